# ncu DRAM bytes per launch for every kernel of every plan (north star: dram bytes/px fused vs unfused)
mkdir -p gpurun_out
for cfg in C3 C2 C4 C3s; do
  for plan in unfused paper b200; do
    timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum --clock-control none --cache-control all --csv \
      --log-file gpurun_out/dram_${cfg}_${plan}.csv python tools/prof_run.py --config $cfg --plan $plan --runs 2 > /dev/null 2>&1; echo "$cfg $plan rc=$?"
  done
done
