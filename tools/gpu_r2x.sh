# r2x: ncu DRAM bytes per pixel of every plan on the final build (cold L2), for the fused-vs-unfused table
mkdir -p gpurun_out/r02_dram
for cfg in C3 C2 C4 C3s; do
  for plan in unfused paper b200; do
    timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum --clock-control none --cache-control all --csv \
      --log-file gpurun_out/r02_dram/dram_${cfg}_${plan}.csv python tools/prof_run.py --config $cfg --plan $plan --runs 2 > /dev/null 2>&1; echo "$cfg $plan rc=$?"
  done
done
python tools/dram_table.py gpurun_out/r02_dram
