mkdir -p gpurun_out
for cfg in C2 C3s; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_${cfg}_final \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}.log 2>&1; echo "ncu $cfg rc=$?"
done
