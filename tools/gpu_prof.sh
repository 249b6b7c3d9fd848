# ncu evidence for the non-headline configs + FP/INT issue-rate microbenchmark.
mkdir -p gpurun_out
cd tools/ubench && nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o fp_rates fp_rates.cu && ./fp_rates > ../../gpurun_out/fp_rates.txt 2>&1; cd ../..
for cfg in C2 C3 C3s C4; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:kf_b -s 2 -c 1 -f -o gpurun_out/prof_${cfg} \
     python tools/prof_run.py --config $cfg --plan b200 > gpurun_out/ncu_${cfg}.log 2>&1; echo "ncu $cfg rc=$?"
done
