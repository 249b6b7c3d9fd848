python tools/repro_case_f32.py 2030000 230 > gpurun_out/repro_a.log 2>&1; cat gpurun_out/repro_a.log
python tools/repro_case_f32.py 2030000 1381 > gpurun_out/repro_b.log 2>&1; cat gpurun_out/repro_b.log
