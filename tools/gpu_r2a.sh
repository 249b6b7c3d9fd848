# r2a: host facts, smoke, the whole GPU suite (no -x: see every failure) with the parity log
mkdir -p gpurun_out
{ nproc; lscpu | grep -E "Model name|^CPU\(s\)|Thread|Socket"; free -g | head -2; nvidia-smi --query-gpu=name,clocks.max.sm --format=csv; } > gpurun_out/host_r2a.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2a.log 2>&1; echo "smoke rc=$?"
KF_PARITY_LOG=gpurun_out/parity_r2a.jsonl timeout 2700 python -m pytest tests -q -m gpu --durations=40 > gpurun_out/tests_r2a.log 2>&1; echo "tests rc=$?"
tail -60 gpurun_out/tests_r2a.log
