#!/bin/bash
# NOTE (round 2): compute-sanitizer is closed on the GPU pool ("runs under it have left GPUs
# needing a reset"); this script is kept for the record of the earlier clean run
# (profiles/r02_sanitize/) and must not be run there again.
# compute-sanitizer over every kernel family: memcheck, racecheck,
# synccheck and initcheck on tests/sanitize_cases.py, plus memcheck on the
# peer-memory halo kernels at 2 ranks (tests/test_gpu_parity.py peer cases).
# Logs under gpurun_out/sanitize/; the summary lines are what profiles/ keeps.
mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "memcheck" ] && extra="--leak-check no"
  timeout 1500 $CS --tool $tool $extra --error-exitcode 9 --print-limit 50 \
      python tests/sanitize_cases.py all > gpurun_out/sanitize/$tool.log 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|sanitize cases ok' gpurun_out/sanitize/$tool.log | tr '\n' ' ')"
done
timeout 1200 $CS --tool memcheck --target-processes all --error-exitcode 9 --print-limit 50 \
    python -m pytest tests/test_gpu_parity.py -q -m gpu -k "peer_halo_steps and (harris-2-False or two_input-2-True)" \
    > gpurun_out/sanitize/memcheck_peer.log 2>&1
echo "memcheck peer rc=$? $(grep -cE 'ERROR SUMMARY: 0 errors' gpurun_out/sanitize/memcheck_peer.log) clean process summaries; $(grep -E 'ERROR SUMMARY: [1-9]' gpurun_out/sanitize/memcheck_peer.log | head -3 | tr '\n' ' ') $(tail -1 gpurun_out/sanitize/memcheck_peer.log)"
