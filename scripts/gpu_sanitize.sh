#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over every kernel at a small size, and the
# n = 1024 flag-race stress at 1000 repetitions
mkdir -p gpurun_out
export NW_SPIN_LIMIT_MS=60000
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_small.py 300 > gpurun_out/san_$tool.txt 2>&1
  echo "== $tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ALL OK|BAD" gpurun_out/san_$tool.txt | head -5
done
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "stress" > gpurun_out/stress.log 2>&1; tail -2 gpurun_out/stress.log
