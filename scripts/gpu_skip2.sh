#!/bin/bash
# Timing attribution: the wave kernel at config 3 with staging work skipped (results invalid).
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for sk in 0 5 9 13 2; do
  NW_DEBUG_SKIP=$sk timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_s$sk.npy $@ > gpurun_out/bench_s$sk.json 2>/dev/null
  echo "skip=$sk $(python -c "import json;j=json.loads(open('gpurun_out/bench_s$sk.json').read().splitlines()[-1]);print(round(j['value'],1),'GCUPS')")"
  python scripts/trace_quick.py gpurun_out/trace_s$sk.npy 32768 | head -2
done
