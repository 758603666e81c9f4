#!/bin/bash
# Staging back-off sweep at config 3 for the default (K=4) and tile 256 (K=8) kernels.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for tile in 0 256; do for sl in 0 32 100 300 1000; do
  NW_STAGE_SLEEP_NS=$sl timeout 300 python bench.py --tile $tile --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_sl.npy > gpurun_out/bench_sl.json 2>/dev/null
  echo "tile=$tile sleep=$sl $(python -c "import json;j=json.loads(open('gpurun_out/bench_sl.json').read().splitlines()[-1]);print(round(j['value'],1),'GCUPS')")"
  python scripts/trace_quick.py gpurun_out/trace_sl.npy 32768 2>/dev/null | sed -n 2p
done; done
