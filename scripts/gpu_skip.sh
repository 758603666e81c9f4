#!/bin/bash
# timing attribution: config 3 with the staging warp's copies skipped (results invalid) vs normal
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for sk in ${SKIPS:-0 1}; do
 for tl in ${TILES:-0 128}; do
  NW_DEBUG_SKIP=$sk timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --tile $tl --trace gpurun_out/trace_s$sk$tl.npy > gpurun_out/bench_s$sk$tl.json 2> gpurun_out/bench_s$sk$tl.err
  python -c "import json;j=json.loads(open('gpurun_out/bench_s$sk$tl.json').read().splitlines()[-1]);print('skip $sk tile $tl:',round(j['value'],1),'GCUPS',round(j['ms_per_step'],3),'ms')"
  python scripts/trace_summary.py gpurun_out/trace_s$sk$tl.npy 32768
 done
done
