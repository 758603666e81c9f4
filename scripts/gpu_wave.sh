#!/bin/bash
# Quick probe of the wave kernel: parity subset, then config 3 at tile 0 (K=2) and 128 (K=4) with traces.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "${PYK:-fill_sizes or sharded or batch or seq or pitch}" > gpurun_out/pytest_w.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_w.log
for tl in ${TILES:-0 128}; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --tile $tl --trace gpurun_out/trace_w$tl.npy $BENCH_ARGS > gpurun_out/bench_w$tl.json 2> gpurun_out/bench_w$tl.err; echo "tile $tl rc=$?"
  tail -3 gpurun_out/bench_w$tl.err
  python -c "import json;j=json.loads(open('gpurun_out/bench_w$tl.json').read().splitlines()[-1]);print('tile $tl:',round(j['value'],1),'GCUPS',round(j['ms_per_step'],3),'ms frac',round(j['roofline']['frac'],3))"
  python scripts/trace_summary.py gpurun_out/trace_w$tl.npy 32768
done
