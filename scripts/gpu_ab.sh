#!/bin/bash
# A/B probe: parity subset once, then config 3 for each tile given (default: 0 128), with traces.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "fill_sizes or sharded or batch or seq or pitch" > gpurun_out/pytest_q.log 2>&1; echo pytest_rc=$?; tail -2 gpurun_out/pytest_q.log
for tl in ${@:-0 128}; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --tile $tl --trace gpurun_out/trace_t$tl.npy > gpurun_out/bench_t$tl.json 2> gpurun_out/bench_t$tl.err; echo "tile $tl rc=$?"
  python -c "import json;j=json.loads(open('gpurun_out/bench_t$tl.json').read().splitlines()[-1]);print('tile $tl:',round(j['value'],1),'GCUPS',round(j['ms_per_step'],3),'ms frac',round(j['roofline']['frac'],3))"
  python scripts/trace_quick.py gpurun_out/trace_t$tl.npy 32768 | tail -6
done
