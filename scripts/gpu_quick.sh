#!/bin/bash
# Quick probe: a parity subset, then bench config 3 with the per-band trace (+ extra bench args).
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "fill_sizes or sharded or batch or seq or pitch" > gpurun_out/pytest_q.log 2>&1; echo pytest_rc=$?; tail -3 gpurun_out/pytest_q.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_q.npy $@ > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; echo rc=$?
tail -2 gpurun_out/bench_q.err
python scripts/trace_quick.py gpurun_out/trace_q.npy 32768
python -c "import json;j=json.loads(open('gpurun_out/bench_q.json').read().splitlines()[-1]);print(j['value'],'GCUPS',j['ms_per_step'],'ms',j['roofline']['frac'])"
