#!/bin/bash
# Quick perf probe: bench config 3 with trace (+ optional extra args), no tests.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_q.npy $@ > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; echo rc=$?
tail -2 gpurun_out/bench_q.err
python scripts/trace_analysis.py gpurun_out/trace_q.npy 32768
python -c "import json;j=json.loads(open('gpurun_out/bench_q.json').read().splitlines()[-1]);print(j['value'],'GCUPS',j['ms_per_step'],'ms',j['roofline']['frac'])"
