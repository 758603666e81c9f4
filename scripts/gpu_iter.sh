#!/bin/bash
# Iteration probe: full GPU parity suite, bench config 3 (+ per-band trace), SEQ variant, config 2.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_i.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_i.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_i.npy $@ > gpurun_out/bench_i.json 2> gpurun_out/bench_i.err; echo rc=$?
tail -2 gpurun_out/bench_i.err
python -c "import json;j=json.loads(open('gpurun_out/bench_i.json').read().splitlines()[-1]);print('c3',j['value'],'GCUPS',j['ms_per_step'],'ms frac',j['roofline']['frac'])"
timeout 300 python bench.py --variant seq --steps 10 --warmup 3 --no-cpu --e2e-steps 0 $@ > gpurun_out/bench_iseq.json 2>&1
python -c "import json;j=json.loads(open('gpurun_out/bench_iseq.json').read().splitlines()[-1]);print('c3 seq',j['value'],'GCUPS',j['ms_per_step'],'ms')"
timeout 300 python bench.py --config 2 --steps 10 --warmup 3 --no-cpu --e2e-steps 0 $@ > gpurun_out/bench_ic2.json 2>&1
python -c "import json;j=json.loads(open('gpurun_out/bench_ic2.json').read().splitlines()[-1]);print('c2',j['value'],'GCUPS',j['ms_per_step'],'ms')"
