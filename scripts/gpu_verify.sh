#!/bin/bash
# One gpurun call: smoke, GPU parity tests, the default bench line, the ncu launch list of that command.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.max.sm,memory.total --format=csv
timeout 180 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -3 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --maxfail=8 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_gpu.log
timeout 400 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo bench_rc=$?; cat gpurun_out/bench_default.json; tail -3 gpurun_out/bench_default.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_default.csv python bench.py --steps 2 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1; echo ncu_rc=$?
