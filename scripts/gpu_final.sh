#!/bin/bash
# One gpurun call: smoke, all GPU tests, the default bench line, batch bench line, ncu launch list,
# ncu --set full of the traceback kernel (single pair, n = 32768).
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 180 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --maxfail=8 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -4 gpurun_out/pytest_gpu.log
timeout 400 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo bench_rc=$?; tail -c 900 gpurun_out/bench_final.json
timeout 600 python bench.py --config 4 --steps 3 --e2e-steps 0 --no-cpu > gpurun_out/bench_final_c4.json 2> gpurun_out/bench_final_c4.err; echo rc=$?
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_final.csv python bench.py --steps 2 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1; echo ncu_rc=$?
PYTHONPATH=. timeout 500 ncu --set full --clock-control none --import-source on -k regex:nw_traceback -c 2 -o gpurun_out/prof_tb_final python scripts/tb_one.py 32768 > gpurun_out/ncu_tb_final.log 2>&1; echo ncu2_rc=$?
