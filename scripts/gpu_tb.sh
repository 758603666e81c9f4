#!/bin/bash
# One gpurun call: traceback parity tests + bench lines that carry the traceback timing.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_traceback.py -q -x > gpurun_out/pytest_tb.log 2>&1; echo pytest_rc=$?; tail -15 gpurun_out/pytest_tb.log
timeout 400 python bench.py --steps 10 --e2e-steps 0 --no-cpu > gpurun_out/bench_tb_c3.json 2> gpurun_out/bench_tb_c3.err; echo rc=$?; tail -c 600 gpurun_out/bench_tb_c3.json; tail -3 gpurun_out/bench_tb_c3.err
timeout 600 python bench.py --config 4 --steps 3 --e2e-steps 0 --no-cpu > gpurun_out/bench_tb_c4.json 2> gpurun_out/bench_tb_c4.err; echo rc=$?; tail -c 600 gpurun_out/bench_tb_c4.json; tail -3 gpurun_out/bench_tb_c4.err
