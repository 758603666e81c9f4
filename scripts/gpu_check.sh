#!/bin/bash
# One gpurun call: smoke, GPU parity tests, bench (headline + ablations), ncu launch list + full capture.
export NW_SPIN_LIMIT_MS=10000
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.max.sm,memory.total --format=csv
timeout 180 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -5 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q --maxfail=8 > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -40 gpurun_out/pytest_gpu.log
timeout 400 python bench.py --steps 10 --warmup 3 --trace gpurun_out/trace_c3.npy > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo bench_rc=$?; cat gpurun_out/bench_c3.json; tail -5 gpurun_out/bench_c3.err
for t in 16 64 128; do timeout 200 python bench.py --config 2 --tile $t --steps 10 --no-cpu --e2e-steps 0 > gpurun_out/bench_c2_t$t.json 2>&1; tail -1 gpurun_out/bench_c2_t$t.json | cut -c1-400; done
timeout 300 python bench.py --config 3 --variant diagonal --steps 3 --no-cpu --e2e-steps 0 > gpurun_out/bench_c3_diag.json 2>&1; tail -1 gpurun_out/bench_c3_diag.json | cut -c1-300
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:nw_ -c 6 --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 2 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1; echo ncu1_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 3 -c 1 -o gpurun_out/prof_c3 python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1; echo ncu2_rc=$?; tail -3 gpurun_out/ncu_full.log
timeout 300 python bench.py --config 3 --variant seq --steps 10 --no-cpu --e2e-steps 0 > gpurun_out/bench_c3_seq.json 2>&1; tail -1 gpurun_out/bench_c3_seq.json | cut -c1-400
