#!/bin/bash
# One ncu --set full capture of the wave kernel at config 3 (+ source-level stalls), tile $1 (default 0).
export NW_SPIN_LIMIT_MS=20000
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 2 -c 1 -o gpurun_out/prof_w${1:-0} python bench.py --steps 1 --warmup 2 --no-cpu --e2e-steps 0 --tile ${1:-0} > gpurun_out/ncu_w.log 2>&1; echo ncu_rc=$?; tail -3 gpurun_out/ncu_w.log
