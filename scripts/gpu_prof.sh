#!/bin/bash
# Quick probe + one ncu --set full capture of the strip kernel at config 3.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
bash scripts/gpu_quick.sh $@
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_strip -s 3 -c 1 -o gpurun_out/prof_q python bench.py --steps 1 --warmup 3 --no-cpu --e2e-steps 0 $@ > gpurun_out/ncu_q.log 2>&1; echo ncu_rc=$?
