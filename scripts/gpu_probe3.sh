#!/bin/bash
mkdir -p gpurun_out/p3
timeout 120 ./scripts/ubench_ops > gpurun_out/p3/ops.txt 2>&1; cat gpurun_out/p3/ops.txt
for s in 1024 1040; do timeout 30 ./scripts/tma_probe $s 1; timeout 30 ./scripts/tma_probe32 $s 1; done
timeout 60 compute-sanitizer --tool memcheck ./scripts/tma_probe 1024 1 2>&1 | head -30
# ncu source-level capture of the headline kernel (one launch)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 1 -c 1 -o gpurun_out/p3/prof_c3 -f python scripts/one_fill.py 32768 0 2 > gpurun_out/p3/ncu.log 2>&1; echo ncu_rc=$?; tail -2 gpurun_out/p3/ncu.log
