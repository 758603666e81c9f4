#!/bin/bash
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
NW_DEBUG_SKIP=${2:-0} timeout 600 ncu --set full --warp-sampling-interval 0 --clock-control none --import-source on -k regex:nw_strip -s 2 -c 1 -o gpurun_out/prof1 python scripts/one_band.py ${1:-128} ${3:-1} > gpurun_out/ncu1.log 2>&1; echo ncu_rc=$?
