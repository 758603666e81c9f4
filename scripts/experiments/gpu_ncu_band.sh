#!/bin/bash
# ncu --set full capture of the round-2 band kernel (one launch)
mkdir -p gpurun_out
N=${1:-16384}; TILE=${2:-0}; TAG=${3:-band}
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nw_band -s 1 -c 1 -o gpurun_out/$TAG -f python scripts/one_fill.py $N $TILE 2 > gpurun_out/$TAG.log 2>&1
tail -3 gpurun_out/$TAG.log
