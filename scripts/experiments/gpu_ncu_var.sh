#!/bin/bash
# ncu --set full of one launch of a build variant: gpu_ncu_var.sh variant n tag
mkdir -p gpurun_out
V=$1; N=${2:-32768}; TAG=${3:-var}
if [ "$V" != default ]; then export NW_LIB=$PWD/build_variants/$V.so; fi
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nw_band -s 1 -c 1 -o gpurun_out/$TAG -f python scripts/one_fill.py $N 0 2 > gpurun_out/$TAG.log 2>&1
tail -2 gpurun_out/$TAG.log
