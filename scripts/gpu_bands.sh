#!/bin/bash
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for tl in ${@:-128 0}; do echo "== tile $tl"; timeout 300 python scripts/probe_bands.py 32768 $tl 2>&1 | grep -v "^\[" | tee -a gpurun_out/bands.txt; done
