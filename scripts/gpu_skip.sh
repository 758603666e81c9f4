#!/bin/bash
# timing attribution on narrow strips: NW_DEBUG_SKIP bits (1 staging, 2 state check, 4 ev arrive, 8 border)
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for sk in 0 1 3 7 15; do echo "== skip $sk"; NW_DEBUG_SKIP=$sk timeout 120 python scripts/probe_bands.py 32768 ${1:-128} 2>&1 | grep -E "bands +(1|4|256) " ; done | tee gpurun_out/skip.txt
