#!/bin/bash
export NW_SPIN_LIMIT_MS=3000
mkdir -p gpurun_out
for args in "700 3 0 4" "700 3 128 4" "700 0 0 2" "1000 3 0 3" "517 10 0 3" "2048 3 0 3"; do
  echo "== $args" >> gpurun_out/dbg.txt
  timeout 120 python scripts/dbg_band.py $args >> gpurun_out/dbg.txt 2>&1
done
