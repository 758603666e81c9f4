#!/bin/bash
export NW_SPIN_LIMIT_MS=2000
mkdir -p gpurun_out
timeout 300 compute-sanitizer --tool memcheck --print-limit 10 python scripts/dbg_band.py 1 10 128 1 > gpurun_out/dbg2.txt 2>&1
tail -40 gpurun_out/dbg2.txt
