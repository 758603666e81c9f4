#!/bin/bash
# one ncu --set full capture (source counters) of the headline kernel, exported as CSV for
# scripts/ncu_steady.py; plus the per-band trace of an NW_TRACE=1 build if present
mkdir -p gpurun_out/ns
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 1 -c 1 -o gpurun_out/ns/prof -f python scripts/one_fill.py 32768 0 2 > gpurun_out/ns/ncu.log 2>&1; echo ncu_rc=$?
ncu -i gpurun_out/ns/prof.ncu-rep --page source --csv --print-source sass > gpurun_out/ns/src.csv 2>/dev/null
ncu -i gpurun_out/ns/prof.ncu-rep --page raw --csv > gpurun_out/ns/raw.csv 2>/dev/null
if [ -f build_variants/trace.so ]; then
  NW_LIB=$PWD/build_variants/trace.so timeout 120 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/ns/tr.npy > gpurun_out/ns/b_trace.json 2>/dev/null
  python scripts/trace_quick.py gpurun_out/ns/tr.npy 32768
fi
