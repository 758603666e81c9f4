#!/bin/bash
# steady-block cycles per step of config 3 at tile 16 (K = 4, two bands per CTA) for experiment builds
for v in "$@"; do
  NW_LIB=$PWD/build_variants/$v.so timeout 120 python bench.py --config 3 --tile 16 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tx16_$v.npy > gpurun_out/tx16_$v.log 2>&1
  echo "$v $(python scripts/trace_quick.py gpurun_out/tx16_$v.npy 32768 2>/dev/null | sed -n '2p;4p;5p' | grep -o 'steady-block.*\|per event.*' | tr '\n' ' ')"
done
