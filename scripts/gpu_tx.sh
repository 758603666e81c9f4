#!/bin/bash
# steady-block cycles per step of config 3 (tile 0) for experiment builds that strip parts of the step
for v in "$@"; do
  NW_LIB=$PWD/build_variants/$v.so timeout 120 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tx_$v.npy > gpurun_out/tx_$v.log 2>&1
  echo "$v $(python scripts/trace_quick.py gpurun_out/tx_$v.npy 32768 2>/dev/null | sed -n 2p | grep -o 'steady-block.*')"
done
