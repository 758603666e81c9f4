#!/bin/bash
# per-band traces (NW_TRACE=1 build) of config 3 for the kernel variants (tile 0 / 16 / 64)
mkdir -p gpurun_out/tt
for t in 0 16 64; do
  NW_LIB=$PWD/build_variants/trace.so timeout 120 python bench.py --config 3 --tile $t --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tt/tr_$t.npy > gpurun_out/tt/b_$t.json 2>/dev/null
  echo "== tile $t"; python scripts/show_bench.py gpurun_out/tt/b_$t.json; python scripts/trace_quick.py gpurun_out/tt/tr_$t.npy 32768 2>/dev/null | head -8
done
