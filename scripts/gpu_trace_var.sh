#!/bin/bash
# per-band traces of config 3 (tile 0) for the NW_TRACE=1 variant builds named on the command line
mkdir -p gpurun_out/tv
for v in "$@"; do
  NW_LIB=$PWD/build_variants/$v.so timeout 120 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tv/tr_$v.npy > gpurun_out/tv/b_$v.json 2>/dev/null
  echo "== $v"; python scripts/show_bench.py gpurun_out/tv/b_$v.json; python scripts/trace_quick.py gpurun_out/tv/tr_$v.npy 32768 2>/dev/null | sed -n '2,4p;11,13p'
done
