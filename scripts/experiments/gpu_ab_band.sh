#!/bin/bash
# A/B of band-kernel build variants (build_variants/*.so via NW_LIB): config 3, both layouts
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
OUT=gpurun_out/ab_${TAG:-x}.jsonl
for v in "$@"; do
  export NW_LIB=$PWD/build_variants/$v.so
  for lay in rodinia aligned; do
    timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/ab.err | tail -1 | sed "s/^/$v-$lay /" >> $OUT
  done
done
