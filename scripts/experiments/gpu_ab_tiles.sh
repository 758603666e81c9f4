#!/bin/bash
# A/B of a build variant over tiles and layouts (config 3)
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
V=$1; shift
if [ "$V" != default ]; then export NW_LIB=$PWD/build_variants/$V.so; fi
for tile in "$@"; do for lay in rodinia aligned; do
  timeout 120 python bench.py --config 3 --tile $tile --layout $lay --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/abt.err | tail -1 | sed "s/^/$V-t$tile-$lay /" >> gpurun_out/abt.jsonl
done; done
