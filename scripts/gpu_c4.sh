#!/bin/bash
# Config 4 (4096 independent n=2048 pairs) on one GPU, both kernels.
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for tile in 0 128; do
  timeout 600 python bench.py --config 4 --tile $tile --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_c4_$tile.json 2> gpurun_out/bench_c4_$tile.err
  echo "tile=$tile rc=$? $(tail -1 gpurun_out/bench_c4_$tile.json | cut -c1-250)"
  tail -2 gpurun_out/bench_c4_$tile.err
done
