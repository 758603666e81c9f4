#!/bin/bash
# configs 2 and 4 across kernels: round-1 (tiles 16/32/64 and the K=8 default was tile 256 before)
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
for tile in 0 128 256 16 64; do
  timeout 120 python bench.py --config 2 --tile $tile --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/c24.err | tail -1 | sed "s/^/c2-t$tile /" >> gpurun_out/c24.jsonl
done
for tile in 0 128 256 64; do
  timeout 300 python bench.py --config 4 --tile $tile --steps 3 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/c24.err | tail -1 | sed "s/^/c4-t$tile /" >> gpurun_out/c24.jsonl
done
