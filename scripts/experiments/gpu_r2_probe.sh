#!/bin/bash
# round-2 first probe: tile sweep at configs 2/3 on the round-1 kernel
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2p_smi.txt
for c in 3 2; do for tile in 0 16 64; do
  timeout 300 python bench.py --config $c --tile $tile --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/r2p.err | tail -1 >> gpurun_out/r2p_bench.jsonl
done; done
if [ -x scripts/ubench_mw ]; then timeout 300 ./scripts/ubench_mw > gpurun_out/r2p_ubench.txt 2>&1; fi
