#!/bin/bash
# per-band trace of the round-1 kernel at n = 32768 (tiles 0 and 16)
export NW_SPIN_LIMIT_MS=10000 NW_LIB=$PWD/build_variants/trace.so
mkdir -p gpurun_out
for tile in 0 16; do
  timeout 300 python bench.py --config 3 --tile $tile --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tr_t$tile.npy 2>>gpurun_out/tr.err | tail -1 > gpurun_out/tr_t$tile.json
  python scripts/trace_quick.py gpurun_out/tr_t$tile.npy 32768 > gpurun_out/tr_t$tile.txt 2>&1
done
