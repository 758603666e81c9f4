#!/bin/bash
export NW_SPIN_LIMIT_MS=5000 NW_LIB=$PWD/build_variants/trace.so
mkdir -p gpurun_out
for lay in rodinia aligned; do
  timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tro_$lay.npy 2>>gpurun_out/tro.err | tail -1 | sed "s/^/tr$lay /" >> gpurun_out/tro_bench.jsonl
  python scripts/trace_band.py gpurun_out/tro_$lay.npy 32768 > gpurun_out/tro_$lay.txt 2>&1
  python scripts/trace_chunks.py gpurun_out/tro_${lay}_chunks.npy 6 >> gpurun_out/tro_$lay.txt 2>&1
done
