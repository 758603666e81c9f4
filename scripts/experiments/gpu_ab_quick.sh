#!/bin/bash
# quick A/B: config 3 bench of build variants (no parity)
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
for v in default "$@"; do
  if [ "$v" = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  timeout 120 python bench.py --config 3 --tile 0 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/abq.err | tail -1 | sed "s/^/$v /" >> gpurun_out/abq.jsonl
done
