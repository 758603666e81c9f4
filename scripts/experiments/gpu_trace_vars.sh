#!/bin/bash
# trace builds with parts of the staging disabled (timing only): steady cycles per step per band
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
for v in trace "$@"; do
  export NW_LIB=$PWD/build_variants/$v.so
  timeout 120 python bench.py --config 3 --tile 0 --steps 2 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trv_$v.npy 2>>gpurun_out/trv.err | tail -1 | sed "s/^/$v /" >> gpurun_out/trv_bench.jsonl
  echo "== $v" >> gpurun_out/trv.txt
  python scripts/trace_band.py gpurun_out/trv_$v.npy 32768 2>&1 | sed -n '2,4p;$p' >> gpurun_out/trv.txt
done
