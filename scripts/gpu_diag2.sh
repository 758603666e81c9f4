#!/bin/bash
# round-2 diagnosis: per-band trace of the headline kernel with parts of the staging disabled
# (timing only: the skip builds produce invalid matrices), and the TMA destination-alignment probe
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out/dg
for s in 1024 1040 1152; do timeout 30 ./scripts/tma_probe $s 1 >> gpurun_out/dg/tma.txt 2>&1; timeout 30 ./scripts/tma_probe $s 7 >> gpurun_out/dg/tma.txt 2>&1; done
cat gpurun_out/dg/tma.txt
for v in trace skipref skipst skipboth; do
  export NW_LIB=$PWD/build_variants/$v.so
  timeout 120 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/dg/tr_$v.npy > gpurun_out/dg/b_$v.json 2>>gpurun_out/dg/err.txt
  echo "== $v"; python scripts/show_bench.py gpurun_out/dg/b_$v.json
  python scripts/trace_quick.py gpurun_out/dg/tr_$v.npy 32768
done
