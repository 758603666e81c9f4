#!/bin/bash
# A/B of experiment builds on the K = 4 configurations (config 3 tiles 16 / 64, config 2 tiles 16 / 64)
for v in default "$@"; do
  if [ $v = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  for c in 3 2; do for t in 16 64; do
    timeout 300 python bench.py --no-cpu --e2e-steps 0 --config $c --tile $t --steps 10 --warmup 3 > gpurun_out/ab4_${v}_c${c}_$t.json 2>/dev/null
    echo -n "$v "; python scripts/show_bench.py gpurun_out/ab4_${v}_c${c}_$t.json
  done; done
done
