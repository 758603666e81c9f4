#!/bin/bash
# A/B of experiment builds (build_variants/<name>.so) on config 3 and config 4, with the default library first
for v in default "$@"; do
  if [ $v = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  for c in 3 4; do
    timeout 300 python bench.py --no-cpu --e2e-steps 0 --config $c --steps $([ $c = 3 ] && echo 10 || echo 3) --warmup 3 > gpurun_out/ab_${v}_c$c.json 2>/dev/null
    echo -n "$v "; python scripts/show_bench.py gpurun_out/ab_${v}_c$c.json
  done
done
