#!/bin/bash
# A/B of experiment builds (build_variants/*.so via NW_LIB) on configs 3 and 4.
export NW_SPIN_LIMIT_MS=10000
for v in default $@; do
  if [ "$v" = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  for tile in 0 128; do
    a=$(timeout 300 python bench.py --tile $tile --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>/dev/null | python -c "import json,sys;print(round(json.loads(sys.stdin.read().splitlines()[-1])['value'],1))")
    b=$(timeout 300 python bench.py --config 4 --tile $tile --steps 3 --warmup 3 --no-cpu --e2e-steps 0 2>/dev/null | python -c "import json,sys;print(round(json.loads(sys.stdin.read().splitlines()[-1])['value'],1))")
    echo "$v tile=$tile c3=$a c4=$b"
  done
done
