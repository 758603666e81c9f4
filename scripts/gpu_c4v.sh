#!/bin/bash
# Config 4 on one GPU: kernel variant (tile) x experiment build (build_variants/*.so via NW_LIB).
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for v in default "$@"; do
  if [ "$v" = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  python -c "
import paper_conf_sc_munksgaardhso22_b200 as nwb
for t in (0, 16, 32):
    print('$v', 'tile', t, nwb.nw_kernel_info(t, 0))" 2>&1 | tail -3
  for tile in 0 32; do
    timeout 300 python bench.py --config 4 --tile $tile --steps 3 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/c4v_${v}_$tile.json 2> gpurun_out/c4v_${v}_$tile.err
    echo "$v tile=$tile rc=$? $(python scripts/show_bench.py gpurun_out/c4v_${v}_$tile.json 2>&1 | tail -1)"
  done
done
