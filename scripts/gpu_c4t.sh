#!/bin/bash
B="timeout 300 python bench.py --no-cpu --e2e-steps 0 --config 4 --steps 3 --warmup 3"
for L in rodinia aligned; do for t in 0 16 64; do $B --layout $L --tile $t > gpurun_out/c4_${L}_$t.json 2>/dev/null; echo -n "$L "; python scripts/show_bench.py gpurun_out/c4_${L}_$t.json; done; done
