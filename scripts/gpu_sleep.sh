#!/bin/bash
bash scripts/gpu_trace_var.sh tr_sleep200 tr_sleep1000
for v in sleep500; do NW_LIB=$PWD/build_variants/$v.so timeout 200 python bench.py --no-cpu --e2e-steps 0 --config 3 --steps 10 --warmup 3 > gpurun_out/tv/b_$v.json 2>/dev/null; python scripts/show_bench.py gpurun_out/tv/b_$v.json; done
