#!/bin/bash
B="timeout 300 python bench.py --no-cpu --e2e-steps 0 --config 3 --steps 10 --warmup 3"
$B > gpurun_out/cl_none.json 2>/dev/null; echo -n "none "; python scripts/show_bench.py gpurun_out/cl_none.json
$B --cluster > gpurun_out/cl_4.json 2>/dev/null; echo -n "cl4 "; python scripts/show_bench.py gpurun_out/cl_4.json
for v in cl2 cl8; do NW_LIB=$PWD/build_variants/$v.so $B --cluster > gpurun_out/cl_$v.json 2>gpurun_out/cl_$v.err; echo -n "$v "; python scripts/show_bench.py gpurun_out/cl_$v.json; tail -2 gpurun_out/cl_$v.err; done
