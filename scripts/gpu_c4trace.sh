#!/bin/bash
NW_LIB=$PWD/build_variants/trace.so timeout 300 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/tr_c4.npy > gpurun_out/tr_c4.log 2>&1; tail -c 300 gpurun_out/tr_c4.log
