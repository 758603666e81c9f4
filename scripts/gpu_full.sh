#!/bin/bash
# full GPU suite + sanitizers + default bench lines (configs 3, 4) of the shipped library
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/full_pytest.log 2>&1; tail -3 gpurun_out/full_pytest.log
bash scripts/gpu_sanitize.sh
timeout 300 python bench.py --config 3 --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>gpurun_out/full_b.err | tail -1 > gpurun_out/full_b3.json
timeout 300 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/full_b.err | tail -1 > gpurun_out/full_b4.json
