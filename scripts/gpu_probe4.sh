#!/bin/bash
./scripts/ubench_step3
for t in 0 16 64 128; do timeout 200 python bench.py --no-cpu --e2e-steps 0 --config 3 --tile $t --steps 10 --warmup 3 > gpurun_out/c3_t$t.json 2>/dev/null; python scripts/show_bench.py gpurun_out/c3_t$t.json; done
