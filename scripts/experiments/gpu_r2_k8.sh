#!/bin/bash
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "sizes or families or pitch or grids or reuse or aligned" > gpurun_out/k8_pytest.log 2>&1
tail -2 gpurun_out/k8_pytest.log
for tile in 256 0; do for lay in rodinia aligned; do
  timeout 120 python bench.py --config 3 --tile $tile --layout $lay --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/k8.err | tail -1 | sed "s/^/t$tile-$lay /" >> gpurun_out/k8_bench.jsonl
done; done
