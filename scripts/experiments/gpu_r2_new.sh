#!/bin/bash
# round-2 band kernel: quick parity + bench
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "sizes or families or pitch or grids or reuse or aligned" > gpurun_out/r2n_pytest.log 2>&1
tail -3 gpurun_out/r2n_pytest.log
for lay in rodinia aligned; do for tile in 0 128; do
  timeout 120 python bench.py --config 3 --tile $tile --layout $lay --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/r2n.err | tail -1 | sed "s/^/$lay /" >> gpurun_out/r2n_bench.jsonl
done; done
for lay in rodinia aligned; do for tile in 0 128; do
  timeout 120 python bench.py --config 2 --tile $tile --layout $lay --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/r2n.err | tail -1 | sed "s/^/$lay /" >> gpurun_out/r2n_bench.jsonl
done; done
