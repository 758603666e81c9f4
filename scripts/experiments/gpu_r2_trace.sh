#!/bin/bash
# parity subset + bench + per-band trace of the band kernel
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "sizes or families or pitch or grids or reuse or aligned" > gpurun_out/r2t_pytest.log 2>&1
tail -2 gpurun_out/r2t_pytest.log
for lay in rodinia aligned; do
  timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 10 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/r2t.err | tail -1 | sed "s/^/$lay /" >> gpurun_out/r2t_bench.jsonl
done
export NW_LIB=$PWD/build_variants/trace.so
for lay in rodinia aligned; do
  timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/r2t_$lay.npy 2>>gpurun_out/r2t.err | tail -1 | sed "s/^/tr$lay /" >> gpurun_out/r2t_bench.jsonl
  python scripts/trace_band.py gpurun_out/r2t_$lay.npy 32768 > gpurun_out/r2t_$lay.txt 2>&1
done
unset NW_LIB
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nw_band -s 1 -c 1 -o gpurun_out/r2t_prof -f python scripts/one_fill.py 32768 0 2 > gpurun_out/r2t_ncu.log 2>&1
