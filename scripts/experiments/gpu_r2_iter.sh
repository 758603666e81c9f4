#!/bin/bash
# one iteration: parity subset, config-3 bench (both layouts) of the default build and variants,
# trace of the trace build
export NW_SPIN_LIMIT_MS=5000
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "sizes or families or pitch or grids or reuse or aligned" > gpurun_out/it_pytest.log 2>&1
tail -2 gpurun_out/it_pytest.log
for v in default "$@"; do
  if [ "$v" = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  for lay in rodinia aligned; do
    timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/it.err | tail -1 | sed "s/^/$v-$lay /" >> gpurun_out/it_bench.jsonl
  done
done
export NW_LIB=$PWD/build_variants/trace.so
for lay in rodinia aligned; do
timeout 120 python bench.py --config 3 --tile 0 --layout $lay --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/it_tr_$lay.npy 2>>gpurun_out/it.err | tail -1 | sed "s/^/trace-$lay /" >> gpurun_out/it_bench.jsonl
python scripts/trace_band.py gpurun_out/it_tr_$lay.npy 32768 > gpurun_out/it_tr_$lay.txt 2>&1
done
