#!/bin/bash
# iteration probe: smoke, fast GPU parity subset, bench lines for configs 3 (tiles 0/16/64) / 4 / 2, trace of tile 16
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out/it
timeout 180 python __graft_entry__.py smoke > gpurun_out/it/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size and not config5 and not config4_full and not stress" > gpurun_out/it/pytest.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/it/pytest.log
B="timeout 300 python bench.py --no-cpu --e2e-steps 0"
for t in 0 16 64; do $B --config 3 --tile $t --steps 10 --warmup 3 > gpurun_out/it/c3_$t.json 2>/dev/null; python scripts/show_bench.py gpurun_out/it/c3_$t.json; done
$B --config 4 --steps 3 --warmup 3 > gpurun_out/it/c4.json 2>/dev/null; python scripts/show_bench.py gpurun_out/it/c4.json
for t in 16 64; do $B --config 2 --tile $t --steps 10 --warmup 3 > gpurun_out/it/c2_$t.json 2>/dev/null; python scripts/show_bench.py gpurun_out/it/c2_$t.json; done
for t in ${TRACE_TILES:-16}; do
  NW_LIB=$PWD/build_variants/trace.so timeout 120 python bench.py --config 3 --tile $t --steps 3 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/it/tr_$t.npy > /dev/null 2>&1
  echo "trace tile $t"; python scripts/trace_quick.py gpurun_out/it/tr_$t.npy 32768 2>/dev/null | sed -n '1,4p'
done
