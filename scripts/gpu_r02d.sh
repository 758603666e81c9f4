#!/bin/bash
# final refresh after the per-kernel tuning: the whole GPU suite and the K = 4 bench lines
export NW_SPIN_LIMIT_MS=10000
O=gpurun_out/r02d; mkdir -p $O
timeout 180 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo smoke_rc=$?; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --maxfail=8 > $O/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -2 $O/pytest_gpu.log
B="timeout 600 python bench.py --no-cpu --e2e-steps 0"
for t in 16 32 64; do $B --config 2 --tile $t --steps 20 --warmup 3 > $O/c2_t$t.json 2>> $O/err; python scripts/show_bench.py $O/c2_t$t.json; done
for t in 16 64; do $B --config 3 --tile $t --steps 10 --warmup 3 > $O/c3_t$t.json 2>> $O/err; python scripts/show_bench.py $O/c3_t$t.json; done
$B --config 3 --steps 20 --warmup 3 > $O/c3.json 2>> $O/err; python scripts/show_bench.py $O/c3.json
$B --config 4 --steps 5 --warmup 3 > $O/c4.json 2>> $O/err; python scripts/show_bench.py $O/c4.json
