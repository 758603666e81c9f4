#!/bin/bash
# round-2 iteration probe: smoke, fast GPU parity subset, bench lines for configs 3 / 4 / 2
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out/it
timeout 180 python __graft_entry__.py smoke > gpurun_out/it/smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/it/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size and not config5 and not config4_full and not stress" > gpurun_out/it/pytest.log 2>&1; echo pytest_rc=$?; tail -4 gpurun_out/it/pytest.log
B="timeout 300 python bench.py --no-cpu --e2e-steps 0"
$B --config 3 --steps 10 --warmup 3 > gpurun_out/it/c3.json 2> gpurun_out/it/c3.err; python scripts/show_bench.py gpurun_out/it/c3.json
$B --config 4 --steps 3 --warmup 3 > gpurun_out/it/c4.json 2> gpurun_out/it/c4.err; python scripts/show_bench.py gpurun_out/it/c4.json
$B --config 2 --tile 64 --steps 10 --warmup 3 > gpurun_out/it/c2.json 2> gpurun_out/it/c2.err; python scripts/show_bench.py gpurun_out/it/c2.json
$B --config 3 --layout aligned --steps 10 --warmup 3 > gpurun_out/it/c3a.json 2> gpurun_out/it/c3a.err; python scripts/show_bench.py gpurun_out/it/c3a.json
