#!/bin/bash
# the round-2 parity tests (range edge, concurrent strips, watchdog, full configs 4 and 5)
mkdir -p gpurun_out
nproc > gpurun_out/nt_nproc.txt; free -g >> gpurun_out/nt_nproc.txt
timeout 2400 python -m pytest tests/test_gpu_parity.py -q -x -k "range_edge or concurrent or watchdog or config5 or config4_full" --durations=20 > gpurun_out/nt_pytest.log 2>&1
tail -30 gpurun_out/nt_pytest.log
