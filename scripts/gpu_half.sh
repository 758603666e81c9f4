#!/bin/bash
export NW_SPIN_LIMIT_MS=10000
timeout 180 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size and not config5 and not config4_full and not stress" 2>&1 | tail -1
bash scripts/gpu_ab.sh half16 half12
bash scripts/gpu_ab.sh half16
