#!/bin/bash
export NW_SPIN_LIMIT_MS=10000
timeout 600 python -m pytest tests -m gpu -q -x -k "host" 2>&1 | tail -3
timeout 600 python bench.py --config 3 --steps 3 --warmup 3 --no-cpu --e2e-steps 3 > gpurun_out/host_c3.json 2> gpurun_out/host_c3.err; python -c "
import json; d=json.loads(open('gpurun_out/host_c3.json').read().strip().splitlines()[-1]); print('c3', d['value'], d['e2e'])"
timeout 600 python bench.py --config 4 --steps 3 --warmup 3 --no-cpu --e2e-steps 3 > gpurun_out/host_c4.json 2> gpurun_out/host_c4.err; python -c "
import json; d=json.loads(open('gpurun_out/host_c4.json').read().strip().splitlines()[-1]); print('c4', d['value'], d['e2e'])"
tail -3 gpurun_out/host_c3.err
