#!/bin/bash
export NW_SPIN_LIMIT_MS=10000
mkdir -p gpurun_out
for tile in 0 128; do
  timeout 300 python bench.py --tile $tile --steps 5 --warmup 3 --no-cpu --e2e-steps 0 --trace gpurun_out/trace_st$tile.npy $@ > gpurun_out/bench_st.json 2>/dev/null
  echo "tile=$tile $(python -c "import json;j=json.loads(open('gpurun_out/bench_st.json').read().splitlines()[-1]);print(round(j['value'],1),'GCUPS')")"
  python scripts/trace_quick.py gpurun_out/trace_st$tile.npy 32768 2>/dev/null
done
