#!/bin/bash
# release/acquire progress words (NW_DEBUG_SKIP=16 build) vs the relaxed default: cost and racecheck
mkdir -p gpurun_out
export NW_SPIN_LIMIT_MS=60000
for v in default strict; do
  if [ "$v" = default ]; then unset NW_LIB; else export NW_LIB=$PWD/build_variants/$v.so; fi
  for c in 3 4; do
    timeout 300 python bench.py --config $c --steps 5 --warmup 3 --no-cpu --e2e-steps 0 2>>gpurun_out/st.err | tail -1 | sed "s/^/$v-c$c /" >> gpurun_out/st_bench.jsonl
  done
done
export NW_LIB=$PWD/build_variants/strict.so
timeout 1200 compute-sanitizer --tool racecheck --print-limit 10 python scripts/sanitize_small.py 300 > gpurun_out/st_racecheck.txt 2>&1
grep -E "RACECHECK SUMMARY|ALL OK|BAD" gpurun_out/st_racecheck.txt
unset NW_LIB
timeout 1200 compute-sanitizer --tool memcheck --print-limit 10 python scripts/sanitize_small.py 300 > gpurun_out/san_memcheck.txt 2>&1
grep -E "ERROR SUMMARY|ALL OK|BAD" gpurun_out/san_memcheck.txt
