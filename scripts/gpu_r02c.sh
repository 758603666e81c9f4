#!/bin/bash
# Round-2 final record: smoke, the whole GPU suite, kept bench lines for every config,
# the launch list of the default bench command and one ncu --set full capture of its kernel.
export NW_SPIN_LIMIT_MS=10000
O=gpurun_out/r02c; mkdir -p $O
timeout 180 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo smoke_rc=$?; tail -1 $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --maxfail=8 > $O/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -3 $O/pytest_gpu.log
B="timeout 600 python bench.py"
$B --config 3 --steps 20 --warmup 3 > $O/c3.json 2> $O/c3.err; echo c3_rc=$?
$B --config 3 --layout aligned --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $O/c3_aligned.json 2>> $O/c3.err
for t in 16 64; do $B --config 3 --tile $t --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > $O/c3_t$t.json 2>> $O/c3.err; done
python scripts/e2e_probe.py > $O/e2e_probe.txt 2>&1
$B --config 1 --steps 50 --warmup 5 > $O/c1.json 2> $O/c1.err
for t in 16 32 64; do $B --config 2 --tile $t --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $O/c2_t$t.json 2>> $O/c2.err; done
$B --config 4 --steps 5 --warmup 3 > $O/c4.json 2> $O/c4.err
$B --config 3 --variant seq --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > $O/c3_seq.json 2>> $O/c3.err
$B --impl reference --config 3 --steps 2 --warmup 3 > $O/ref_c3.json 2> $O/ref.err
for f in $O/c3.json $O/c3_aligned.json $O/c1.json $O/c2_t16.json $O/c2_t32.json $O/c2_t64.json $O/c4.json $O/c3_seq.json; do python scripts/show_bench.py $f; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 3 -c 40 --csv --log-file $O/launches_c3.csv python bench.py --config 3 --steps 2 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1; echo ncu1_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 1 -c 1 -o $O/prof_c3 -f python scripts/one_fill.py 32768 0 2 > $O/ncu.log 2>&1; echo ncu2_rc=$?
