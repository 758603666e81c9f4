#!/bin/bash
# round-2 kept bench lines: every config, config 2's three tiles, the paper's Opt / Unopt pair,
# the ref-from-sequences variant, the aligned layout; then the launch list and one ncu --set full
# capture of the default config-3 kernel (profiles/)
mkdir -p gpurun_out/bl
B="timeout 600 python bench.py"
$B --config 3 --steps 20 --warmup 3 > gpurun_out/bl/c3.json 2> gpurun_out/bl/c3.err
$B --config 1 --steps 50 --warmup 5 > gpurun_out/bl/c1.json 2> gpurun_out/bl/c1.err
for t in 16 32 64; do $B --config 2 --tile $t --steps 20 --warmup 3 --no-cpu > gpurun_out/bl/c2_t$t.json 2>>gpurun_out/bl/c2.err; done
$B --config 2 --tile 64 --steps 20 --warmup 3 > gpurun_out/bl/c2_cpu.json 2>>gpurun_out/bl/c2.err
$B --config 4 --steps 5 --warmup 3 > gpurun_out/bl/c4.json 2> gpurun_out/bl/c4.err
for n in 2 3; do for v in diagonal unopt; do
  $B --config $n --variant $v --tile 16 --steps 5 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bl/c${n}_$v.json 2>>gpurun_out/bl/opt.err
done; done
$B --config 3 --variant seq --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bl/c3_seq.json 2>>gpurun_out/bl/seq.err
$B --config 3 --layout aligned --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/bl/c3_aligned.json 2>>gpurun_out/bl/al.err
$B --impl reference --config 3 --steps 2 --warmup 3 > gpurun_out/bl/ref_c3.json 2>>gpurun_out/bl/ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -s 3 -c 40 --csv --log-file gpurun_out/bl/launches_c3.csv python bench.py --config 3 --steps 2 --warmup 3 --no-cpu --e2e-steps 0 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nw_wave -s 1 -c 1 -o gpurun_out/bl/prof_c3 -f python scripts/one_fill.py 32768 0 2 > gpurun_out/bl/ncu.log 2>&1
ls -la gpurun_out/bl
