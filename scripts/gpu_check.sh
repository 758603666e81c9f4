set -x
nvidia-smi --query-gpu=name,clocks.max.sm,memory.total --format=csv
python -c "import torch;print(torch.cuda.get_device_name())"
timeout 180 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?; tail -5 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -q --maxfail=8 -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest_rc=$?; tail -40 gpurun_out/pytest_gpu.log
timeout 400 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo bench_rc=$?; cat gpurun_out/bench_c3.json; tail -5 gpurun_out/bench_c3.err
