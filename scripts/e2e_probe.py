"""End-to-end nw_fill_host timing at n = 32768 for host modes / pipeline block sizes:
python scripts/e2e_probe.py"""
import sys, time
import torch
sys.path.insert(0, ".")
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb
n, p = 32768, 10
S, R = inputs.device_problem(n, p, device="cuda")
hs = torch.empty(S.shape, dtype=torch.int32).pin_memory(); hs.copy_(S.cpu())
hr = torch.empty(R.shape, dtype=torch.int32).pin_memory(); hr.copy_(R.cpu())
del S, R
for mode, rows in [(2, 0), (2, 128), (2, 512), (2, 1024), (2, 4096), (1, 0), (0, 0)]:
    nwb.nw_debug_set_host_mode(mode); nwb.nw_debug_set_host_block_rows(rows)
    ts = []
    for _ in range(3):
        t0 = time.perf_counter(); nwb.nw_fill_host(hs.numpy(), hr.numpy(), p, 0, 0); ts.append(time.perf_counter() - t0)
    print(f"mode {mode} block_rows {rows:5d}: {min(ts) * 1e3:7.1f} ms  {n * n / min(ts) / 1e9:5.2f} GCUPS", flush=True)
nwb.nw_debug_set_host_mode(2); nwb.nw_debug_set_host_block_rows(0)
