"""Traceback timing probe for a batch: 4096 pairs x n = 2048 (config 4 shape), fill then traceback."""
import torch
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb

B, n = 4096, 2048
S = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
R = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
for k in range(B):
    inputs.device_problem(n, 10, seed=inputs.pair_seed(k), device="cuda", score=S[k], ref=R[k])
nwb.nw_fill_batch(S, R, 10)
ts = []
for _ in range(5):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ops, length = nwb.nw_traceback_batch(S, R, 10)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
print(f"batch B={B} n={n} steps={int(length.to(torch.int64).sum())} ms={sorted(ts)[2]:.3f} min={min(ts):.3f} bad={int((length < 0).sum())}")
