"""Traceback timing probe: per-window cost vs n (L2-resident vs HBM-resident matrices)."""
import torch
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb

for n in (1024, 4096, 16384, 32768):
    S, R = inputs.device_problem(n, 10, device="cuda")
    nwb.nw_fill(S, R, 10)
    ts = []
    for _ in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ops, length = nwb.nw_traceback(S, R, 10)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    L = int(length.item())
    ms = sorted(ts)[2]
    print(f"n={n} len={L} ms={ms:.3f} us/step={ms*1e3/L:.4f} us/window(~{L/33:.0f})={ms*1e3/(L/33):.2f}")
    del S, R
