"""One fill + traceback at n (argv[1]) for ncu captures of the traceback kernels."""
import sys
import torch
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
S, R = inputs.device_problem(n, 10, device="cuda")
nwb.nw_fill(S, R, 10)
for _ in range(2):
    ops, length = nwb.nw_traceback(S, R, 10)
torch.cuda.synchronize()
print("len", int(length.item()))
