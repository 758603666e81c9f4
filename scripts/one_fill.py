"""One nw_fill (for ncu captures): python scripts/one_fill.py n tile [reps]"""
import sys
import torch
sys.path.insert(0, ".")
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb
n = int(sys.argv[1]); tile = int(sys.argv[2]); reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
S, R = inputs.device_problem(n, 10, device="cuda")
for _ in range(reps):
    nwb.nw_fill(S, R, 10, tile)
torch.cuda.synchronize()
