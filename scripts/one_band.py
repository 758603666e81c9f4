import sys, torch
sys.path.insert(0, ".")
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb
n = 32768; tile = int(sys.argv[1]) if len(sys.argv) > 1 else 128
W = nwb.nw_band_width(tile)
S, R = inputs.device_problem(n, 10, device="cuda")
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 1
S1, R1 = S[:, : nb * W + 1], R[:, : nb * W + 1]
for _ in range(3):
    nwb.nw_fill_sharded(S1, R1, 10, tile=tile)
torch.cuda.synchronize()
