import sys, torch, numpy as np
sys.path.insert(0, ".")
import inputs
import paper_conf_sc_munksgaardhso22_b200 as nwb
n = 32768; tile = int(sys.argv[1]) if len(sys.argv) > 1 else 128; nb = int(sys.argv[2]) if len(sys.argv) > 2 else 3
W = nwb.nw_band_width(tile)
S, R = inputs.device_problem(n, 10, device="cuda")
S1, R1 = S[:, : nb * W + 1], R[:, : nb * W + 1]
for _ in range(2):
    nwb.nw_fill_sharded(S1, R1, 10, tile=tile)
tb = torch.zeros(16 * nb, dtype=torch.int64, device="cuda")
nwb.nw_debug_set_trace(tb[: 8 * nb].view(nb, 8))
nwb.nw_fill_sharded(S1, R1, 10, tile=tile)
torch.cuda.synchronize()
nwb.nw_debug_set_trace(None)
t = tb.cpu().numpy().astype(np.int64)
tr = t[: 8 * nb].reshape(nb, 8); t2 = t[8 * nb:].reshape(nb, 8)
t0 = tr[:, 1].min()
for b in range(nb):
    r = tr[b]; blk = r[3] >> 16
    print(f"band {b}: start {(r[1]-t0)/1e3:8.1f} us end {(r[2]-t0)/1e3:8.1f} us cyc/row {r[7]/n:6.1f} blk {blk/n:6.1f} "
          f"ev {r[4]/n:6.1f} wait {r[5]/n:5.1f} spin {r[6]/n:6.1f} | stage busy {t2[b,0]/n:6.1f} wait {t2[b,1]/n:6.1f}"
          f" | phases state {t2[b,2]/n:5.1f} arrive {t2[b,3]/n:5.1f} border {t2[b,4]/n:5.1f} ready {t2[b,5]/n:5.1f} bp {t2[b,6]/n:5.1f}")
