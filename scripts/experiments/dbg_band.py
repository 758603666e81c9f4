"""Parity debugging of the band kernel: python scripts/dbg_band.py n p tile reps [family]"""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import inputs
import oracle
import paper_conf_sc_munksgaardhso22_b200 as nwb
n, p, tile, reps = (int(x) for x in sys.argv[1:5])
fam = sys.argv[5] if len(sys.argv) > 5 else "random"
score, ref = inputs.make_problem(n, p, seed=3, family=fam)
want = oracle.nw_ref(score.copy(), ref, p)
W = nwb.nw_band_width(tile)
for rep in range(reps):
    s = torch.from_numpy(score.copy()).cuda()
    r = torch.from_numpy(ref.copy()).cuda()
    nwb.nw_fill(s, r, p, tile)
    torch.cuda.synchronize()
    got = s.cpu().numpy()
    bad = np.argwhere(got != want)
    if len(bad) == 0:
        print(f"rep {rep}: ok")
        continue
    i0, j0 = bad[np.lexsort((bad[:, 0], bad[:, 1]))][0]
    bands = np.bincount((bad[:, 1] - 1) // W)
    first_rows = {int(b): int(bad[(bad[:, 1] - 1) // W == b][:, 0].min()) for b in np.unique((bad[:, 1] - 1) // W)}
    print(f"rep {rep}: {len(bad)} bad; first (row {i0}, col {j0}) band {(j0-1)//W} got {got[i0,j0]} want {want[i0,j0]};"
          f" first bad row per band {first_rows}")
    # first bad column within the earliest band, and rows
    b0 = (j0 - 1) // W
    inb = bad[(bad[:, 1] - 1) // W == b0]
    print("   earliest band cols:", sorted(set((inb[:, 1] - 1 - b0 * W).tolist()))[:20], " rows:", sorted(set(inb[:, 0].tolist()))[:20])
