"""Debug: print where the GPU fill differs from the oracle for a few sizes / tiles."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import inputs, oracle
import paper_conf_sc_munksgaardhso22_b200 as nwb
for n in [int(x) for x in sys.argv[1].split(",")]:
    for tile in (0, 128):
        score, ref = inputs.make_problem(n, 10, seed=n)
        want = oracle.nw_ref(score.copy(), ref, 10)
        s = torch.from_numpy(score).cuda(); r = torch.from_numpy(ref).cuda()
        nwb.nw_fill(s, r, 10, tile); torch.cuda.synchronize()
        got = s.cpu().numpy()
        bad = np.argwhere(got != want)
        print(f"n={n} tile={tile}: {len(bad)} bad", end="")
        if len(bad):
            rows = np.unique(bad[:, 0]); cols = np.unique(bad[:, 1])
            print(f" rows {rows[:20].tolist()} cols {cols[:20].tolist()} first {bad[:4].tolist()} got {got[tuple(bad[0])]} want {want[tuple(bad[0])]}")
        else:
            print()
