"""Every kernel of libnwb200.so once at a small size (for compute-sanitizer memcheck / racecheck /
synccheck runs, scripts/gpu_sanitize.sh): single pairs (every tile), a batch in pair mode, strips
with halos, the ref-from-sequences kernels, the diagonal / Unopt baselines, the traceback."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import inputs
import oracle
import paper_conf_sc_munksgaardhso22_b200 as nwb

bad = []


def check(name, got, want):
    if not np.array_equal(got, want):
        bad.append(name)


n, p = int(sys.argv[1]) if len(sys.argv) > 1 else 300, 10
s, r = inputs.make_problem(n, p, seed=3)
want = oracle.nw_ref(s.copy(), r, p)
for tile in (0, 16, 32, 64, 128, 256):
    S, R = torch.from_numpy(s.copy()).cuda(), torch.from_numpy(r).cuda()
    nwb.nw_fill(S, R, p, tile); torch.cuda.synchronize()
    check(f"fill{tile}", S.cpu().numpy(), want)
for fn in (nwb.nw_fill_diagonal, nwb.nw_fill_unopt):
    S = torch.from_numpy(s.copy()).cuda()
    fn(S, R, p, 16); torch.cuda.synchronize()
    check(fn.__name__, S.cpu().numpy(), want)
nwb.nw_debug_set_cluster(True)
S = torch.from_numpy(s.copy()).cuda(); nwb.nw_fill(S, R, p, 0); torch.cuda.synchronize()
check("cluster", S.cpu().numpy(), want)
nwb.nw_debug_set_cluster(False)
B = 3
ss = [inputs.make_problem(n, p, seed=inputs.pair_seed(k)) for k in range(B)]
SB = torch.from_numpy(np.stack([a for a, _ in ss])).cuda(); RB = torch.from_numpy(np.stack([b for _, b in ss])).cuda()
nwb.nw_debug_set_pair_mode(1); nwb.nw_fill_batch(SB, RB, p, 0); torch.cuda.synchronize(); nwb.nw_debug_set_pair_mode(0)
for k in range(B):
    check(f"batch{k}", SB[k].cpu().numpy(), oracle.nw_ref(ss[k][0].copy(), ss[k][1], p))
# two strips with a halo
W = nwb.nw_band_width(0)
w0 = W
ls0, lr0 = s[:, :w0 + 1].copy(), r[:, :w0 + 1].copy()
ls1, lr1 = s[:, w0:].copy(), r[:, w0:].copy()
ls1[1:, 0] = inputs.SENTINEL
halo = torch.zeros(n + 2, dtype=torch.int64, device="cuda")
S0, S1 = torch.from_numpy(ls0).cuda(), torch.from_numpy(ls1).cuda()
nwb.nw_fill_sharded(S0, torch.from_numpy(lr0).cuda(), p, halo_out=halo, epoch=1)
nwb.nw_fill_sharded(S1, torch.from_numpy(lr1).cuda(), p, halo_in=halo, epoch=1)
torch.cuda.synchronize()
check("strip0", S0.cpu().numpy()[:, 1:], want[:, 1:w0 + 1]); check("strip1", S1.cpu().numpy()[:, 1:], want[:, w0 + 1:])
a, b = inputs.gen_pair(n, 11)
rs = inputs.build_ref(a, b)
s2 = inputs.init_borders(inputs.aligned_matrix(n), p)
inputs.fill_interior(s2, inputs.SENTINEL)
for tile in (0, 64):
    S = torch.from_numpy(s2.copy()).cuda()
    nwb.nw_fill_seq(S, torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda(), inputs.blosum62(), p, tile)
    torch.cuda.synchronize()
    check(f"seq{tile}", S.cpu().numpy(), oracle.nw_ref(s2.copy(), rs, p))
S, R = torch.from_numpy(want.copy()).cuda(), torch.from_numpy(r).cuda()
ops, length = nwb.nw_traceback(S, R, p)
torch.cuda.synchronize()
tw = oracle.nw_traceback_ref(want, r, p)
check("traceback", ops[: int(length.item())].cpu().numpy(), tw)
print("BAD", bad) if bad else print("ALL OK")
