"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

The bar is BIT-EXACT on every cell (integer work): the recurrence plus the
borders determine the matrix uniquely (reading R13), so any schedule must reproduce the
oracle's int32 values exactly.  The interior is pre-filled with the sentinel 0x80000000, so an
unwritten cell fails too.  Inputs come from the seeded generator in inputs/ (no arithmetic of
the method there); expected values only ever come from oracle/.
"""
import os

import numpy as np
import pytest

import inputs
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

torch = pytest.importorskip("torch")
import paper_conf_sc_munksgaardhso22_b200 as nwb  # noqa: E402

pytestmark = pytest.mark.gpu


def to_dev(a, ld=None, offset=0):
    """(n+1, n+1) host matrix -> CUDA int32 view with pitch ld and a base shifted by `offset`
    elements inside a larger allocation (exercises every 16-byte phase of the rows)."""
    n1 = a.shape[0]
    ld = a.shape[1] if ld is None else ld
    buf = torch.full((offset + n1 * ld + 8,), -7, dtype=torch.int32, device="cuda")
    view = buf[offset:offset + n1 * ld].view(n1, ld)
    view[:, : a.shape[1]] = torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return view


def expect(score, ref, p):
    return oracle.nw_ref(score.copy(), ref, p)


def gpu_fill(score, ref, p, tile, fn=None, ld=None, offset=0, ref_offset=None):
    n = score.shape[0] - 1
    s = to_dev(score, ld, offset)
    r = to_dev(ref, ld, (offset * 3) % 4 if ref_offset is None else ref_offset)
    (fn or nwb.nw_fill)(s, r, p, tile)
    torch.cuda.synchronize()
    return s[:, : n + 1].cpu().numpy()


SIZES = [1, 2, 3, 15, 16, 17, 31, 32, 33, 63, 64, 65, 100, 127, 128, 129, 255, 256, 257, 1000, 1024]


@pytest.mark.parametrize("tile", [0, 16, 64])
@pytest.mark.parametrize("n", SIZES)
def test_fill_sizes(n, tile):
    score, ref = inputs.make_problem(n, 10, seed=n)
    np.testing.assert_array_equal(gpu_fill(score, ref, 10, tile), expect(score, ref, 10))


@pytest.mark.parametrize("p", [0, 1, 3, 10, 1000])
@pytest.mark.parametrize("family", ["random", "homologous", "const", "borders"])
def test_fill_families(family, p):
    n = 700
    kw = {"family": "const", "const_ref": 5} if family == "const" else {"family": family}
    if family == "borders":
        kw = {"family": "random", "border_seed": 99}
    score, ref = inputs.make_problem(n, p, seed=3, **kw)
    for tile in (0, 128):
        np.testing.assert_array_equal(gpu_fill(score, ref, p, tile), expect(score, ref, p))


@pytest.mark.parametrize("ld_extra,offset", [(0, 1), (0, 2), (0, 3), (3, 0), (4, 0), (7, 1), (31, 2)])
def test_fill_pitch_and_alignment(ld_extra, offset):
    n = 517
    score, ref = inputs.make_problem(n, 10, seed=11)
    got = gpu_fill(score, ref, 10, 0, ld=n + 1 + ld_extra, offset=offset)
    np.testing.assert_array_equal(got, expect(score, ref, 10))


@pytest.mark.parametrize("tile", [0, 128])
@pytest.mark.parametrize("n", [1, 2, 17, 100, 128, 129, 257, 1000, 1024, 1531])
def test_fill_aligned_layout(n, tile):
    """16-byte aligned interior rows (pitch 0 mod 4, element (0, 1) on a 16-byte boundary)."""
    score, ref = inputs.make_problem(n, 10, seed=100 + n)
    ld = (n + 1 + 3) & ~3
    got = gpu_fill(score, ref, 10, tile, ld=ld, offset=3, ref_offset=3)
    np.testing.assert_array_equal(got, expect(score, ref, 10))


@pytest.mark.parametrize("tile", [0, 16, 64])
def test_range_edge_bit_exact(tile):
    """At the edge of the range contract: n = 64, p = 8259040 (65 (2p + 1024) just below 2^30),
    borders of magnitude 2^30 - 1 (the caller's promise) with random signs, ref at +-NW_REF_MAX:
    the gap-normalised intermediates reach ~2^31 - 2^10 and the result must still be bit-exact."""
    n, p = 64, 8259040
    rng = np.random.default_rng(5)
    score = np.zeros((n + 1, n + 1), dtype=np.int32)
    big = (1 << 30) - 1
    score[0, :] = rng.choice([-big, big], n + 1)
    score[:, 0] = rng.choice([-big, big], n + 1)
    score[1:, 1:] = inputs.SENTINEL
    ref = np.zeros((n + 1, n + 1), dtype=np.int32)
    ref[1:, 1:] = rng.choice([-nwb.NW_REF_MAX, nwb.NW_REF_MAX, 0, 7], (n, n))
    want = expect(score, ref, p)
    np.testing.assert_array_equal(gpu_fill(score, ref, p, tile), want)
    np.testing.assert_array_equal(gpu_fill(score, ref, p, 16, fn=nwb.nw_fill_diagonal), want)
    # one past the edge, and round 1's counterexample, are rejected before any work
    for bad in (p + 1, 16776703):
        with pytest.raises(nwb.NwError):
            gpu_fill(score, ref, bad, tile)


def test_config1_bit_exact_and_idempotent():
    """BASELINE.json config 1: n=1024, p=10, tile=16, repeated back to back (Table I ran 1000x)."""
    n, p = 1024, 10
    score, ref = inputs.make_problem(n, p)
    want = expect(score, ref, p)
    s, r = to_dev(score), to_dev(ref)
    for _ in range(200):
        nwb.nw_fill(s, r, p, 16)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(s.cpu().numpy(), want)


@pytest.mark.parametrize("tile", [0, 16, 64])
def test_flag_race_stress_1000(tile):
    """The band-to-band handoff under repetition (Table I ran 1000 times):
    n = 1024, 1000 launches, each on a sentinel-reset interior and each compared on the device
    with the oracle's matrix (a stale or torn border entry would show as a wrong cell)."""
    n, p = 1024, 10
    score, ref = inputs.make_problem(n, p, seed=1000 + tile)
    want = torch.from_numpy(expect(score, ref, p)).cuda()
    s, r = to_dev(score), to_dev(ref)
    bad = []
    for rep in range(1000):
        s[1:, 1:] = inputs.SENTINEL
        nwb.nw_fill(s, r, p, tile)
        if not torch.equal(s, want):
            bad.append(rep)
    torch.cuda.synchronize()
    assert not bad, bad[:10]


@pytest.mark.parametrize("grid", [1, 3])
def test_small_grids_deadlock_free(grid):
    """Ticket order => a CTA only waits on bands held by running CTAs: a 1-CTA grid must finish."""
    n = 600
    score, ref = inputs.make_problem(n, 10, seed=5)
    try:
        nwb.nw_debug_set_grid(grid)
        got = gpu_fill(score, ref, 10, 16)
    finally:
        nwb.nw_debug_set_grid(0)
    np.testing.assert_array_equal(got, expect(score, ref, 10))


def test_workspace_reuse_across_sizes():
    """Epoch tags keep stale band borders of earlier calls (other n, other tile) harmless."""
    for n, tile in [(300, 0), (1000, 128), (129, 0), (2000, 16), (300, 128)]:
        score, ref = inputs.make_problem(n, 10, seed=n + tile)
        np.testing.assert_array_equal(gpu_fill(score, ref, 10, tile), expect(score, ref, 10))


@pytest.mark.parametrize("tile", [16, 32, 64])
@pytest.mark.parametrize("n", [1, 16, 47, 64, 200, 1024])
def test_diagonal_and_unopt(n, tile):
    score, ref = inputs.make_problem(n, 10, seed=7 + n)
    want = expect(score, ref, 10)
    np.testing.assert_array_equal(gpu_fill(score, ref, 10, tile, fn=nwb.nw_fill_diagonal), want)
    np.testing.assert_array_equal(gpu_fill(score, ref, 10, tile, fn=nwb.nw_fill_unopt), want)


def test_fill_host_e2e():
    n = 999
    score, ref = inputs.make_problem(n, 10, seed=21)
    want = expect(score, ref, 10)
    got = score.copy()
    nwb.nw_fill_host(got, ref, 10, 0, 0)
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("mode,block_rows", [(1, 0), (0, 0), (2, 0), (2, 37), (2, 256)])
@pytest.mark.parametrize("n,tile", [(999, 0), (1500, 64), (3000, 0), (1000, 16)])
def test_fill_host_pinned(n, tile, mode, block_rows):
    """Pinned host buffers in every host mode: zero copy (the kernel on the host link), staged, and
    the copy-engine pipeline (ref blocks gated into the kernel, score blocks released back as every
    band stores them) with automatic, odd and tile-sized row blocks."""
    score, ref = inputs.make_problem(n, 10, seed=23)
    want = expect(score, ref, 10)
    hs = torch.from_numpy(score.copy()).pin_memory()
    hr = torch.from_numpy(ref).pin_memory()
    try:
        nwb.nw_debug_set_host_mode(mode)
        nwb.nw_debug_set_host_block_rows(block_rows)
        nwb.nw_fill_host(hs.numpy(), hr.numpy(), 10, tile, 0)
    finally:
        nwb.nw_debug_set_host_mode(2)
        nwb.nw_debug_set_host_block_rows(0)
    np.testing.assert_array_equal(hs.numpy(), want)


@pytest.mark.parametrize("pinned,mode,block_rows", [(False, 2, 0), (True, 1, 0), (True, 2, 0), (True, 2, 50), (True, 2, 301),
                                                    (True, 2, 7)])
def test_fill_batch_host(pinned, mode, block_rows):
    """Batched end to end from host arrays: staged (pageable), zero copy and the pipeline (pinned),
    with row blocks inside pairs (50, 7), equal to a pair (301 = n + 1) and automatic."""
    B, n = 5, 300
    ss, rs, want = [], [], []
    for k in range(B):
        s, r = inputs.make_problem(n, 10, seed=inputs.pair_seed(k))
        ss.append(s); rs.append(r); want.append(expect(s, r, 10))
    S, R = np.stack(ss), np.stack(rs)
    if pinned:
        St, Rt = torch.from_numpy(S).pin_memory(), torch.from_numpy(R).pin_memory()
        S, R = St.numpy(), Rt.numpy()
    try:
        nwb.nw_debug_set_host_mode(mode)
        nwb.nw_debug_set_host_block_rows(block_rows)
        nwb.nw_fill_batch_host(S, R, 10, 0, 0)
    finally:
        nwb.nw_debug_set_host_mode(2)
        nwb.nw_debug_set_host_block_rows(0)
    for k in range(B):
        np.testing.assert_array_equal(S[k], want[k])


@pytest.mark.parametrize("B,n,tile", [(1, 64, 0), (5, 100, 16), (7, 257, 0), (33, 64, 64), (3, 2048, 0), (4, 700, 128)])
def test_batch(B, n, tile):
    probs = [inputs.make_problem(n, 10, seed=inputs.pair_seed(k)) for k in range(B)]
    S = torch.from_numpy(np.stack([s for s, _ in probs])).cuda()
    R = torch.from_numpy(np.stack([r for _, r in probs])).cuda()
    nwb.nw_fill_batch(S, R, 10, tile)
    torch.cuda.synchronize()
    got = S.cpu().numpy()
    for k, (s, r) in enumerate(probs):
        np.testing.assert_array_equal(got[k], expect(s, r, 10), err_msg=f"pair {k}")


def split_strips(score, ref, G, tile):
    """Cut a global problem into G column strips (local (n+1) x (w+1) matrices, col 0 = halo)
    with the multi-GPU driver's bounds (widths multiples of the band width; last one ragged)."""
    from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
    n = score.shape[0] - 1
    out = []
    for st in nwdist.strip_bounds(n, G, align=nwb.nw_band_width(tile)):
        a, b = st.col0, st.col0 + st.w
        ls = score[:, a:b + 1].copy()
        lr = ref[:, a:b + 1].copy()
        if st.rank > 0:
            ls[1:, 0] = inputs.SENTINEL  # the halo must come from the left rank, not from here
        out.append((a, b, ls, lr))
    return out


@pytest.mark.parametrize("G,n,tile", [(2, 256, 0), (3, 500, 16), (4, 1024, 0), (8, 1000, 64), (3, 1111, 128), (2, 600, 128), (4, 1500, 0)])
def test_sharded_single_device(G, n, tile):
    """Config 5's protocol on one GPU: G strips launched in rank order on one stream, each
    pushing its right border into the next strip's halo (epoch-tagged entries)."""
    score, ref = inputs.make_problem(n, 10, seed=17)
    want = expect(score, ref, 10)
    strips = split_strips(score, ref, G, tile)
    halos = [torch.zeros(n + 2, dtype=torch.int64, device="cuda") for _ in range(G + 1)]  # n+2: see nw.h
    for epoch in (1, 2, 7):                        # re-use of halo buffers across calls
        locs = []
        for g, (a, b, ls, lr) in enumerate(strips):
            if b == a:
                locs.append(None)
                continue
            s_dev, r_dev = to_dev(ls), to_dev(lr)
            nwb.nw_fill_sharded(s_dev, r_dev, 10, halo_in=halos[g] if g > 0 else None,
                                halo_out=halos[g + 1] if g < G - 1 else None, epoch=epoch, tile=tile)
            locs.append(s_dev)
        torch.cuda.synchronize()
        for g, (a, b, ls, lr) in enumerate(strips):
            if locs[g] is None:
                continue
            got = locs[g].cpu().numpy()
            np.testing.assert_array_equal(got[:, 1:], want[:, a + 1:b + 1], err_msg=f"strip {g} epoch {epoch}")
        # halo entries carry the tag and the left neighbour's last column
        h = halos[1].cpu().numpy().view(np.uint64)[: n + 1]
        assert (h[1:] >> np.uint64(32) == epoch).all()
        np.testing.assert_array_equal((h[1:] & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32),
                                      want[1:, strips[0][1]])


@pytest.mark.parametrize("G,n,tile", [(2, 4096, 0), (3, 3000, 64), (4, 8192, 0), (2, 2100, 128)])
def test_sharded_concurrent_streams(G, n, tile):
    """Config 5's protocol with the strips running CONCURRENTLY on one GPU: each strip on its own
    stream, launched in reverse rank order, so every consumer is already spinning on its halo tags
    while its producer pushes the right border column row by row (system-scope stores, as to a
    peer GPU: halo_out_is_peer); grids capped so all strips are co-resident; the halo buffers are
    reused across three calls (epochs 5, 6, 9)."""
    score, ref = inputs.make_problem(n, 10, seed=21)
    want = expect(score, ref, 10)
    strips = split_strips(score, ref, G, tile)
    halos = [torch.zeros(n + 2, dtype=torch.int64, device="cuda") for _ in range(G + 1)]
    streams = [torch.cuda.Stream() for _ in range(G)]
    devs = [(to_dev(ls), to_dev(lr)) for (a, b, ls, lr) in strips]
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    torch.cuda.synchronize()
    try:
        nwb.nw_debug_set_grid(max(1, sms // G))
        for epoch in (5, 6, 9):
            for s_dev, _ in devs:
                s_dev[1:, 1:] = inputs.SENTINEL
            torch.cuda.synchronize()
            for g in reversed(range(G)):
                s_dev, r_dev = devs[g]
                nwb.nw_fill_sharded(s_dev, r_dev, 10, halo_in=halos[g] if g > 0 else None,
                                    halo_out=halos[g + 1] if g < G - 1 else None, epoch=epoch,
                                    halo_out_is_peer=True, tile=tile, stream=streams[g])
            torch.cuda.synchronize()
            for g, (a, b, ls, lr) in enumerate(strips):
                got = devs[g][0].cpu().numpy()
                np.testing.assert_array_equal(got[:, 1:], want[:, a + 1:b + 1], err_msg=f"strip {g} epoch {epoch}")
    finally:
        nwb.nw_debug_set_grid(0)


def test_watchdog_traps_a_missing_halo():
    """The spin watchdog: a strip whose halo is never written must not hang the GPU.
    With NW_SPIN_LIMIT_MS=300 the kernel traps, the caller sees a CUDA error at synchronisation
    (a sticky error: that process's context is gone), and a fresh process then fills correctly."""
    import subprocess
    import sys
    hang = r'''
import sys; sys.path.insert(0, %r)
import numpy as np, torch, inputs, paper_conf_sc_munksgaardhso22_b200 as nwb
s, r = inputs.make_problem(512, 10)
S = torch.from_numpy(s).cuda(); R = torch.from_numpy(r).cuda()
halo = torch.zeros(514, dtype=torch.int64, device="cuda")      # never written: tags stay 0
nwb.nw_fill_sharded(S, R, 10, halo_in=halo, epoch=7, tile=0)   # enqueued fine ...
try:
    torch.cuda.synchronize()
    print("no-error")
except Exception as e:
    print("cuda-error", type(e).__name__)
''' % ROOT
    env = dict(os.environ, NW_SPIN_LIMIT_MS="300")
    out = subprocess.run([sys.executable, "-c", hang], env=env, capture_output=True, text=True, timeout=300)
    assert "cuda-error" in out.stdout, (out.stdout, out.stderr[-2000:])
    ok = r'''
import sys; sys.path.insert(0, %r)
import numpy as np, torch, inputs, oracle, paper_conf_sc_munksgaardhso22_b200 as nwb
s, r = inputs.make_problem(512, 10)
want = oracle.nw_ref(s.copy(), r, 10)
S = torch.from_numpy(s).cuda(); R = torch.from_numpy(r).cuda()
nwb.nw_fill(S, R, 10, 0); torch.cuda.synchronize()
print("ok" if np.array_equal(S.cpu().numpy(), want) else "mismatch")
''' % ROOT
    out = subprocess.run([sys.executable, "-c", ok], capture_output=True, text=True, timeout=300)
    assert "ok" in out.stdout, (out.stdout, out.stderr[-2000:])


def _stream_compare(s_dev, score_row0, ref, n, p, chunk=2048):
    """Full-size check with the O(n)-memory streaming oracle, rows in chunks."""
    st = oracle.NwRefStream(n, p, score_row0)
    for i0 in range(1, n + 1, chunk):
        i1 = min(n + 1, i0 + chunk)
        got = s_dev[i0:i1].cpu().numpy()
        want = st.rows(ref[i0:i1], got[:, 0].copy())
        np.testing.assert_array_equal(got, want, err_msg=f"rows {i0}..{i1}")
    st.close()


@pytest.mark.parametrize("n,tile", [(16384, 128), (16384, 64), (32768, 0)])
def test_full_size_configs_bit_exact(n, tile):
    """BASELINE.json configs 2/3 at full size, in the launch configuration bench.py times:
    every cell against the streaming oracle."""
    p = 10
    a, b = inputs.gen_pair(n, inputs.SEED)
    ref = inputs.build_ref(a, b)
    score = inputs.init_borders(inputs.aligned_matrix(n), p)
    s_dev, r_dev = torch.from_numpy(score).cuda(), torch.from_numpy(ref).cuda()
    s_dev[1:, 1:] = inputs.SENTINEL
    nwb.nw_fill(s_dev, r_dev, p, tile)
    nwb.nw_fill(s_dev, r_dev, p, tile)
    torch.cuda.synchronize()
    _stream_compare(s_dev, score[0], ref, n, p)


def _stream_compare_strips(parts, n, p, seed=inputs.SEED, chunk=2048):
    """Config-5 size check: the streaming oracle over the full width, each row chunk compared with
    the strips' local columns (parts: list of (col0, w, local score on the device))."""
    a, b = inputs.gen_pair(n, seed)
    row0 = -np.arange(n + 1, dtype=np.int32) * p
    st = oracle.NwRefStream(n, p, row0)
    for i0 in range(1, n + 1, chunk):
        i1 = min(n + 1, i0 + chunk)
        ref_rows = inputs.build_ref_block(a, b, i0, i1)
        want = st.rows(ref_rows, -np.arange(i0, i1, dtype=np.int32) * p)
        for col0, w, s_dev in parts:
            got = s_dev[i0:i1, 1:w + 1].cpu().numpy()
            np.testing.assert_array_equal(got, want[:, col0 + 1:col0 + w + 1], err_msg=f"rows {i0}..{i1} strip at {col0}")
    st.close()


@pytest.mark.parametrize("G", [1, 2, 4, 8])
def test_config5_full_size_strips(G):
    """BASELINE.json config 5 at its size, n = 65536 (the one matrix above 2^31 elements: the
    kernels' 64-bit addressing): G = 1 is nw_fill on the whole matrix; G = 2, 4, 8 are the strips
    the multi-GPU driver cuts (widths multiples of the band width), run on one device in rank order
    with each strip pushing its right border into the next strip's halo.  Every cell is checked
    against the streaming oracle."""
    from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
    n, p, tile = 65536, 10, 0
    free, _ = torch.cuda.mem_get_info()
    if free < 40e9:
        pytest.skip("needs ~35 GB of device memory")
    parts = []
    if G == 1:
        S, R = inputs.device_problem(n, p, device="cuda")
        nwb.nw_fill(S, R, p, tile)
        torch.cuda.synchronize()
        del R
        parts.append((0, n, S))
    else:
        halos = [torch.zeros(n + 2, dtype=torch.int64, device="cuda") for _ in range(G + 1)]
        for st in nwdist.strip_bounds(n, G, align=nwb.nw_band_width(tile)):
            S, R = inputs.device_strip(n, p, st.col0, st.w)
            nwb.nw_fill_sharded(S, R, p, halo_in=halos[st.rank] if st.rank > 0 else None,
                                halo_out=halos[st.rank + 1] if st.rank < G - 1 else None, epoch=3, tile=tile)
            torch.cuda.synchronize()
            del R
            parts.append((st.col0, st.w, S))
    _stream_compare_strips(parts, n, p)


def test_config4_full_batch_bit_exact():
    """BASELINE.json config 4 in full: 4096 pairs of n = 2048 built on the device as bench.py builds
    them, one nw_fill_batch launch (pair mode), every cell of every pair checked with the oracle
    (pairs copied back in groups; threads: ctypes drops the GIL)."""
    from concurrent.futures import ThreadPoolExecutor
    n, p, B = 2048, 10, 4096
    free, _ = torch.cuda.mem_get_info()
    if free < 150e9:
        pytest.skip("needs ~140 GB of device memory")
    S = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
    R = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
    for k in range(B):
        inputs.device_problem(n, p, seed=inputs.pair_seed(k), device="cuda", score=S[k], ref=R[k])
    nwb.nw_fill_batch(S, R, p, 0)
    torch.cuda.synchronize()
    del R

    def check(args):
        k, got = args
        s, r = inputs.make_problem(n, p, seed=inputs.pair_seed(k))
        return bool(np.array_equal(got, oracle.nw_ref(s, r, p)))

    bad = []
    with ThreadPoolExecutor(max(4, os.cpu_count() or 4)) as ex:
        for g0 in range(0, B, 256):
            got = S[g0:g0 + 256].cpu().numpy()
            ok = list(ex.map(check, [(g0 + i, got[i]) for i in range(got.shape[0])]))
            bad += [g0 + i for i, v in enumerate(ok) if not v]
    assert not bad, bad[:10]


@pytest.mark.parametrize("tile", [0, 64, 128])
@pytest.mark.parametrize("n", [1, 5, 31, 64, 129, 1000, 4096])
def test_fill_seq_next2(n, tile):
    """NEXT-2: ref generated on chip from (a, b, BLOSUM62) == nw_fill on the materialised ref."""
    a, b = inputs.gen_pair(n, 100 + n)
    ref = inputs.build_ref(a, b)
    score = inputs.init_borders(inputs.aligned_matrix(n), 10)
    inputs.fill_interior(score, inputs.SENTINEL)
    want = expect(score, ref, 10)
    s = to_dev(score)
    nwb.nw_fill_seq(s, torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda(), inputs.blosum62(), 10, tile)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(s.cpu().numpy(), want)


def test_fill_seq_batch_next2():
    B, n = 6, 300
    pairs = [inputs.gen_pair(n, inputs.pair_seed(k)) for k in range(B)]
    want = []
    S = np.empty((B, n + 1, n + 1), dtype=np.int32)
    for k, (a, b) in enumerate(pairs):
        s0 = inputs.init_borders(inputs.aligned_matrix(n), 10)
        inputs.fill_interior(s0, inputs.SENTINEL)
        S[k] = s0
        want.append(expect(s0, inputs.build_ref(a, b), 10))
    Sd = torch.from_numpy(S).cuda()
    Ad = torch.from_numpy(np.stack([a for a, _ in pairs])).cuda()
    Bd = torch.from_numpy(np.stack([b for _, b in pairs])).cuda()
    nwb.nw_fill_seq_batch(Sd, Ad, Bd, inputs.blosum62(), 10, 0)
    torch.cuda.synchronize()
    got = Sd.cpu().numpy()
    for k in range(B):
        np.testing.assert_array_equal(got[k], want[k], err_msg=f"pair {k}")


def test_config4_shape_batch_bit_exact():
    """BASELINE.json config 4 shape (n=2048 pairs seeded 7 ^ k*C) on 512 pairs, built on the device
    as bench.py builds them, every cell checked with the oracle (threads: ctypes drops the GIL)."""
    from concurrent.futures import ThreadPoolExecutor
    n, p, B = 2048, 10, 512
    S = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
    R = torch.empty((B, n + 1, n + 1), dtype=torch.int32, device="cuda")
    for k in range(B):
        inputs.device_problem(n, p, seed=inputs.pair_seed(k), device="cuda", score=S[k], ref=R[k])
    nwb.nw_fill_batch(S, R, p, 0)
    torch.cuda.synchronize()
    got = S.cpu().numpy()

    def check(k):
        s, r = inputs.make_problem(n, p, seed=inputs.pair_seed(k))
        return bool(np.array_equal(got[k], oracle.nw_ref(s, r, p)))

    with ThreadPoolExecutor(8) as ex:
        ok = list(ex.map(check, range(B)))
    assert all(ok), [k for k, v in enumerate(ok) if not v][:10]


def test_cluster_dsmem_handoff_opt_in():
    """nw_debug_set_cluster(1) (opt-in): single pairs run as clusters of 4 CTAs whose border
    columns pass through distributed shared memory; bit-exact against the oracle."""
    try:
        nwb.nw_debug_set_cluster(True)
        for n in (1, 255, 256, 1000, 1024, 3000):
            s, r = inputs.make_problem(n, 10)
            np.testing.assert_array_equal(gpu_fill(s, r, 10, 0), expect(s, r, 10), err_msg=str(n))
    finally:
        nwb.nw_debug_set_cluster(False)


def test_pair_mode_batches_forced():
    """Pair mode (a CTA sweeps all bands of a pair in turn; automatic for large batches) forced
    on small ragged batches (nw_debug_set_pair_mode(1)), both one-band-per-CTA kernels (tiles 0,
    64); and switched off (-1) for a batch large enough to enable it automatically."""
    try:
        for mode, cases in ((1, ((3, 700, 0), (5, 257, 64), (2, 1024, 0), (4, 1500, 64), (3, 100, 0))),
                            (-1, ((600, 64, 0),))):
            nwb.nw_debug_set_pair_mode(mode)
            for B, n, tile in cases:
                ss, rs, want = [], [], []
                for k in range(B):
                    s, r = inputs.make_problem(n, 10, seed=inputs.pair_seed(k))
                    ss.append(s), rs.append(r), want.append(expect(s, r, 10))
                S = torch.from_numpy(np.stack(ss)).cuda()
                R = torch.from_numpy(np.stack(rs)).cuda()
                nwb.nw_fill_batch(S, R, 10, tile)
                torch.cuda.synchronize()
                got = S.cpu().numpy()
                for k in range(B):
                    np.testing.assert_array_equal(got[k], want[k], err_msg=f"{mode} {B} {n} {tile} {k}")
    finally:
        nwb.nw_debug_set_pair_mode(0)
