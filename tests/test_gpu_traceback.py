"""GPU parity for the traceback (NEXT-3): nw_traceback[_batch] through the C ABI against the
oracle's nw_traceback_ref, bit-exact on the op sequence and the length.

The matrices come from the oracle (so the traceback is tested on its own), and end to end from
nw_fill (the product path: fill then traceback on the device).  Tie-heavy families exercise the
diagonal > up > left rule (R12); a corrupted matrix must give length -1.
"""
import numpy as np
import pytest

import inputs
import oracle

torch = pytest.importorskip("torch")
import paper_conf_sc_munksgaardhso22_b200 as nwb  # noqa: E402

pytestmark = pytest.mark.gpu


def problem(n, p, seed, family):
    if family == "ties":
        rng = np.random.default_rng(seed)
        ref = np.zeros((n + 1, n + 1), dtype=np.int32)
        ref[1:, 1:] = rng.integers(-1, 2, size=(n, n))
        score = inputs.init_borders(inputs.aligned_matrix(n), p)
        return score, ref
    if family == "borders":        # arbitrary row 0 / column 0 (reading R5)
        return inputs.make_problem(n, p, seed=seed, border_seed=seed + 1)
    return inputs.make_problem(n, p, seed=seed, family=family)


def run_gpu(score, ref, p):
    ops, length = nwb.nw_traceback(torch.from_numpy(score).cuda(), torch.from_numpy(ref).cuda(), p)
    torch.cuda.synchronize()
    L = int(length.item())
    return ops[:max(L, 0)].cpu().numpy(), L


@pytest.mark.parametrize("n", [1, 2, 5, 31, 32, 33, 64, 65, 100, 257, 1000, 2048])
@pytest.mark.parametrize("p,family", [(10, "random"), (3, "homologous"), (0, "ties"), (1, "ties"),
                                      (1000, "random"), (10, "borders"), (0, "const")])
def test_traceback_matches_oracle(n, p, family):
    score, ref = problem(n, p, n + p, family)
    oracle.nw_ref(score, ref, p)
    want = oracle.nw_traceback_ref(score, ref, p)
    got, L = run_gpu(score, ref, p)
    assert L == len(want)
    np.testing.assert_array_equal(got, want)


def test_traceback_zero_and_pitched():
    ops, length = nwb.nw_traceback(torch.zeros((1, 1), dtype=torch.int32, device="cuda"),
                                   torch.zeros((1, 1), dtype=torch.int32, device="cuda"), 10)
    torch.cuda.synchronize()
    assert int(length.item()) == 0
    n, p = 300, 10
    score, ref = problem(n, p, 4, "random")
    oracle.nw_ref(score, ref, p)
    want = oracle.nw_traceback_ref(score, ref, p)
    s = torch.full((n + 1, n + 13), 99, dtype=torch.int32, device="cuda")
    r = torch.full((n + 1, n + 7), 99, dtype=torch.int32, device="cuda")
    s[:, : n + 1] = torch.from_numpy(score).cuda()
    r[:, : n + 1] = torch.from_numpy(ref).cuda()
    ops, length = nwb.nw_traceback(s[:, : n + 1], r[:, : n + 1], p)
    torch.cuda.synchronize()
    assert int(length.item()) == len(want)
    np.testing.assert_array_equal(ops[: len(want)].cpu().numpy(), want)


def test_traceback_corrupted_matrix():
    n, p = 200, 10
    score, ref = problem(n, p, 9, "random")
    oracle.nw_ref(score, ref, p)
    score[n, n] += 1000
    _, L = run_gpu(score, ref, p)
    assert L == -1


@pytest.mark.parametrize("B,n", [(7, 64), (33, 129), (300, 40), (1100, 17)])   # > 296: one warp per pair
def test_traceback_batch_after_device_fill(B, n):
    p = 10
    pairs = [inputs.make_problem(n, p, seed=inputs.pair_seed(k)) for k in range(B)]
    s = torch.from_numpy(np.stack([q[0] for q in pairs])).cuda()
    r = torch.from_numpy(np.stack([q[1] for q in pairs])).cuda()
    nwb.nw_fill_batch(s, r, p)
    ops, length = nwb.nw_traceback_batch(s, r, p)
    torch.cuda.synchronize()
    for k, (score, ref) in enumerate(pairs):
        oracle.nw_ref(score, ref, p)
        want = oracle.nw_traceback_ref(score, ref, p)
        assert int(length[k]) == len(want)
        np.testing.assert_array_equal(ops[k, : len(want)].cpu().numpy(), want)


@pytest.mark.parametrize("n", [16384])
def test_traceback_full_size_after_device_fill(n):
    """n = 16384 end to end on the device (fill + traceback) against the full oracle (1 GB matrix)."""
    p = 10
    score, ref = inputs.make_problem(n, p)
    s = torch.from_numpy(score).cuda()
    r = torch.from_numpy(ref).cuda()
    nwb.nw_fill(s, r, p)
    ops, length = nwb.nw_traceback(s, r, p)
    torch.cuda.synchronize()
    oracle.nw_ref(score, ref, p)
    want = oracle.nw_traceback_ref(score, ref, p)
    assert int(length.item()) == len(want)
    np.testing.assert_array_equal(ops[: len(want)].cpu().numpy(), want)
