"""The shared input generator (inputs/): determinism, ranges, known vectors, BLOSUM62."""
import numpy as np

import inputs


def test_splitmix64_known_vector():
    # splitmix64 (Steele/Lea/Flood) from state 0: first output 0xE220A8397B1DCDAF.
    assert inputs.splitmix64(0, 1)[0] == 0xE220A8397B1DCDAF


def test_pair_deterministic_and_range():
    a1, b1 = inputs.gen_pair(4096, 7)
    a2, b2 = inputs.gen_pair(4096, 7)
    assert (a1 == a2).all() and (b1 == b2).all()
    assert a1.min() >= 1 and a1.max() <= 10 and b1.min() >= 1 and b1.max() <= 10
    counts = np.bincount(a1, minlength=11)[1:]
    assert counts.min() > 300          # roughly uniform over 10 residues
    a3, _ = inputs.gen_pair(4096, inputs.pair_seed(1))
    assert (a3 != a1).any()


def test_pair_seed_formula():
    assert inputs.pair_seed(0) == 7
    assert inputs.pair_seed(3) == 7 ^ ((3 * inputs.PAIR_SEED_MUL) & (2**64 - 1))


def test_homologous_identity():
    a, b = inputs.gen_homologous(10000, 7, 100)
    frac_same = (a == b).mean()
    assert 0.88 < frac_same < 0.94    # 10 % substituted, 1/10 of those by the same residue


def test_blosum62_known_entries():
    B = inputs.blosum62()
    al = inputs.alphabet()
    assert al == "ARNDCQEGHILKMFPSTWYVBZX*"
    assert (B == B.T).all()
    idx = al.index
    assert B[idx("W"), idx("W")] == 11 and B[idx("C"), idx("C")] == 9
    assert B[idx("A"), idx("A")] == 4 and B[idx("*"), idx("*")] == 1
    assert B[idx("W"), idx("D")] == -4 and B[idx("R"), idx("K")] == 2
    sub = B[1:11, 1:11]
    assert sub.min() == -4 and sub.max() == 9


def test_build_ref_and_block():
    n = 50
    a, b = inputs.gen_pair(n, 3)
    B = inputs.blosum62()
    ref = inputs.build_ref(a, b)
    np.testing.assert_array_equal(ref[1:, 1:], B[a][:, b])
    assert (ref[0] == 0).all() and (ref[:, 0] == 0).all()
    blk = inputs.build_ref_block(a, b, 10, 20)
    np.testing.assert_array_equal(blk, ref[10:20])


def test_borders():
    s = inputs.init_borders(inputs.aligned_matrix(5, ld=9), 10)
    assert list(s[0, :6]) == [0, -10, -20, -30, -40, -50]
    assert list(s[:, 0]) == [0, -10, -20, -30, -40, -50]


def test_device_problem_matches_host_builder():
    """The device-side recipe (used by bench.py for the big configs) builds the same problem."""
    import torch
    for n, seed in [(1, 7), (50, 3), (129, 11)]:
        s, r = inputs.make_problem(n, 10, seed=seed)
        ds, dr = inputs.device_problem(n, 10, seed=seed, device="cpu", chunk_rows=17)
        np.testing.assert_array_equal(ds.numpy(), s)
        np.testing.assert_array_equal(dr.numpy(), r)
