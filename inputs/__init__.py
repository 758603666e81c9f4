"""Seeded synthetic input generator for NW (shared by oracle side and CUDA side).

Holds none of the method's arithmetic (see ``include/nw_inputs.h``): sequences from
splitmix64, the BLOSUM62 lookup that turns a pair of sequences into ``ref``, the
global-alignment border convention, and the test families (random, homologous, constant
ref, random borders).  The C implementation is ``inputs/nw_inputs.c``; this module
builds it with ``cc`` and wraps it with ctypes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_HERE)
_SRC = os.path.join(_HERE, "nw_inputs.c")
_HDR = os.path.join(_ROOT, "include", "nw_inputs.h")
_LIB_PATH = os.path.join(_HERE, "libnwinputs.so")
_lock = threading.Lock()
_lib = None

SEED = 7                      # Rodinia's srand(7), reading C2
PAIR_SEED_MUL = 0xD1B54A32D192ED03
_i32p = ctypes.POINTER(ctypes.c_int32)
_u8p = ctypes.POINTER(ctypes.c_uint8)


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
        os.path.getmtime(_SRC), os.path.getmtime(_HDR)
    ):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["cc", "-O2", "-std=c11", "-shared", "-fPIC",
                               "-I", os.path.join(_ROOT, "include"), _SRC, "-o", tmp])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib() -> ctypes.CDLL:
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            L.nw_splitmix64_next.argtypes = [ctypes.POINTER(ctypes.c_uint64)]
            L.nw_splitmix64_next.restype = ctypes.c_uint64
            L.nw_pair_seed.argtypes = [ctypes.c_uint64, ctypes.c_int64]
            L.nw_pair_seed.restype = ctypes.c_uint64
            L.nw_gen_pair.argtypes = [ctypes.c_uint64, ctypes.c_int64, _u8p, _u8p]
            L.nw_gen_homologous.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, _u8p, _u8p]
            L.nw_blosum62.restype = ctypes.POINTER(ctypes.c_int8)
            L.nw_blosum62_alphabet.restype = ctypes.c_char_p
            L.nw_build_ref_rows.argtypes = [_i32p, ctypes.c_int64, _u8p, _u8p, ctypes.c_int64,
                                            ctypes.c_int64, ctypes.c_int64]
            L.nw_build_ref_block.argtypes = [_i32p, ctypes.c_int64, _u8p, _u8p, ctypes.c_int64,
                                             ctypes.c_int64, ctypes.c_int64]
            L.nw_init_borders.argtypes = [_i32p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int32]
            L.nw_fill_interior.argtypes = [_i32p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int32]
            _lib = L
    return _lib


def splitmix64(state: int, count: int) -> list[int]:
    s = ctypes.c_uint64(state)
    return [lib().nw_splitmix64_next(ctypes.byref(s)) for _ in range(count)]


def pair_seed(k: int, base: int = SEED) -> int:
    return lib().nw_pair_seed(base, k)


def blosum62() -> np.ndarray:
    p = lib().nw_blosum62()
    return np.ctypeslib.as_array(p, shape=(24 * 24,)).reshape(24, 24).astype(np.int32)


def alphabet() -> str:
    return lib().nw_blosum62_alphabet().decode()


def gen_pair(n: int, seed: int = SEED) -> tuple[np.ndarray, np.ndarray]:
    """Rodinia-style random pair: residues uniform on BLOSUM62 indices 1..10."""
    a = np.empty(n, dtype=np.uint8)
    b = np.empty(n, dtype=np.uint8)
    lib().nw_gen_pair(seed, n, a.ctypes.data_as(_u8p), b.ctypes.data_as(_u8p))
    return a, b


def gen_homologous(n: int, seed: int = SEED, sub_per_mille: int = 100):
    a = np.empty(n, dtype=np.uint8)
    b = np.empty(n, dtype=np.uint8)
    lib().nw_gen_homologous(seed, n, sub_per_mille, a.ctypes.data_as(_u8p), b.ctypes.data_as(_u8p))
    return a, b


def encode(s: str) -> np.ndarray:
    """Residue letters -> BLOSUM62 indices (for hand-worked examples)."""
    al = alphabet()
    return np.array([al.index(c) for c in s], dtype=np.uint8)


def aligned_matrix(n: int, ld: int | None = None, align_col1: bool = False) -> np.ndarray:
    """An (n+1) x ld int32 host matrix view (ld defaults to n+1)."""
    ld = n + 1 if ld is None else ld
    assert ld >= n + 1
    return np.zeros((n + 1, ld), dtype=np.int32)


def build_ref(a: np.ndarray, b: np.ndarray, ld: int | None = None, out: np.ndarray | None = None) -> np.ndarray:
    """ref[i][j] = B62[a[i-1]][b[j-1]] (i, j >= 1); row/col 0 are zero (unused)."""
    n = len(a)
    assert len(b) == n
    a = np.ascontiguousarray(a, dtype=np.uint8)
    b = np.ascontiguousarray(b, dtype=np.uint8)
    ref = aligned_matrix(n, ld) if out is None else out
    lib().nw_build_ref_rows(ref.ctypes.data_as(_i32p), ref.strides[0] // 4, a.ctypes.data_as(_u8p),
                            b.ctypes.data_as(_u8p), n, 1, n + 1)
    return ref


def build_ref_block(a: np.ndarray, b: np.ndarray, row_begin: int, row_end: int, out: np.ndarray | None = None) -> np.ndarray:
    """Rows [row_begin, row_end) of ref as a (rows, n+1) block (col 0 zero)."""
    n = len(a)
    a = np.ascontiguousarray(a, dtype=np.uint8)
    b = np.ascontiguousarray(b, dtype=np.uint8)
    rows = row_end - row_begin
    if out is None:
        out = np.zeros((rows, n + 1), dtype=np.int32)
    lib().nw_build_ref_block(out.ctypes.data_as(_i32p), out.strides[0] // 4, a.ctypes.data_as(_u8p),
                             b.ctypes.data_as(_u8p), n, row_begin, row_end)
    return out


def init_borders(score: np.ndarray, p: int) -> np.ndarray:
    n = score.shape[0] - 1
    lib().nw_init_borders(score.ctypes.data_as(_i32p), score.strides[0] // 4, n, int(p))
    return score


def fill_interior(score: np.ndarray, value: int) -> np.ndarray:
    n = score.shape[0] - 1
    lib().nw_fill_interior(score.ctypes.data_as(_i32p), score.strides[0] // 4, n, int(value))
    return score


SENTINEL = -(2**31)  # 0x80000000: marks never-written interior cells


def make_problem(n: int, p: int = 10, seed: int = SEED, family: str = "random", ld: int | None = None,
                 const_ref: int = 0, border_seed: int | None = None, sentinel: bool = True):
    """(score, ref) host pair for one test case.

    family: "random" (Rodinia), "homologous" (10 % substitutions), "const" (ref == const_ref).
    border_seed: if set, row 0 / col 0 get arbitrary values in [-2^20, 2^20) instead of the
    global-alignment borders (the strip halo needs arbitrary borders, reading C5).
    """
    ld = n + 1 if ld is None else ld
    score = aligned_matrix(n, ld)
    if family == "const":
        ref = aligned_matrix(n, ld)
        ref[1:, 1:n + 1] = const_ref
    else:
        a, b = gen_pair(n, seed) if family == "random" else gen_homologous(n, seed)
        ref = build_ref(a, b, ld)
    init_borders(score, p)
    if border_seed is not None:
        rng = np.random.default_rng(border_seed)
        score[0, : n + 1] = rng.integers(-(1 << 20), 1 << 20, n + 1, dtype=np.int32)
        score[:, 0] = rng.integers(-(1 << 20), 1 << 20, n + 1, dtype=np.int32)
    if sentinel:
        fill_interior(score, SENTINEL)
    return score, ref


def device_aligned_matrix(n: int, device="cuda"):
    """An (n+1) x (n+1) int32 CUDA view whose interior rows start 16-byte aligned: pitch a multiple of 4
    elements and element (0, 1) on a 16-byte boundary (a layout, no data)."""
    import torch
    ld = (n + 1 + 3) & ~3
    buf = torch.empty((n + 1) * ld + 4, dtype=torch.int32, device=device)
    return buf[3:3 + (n + 1) * ld].view(n + 1, ld)[:, : n + 1]


def device_aligned_batch(b: int, n: int, device="cuda"):
    """A (b, n+1, n+1) int32 CUDA view of b pairs whose interior rows all start 16-byte aligned
    (pitch and pair stride multiples of 4 elements, element (k, 0, 1) on a 16-byte boundary)."""
    import torch
    ld = (n + 1 + 3) & ~3
    buf = torch.empty(b * (n + 1) * ld + 4, dtype=torch.int32, device=device)
    return buf[3:3 + b * (n + 1) * ld].view(b, n + 1, ld)[:, :, : n + 1]


def device_problem(n: int, p: int = 10, seed: int = SEED, device="cuda", score=None, ref=None,
                   sentinel: bool = True, chunk_rows: int = 4096, layout: str = "rodinia"):
    """The same Rodinia-style problem as make_problem(n, p, seed), built ON THE DEVICE (for the
    large bench configs): sequences from the C splitmix64 generator, ref = B62[a_i][b_j] by a
    table gather in row chunks, global-alignment borders.  Optionally fills preallocated
    (n+1, >= n+1) int32 views `score` / `ref` (e.g. one pair of a batch)."""
    import torch
    a, b = gen_pair(n, seed)
    table = torch.from_numpy(blosum62()).to(device=device, dtype=torch.int32)
    ta = torch.from_numpy(a.astype(np.int64)).to(device)
    tb = torch.from_numpy(b.astype(np.int64)).to(device)
    if score is None:
        score = device_aligned_matrix(n, device) if layout == "aligned" else torch.empty((n + 1, n + 1), dtype=torch.int32, device=device)
    if ref is None:
        ref = device_aligned_matrix(n, device) if layout == "aligned" else torch.empty((n + 1, n + 1), dtype=torch.int32, device=device)
    ref[0, : n + 1] = 0
    ref[:, 0] = 0
    rows_b = table[:, tb]                       # (24, n): B62[x][b_j] for every residue x
    for i0 in range(0, n, chunk_rows):
        i1 = min(n, i0 + chunk_rows)
        ref[1 + i0:1 + i1, 1:n + 1] = rows_b[ta[i0:i1]]
    steps = torch.arange(n + 1, device=device, dtype=torch.int64) * (-p)
    score[0, : n + 1] = steps.to(torch.int32)
    score[:, 0] = steps.to(torch.int32)
    if sentinel:
        score[1:, 1:n + 1] = SENTINEL
    return score, ref


def device_strip(n: int, p: int, col0: int, w: int, seed: int = SEED, device="cuda", chunk_rows: int = 4096):
    """Column strip (global columns col0+1 .. col0+w) of device_problem(n, p, seed) as the local
    (n+1) x (w+1) matrices a sharded rank holds (nw.h nw_strip): local column j = global column
    col0 + j; row 0 = the global row 0 there; local column 0 (rows >= 1) = the global left border
    on the first strip (col0 == 0), else SENTINEL (a halo supplies it); interior SENTINEL."""
    import torch
    a, b = gen_pair(n, seed)
    table = torch.from_numpy(blosum62()).to(device=device, dtype=torch.int32)
    ta = torch.from_numpy(a.astype(np.int64)).to(device)
    tb = torch.from_numpy(b[col0:col0 + w].astype(np.int64)).to(device)
    score = torch.empty((n + 1, w + 1), dtype=torch.int32, device=device)
    ref = torch.zeros((n + 1, w + 1), dtype=torch.int32, device=device)
    rows_b = table[:, tb]                       # (24, w): B62[x][b_j] for the strip's columns
    for i0 in range(0, n, chunk_rows):
        i1 = min(n, i0 + chunk_rows)
        ref[1 + i0:1 + i1, 1:] = rows_b[ta[i0:i1]]
    score[0, :] = (torch.arange(col0, col0 + w + 1, device=device, dtype=torch.int64) * (-p)).to(torch.int32)
    if col0 == 0:
        score[1:, 0] = (torch.arange(1, n + 1, device=device, dtype=torch.int64) * (-p)).to(torch.int32)
    else:
        score[1:, 0] = SENTINEL
    score[1:, 1:] = SENTINEL
    return score, ref
