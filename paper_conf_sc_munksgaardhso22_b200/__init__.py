"""paper_conf_sc_munksgaardhso22_b200 — B200-native Needleman–Wunsch wavefront.

Thin Python binding of the C-ABI library ``libnwb200.so`` (``include/nw.h``).  This module does
argument marshalling only — dtype/device/shape checks, pointers, pitches and the current CUDA
stream — every step of the fill runs in the library's sm_100a kernels.  There is no CPU
fallback: if the library is missing the calls raise.

PyTorch supplies device memory, streams and (in ``dist.py``) process groups.

The computed matrix is the paper's NW fill (Fig. 2; Rodinia's cell
function, BASELINE.json north_star):
    score[i][j] = max(score[i-1][j-1] + ref[i][j], score[i-1][j] - p, score[i][j-1] - p)
with row 0 / column 0 of ``score`` as inputs and the interior written in place.
"""
from __future__ import annotations

import ctypes
import os
import threading

from ._build import LIB_PATH, build  # noqa: F401  (build() is re-exported for __graft_entry__)

__all__ = [
    "NwError", "lib", "nw_fill", "nw_fill_batch", "nw_fill_seq", "nw_fill_seq_batch", "nw_fill_sharded", "nw_fill_host", "nw_fill_batch_host",
    "nw_fill_diagonal", "nw_fill_unopt", "nw_traceback", "nw_traceback_batch", "nw_band_width", "nw_launch_count", "nw_diag_lmad",
    "nw_kernel_info", "nw_strip_map", "nw_debug_set_grid", "nw_debug_set_trace", "nw_release_workspace", "nw_status_str",
    "nw_debug_set_pair_mode", "nw_debug_set_cluster", "nw_debug_set_host_zero_copy", "nw_debug_set_host_mode",
    "nw_debug_set_host_block_rows",
]

NW_OK, NW_EINVAL, NW_ERANGE, NW_ECUDA, NW_ECOMM = range(5)  # SURVEY.md §8(b) numbering
NW_REF_MAX = 1024

_lock = threading.Lock()
_lib = None
_i32p = ctypes.c_void_p
_i64 = ctypes.c_int64
_i32 = ctypes.c_int32


class NwError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib().nw_status_str(status).decode()
        if status == NW_ECUDA:
            msg += f" (cudaError {lib().nw_last_cuda_error()})"
        super().__init__(f"{where}: {msg}")


class NwStrip(ctypes.Structure):
    _fields_ = [
        ("score", ctypes.c_void_p), ("ld_score", _i64),
        ("ref", ctypes.c_void_p), ("ld_ref", _i64),
        ("n", _i64), ("w", _i64),
        ("halo_in", ctypes.c_void_p), ("halo_out", ctypes.c_void_p),
        ("epoch", ctypes.c_uint32), ("halo_out_is_peer", _i32),
    ]


def lib() -> ctypes.CDLL:
    """Load libnwb200.so (raises if it has not been built: no silent fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError(f"{LIB_PATH} is missing: run __graft_entry__.build() first")
            L = ctypes.CDLL(os.environ.get("NW_LIB") or LIB_PATH)  # NW_LIB: experiment builds only
            vp = ctypes.c_void_p
            L.nw_status_str.argtypes = [ctypes.c_int]
            L.nw_status_str.restype = ctypes.c_char_p
            L.nw_abi_version.restype = ctypes.c_int
            L.nw_last_cuda_error.restype = ctypes.c_int
            L.nw_fill.argtypes = [vp, vp, _i64, _i32, _i32, vp]
            L.nw_fill_ld.argtypes = [vp, _i64, vp, _i64, _i64, _i32, _i32, vp]
            L.nw_fill_batch.argtypes = [vp, vp, _i64, _i64, _i32, _i32, vp]
            L.nw_fill_batch_ld.argtypes = [vp, _i64, _i64, vp, _i64, _i64, _i64, _i64, _i32, _i32, vp]
            L.nw_fill_sharded.argtypes = [ctypes.POINTER(NwStrip), _i32, _i32, vp]
            L.nw_fill_seq.argtypes = [vp, _i64, vp, vp, _i64, vp, _i32, _i32, _i32, vp]
            L.nw_fill_seq_batch.argtypes = [vp, _i64, _i64, vp, vp, _i64, _i64, _i64, vp, _i32, _i32, _i32, vp]
            L.nw_fill_host.argtypes = [vp, vp, _i64, _i32, _i32, _i32]
            L.nw_fill_batch_host.argtypes = [vp, vp, _i64, _i64, _i32, _i32, _i32]
            L.nw_fill_diagonal.argtypes = [vp, _i64, vp, _i64, _i64, _i32, _i32, vp]
            L.nw_fill_unopt.argtypes = [vp, _i64, vp, _i64, _i64, _i32, _i32, vp]
            L.nw_traceback.argtypes = [vp, _i64, vp, _i64, _i64, _i32, vp, vp, vp]
            L.nw_traceback_batch.argtypes = [vp, _i64, _i64, vp, _i64, _i64, _i64, _i64, _i32, vp, _i64, vp, vp]
            L.nw_band_width.argtypes = [_i32]
            L.nw_band_width.restype = _i32
            L.nw_launch_count.argtypes = [_i32, _i64, _i32]
            L.nw_launch_count.restype = _i64
            L.nw_diag_lmad.argtypes = [_i64, _i64, _i32, _i64, ctypes.POINTER(_i64)]
            L.nw_diag_lmad.restype = _i32
            L.nw_kernel_info.argtypes = [_i32, _i32, ctypes.POINTER(_i64), ctypes.POINTER(_i32),
                                         ctypes.POINTER(_i32)]
            L.nw_strip_map.argtypes = [_i64, _i64, _i32, _i32, _i32, _i32, ctypes.POINTER(_i64)]
            L.nw_strip_map.restype = _i32
            L.nw_debug_set_trace.argtypes = [vp, _i64]
            L.nw_debug_set_trace.restype = None
            L.nw_debug_set_grid.argtypes = [_i32]
            L.nw_debug_set_grid.restype = None
            for f in ("nw_debug_set_pair_mode", "nw_debug_set_cluster", "nw_debug_set_host_zero_copy", "nw_debug_set_host_mode"):
                getattr(L, f).argtypes = [_i32]
                getattr(L, f).restype = None
            L.nw_debug_set_host_block_rows.argtypes = [_i64]
            L.nw_debug_set_host_block_rows.restype = None
            L.nw_release_workspace.restype = None
            for f in ("nw_fill", "nw_fill_ld", "nw_fill_batch", "nw_fill_batch_ld", "nw_fill_sharded",
                      "nw_fill_host", "nw_fill_batch_host", "nw_fill_diagonal", "nw_fill_unopt", "nw_kernel_info", "nw_fill_seq",
                      "nw_fill_seq_batch", "nw_traceback", "nw_traceback_batch"):
                getattr(L, f).restype = ctypes.c_int
            _lib = L
    return _lib


def nw_status_str(status: int) -> str:
    return lib().nw_status_str(status).decode()


def _check(status: int, where: str):
    if status != NW_OK:
        raise NwError(status, where)


def _stream_ptr(stream, device):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return ctypes.c_void_p(s.cuda_stream)


def _mat(t, name):
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if t.dtype != torch.int32:
        raise TypeError(f"{name} must be int32, got {t.dtype}")
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if t.stride(-1) != 1:
        raise ValueError(f"{name} rows must be contiguous (stride(-1) == 1)")
    return t


def nw_fill(score, ref, penalty: int, tile: int = 0, stream=None):
    """Fill score[1:, 1:] in place.  score, ref: int32 CUDA tensors of shape (n+1, >= n+1)."""
    import torch
    _mat(score, "score"), _mat(ref, "ref")
    if score.dim() != 2 or ref.dim() != 2:
        raise ValueError("score/ref must be 2-D")
    n = score.shape[0] - 1
    if score.shape[1] < n + 1 or ref.shape[0] < n + 1 or ref.shape[1] < n + 1:
        raise ValueError(f"shapes {tuple(score.shape)} / {tuple(ref.shape)} do not hold an (n+1)^2 matrix")
    if score.device != ref.device:
        raise ValueError("score and ref must be on the same device")
    with torch.cuda.device(score.device):
        _check(lib().nw_fill_ld(score.data_ptr(), score.stride(0), ref.data_ptr(), ref.stride(0), n,
                                int(penalty), int(tile), _stream_ptr(stream, score.device)), "nw_fill")
    return score


def nw_fill_batch(score, ref, penalty: int, tile: int = 0, stream=None):
    """Batch of independent pairs: score, ref int32 CUDA tensors (B, n+1, >= n+1)."""
    import torch
    _mat(score, "score"), _mat(ref, "ref")
    if score.dim() != 3 or ref.dim() != 3 or score.shape[0] != ref.shape[0]:
        raise ValueError("score/ref must be (B, n+1, >= n+1)")
    b, n = score.shape[0], score.shape[1] - 1
    if score.shape[2] < n + 1 or ref.shape[1] < n + 1 or ref.shape[2] < n + 1:
        raise ValueError("bad batch shapes")
    with torch.cuda.device(score.device):
        _check(lib().nw_fill_batch_ld(score.data_ptr(), score.stride(1), score.stride(0), ref.data_ptr(),
                                      ref.stride(1), ref.stride(0), b, n, int(penalty), int(tile),
                                      _stream_ptr(stream, score.device)), "nw_fill_batch")
    return score


def nw_fill_sharded(score, ref, penalty: int, *, halo_in=None, halo_out=None, epoch: int = 0,
                    halo_out_is_peer: bool = False, tile: int = 0, stream=None):
    """One rank's column strip.  score/ref: local (n+1, >= w+1) int32 CUDA tensors.

    halo_in: None (rank 0: left border = score[:, 0]) or an int64 CUDA tensor of n+2 tagged
    entries written by the left neighbour.  halo_out: None, an int64 tensor (same device) or an
    integer device address (peer-mapped, e.g. from torch symmetric memory)."""
    import torch
    _mat(score, "score"), _mat(ref, "ref")
    n, w = score.shape[0] - 1, score.shape[1] - 1
    if ref.shape[0] < n + 1 or ref.shape[1] < w + 1:
        raise ValueError("ref smaller than score")

    def ptr(h):
        if h is None:
            return None
        if isinstance(h, int):
            return h
        if h.dtype not in (torch.int64, torch.uint64) or not h.is_cuda or h.numel() < n + 2:
            raise ValueError("halo tensors must be int64 CUDA tensors with >= n+2 entries")
        return h.data_ptr()

    st = NwStrip(score.data_ptr(), score.stride(0), ref.data_ptr(), ref.stride(0), n, w,
                 ptr(halo_in), ptr(halo_out), int(epoch) & 0xFFFFFFFF, int(bool(halo_out_is_peer)))
    with torch.cuda.device(score.device):
        _check(lib().nw_fill_sharded(ctypes.byref(st), int(penalty), int(tile),
                                     _stream_ptr(stream, score.device)), "nw_fill_sharded")
    return score


def _subst_host(subst):
    import numpy as np
    t = np.ascontiguousarray(np.asarray(subst), dtype=np.int32)
    if t.ndim != 2 or t.shape[0] != t.shape[1]:
        raise ValueError("subst must be a square (alphabet x alphabet) table")
    return t


def nw_fill_seq(score, a, b, subst, penalty: int, tile: int = 0, stream=None):
    """NEXT-2: fill score from the two sequences directly (ref never materialised).
    score: int32 CUDA (n+1, >= n+1); a, b: uint8 CUDA (n,) residue codes; subst: host table."""
    import torch
    _mat(score, "score")
    n = score.shape[0] - 1
    for v, nm in ((a, "a"), (b, "b")):
        if v.dtype != torch.uint8 or not v.is_cuda or v.dim() != 1 or v.numel() < n or v.stride(0) != 1:
            raise ValueError(f"{nm} must be a contiguous uint8 CUDA vector of length >= n")
    tab = _subst_host(subst)
    with torch.cuda.device(score.device):
        _check(lib().nw_fill_seq(score.data_ptr(), score.stride(0), a.data_ptr(), b.data_ptr(), n,
                                 tab.ctypes.data, tab.shape[0], int(penalty), int(tile),
                                 _stream_ptr(stream, score.device)), "nw_fill_seq")
    return score


def nw_fill_seq_batch(score, a, b, subst, penalty: int, tile: int = 0, stream=None):
    """Batch NEXT-2: score (B, n+1, >= n+1) int32; a, b (B, n) uint8 CUDA, contiguous rows."""
    import torch
    _mat(score, "score")
    B, n = score.shape[0], score.shape[1] - 1
    if a.shape != b.shape or a.dim() != 2 or a.shape[0] != B or a.shape[1] < n or a.dtype != torch.uint8 \
            or b.dtype != torch.uint8 or a.stride(1) != 1 or b.stride(1) != 1 or a.stride(0) != b.stride(0):
        raise ValueError("a, b must be (B, >= n) uint8 CUDA tensors with equal strides")
    tab = _subst_host(subst)
    with torch.cuda.device(score.device):
        _check(lib().nw_fill_seq_batch(score.data_ptr(), score.stride(1), score.stride(0), a.data_ptr(),
                                       b.data_ptr(), a.stride(0), B, n, tab.ctypes.data, tab.shape[0],
                                       int(penalty), int(tile), _stream_ptr(stream, score.device)),
               "nw_fill_seq_batch")
    return score


def nw_fill_host(score, ref, penalty: int, tile: int = 0, device: int = 0):
    """End-to-end from host numpy arrays ((n+1, n+1) int32, C-contiguous); synchronous."""
    import numpy as np
    if score.dtype != np.int32 or ref.dtype != np.int32 or not score.flags.c_contiguous \
            or not ref.flags.c_contiguous:
        raise ValueError("host arrays must be C-contiguous int32")
    n = score.shape[0] - 1
    if score.shape != (n + 1, n + 1) or ref.shape != (n + 1, n + 1):
        raise ValueError("host arrays must be (n+1, n+1)")
    _check(lib().nw_fill_host(score.ctypes.data, ref.ctypes.data, n, int(penalty), int(tile),
                              int(device)), "nw_fill_host")
    return score


def nw_fill_batch_host(score, ref, penalty: int, tile: int = 0, device: int = 0):
    """End-to-end from host numpy arrays ((B, n+1, n+1) int32, C-contiguous); synchronous.
    Pinned (e.g. torch pin_memory) arrays take the zero-copy path."""
    import numpy as np
    if score.dtype != np.int32 or ref.dtype != np.int32 or not score.flags.c_contiguous \
            or not ref.flags.c_contiguous:
        raise ValueError("host arrays must be C-contiguous int32")
    if score.ndim != 3 or score.shape != ref.shape or score.shape[1] != score.shape[2]:
        raise ValueError("host arrays must be (B, n+1, n+1)")
    B, n = score.shape[0], score.shape[1] - 1
    _check(lib().nw_fill_batch_host(score.ctypes.data, ref.ctypes.data, B, n, int(penalty), int(tile),
                                    int(device)), "nw_fill_batch_host")
    return score


def _diag(fn, name, score, ref, penalty, tile, stream):
    import torch
    _mat(score, "score"), _mat(ref, "ref")
    n = score.shape[0] - 1
    with torch.cuda.device(score.device):
        _check(getattr(lib(), fn)(score.data_ptr(), score.stride(0), ref.data_ptr(), ref.stride(0), n,
                                  int(penalty), int(tile), _stream_ptr(stream, score.device)), name)
    return score


def nw_fill_diagonal(score, ref, penalty: int, tile: int = 16, stream=None):
    """The paper's/Rodinia's structure: one launch per tile anti-diagonal, in place (Opt)."""
    return _diag("nw_fill_diagonal", "nw_fill_diagonal", score, ref, penalty, tile, stream)


def nw_fill_unopt(score, ref, penalty: int, tile: int = 16, stream=None):
    """The paper's Unopt variant: per diagonal, tiles -> temporary X, then a copy A[W] = X."""
    return _diag("nw_fill_unopt", "nw_fill_unopt", score, ref, penalty, tile, stream)


def nw_traceback(score, ref, penalty: int, stream=None):
    """Traceback of one filled pair (NEXT-3): returns (ops, length) CUDA tensors.

    ops: uint8 (2n,), ops[:length] = the path in forward order (0 diagonal, 1 up, 2 left; ties
    diagonal > up > left); length: int32 (1,), -1 if the matrix is not a fill of (ref, penalty)."""
    ops, length = nw_traceback_batch(score.unsqueeze(0), ref.unsqueeze(0), penalty, stream)
    return ops[0], length


def nw_traceback_batch(score, ref, penalty: int, stream=None):
    """Traceback of B filled pairs: score/ref (B, n+1, >= n+1) -> ops uint8 (B, 2n), length int32 (B,)."""
    import torch
    _mat(score, "score"), _mat(ref, "ref")
    if score.dim() != 3 or ref.dim() != 3 or score.shape[0] != ref.shape[0]:
        raise ValueError("score/ref must be (B, n+1, >= n+1)")
    b, n = score.shape[0], score.shape[1] - 1
    if score.shape[2] < n + 1 or ref.shape[1] < n + 1 or ref.shape[2] < n + 1:
        raise ValueError("bad batch shapes")
    ops = torch.empty((b, max(2 * n, 1)), dtype=torch.uint8, device=score.device)
    length = torch.empty((b,), dtype=torch.int32, device=score.device)
    with torch.cuda.device(score.device):
        _check(lib().nw_traceback_batch(score.data_ptr(), score.stride(1), score.stride(0), ref.data_ptr(),
                                        ref.stride(1), ref.stride(0), b, n, int(penalty), ops.data_ptr(),
                                        ops.stride(0), length.data_ptr(), _stream_ptr(stream, score.device)),
               "nw_traceback")
    return ops, length


def nw_band_width(tile: int = 0) -> int:
    return lib().nw_band_width(int(tile))


def nw_launch_count(kind: int, n: int, tile: int = 0) -> int:
    return lib().nw_launch_count(int(kind), int(n), int(tile))


def nw_diag_lmad(n: int, N: int, tile: int, d: int):
    out = (_i64 * 10)()
    if lib().nw_diag_lmad(int(n), int(N), int(tile), int(d), out) != 0:
        raise ValueError("nw_diag_lmad: bad arguments")
    return list(out)


def nw_strip_map(n: int, width: int, tile: int, band: int, step: int, lane: int):
    """(row, first column, #columns) lane `lane` of band `band` computes at `step`."""
    out = (_i64 * 3)()
    if lib().nw_strip_map(int(n), int(width), int(tile), int(band), int(step), int(lane), out) != 0:
        raise ValueError("nw_strip_map: bad arguments")
    return tuple(out)


def nw_kernel_info(tile: int = 0, device: int = 0):
    smem, occ, sms = _i64(), _i32(), _i32()
    _check(lib().nw_kernel_info(int(tile), int(device), ctypes.byref(smem), ctypes.byref(occ),
                                ctypes.byref(sms)), "nw_kernel_info")
    return {"smem_bytes": smem.value, "ctas_per_sm": occ.value, "num_sms": sms.value}


def nw_debug_set_grid(grid: int):
    lib().nw_debug_set_grid(int(grid))


def nw_debug_set_pair_mode(mode: int):
    """0 automatic, 1 whole pairs per ticket for any batch >= 2, -1 never (nw.h)."""
    lib().nw_debug_set_pair_mode(int(mode))


def nw_debug_set_cluster(on: bool):
    lib().nw_debug_set_cluster(int(bool(on)))


def nw_debug_set_host_zero_copy(on: bool):
    lib().nw_debug_set_host_zero_copy(int(bool(on)))


def nw_debug_set_host_block_rows(rows: int):
    """Row-block size of the host pipeline (0: automatic, ~64 MB)."""
    lib().nw_debug_set_host_block_rows(int(rows))


def nw_debug_set_host_mode(mode: int):
    """Pinned host buffers in nw_fill[_batch]_host: 2 copy-engine pipeline (default), 1 zero copy, 0 staged."""
    lib().nw_debug_set_host_mode(int(mode))


def nw_debug_set_trace(buf=None):
    """buf: int64 CUDA tensor of shape (>= tasks, 8) or None (off)."""
    if buf is None:
        lib().nw_debug_set_trace(None, 0)
    else:
        lib().nw_debug_set_trace(buf.data_ptr(), buf.shape[0])


def nw_release_workspace():
    lib().nw_release_workspace()
