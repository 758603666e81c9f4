"""CPU oracle for the NW score-matrix fill — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_sc_munksgaardhso22_b200``) never imports it and shares no code with it.

The arithmetic lives in plain C (``oracle/nw_ref.c``): the paper's "Golden Sequential"
loop (Fig. 2) with Rodinia's cell function (BASELINE.json north_star).
This module only builds that C file with ``cc`` and marshals numpy arrays through ctypes.
Every function is pinned by ``tests/test_oracle.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "nw_ref.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_i32p = ctypes.POINTER(ctypes.c_int32)


def build(force: bool = False) -> str:
    """Compile ``oracle/nw_ref.c`` -> ``oracle/liboracle.so`` (cc -O2 -std=c11, 1 thread)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "nw_ref.h"))
    ):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(
            ["cc", "-O2", "-std=c11", "-shared", "-fPIC", "-I", _HERE, _SRC, "-o", tmp]
        )
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib() -> ctypes.CDLL:
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            L.nw_ref.argtypes = [_i32p, ctypes.c_int64, _i32p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int32]
            L.nw_ref.restype = ctypes.c_int
            L.nw_ref_stream_new.argtypes = [ctypes.c_int64, ctypes.c_int32, _i32p]
            L.nw_ref_stream_new.restype = ctypes.c_void_p
            L.nw_ref_stream_rows.argtypes = [ctypes.c_void_p, _i32p, ctypes.c_int64, _i32p,
                                             ctypes.c_int64, _i32p, ctypes.c_int64]
            L.nw_ref_stream_rows.restype = ctypes.c_int
            L.nw_ref_stream_last.argtypes = [ctypes.c_void_p]
            L.nw_ref_stream_last.restype = _i32p
            L.nw_ref_stream_free.argtypes = [ctypes.c_void_p]
            L.nw_ref_stream_free.restype = None
            L.nw_traceback_ref.argtypes = [_i32p, ctypes.c_int64, _i32p, ctypes.c_int64, ctypes.c_int64,
                                           ctypes.c_int32, ctypes.POINTER(ctypes.c_uint8)]
            L.nw_traceback_ref.restype = ctypes.c_int64
            _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(_i32p)


def nw_ref(score: np.ndarray, ref: np.ndarray, p: int) -> np.ndarray:
    """Fill the interior of ``score`` in place (borders row 0 / col 0 are inputs).

    ``score`` and ``ref``: 2-D C-contiguous-rows int32 arrays of shape (n+1, ld>=n+1).
    Returns ``score``.  Raises OverflowError if a cell leaves int32.
    """
    assert score.dtype == np.int32 and ref.dtype == np.int32
    assert score.ndim == 2 and ref.ndim == 2 and score.strides[1] == 4 and ref.strides[1] == 4
    n = score.shape[0] - 1
    assert score.shape[1] >= n + 1 and ref.shape[0] >= n + 1 and ref.shape[1] >= n + 1
    rc = lib().nw_ref(_ptr(score), score.strides[0] // 4, _ptr(ref), ref.strides[0] // 4, n, int(p))
    if rc != 0:
        raise OverflowError("nw_ref: a cell value does not fit in int32")
    return score


def nw_traceback_ref(score: np.ndarray, ref: np.ndarray, p: int) -> np.ndarray:
    """Traceback of a filled ``score`` (NEXT-3): uint8 ops in forward order (0 diagonal, 1 up,
    2 left; ties diagonal > up > left).  Raises ValueError if a cell matches none of its moves."""
    assert score.dtype == np.int32 and ref.dtype == np.int32
    assert score.strides[1] == 4 and ref.strides[1] == 4
    n = score.shape[0] - 1
    ops = np.zeros(max(2 * n, 1), dtype=np.uint8)
    L = lib().nw_traceback_ref(_ptr(score), score.strides[0] // 4, _ptr(ref), ref.strides[0] // 4, n, int(p),
                               ops.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)))
    if L < 0:
        raise ValueError("nw_traceback_ref: a cell matches none of its three moves")
    return ops[:L].copy()


class NwRefStream:
    """Row-streaming oracle (O(n) memory): feed ref rows, get score rows."""

    def __init__(self, n: int, p: int, row0: np.ndarray):
        row0 = np.ascontiguousarray(row0, dtype=np.int32)
        assert row0.shape == (n + 1,)
        self.n = n
        self._h = lib().nw_ref_stream_new(n, int(p), _ptr(row0))
        if not self._h:
            raise MemoryError("nw_ref_stream_new")

    def rows(self, ref_rows: np.ndarray, col0: np.ndarray, want_out: bool = True):
        ref_rows = np.ascontiguousarray(ref_rows, dtype=np.int32)
        col0 = np.ascontiguousarray(col0, dtype=np.int32)
        k = ref_rows.shape[0]
        assert ref_rows.shape[1] >= self.n + 1 and col0.shape == (k,)
        out = np.empty((k, self.n + 1), dtype=np.int32) if want_out else None
        rc = lib().nw_ref_stream_rows(
            self._h, _ptr(ref_rows), ref_rows.strides[0] // 4, _ptr(col0), k,
            _ptr(out) if out is not None else None, self.n + 1,
        )
        if rc != 0:
            raise OverflowError("nw_ref_stream_rows: a cell value does not fit in int32")
        return out

    def last(self) -> np.ndarray:
        p = lib().nw_ref_stream_last(self._h)
        return np.ctypeslib.as_array(p, shape=(self.n + 1,)).copy()

    def close(self):
        if self._h:
            lib().nw_ref_stream_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
