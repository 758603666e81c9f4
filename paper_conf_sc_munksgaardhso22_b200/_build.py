"""Build libnwb200.so (the C-ABI library of include/nw.h) in-tree with nvcc for sm_100a.

nvcc cross-compiles without a GPU, so this runs on the CPU dev host too; the resulting .so is
what tests, bench.py and __graft_entry__.smoke() load.
"""
from __future__ import annotations

import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB_PATH = os.path.join(PKG, "libnwb200.so")
SOURCES = ["nw_lib.cu"]
DEPS = ["nw_lib.cu", "nw_common.cuh", "nw_wave.cuh", "nw_diag.cuh", "nw_ptx.cuh", "nw_traceback.cuh"]

NVCC_FLAGS = [
    "-O3", "-std=c++20", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-Xcompiler", "-fPIC", "-shared", "--cudart", "static",
    "-Xptxas", "-v",
]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(LIB_PATH):
        return True
    t = os.path.getmtime(LIB_PATH)
    deps = [os.path.join(CSRC, d) for d in DEPS] + [os.path.join(INCLUDE, "nw.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB_PATH
    tmp = LIB_PATH + f".tmp{os.getpid()}"
    trace = ["-DNW_TRACE=1"] if os.environ.get("NW_TRACE") == "1" else []  # diagnostics build only
    cmd = [nvcc(), *NVCC_FLAGS, *trace, "-I", INCLUDE, "-I", CSRC,
           *[os.path.join(CSRC, s) for s in SOURCES], "-o", tmp]
    r = subprocess.run(cmd, capture_output=True, text=True)
    log = os.path.join(PKG, "build.log")
    with open(log, "w") as f:
        f.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed ({r.returncode}):\n{r.stderr[-4000:]}")
    if verbose:
        print(r.stderr)
    os.replace(tmp, LIB_PATH)
    return LIB_PATH


def build_variant(out_path: str, defines) -> str:
    """Experiments only: the library with extra -D flags at out_path (loaded via NW_LIB)."""
    cmd = [nvcc(), *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", INCLUDE, "-I", CSRC,
           *[os.path.join(CSRC, s) for s in SOURCES], "-o", out_path]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed ({r.returncode}):\n{r.stderr[-4000:]}")
    return out_path


if __name__ == "__main__":
    print(build(force=True, verbose=True))
