"""oracle/ -- TEST INFRASTRUCTURE ONLY (not part of the product path).

Two independent oracles written from PAPER.md (Prajapati et al., PPoPP'17):

* ``stencil_oracle.c`` (wrapped here): naive two-plane time stepping of
  Eq. 1 in fp32, in the canonical per-point expression
  order of DESIGN.md reading R4, "plain" (separate mul/add) or "fused" (fmaf).
* ``model_oracle.py``: the execution-time model, Eqs. 2-30, and the tile
  optimisation problem, Eq. 31 (§4, §6.1), in fp64.

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this package.  Nothing here imports the
product package and the product never imports this (tests/test_independence.py
checks both directions).  Pins (tests/test_oracle_*.py) tie these oracles to
the paper and to mathematics, not to themselves; see DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stencil_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

JACOBI2D_5PT, HEAT2D_9PT, GRADIENT2D, HEAT3D_7PT, LAPLACIAN3D_27PT, LAPLACIAN2D_5PT = 1, 2, 3, 4, 5, 6
JACOBI1D_3PT = 7
BINOM1D_R2, BINOM1D_R3, BINOM1D_R4 = 8, 9, 10      # radius-r 1D binomial smoothers
KIND_NDIMS = {1: 2, 2: 2, 3: 2, 4: 3, 5: 3, 6: 2, 7: 1, 8: 1, 9: 1, 10: 1}
KIND_RADIUS = {8: 2, 9: 3, 10: 4}
PLAIN, FUSED = 0, 1

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared", "-fPIC"]


def build(force: bool = False) -> str:
    """Compile the C oracle (gcc).  Called by __graft_entry__.build() too:
    building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.oracle_run.restype = ctypes.c_int
        lib.oracle_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
                                   ctypes.POINTER(ctypes.c_float), ctypes.c_int,
                                   ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                   ctypes.c_int, ctypes.c_int]
        lib.oracle_stencil_info.restype = ctypes.c_int
        lib.oracle_stencil_info.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_int),
                                            ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_float)]
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def run(kind: int, field: np.ndarray, T: int, mode: int = PLAIN, coeffs=None,
        nthreads: int = 0) -> np.ndarray:
    """A_T from A_0 = field (full extents incl. the fixed ring)."""
    lib = _load()
    a = np.ascontiguousarray(field, dtype=np.float32)
    out = np.empty_like(a)
    dims = (ctypes.c_int64 * a.ndim)(*a.shape)
    if coeffs is None:
        cp, nc = None, 0
    else:
        c = np.ascontiguousarray(coeffs, dtype=np.float32)
        cp, nc = c.ctypes.data_as(ctypes.POINTER(ctypes.c_float)), int(c.size)
    rc = lib.oracle_run(int(kind), a.ndim, dims, cp, nc, a.ctypes.data, out.ctypes.data,
                        int(T), int(mode), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_run rejected arguments (rc={rc})")
    return out


def stencil_info(kind: int):
    """(offsets [n,3] int, default weights [n] float32) in canonical order."""
    lib = _load()
    n = ctypes.c_int()
    offs = (ctypes.c_int * 81)()
    w = (ctypes.c_float * 27)()
    if lib.oracle_stencil_info(int(kind), ctypes.byref(n), offs, w) != 0:
        raise ValueError(kind)
    k = n.value
    return (np.array(offs[:3 * k], dtype=np.int64).reshape(k, 3),
            np.array(w[:k], dtype=np.float32))


def max_threads() -> int:
    return _load().oracle_max_threads()
