"""CPU oracle for the PDL-mapped blocked matmul -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and the ``cpu_baseline`` /
``--impl reference`` legs of ``bench.py`` may import this package.  The product
path (``paper_conf_ipps_sandrieserbp11_b200``) never imports it and shares no
code with it: the C source ``oracle.c`` is compiled into its own
``liboracle.so`` with gcc, no CUDA, no shared headers.

What it computes -- the plain definition the paper's DGEMM task reaches
(SS IV-D: "double precision matrix multiplication of two
8192x8192 matrices (DGEMM)"; tasks keep one signature and functionality across
implementation variants, L1032-1039)::

    Cref[i, j] = sum_k A[i, k] * B[k, j]     (k ascending, double accumulator)
    D[i, j]    = sum_k |A[i, k]| * |B[k, j]|

Pins (tests/test_oracle_pins.py) tie it to exact rational arithmetic
(fractions.Fraction brute force), identity/permutation products, rank-1 closed
forms, integer matrices and the gamma_K error bound -- none of which re-use this
code.  Parity with the paper's own numbers is unpinned: PAPER.md prints no
DGEMM output (Figure 5's bars are missing, L1390-1394).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (no CUDA).  Returns the library path."""
    if (not force and os.path.exists(_LIB)
            and os.path.getmtime(_LIB) >= os.path.getmtime(_SRC)):
        return _LIB
    cmd = ["gcc", "-O3", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
           "-shared", "-fPIC", "-o", _LIB, _SRC, "-lm"]
    subprocess.check_call(cmd)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        # ORACLE_LIB: load another build of oracle.c (mutation tests only)
        path = os.environ.get("ORACLE_LIB") or build()
        lib = ctypes.CDLL(path)
        i64 = ctypes.c_int64
        vp = ctypes.c_void_p
        lib.oracle_matmul_rows.argtypes = [ctypes.c_int, vp, vp, i64, i64, i64,
                                           vp, i64, vp, vp, ctypes.c_int]
        lib.oracle_matmul_rows.restype = ctypes.c_int
        lib.oracle_matmul.argtypes = [ctypes.c_int, vp, vp, i64, i64, i64,
                                      vp, vp, ctypes.c_int]
        lib.oracle_matmul.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _dtype_code(a: np.ndarray) -> int:
    if a.dtype == np.float64:
        return 0
    if a.dtype == np.float32:
        return 1
    raise TypeError(f"oracle supports float64/float32 inputs, got {a.dtype}")


def matmul(A: np.ndarray, B: np.ndarray, rows=None, nthreads: int = 0,
           with_mag: bool = True):
    """Return (Cref, D) in float64 for the given rows (all rows if None).

    A: (M, K), B: (K, N), same dtype (float64 or float32), C-contiguous.
    """
    A = np.ascontiguousarray(A)
    B = np.ascontiguousarray(B)
    if A.ndim != 2 or B.ndim != 2 or A.shape[1] != B.shape[0]:
        raise ValueError(f"bad shapes {A.shape} x {B.shape}")
    if A.dtype != B.dtype:
        raise TypeError("A and B must share a dtype")
    M, K = A.shape
    N = B.shape[1]
    code = _dtype_code(A)
    if rows is None:
        nrows = M
        rows_arr = None
    else:
        rows_arr = np.ascontiguousarray(np.asarray(rows, dtype=np.int64))
        nrows = rows_arr.size
    C = np.empty((nrows, N), dtype=np.float64)
    D = np.empty((nrows, N), dtype=np.float64) if with_mag else None
    lib = _load()
    rc = lib.oracle_matmul_rows(
        code, A.ctypes.data if A.size else None, B.ctypes.data if B.size else None,
        M, N, K,
        rows_arr.ctypes.data if rows_arr is not None and nrows else None, nrows,
        C.ctypes.data if C.size else None,
        D.ctypes.data if (D is not None and D.size) else None, int(nthreads))
    if rc != 0:
        raise RuntimeError(f"oracle_matmul_rows failed ({rc})")
    return C, D


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def scaled_error(C: np.ndarray, Cref: np.ndarray, D: np.ndarray):
    """Element-wise error |C - Cref| / D (R13).

    Where D == 0 the exact product is 0 and C must be exactly 0 (error 0 if so,
    inf otherwise).  Non-finite C where the inputs were finite gives inf.
    Returns the error array (float64).
    """
    C = np.asarray(C, dtype=np.float64)
    diff = np.abs(C - Cref)
    with np.errstate(divide="ignore", invalid="ignore"):
        err = np.where(D > 0, diff / np.where(D > 0, D, 1.0),
                       np.where(C == 0, 0.0, np.inf))
    err = np.where(np.isfinite(C), err, np.inf)
    return err
