"""oracle -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU reference for the DTC-SpMM hot path
(SURVEY.md §8(c)).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA path (``paper_conf_asplos_fan0024_b200``)
and never imports it.

Functions and the passage each follows:

* :func:`spmm` / :func:`spmm_at` -- O1, the definition C = A·B (PAPER.md:68,
  §2.2) in FP64, with Bound = |A|·|B| for the tolerance of BASELINE.json's
  north_star.  Pinned (tests/test_oracle_pins.py) by dense brute force,
  identity, permutation and row-sum cases.
* :func:`condense` -- O2, SGT condensation into ME-TCF (§2.3,
  PAPER.md:180 §4.2) under DESIGN.md readings C3-C7.  Pinned by the decode
  round trip, a brute-force dense-window condensation on tiny inputs, and the
  closed forms of P9/P10.
* :func:`metcf_elements`, :func:`csr_elements`, :func:`tcf_elements` -- the
  storage formulas of PAPER.md:180 and PAPER.md:127 (pinned by exact integer
  equality against the arrays actually built).
* :func:`within_tolerance` -- |C - C_ref| <= rtol·Bound + atol, the acceptance
  test of BASELINE.json (rtol 2e-3 TF32, 1e-2 FP16; atol 1e-6).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

WINDOW = 16
TCW = 8

TOL = {"tf32": 2e-3, "fp16": 1e-2}
ATOL = 1e-6


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11",
                               src, "-o", _SO, "-lm"])
    return _SO


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_SO)
            i64, vp = ctypes.c_int64, ctypes.c_void_p
            L.oracle_spmm.argtypes = [i64, i64, i64, vp, vp, vp, vp, i64, i64, i64, vp, vp]
            L.oracle_spmm.restype = ctypes.c_int
            L.oracle_spmm_at.argtypes = [i64, vp, vp, vp, vp, i64, i64, vp, vp, vp, vp]
            L.oracle_spmm_at.restype = ctypes.c_int
            L.oracle_condense_count_wh.argtypes = [i64, vp, vp, i64, vp]
            L.oracle_condense_count_wh.restype = i64
            L.oracle_condense_fill_wh.argtypes = [i64, vp, vp, i64, vp, i64, vp, vp, vp, vp, vp]
            L.oracle_condense_fill_wh.restype = ctypes.c_int
            L.oracle_max_threads.argtypes = []
            L.oracle_max_threads.restype = ctypes.c_int
            L.oracle_set_threads.argtypes = [ctypes.c_int]
            L.oracle_set_threads.restype = None
            _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def set_threads(n: int) -> None:
    lib().oracle_set_threads(int(n))


def spmm(M, K, rowptr, colidx, vals, B, r0: int = 0, r1: int | None = None, bound: bool = True):
    """O1: rows [r0, r1) of C = A·B and Bound = |A|·|B|, FP64.

    vals: float32 (FP16 inputs are passed upcast -- exact).  B: float32 (K, N),
    any row stride."""
    rowptr = _c(rowptr, np.int32)
    colidx = _c(colidx, np.int32)
    vals = _c(vals, np.float32)
    B = np.asarray(B, dtype=np.float32)
    if B.ndim != 2 or B.strides[1] != 4:
        B = np.ascontiguousarray(B)
    N = B.shape[1]
    ldb = B.strides[0] // 4
    r1 = M if r1 is None else r1
    C = np.empty((r1 - r0, N), dtype=np.float64)
    Bd = np.empty((r1 - r0, N), dtype=np.float64) if bound else None
    rc = lib().oracle_spmm(M, K, N, _p(rowptr), _p(colidx), _p(vals), _p(B), ldb, r0, r1, _p(C), _p(Bd))
    if rc != 0:
        raise ValueError("oracle_spmm: bad row range")
    return (C, Bd) if bound else C


def spmm_at(M, rowptr, colidx, vals, B, rows, cols):
    """O1 at sampled entries (rows[s], cols[s]) -> (C[s], Bound[s])."""
    rowptr = _c(rowptr, np.int32)
    colidx = _c(colidx, np.int32)
    vals = _c(vals, np.float32)
    B = np.asarray(B, dtype=np.float32)
    ldb = B.strides[0] // 4
    rows = _c(rows, np.int64)
    cols = _c(cols, np.int64)
    C = np.empty(len(rows), dtype=np.float64)
    Bd = np.empty(len(rows), dtype=np.float64)
    lib().oracle_spmm_at(M, _p(rowptr), _p(colidx), _p(vals), _p(B), ldb, len(rows),
                         _p(rows), _p(cols), _p(C), _p(Bd))
    return C, Bd


def condense_count(M, rowptr, colidx, window: int = WINDOW):
    """O2 steps 1-2: RowWindowOffset and NumTCBlock (window = rows per window: 16, the paper's
    BLOCK_HEIGHT, or 32 for the NEXT-2 tall windows, reading C2b)."""
    W = (M + window - 1) // window
    rwo = np.zeros(W + 1, dtype=np.int32)
    T = lib().oracle_condense_count_wh(M, _p(_c(rowptr, np.int32)), _p(_c(colidx, np.int32)), window, _p(rwo))
    if T < 0:
        raise ValueError("NumTCBlock overflows int32")
    return rwo, int(T)


def condense(M, rowptr, colidx, vals=None, window: int = WINDOW):
    """O2: CSR -> ME-TCF arrays (dict).  vals may be float32 or float16 (copied
    bit-for-bit into TCValues), or None (pattern only)."""
    rowptr = _c(rowptr, np.int32)
    colidx = _c(colidx, np.int32)
    nnz = int(rowptr[-1]) if len(rowptr) else 0
    rwo, T = condense_count(M, rowptr, colidx, window)
    if vals is None:
        vals = np.zeros(nnz, dtype=np.float32)
    vals = np.ascontiguousarray(vals)
    tco = np.zeros(T + 1, dtype=np.int32)
    lid = np.zeros(max(nnz, 1), dtype=np.uint8)
    atob = np.zeros(max(8 * T, 1), dtype=np.int32)
    tv = np.zeros(max(nnz, 1), dtype=vals.dtype)
    rc = lib().oracle_condense_fill_wh(M, _p(rowptr), _p(colidx), window, _p(vals), vals.itemsize, _p(rwo),
                                       _p(tco), _p(lid), _p(atob), _p(tv))
    if rc != 0:
        raise RuntimeError("oracle_condense_fill failed")
    return {
        "num_windows": len(rwo) - 1,
        "num_tc_blocks": T,
        "row_window_offset": rwo,
        "tc_offset": tco,
        "tc_local_id": lid[:nnz],
        "sparse_a_to_b": atob[: 8 * T],
        "tc_values": tv[:nnz],
    }


# ---------------------------------------------------------------- sizes
def metcf_elements(M: int, T: int, nnz: int) -> float:
    """ceil(M/16) + NumTCBlock*9 + NNZ/4 + 2 (32-bit elements)."""
    return -(-M // 16) + 9 * T + nnz / 4 + 2


def csr_elements(M: int, nnz: int) -> int:
    """CSR index storage M + 1 + NNZ elements."""
    return M + 1 + nnz


def tcf_elements(M: int, nnz: int) -> int:
    """TCF = ceil(M/16) + M + 1 + 3*NNZ elements."""
    return -(-M // 16) + M + 1 + 3 * nnz


def within_tolerance(C, Cref, Bound, rtol: float, atol: float = ATOL):
    """Elementwise |C - Cref| <= rtol*Bound + atol; returns (ok, worst_ratio)."""
    C = np.asarray(C, dtype=np.float64)
    err = np.abs(C - Cref)
    lim = rtol * Bound + atol
    ok = bool(np.all(err <= lim)) and bool(np.all(np.isfinite(C)))
    ratio = float(np.max(err / lim)) if err.size else 0.0
    return ok, ratio
