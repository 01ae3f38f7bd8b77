"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This module holds none of the method's arithmetic (no condensation, no SpMM):
it only draws canonical CSR sparsity patterns and value arrays from a
counter-based generator (``gen.c``), so every array is a pure function of its
seed and independent of the thread count.  The recipes are stated in
DESIGN.md §"Input recipe".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libdatagen.so")
_lock = threading.Lock()
_lib = None

# counter-stream ids for the value arrays (the pattern streams live in gen.c)
STREAM_AVALS = 11
STREAM_B = 12


def build(force: bool = False) -> str:
    """Compile gen.c into libdatagen.so (gcc, OpenMP)."""
    src = os.path.join(_HERE, "gen.c")
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
            i64, u64, dbl, f32 = ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_float
            vp = ctypes.c_void_p
            L.dg_powerlaw_degrees.argtypes = [i64, i64, dbl, i64, u64, vp]
            L.dg_powerlaw_degrees.restype = i64
            L.dg_zipf_table.argtypes = [i64, dbl, u64, vp, vp]
            L.dg_zipf_table.restype = ctypes.c_int
            L.dg_powerlaw_fill.argtypes = [i64, i64, vp, dbl, i64, vp, vp, u64, vp]
            L.dg_powerlaw_fill.restype = ctypes.c_int
            L.dg_banded_degrees.argtypes = [i64, i64, i64, i64, i64, i64, u64, vp, vp]
            L.dg_banded_degrees.restype = i64
            L.dg_banded_fill.argtypes = [i64, i64, vp, i64, i64, vp, u64, vp]
            L.dg_banded_fill.restype = ctypes.c_int
            L.dg_uniform_f32.argtypes = [u64, u64, i64, f32, f32, vp]
            L.dg_uniform_f32.restype = None
            L.dg_int_f32.argtypes = [u64, u64, i64, i64, i64, vp]
            L.dg_int_f32.restype = None
            L.dg_dyadic_f32.argtypes = [u64, u64, i64, i64, i64, vp]
            L.dg_dyadic_f32.restype = None
            _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def zipf_beta_for(K: int, draws: float, top_count: float) -> float:
    """Zipf exponent beta such that the most popular column expects `top_count`
    of `draws` global draws: Z(beta) = sum_{r<=K} r^-beta = draws / top_count."""
    target = max(draws / max(top_count, 1.0), 1.0 + 1e-9)
    r = np.arange(1, K + 1, dtype=np.float64)
    lo, hi = 0.0, 4.0
    for _ in range(60):
        mid = 0.5 * (lo + hi)
        z = float(np.sum(r ** -mid))
        if z > target:
            lo = mid
        else:
            hi = mid
    return 0.5 * (lo + hi)


def powerlaw_csr(M: int, K: int, nnz: int, alpha: float, d_max: int, p_local: float,
                 S: int, beta: float, seed: int):
    """G1: locality power-law graph -> (rowptr int32[M+1], colidx int32[nnz'])."""
    L = lib()
    deg = np.empty(M, dtype=np.int32)
    L.dg_powerlaw_degrees(M, nnz, alpha, min(d_max, K), seed, _p(deg))
    rowptr = np.zeros(M + 1, dtype=np.int64)
    np.cumsum(deg, out=rowptr[1:])
    cdf = np.empty(K, dtype=np.float64)
    perm = np.empty(K, dtype=np.int32)
    L.dg_zipf_table(K, beta, seed, _p(cdf), _p(perm))
    col = np.empty(int(rowptr[-1]), dtype=np.int32)
    rc = L.dg_powerlaw_fill(M, K, _p(rowptr), p_local, S, _p(cdf), _p(perm), seed, _p(col))
    if rc != 0:
        raise ValueError("row degree exceeds K")
    return rowptr.astype(np.int32), col


def banded_csr(M: int, K: int, per_row: int, half_band: int, n_out: int, out_len: int, seed: int):
    """G2: banded/FEM pattern with n_out long-row outliers."""
    L = lib()
    deg = np.empty(M, dtype=np.int32)
    out_rows = np.zeros(max(n_out, 1), dtype=np.int64)
    L.dg_banded_degrees(M, K, per_row, half_band, n_out, out_len, seed, _p(deg), _p(out_rows))
    rowptr = np.zeros(M + 1, dtype=np.int64)
    np.cumsum(deg, out=rowptr[1:])
    col = np.empty(int(rowptr[-1]), dtype=np.int32)
    L.dg_banded_fill(M, K, _p(rowptr), half_band, n_out, _p(out_rows), seed, _p(col))
    return rowptr.astype(np.int32), col


def random_csr(M: int, K: int, density: float, seed: int, row_cap: int | None = None):
    """Small uniform-random pattern (tests): each of the M*K entries kept with
    probability `density`, drawn from the counter-based generator."""
    u = uniform(seed, 99, M * K, 0.0, 1.0).reshape(M, K)
    mask = u < density
    if row_cap is not None:
        for i in range(M):
            nz = np.flatnonzero(mask[i])
            if len(nz) > row_cap:
                mask[i, nz[row_cap:]] = False
    rowptr = np.zeros(M + 1, dtype=np.int32)
    rowptr[1:] = np.cumsum(mask.sum(axis=1))
    col = np.nonzero(mask)[1].astype(np.int32)
    return rowptr, col


def uniform(seed: int, stream: int, n: int, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    out = np.empty(n, dtype=np.float32)
    lib().dg_uniform_f32(seed, stream, n, lo, hi, _p(out))
    return out


def integers(seed: int, stream: int, n: int, lo: int = -4, hi: int = 4) -> np.ndarray:
    out = np.empty(n, dtype=np.float32)
    lib().dg_int_f32(seed, stream, n, lo, hi, _p(out))
    return out


def dyadic(seed: int, stream: int, n: int, lo: int = -2, hi: int = 2) -> np.ndarray:
    out = np.empty(n, dtype=np.float32)
    lib().dg_dyadic_f32(seed, stream, n, lo, hi, _p(out))
    return out


def values(kind: str, seed: int, stream: int, n: int) -> np.ndarray:
    """Value recipe by name: 'uniform' U(-1,1), 'int' {-4..4}, 'dyadic' k/8 in [-2,2], 'ones'."""
    if kind == "uniform":
        return uniform(seed, stream, n)
    if kind == "int":
        return integers(seed, stream, n)
    if kind == "dyadic":
        return dyadic(seed, stream, n)
    if kind == "ones":
        return np.ones(n, dtype=np.float32)
    raise ValueError(kind)
