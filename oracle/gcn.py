"""oracle.gcn -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

GraphConv layer, §5.4 Eq. (2): H_{l+1} = sigma((A x H_l) x w_l + b_l),
in FP64 and in the paper's order:

1. AH = A x H_l         -- O1 (oracle.spmm, the FP64 definition of SpMM)
2. Z  = AH x w_l + b_l  -- a dense FP64 matmul (library primitive) plus the bias row
3. H_{l+1} = sigma(Z)   -- sigma = ReLU or identity

Tolerance bound (GraphConv): the SpMM step errs by at most
rtol_spmm * (|A|·|H|) (+atol), the TF32 GEMM by about 2e-3 * (|AH|·|w|) <= 2e-3 * ((|A|·|H|)·|w|),
and ReLU is 1-Lipschitz, so |Y - Y_ref| <= (rtol_spmm + 2e-3) * Bound + atol * (1 + sum_k |w_kj|)
with Bound = (|A|·|H|)·|w| + 2^-22 |b|.

Pinned by tests/test_gcn_oracle.py: pure-Python triple loops on tiny inputs, identity
weights reducing to O1, identity A reducing to a dense layer, associativity
(A·H)·w = A·(H·w), and ReLU's sign pattern.
"""
from __future__ import annotations

import numpy as np

from . import spmm as _spmm

GEMM_RTOL = 2e-3   # TF32 inputs (2 x 2^-10 worst case per product) + FP32 accumulation


def graphconv(M, K, rowptr, colidx, vals, H, W, bias=None, relu=True):
    """Returns (Y, Bound, AH) in FP64."""
    AH, BdAH = _spmm(M, K, rowptr, colidx, vals, np.asarray(H, dtype=np.float32))
    Wd = np.asarray(W, dtype=np.float64)
    Z = AH @ Wd
    Bound = BdAH @ np.abs(Wd)
    if bias is not None:
        bd = np.asarray(bias, dtype=np.float64)
        Z = Z + bd[None, :]
        Bound = Bound + 2.0 ** -22 * np.abs(bd)[None, :]
    Y = np.maximum(Z, 0.0) if relu else Z
    return Y, Bound, AH


def tolerance(dtype: str, W, atol: float = 1e-6):
    """(rtol, atol per output column) for graphconv outputs (see the module docstring)."""
    from . import TOL
    col_abs = np.abs(np.asarray(W, dtype=np.float64)).sum(axis=0)
    return TOL[dtype] + GEMM_RTOL, atol * (1.0 + col_abs)[None, :]
