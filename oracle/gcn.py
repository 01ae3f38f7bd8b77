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

Backward (graphconv_backward, softmax_xent): the chain rule of Eq. (2) and the mean softmax
cross-entropy, pinned by central finite differences of the forward (independent of the backward
formulas), the transpose by a dense A.T, and softmax-xent closed forms (uniform logits: log C).
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


# ------------------------------------------------------------------ backward (NEXT-3 training)
def csr_transpose(M, K, rowptr, colidx, vals):
    """CSR of A^T (K x M) by a stable argsort of the column indices (a library sort as a step):
    rows of A^T = columns of A, entries in ascending original row."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    colidx = np.asarray(colidx, dtype=np.int64)
    rows = np.repeat(np.arange(M, dtype=np.int64), np.diff(rowptr))
    order = np.argsort(colidx, kind="stable")          # CSR order is row-major, so ties keep row order
    rp_t = np.zeros(K + 1, dtype=np.int64)
    np.add.at(rp_t, colidx + 1, 1)
    rp_t = np.cumsum(rp_t)
    return rp_t.astype(np.int32), rows[order].astype(np.int32), np.asarray(vals)[order]


def graphconv_backward(M, K, rowptr, colidx, vals, H, W, dY, mask=None):
    """Chain rule of Eq. (2) in FP64, in the order the library computes it:
    dZ = dY * mask (mask = [Y > 0] for ReLU, taken from the caller's forward so both sides make the
    same sign decision; None = identity), dW = AH^T dZ, db = sum_rows dZ, dAH = dZ W^T, dH = A^T dAH.
    Returns dict of the gradients and their error bounds (|.|-products of the same expressions)."""
    AH, BdAH = _spmm(M, K, rowptr, colidx, vals, np.asarray(H, dtype=np.float32))
    dY = np.asarray(dY, dtype=np.float64)
    dZ = dY * mask if mask is not None else dY
    Wd = np.asarray(W, dtype=np.float64)
    aZ = np.abs(dZ)
    out = {"dZ": dZ, "dW": AH.T @ dZ, "bound_dW": BdAH.T @ aZ, "db": dZ.sum(axis=0), "bound_db": aZ.sum(axis=0),
           "dAH": dZ @ Wd.T, "bound_dAH": aZ @ np.abs(Wd).T}
    rp_t, ci_t, v_t = csr_transpose(M, K, rowptr, colidx, vals)
    out["dH"] = _spmm(K, M, rp_t, ci_t, np.asarray(v_t, dtype=np.float32), out["dAH"].astype(np.float32),
                      bound=False)
    # |A^T| (|dZ| |W|^T): O1 on the absolute values (non-negative inputs; float32 is ample for a bound)
    out["bound_dH"] = _spmm(K, M, rp_t, ci_t, np.abs(np.asarray(v_t, dtype=np.float32)),
                            out["bound_dAH"].astype(np.float32), bound=False)
    return out


def backward_tolerance(dtype: str, M: int):
    """rtol of (dW, db, dAH, dH) on their bounds: the SpMM rtol and a TF32 GEMM (2e-3) compounded
    (AH and dAH carry their own errors into the next product), db an FP32 sum of M terms."""
    from . import TOL
    r_s = TOL[dtype]
    chain = r_s + GEMM_RTOL * (1.0 + r_s)
    return {"dW": chain, "db": max(M, 1) * 2.0 ** -23, "dAH": GEMM_RTOL, "dH": r_s + GEMM_RTOL * (1.0 + r_s)}


def softmax_xent(logits, labels):
    """Mean softmax cross-entropy in FP64: (loss, dlogits) with dlogits = (softmax - onehot) / M."""
    z = np.asarray(logits, dtype=np.float64)
    M = z.shape[0]
    mx = z.max(axis=1, keepdims=True)
    e = np.exp(z - mx)
    se = e.sum(axis=1, keepdims=True)
    lab = np.asarray(labels, dtype=np.int64)
    loss = float(np.mean(np.log(se[:, 0]) + mx[:, 0] - z[np.arange(M), lab])) if M else 0.0
    g = e / se
    g[np.arange(M), lab] -= 1.0
    return loss, g / max(M, 1)
