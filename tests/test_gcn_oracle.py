"""Pins for the GraphConv oracle (oracle/gcn.py, Eq. (2)) -- CPU only."""
import numpy as np
import pytest

import datagen
from oracle import gcn as ogcn


def _dense(M, K, rowptr, colidx, vals):
    A = np.zeros((M, K))
    for i in range(M):
        for p in range(rowptr[i], rowptr[i + 1]):
            A[i, colidx[p]] = vals[p]
    return A


def _layer_loops(A, H, W, b, relu):
    """Eq. (2) written out with explicit loops: ((A x H) x W + b), then sigma."""
    M, K = A.shape
    Fi, Fo = W.shape
    AH = [[sum(A[i, k] * float(H[k, f]) for k in range(K)) for f in range(Fi)] for i in range(M)]
    Y = np.zeros((M, Fo))
    for i in range(M):
        for j in range(Fo):
            z = sum(AH[i][f] * float(W[f, j]) for f in range(Fi)) + (float(b[j]) if b is not None else 0.0)
            Y[i, j] = max(z, 0.0) if relu else z
    return Y


def _case(M, K, Fi, Fo, density, seed, kind="int"):
    rp, ci = datagen.random_csr(M, K, density, seed)
    v = datagen.values(kind, seed, 1, len(ci))
    H = datagen.values(kind, seed, 2, K * Fi).reshape(K, Fi)
    W = datagen.values(kind, seed, 3, Fi * Fo).reshape(Fi, Fo)
    b = datagen.values(kind, seed, 4, Fo)
    return rp, ci, v, H, W, b


@pytest.mark.parametrize("relu", [True, False])
@pytest.mark.parametrize("shape", [(5, 7, 3, 4), (17, 9, 6, 2), (1, 1, 1, 1)])
def test_brute_force_integers_exact(shape, relu):
    M, K, Fi, Fo = shape
    rp, ci, v, H, W, b = _case(M, K, Fi, Fo, 0.4, sum(shape))
    Y, Bound, AH = ogcn.graphconv(M, K, rp, ci, v, H, W, b, relu)
    ref = _layer_loops(_dense(M, K, rp, ci, v), H, W, b, relu)
    assert np.array_equal(Y, ref)          # small integers: every step exact in FP64


def test_identity_weights_reduce_to_spmm():
    import oracle
    rp, ci, v, H, _, _ = _case(23, 19, 5, 5, 0.3, 7, "uniform")
    Y, _, AH = ogcn.graphconv(23, 19, rp, ci, v, H, np.eye(5, dtype=np.float32), None, relu=False)
    C, _ = oracle.spmm(23, 19, rp, ci, v, H)
    assert np.array_equal(Y, C) and np.array_equal(AH, C)


def test_identity_adjacency_is_a_dense_layer():
    n = 11
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    v = np.ones(n, np.float32)
    _, _, _, H, W, b = _case(n, n, 4, 3, 0.0, 3)
    Y, _, _ = ogcn.graphconv(n, n, rp, ci, v, H, W, b, relu=True)
    ref = _layer_loops(np.eye(n), H, W, b, True)
    assert np.array_equal(Y, ref)


def test_associativity_catches_transposed_operands():
    rp, ci, v, H, W, _ = _case(31, 29, 6, 4, 0.2, 11, "uniform")
    Y, _, _ = ogcn.graphconv(31, 29, rp, ci, v, H, W, None, relu=False)
    A = _dense(31, 29, rp, ci, v)
    np.testing.assert_allclose(Y, A @ (H.astype(np.float64) @ W.astype(np.float64)), rtol=1e-12, atol=1e-12)


def test_relu_sign_pattern_and_bound():
    rp, ci, v, H, W, b = _case(40, 40, 8, 8, 0.2, 5, "uniform")
    Y, Bound, AH = ogcn.graphconv(40, 40, rp, ci, v, H, W, b, relu=True)
    Z, _, _ = ogcn.graphconv(40, 40, rp, ci, v, H, W, b, relu=False)
    assert np.all(Y >= 0) and np.array_equal(Y > 0, Z > 0)
    assert np.array_equal(Y[Z > 0], Z[Z > 0])
    assert np.all(np.abs(Z - b[None, :].astype(np.float64)) <= Bound + 1e-12)
    rtol, atol = ogcn.tolerance("tf32", W)
    assert rtol == pytest.approx(4e-3) and atol.shape == (1, 8)
