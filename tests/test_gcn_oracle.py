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


# ------------------------------------------------------------------ backward pins (finite differences)
def _tiny(seed, M=9, K=11, Fi=3, Fo=2, density=0.35):
    rng = np.random.default_rng(seed)
    Ad = (rng.random((M, K)) < density) * rng.uniform(-1, 1, (M, K))
    rp = np.concatenate([[0], np.cumsum((Ad != 0).sum(1))]).astype(np.int32)
    ci = np.nonzero(Ad)[1].astype(np.int32)
    v = Ad[Ad != 0].astype(np.float32)
    H = rng.uniform(-1, 1, (K, Fi)).astype(np.float32)
    W = rng.uniform(-1, 1, (Fi, Fo))
    b = rng.uniform(-1, 1, Fo)
    R = rng.uniform(-1, 1, (M, Fo))
    return Ad.astype(np.float32).astype(np.float64), rp, ci, v, H, W, b, R


def _loss(Ad, H, W, b, R, relu):
    Z = Ad @ H.astype(np.float64) @ W + b
    Y = np.maximum(Z, 0) if relu else Z
    return float((Y * R).sum()), Y


@pytest.mark.parametrize("relu", [False, True])
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_backward_matches_finite_differences(seed, relu):
    """L = sum(Y * R) so dY = R; every gradient the oracle returns equals the central difference of
    the FORWARD (a dense FP64 expression, independent of the backward formulas) -- a dropped term,
    a transposed operand or a wrong sign in dW, db, dH fails."""
    Ad, rp, ci, v, H, W, b, R = _tiny(seed)
    M, K = Ad.shape
    _, Y = _loss(Ad, H, W, b, R, relu)
    mask = (Y > 0).astype(np.float64) if relu else None
    g = ogcn.graphconv_backward(M, K, rp, ci, v, H, W, R, mask=mask)
    eps = 1e-6
    for (i, j) in [(0, 0), (1, 1), (2, 0)]:
        Wp, Wm = W.copy(), W.copy()
        Wp[i, j] += eps
        Wm[i, j] -= eps
        fd = (_loss(Ad, H, Wp, b, R, relu)[0] - _loss(Ad, H, Wm, b, R, relu)[0]) / (2 * eps)
        assert g["dW"][i, j] == pytest.approx(fd, rel=1e-6, abs=1e-7)
    for j in range(W.shape[1]):
        bp, bm = b.copy(), b.copy()
        bp[j] += eps
        bm[j] -= eps
        fd = (_loss(Ad, H, W, bp, R, relu)[0] - _loss(Ad, H, W, bm, R, relu)[0]) / (2 * eps)
        assert g["db"][j] == pytest.approx(fd, rel=1e-6, abs=1e-7)
    for (k, f) in [(0, 0), (4, 2), (10, 1)]:
        Hp, Hm = H.astype(np.float64), H.astype(np.float64).copy()
        Hp = Hp.copy()
        Hp[k, f] += eps
        Hm[k, f] -= eps
        fd = (_loss(Ad, Hp, W, b, R, relu)[0] - _loss(Ad, Hm, W, b, R, relu)[0]) / (2 * eps)
        assert g["dH"][k, f] == pytest.approx(fd, rel=1e-5, abs=1e-6)


def test_csr_transpose_is_dense_transpose():
    Ad, rp, ci, v, *_ = _tiny(7, M=13, K=6)
    rp_t, ci_t, v_t = ogcn.csr_transpose(13, 6, rp, ci, v)
    D = np.zeros((6, 13))
    for r in range(6):
        for p in range(rp_t[r], rp_t[r + 1]):
            D[r, ci_t[p]] = v_t[p]
        assert np.all(np.diff(ci_t[rp_t[r]:rp_t[r + 1]]) > 0)   # canonical: ascending original row
    assert np.array_equal(D, Ad.T)


def test_softmax_xent_closed_forms_and_fd():
    C = 7
    loss, g = ogcn.softmax_xent(np.zeros((5, C)), np.arange(5) % C)
    assert loss == pytest.approx(np.log(C))
    assert np.allclose(g.sum(axis=1), 0.0)
    rng = np.random.default_rng(4)
    z = rng.normal(size=(4, C))
    lab = rng.integers(0, C, 4)
    _, g = ogcn.softmax_xent(z, lab)
    eps = 1e-6
    for (i, j) in [(0, 0), (2, 5), (3, int(lab[3]))]:
        zp, zm = z.copy(), z.copy()
        zp[i, j] += eps
        zm[i, j] -= eps
        fd = (ogcn.softmax_xent(zp, lab)[0] - ogcn.softmax_xent(zm, lab)[0]) / (2 * eps)
        assert g[i, j] == pytest.approx(fd, rel=1e-6, abs=1e-9)
