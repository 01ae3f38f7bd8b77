"""Pins for oracle O1 (SpMM) against things other than itself.

SURVEY.md §8(c) pins P1, P3, P4, P5, P11 (+ the |A|·|B| bound and the row-range
chunking used by the full-size comparisons).  Every expected value here comes
from a different computation: a dense triple loop, numpy's dense matmul, or a
closed form (identity / permutation / row sums).
"""
import numpy as np
import pytest

import datagen
import oracle


def _dense(M, K, rowptr, colidx, vals):
    A = np.zeros((M, K), dtype=np.float64)
    for i in range(M):
        for p in range(rowptr[i], rowptr[i + 1]):
            A[i, colidx[p]] = vals[p]
    return A


def _triple_loop(A, B):
    M, K = A.shape
    N = B.shape[1]
    C = np.zeros((M, N), dtype=np.float64)
    for i in range(M):
        for j in range(N):
            s = 0.0
            for k in range(K):
                s += A[i, k] * float(B[k, j])
            C[i, j] = s
    return C


@pytest.mark.parametrize("density", [0.0, 0.05, 0.5, 1.0])
@pytest.mark.parametrize("shape", [(7, 5, 3), (33, 64, 16), (64, 17, 9)])
def test_p1_dense_brute_force_integers_bit_exact(density, shape):
    """P1: small integers -> every product and partial sum is exact in FP64."""
    M, K, N = shape
    rp, ci = datagen.random_csr(M, K, density, seed=M * 131 + K)
    v = datagen.integers(7, 1, len(ci))
    B = datagen.integers(8, 2, K * N).reshape(K, N)
    C, Bd = oracle.spmm(M, K, rp, ci, v, B)
    A = _dense(M, K, rp, ci, v)
    assert np.array_equal(C, _triple_loop(A, B))
    assert np.array_equal(Bd, _triple_loop(np.abs(A), np.abs(B)))


@pytest.mark.parametrize("density", [0.05, 0.5])
def test_p1_dense_matmul_uniform(density):
    """P1 with U(-1,1) values against numpy's dense FP64 GEMM (library routine)."""
    M, K, N = 48, 40, 12
    rp, ci = datagen.random_csr(M, K, density, seed=3)
    v = datagen.uniform(5, 1, len(ci))
    B = datagen.uniform(6, 2, K * N).reshape(K, N)
    C, Bd = oracle.spmm(M, K, rp, ci, v, B)
    A = _dense(M, K, rp, ci, v)
    np.testing.assert_allclose(C, A @ B.astype(np.float64), rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(Bd, np.abs(A) @ np.abs(B.astype(np.float64)), rtol=1e-13, atol=1e-14)


def test_p3_identity():
    """P3: A = I  ->  C = B exactly."""
    M = 100
    rp = np.arange(M + 1, dtype=np.int32)
    ci = np.arange(M, dtype=np.int32)
    v = np.ones(M, dtype=np.float32)
    B = datagen.uniform(9, 2, M * 24).reshape(M, 24)
    C, _ = oracle.spmm(M, M, rp, ci, v, B)
    assert np.array_equal(C, B.astype(np.float64))


def test_p4_permutation():
    """P4: A = P (a permutation)  ->  C = row-permuted B exactly."""
    M = 257
    perm = np.random.default_rng(0).permutation(M).astype(np.int32)
    rp = np.arange(M + 1, dtype=np.int32)
    v = np.ones(M, dtype=np.float32)
    B = datagen.uniform(10, 2, M * 8).reshape(M, 8)
    C, _ = oracle.spmm(M, M, rp, perm, v, B)
    assert np.array_equal(C, B[perm].astype(np.float64))


def test_p5_row_sums():
    """P5: B = ones, dyadic A  ->  C[i, j] = sum_k A_ik for all j (exact)."""
    M, K, N = 300, 500, 7
    rp, ci = datagen.random_csr(M, K, 0.03, seed=11)
    v = datagen.dyadic(12, 1, len(ci))
    C, _ = oracle.spmm(M, K, rp, ci, v, np.ones((K, N), dtype=np.float32))
    rows = np.repeat(np.arange(M), np.diff(rp))
    sums = np.zeros(M)
    np.add.at(sums, rows, v.astype(np.float64))   # exact: dyadic values, small sums
    for j in range(N):
        assert np.array_equal(C[:, j], sums)


def test_p11_linearity():
    M, K, N = 120, 90, 10
    rp, ci = datagen.random_csr(M, K, 0.1, seed=13)
    v = datagen.uniform(14, 1, len(ci))
    B1 = datagen.uniform(15, 2, K * N).reshape(K, N)
    B2 = datagen.uniform(16, 2, K * N).reshape(K, N)
    C1, _ = oracle.spmm(M, K, rp, ci, v, B1)
    C2, _ = oracle.spmm(M, K, rp, ci, v, B2)
    C12, _ = oracle.spmm(M, K, rp, ci, v, (B1.astype(np.float64) + B2).astype(np.float32))
    # B1+B2 is rounded to fp32 once; the FP64 sum is otherwise exact-ish
    np.testing.assert_allclose(C12, C1 + C2, rtol=1e-6, atol=1e-6)


def test_empty_rows_and_row_ranges():
    M, K, N = 50, 30, 5
    rp, ci = datagen.random_csr(M, K, 0.1, seed=17)
    # force some empty rows
    keep = np.ones(len(ci), dtype=bool)
    rows = np.repeat(np.arange(M), np.diff(rp))
    keep[(rows % 7) == 3] = False
    ci2 = ci[keep]
    rp2 = np.zeros(M + 1, dtype=np.int32)
    rp2[1:] = np.cumsum(np.bincount(rows[keep], minlength=M))
    v = datagen.uniform(18, 1, len(ci2))
    B = datagen.uniform(19, 2, K * N).reshape(K, N)
    C, _ = oracle.spmm(M, K, rp2, ci2, v, B)
    assert np.all(C[3::7] == 0.0)
    Cpart, _ = oracle.spmm(M, K, rp2, ci2, v, B, r0=10, r1=37)
    assert np.array_equal(Cpart, C[10:37])
    rs = np.array([0, 5, 49, 3, 10], dtype=np.int64)
    cs = np.array([0, 4, 2, 1, 3], dtype=np.int64)
    Cs, _ = oracle.spmm_at(M, rp2, ci2, v, B, rs, cs)
    assert np.array_equal(Cs, C[rs, cs])


def test_strided_B():
    """ldb > N: the oracle reads rows with the given stride."""
    M, K, N = 20, 30, 6
    rp, ci = datagen.random_csr(M, K, 0.2, seed=21)
    v = datagen.integers(22, 1, len(ci))
    Bfull = datagen.integers(23, 2, K * 10).reshape(K, 10)
    C, _ = oracle.spmm(M, K, rp, ci, v, Bfull[:, :N])
    A = _dense(M, K, rp, ci, v)
    assert np.array_equal(C, _triple_loop(A, Bfull[:, :N]))


def test_tolerance_helper():
    C = np.array([1.0, 2.0])
    ok, r = oracle.within_tolerance(C + np.array([1e-4, 0.0]), C, np.array([1.0, 1.0]), 2e-3)
    assert ok and r < 1
    ok, _ = oracle.within_tolerance(C + np.array([1e-2, 0.0]), C, np.array([1.0, 1.0]), 2e-3)
    assert not ok
    ok, _ = oracle.within_tolerance(np.array([np.nan, 2.0]), C, np.array([1.0, 1.0]), 2e-3)
    assert not ok
