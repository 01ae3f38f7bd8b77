"""Pins for oracle O2 (reference ME-TCF condensation).

* a hand-worked example derived on paper from the ME-TCF definition
  under DESIGN.md readings C3-C6;
* a brute-force dense-window condensation (scan every column k=0..K-1 of the
  densified window, enumerate local ids 0..127 in order) on tiny inputs;
* the decode round trip ME-TCF -> CSR on larger inputs (P7);
* closed forms: fully dense A (P9), block-diagonal 16x8 blocks (P10), the
  storage formulas of P:180 and P:127 (P8).
"""
import json
import math
import os

import numpy as np
import pytest

import datagen
import oracle

HERE = os.path.dirname(os.path.abspath(__file__))


def _csr_from_rows(M, rows):
    rp = [0]
    ci = []
    for i in range(M):
        cols = sorted(rows.get(i, []))
        ci += cols
        rp.append(len(ci))
    return np.array(rp, dtype=np.int32), np.array(ci, dtype=np.int32)


def test_hand_worked_example():
    """Two windows (M=20, K=12); derivation in the comments.

    window 0 (rows 0-15): row0 {3,7}, row1 {7}, row5 {1,3,9,10,11}, row15 {0}
      U = [0,1,3,7,9,10,11] -> u=7 -> 1 block, AtoB=[0,1,3,7,9,10,11,-1]
      ids = row*8 + rank: r0c3 -> 2, r0c7 -> 3, r1c7 -> 11, r5: c1->41 c3->42 c9->44
      c10->45 c11->46, r15c0 -> 120
    window 1 (rows 16-19): row16 {0,2,4,5,6,7,8,9,10}, row18 {2,11}
      U = [0,2,4,5,6,7,8,9,10,11] -> u=10 -> 2 blocks
      block a: cols [0,2,4,5,6,7,8,9]: r16 ids 0..7, r18c2 -> 2*8+1 = 17
      block b: cols [10,11,-1 x6]: r16c10 -> 0, r18c11 -> 17
    values = 1..20 in CSR order.
    """
    rows = {0: [3, 7], 1: [7], 5: [1, 3, 9, 10, 11], 15: [0],
            16: [0, 2, 4, 5, 6, 7, 8, 9, 10], 18: [2, 11]}
    rp, ci = _csr_from_rows(20, rows)
    vals = np.arange(1, 21, dtype=np.float32)
    f = oracle.condense(20, rp, ci, vals)
    assert f["num_tc_blocks"] == 3
    assert f["row_window_offset"].tolist() == [0, 1, 3]
    assert f["tc_offset"].tolist() == [0, 9, 18, 20]
    assert f["tc_local_id"].tolist() == [2, 3, 11, 41, 42, 44, 45, 46, 120,
                                         0, 1, 2, 3, 4, 5, 6, 7, 17, 0, 17]
    assert f["sparse_a_to_b"].tolist() == [0, 1, 3, 7, 9, 10, 11, -1,
                                           0, 2, 4, 5, 6, 7, 8, 9,
                                           10, 11, -1, -1, -1, -1, -1, -1]
    assert f["tc_values"].tolist() == [1, 2, 3, 4, 5, 6, 7, 8, 9,
                                       10, 11, 12, 13, 14, 15, 16, 17, 19, 18, 20]
    # P:180 size: ceil(20/16) + 3*9 + 20/4 + 2 = 36 elements = 144 index bytes
    assert oracle.metcf_elements(20, 3, 20) == 36


def brute_condense(M, K, rp, ci, vals, WH=16):
    """Dense-window brute force: scan k = 0..K-1, enumerate ids 0..8*WH-1 (windows of WH rows)."""
    A = np.zeros((M, K), dtype=np.float64)
    mask = np.zeros((M, K), dtype=bool)
    for i in range(M):
        for p in range(rp[i], rp[i + 1]):
            A[i, ci[p]] = vals[p]
            mask[i, ci[p]] = True
    W = -(-M // WH)
    rwo, atob, tco, lid, tv = [0], [], [], [], []
    for w in range(W):
        r0, r1 = WH * w, min(WH * w + WH, M)
        cols = [k for k in range(K) if mask[r0:r1, k].any()]
        nb = -(-len(cols) // 8)
        for b in range(nb):
            bc = cols[8 * b: 8 * b + 8]
            atob += bc + [-1] * (8 - len(bc))
            tco.append(len(lid))
            for lid_ in range(8 * WH):
                r, c = divmod(lid_, 8)
                if r0 + r < r1 and c < len(bc) and mask[r0 + r, bc[c]]:
                    lid.append(lid_)
                    tv.append(A[r0 + r, bc[c]])
        rwo.append(rwo[-1] + nb)
    tco.append(len(lid))
    return rwo, tco, lid, atob, tv


@pytest.mark.parametrize("M,K,density,seed", [
    (1, 1, 1.0, 1), (15, 9, 0.3, 2), (16, 8, 1.0, 3), (17, 40, 0.2, 4), (40, 70, 0.05, 5),
    (48, 130, 0.5, 6), (33, 300, 0.02, 7), (64, 12, 0.0, 8), (20, 200, 0.9, 9),
])
@pytest.mark.parametrize("WH", [16, 32])
def test_brute_force_condensation(M, K, density, seed, WH):
    """O2 (16-row ME-TCF and the 32-row windows of NEXT-2) against a dense brute force."""
    rp, ci = datagen.random_csr(M, K, density, seed)
    v = datagen.uniform(seed, 1, len(ci))
    f = oracle.condense(M, rp, ci, v, window=WH)
    rwo, tco, lid, atob, tv = brute_condense(M, K, rp, ci, v, WH)
    assert f["row_window_offset"].tolist() == rwo
    assert f["tc_offset"].tolist() == tco
    assert f["tc_local_id"].tolist() == lid
    assert f["sparse_a_to_b"].tolist() == atob
    assert np.array_equal(f["tc_values"].astype(np.float64), np.array(tv, dtype=np.float64))


def decode(M, f, WH=16):
    """ME-TCF -> (rows, cols, vals) sorted by (row, col)."""
    rwo, tco, lid = f["row_window_offset"], f["tc_offset"], f["tc_local_id"].astype(np.int64)
    atob, tv = f["sparse_a_to_b"], f["tc_values"]
    T = f["num_tc_blocks"]
    blk_of_window = np.repeat(np.arange(len(rwo) - 1), np.diff(rwo))
    blk_of_nnz = np.repeat(np.arange(T), np.diff(tco))
    rows = WH * blk_of_window[blk_of_nnz] + (lid >> 3)
    cols = atob[8 * blk_of_nnz + (lid & 7)]
    order = np.lexsort((cols, rows))
    return rows[order], cols[order], tv[order]


def check_invariants(M, rp, ci, f):
    """P7 format invariants."""
    T, W = f["num_tc_blocks"], f["num_windows"]
    rwo, tco, lid, atob = f["row_window_offset"], f["tc_offset"], f["tc_local_id"], f["sparse_a_to_b"]
    nnz = len(ci)
    assert W == -(-M // 16) and rwo[0] == 0 and rwo[W] == T
    assert np.all(np.diff(rwo) >= 0) and np.all(np.diff(tco) >= 0)
    assert tco[T] == nnz and (T == 0 or tco[0] == 0)
    for w in range(W):
        b0, b1 = rwo[w], rwo[w + 1]
        cols = atob[8 * b0: 8 * b1]
        valid = cols[cols >= 0]
        assert np.all(np.diff(valid) > 0)                      # strictly increasing per window
        if b1 > b0:
            assert np.all(atob[8 * b0: 8 * (b1 - 1)] >= 0)     # only the last block is padded
            assert atob[8 * (b1 - 1)] >= 0                     # ... and has >= 1 column
        rows_in_w = min(16, M - 16 * w)
        for b in range(b0, b1):
            ids = lid[tco[b]: tco[b + 1]].astype(np.int64)
            assert len(ids) >= 1
            assert np.all(np.diff(ids) > 0) and np.all(ids < 128)
            assert np.all((ids >> 3) < rows_in_w)
            assert np.all(atob[8 * b + (ids & 7)] >= 0)
    # T = sum ceil(u_w / 8)
    u = [len(np.unique(ci[rp[16 * w]: rp[min(16 * w + 16, M)]])) for w in range(W)]
    assert T == sum(-(-x // 8) for x in u)


@pytest.mark.parametrize("name", ["c1"])
def test_decode_round_trip_config(name):
    from datagen import configs
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = oracle.condense(cfg.M, rp, ci, v)
    check_invariants(cfg.M, rp, ci, f)
    r, c, vv = decode(cfg.M, f)
    assert np.array_equal(r, np.repeat(np.arange(cfg.M), np.diff(rp)))
    assert np.array_equal(c, ci)
    assert np.array_equal(vv, v)
    mean = len(ci) / f["num_tc_blocks"]
    assert 0.9 * cfg.mean_nnz_tc_target < mean < 1.2 * cfg.mean_nnz_tc_target


@pytest.mark.parametrize("M,K,density,seed", [(100, 5000, 0.01, 1), (333, 333, 0.1, 2), (1000, 64, 0.3, 3)])
def test_decode_round_trip_random(M, K, density, seed):
    rp, ci = datagen.random_csr(M, K, density, seed)
    v = datagen.uniform(seed, 1, len(ci)).astype(np.float16)
    f = oracle.condense(M, rp, ci, v)
    check_invariants(M, rp, ci, f)
    r, c, vv = decode(M, f)
    assert np.array_equal(r, np.repeat(np.arange(M), np.diff(rp)))
    assert np.array_equal(c, ci)
    assert np.array_equal(vv.view(np.uint16), v.view(np.uint16))


@pytest.mark.parametrize("M,K", [(32, 24), (48, 64), (20, 13)])
def test_p9_fully_dense(M, K):
    rp = (np.arange(M + 1) * K).astype(np.int32)
    ci = np.tile(np.arange(K, dtype=np.int32), M)
    f = oracle.condense(M, rp, ci)
    W = -(-M // 16)
    assert f["num_tc_blocks"] == W * math.ceil(K / 8)
    if M % 16 == 0 and K % 8 == 0:
        assert len(ci) / f["num_tc_blocks"] == 128
    # every full block has ids 0..127 in order
    if M % 16 == 0 and K % 8 == 0:
        assert np.array_equal(f["tc_local_id"][:128], np.arange(128))


def test_p10_block_diagonal():
    nw = 37
    M, K = 16 * nw, 8 * nw
    rows = {i: list(range(8 * (i // 16), 8 * (i // 16) + 8)) for i in range(M)}
    rp, ci = _csr_from_rows(M, rows)
    f = oracle.condense(M, rp, ci)
    assert f["num_tc_blocks"] == nw
    assert np.array_equal(f["row_window_offset"], np.arange(nw + 1))
    assert np.array_equal(np.diff(f["tc_offset"]), np.full(nw, 128))
    assert np.array_equal(f["sparse_a_to_b"], np.arange(K))


def test_p8_size_closed_form():
    rp, ci = datagen.random_csr(300, 400, 0.05, 9)
    f = oracle.condense(300, rp, ci)
    W, T, nnz = f["num_windows"], f["num_tc_blocks"], len(ci)
    index_bytes = (f["row_window_offset"].nbytes + f["tc_offset"].nbytes
                   + f["tc_local_id"].nbytes + f["sparse_a_to_b"].nbytes)
    assert index_bytes == 4 * oracle.metcf_elements(300, T, nnz)
    assert W == 19


def test_p8_tcf_formula_reproduces_paper_percentage():
    """P:127 TCF formula on Table 1 shapes vs the +168.41% printed at P:129.

    The mean of per-matrix (TCF/CSR - 1) is ~170.4%; the paper's 168.41% is
    not reproduced exactly (reading C8) -- we pin it within 2.5%."""
    g = json.load(open(os.path.join(HERE, "golden", "paper_tables.json")))
    t1 = {k: v for k, v in g["table1_matrices"].items() if not k.startswith("_")}
    pct = [100.0 * (oracle.tcf_elements(m["M"], m["nnz"]) / oracle.csr_elements(m["M"], m["nnz"]) - 1)
           for m in t1.values()]
    assert abs(np.mean(pct) - g["tcf_vs_csr_extra_pct"]["value"]) < 2.5
    # AvgRowL column = NNZ / M
    for m in t1.values():
        assert abs(m["nnz"] / m["M"] - m["avg_row_len"]) < 0.006


@pytest.mark.parametrize("M,K,density,seed", [(100, 80, 0.05, 11), (77, 300, 0.3, 12), (64, 64, 1.0, 13)])
def test_decode_round_trip_tall_windows(M, K, density, seed):
    """32-row windows (NEXT-2): ids < 256 still fit uint8, and the decode reproduces the CSR."""
    rp, ci = datagen.random_csr(M, K, density, seed)
    v = datagen.uniform(seed, 1, len(ci))
    f = oracle.condense(M, rp, ci, v, window=32)
    rows, cols, vv = decode(M, f, WH=32)
    ref_rows = np.repeat(np.arange(M), np.diff(rp))
    assert np.array_equal(rows, ref_rows) and np.array_equal(cols, ci) and np.array_equal(vv, v)
    assert f["num_windows"] == -(-M // 32) and int(f["tc_local_id"].max(initial=0)) < 256
