"""TCA reordering (NEXT-1, Alg. 1): native implementation vs the
step-by-step Python oracle (exact permutation equality), and pins of the oracle."""
import numpy as np
import pytest

import datagen
import oracle
from oracle import tca as otca
import paper_conf_asplos_fan0024_b200 as dtc
from datagen import configs


def _shuffle_rows(M, rp, ci, seed):
    perm = np.random.default_rng(seed).permutation(M)
    deg = np.diff(rp)[perm]
    nrp = np.zeros(M + 1, np.int32)
    nrp[1:] = np.cumsum(deg)
    nci = np.concatenate([ci[rp[r]:rp[r + 1]] for r in perm]).astype(np.int32) if M else ci
    return nrp, nci


def _permute(rp, ci, perm):
    deg = np.diff(rp)[perm]
    nrp = np.zeros(len(perm) + 1, np.int32)
    nrp[1:] = np.cumsum(deg)
    nci = np.concatenate([ci[rp[r]:rp[r + 1]] for r in perm]).astype(np.int32)
    return nrp, nci


@pytest.mark.parametrize("M,K,density,seed", [(100, 60, 0.1, 3), (500, 300, 0.02, 4), (64, 64, 0.3, 5),
                                              (257, 1000, 0.01, 6), (40, 8, 0.5, 7), (1, 1, 1.0, 8)])
def test_native_matches_oracle_exactly(M, K, density, seed):
    rp, ci = datagen.random_csr(M, K, density, seed)
    p_native = dtc.tca_reorder(M, K, rp, ci)
    p_oracle = otca.tca_reorder(M, rp, ci)
    assert list(p_native) == p_oracle
    assert sorted(p_oracle) == list(range(M))


@pytest.mark.parametrize("sm_num", [1, 4, 148])
def test_native_matches_oracle_structured(sm_num):
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    srp, sci = _shuffle_rows(cfg.M, rp, ci, 11)
    assert list(dtc.tca_reorder(cfg.M, cfg.K, srp, sci, sm_num)) == otca.tca_reorder(cfg.M, srp, sci, sm_num)


def test_oracle_restores_shuffled_block_diagonal():
    """Pin: 16-row groups of identical rows (dense 16x8 blocks), rows shuffled.  Jaccard is 1
    inside a group and 0 across groups, so Hierarchy I must rebuild exactly the groups and
    Reid must put each group in one window: one TC block per window, MeanNnzTC = 128 (P9/P10)."""
    nw = 20
    M, K = 16 * nw, 8 * nw
    rp = (np.arange(M + 1) * 8).astype(np.int32)
    ci = np.concatenate([np.arange(8 * (i // 16), 8 * (i // 16) + 8) for i in range(M)]).astype(np.int32)
    srp, sci = _shuffle_rows(M, rp, ci, 3)
    f0 = oracle.condense(M, srp, sci)
    assert f0["num_tc_blocks"] > nw
    perm = np.array(otca.tca_reorder(M, srp, sci))
    prp, pci = _permute(srp, sci, perm)
    f = oracle.condense(M, prp, pci)
    assert f["num_tc_blocks"] == nw
    assert np.array_equal(np.diff(f["tc_offset"]), np.full(nw, 128))


def test_oracle_hierarchy_limits():
    """Row clusters never exceed 2*16-1 rows and Hierarchy I merges only similar rows."""
    rp, ci = datagen.random_csr(300, 120, 0.05, 9)
    rows = [[int(c) for c in ci[rp[i]:rp[i + 1]]] for i in range(300)]
    rc = otca.merge(300, otca.priority_queue(otca.minhash_lsh(rows)), otca.BLOCK_HEIGHT)
    assert sorted(x for c in rc for x in c) == list(range(300))
    assert max(len(c) for c in rc) <= 2 * otca.BLOCK_HEIGHT - 1
    # every multi-row cluster is connected by pairs with J > 0
    for c in rc:
        if len(c) > 1:
            assert any(set(rows[a]) & set(rows[b]) for a in c for b in c if a < b)


def test_tca_raises_mean_nnz_tc_on_shuffled_graph():
    """The point of Hierarchy I: on a row-shuffled community graph TCA recovers
    dense TC blocks (MeanNnzTC up, NumTCBlocks down)."""
    cfg = configs.get("c2")
    rp, ci = configs.make_pattern(cfg)
    srp, sci = _shuffle_rows(cfg.M, rp, ci, 5)
    _, T_shuf = oracle.condense_count(cfg.M, srp, sci)
    perm = dtc.tca_reorder(cfg.M, cfg.K, srp, sci)
    prp, pci = _permute(srp, sci, perm)
    _, T_tca = oracle.condense_count(cfg.M, prp, pci)
    assert T_tca < 0.8 * T_shuf


def _permuted(rp, ci, perm):
    rows = [ci[rp[r]:rp[r + 1]] for r in perm]
    rp2 = np.concatenate([[0], np.cumsum([len(x) for x in rows])]).astype(np.int32)
    return rp2, (np.concatenate(rows) if rows else np.zeros(0, np.int32)).astype(np.int32)


@pytest.mark.parametrize("name", ["c1", "c4small", "shuffled"])
def test_tca_checked_keeps_identity_unless_T_drops(name):
    """dtc_tca_reorder_checked: the T counts equal O2's NumTCBlock (oracle.condense_count) of the two
    row orders, and the TCA order is applied exactly when it lowers T (else the identity)."""
    import oracle
    if name == "c1":
        cfg = configs.get("c1")
        rp, ci = configs.make_pattern(cfg)
        M, K = cfg.M, cfg.K
    elif name == "c4small":   # banded: already in its best order, TCA cannot lower T
        M = K = 4000
        rows = [sorted(set(range(max(0, i - 3), min(K, i + 4)))) for i in range(M)]
        rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int32)
        ci = np.concatenate(rows).astype(np.int32)
    else:                     # shuffled block diagonal (16-row blocks of 8 columns): TCA restores them
        nb = 64
        rows = [list(range(8 * (i // 16), 8 * (i // 16) + 8)) for i in range(16 * nb)]
        rp0 = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int32)
        ci0 = np.concatenate(rows).astype(np.int32)
        M, K = 16 * nb, 8 * nb
        rp, ci = _shuffle_rows(M, rp0, ci0, 5)
    perm, info = dtc.tca_reorder_checked(M, K, rp, ci, 148)
    raw = dtc.tca_reorder(M, K, rp, ci, 148)
    _, t0 = oracle.condense_count(M, rp, ci)
    rpp, cip = _permuted(rp, ci, raw)
    _, t1 = oracle.condense_count(M, rpp, cip)
    assert (info["T_identity"], info["T_reordered"]) == (t0, t1)
    assert info["applied"] == (t1 < t0)
    assert np.array_equal(perm, raw if t1 < t0 else np.arange(M, dtype=np.int32))
    if name == "c4small":
        assert not info["applied"]
    if name == "shuffled":
        assert info["applied"]
