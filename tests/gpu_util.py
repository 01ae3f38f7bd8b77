"""Shared helpers for the -m gpu parity tests (test infrastructure)."""
import numpy as np

import oracle

TOL = oracle.TOL


def dev(a, dtype=None):
    import torch
    t = torch.from_numpy(np.ascontiguousarray(a))
    if dtype is not None:
        t = t.to(dtype)
    return t.cuda()


def build(M, K, rp, ci, v, dtype="tf32", options=None, **kw):
    """Format.build through the C ABI; `options` = per-handle launch options (dtc_format_set_option)."""
    from paper_conf_asplos_fan0024_b200 import Format
    vv = v.astype(np.float16) if dtype == "fp16" else v.astype(np.float32)
    f = Format.build(dev(rp.astype(np.int32)), dev(ci.astype(np.int32)), dev(vv), M, K, dtype=dtype, **kw)
    for k, x in (options or {}).items():
        f.set_option(k, x)
    return f


def assert_format_equal(got: dict, ref: dict):
    assert got["num_tc_blocks"] == ref["num_tc_blocks"]
    for k in ("row_window_offset", "tc_offset", "tc_local_id", "sparse_a_to_b"):
        assert np.array_equal(got[k], ref[k]), k
    g, r = got["tc_values"], ref["tc_values"]
    assert g.dtype.itemsize == r.dtype.itemsize
    assert np.array_equal(g.view(np.uint8), r.view(np.uint8)), "tc_values"


def check_units(f: dict, M: int):
    """F4 schedule invariants (vectorised, any size): every TC block is covered by exactly one
    unit; every window's rows by one non-split unit or by the pieces of its split, whose pieces
    have distinct workspace slots and consistent piece counts."""
    units, rwo = np.asarray(f["units"], dtype=np.int64), np.asarray(f["row_window_offset"], dtype=np.int64)
    W, T = len(rwo) - 1, int(f["num_tc_blocks"])
    if len(units) == 0:
        assert T == 0
        return
    wb, we, bb, be, sid, piece, npc, slot = units.T
    assert np.all((0 <= bb) & (bb <= be) & (be <= T))
    assert np.all((0 <= wb) & (wb <= we) & (we <= W))
    cov = np.zeros(T + 1, np.int64)
    np.add.at(cov, bb, 1)
    np.add.at(cov, be, -1)
    assert np.all(np.cumsum(cov)[:T] == 1), "TC blocks not covered exactly once"
    whole = sid < 0
    assert np.all(rwo[wb[whole]] == bb[whole]) and np.all(rwo[we[whole]] == be[whole])
    wcov = np.zeros(W + 1, np.int64)
    np.add.at(wcov, wb[whole], 1)
    np.add.at(wcov, we[whole], -1)
    wcov = np.cumsum(wcov)[:W]
    sp = ~whole
    assert np.all(we[sp] == wb[sp] + 1) and np.all(rwo[wb[sp]] <= bb[sp]) and np.all(be[sp] <= rwo[we[sp]])
    assert np.all((0 <= piece[sp]) & (piece[sp] < npc[sp]))
    np.add.at(wcov, wb[sp & (piece == 0)], 1)
    assert np.all(wcov == 1), "windows not covered exactly once"
    slots = slot[sp] + piece[sp]
    assert len(np.unique(slots)) == len(slots), "split pieces share a workspace slot"
    # every piece of a split window agrees on npieces and slot_base, and all pieces are present
    order = np.lexsort((piece[sp], wb[sp]))
    w_s, p_s, n_s, b_s = wb[sp][order], piece[sp][order], npc[sp][order], slot[sp][order]
    if len(w_s):
        first = np.r_[True, w_s[1:] != w_s[:-1]]
        grp = np.cumsum(first) - 1
        assert np.all(n_s == n_s[first][grp]) and np.all(b_s == b_s[first][grp])
        assert np.all(p_s == np.arange(len(p_s)) - np.flatnonzero(first)[grp])
        assert np.all(np.bincount(grp) == n_s[first])


def spmm(fmt, B, N=None):
    import torch
    Bt = dev(B)
    C = fmt.spmm(Bt)
    torch.cuda.synchronize()
    return C.cpu().numpy()


def compare_chunked(C, M, K, rp, ci, v, B, dtype=None, exact=False, chunk=65536):
    """Every element of C against oracle O1, 64k rows at a time: within the
    north_star tolerance (returns the worst err/limit) or, with exact=True, bit for bit (returns 0)."""
    vf = v.astype(np.float32, copy=False)
    Bf = B.astype(np.float32, copy=False)
    worst = 0.0
    for r0 in range(0, M, chunk):
        r1 = min(M, r0 + chunk)
        if exact:
            Cr = oracle.spmm(M, K, rp, ci, vf, Bf, r0=r0, r1=r1, bound=False)
            bad = np.flatnonzero((C[r0:r1].astype(np.float64) != Cr).any(axis=1))
            assert bad.size == 0, f"rows {r0 + bad[:5]} differ from O1"
        else:
            Cr, Bd = oracle.spmm(M, K, rp, ci, vf, Bf, r0=r0, r1=r1)
            ok, ratio = oracle.within_tolerance(C[r0:r1], Cr, Bd, TOL[dtype])
            assert ok, f"rows [{r0},{r1}): max err/limit {ratio:.3g}"
            worst = max(worst, ratio)
    return worst


def check_tol(Cg, M, K, rp, ci, v, B, dtype, r0=0, r1=None):
    Cr, Bd = oracle.spmm(M, K, rp, ci, v.astype(np.float32), B.astype(np.float32), r0=r0, r1=r1)
    ok, ratio = oracle.within_tolerance(Cg, Cr, Bd, TOL[dtype])
    assert ok, f"tolerance violated: max err/limit = {ratio:.3g}"
    return ratio
