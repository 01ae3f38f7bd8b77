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


def build(M, K, rp, ci, v, dtype="tf32", **kw):
    from paper_conf_asplos_fan0024_b200 import Format
    vv = v.astype(np.float16) if dtype == "fp16" else v.astype(np.float32)
    return Format.build(dev(rp.astype(np.int32)), dev(ci.astype(np.int32)), dev(vv), M, K, dtype=dtype, **kw)


def assert_format_equal(got: dict, ref: dict):
    assert got["num_tc_blocks"] == ref["num_tc_blocks"]
    for k in ("row_window_offset", "tc_offset", "tc_local_id", "sparse_a_to_b"):
        assert np.array_equal(got[k], ref[k]), k
    g, r = got["tc_values"], ref["tc_values"]
    assert g.dtype.itemsize == r.dtype.itemsize
    assert np.array_equal(g.view(np.uint8), r.view(np.uint8)), "tc_values"


def check_units(f: dict, M: int):
    """Every TC block is covered by exactly one unit; every window's rows by one
    non-split unit or by the pieces of its split."""
    units, rwo = f["units"], f["row_window_offset"]
    W, T = len(rwo) - 1, f["num_tc_blocks"]
    covered = np.zeros(T, dtype=np.int64)
    wcov = np.zeros(W, dtype=np.int64)
    for wb, we, bb, be, sid, piece, npc, slot in units:
        assert 0 <= bb <= be <= T
        covered[bb:be] += 1
        if sid < 0:
            assert rwo[wb] == bb and rwo[we] == be
            wcov[wb:we] += 1
        else:
            assert we == wb + 1 and rwo[wb] <= bb and be <= rwo[we]
            if piece == 0:
                wcov[wb] += 1
    assert np.all(covered == 1)
    assert np.all(wcov == 1)


def spmm(fmt, B, N=None):
    import torch
    Bt = dev(B)
    C = fmt.spmm(Bt)
    torch.cuda.synchronize()
    return C.cpu().numpy()


def check_tol(Cg, M, K, rp, ci, v, B, dtype, r0=0, r1=None):
    Cr, Bd = oracle.spmm(M, K, rp, ci, v.astype(np.float32), B.astype(np.float32), r0=r0, r1=r1)
    ok, ratio = oracle.within_tolerance(Cg, Cr, Bd, TOL[dtype])
    assert ok, f"tolerance violated: max err/limit = {ratio:.3g}"
    return ratio
