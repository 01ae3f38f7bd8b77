"""dtc_dist_* on one GPU: NCCL path with a 1-rank communicator, and P12 (shards
built by dtc_dist_create for world = 2..4, run one after another on the same
device, concatenate to the single-GPU result)."""
import numpy as np
import pytest

import datagen
import oracle
from datagen import configs

from gpu_util import build, dev, check_tol

pytestmark = pytest.mark.gpu


def _inputs(name, N, ints=False):
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    if ints:
        v = datagen.integers(cfg.seed_a, 5, len(ci))
        B = datagen.integers(cfg.seed_b, 6, cfg.K * N).reshape(cfg.K, N)
    else:
        v = configs.make_values(cfg, len(ci))
        B = configs.make_B(cfg, N)
    return cfg, rp, ci, v, B


def test_one_rank_communicator_broadcast_and_gather():
    import torch
    from paper_conf_asplos_fan0024_b200 import Dist, nccl_unique_id
    cfg, rp, ci, v, B = _inputs("c1", 32)
    d = Dist(dev(rp), dev(ci), dev(v), cfg.M, cfg.K, "tf32", 0, 1, nccl_unique_id())
    assert (d.row_begin, d.row_end) == (0, cfg.M)
    Bd = dev(B)
    C = torch.full((cfg.M, 32), float("nan"), device="cuda")
    d.spmm(Bd, C, root=0, gather_c=True)
    torch.cuda.synchronize()
    check_tol(C.cpu().numpy(), cfg.M, cfg.K, rp, ci, v, B, "tf32")
    d.close()


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("name", ["c1", "c2"])
def test_p12_shards_concatenate(name, world):
    import torch
    from paper_conf_asplos_fan0024_b200 import Dist
    N = 64
    cfg, rp, ci, v, B = _inputs(name, N, ints=True)
    Bd = dev(B)
    parts = []
    bounds = []
    for r in range(world):
        d = Dist(dev(rp), dev(ci), dev(v), cfg.M, cfg.K, "tf32", r, world, None)
        rows = d.row_end - d.row_begin
        bounds.append((d.row_begin, d.row_end))
        Cl = torch.zeros((max(rows, 1), N), device="cuda")
        d.local_spmm(Bd, Cl)
        torch.cuda.synchronize()
        parts.append(Cl[:rows].cpu().numpy())
        d.close()
    assert bounds[0][0] == 0 and bounds[-1][1] == cfg.M
    assert all(bounds[i][1] == bounds[i + 1][0] for i in range(world - 1))
    C = np.concatenate(parts)
    f = build(cfg.M, cfg.K, rp, ci, v)
    C1 = f.spmm(Bd).cpu().numpy()
    Cref, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B)
    # integer inputs: every path is exact, so shards == single GPU == oracle
    assert np.array_equal(C.astype(np.float64), Cref)
    assert np.array_equal(C, C1)


@pytest.mark.parametrize("chunks", [0, 1, 2, 3, 8])
@pytest.mark.parametrize("dtype,N", [("tf32", 256), ("tf32", 200), ("fp16", 256), ("tf32", 33)])
def test_chunked_broadcast_bit_identical(chunks, dtype, N):
    """dtc_spmm_dist with a 1-rank communicator runs the whole pipelined path (root packs column
    chunks into the staging buffer, NCCL broadcast on the library stream, kernel per chunk): C
    must equal one dtc_spmm over all N columns bit for bit, gathered or not."""
    import torch
    from paper_conf_asplos_fan0024_b200 import Dist, nccl_unique_id
    cfg = configs.get("c2")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    d = Dist(dev(rp), dev(ci), dev(v), cfg.M, cfg.K, dtype, 0, 1, nccl_unique_id())
    d.set_chunks(chunks)
    Bd = dev(B)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype)
    C1 = f.spmm(Bd)
    for gather in (True, False):
        C = torch.full((cfg.M, N), float("nan"), device="cuda")
        d.spmm(Bd, C, root=0, gather_c=gather)
        d.spmm(Bd, C, root=0, gather_c=gather)   # staging buffer reuse
        torch.cuda.synchronize()
        assert torch.equal(C, C1)
    d.close()


def test_dist_partition_from_counts_matches_format():
    """dtc_dist_create partitions by the F0-F2 window counts: the same boundaries dtc_partition_windows
    gives on the full format's RowWindowOffset."""
    from paper_conf_asplos_fan0024_b200 import Dist, partition_windows
    cfg = configs.get("c2")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    rwo = build(cfg.M, cfg.K, rp, ci, v).export()["row_window_offset"]
    for world in (2, 3, 5, 8):
        wb = partition_windows(rwo, world)
        for r in range(world):
            d = Dist(dev(rp), dev(ci), dev(v), cfg.M, cfg.K, "tf32", r, world, None)
            assert (d.row_begin, d.row_end) == (min(16 * int(wb[r]), cfg.M), min(16 * int(wb[r + 1]), cfg.M))
            d.close()
