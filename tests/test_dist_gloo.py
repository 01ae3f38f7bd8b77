"""Multi-process (world_size 2, gloo, CPU) test of the row-window sharding plumbing.

Each rank computes the window partition with the library's host partitioner
(dtc_partition_windows, the same function dtc_dist_create uses), computes its
C rows with the FP64 oracle, and the shards are all-gathered over gloo; the
concatenation must equal the unsharded result bit-exactly.
No GPU is used: this pins the host-side logic the NCCL path relies on.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch
    import torch.distributed as dist

    import oracle
    import paper_conf_asplos_fan0024_b200 as dtc
    from datagen import configs

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    N = 16
    B = configs.make_B(cfg, N)
    rwo, T = oracle.condense_count(cfg.M, rp, ci)
    wb = dtc.partition_windows(rwo, world)
    r0, r1 = min(16 * int(wb[rank]), cfg.M), min(16 * int(wb[rank + 1]), cfg.M)
    C_local, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B, r0, r1)
    # variable-size all-gather over gloo: pad to the largest shard
    sizes = [min(16 * int(wb[r + 1]), cfg.M) - min(16 * int(wb[r]), cfg.M) for r in range(world)]
    mx = max(sizes)
    pad = torch.zeros((mx, N), dtype=torch.float64)
    pad[: r1 - r0] = torch.from_numpy(C_local)
    gathered = [torch.zeros_like(pad) for _ in range(world)]
    dist.all_gather(gathered, pad)
    if rank == 0:
        C = np.concatenate([g[:s].numpy() for g, s in zip(gathered, sizes)])
        Cref, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B)
        blocks = [int(rwo[wb[r + 1]] - rwo[wb[r]]) for r in range(world)]
        out_q.put((bool(np.array_equal(C, Cref)), sizes, blocks, int(T)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,world", [("c1", 2), ("c2", 2)])
def test_sharded_oracle_matches_unsharded(name, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    equal, sizes, blocks, T = res
    assert equal
    assert sum(sizes) > 0 and sum(blocks) == T
    # TC-block balance: no rank more than one window's worth above T/world
    assert max(blocks) <= T / world + 2048
