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


def test_dist_chunks_plan():
    """The column chunks of dtc_spmm_dist (host): cover [0, N), widths multiples of 32 (but the last),
    >= 128 KB each when more than one, at most the requested count (8 max)."""
    import paper_conf_asplos_fan0024_b200 as dtc
    for K, N, elt in [(169343, 128, 4), (2449029, 512, 4), (232965, 256, 2), (100, 33, 4), (10, 1, 4), (0, 64, 4)]:
        for mx in (0, 1, 2, 4, 8):
            cb = dtc.dist_chunks(K, N, elt, mx)
            n = len(cb) - 1
            assert cb[0] == 0 and cb[-1] == N and np.all(np.diff(cb) > 0)
            assert n <= (mx if mx else 4) and n <= 8
            assert np.all(np.diff(cb)[:-1] % 32 == 0)
            if n > 1:
                assert np.all(K * np.diff(cb)[:-1] * elt >= 128 << 10)


def _chunk_worker(rank, world, port, name, out_q):
    """The chunked-broadcast schedule of dtc_spmm_dist emulated over gloo: the root sends B's column
    chunks one at a time (dtc_dist_chunks), every rank computes its row windows' C for that chunk with
    the FP64 oracle; the assembled C must equal the unsharded product bit for bit."""
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
    N = 96
    B_root = configs.make_B(cfg, N) if rank == 0 else None
    rwo, T = oracle.condense_count(cfg.M, rp, ci)
    wb = dtc.partition_windows(rwo, world)
    r0, r1 = min(16 * int(wb[rank]), cfg.M), min(16 * int(wb[rank + 1]), cfg.M)
    cb = dtc.dist_chunks(cfg.K, N, 4, 3)
    C_local = np.zeros((r1 - r0, N))
    for j in range(len(cb) - 1):
        nc = int(cb[j + 1] - cb[j])
        chunk = torch.from_numpy(np.ascontiguousarray(B_root[:, cb[j]:cb[j + 1]])) if rank == 0 \
            else torch.zeros((cfg.K, nc), dtype=torch.float32)
        dist.broadcast(chunk, src=0)
        C_local[:, cb[j]:cb[j + 1]] = oracle.spmm(cfg.M, cfg.K, rp, ci, v, chunk.numpy(), r0, r1, bound=False)
    sizes = [min(16 * int(wb[r + 1]), cfg.M) - min(16 * int(wb[r]), cfg.M) for r in range(world)]
    pad = torch.zeros((max(sizes), N), dtype=torch.float64)
    pad[: r1 - r0] = torch.from_numpy(C_local)
    gathered = [torch.zeros_like(pad) for _ in range(world)]
    dist.all_gather(gathered, pad)
    if rank == 0:
        C = np.concatenate([g[:s].numpy() for g, s in zip(gathered, sizes)])
        Cref = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B_root, bound=False)
        out_q.put((bool(np.array_equal(C, Cref)), len(cb) - 1))
    dist.barrier()
    dist.destroy_process_group()


def test_chunked_broadcast_schedule_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_chunk_worker, args=(r, 2, port, "c2", q)) for r in range(2)]
    for p in procs:
        p.start()
    equal, nch = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert equal and nch == 3
