"""Run bench.py's multi-GPU leg (run_dist) in a 1-rank NCCL process group on one GPU: exercises the
dtc_dist_* path end to end (partition, pipelined broadcast, local kernel, C all-gather, e2e legs).
The numbers are a 1-rank smoke test, not a scaling measurement."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torch.distributed as tdist
    import bench
    from datagen import configs
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29533")
    torch.cuda.set_device(0)
    tdist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    args = argparse.Namespace(steps=5, warmup=3, no_e2e=False)
    cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "c2")
    dev = torch.device("cuda", 0)
    flush = torch.empty(bench.L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    bench.run_dist(args, cfg, cfg.N, 0, 1, 0, dev, torch.cuda.current_stream(), flush)
    tdist.destroy_process_group()


if __name__ == "__main__":
    main()
