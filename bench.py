#!/usr/bin/env python
"""bench.py -- SpMM GFLOP/s (2*nnz*N/t) of the DTC-SpMM hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--n N] [--impl dtc|reference]

One step = one pass of the whole hot path (dtc_spmm: S1-S5) over the config's
synthetic matrix (the ME-TCF format is built once beforehand, as the paper
converts once and reuses A; its build time is reported as
format_build_ms).  Timing: CUDA events on the launching stream around each step,
L2 flushed (256 MiB memset, outside the events) between steps, W warm-up steps,
barrier + synchronize on both sides, max over ranks.  Rank 0 prints ONE JSON line.

--impl reference times the FP64 CPU oracle (the only reference this tier has) on
the host cores on bounded samples of the same workload.
Under torchrun (N > 1) the row windows are partitioned across ranks
(dtc_spmm_dist); value = whole-job GFLOP/s with B resident on every GPU, e2e adds
the NCCL broadcast of B from the root's pinned host copy and the C readback.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMM GFLOP/s (2*nnz*N/t)"
UNIT = "GFLOP/s"
L2_FLUSH_BYTES = 256 << 20


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=200)
    p.add_argument("--warmup", type=int, default=10)
    p.add_argument("--impl", default="dtc", choices=["dtc", "reference"])
    p.add_argument("--config", default="c2")
    p.add_argument("--n", type=int, default=0, help="override N (columns of B)")
    p.add_argument("--unit-blocks", type=int, default=0)
    p.add_argument("--guided", type=int, default=0, help="F4 guided tail (1 on, -1 off, 0 auto)")
    p.add_argument("--no-cusparse", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--minimal", action="store_true", help="only the timed dtc loop (for ncu launch lists)")
    p.add_argument("--tca", type=int, default=-1,
                   help="also time the SpMM on the TCA-reordered matrix (NEXT-1, dtc_tca_reorder + row_perm; "
                        "C still in the original order): 1 on, 0 off, -1 on when nnz < 10M")
    p.add_argument("--graphconv", type=int, default=-1,
                   help="also time one GraphConv layer (dtc_graphconv, NEXT-3) with F_in=N and this F_out "
                        "(-1: F_out=N; 0: off)")
    return p.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """NVML sampling of SM clock and throttle reasons DURING the timed region."""
    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x2: "applications_clocks_setting",
               0x1: "gpu_idle"}

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self._nv = None

    def _run(self):
        nv = self._nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                self.reasons |= nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self._nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._nv:
            self._t.join()

    def summary(self):
        if not self._nv:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"], "samples": 0}
        names = [n for bit, n in self.REASONS.items() if self.reasons & bit and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


# ------------------------------------------------------------------ workload
def load_workload(cfg, N):
    from datagen import configs
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    return rp, ci, v, B


def algorithmic_bytes(exp: dict, M: int, N: int, elt: int):
    """per TC block 4 (TCOffset) + 32 (SparseAtoB) + nnz_t*(1+elt)
    + u_t*N*elt (gathered B rows); per window 4 (RowWindowOffset) + rows*N*4 (C)."""
    T, W = exp["num_tc_blocks"], exp["num_windows"]
    nnz = len(exp["tc_local_id"])
    atob = exp["sparse_a_to_b"]
    sum_u = int(np.count_nonzero(atob >= 0))
    fmt = 4 * (T + 1) + 32 * T + nnz * (1 + elt) + 4 * (W + 1)
    literal = fmt + sum_u * N * elt + M * N * 4
    distinct_rows = int(np.unique(atob[atob >= 0]).size)
    compulsory = fmt + distinct_rows * N * elt + M * N * 4
    return literal, compulsory, sum_u


def time_loop(fn, steps, warmup, stream, flush_buf=None):
    import torch
    for _ in range(warmup):
        if flush_buf is not None:
            flush_buf.zero_()
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for a, b in ev:
        if flush_buf is not None:
            flush_buf.zero_()
        a.record(stream)
        fn()
        b.record(stream)
    torch.cuda.synchronize()
    return [a.elapsed_time(b) for a, b in ev]


def traffic_from_profiles(name, N):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(f"{name}_N{N}")
    except Exception:
        return None


def cpu_baseline(cfg, rp, ci, v, B, N, budget_s=10.0):
    """The oracle as it stands, timed on the host cores on a bounded sample."""
    import oracle
    cores = oracle.max_threads()
    M, K = cfg.M, cfg.K
    vf = v.astype(np.float32)
    Bf = B.astype(np.float32) if B.dtype != np.float32 else B
    # probe on a small row block to size the sample
    r_probe = min(M, 4096)
    t0 = time.perf_counter()
    oracle.spmm(M, K, rp, ci, vf, Bf, 0, r_probe, bound=False)
    dt = max(time.perf_counter() - t0, 1e-4)
    nnz_probe = int(rp[r_probe])
    rate = max(nnz_probe, 1) / dt                     # nnz per second
    full_s = len(ci) / rate
    if full_s <= budget_s:
        r1, reps = M, max(1, int(budget_s / max(full_s, 1e-4)))
        reps = min(reps, 2000)
    else:
        target_nnz = rate * budget_s
        r1 = int(np.searchsorted(rp, target_nnz))
        r1 = max(1, min(M, r1))
        reps = 1
    t0 = time.perf_counter()
    done = 0
    while True:   # at least `reps`, and at least budget_s of CPU work
        oracle.spmm(M, K, rp, ci, vf, Bf, 0, r1, bound=False)
        done += 1
        el = time.perf_counter() - t0
        if done >= reps and el >= 0.8 * budget_s:
            break
    reps = done
    nnz_s = int(rp[r1])
    gflops = 2.0 * nnz_s * N * reps / el / 1e9
    return {"value": round(gflops, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"rows [0,{r1}) of {M} ({nnz_s} of {len(ci)} nnz), N={N}, FP64 C only, "
                      f"x{reps} reps, {el:.1f} s, OpenMP {cores} threads"}


# ------------------------------------------------------------------ dtc arm
def run_dtc(args, cfg, N, rank, world, local_rank):
    import torch
    import paper_conf_asplos_fan0024_b200 as dtc

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    stream = torch.cuda.current_stream()
    rp, ci, v, B = load_workload(cfg, N)
    M, K, nnz = cfg.M, cfg.K, len(ci)
    elt = 2 if cfg.dtype == "fp16" else 4
    rp_d = torch.from_numpy(rp).to(dev)
    ci_d = torch.from_numpy(ci).to(dev)
    v_d = torch.from_numpy(v).to(dev)
    B_d = torch.from_numpy(B).to(dev)
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    flops = 2.0 * nnz * N

    if world == 1:
        # format build (F0-F4): first call (includes one-time module/pool setup) and a warm rebuild
        build_ms_runs = []
        for _ in range(2):
            torch.cuda.synchronize()
            tb0 = time.perf_counter()
            fmt = dtc.Format.build(rp_d, ci_d, v_d, M, K, dtype=cfg.dtype, unit_blocks=args.unit_blocks,
                                   guided=args.guided)
            torch.cuda.synchronize()
            build_ms_runs.append((time.perf_counter() - tb0) * 1e3)
        build_ms = build_ms_runs[-1]
        C_d = torch.empty((M, N), dtype=torch.float32, device=dev)
        fn = lambda: fmt.spmm(B_d, C_d)  # noqa: E731
        T = fmt.num_tc_blocks
    else:
        import torch.distributed as tdist
        uid = [dtc.nccl_unique_id() if rank == 0 else None]
        tdist.broadcast_object_list(uid, src=0)
        torch.cuda.synchronize()
        tb0 = time.perf_counter()
        dd = dtc.Dist(rp_d, ci_d, v_d, M, K, cfg.dtype, rank, world, uid[0])
        torch.cuda.synchronize()
        build_ms = (time.perf_counter() - tb0) * 1e3
        rows = dd.row_end - dd.row_begin
        C_d = torch.empty((max(rows, 1), N), dtype=torch.float32, device=dev)
        # kernel-only step: B resident on every rank, local row windows only
        fn = lambda: dd.local_spmm(B_d, C_d)  # noqa: E731
        T = None

    if world > 1:
        import torch.distributed as tdist
        tdist.barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local_rank)
    with sampler:
        t_wall0 = time.perf_counter()
        ms = time_loop(fn, args.steps, args.warmup, stream, flush)
        t_wall = time.perf_counter() - t_wall0
    if world > 1:
        tdist.barrier()
    torch.cuda.synchronize()
    total_ms = float(sum(ms))
    if world > 1:
        t = torch.tensor([total_ms], device=dev)
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = flops / (ms_per_step * 1e-3) / 1e9

    if args.minimal:
        if rank == 0:
            print(json.dumps({"metric": METRIC, "value": round(value, 2), "unit": UNIT, "ms_per_step": ms_per_step,
                              "minimal": True, "config": {"workload": cfg.name, "N": N}}))
        return

    out = {"metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms_per_step, 5), "higher_is_better": True,
           "scaling": "strong" if world > 1 else "weak", "vs_baseline": None,
           "dtype": cfg.dtype, "data": "synthetic (seeded generators, datagen/; DESIGN.md §3)"}
    cfgd = {"workload": f"{cfg.name}: {cfg.desc}", "M": M, "K": K, "nnz": nnz, "N": N,
            "parallelism": f"row-window dp{world}", "l2": "flushed between steps (256 MiB memset outside the events)",
            "timing": "CUDA events per step on the launching stream; sum over steps; max over ranks"}
    hbm, peak_src = peaks()
    if world == 1:
        exp = fmt.export()
        lit, comp, sum_u = algorithmic_bytes(exp, M, N, elt)
        cfgd.update({"num_tc_blocks": T, "mean_nnz_tc": round(nnz / max(T, 1), 3), "sum_u": sum_u,
                     "unit_blocks": fmt.unit_blocks, "num_units": fmt.num_units,
                     "split_windows": fmt.num_split_windows})
        # the paper's Selector, as a diagnostic: AR of one-CTA-per-window
        sel = dtc.selector_ar(exp["row_window_offset"], torch.cuda.get_device_properties(0).multi_processor_count, 6)
        cfgd["selector"] = {"ar": round(sel["ar"], 3), "occupancy": 6, "balanced_by_paper_rule": sel["ar"] > 1.2}
        kern_ms = statistics.mean(ms)
        achieved = lit / (kern_ms * 1e-3) / 1e9
        out["roofline"] = {"bound": "hbm", "achieved": round(achieved, 1), "peak": hbm, "unit": "GB/s",
                           "frac": round(achieved / hbm, 4), "traffic": traffic_from_profiles(cfg.name, N),
                           "peak_source": peak_src,
                           "bytes_per_launch": lit,
                           "bytes_def": "literal algorithmic bytes, SURVEY §8(d): format + sum_t u_t*N*elt + M*N*4",
                           "compulsory_bytes_per_launch": comp,
                           "compulsory_frac": round(comp / (kern_ms * 1e-3) / 1e9 / hbm, 4),
                           "kernel": "k_spmm (dtc_spmm)", "kernel_ms_mean": round(kern_ms, 5),
                           "kernel_ms_median": round(statistics.median(ms), 5)}
        out["format_build_ms"] = round(build_ms, 3)
        out["format_build_first_call_ms"] = round(build_ms_runs[0], 3)
        out["format_build_x_spmm"] = round(build_ms / kern_ms, 2)
    out["config"] = cfgd
    out["gpu_launches"] = args.steps * dtc.launches_per_call()
    out["clocks"] = sampler.summary()
    out["wall_s_timed_region"] = round(t_wall, 4)

    # ---- e2e through the public API with HOST buffers (pinned), 1 GPU
    if not args.no_e2e and world == 1:
        Bh = torch.from_numpy(B).pin_memory()
        Ch = torch.empty((M, N), dtype=torch.float32).pin_memory()
        for _ in range(max(1, args.warmup // 2)):
            fmt.spmm_host(Bh, Ch)
        e2e_steps = max(3, min(args.steps, 20))
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            fmt.spmm_host(Bh, Ch)
        e2e_s = (time.perf_counter() - t0) / e2e_steps
        out["e2e"] = {"value": round(flops / e2e_s / 1e9, 2), "unit": UNIT,
                      "h2d_bytes_per_step": int(B.nbytes), "d2h_bytes_per_step": int(M * N * 4),
                      "ms_per_step": round(e2e_s * 1e3, 4), "api": "dtc_spmm_host (pinned host B and C; column-chunk copy pipeline)",
                      "steps": e2e_steps}
        # parity spot check of the timed result (sampled, oracle lives in tests; here a cheap self-check)
        out["e2e_matches_device"] = bool(torch.equal(Ch, C_d.cpu()))

    # ---- e2e at N > 1: root copies B from pinned host memory, dtc_spmm_dist broadcasts it over
    # NCCL and runs the local row windows, every rank reads its C rows back; max over ranks
    if not args.no_e2e and world > 1:
        import torch.distributed as tdist
        Bh = torch.from_numpy(B).pin_memory() if rank == 0 else None
        Ch = torch.empty(tuple(C_d.shape), dtype=torch.float32).pin_memory()

        def e2e_step():
            if rank == 0:
                B_d.copy_(Bh, non_blocking=True)
            dd.spmm(B_d, C_d, root=0, gather_c=False)
            Ch.copy_(C_d, non_blocking=True)
            torch.cuda.synchronize()

        for _ in range(2):
            e2e_step()
        tdist.barrier()
        e2e_steps = max(3, min(args.steps, 20))
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        el = torch.tensor([(time.perf_counter() - t0) / e2e_steps], device=dev)
        tdist.all_reduce(el, op=tdist.ReduceOp.MAX)
        e2e_s = float(el.item())
        out["e2e"] = {"value": round(flops / e2e_s / 1e9, 2), "unit": UNIT,
                      "h2d_bytes_per_step": int(B.nbytes), "d2h_bytes_per_step": int(M * N * 4),
                      "ms_per_step": round(e2e_s * 1e3, 4),
                      "api": "dtc_spmm_dist (root H2D of B, NCCL broadcast, local kernel, per-rank C D2H)",
                      "steps": e2e_steps}
        out["format_build_ms"] = round(build_ms, 3)

    # ---- TCA reordering (NEXT-1, Alg. 1): host preprocessing, then the same kernel on
    # the permuted ME-TCF (rows permuted inside the library, C written in the original row order)
    if (args.tca == 1 or (args.tca < 0 and nnz < 10_000_000)) and world == 1 and not args.minimal:
        try:
            t0 = time.perf_counter()
            perm = dtc.tca_reorder(M, K, rp, ci, torch.cuda.get_device_properties(dev).multi_processor_count)
            reorder_s = time.perf_counter() - t0
            perm_d = torch.from_numpy(perm).to(dev)
            fmt_t = dtc.Format.build(rp_d, ci_d, v_d, M, K, dtype=cfg.dtype, unit_blocks=args.unit_blocks,
                                     guided=args.guided, row_perm=perm_d)
            C_t = torch.empty((M, N), dtype=torch.float32, device=dev)
            ms_t = time_loop(lambda: fmt_t.spmm(B_d, C_t), max(10, min(args.steps, 100)), 3, stream, flush)
            tms = statistics.mean(ms_t)
            out["tca"] = {"value": round(flops / (tms * 1e-3) / 1e9, 2), "unit": UNIT, "ms_per_step": round(tms, 5),
                          "num_tc_blocks": fmt_t.num_tc_blocks, "mean_nnz_tc": round(nnz / max(fmt_t.num_tc_blocks, 1), 3),
                          "reorder_host_s": round(reorder_s, 3), "speedup_vs_unordered": round(kern_ms / tms, 3),
                          "matches_unordered": bool(torch.allclose(C_t, C_d, rtol=1e-2, atol=1e-2))}
            fmt_t.close()
        except Exception as e:  # noqa: BLE001
            out["tca"] = {"error": str(e)}

    # ---- GraphConv layer (NEXT-3, Eq. (2)): (A x H) x W + b, ReLU, with H = B
    if args.graphconv != 0 and world == 1 and not args.minimal:
        try:
            F_out = N if args.graphconv < 0 else args.graphconv
            Wg = torch.empty((N, F_out), dtype=torch.float32, device=dev).uniform_(-0.1, 0.1)
            bg = torch.empty((F_out,), dtype=torch.float32, device=dev).uniform_(-0.1, 0.1)
            AH = torch.empty((M, N), dtype=torch.float32, device=dev)
            Yg = torch.empty((M, F_out), dtype=torch.float32, device=dev)
            gsteps = max(5, min(args.steps, 50))
            ms_g = time_loop(lambda: fmt.graphconv(B_d, Wg, bg, relu=True, AH=AH, Y=Yg), gsteps, 3, stream, flush)
            gms = statistics.mean(ms_g)
            out["graphconv"] = {"F_in": N, "F_out": F_out, "ms": round(gms, 5), "spmm_ms": round(kern_ms, 5),
                                "dense_ms": round(gms - kern_ms, 5),
                                "gflops_total": round((flops + 2.0 * M * N * F_out) / (gms * 1e-3) / 1e9, 1),
                                "steps": gsteps, "api": "dtc_graphconv (DTC-SpMM + cuBLASLt TF32 bias/ReLU epilogue)"}
        except Exception as e:  # noqa: BLE001
            out["graphconv"] = {"error": str(e)}

    # ---- cuSPARSE on the same box (comparison system)
    if not args.no_cusparse and world == 1:
        try:
            from tools.cusparse_ref import CuSparseSpMM
            res = {}
            C2 = torch.empty((M, N), dtype=torch.float32, device=dev)
            for alg in ("ALG_DEFAULT", "CSR_ALG1", "CSR_ALG2", "CSR_ALG3"):
                cs = CuSparseSpMM(M, K, rp_d, ci_d, v_d, B_d, C2, alg)
                if not cs.ok:
                    res[alg] = f"unsupported (status {cs.status})"
                    continue
                try:
                    ms2 = time_loop(cs.run, max(5, args.steps // 4), 3, stream, flush)
                    res[alg] = round(flops / (statistics.mean(ms2) * 1e-3) / 1e9, 2)
                except Exception as e:  # noqa: BLE001
                    res[alg] = f"error: {e}"
                cs.close()
            nums = {k: x for k, x in res.items() if isinstance(x, float)}
            out["cusparse"] = {"gflops": res, "best": max(nums.values()) if nums else None,
                               "speedup_vs_default": round(value / nums["ALG_DEFAULT"], 3)
                               if "ALG_DEFAULT" in nums else None,
                               "speedup_vs_best": round(value / max(nums.values()), 3) if nums else None}
        except Exception as e:  # noqa: BLE001
            out["cusparse"] = {"error": str(e)}

    if not args.no_cpu and rank == 0 and world == 1:
        out["cpu_baseline"] = cpu_baseline(cfg, rp, ci, v, B, N)
    if rank == 0:
        print(json.dumps(out))


# ------------------------------------------------------------------ reference arm
def run_reference(args, cfg, N, rank, world):
    if rank != 0:
        return
    import oracle
    rp, ci, v, B = load_workload(cfg, N)
    vf = v.astype(np.float32)
    Bf = B.astype(np.float32)
    M, K = cfg.M, cfg.K
    cores = oracle.max_threads()
    # size one step to ~1 s of CPU work (the whole workload if it is shorter)
    r_probe = min(M, 4096)
    t0 = time.perf_counter()
    oracle.spmm(M, K, rp, ci, vf, Bf, 0, r_probe, bound=False)
    rate = max(int(rp[r_probe]), 1) / max(time.perf_counter() - t0, 1e-4)
    r1 = M if len(ci) / rate <= 1.0 else max(1, int(np.searchsorted(rp, rate * 1.0)))
    nnz_s = int(rp[r1])
    for _ in range(args.warmup):
        oracle.spmm(M, K, rp, ci, vf, Bf, 0, r1, bound=False)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.spmm(M, K, rp, ci, vf, Bf, 0, r1, bound=False)
    el = time.perf_counter() - t0
    ms = el / args.steps * 1e3
    value = 2.0 * nnz_s * N / (ms * 1e-3) / 1e9
    sample = f"rows [0,{r1}) of {M} ({nnz_s} of {len(ci)} nnz) per step, N={N}, FP64, OpenMP {cores} threads"
    out = {"metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded generators, datagen/)", "impl": "reference",
           "config": {"workload": f"{cfg.name}: {cfg.desc}", "M": M, "K": K, "nnz": len(ci), "N": N,
                      "parallelism": "host cores"},
           "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
                            "sample": sample},
           "e2e": {"value": round(value, 3), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "gpu_launches": 0}
    print(json.dumps(out))


def main():
    args = parse_args()
    from datagen import configs
    cfg = configs.get(args.config)
    N = args.n or cfg.N
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, cfg, N, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as tdist
        torch.cuda.set_device(local_rank)
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    run_dtc(args, cfg, N, rank, world, local_rank)
    if world > 1:
        import torch.distributed as tdist
        tdist.barrier()
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
