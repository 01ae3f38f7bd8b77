#!/usr/bin/env python
"""bench.py -- SpMM GFLOP/s (2*nnz*N/t) of the DTC-SpMM hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--legs ...] [--impl dtc|reference]

One step = one pass of the whole hot path (dtc_spmm: S1-S5) over one batch of the config's
synthetic input (the ME-TCF format is built once beforehand, as the paper converts once and
reuses A; its build time is reported as format_build_ms).  The headline workload
is c3 (Reddit-shaped, TF32, N=256): the largest BASELINE config that fits one GPU's kernel
launch with the roofline accounting below; c2, c3h, c4 (N=64/128/256) and c5 run as nested
`legs` with their own roofline, cuSPARSE comparison and e2e.

Timing: CUDA events on the launching stream around each step, L2 flushed (256 MiB memset,
outside the events) between steps, W warm-up steps, barrier + synchronize on both sides, max over
ranks.  Rank 0 prints ONE JSON line.

roofline (per leg): `frac` = literal algorithmic bytes (format + sum_t u_t*N*elt +
M*N*4) / mean kernel time / measured HBM peak; `dram_frac` = DRAM bytes actually moved (ncu
dram__bytes_read+write of ONE launch of this commit, captured by a subprocess under ncu in this
run) / mean kernel time / peak; `compulsory_frac` counts every distinct B row once; `gather_frac`
= gathered B bytes / time / the measured TMA gather4-from-L2 peak for the slice width (profiles/r02_gather_issue_sweep.txt).
`bound_by` names the largest of these fractions.

--impl reference times the FP64 CPU oracle (the only reference this tier has) on the host cores on
bounded samples of the same workload.  Under torchrun (N > 1) the row windows are partitioned
across ranks (dtc_spmm_dist); value = whole-job GFLOP/s with B resident on every GPU.
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import shutil
import statistics
import subprocess
import sys
import tempfile
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMM GFLOP/s (2*nnz*N/t)"
UNIT = "GFLOP/s"
L2_FLUSH_BYTES = 256 << 20
HEADLINE = "c3"
DEFAULT_LEGS = "c2,c3h,c4:64,c4:128,c4:256,c5"
# TMA tile::gather4 peak from an L2-resident B (77 MB), 148 SMs, best over CTAs/SM x gather ops per
# stage x stages (tools/gather_bw2.py --issue, profiles/r02_gather_issue_sweep.txt), per row-slice
# width the kernel gathers: 1 KB slices (B rows >= 1 KB) and 512 B slices.  (Round 1's 9.3 TB/s was
# the rate of one 2-op stage per CTA at 3 CTAs/SM, not the engine's peak.)
GATHER4_L2_PEAK_GBS = {1024: 18670.0, 512: 12777.0}


def gather_peak(N, elt):
    """the slice width k_spmm_pad gathers for N columns (pad_geometry) -> its measured gather4 peak"""
    return GATHER4_L2_PEAK_GBS[1024 if (N * elt >= 1024 and (N * elt) % 8 == 0) else 512]


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="dtc", choices=["dtc", "reference"])
    p.add_argument("--config", default=HEADLINE)
    p.add_argument("--n", type=int, default=0, help="override N (columns of B) of the headline config")
    p.add_argument("--legs", default=DEFAULT_LEGS,
                   help="nested legs 'cfg[:N],...' measured after the headline ('none' = off)")
    p.add_argument("--unit-blocks", type=int, default=0)
    p.add_argument("--guided", type=int, default=0, help="F4 guided tail (1 on, -1 off, 0 auto)")
    p.add_argument("--persistent", type=int, default=0, help="DTC_OPT_PERSISTENT for the timed launches")
    p.add_argument("--window-rows", type=int, default=0,
                   help="32: NEXT-2 tall windows (TF32 workloads; FP16 legs keep 16-row ME-TCF)")
    p.add_argument("--selector", type=int, default=2,
                   help="B200 Selector (NEXT-4): 1 = plan U by simulation + window height, 2 = window height only "
                        "(32-row NEXT-2 windows where they pay), 0 = fixed rule, 16-row windows")
    p.add_argument("--ncu", default="auto", choices=["auto", "off"],
                   help="capture DRAM traffic of one launch per leg under ncu (subprocess)")
    p.add_argument("--no-cusparse", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--minimal", action="store_true", help="only the timed dtc loop (for ncu launch lists)")
    p.add_argument("--tca", type=int, default=-1,
                   help="also time the SpMM on the TCA-reordered matrix (NEXT-1): 1 on, 0 off, -1 on when nnz < 10M")
    p.add_argument("--graphconv", type=int, default=-1,
                   help="also time one GraphConv layer + its backward (NEXT-3) with F_in=N and this F_out "
                        "(-1: F_out=N; 0: off)")
    return p.parse_args()


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def parse_legs(spec: str, headline: tuple):
    if spec in ("", "none", "off"):
        return []
    from datagen import configs
    out = []
    for item in spec.split(","):
        name, _, n = item.partition(":")
        cfg = configs.get(name)
        leg = (name, int(n) if n else cfg.N)
        if leg != headline:
            out.append(leg)
    return out


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
_PATTERNS = {}


def load_pattern(cfg):
    if cfg.name not in _PATTERNS:
        from datagen import configs
        base = "c3" if cfg.name == "c3h" else cfg.name       # c3h: the c3 pattern with fp16 values
        if base in _PATTERNS:
            _PATTERNS[cfg.name] = _PATTERNS[base]
        else:
            _PATTERNS[cfg.name] = configs.make_pattern(cfg)
    return _PATTERNS[cfg.name]


def load_workload(cfg, N):
    from datagen import configs
    rp, ci = load_pattern(cfg)
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
    gathered = sum_u * N * elt
    literal = fmt + gathered + M * N * 4
    distinct_rows = int(np.unique(atob[atob >= 0]).size)
    compulsory = fmt + distinct_rows * N * elt + M * N * 4
    return {"literal": literal, "compulsory": compulsory, "gathered": gathered, "sum_u": sum_u, "format": fmt}


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


# ------------------------------------------------------------------ ncu traffic (subprocess)
def ncu_traffic(legs, cache_dir, timeout_s=600):
    """DRAM bytes (read + write), kernel time and L2 bytes of ONE launch per leg of THIS build,
    from `ncu` over tools/ncu_traffic.py (one process for all legs; inputs from cache_dir)."""
    ncu = shutil.which("ncu") or "/usr/local/cuda/bin/ncu"
    if not os.path.exists(ncu):
        return {"error": "ncu not found"}
    spec = ",".join(f"{n}:{N}" for n, N in legs)
    log = os.path.join(cache_dir, "ncu.csv")
    metrics = "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_bytes.sum"
    cmd = [ncu, "--metrics", metrics, "--clock-control", "none", "-k", "regex:k_spmm_(pad|ldg)", "--csv",
           "--log-file", log, sys.executable, os.path.join(ROOT, "tools", "ncu_traffic.py"), "--cache", cache_dir,
           "--legs", spec]
    try:
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout_s)
    except subprocess.TimeoutExpired:
        return {"error": f"ncu timed out after {timeout_s} s"}
    if r.returncode != 0 or not os.path.exists(log):
        return {"error": f"ncu rc={r.returncode}: {(r.stderr or r.stdout)[-300:]}"}
    import csv
    rows = [x for x in csv.reader(open(log)) if x]
    hdr = None
    per_launch = []
    for x in rows:
        if "Metric Name" in x and "ID" in x:
            hdr = x
            continue
        if hdr and len(x) == len(hdr):
            d = dict(zip(hdr, x))
            per_launch.append(d)
    # group by launch ID, in launch order (one launch per leg)
    launches = {}
    for d in per_launch:
        launches.setdefault(int(d["ID"]), {})[d["Metric Name"]] = (float(d["Metric Value"].replace(",", "")),
                                                                   d["Metric Unit"])
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "nsecond": 1e-9, "usecond": 1e-6,
             "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}
    out = {}
    ids = sorted(launches)
    if len(ids) != len(legs):
        return {"error": f"expected {len(legs)} launches, ncu saw {len(ids)}"}
    for (name, N), i in zip(legs, ids):
        m = launches[i]
        g = lambda k: m[k][0] * scale.get(m[k][1], 1.0) if k in m else None  # noqa: E731
        rd, wr = g("dram__bytes_read.sum"), g("dram__bytes_write.sum")
        out[f"{name}:{N}"] = {"dram_bytes": int(rd + wr) if rd is not None and wr is not None else None,
                              "kernel_s": g("gpu__time_duration.sum"), "l2_bytes": g("lts__t_bytes.sum"),
                              "time_unit": m.get("gpu__time_duration.sum", (0, "?"))[1]}
    return out


# ------------------------------------------------------------------ cpu baseline
def cpu_info():
    model = platform.processor() or ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


def _oracle_rate(oracle, cfg, rp, ci, vf, Bf, N, budget_s):
    M, K = cfg.M, cfg.K
    r_probe = min(M, 4096)
    t0 = time.perf_counter()
    oracle.spmm(M, K, rp, ci, vf, Bf, 0, r_probe, bound=False)
    rate = max(int(rp[r_probe]), 1) / max(time.perf_counter() - t0, 1e-4)   # nnz per second
    if len(ci) / rate <= budget_s:
        r1, reps = M, max(1, min(2000, int(budget_s / max(len(ci) / rate, 1e-4))))
    else:
        r1, reps = max(1, min(M, int(np.searchsorted(rp, rate * budget_s)))), 1
    t0 = time.perf_counter()
    done = 0
    while True:   # at least `reps`, and at least ~budget_s of CPU work
        oracle.spmm(M, K, rp, ci, vf, Bf, 0, r1, bound=False)
        done += 1
        el = time.perf_counter() - t0
        if done >= reps and el >= 0.8 * budget_s:
            break
    nnz_s = int(rp[r1])
    return 2.0 * nnz_s * N * done / el / 1e9, r1, nnz_s, done, el


def cpu_baseline(cfg, rp, ci, v, B, N, budget_s=10.0):
    """The oracle as it stands, timed on the host cores on a bounded sample of the workload, plus
    1-thread runs on c1 and c2."""
    import oracle
    from datagen import configs
    cores = oracle.max_threads()
    vf = v.astype(np.float32)
    Bf = B.astype(np.float32, copy=False)
    g, r1, nnz_s, reps, el = _oracle_rate(oracle, cfg, rp, ci, vf, Bf, N, budget_s)
    out = {"value": round(g, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
           "sample": f"{cfg.name}: rows [0,{r1}) of {cfg.M} ({nnz_s} of {len(ci)} nnz), N={N}, FP64 C only, "
                     f"x{reps} reps, {el:.1f} s, OpenMP {cores} threads", **cpu_info()}
    single = {}
    oracle.set_threads(1)
    try:
        for name in ("c1", "c2"):
            c = configs.get(name)
            rp1, ci1 = load_pattern(c)
            v1 = configs.make_values(c, len(ci1)).astype(np.float32)
            B1 = configs.make_B(c, c.N).astype(np.float32, copy=False)
            g1, r11, nnz1, reps1, el1 = _oracle_rate(oracle, c, rp1, ci1, v1, B1, c.N, 2.0)
            single[name] = {"value": round(g1, 3), "unit": UNIT, "threads": 1,
                            "sample": f"rows [0,{r11}) of {c.M}, N={c.N}, x{reps1}, {el1:.1f} s"}
    finally:
        oracle.set_threads(cores)
    out["single_thread"] = single
    return out


# ------------------------------------------------------------------ one leg (1 GPU)
def run_leg(args, cfg, N, dev, stream, flush, full: bool, cache_dir=None):
    """Time dtc_spmm on one workload; returns the leg's JSON object (+ the objects the headline
    reuses).  full=False skips the extras (TCA / graphconv) that only the headline reports."""
    import torch
    import paper_conf_asplos_fan0024_b200 as dtc
    rp, ci, v, B = load_workload(cfg, N)
    M, K, nnz = cfg.M, cfg.K, len(ci)
    elt = 2 if cfg.dtype == "fp16" else 4
    rp_d = torch.from_numpy(rp).to(dev)
    ci_d = torch.from_numpy(ci).to(dev)
    v_d = torch.from_numpy(v).to(dev)
    B_d = torch.from_numpy(B).to(dev)
    flops = 2.0 * nnz * N
    if cache_dir is not None:   # inputs for the ncu subprocess (this run only; removed at exit)
        d = os.path.join(cache_dir, f"{cfg.name}")
        if not os.path.exists(d + ".rp.npy"):
            np.save(d + ".rp.npy", rp)
            np.save(d + ".ci.npy", ci)
    build_ms_runs = []
    for _ in range(2):   # first call (one-time module/pool setup) and a warm rebuild
        torch.cuda.synchronize()
        tb0 = time.perf_counter()
        fmt = dtc.Format.build(rp_d, ci_d, v_d, M, K, dtype=cfg.dtype, unit_blocks=args.unit_blocks,
                               guided=args.guided, n_hint=N, selector=args.selector,
                               window_rows=args.window_rows if cfg.dtype == "tf32" else 0)
        torch.cuda.synchronize()
        build_ms_runs.append((time.perf_counter() - tb0) * 1e3)
    fmt.set_option("persistent", args.persistent)
    C_d = torch.empty((M, N), dtype=torch.float32, device=dev)
    fn = lambda: fmt.spmm(B_d, C_d)  # noqa: E731
    sampler = ClockSampler(dev.index or 0)
    with sampler:
        t_wall0 = time.perf_counter()
        ms = time_loop(fn, args.steps, args.warmup, stream, flush)
        t_wall = time.perf_counter() - t_wall0
    kern_ms = statistics.mean(ms)
    value = flops / (kern_ms * 1e-3) / 1e9
    leg = {"workload": f"{cfg.name}: {cfg.desc}", "config": cfg.name, "M": M, "K": K, "nnz": nnz, "N": N,
           "dtype": cfg.dtype, "value": round(value, 2), "unit": UNIT, "ms_per_step": round(kern_ms, 5),
           "ms_median": round(statistics.median(ms), 5), "steps": args.steps, "warmup": args.warmup,
           "kernel": "k_spmm_pad" if fmt.get_option("last_kernel") == 4 else "k_spmm_ldg",
           "clocks": sampler.summary(), "wall_s_timed_region": round(t_wall, 4)}
    exp = fmt.export()
    ab = algorithmic_bytes(exp, M, N, elt)
    T = fmt.num_tc_blocks
    leg.update({"num_tc_blocks": T, "mean_nnz_tc": round(nnz / max(T, 1), 3), "sum_u": ab["sum_u"],
                "unit_blocks": fmt.unit_blocks, "num_units": fmt.num_units,
                "split_windows": fmt.num_split_windows, "guided": fmt.get_option("guided"),
                "f4_plan": {0: "rule", 1: "selector", 2: "rule + selector window height"}[args.selector],
                "window_rows": fmt.window_rows,
                "selector_predicted_ms": round(fmt.get_option("plan_makespan_ns") / 1e6, 4) or None,
                "format_build_ms": round(build_ms_runs[-1], 3),
                "format_build_first_call_ms": round(build_ms_runs[0], 3),
                "format_build_x_spmm": round(build_ms_runs[-1] / kern_ms, 2)})
    hbm, peak_src = peaks()
    t = kern_ms * 1e-3
    leg["roofline"] = {"bound": "hbm", "achieved": round(ab["literal"] / t / 1e9, 1), "peak": hbm, "unit": "GB/s",
                       "frac": round(ab["literal"] / t / 1e9 / hbm, 4), "traffic": None, "peak_source": peak_src,
                       "bytes_per_launch": ab["literal"],
                       "bytes_def": "literal algorithmic bytes, SURVEY §8(d): format + sum_t u_t*N*elt + M*N*4",
                       "compulsory_bytes_per_launch": ab["compulsory"],
                       "compulsory_frac": round(ab["compulsory"] / t / 1e9 / hbm, 4),
                       "gathered_bytes_per_launch": ab["gathered"],
                       "gather_ceiling_gbs": gather_peak(N, elt),
                       "gather_frac": round(ab["gathered"] / t / 1e9 / gather_peak(N, elt), 4),
                       "kernel_ms_mean": round(kern_ms, 5)}

    # ---- e2e through the public API with HOST buffers (pinned): every step copies its B in and
    # its C out.  Headline: the streaming API (dtc_spmm_host_async, consecutive steps overlap their
    # copies with the previous kernel; one wait after the K steps); e2e_sync: one blocking
    # dtc_spmm_host per step.
    if not args.no_e2e:
        Bh = [torch.from_numpy(B).pin_memory(), torch.from_numpy(B.copy()).pin_memory()]
        Ch = [torch.empty((M, N), dtype=torch.float32).pin_memory() for _ in range(2)]
        e2e_steps = max(3, min(args.steps, 10 if nnz > 50_000_000 else 20))
        for j in range(2):
            fmt.spmm_host_async(Bh[j], Ch[j])
        fmt.wait()
        t0 = time.perf_counter()
        for j in range(e2e_steps):
            fmt.spmm_host_async(Bh[j % 2], Ch[j % 2])
        fmt.wait()
        e2e_s = (time.perf_counter() - t0) / e2e_steps
        mode = fmt.get_option("last_host_mode")
        zc = bool(mode & 1)
        c_transfer = ("zero-copy: the kernel stores C into pinned mapped host memory over PCIe "
                      "(M*N*4 bytes cross to the host, no cudaMemcpy)") if zc else "cudaMemcpy2DAsync device->host"
        leg["e2e"] = {"value": round(flops / e2e_s / 1e9, 2), "unit": UNIT,
                      "h2d_bytes_per_step": int(B.nbytes), "d2h_bytes_per_step": int(M * N * 4),
                      "ms_per_step": round(e2e_s * 1e3, 4), "steps": e2e_steps,
                      "api": "dtc_spmm_host_async x K, dtc_spmm_host_wait (pinned host B and C; each step copies "
                             "its own B in and C out; step j+1's copy-in overlaps step j's kernel)",
                      "c_transfer": c_transfer, "wall_clock": "perf_counter around the K steps and the final wait"}
        leg["e2e_matches_device"] = bool(torch.equal(Ch[(e2e_steps - 1) % 2], C_d.cpu()))
        for _ in range(2):
            fmt.spmm_host(Bh[0], Ch[0])
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            fmt.spmm_host(Bh[0], Ch[0])
        e2e_sync_s = (time.perf_counter() - t0) / e2e_steps
        mode = fmt.get_option("last_host_mode")
        leg["e2e_sync"] = {"value": round(flops / e2e_sync_s / 1e9, 2), "unit": UNIT,
                           "ms_per_step": round(e2e_sync_s * 1e3, 4), "steps": e2e_steps,
                           "api": "dtc_spmm_host (blocking; column chunks pipelined within the call)",
                           "column_chunks": mode // 2, "zero_copy_c": bool(mode & 1)}
        del Bh, Ch

    # ---- cuSPARSE on the same box (comparison system)
    if not args.no_cusparse:
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
                    ms2 = time_loop(cs.run, max(3, min(args.steps, 10)), 2, stream, flush)
                    res[alg] = round(flops / (statistics.mean(ms2) * 1e-3) / 1e9, 2)
                except Exception as e:  # noqa: BLE001
                    res[alg] = f"error: {e}"
                cs.close()
            nums = {k: x for k, x in res.items() if isinstance(x, float)}
            leg["cusparse"] = {"gflops": res, "best": max(nums.values()) if nums else None,
                               "speedup_vs_best": round(value / max(nums.values()), 3) if nums else None}
            del C2
        except Exception as e:  # noqa: BLE001
            leg["cusparse"] = {"error": str(e)}

    extras = {"fmt": fmt, "B_d": B_d, "C_d": C_d, "rp": rp, "ci": ci, "v": v, "B": B, "rp_d": rp_d,
              "ci_d": ci_d, "v_d": v_d, "kern_ms": kern_ms, "flops": flops, "exp": exp}
    return leg, extras


def headline_extras(args, cfg, N, dev, stream, flush, leg, x):
    """NEXT rows on the headline workload: Selector (NEXT-4), TCA (NEXT-1), GraphConv (NEXT-3)."""
    import torch
    import paper_conf_asplos_fan0024_b200 as dtc
    fmt, B_d, C_d = x["fmt"], x["B_d"], x["C_d"]
    M, K, nnz = cfg.M, cfg.K, len(x["ci"])
    sm = torch.cuda.get_device_properties(dev).multi_processor_count
    try:
        leg["selector"] = dtc.selector_report(x["exp"]["row_window_offset"], sm, cfg.dtype, N)
    except Exception as e:  # noqa: BLE001
        leg["selector"] = {"error": str(e)}
    if args.tca == 1 or (args.tca < 0 and nnz < 10_000_000):
        try:
            t0 = time.perf_counter()
            perm, tinfo = dtc.tca_reorder_checked(M, K, x["rp"], x["ci"], sm)
            reorder_s = time.perf_counter() - t0
            perm_d = torch.from_numpy(perm).to(dev)
            fmt_t = dtc.Format.build(x["rp_d"], x["ci_d"], x["v_d"], M, K, dtype=cfg.dtype, row_perm=perm_d)
            C_t = torch.empty((M, N), dtype=torch.float32, device=dev)
            ms_t = time_loop(lambda: fmt_t.spmm(B_d, C_t), max(10, min(args.steps, 50)), 3, stream, flush)
            tms = statistics.mean(ms_t)
            leg["tca"] = {"value": round(x["flops"] / (tms * 1e-3) / 1e9, 2), "unit": UNIT, **tinfo,
                          "ms_per_step": round(tms, 5), "num_tc_blocks": fmt_t.num_tc_blocks,
                          "reorder_host_s": round(reorder_s, 3), "speedup_vs_unordered": round(x["kern_ms"] / tms, 3),
                          "matches_unordered": bool(torch.allclose(C_t, C_d, rtol=1e-2, atol=1e-2))}
            fmt_t.close()
        except Exception as e:  # noqa: BLE001
            leg["tca"] = {"error": str(e)}
    if args.graphconv != 0:
        try:
            leg["graphconv"] = graphconv_leg(args, cfg, N, dev, stream, flush, x)
        except Exception as e:  # noqa: BLE001
            leg["graphconv"] = {"error": str(e)}


def graphconv_leg(args, cfg, N, dev, stream, flush, x):
    """One GCN layer forward (Eq. (2)) and its backward through the library."""
    import torch
    fmt, B_d = x["fmt"], x["B_d"]
    M = cfg.M
    F_out = N if args.graphconv < 0 else args.graphconv
    g = torch.Generator(device=dev).manual_seed(7)
    Wg = torch.empty((N, F_out), dtype=torch.float32, device=dev).uniform_(-0.1, 0.1, generator=g)
    bg = torch.empty((F_out,), dtype=torch.float32, device=dev).uniform_(-0.1, 0.1, generator=g)
    AH = torch.empty((M, N), dtype=torch.float32, device=dev)
    Yg = torch.empty((M, F_out), dtype=torch.float32, device=dev)
    gsteps = max(5, min(args.steps, 20))
    ms_g = time_loop(lambda: fmt.graphconv(B_d, Wg, bg, relu=True, AH=AH, Y=Yg), gsteps, 3, stream, flush)
    gms = statistics.mean(ms_g)
    return {"F_in": N, "F_out": F_out, "ms": round(gms, 5), "spmm_ms": round(x["kern_ms"], 5),
            "dense_ms": round(gms - x["kern_ms"], 5), "steps": gsteps,
            "api": "dtc_graphconv (DTC-SpMM + cuBLASLt TF32 bias/ReLU epilogue)"}


# ------------------------------------------------------------------ dtc arm
def run_dtc(args, cfg, N, rank, world, local_rank):
    import torch
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    stream = torch.cuda.current_stream()
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    if world > 1:
        return run_dist(args, cfg, N, rank, world, local_rank, dev, stream, flush)

    legs = parse_legs(args.legs, (cfg.name, N)) if not args.minimal else []
    cache_dir = tempfile.mkdtemp(prefix="dtc_bench_") if (args.ncu == "auto" and not args.minimal) else None
    try:
        if args.minimal:
            a2 = argparse.Namespace(**{**vars(args), "no_e2e": True, "no_cusparse": True})
            leg, _ = run_leg(a2, cfg, N, dev, stream, flush, full=False)
            print(json.dumps({"metric": METRIC, "value": leg["value"], "unit": UNIT, "ms_per_step": leg["ms_per_step"],
                              "minimal": True, "config": {"workload": cfg.name, "N": N}}))
            return
        head, x = run_leg(args, cfg, N, dev, stream, flush, full=True, cache_dir=cache_dir)
        headline_extras(args, cfg, N, dev, stream, flush, head, x)
        del x
        torch.cuda.empty_cache()
        from datagen import configs
        leg_objs = []
        for name, n in legs:
            c = configs.get(name)
            lg, xx = run_leg(args, c, n, dev, stream, flush, full=False, cache_dir=cache_dir)
            del xx
            torch.cuda.empty_cache()
            leg_objs.append(lg)
        # DRAM traffic of one launch per workload, this build, under ncu (subprocess; not timed)
        all_legs = [(cfg.name, N)] + list(legs)
        traffic = ncu_traffic(all_legs, cache_dir) if cache_dir else {"error": "disabled (--ncu off)"}
        hbm, _ = peaks()
        for (name, n), lg in zip(all_legs, [head] + leg_objs):
            tr = traffic.get(f"{name}:{n}") if "error" not in traffic else None
            rf = lg["roofline"]
            t = lg["ms_per_step"] * 1e-3
            if tr and tr.get("dram_bytes") is not None:
                rf["traffic"] = tr["dram_bytes"]
                rf["traffic_source"] = "ncu dram__bytes_read.sum + dram__bytes_write.sum, one launch, this run"
                rf["dram_frac"] = round(tr["dram_bytes"] / t / 1e9 / hbm, 4)
                rf["ncu_kernel_ms"] = round(tr["kernel_s"] * 1e3, 5) if tr.get("kernel_s") else None
                rf["l2_bytes"] = tr.get("l2_bytes")
            else:
                rf["traffic_source"] = traffic.get("error", "unavailable")
            fr = {"hbm_literal": rf["frac"], "dram_measured": rf.get("dram_frac"), "tma_gather4": rf["gather_frac"]}
            real = {k: val for k, val in fr.items() if k != "hbm_literal" and val is not None}
            rf["bound_by"] = max(real, key=real.get) if real else "hbm_literal"
            rf["fracs"] = fr
    finally:
        if cache_dir:
            shutil.rmtree(cache_dir, ignore_errors=True)

    out = {"metric": METRIC, "value": head["value"], "unit": UNIT, "n_gpus": 1, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": head["ms_per_step"], "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": cfg.dtype,
           "data": "synthetic (seeded generators, datagen/; DESIGN.md §3)"}
    cfgd = {"workload": head["workload"], "M": head["M"], "K": head["K"], "nnz": head["nnz"], "N": N,
            "parallelism": "row-window dp1", "l2": "flushed between steps (256 MiB memset outside the events)",
            "timing": "CUDA events per step on the launching stream; mean over steps"}
    for k in ("num_tc_blocks", "mean_nnz_tc", "sum_u", "unit_blocks", "num_units", "split_windows", "window_rows",
              "f4_plan"):
        cfgd[k] = head[k]
    out["config"] = cfgd
    out["roofline"] = head["roofline"]
    for k in ("e2e", "e2e_sync", "e2e_matches_device", "cusparse", "clocks", "wall_s_timed_region", "format_build_ms",
              "format_build_first_call_ms", "format_build_x_spmm", "kernel", "selector", "tca", "graphconv"):
        if k in head:
            out[k] = head[k]
    out["gpu_launches"] = args.steps * launches_per_call()
    out["legs"] = leg_objs
    if not args.no_cpu:
        rp, ci = load_pattern(cfg)
        from datagen import configs
        out["cpu_baseline"] = cpu_baseline(cfg, rp, ci, configs.make_values(cfg, len(ci)), configs.make_B(cfg, N), N)
    print(json.dumps(out))


def launches_per_call():
    import paper_conf_asplos_fan0024_b200 as dtc
    return dtc.launches_per_call()


def run_dist(args, cfg, N, rank, world, local_rank, dev, stream, flush):
    """N > 1: row windows partitioned across ranks by TC-block count (dtc_spmm_dist); kernel-only
    value with B resident on every rank; e2e = B broadcast over NVLink from the root's device copy,
    the local kernel, and C all-gathered (device resident)."""
    import torch
    import torch.distributed as tdist
    import paper_conf_asplos_fan0024_b200 as dtc
    rp, ci, v, B = load_workload(cfg, N)
    M, K, nnz = cfg.M, cfg.K, len(ci)
    flops = 2.0 * nnz * N
    rp_d = torch.from_numpy(rp).to(dev)
    ci_d = torch.from_numpy(ci).to(dev)
    v_d = torch.from_numpy(v).to(dev)
    B_d = torch.from_numpy(B).to(dev)
    uid = [dtc.nccl_unique_id() if rank == 0 else None]
    tdist.broadcast_object_list(uid, src=0)
    torch.cuda.synchronize()
    tb0 = time.perf_counter()
    dd = dtc.Dist(rp_d, ci_d, v_d, M, K, cfg.dtype, rank, world, uid[0])
    torch.cuda.synchronize()
    build_ms = (time.perf_counter() - tb0) * 1e3
    rows = dd.row_end - dd.row_begin
    C_d = torch.empty((max(rows, 1), N), dtype=torch.float32, device=dev)
    fn = lambda: dd.local_spmm(B_d, C_d)  # noqa: E731
    tdist.barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local_rank)
    with sampler:
        ms = time_loop(fn, args.steps, args.warmup, stream, flush)
    tdist.barrier()
    torch.cuda.synchronize()
    t = torch.tensor([float(sum(ms))], device=dev)
    tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    ms_per_step = float(t.item()) / args.steps
    value = flops / (ms_per_step * 1e-3) / 1e9
    out = {"metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms_per_step, 5), "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": cfg.dtype,
           "data": "synthetic (seeded generators, datagen/; DESIGN.md §3)",
           "config": {"workload": f"{cfg.name}: {cfg.desc}", "M": M, "K": K, "nnz": nnz, "N": N,
                      "parallelism": f"row-window dp{world}", "l2": "flushed between steps",
                      "timing": "CUDA events per step; sum over steps; max over ranks"},
           "clocks": sampler.summary(), "format_build_ms": round(build_ms, 3),
           "gpu_launches": args.steps * launches_per_call()}
    if not args.no_e2e:
        Cfull = torch.empty((M, N), dtype=torch.float32, device=dev)
        Bh = torch.from_numpy(B).pin_memory() if rank == 0 else None
        Ch = torch.empty((M, N), dtype=torch.float32).pin_memory() if rank == 0 else None

        def e2e_step():
            if rank == 0:
                B_d.copy_(Bh, non_blocking=True)
            dd.spmm(B_d, Cfull, root=0, gather_c=True)
            if rank == 0:
                Ch.copy_(Cfull, non_blocking=True)
            torch.cuda.synchronize()

        for _ in range(2):
            e2e_step()
        tdist.barrier()
        e2e_steps = max(3, min(args.steps, 10))
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        el = torch.tensor([(time.perf_counter() - t0) / e2e_steps], device=dev)
        tdist.all_reduce(el, op=tdist.ReduceOp.MAX)
        e2e_s = float(el.item())
        out["e2e"] = {"value": round(flops / e2e_s / 1e9, 2), "unit": UNIT,
                      "h2d_bytes_per_step": int(B.nbytes), "d2h_bytes_per_step": int(M * N * 4),
                      "ms_per_step": round(e2e_s * 1e3, 4), "steps": e2e_steps,
                      "api": "root H2D of B, dtc_spmm_dist (NCCL broadcast of B pipelined with the local "
                             "kernel, C all-gathered), root D2H of C"}

        # device-resident variant: B already in the root's HBM, NVLink broadcast + kernel + all-gather
        def dev_step():
            dd.spmm(B_d if rank == 0 else None, Cfull, root=0, gather_c=True, N=N)
            torch.cuda.synchronize()

        for _ in range(2):
            dev_step()
        tdist.barrier()
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            dev_step()
        el = torch.tensor([(time.perf_counter() - t0) / e2e_steps], device=dev)
        tdist.all_reduce(el, op=tdist.ReduceOp.MAX)
        out["e2e_device_b"] = {"value": round(flops / float(el.item()) / 1e9, 2), "unit": UNIT,
                               "ms_per_step": round(float(el.item()) * 1e3, 4), "steps": e2e_steps,
                               "api": "dtc_spmm_dist with B resident on the root: chunked NCCL broadcast over "
                                      "NVLink pipelined with the kernel, C all-gathered; max over ranks"}
    if rank == 0:
        print(json.dumps(out))


# ------------------------------------------------------------------ reference arm
def run_reference(args, cfg, N, rank, world):
    if rank != 0:
        return
    import oracle
    rp, ci, v, B = load_workload(cfg, N)
    vf = v.astype(np.float32)
    Bf = B.astype(np.float32, copy=False)
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
    sample = (f"{cfg.name}: rows [0,{r1}) of {M} ({nnz_s} of {len(ci)} nnz) per step (~1 s of CPU work), N={N}, "
              f"FP64, OpenMP {cores} threads")
    out = {"metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded generators, datagen/)", "impl": "reference",
           "config": {"workload": f"{cfg.name}: {cfg.desc}", "M": M, "K": K, "nnz": len(ci), "N": N,
                      "parallelism": "host cores"},
           "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
                            "sample": sample, **cpu_info()},
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
