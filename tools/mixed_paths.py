"""Experiment: register-gather kernel and TMA-gather kernel on disjoint column halves, concurrently."""
import ctypes, os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from datagen import configs
import paper_conf_asplos_fan0024_b200._binding as bnd

def load(path):
    L = ctypes.CDLL(path)
    vp, i64 = ctypes.c_void_p, ctypes.c_int64
    L.dtc_format_build_ex.argtypes = [ctypes.POINTER(bnd._Csr), ctypes.POINTER(bnd._Opts), vp, ctypes.POINTER(vp)]
    L.dtc_spmm.argtypes = [vp, vp, i64, i64, vp, i64, vp]
    return L

def main(name):
    cfg = configs.get(name); N = cfg.N
    rp, ci = configs.make_pattern(cfg); v = configs.make_values(cfg, len(ci)); B = configs.make_B(cfg, N)
    rpd, cid, vd, Bd = [torch.from_numpy(x).cuda() for x in (rp, ci, v, B)]
    C = torch.empty((cfg.M, N), device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    libs = {"ldg": load(os.path.abspath("paper_conf_asplos_fan0024_b200/libdtc.so")),
            "tma": load(os.path.abspath("build_variants/libdtc_tmadefault.so"))}
    hs = {}
    for k, L in libs.items():
        csr = bnd._make_csr(rpd, cid, vd, cfg.M, cfg.K, cfg.dtype); h = ctypes.c_void_p(); o = bnd._Opts(0, 0, 0)
        assert L.dtc_format_build_ex(ctypes.byref(csr), ctypes.byref(o), None, ctypes.byref(h)) == 0
        hs[k] = h
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    esz = 4 if cfg.dtype != "fp16" else 2
    def run(mode):
        if mode in ("ldg", "tma"):
            libs[mode].dtc_spmm(hs[mode], Bd.data_ptr(), N, N, C.data_ptr(), N, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
        else:
            frac = {"mix50": 0.5, "mix25": 0.25, "mix75": 0.75}[mode]
            n_t = int(round(N * frac / 64)) * 64
            cur = torch.cuda.current_stream()
            ev = torch.cuda.Event(); ev.record(cur); s1.wait_event(ev); s2.wait_event(ev)
            libs["ldg"].dtc_spmm(hs["ldg"], Bd.data_ptr(), N - n_t, N, C.data_ptr(), N, ctypes.c_void_p(s1.cuda_stream))
            libs["tma"].dtc_spmm(hs["tma"], Bd.data_ptr() + (N - n_t) * esz, n_t, N, C.data_ptr() + (N - n_t) * 4, N, ctypes.c_void_p(s2.cuda_stream))
            e1, e2 = torch.cuda.Event(), torch.cuda.Event(); e1.record(s1); e2.record(s2); cur.wait_event(e1); cur.wait_event(e2)
    res = {}
    for mode in ("ldg", "tma", "mix25", "mix50", "mix75"):
        ts = []
        for it in range(13):
            flush.zero_(); torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); run(mode); b.record(); torch.cuda.synchronize()
            if it >= 3: ts.append(a.elapsed_time(b))
        res[mode] = statistics.median(ts)
        ref = C.clone() if mode == "ldg" else ref
        if mode != "ldg":
            assert torch.allclose(C, ref, rtol=1e-3, atol=1e-3), mode
    fl = 2.0 * len(ci) * N
    print(name, {k: f"{v:.3f} ms {fl / v / 1e6:.0f} GFLOP/s" for k, v in res.items()}, flush=True)

for n in sys.argv[1:]:
    main(n)
