"""Run tools/gather_bw2.cu on the GPU box: TMA gather4 vs 1D bulk copies of random B rows."""
import ctypes
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libgather_bw2.so")


def issue_sweep(L, torch, sink):
    """Bytes in flight vs ops per stage: is the per-SM gather rate set by in-flight bytes or by ops/stage?"""
    for total, tag in ((77 << 20, "L2-resident 77 MB"), (238 << 20, "c3-sized 238 MB")):
        for row in (1024, 512):
            K = total // row
            B = torch.empty(K * row, dtype=torch.uint8, device="cuda").random_()
            for cps in (1, 2, 3):
                for ops, R in ((2, 4), (2, 6), (2, 8), (2, 12), (2, 16), (4, 4), (4, 6), (4, 8), (8, 2), (8, 3), (8, 4)):
                    by = ctypes.c_double(0)
                    ms = L.gather_bw2(B.data_ptr(), K, row, 0, ops, R, 148 * cps, 3000, sink.data_ptr(), ctypes.byref(by))
                    gbs = by.value / ms / 1e6 if ms > 0 else ms
                    kb = cps * ops * R * 4 * row / 1024
                    print(f"{tag} row {row:5d} B ctas/SM {cps} ops/stage {ops:2d} R {R:2d} (in flight <= {kb:4.0f} KB/SM):"
                          f" {gbs:8.0f} GB/s", flush=True)
            del B


def main():
    import sys
    import torch
    if not os.path.exists(SO):
        subprocess.check_call(["nvcc", "-O3", "-shared", "-Xcompiler", "-fPIC", "-gencode", "arch=compute_100a,code=sm_100a",
                               os.path.join(HERE, "gather_bw2.cu"), "-o", SO, "-lcuda"])
    L = ctypes.CDLL(SO)
    L.gather_bw2.restype = ctypes.c_float
    L.gather_bw2.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                             ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(ctypes.c_double)]
    sink = torch.zeros(4, dtype=torch.int32, device="cuda")
    if "--issue" in sys.argv:
        return issue_sweep(L, torch, sink)
    for total, tag in ((77 << 20, "L2-resident 77 MB"), (1 << 30, "DRAM 1 GB")):
        for row in (512, 1024, 2048):
            K = total // row
            B = torch.empty(K * row, dtype=torch.uint8, device="cuda").random_()
            for mode, name in ((0, "gather4"), (1, "bulk1D")):
                for cps in (2, 3, 4):
                    for ops, R in (((2, 4), (4, 4), (8, 4)) if mode == 0 else ((8, 4), (16, 4), (32, 2))):
                        by = ctypes.c_double(0)
                        ms = L.gather_bw2(B.data_ptr(), K, row, mode, ops, R, 148 * cps, 3000, sink.data_ptr(),
                                          ctypes.byref(by))
                        gbs = by.value / ms / 1e6 if ms > 0 else ms
                        print(f"{tag} row {row:5d} B {name:8s} ctas/SM {cps} ops/stage {ops:2d} R {R}: {gbs:8.0f} GB/s",
                              flush=True)
            del B


if __name__ == "__main__":
    main()
