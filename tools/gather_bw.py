"""Run the row-gather microbenchmark (tools/gather_bw.cu) on the GPU box."""
import ctypes
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libgather_bw.so")


def build():
    subprocess.check_call(["nvcc", "-O3", "-shared", "-Xcompiler", "-fPIC", "-gencode", "arch=compute_100a,code=sm_100a",
                           os.path.join(HERE, "gather_bw.cu"), "-o", SO])


def main():
    import torch
    if not os.path.exists(SO):
        build()
    L = ctypes.CDLL(SO)
    L.gather_bw.restype = ctypes.c_float
    L.gather_bw.argtypes = [ctypes.c_int, ctypes.c_void_p] + [ctypes.c_int] * 9 + [ctypes.c_void_p,
                                                                                       ctypes.POINTER(ctypes.c_double)]
    for K, ldb, tag in [(2_000_000, 128, "B=1GB (DRAM)"), (150_000, 128, "B=77MB (L2-resident)")]:
        B = torch.randn(K, ldb, device="cuda")
        sink = torch.zeros(4, dtype=torch.int32, device="cuda")
        print(f"--- {tag}")

        def run(mode, box=32, sw=1, ops=8, R=8, ctas=148 * 4, threads=128, iters=4000):
            by = ctypes.c_double(0)
            ms = L.gather_bw(mode, B.data_ptr(), K, ldb, box, sw, ops, R, ctas, threads, iters, sink.data_ptr(),
                             ctypes.byref(by))
            return by.value / ms / 1e6 if ms > 0 else -1

        for ctas_per_sm in (1, 2, 4):
            for ops, R in ((2, 16), (8, 8), (16, 8), (32, 4)):
                print(f"TMA box32 sw128 ctas/SM={ctas_per_sm} ops/stage={ops} R={R}: "
                      f"{run(0, 32, 1, ops, R, 148 * ctas_per_sm, 64, 2000):.0f} GB/s")
            for ops, R in ((2, 8), (8, 4)):
                print(f"TMA box128 nosw ctas/SM={ctas_per_sm} ops/stage={ops} R={R}: "
                      f"{run(0, 128, 0, ops, R, 148 * ctas_per_sm, 64, 2000):.0f} GB/s")
        for mode, name in ((1, "LDG frag-order"), (2, "LDG coalesced"), (3, "cp.async coalesced")):
            for warps in (4, 8, 16):
                for cps in (2, 4, 8):
                    if mode == 3 and warps * cps * 8 > 200:
                        continue
                    print(f"{name} warps/CTA={warps} ctas/SM={cps}: "
                          f"{run(mode, ctas=148 * cps, threads=32 * warps, iters=2000):.0f} GB/s")


if __name__ == "__main__":
    main()
