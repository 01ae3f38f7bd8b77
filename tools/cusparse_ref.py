"""ctypes wrapper for the cuSPARSE comparator (bench only)."""
import ctypes
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libcusparse_ref.so")
ALGS = {"ALG_DEFAULT": 0, "CSR_ALG1": 1, "CSR_ALG2": 2, "CSR_ALG3": 3}
_lib = None


def build(force=False):
    src = os.path.join(HERE, "cusparse_ref.cu")
    if force or not os.path.exists(SO) or os.path.getmtime(SO) < os.path.getmtime(src):
        subprocess.check_call(["nvcc", "-O2", "-shared", "-Xcompiler", "-fPIC", "-gencode",
                               "arch=compute_100a,code=sm_100a", src, "-o", SO, "-lcusparse"])
    return SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(SO)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.cusp_create.argtypes = [i64, i64, i64, vp, vp, vp, ctypes.c_int, vp, i64, vp, ctypes.c_int, vp,
                                  ctypes.POINTER(ctypes.c_int)]
        L.cusp_create.restype = vp
        L.cusp_run.argtypes = [vp]
        L.cusp_run.restype = ctypes.c_int
        L.cusp_destroy.argtypes = [vp]
        L.cusp_destroy.restype = None
        _lib = L
    return _lib


class CuSparseSpMM:
    def __init__(self, M, K, rowptr, colidx, vals, B, C, alg="ALG_DEFAULT", stream=None):
        import torch
        st = ctypes.c_int(0)
        s = (stream or torch.cuda.current_stream()).cuda_stream
        self._h = lib().cusp_create(M, K, colidx.numel(), rowptr.data_ptr(), colidx.data_ptr(), vals.data_ptr(),
                                    int(vals.dtype == torch.float16), B.data_ptr(), B.shape[1], C.data_ptr(),
                                    ALGS[alg], s, ctypes.byref(st))
        self.status = st.value
        self.ok = bool(self._h)

    def run(self):
        rc = lib().cusp_run(self._h)
        if rc != 0:
            raise RuntimeError(f"cusparseSpMM status {rc}")

    def close(self):
        if self._h:
            lib().cusp_destroy(self._h)
        self._h = None
