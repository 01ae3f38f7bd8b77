"""ctypes marshalling for include/dtc.h.  No computation happens here."""
from __future__ import annotations

import ctypes
import os
import re
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.environ.get("DTC_LIBRARY") or os.path.join(_HERE, "libdtc.so")  # override: experiments only
_HEADER = os.path.join(os.path.dirname(_HERE), "include", "dtc.h")

DTC_OK = 0
DTC_ERR_INVALID = -1
DTC_ERR_UNSORTED = -2
DTC_ERR_DUPLICATE = -3
DTC_ERR_RANGE = -4
DTC_ERR_OOM = -5
DTC_ERR_CUDA = -6
DTC_ERR_NCCL = -7
DTC_ERR_UNSUPPORTED = -8
DTC_TF32 = 0
DTC_FP16 = 1

_i64, _i32, _vp = ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p


class _Csr(ctypes.Structure):
    _fields_ = [("M", _i64), ("K", _i64), ("nnz", _i64), ("rowptr", _vp), ("colidx", _vp),
                ("vals", _vp), ("dtype", _i32)]


class _View(ctypes.Structure):
    _fields_ = [("M", _i64), ("K", _i64), ("nnz", _i64), ("num_windows", _i64), ("num_tc_blocks", _i64),
                ("num_units", _i64), ("num_split_windows", _i64), ("dtype", _i32), ("unit_blocks", _i32),
                ("window_rows", _i32),
                ("row_window_offset", _vp), ("tc_offset", _vp), ("tc_local_id", _vp),
                ("sparse_a_to_b", _vp), ("tc_values", _vp), ("units", _vp)]


class _Opts(ctypes.Structure):
    _fields_ = [("unit_blocks", _i32), ("dedup_path", _i32), ("guided", _i32), ("window_order", _i32),
                ("row_perm", _vp), ("n_hint", _i32), ("selector", _i32), ("transpose", _i32),
                ("window_rows", _i32)]


class SchedModel(ctypes.Structure):
    """dtc_sched_model_t: the B200 Selector's launch model."""
    _fields_ = [("num_sms", _i32), ("occupancy", _i32), ("cta_ns", ctypes.c_double), ("block_ns", ctypes.c_double),
                ("fixup_ns", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class _Plan(ctypes.Structure):
    _fields_ = [("unit_blocks", _i32), ("guided", _i32), ("num_units", _i64), ("makespan_ns", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class DtcError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__(f"{where}: {_status_name(status)} ({status}): {detail}")


_lock = threading.Lock()
_lib = None


def library_path() -> str:
    return _SO


def lib():
    """Load libdtc.so; raise loudly if it has not been built (no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(_SO):
                raise ImportError(f"{_SO} is missing: build it with `python -c 'import __graft_entry__ as g; "
                                  f"g.build()'` (there is no CPU fallback)")
            L = ctypes.CDLL(_SO)
            P = ctypes.POINTER
            L.dtc_format_build.argtypes = [P(_Csr), _vp, P(_vp)]
            L.dtc_format_build_ex.argtypes = [P(_Csr), P(_Opts), _vp, P(_vp)]
            L.dtc_format_query.argtypes = [_vp, P(_View)]
            L.dtc_format_export.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp]
            L.dtc_spmm.argtypes = [_vp, _vp, _i64, _i64, _vp, _i64, _vp]
            L.dtc_spmm_host.argtypes = [_vp, _vp, _i64, _i64, _vp, _i64, _vp]
            L.dtc_spmm_launches_per_call.argtypes = []
            L.dtc_spmm_host_async.argtypes = [_vp, _vp, _i64, _i64, _vp, _i64, _vp]
            L.dtc_spmm_host_wait.argtypes = [_vp]
            L.dtc_format_set_option.argtypes = [_vp, _i32, _i64]
            L.dtc_format_get_option.argtypes = [_vp, _i32, _vp]
            L.dtc_format_set_trace.argtypes = [_vp, _vp, _i64]
            L.dtc_format_destroy.argtypes = [_vp]
            L.dtc_format_destroy.restype = None
            L.dtc_partition_windows.argtypes = [_vp, _i64, _i32, _vp]
            L.dtc_graphconv.argtypes = [_vp, _vp, _i64, _vp, _i64, _vp, _i32, _vp, _vp, _vp]
            L.dtc_graphconv_launches_per_call.argtypes = []
            L.dtc_graphconv_backward.argtypes = [_vp, _vp, _vp, _vp, _i64, _i64, _i32, _vp, _vp, _vp, _vp, _vp, _vp,
                                                 _vp, _vp]
            L.dtc_softmax_xent.argtypes = [_vp, _vp, _i64, _i64, _vp, _vp, _vp]
            L.dtc_sgd_update.argtypes = [_vp, _vp, _i64, ctypes.c_float, _vp]
            L.dtc_selector_ar.argtypes = [_vp, _i64, _i32, _i32, _vp, _vp, _vp]
            L.dtc_sched_model.argtypes = [_i32, _i64, P(SchedModel)]
            L.dtc_selector_plan.argtypes = [_vp, _i64, P(SchedModel), _vp, _i32, _i32, _vp, P(_Plan)]
            L.dtc_selector_simulate.argtypes = [_vp, _i64, P(SchedModel), P(ctypes.c_double)]
            L.dtc_tca_reorder.argtypes = [_i64, _i64, _vp, _vp, _i32, _vp]
            L.dtc_tca_reorder_checked.argtypes = [_i64, _i64, _vp, _vp, _i32, _vp, _vp, _vp, _vp]
            L.dtc_nccl_unique_id.argtypes = [_vp]
            L.dtc_dist_create.argtypes = [P(_Csr), _i32, _i32, _vp, _vp, P(_vp)]
            L.dtc_dist_query.argtypes = [_vp, P(_i64), P(_i64), P(_vp)]
            L.dtc_spmm_dist.argtypes = [_vp, _vp, _i32, _i64, _vp, _i32, _vp]
            L.dtc_dist_chunks.argtypes = [_i64, _i64, _i32, _i32, _vp]
            L.dtc_dist_set_chunks.argtypes = [_vp, _i32]
            L.dtc_dist_destroy.argtypes = [_vp]
            L.dtc_dist_destroy.restype = None
            L.dtc_status_string.argtypes = [ctypes.c_int]
            L.dtc_status_string.restype = ctypes.c_char_p
            L.dtc_last_error.argtypes = []
            L.dtc_last_error.restype = ctypes.c_char_p
            L.dtc_version.argtypes = []
            L.dtc_version.restype = ctypes.c_char_p
            _lib = L
    return _lib


def _status_name(st: int) -> str:
    try:
        return lib().dtc_status_string(st).decode()
    except Exception:
        return str(st)


def _check(st: int, where: str):
    if st != DTC_OK:
        raise DtcError(st, where, lib().dtc_last_error().decode())


def exported_symbols() -> list[str]:
    """Function names declared in include/dtc.h."""
    txt = open(_HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(dtc_[a-z0-9_]+)\s*\(", txt)))


def version() -> str:
    return lib().dtc_version().decode()


def launches_per_call() -> int:
    return int(lib().dtc_spmm_launches_per_call())


# per-handle launch options (include/dtc.h dtc_option_t)
OPTIONS = {"kernel": 1, "persistent": 2, "first_records": 3, "host_chunks": 4, "host_zero_copy": 5,
           "slice_bytes": 6, "last_kernel": 100, "last_host_mode": 101, "guided": 102, "plan_makespan_ns": 103}
KERNELS = {"auto": 0, "ldg": 1, "pad": 4}


def _dtype_code(dtype) -> int:
    if dtype in ("tf32", "fp32", DTC_TF32):
        return DTC_TF32
    if dtype in ("fp16", "f16", DTC_FP16):
        return DTC_FP16
    raise ValueError(f"dtype {dtype!r}")


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dptr(t) -> int:
    return 0 if t is None else int(t.data_ptr())


def _make_csr(rowptr, colidx, vals, M, K, dtype) -> _Csr:
    import torch
    code = _dtype_code(dtype)
    for name, t, dt in (("rowptr", rowptr, torch.int32), ("colidx", colidx, torch.int32)):
        if t.dtype != dt or not t.is_cuda or not t.is_contiguous():
            raise TypeError(f"{name} must be a contiguous CUDA int32 tensor")
    want = torch.float16 if code == DTC_FP16 else torch.float32
    if vals.dtype != want or not vals.is_cuda or not vals.is_contiguous():
        raise TypeError(f"vals must be a contiguous CUDA {want} tensor")
    return _Csr(int(M), int(K), int(colidx.numel()), _dptr(rowptr), _dptr(colidx), _dptr(vals), code)


class Format:
    """An ME-TCF handle (library-owned device memory)."""

    def __init__(self, handle: int, keep=(), device: int = 0):
        self._h = ctypes.c_void_p(handle)
        self._keep = keep
        v = self.query()
        self.M, self.K, self.nnz = v.M, v.K, v.nnz
        self.num_windows, self.num_tc_blocks = v.num_windows, v.num_tc_blocks
        self.num_units, self.num_split_windows = v.num_units, v.num_split_windows
        self.unit_blocks = v.unit_blocks
        self.window_rows = v.window_rows
        self.dtype = "fp16" if v.dtype == DTC_FP16 else "tf32"
        self.device = device
        self._trace = None

    @classmethod
    def build(cls, rowptr, colidx, vals, M: int, K: int, dtype="tf32", stream=None,
              unit_blocks: int = 0, dedup_path: int = 0, guided: int = 0, row_perm=None,
              window_order: bool = False, n_hint: int = 0, selector: int = 0,
              transpose: bool = False, window_rows: int = 0) -> "Format":
        """row_perm: optional CUDA int32 tensor [M], new row -> original row (e.g. tca_reorder);
        C is still produced in the original row order.  selector=1 (with unit_blocks=0): F4 cut by
        the B200 Selector's plan for N = n_hint columns (dtc_selector_plan).  transpose=True condenses
        A^T (K x M) from A's CSR (e.g. for the GCN backward).  window_rows=32: the NEXT-2 tall-window
        layout (two 16-row windows share their gathered B rows; TF32)."""
        csr = _make_csr(rowptr, colidx, vals, M, K, dtype)
        h = ctypes.c_void_p()
        if row_perm is not None:
            import torch
            if row_perm.dtype != torch.int32 or not row_perm.is_cuda or row_perm.numel() != M:
                raise TypeError("row_perm must be a CUDA int32 tensor of length M")
        opts = _Opts(int(unit_blocks), int(dedup_path), int(guided), int(bool(window_order)), _dptr(row_perm),
                     int(n_hint), int(selector), int(bool(transpose)), int(window_rows))
        _check(lib().dtc_format_build_ex(ctypes.byref(csr), ctypes.byref(opts), _stream_ptr(stream),
                                         ctypes.byref(h)), "dtc_format_build")
        return cls(h.value, device=rowptr.device.index or 0)

    @property
    def handle(self):
        return self._h

    def query(self) -> _View:
        v = _View()
        _check(lib().dtc_format_query(self._h, ctypes.byref(v)), "dtc_format_query")
        return v

    def export(self) -> dict:
        """Copy the ME-TCF arrays to host numpy arrays (bit-exact checks)."""
        W, T, nnz, nu = self.num_windows, self.num_tc_blocks, self.nnz, self.num_units
        out = {
            "row_window_offset": np.zeros(W + 1, np.int32),
            "tc_offset": np.zeros(T + 1, np.int32),
            "tc_local_id": np.zeros(max(nnz, 1), np.uint8),
            "sparse_a_to_b": np.zeros(max(8 * T, 1), np.int32),
            "tc_values": np.zeros(max(nnz, 1), np.float16 if self.dtype == "fp16" else np.float32),
            "units": np.zeros((max(nu, 1), 8), np.int32),
        }
        p = {k: v.ctypes.data_as(_vp) for k, v in out.items()}
        _check(lib().dtc_format_export(self._h, p["row_window_offset"], p["tc_offset"], p["tc_local_id"],
                                       p["sparse_a_to_b"], p["tc_values"], p["units"]), "dtc_format_export")
        out["tc_local_id"] = out["tc_local_id"][:nnz]
        out["tc_values"] = out["tc_values"][:nnz]
        out["sparse_a_to_b"] = out["sparse_a_to_b"][: 8 * T]
        out["units"] = out["units"][:nu]
        out["num_windows"] = W
        out["num_tc_blocks"] = T
        return out

    def set_option(self, name, value) -> None:
        """Per-handle launch option (dtc_format_set_option): kernel ("auto" | "ldg" | "pad"),
        persistent, first_records, host_chunks, host_zero_copy, slice_bytes."""
        if name == "kernel" and isinstance(value, str):
            value = KERNELS[value]
        _check(lib().dtc_format_set_option(self._h, OPTIONS[name], int(value)), "dtc_format_set_option")

    def get_option(self, name) -> int:
        v = _i64()
        _check(lib().dtc_format_get_option(self._h, OPTIONS[name], ctypes.byref(v)), "dtc_format_get_option")
        return int(v.value)

    def set_trace(self, buf=None) -> None:
        """Enable (CUDA int64 tensor of shape [ctas, 8]) or disable (None) the per-CTA timeline."""
        if buf is None:
            _check(lib().dtc_format_set_trace(self._h, None, 0), "dtc_format_set_trace")
            self._trace = None
            return
        import torch
        if buf.dtype != torch.int64 or not buf.is_cuda or buf.dim() != 2 or buf.shape[1] != 8 or not buf.is_contiguous():
            raise TypeError("trace buffer must be a contiguous CUDA int64 tensor [ctas, 8]")
        _check(lib().dtc_format_set_trace(self._h, ctypes.c_void_p(buf.data_ptr()), buf.shape[0]),
               "dtc_format_set_trace")
        self._trace = buf   # keep it alive while the library may write to it

    def _want(self):
        import torch
        return torch.float16 if self.dtype == "fp16" else torch.float32

    def spmm(self, B, C=None, stream=None):
        """C := A @ B on the GPU (B: CUDA tensor K x N of the handle dtype, row stride ldb)."""
        import torch
        if not isinstance(B, torch.Tensor) or B.dim() != 2 or not B.is_cuda or B.stride(1) != 1:
            raise TypeError("B must be a 2-D CUDA tensor with unit column stride")
        if B.dtype != self._want():
            raise TypeError(f"B must be {self._want()}")
        if B.shape[0] != self.K:
            raise ValueError(f"B must have K = {self.K} rows, got {B.shape[0]}")
        if B.device.index != self.device:
            raise ValueError(f"B is on {B.device}, the handle on cuda:{self.device}")
        N = B.shape[1]
        if C is None:
            C = torch.empty((self.M, N), dtype=torch.float32, device=B.device)
        if (not isinstance(C, torch.Tensor) or C.dtype != torch.float32 or not C.is_cuda or C.dim() != 2
                or C.stride(1) != 1 or C.shape[0] != self.M or C.shape[1] != N):
            raise TypeError("C must be a float32 (M x N) CUDA tensor with unit column stride")
        if C.device.index != self.device:
            raise ValueError(f"C is on {C.device}, the handle on cuda:{self.device}")
        _check(lib().dtc_spmm(self._h, _dptr(B), N, B.stride(0), _dptr(C), C.stride(0), _stream_ptr(stream)),
               "dtc_spmm")
        return C

    def graphconv(self, H, W, bias=None, relu=True, AH=None, Y=None, stream=None):
        """One GCN layer (dtc_graphconv, Eq. (2)): Y = act((A @ H) @ W + b).
        H: CUDA K x F_in (handle dtype), W: CUDA fp32 F_in x F_out, bias fp32 F_out or None.
        Returns (Y, AH); all tensors contiguous row-major."""
        import torch
        want = self._want()
        if H.dtype != want or not H.is_cuda or not H.is_contiguous() or H.dim() != 2:
            raise TypeError(f"H must be a contiguous 2-D CUDA {want} tensor")
        if H.shape[0] != self.K:
            raise ValueError(f"H must have K = {self.K} rows, got {H.shape[0]}")
        F_in, F_out = H.shape[1], W.shape[1]
        if W.dtype != torch.float32 or not W.is_contiguous() or W.shape[0] != F_in:
            raise TypeError("W must be a contiguous fp32 (F_in x F_out) tensor")
        if bias is not None and (bias.dtype != torch.float32 or bias.numel() != F_out or not bias.is_contiguous()):
            raise TypeError("bias must be a contiguous fp32 tensor of F_out elements")
        if AH is None:
            AH = torch.empty((self.M, F_in), dtype=torch.float32, device=H.device)
        if Y is None:
            Y = torch.empty((self.M, F_out), dtype=torch.float32, device=H.device)
        for t, shape in ((AH, (self.M, F_in)), (Y, (self.M, F_out))):
            if t.dtype != torch.float32 or not t.is_contiguous() or tuple(t.shape) != shape:
                raise TypeError(f"workspace/output must be contiguous fp32 {shape}")
        _check(lib().dtc_graphconv(self._h, _dptr(H), F_in, _dptr(W), F_out, _dptr(bias), 1 if relu else 0,
                                   _dptr(AH), _dptr(Y), _stream_ptr(stream)), "dtc_graphconv")
        return Y, AH

    def graphconv_backward(self, AH, W, Y, dY, relu=True, At=None, want_dH=True, bias=True, stream=None):
        """Backward of graphconv (dtc_graphconv_backward): returns dict dW, db (or None), dAH, dH (or None).
        At: the Format of A^T (Format.build(..., transpose=True)), needed for dH."""
        import torch
        M, F_in = AH.shape
        F_out = W.shape[1]
        for name, t, shape in (("AH", AH, (self.M, None)), ("W", W, (F_in, None)), ("Y", Y, (self.M, F_out)),
                               ("dY", dY, (self.M, F_out))):
            _dense(t, name, shape, torch.float32)
        dev = AH.device
        out = {"dZ": torch.empty((self.M, F_out), dtype=torch.float32, device=dev),
               "dW": torch.empty((F_in, F_out), dtype=torch.float32, device=dev),
               "db": torch.empty((F_out,), dtype=torch.float32, device=dev) if bias else None,
               "dAH": torch.empty((self.M, F_in), dtype=torch.float32, device=dev),
               "dH": torch.empty((self.K, F_in), dtype=torch.float32, device=dev) if want_dH else None}
        _check(lib().dtc_graphconv_backward(self._h, At.handle if At is not None else None, _dptr(AH), _dptr(W),
                                            F_in, F_out, 1 if relu else 0, _dptr(Y), _dptr(dY), _dptr(out["dZ"]),
                                            _dptr(out["dW"]), _dptr(out["db"]), _dptr(out["dAH"]), _dptr(out["dH"]),
                                            _stream_ptr(stream)), "dtc_graphconv_backward")
        return out

    def spmm_raw(self, B_ptr: int, N: int, ldb: int, C_ptr: int, ldc: int, stream=None):
        _check(lib().dtc_spmm(self._h, B_ptr, N, ldb, C_ptr, ldc, _stream_ptr(stream)), "dtc_spmm")

    def spmm_host(self, B_host, C_host=None, stream=None):
        """End-to-end C = A @ B with HOST buffers (numpy or pinned torch CPU tensors).  The library
        cannot see host extents, so B (K x N, handle dtype) and C (M x N, float32) are checked here."""
        bp, (K, N), ldb, bdt = _host_ptr(B_host, "B_host")
        want = np.float16 if self.dtype == "fp16" else np.float32
        if bdt != np.dtype(want):
            raise TypeError(f"B_host must be {np.dtype(want)}, got {bdt}")
        if K != self.K:
            raise ValueError(f"B_host must have K = {self.K} rows, got {K}")
        if C_host is None:
            C_host = np.empty((self.M, N), dtype=np.float32)
        cp, (M, Nc), ldc, cdt = _host_ptr(C_host, "C_host")
        if cdt != np.dtype(np.float32) or (M, Nc) != (self.M, N):
            raise TypeError(f"C_host must be float32 of shape ({self.M}, {N}), got {cdt} {(M, Nc)}")
        _check(lib().dtc_spmm_host(self._h, bp, N, ldb, cp, ldc, _stream_ptr(stream)), "dtc_spmm_host")
        return C_host

    def spmm_host_async(self, B_host, C_host, stream=None):
        """Streaming C_host = A @ B_host (dtc_spmm_host_async): returns at once; consecutive calls
        overlap their copies with the previous kernel.  Keep B_host unchanged and do not read C_host
        until wait()."""
        bp, (K, N), ldb, bdt = _host_ptr(B_host, "B_host")
        want = np.float16 if self.dtype == "fp16" else np.float32
        if bdt != np.dtype(want) or K != self.K:
            raise TypeError(f"B_host must be {np.dtype(want)} with K = {self.K} rows")
        cp, (M, Nc), ldc, cdt = _host_ptr(C_host, "C_host")
        if cdt != np.dtype(np.float32) or (M, Nc) != (self.M, N):
            raise TypeError(f"C_host must be float32 of shape ({self.M}, {N})")
        _check(lib().dtc_spmm_host_async(self._h, bp, N, ldb, cp, ldc, _stream_ptr(stream)), "dtc_spmm_host_async")
        return C_host

    def wait(self):
        """Wait for every spmm_host_async call of this handle (dtc_spmm_host_wait)."""
        _check(lib().dtc_spmm_host_wait(self._h), "dtc_spmm_host_wait")

    def close(self):
        if self._h is not None and self._h.value:
            lib().dtc_format_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _host_ptr(a, name):
    """(pointer, shape, row stride in elements, numpy dtype) of a 2-D host buffer with unit column stride."""
    if isinstance(a, np.ndarray):
        if a.ndim != 2 or a.strides[1] != a.itemsize or a.strides[0] % a.itemsize or a.strides[0] < 0:
            raise TypeError(f"{name} must be a 2-D array with unit column stride")
        return a.ctypes.data, a.shape, a.strides[0] // a.itemsize, a.dtype
    import torch
    if not isinstance(a, torch.Tensor) or a.is_cuda or a.dim() != 2 or a.stride(1) != 1:
        raise TypeError(f"{name} must be a 2-D host array/tensor with unit column stride")
    dt = {torch.float32: np.dtype(np.float32), torch.float16: np.dtype(np.float16)}.get(a.dtype, None)
    if dt is None:
        raise TypeError(f"{name} has unsupported dtype {a.dtype}")
    return a.data_ptr(), tuple(a.shape), a.stride(0), dt


def _dense(t, name, shape, dtype):
    """Raise unless t is a contiguous 2-D CUDA tensor of `dtype` whose shape matches (None = any)."""
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dim() != 2 or not t.is_contiguous():
        raise TypeError(f"{name} must be a contiguous 2-D CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    for got, want in zip(t.shape, shape):
        if want is not None and got != want:
            raise ValueError(f"{name} must have shape {shape}, got {tuple(t.shape)}")


def partition_windows(rwo, world: int) -> np.ndarray:
    """Host-side window partition by TC-block prefix (dtc_partition_windows)."""
    rwo = np.ascontiguousarray(rwo, dtype=np.int32)
    out = np.zeros(world + 1, dtype=np.int64)
    _check(lib().dtc_partition_windows(rwo.ctypes.data_as(_vp), len(rwo) - 1, world, out.ctypes.data_as(_vp)),
           "dtc_partition_windows")
    return out


def selector_ar(rwo, num_sms: int = 148, occupancy: int = 6) -> dict:
    """Simulation-based Selector diagnostic (dtc_selector_ar): makespans of the
    one-block-per-window kernel and of strict balance, and AR = their ratio (> 1.2: balance pays)."""
    rwo = np.ascontiguousarray(rwo, dtype=np.int32)
    out = np.zeros(3, dtype=np.float64)
    a = out.ctypes.data
    _check(lib().dtc_selector_ar(rwo.ctypes.data_as(_vp), len(rwo) - 1, num_sms, occupancy,
                                 ctypes.c_void_p(a), ctypes.c_void_p(a + 8), ctypes.c_void_p(a + 16)),
           "dtc_selector_ar")
    return {"makespan_base": float(out[0]), "makespan_balanced": float(out[1]), "ar": float(out[2]),
            "num_sms": num_sms, "occupancy": occupancy}


def softmax_xent(logits, labels, stream=None):
    """(loss as a 1-element CUDA tensor, dlogits) of the mean softmax cross-entropy (dtc_softmax_xent)."""
    import torch
    _dense(logits, "logits", (None, None), torch.float32)
    if labels.dtype != torch.int32 or not labels.is_cuda or labels.numel() != logits.shape[0]:
        raise TypeError("labels must be a CUDA int32 tensor with one entry per row")
    loss = torch.empty((1,), dtype=torch.float32, device=logits.device)
    dz = torch.empty_like(logits)
    _check(lib().dtc_softmax_xent(_dptr(logits), _dptr(labels), logits.shape[0], logits.shape[1], _dptr(loss),
                                  _dptr(dz), _stream_ptr(stream)), "dtc_softmax_xent")
    return loss, dz


def sgd_update(param, grad, lr: float, stream=None):
    """param -= lr * grad (dtc_sgd_update), in place."""
    import torch
    if param.dtype != torch.float32 or grad.dtype != torch.float32 or param.numel() != grad.numel() \
            or not param.is_contiguous() or not grad.is_contiguous():
        raise TypeError("param and grad must be contiguous fp32 tensors of equal size")
    _check(lib().dtc_sgd_update(_dptr(param), _dptr(grad), param.numel(), float(lr), _stream_ptr(stream)),
           "dtc_sgd_update")


class GCN2:
    """Two GraphConv layers (Eq. (2)) trained with softmax cross-entropy and SGD, every
    step through the library: H1 = ReLU((A X) W1 + b1), Z = (A H1) W2 + b2, loss = xent(Z, labels);
    backward dtc_graphconv_backward x 2 (the second needs A^T for dH1), dtc_sgd_update x 4.  This
    class only sequences C ABI calls (no arithmetic here)."""

    def __init__(self, A, At, F_in: int, F_hid: int, n_classes: int, seed: int = 0):
        import torch
        if A.dtype != "tf32" or At.dtype != "tf32" or At.M != A.K or At.K != A.M:
            raise ValueError("GCN2 needs a TF32 handle of A and of A^T")
        dev = torch.device("cuda", A.device)
        g = torch.Generator(device=dev).manual_seed(seed)
        s1, s2 = (6.0 / (F_in + F_hid)) ** 0.5, (6.0 / (F_hid + n_classes)) ** 0.5
        self.A, self.At = A, At
        self.W1 = torch.empty((F_in, F_hid), device=dev).uniform_(-s1, s1, generator=g)
        self.b1 = torch.zeros((F_hid,), device=dev)
        self.W2 = torch.empty((F_hid, n_classes), device=dev).uniform_(-s2, s2, generator=g)
        self.b2 = torch.zeros((n_classes,), device=dev)

    def forward(self, X):
        Y1, AH1 = self.A.graphconv(X, self.W1, self.b1, relu=True)
        Z, AH2 = self.A.graphconv(Y1, self.W2, self.b2, relu=False)
        return Z, (Y1, AH1, AH2)

    def train_step(self, X, labels, lr: float):
        """One SGD step; returns the loss (1-element CUDA tensor, computed before the update)."""
        Z, (Y1, AH1, AH2) = self.forward(X)
        loss, dZ = softmax_xent(Z, labels)
        g2 = self.A.graphconv_backward(AH2, self.W2, Z, dZ, relu=False, At=self.At, want_dH=True)
        g1 = self.A.graphconv_backward(AH1, self.W1, Y1, g2["dH"], relu=True, want_dH=False)
        for p, gr in ((self.W2, g2["dW"]), (self.b2, g2["db"]), (self.W1, g1["dW"]), (self.b1, g1["db"])):
            sgd_update(p, gr, lr)
        return loss


def sched_model(dtype="tf32", N: int = 128) -> SchedModel:
    """The default B200 launch model for dtype and N on the current device (dtc_sched_model)."""
    m = SchedModel()
    _check(lib().dtc_sched_model(_dtype_code(dtype), int(N), ctypes.byref(m)), "dtc_sched_model")
    return m


def make_model(num_sms: int, occupancy: int, cta_ns: float, block_ns: float, fixup_ns: float) -> SchedModel:
    return SchedModel(int(num_sms), int(occupancy), float(cta_ns), float(block_ns), float(fixup_ns))


def selector_plan(rwo, model: SchedModel, candidates=None, guided: int = 0) -> dict:
    """B200 Selector (dtc_selector_plan): every candidate plan's simulated makespan and the best."""
    rwo = np.ascontiguousarray(rwo, dtype=np.int32)
    cand = None if candidates is None else np.ascontiguousarray(candidates, dtype=np.int32)
    nc = 11 if cand is None else len(cand)
    plans = (_Plan * (2 * nc))()
    best = _Plan()
    _check(lib().dtc_selector_plan(rwo.ctypes.data_as(_vp), len(rwo) - 1, ctypes.byref(model),
                                   None if cand is None else cand.ctypes.data_as(_vp), 0 if cand is None else nc,
                                   int(guided), ctypes.cast(plans, _vp), ctypes.byref(best)), "dtc_selector_plan")
    return {"best": best.as_dict(), "plans": [p.as_dict() for p in plans]}


def selector_simulate(units, model: SchedModel) -> float:
    """Simulated makespan (ns) of an explicit unit list [nu, 8] (dtc_selector_simulate)."""
    u = np.ascontiguousarray(units, dtype=np.int32).reshape(-1, 8)
    out = ctypes.c_double()
    _check(lib().dtc_selector_simulate(u.ctypes.data_as(_vp), len(u), ctypes.byref(model), ctypes.byref(out)),
           "dtc_selector_simulate")
    return float(out.value)


def selector_report(rwo, num_sms: int = 148, dtype="tf32", N: int = 128, occupancy_paper: int = 6) -> dict:
    """The paper's AR (Eq. (1) model) and the B200 Selector's plan for this RowWindowOffset."""
    ar = selector_ar(rwo, num_sms, occupancy_paper)
    m = sched_model(dtype, N)
    plan = selector_plan(rwo, m)
    return {"paper_ar": round(ar["ar"], 3), "paper_rule_balanced": ar["ar"] > 1.2, "model": m.as_dict(),
            "plan": plan["best"],
            "candidates": {f"U{p['unit_blocks']}{'g' if p['guided'] else ''}": round(p["makespan_ns"] / 1e3, 2)
                           for p in plan["plans"] if p["makespan_ns"] >= 0}}


def tca_reorder(M: int, K: int, rowptr, colidx, sm_num: int = 148) -> np.ndarray:
    """TCA row reordering (dtc_tca_reorder, host): perm[new_row] = original row."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int32)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    perm = np.zeros(max(M, 1), dtype=np.int32)
    _check(lib().dtc_tca_reorder(M, K, rowptr.ctypes.data_as(_vp), colidx.ctypes.data_as(_vp), sm_num,
                                 perm.ctypes.data_as(_vp)), "dtc_tca_reorder")
    return perm[:M]


def tca_reorder_checked(M: int, K: int, rowptr, colidx, sm_num: int = 148):
    """TCA reordering kept only when it lowers NumTCBlock (dtc_tca_reorder_checked):
    returns (perm, {"T_identity", "T_reordered", "applied"})."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int32)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    perm = np.zeros(max(M, 1), dtype=np.int32)
    t0, t1, ap = _i64(), _i64(), _i32()
    _check(lib().dtc_tca_reorder_checked(M, K, rowptr.ctypes.data_as(_vp), colidx.ctypes.data_as(_vp), sm_num,
                                         perm.ctypes.data_as(_vp), ctypes.byref(t0), ctypes.byref(t1),
                                         ctypes.byref(ap)), "dtc_tca_reorder_checked")
    return perm[:M], {"T_identity": t0.value, "T_reordered": t1.value, "applied": bool(ap.value)}


def dist_chunks(K: int, N: int, elt: int, max_chunks: int = 0) -> np.ndarray:
    """Column chunk boundaries of dtc_spmm_dist's pipelined broadcast (dtc_dist_chunks, host)."""
    out = np.zeros(9, dtype=np.int64)
    n = lib().dtc_dist_chunks(int(K), int(N), int(elt), int(max_chunks), out.ctypes.data_as(_vp))
    if n < 1:
        _check(n, "dtc_dist_chunks")
    return out[: n + 1]


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().dtc_nccl_unique_id(buf), "dtc_nccl_unique_id")
    return buf.raw


class Dist:
    """One rank's share of a row-window-partitioned SpMM (dtc_dist_*)."""

    def __init__(self, rowptr, colidx, vals, M, K, dtype, rank: int, world: int, nccl_id: bytes | None,
                 stream=None):
        csr = _make_csr(rowptr, colidx, vals, M, K, dtype)
        h = ctypes.c_void_p()
        idbuf = ctypes.create_string_buffer(nccl_id, 128) if nccl_id is not None else None
        _check(lib().dtc_dist_create(ctypes.byref(csr), rank, world, idbuf, _stream_ptr(stream), ctypes.byref(h)),
               "dtc_dist_create")
        self._h = h
        self.M, self.K, self.rank, self.world = M, K, rank, world
        self.dtype = "fp16" if _dtype_code(dtype) == DTC_FP16 else "tf32"
        rb, re_, loc = _i64(), _i64(), _vp()
        _check(lib().dtc_dist_query(self._h, ctypes.byref(rb), ctypes.byref(re_), ctypes.byref(loc)),
               "dtc_dist_query")
        self.row_begin, self.row_end = rb.value, re_.value
        self._local = loc

    def _want(self):
        import torch
        return torch.float16 if self.dtype == "fp16" else torch.float32

    def local_spmm(self, B, C_local, stream=None):
        """This rank's rows only, B already resident (no collective): C_local = A[rows] @ B."""
        import torch
        _dense(B, "B", (self.K, None), self._want())
        N = B.shape[1]
        _dense(C_local, "C_local", (max(self.row_end - self.row_begin, 1), N), torch.float32)
        _check(lib().dtc_spmm(self._local, _dptr(B), N, N, _dptr(C_local), N, _stream_ptr(stream)), "dtc_spmm")
        return C_local

    def set_chunks(self, chunks: int) -> None:
        """Column chunks of the pipelined broadcast (dtc_dist_set_chunks): 0 = auto, 1 = unpipelined."""
        _check(lib().dtc_dist_set_chunks(self._h, int(chunks)), "dtc_dist_set_chunks")

    def spmm(self, B, C, root: int = 0, gather_c: bool = True, stream=None, N: int | None = None):
        """dtc_spmm_dist: B (K x N) is read on root only (None elsewhere, then pass N) and broadcast in
        column chunks pipelined with the kernel; C is M x N (gather_c) or this rank's rows."""
        import torch
        if B is not None:
            _dense(B, "B", (self.K, None), self._want())
            N = B.shape[1]
        elif N is None or self.rank == root:
            raise ValueError("B is required on the root (elsewhere pass N)")
        rows = self.M if gather_c else max(self.row_end - self.row_begin, 1)
        _dense(C, "C", (rows, N), torch.float32)
        _check(lib().dtc_spmm_dist(self._h, _dptr(B), root, N, _dptr(C), int(gather_c), _stream_ptr(stream)),
               "dtc_spmm_dist")
        return C

    def close(self):
        if self._h is not None and self._h.value:
            lib().dtc_dist_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
