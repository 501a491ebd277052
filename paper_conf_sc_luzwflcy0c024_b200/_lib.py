"""ctypes binding of libamgt.so (include/amgt.h) — argument marshalling only.

Every computation runs in the library's CUDA kernels.  torch supplies device memory
(the caching allocator is handed to the library as its amgt_allocator), the current
stream, and tensor views of library-owned arrays.  There is no CPU fallback: if
libamgt.so is missing this module raises on import.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AMGT_LIB_PATH") or os.path.join(_HERE, "libamgt.so")  # override: kernel experiments

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built — run `python __graft_entry__.py build` "
                      "(there is no CPU fallback for the AmgT kernels)")
_L = ctypes.CDLL(LIB_PATH)

FP64, FP32, FP16 = 0, 1, 2
PREC = {"f64": FP64, "f32": FP32, "f16": FP16, FP64: FP64, FP32: FP32, FP16: FP16}
PREC_DTYPE = {FP64: torch.float64, FP32: torch.float32, FP16: torch.float16}
PREC_NAME = {FP64: "f64", FP32: "f32", FP16: "f16"}
STATUS = {0: "OK", 1: "ERR_ARG", 2: "ERR_FORMAT", 3: "ERR_ALLOC", 4: "ERR_CUDA", 5: "ERR_NCCL", 6: "ERR_RANGE",
          7: "ERR_UNSUPPORTED"}


class AmgtError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class c_mbsr(ctypes.Structure):
    _fields_ = [("m", ctypes.c_int64), ("n", ctypes.c_int64), ("blc_row", ctypes.c_int64),
                ("blc_col", ctypes.c_int64), ("blc_num", ctypes.c_int64), ("blc_ptr", ctypes.c_void_p),
                ("blc_idx", ctypes.c_void_p), ("blc_map", ctypes.c_void_p), ("blc_val", ctypes.c_void_p),
                ("prec", ctypes.c_int), ("own", ctypes.c_uint32), ("aux", ctypes.c_void_p),
                ("row_max", ctypes.c_int64)]


_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)


class c_allocator(ctypes.Structure):
    _fields_ = [("alloc", _ALLOC_FN), ("free", _FREE_FN), ("ctx", ctypes.c_void_p)]


class c_spgemm_info(ctypes.Structure):
    _fields_ = [("bin_rows", ctypes.c_int64 * 8), ("cub_total", ctypes.c_int64), ("pairs_nonzero", ctypes.c_int64),
                ("pairs_tc", ctypes.c_int64), ("scalar_products", ctypes.c_int64),
                ("numeric_rows", ctypes.c_int64 * 3)]

    def as_dict(self):
        return {"bin_rows": list(self.bin_rows), "cub_total": self.cub_total, "pairs_nonzero": self.pairs_nonzero,
                "pairs_tc": self.pairs_tc, "scalar_products": self.scalar_products,
                "numeric_rows": list(self.numeric_rows)}


class c_spmv_stats(ctypes.Structure):
    _fields_ = [("avg_nnz_blc", ctypes.c_double), ("variation", ctypes.c_double), ("long_rows", ctypes.c_int64),
                ("chunks", ctypes.c_int64), ("tc_tiles", ctypes.c_int64)]


class c_vcycle_opts(ctypes.Structure):
    _fields_ = [("max_levels", ctypes.c_int), ("nu1", ctypes.c_int), ("nu2", ctypes.c_int), ("omega", ctypes.c_double),
                ("level_prec", ctypes.c_int * 8), ("smoother", ctypes.c_int), ("interp", ctypes.c_int),
                ("theta", ctypes.c_double), ("omega_p", ctypes.c_double), ("max_coarse_size", ctypes.c_int),
                ("max_row_sum", ctypes.c_double), ("seed", ctypes.c_uint64)]


class c_dist_piece(ctypes.Structure):
    _fields_ = [("peer", ctypes.c_int32), ("begin", ctypes.c_int64), ("end", ctypes.c_int64)]


class c_dist_hier_info(ctypes.Structure):
    _fields_ = [("nlev", ctypes.c_int), ("agg_level", ctypes.c_int), ("rows", ctypes.c_int64 * 8),
                ("tiles", ctypes.c_int64 * 8), ("row_begin", ctypes.c_int64 * 8), ("ext_begin", ctypes.c_int64 * 8),
                ("ext_end", ctypes.c_int64 * 8), ("halo_recv", ctypes.c_int * 8), ("halo_send", ctypes.c_int * 8),
                ("interior", (ctypes.c_int64 * 2) * 8)]


class c_sweep_stage(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int), ("x", ctypes.c_void_p), ("y", ctypes.c_void_p)]


_vp, _i64, _i32, _int = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_int
_P = ctypes.POINTER
_sigs = {
    "amgt_last_error": (ctypes.c_char_p, []),
    "amgt_version": (ctypes.c_char_p, []),
    "amgt_csr_to_mbsr": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _int, _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_mbsr_nnz": (_int, [_P(c_mbsr), _P(_i64), _vp]),
    "amgt_mbsr_to_csr": (_int, [_P(c_mbsr), _vp, _vp, _vp, _vp]),
    "amgt_mbsr_cast": (_int, [_P(c_mbsr), _int, _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_mbsr_free": (_int, [_P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_mbsr_transpose": (_int, [_P(c_mbsr), _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_mbsr_wrap": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _vp, _int, _P(c_mbsr)]),
    "amgt_spgemm_symbolic": (_int, [_P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _P(c_spgemm_info), _P(c_allocator), _vp]),
    "amgt_spgemm_numeric": (_int, [_P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _vp]),
    "amgt_set_tc_threshold": (_int, [_int, _int]),
    "amgt_rap": (_int, [_P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_spmv_analyze": (_int, [_P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_spmv_get_stats": (_int, [_P(c_mbsr), _P(c_spmv_stats)]),
    "amgt_spmv": (_int, [_P(c_mbsr), _vp, _int, _vp, _int, _vp]),
    "amgt_spmv_fused": (_int, [_P(c_mbsr), _vp, _int, _vp, _int, _int, _vp, _vp, ctypes.c_double, _vp]),
    "amgt_pcg": (_int, [_vp, _vp, _vp, _int, ctypes.c_double, _vp, _P(ctypes.c_int), _P(ctypes.c_int64), _vp]),
    "amgt_spmv_fused_r": (_int, [_P(c_mbsr), _vp, _int, _vp, _int, _vp, _vp, ctypes.c_double, _vp, _vp]),
    "amgt_hierarchy_create": (_int, [_P(c_mbsr), _P(_P(c_mbsr)), _int, _P(c_vcycle_opts), _P(c_allocator), _vp,
                                     _P(_vp)]),
    "amgt_hierarchy_level": (_int, [_vp, _int, _P(_P(c_mbsr)), _P(_P(c_mbsr)), _P(_P(c_mbsr))]),
    "amgt_hierarchy_nlev": (_int, [_vp]),
    "amgt_vcycle": (_int, [_vp, _vp, _vp, _int, _P(ctypes.c_double), _P(_i64), _vp]),
    "amgt_hierarchy_destroy": (_int, [_vp]),
    "amgt_timing_enable": (_int, [_int]),
    "amgt_timing_reset": (_int, []),
    "amgt_timing_sample": (_int, [_int]),
    "amgt_timing_read": (_int, [_P(ctypes.c_double), _P(_i64), _P(ctypes.c_double)]),
    "amgt_launch_count": (_i64, []),
    "amgt_spmv_fused_range": (_int, [_P(c_mbsr), _i64, _i64, _vp, _int, _vp, _int, _int, _vp, _vp, _vp, ctypes.c_double,
                                     _vp]),
    "amgt_csr_to_mbsr_ex": (_int, [_i64, _i64, _i64, _vp, _vp, _vp, _i64, _int, _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_mbsr_shift_cols": (_int, [_P(c_mbsr), _i64, _i64, _vp]),
    "amgt_csr_col_range": (_int, [_i64, _vp, _vp, _i64, _P(_i64), _vp]),
    "amgt_mbsr_col_range": (_int, [_P(c_mbsr), _i64, _P(_i64), _vp]),
    "amgt_dinv": (_int, [_P(c_mbsr), _i64, _vp, _int, _vp]),
    "amgt_dense_spd_inverse": (_int, [_i64, _vp, _vp]),
    "amgt_dense_matvec": (_int, [_i64, _i64, _vp, _vp, _vp, _int, _vp]),
    "amgt_norm2sq": (_int, [_i64, _vp, _vp, _vp]),
    "amgt_sweep_plan_create": (_int, [_P(c_mbsr), _P(c_allocator), _vp, _P(_vp)]),
    "amgt_sweep_plan_destroy": (_int, [_vp, _vp]),
    "amgt_sweep_plan_stats": (_int, [_vp, _vp, _vp]),
    "amgt_spmv_sweeps": (_int, [_vp, _P(c_mbsr), _int, _P(c_sweep_stage), _vp, _vp, ctypes.c_double, _vp, _vp]),
    "amgt_strength_filter": (_int, [_P(c_mbsr), ctypes.c_double, ctypes.c_double, _P(c_mbsr), _vp, _P(c_allocator),
                                     _vp]),
    "amgt_sa_interp": (_int, [_P(c_mbsr), _P(c_mbsr), ctypes.c_double, ctypes.c_double, _P(c_mbsr), _P(c_allocator),
                               _vp]),
    "amgt_pmis_aggregate": (_int, [_P(c_mbsr), ctypes.c_double, ctypes.c_double, _vp, ctypes.c_uint64, _int, _vp, _vp,
                                   _P(_i64), _P(_int), _vp]),
    "amgt_aggregation_p": (_int, [_i64, _i64, _vp, _int, _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_nccl_unique_id": (_int, [_vp]),
    "amgt_dist_create": (_int, [_vp, _int, _int, _i64, _i64, _P(_vp)]),
    "amgt_dist_group_create": (_int, [_int, _P(_vp)]),
    "amgt_dist_group_destroy": (_int, [_vp]),
    "amgt_dist_group_abort": (_int, [_vp]),
    "amgt_dist_create_loopback": (_int, [_vp, _int, _i64, _i64, _P(_vp)]),
    "amgt_dist_destroy": (_int, [_vp]),
    "amgt_dist_allreduce_sum": (_int, [_vp, _vp, _i64, _vp]),
    "amgt_dist_spmv": (_int, [_vp, _P(c_mbsr), _vp, _vp, _vp]),
    "amgt_dist_rap": (_int, [_vp, _P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_dist_allgather_mbsr": (_int, [_vp, _P(c_mbsr), _P(c_mbsr), _P(c_allocator), _vp]),
    "amgt_dist_hierarchy_create": (_int, [_vp, _P(c_mbsr), _P(_P(c_mbsr)), _int, _P(c_vcycle_opts), _i64,
                                          _P(c_allocator), _vp, _P(_vp)]),
    "amgt_dist_vcycle": (_int, [_vp, _vp, _vp, _int, _P(ctypes.c_double), _P(_i64), _vp]),
    "amgt_dist_hierarchy_info": (_int, [_vp, _P(c_dist_hier_info)]),
    "amgt_dist_hierarchy_destroy": (_int, [_vp]),
    "amgt_dist_plan_host": (_int, [_int, _int, _vp, _vp, _vp, _vp, _P(c_dist_piece), _P(_int), _P(c_dist_piece),
                                   _P(_int), _int]),
}
for _name, (_res, _args) in _sigs.items():
    _f = getattr(_L, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_sigs)


def _check(st: int):
    if st != 0:
        raise AmgtError(st, _L.amgt_last_error().decode(errors="replace"))


def version() -> str:
    return _L.amgt_version().decode()


def _stream(stream=None) -> int:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


# ------------------------------------------------------------------ allocator (torch caching allocator)
_live: dict[int, int] = {}


_ext_streams: dict[int, "torch.cuda.ExternalStream"] = {}  # stream handle -> wrapper (built once)


@_ALLOC_FN
def _torch_alloc(nbytes, stream, ctx):
    try:
        st = None
        if stream:
            st = _ext_streams.get(stream)
            if st is None:
                st = _ext_streams[stream] = torch.cuda.ExternalStream(stream)
        p = torch.cuda.caching_allocator_alloc(int(nbytes), st.device_index if st is not None else
                                               torch.cuda.current_device(), st)
        _live[p] = int(nbytes)
        return p
    except Exception:  # allocation failure is reported by the library as AMGT_ERR_ALLOC
        return None


@_FREE_FN
def _torch_free(p, nbytes, stream, ctx):
    if p:
        _live.pop(p, None)
        torch.cuda.caching_allocator_delete(p)


ALLOCATOR = c_allocator(_torch_alloc, _torch_free, None)
_AL = ctypes.byref(ALLOCATOR)


class _DevView:
    """__cuda_array_interface__ for a library-owned device array (keeps its owner alive)."""

    def __init__(self, owner, ptr: int, n: int, typestr: str):
        self.owner = owner
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr, "data": (int(ptr or 0), False),
                                         "version": 3, "strides": None, "stream": None}


def _view(owner, ptr, n, dtype) -> torch.Tensor:
    if n == 0 or not ptr:
        return torch.empty(0, dtype=dtype, device="cuda")
    ts = {torch.int64: "<i8", torch.int32: "<i4", torch.int16: "<i2", torch.float64: "<f8", torch.float32: "<f4",
          torch.float16: "<f2"}[dtype]
    return torch.as_tensor(_DevView(owner, ptr, n, ts), device="cuda")


# ------------------------------------------------------------------ mBSR handle
class Mbsr:
    """An mBSR matrix in device memory (library-owned arrays, torch-allocated)."""

    def __init__(self, c: c_mbsr | None = None, keep=()):
        self.c = c if c is not None else c_mbsr()
        self._keep = list(keep)  # tensors this matrix borrows from

    # -- properties
    m = property(lambda s: s.c.m)
    n = property(lambda s: s.c.n)
    blc_row = property(lambda s: s.c.blc_row)
    blc_col = property(lambda s: s.c.blc_col)
    blc_num = property(lambda s: s.c.blc_num)
    prec = property(lambda s: s.c.prec)

    @property
    def blc_ptr(self):
        return _view(self, self.c.blc_ptr, self.c.blc_row + 1, torch.int64)

    @property
    def blc_idx(self):
        return _view(self, self.c.blc_idx, self.c.blc_num, torch.int32)

    @property
    def blc_map(self):
        """uint16 bitmaps (returned as int16 storage; use .to(torch.int32) & 0xFFFF)."""
        return _view(self, self.c.blc_map, self.c.blc_num, torch.int16)

    @property
    def blc_val(self):
        return _view(self, self.c.blc_val, 16 * self.c.blc_num, PREC_DTYPE[self.c.prec])

    def map_u16(self) -> torch.Tensor:
        return self.blc_map.to(torch.int32) & 0xFFFF

    def free(self):
        if self.c.own or self.c.aux:
            _check(_L.amgt_mbsr_free(ctypes.byref(self.c), _AL, _stream()))
        self.c = c_mbsr()

    def __del__(self):
        try:
            if self.c.own or self.c.aux:
                torch.cuda.synchronize()
                _L.amgt_mbsr_free(ctypes.byref(self.c), _AL, _stream())
        except Exception:
            pass

    # -- operations
    def nnz(self, stream=None) -> int:
        v = ctypes.c_int64(0)
        _check(_L.amgt_mbsr_nnz(ctypes.byref(self.c), ctypes.byref(v), _stream(stream)))
        return int(v.value)

    def to_csr(self, stream=None):
        nnz = self.nnz(stream)
        rp = torch.empty(self.m + 1, dtype=torch.int64, device="cuda")
        ci = torch.empty(max(nnz, 1), dtype=torch.int32, device="cuda")
        v = torch.empty(max(nnz, 1), dtype=torch.float64, device="cuda")
        _check(_L.amgt_mbsr_to_csr(ctypes.byref(self.c), rp.data_ptr(), ci.data_ptr(), v.data_ptr(), _stream(stream)))
        return rp, ci[:nnz], v[:nnz]

    def cast(self, prec, stream=None) -> "Mbsr":
        out = Mbsr(keep=[self])
        _check(_L.amgt_mbsr_cast(ctypes.byref(self.c), PREC[prec], ctypes.byref(out.c), _AL, _stream(stream)))
        return out

    def transpose(self, stream=None) -> "Mbsr":
        out = Mbsr()
        _check(_L.amgt_mbsr_transpose(ctypes.byref(self.c), ctypes.byref(out.c), _AL, _stream(stream)))
        return out

    def analyze(self, stream=None) -> "Mbsr":
        _check(_L.amgt_spmv_analyze(ctypes.byref(self.c), _AL, _stream(stream)))
        return self

    def spmv_stats(self) -> dict:
        st = c_spmv_stats()
        _check(_L.amgt_spmv_get_stats(ctypes.byref(self.c), ctypes.byref(st)))
        return {k: getattr(st, k) for k, _ in c_spmv_stats._fields_}


def csr_to_mbsr(m, n, row_ptr: torch.Tensor, col: torch.Tensor, val: torch.Tensor, prec="f64", stream=None) -> Mbsr:
    """amgt_csr_to_mbsr on device CSR arrays (int64 / int32 / float64, CUDA tensors)."""
    for t, dt in ((row_ptr, torch.int64), (col, torch.int32), (val, torch.float64)):
        if not t.is_cuda or t.dtype != dt or not t.is_contiguous():
            raise TypeError(f"expected contiguous CUDA {dt}, got {t.dtype} on {t.device}")
    out = Mbsr()
    _check(_L.amgt_csr_to_mbsr(int(m), int(n), int(col.numel()), row_ptr.data_ptr(), col.data_ptr(), val.data_ptr(),
                               PREC[prec], ctypes.byref(out.c), _AL, _stream(stream)))
    return out


def from_csr(A, prec="f64", stream=None) -> Mbsr:
    """gen.CSR (any device) -> Mbsr via amgt_csr_to_mbsr."""
    d = A.to("cuda")
    return csr_to_mbsr(d.m, d.n, d.row_ptr.contiguous(), d.col.contiguous(), d.val.contiguous(), prec, stream)


def spgemm_symbolic(A: Mbsr, B: Mbsr, stream=None, info: bool = False):
    C = Mbsr()
    inf = c_spgemm_info() if info else None
    _check(_L.amgt_spgemm_symbolic(ctypes.byref(A.c), ctypes.byref(B.c), ctypes.byref(C.c),
                                   ctypes.byref(inf) if info else None, _AL, _stream(stream)))
    return (C, inf.as_dict()) if info else C


def spgemm_numeric(A: Mbsr, B: Mbsr, C: Mbsr, stream=None) -> Mbsr:
    _check(_L.amgt_spgemm_numeric(ctypes.byref(A.c), ctypes.byref(B.c), ctypes.byref(C.c), _stream(stream)))
    return C


def spgemm(A: Mbsr, B: Mbsr, stream=None, info: bool = False):
    r = spgemm_symbolic(A, B, stream, info)
    C = r[0] if info else r
    spgemm_numeric(A, B, C, stream)
    return r


def rap(R: Mbsr, A: Mbsr, P: Mbsr, stream=None) -> Mbsr:
    C = Mbsr()
    _check(_L.amgt_rap(ctypes.byref(R.c), ctypes.byref(A.c), ctypes.byref(P.c), ctypes.byref(C.c), _AL,
                       _stream(stream)))
    return C


def set_tc_threshold(spgemm: int = 17, spmv: int = 17):
    _check(_L.amgt_set_tc_threshold(int(spgemm), int(spmv)))


def spmv(A: Mbsr, x: torch.Tensor, y: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """y = A x.  x: CUDA float64/float32 of length >= 4*blc_col (padding read as given);
    y: float64/float32 of length 4*blc_row (allocated as float64 if None)."""
    xp = {torch.float64: FP64, torch.float32: FP32}[x.dtype]
    if x.numel() < 4 * A.blc_col:
        xx = torch.zeros(4 * A.blc_col, dtype=x.dtype, device=x.device)
        xx[:x.numel()] = x
        x = xx
    if y is None:
        y = torch.empty(4 * A.blc_row, dtype=torch.float64, device="cuda")
    yp = {torch.float64: FP64, torch.float32: FP32}[y.dtype]
    assert y.numel() >= 4 * A.blc_row and x.is_contiguous() and y.is_contiguous()
    _check(_L.amgt_spmv(ctypes.byref(A.c), x.data_ptr(), xp, y.data_ptr(), yp, _stream(stream)))
    return y


EPI = {"y": 0, "jacobi": 1, "residual": 2, "accum": 3}


def spmv_fused(A: Mbsr, x: torch.Tensor, y: torch.Tensor, mode: str, b: torch.Tensor | None = None,
               dinv: torch.Tensor | None = None, omega: float = 2.0 / 3.0, stream=None) -> torch.Tensor:
    """amgt_spmv_fused: y = epilogue((A x)_i) — see include/amgt.h (AMGT_EPI_*)."""
    xp = {torch.float64: FP64, torch.float32: FP32}[x.dtype]
    yp = {torch.float64: FP64, torch.float32: FP32}[y.dtype]
    _check(_L.amgt_spmv_fused(ctypes.byref(A.c), x.data_ptr(), xp, y.data_ptr(), yp, EPI[mode],
                              b.data_ptr() if b is not None else None, dinv.data_ptr() if dinv is not None else None,
                              float(omega), _stream(stream)))
    return y


def spmv_jacobi_res(A: Mbsr, x: torch.Tensor, y: torch.Tensor, b: torch.Tensor, dinv: torch.Tensor,
                    r: torch.Tensor, omega: float = 2.0 / 3.0, stream=None) -> torch.Tensor:
    """amgt_spmv_fused_r: r = b - A x and y = x + omega dinv .* r in one pass over A."""
    p = {torch.float64: FP64, torch.float32: FP32}[x.dtype]
    _check(_L.amgt_spmv_fused_r(ctypes.byref(A.c), x.data_ptr(), p, y.data_ptr(), p, b.data_ptr(), dinv.data_ptr(),
                                float(omega), r.data_ptr(), _stream(stream)))
    return y


def spmv_range(A: Mbsr, blk_begin: int, blk_end: int, x: torch.Tensor, y: torch.Tensor, mode: str = "y",
               b: torch.Tensor | None = None, dinv: torch.Tensor | None = None, xs: torch.Tensor | None = None,
               omega: float = 2.0 / 3.0, stream=None) -> torch.Tensor:
    """amgt_spmv_fused_range: block rows [blk_begin, blk_end) only."""
    xp = {torch.float64: FP64, torch.float32: FP32}[x.dtype]
    yp = {torch.float64: FP64, torch.float32: FP32}[y.dtype]
    ptr = lambda t: t.data_ptr() if t is not None else None
    _check(_L.amgt_spmv_fused_range(ctypes.byref(A.c), int(blk_begin), int(blk_end), x.data_ptr(), xp, y.data_ptr(), yp,
                                    EPI[mode], ptr(b), ptr(dinv), ptr(xs), float(omega), _stream(stream)))
    return y


SWEEP = {"jacobi": 1, "jacobi_res": 2, "residual": 3, "residual_norm": 4}


class SweepPlan:
    """amgt_sweep_plan_create / amgt_spmv_sweeps / amgt_sweep_plan_destroy (FP64 square A)."""

    def __init__(self, A: Mbsr, stream=None):
        h = ctypes.c_void_p()
        _check(_L.amgt_sweep_plan_create(ctypes.byref(A.c), _AL, _stream(stream), ctypes.byref(h)))
        self.h, self.A = h, A

    def run(self, stages, b: torch.Tensor, dinv: torch.Tensor | None = None, omega: float = 2.0 / 3.0,
            norm: torch.Tensor | None = None, stream=None):
        """stages: [(mode, x, y), ...] with mode in SWEEP; norm: 1-element FP64 tensor for the
        squared residual norm of a jacobi_res / residual_norm stage."""
        arr = (c_sweep_stage * len(stages))(*[c_sweep_stage(SWEEP[m], x.data_ptr(), y.data_ptr())
                                              for m, x, y in stages])
        _check(_L.amgt_spmv_sweeps(self.h, ctypes.byref(self.A.c), len(stages), arr, b.data_ptr(),
                                   dinv.data_ptr() if dinv is not None else None, float(omega),
                                   norm.data_ptr() if norm is not None else None, _stream(stream)))

    def stats(self) -> dict:
        """SW_STATS builds only: per-item SM-cycle accounting since the last read."""
        o = (ctypes.c_uint64 * 6)()
        _check(_L.amgt_sweep_plan_stats(self.h, o, _stream(None)))
        return dict(zip(("cyc_s0", "n_s0", "cyc_later", "n_later", "cyc_wait", "polls"), list(o)))

    def close(self):
        if self.h:
            _L.amgt_sweep_plan_destroy(self.h, _stream(None))
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def strength_filter(A: Mbsr, theta: float = 0.25, omega: float = 2.0 / 3.0, stream=None):
    """amgt_strength_filter: (A_F, s = omega / diag(A_F))."""
    out = Mbsr()
    sd = torch.float64 if A.prec == FP64 else torch.float32
    sv = torch.zeros(max(4 * A.blc_row, 1), dtype=sd, device="cuda")
    _check(_L.amgt_strength_filter(ctypes.byref(A.c), float(theta), float(omega), ctypes.byref(out.c), sv.data_ptr(),
                                   _AL, _stream(stream)))
    return out, sv


def sa_interp(A: Mbsr, Pt: Mbsr, theta: float = 0.25, omega: float = 2.0 / 3.0, stream=None) -> Mbsr:
    """amgt_sa_interp: P = (I - omega D_F^-1 A_F) Pt through one SpGEMM call."""
    out = Mbsr()
    _check(_L.amgt_sa_interp(ctypes.byref(A.c), ctypes.byref(Pt.c), float(theta), float(omega), ctypes.byref(out.c),
                             _AL, _stream(stream)))
    return out


def pmis_aggregate(A: Mbsr, theta: float = 0.25, max_row_sum: float = 0.8, weights: torch.Tensor | None = None,
                   seed: int = 0, level: int = 0, stream=None):
    """amgt_pmis_aggregate: (agg int32[m], is_c int8[m], n_agg, rounds) on the device."""
    agg = torch.empty(max(A.m, 1), dtype=torch.int32, device="cuda")
    isc = torch.empty(max(A.m, 1), dtype=torch.int8, device="cuda")
    if weights is not None:
        assert weights.dtype == torch.float64 and weights.is_cuda and weights.numel() >= A.m
    n, r = ctypes.c_int64(0), ctypes.c_int(0)
    _check(_L.amgt_pmis_aggregate(ctypes.byref(A.c), float(theta), float(max_row_sum),
                                  weights.data_ptr() if weights is not None else None, int(seed) & 0xFFFFFFFFFFFFFFFF,
                                  int(level), agg.data_ptr(), isc.data_ptr(), ctypes.byref(n), ctypes.byref(r),
                                  _stream(stream)))
    return agg[:A.m], isc[:A.m], int(n.value), int(r.value)


def aggregation_p(agg: torch.Tensor, n_agg: int, prec="f64", stream=None) -> Mbsr:
    """amgt_aggregation_p: Pt(i, agg_i) = 1."""
    out = Mbsr()
    _check(_L.amgt_aggregation_p(int(agg.numel()), int(n_agg), agg.data_ptr(), PREC[prec], ctypes.byref(out.c), _AL,
                                 _stream(stream)))
    return out


def csr_to_mbsr_ex(m, n, row_ptr, col, val, col_offset: int, prec="f64", stream=None) -> Mbsr:
    out = Mbsr()
    _check(_L.amgt_csr_to_mbsr_ex(int(m), int(n), int(col.numel()), row_ptr.data_ptr(), col.data_ptr(), val.data_ptr(),
                                  int(col_offset), PREC[prec], ctypes.byref(out.c), _AL, _stream(stream)))
    return out


def shift_cols(A: Mbsr, delta_tiles: int, new_n: int, stream=None) -> Mbsr:
    _check(_L.amgt_mbsr_shift_cols(ctypes.byref(A.c), int(delta_tiles), int(new_n), _stream(stream)))
    return A


def csr_col_range(m, row_ptr, col, row_offset: int, stream=None):
    out = (ctypes.c_int64 * 3)()
    _check(_L.amgt_csr_col_range(int(m), row_ptr.data_ptr(), col.data_ptr() if col.numel() else None, int(row_offset),
                                 out, _stream(stream)))
    return tuple(out)


def mbsr_col_range(A: Mbsr, blk_row_offset: int, stream=None):
    out = (ctypes.c_int64 * 3)()
    _check(_L.amgt_mbsr_col_range(ctypes.byref(A.c), int(blk_row_offset), out, _stream(stream)))
    return tuple(out)


def dinv(A: Mbsr, diag_tile_offset: int, dtype=torch.float64, stream=None) -> torch.Tensor:
    d = torch.zeros(4 * A.blc_row, dtype=dtype, device="cuda")
    _check(_L.amgt_dinv(ctypes.byref(A.c), int(diag_tile_offset), d.data_ptr(), {torch.float64: FP64, torch.float32: FP32}[dtype],
                        _stream(stream)))
    return d


def dense_spd_inverse(a):
    """Host Cholesky-based inverse (numpy float64 n x n -> numpy)."""
    import numpy as np
    a = np.ascontiguousarray(a, dtype=np.float64)
    inv = np.empty_like(a)
    _check(_L.amgt_dense_spd_inverse(a.shape[0], a.ctypes.data, inv.ctypes.data))
    return inv


def dense_matvec(n: int, Ainv: torch.Tensor, b: torch.Tensor, x: torch.Tensor, stream=None) -> torch.Tensor:
    _check(_L.amgt_dense_matvec(int(n), int(x.numel()), Ainv.data_ptr(), b.data_ptr(), x.data_ptr(),
                                {torch.float64: FP64, torch.float32: FP32}[x.dtype], _stream(stream)))
    return x


def norm2sq(r: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    if out is None:
        out = torch.empty(1, dtype=torch.float64, device="cuda")
    _check(_L.amgt_norm2sq(int(r.numel()), r.data_ptr(), out.data_ptr(), _stream(stream)))
    return out


def wrap(m, n, blc_ptr, blc_idx, blc_map, blc_val, prec) -> Mbsr:
    out = Mbsr(keep=[blc_ptr, blc_idx, blc_map, blc_val])
    _check(_L.amgt_mbsr_wrap(int(m), int(n), int(blc_idx.numel()), blc_ptr.data_ptr(), blc_idx.data_ptr(),
                             blc_map.data_ptr(), blc_val.data_ptr(), PREC[prec], ctypes.byref(out.c)))
    return out


# ------------------------------------------------------------------ hierarchy / V-cycle
class Hierarchy:
    """amgt_hierarchy_create / amgt_vcycle / amgt_hierarchy_destroy."""

    def __init__(self, A: Mbsr, Ps: list, level_prec=("f64", "f32", "f16", "f16", "f16", "f16", "f16", "f16"),
                 nu1=1, nu2=1, omega=2.0 / 3.0, smoother="jacobi", interp="given", theta=0.25,
                 omega_p=2.0 / 3.0, max_levels=None, max_coarse_size=0, max_row_sum=0.8, seed=0, stream=None):
        # interp "pmis": no Ps; every level coarsened on the device (amgt_pmis_aggregate + SA),
        # up to max_levels levels (L300: PMIS, str_thr, max_row_sum, max_coarse_size)
        self.nlev = int(max_levels) if interp == "pmis" else len(Ps) + 1
        o = c_vcycle_opts()
        o.max_levels = self.nlev
        o.nu1, o.nu2, o.omega = int(nu1), int(nu2), float(omega)
        o.smoother = {"jacobi": 0, "l1_jacobi": 1}[smoother]
        o.interp = {"given": 0, "sa": 1, "pmis": 2}[interp]  # "sa": Ps are tentative; P_k by amgt_sa_interp
        o.theta, o.omega_p = float(theta), float(omega_p)
        o.max_coarse_size, o.max_row_sum, o.seed = int(max_coarse_size), float(max_row_sum), int(seed)
        lp = list(level_prec) + ["f16"] * 8
        for k in range(8):
            o.level_prec[k] = PREC[lp[k]]
        self._keep = [A, *Ps]
        self.npad = 4 * A.blc_row  # length of the level-1 vectors the library reads and writes
        arr = (_P(c_mbsr) * max(len(Ps), 1))(*[ctypes.pointer(p.c) for p in Ps])
        h = ctypes.c_void_p()
        _check(_L.amgt_hierarchy_create(ctypes.byref(A.c), arr, self.nlev, ctypes.byref(o), _AL, _stream(stream),
                                        ctypes.byref(h)))
        self.h = h
        self.nlev = int(_L.amgt_hierarchy_nlev(h))

    def level(self, k: int):
        a, p, r = _P(c_mbsr)(), _P(c_mbsr)(), _P(c_mbsr)()
        _check(_L.amgt_hierarchy_level(self.h, k, ctypes.byref(a), ctypes.byref(p), ctypes.byref(r)))

        def mk(ptr):
            if not ptr:
                return None
            M = Mbsr(c_mbsr.from_buffer_copy(ptr.contents), keep=[self])
            M.c.own = 0
            M.c.aux = None
            return M
        return mk(a), mk(p), mk(r)

    def _check_vectors(self, b: torch.Tensor, x: torch.Tensor):
        """The ABI reads b and writes x over 4*blc_row(A_1) elements (include/amgt.h)."""
        for name, t in (("b", b), ("x", x)):
            if t.dtype != torch.float64 or not t.is_cuda or not t.is_contiguous():
                raise TypeError(f"{name}: expected a contiguous CUDA float64 tensor")
            if t.numel() < self.npad:
                raise ValueError(f"{name} has {t.numel()} elements; the level-1 vectors need 4*blc_row = {self.npad} "
                                 "(zero-pad to a multiple of 4)")

    def vcycle(self, b: torch.Tensor, x: torch.Tensor, ncycles: int, stream=None):
        self._check_vectors(b, x)
        res = (ctypes.c_double * (ncycles + 1))()
        calls = ctypes.c_int64(0)
        _check(_L.amgt_vcycle(self.h, b.data_ptr(), x.data_ptr(), int(ncycles), res, ctypes.byref(calls),
                              _stream(stream)))
        return list(res), int(calls.value)

    def pcg(self, b: torch.Tensor, x: torch.Tensor, maxit: int, rtol: float = 0.0, stream=None):
        """amgt_pcg: V-cycle-preconditioned CG; returns (residual norms, iterations, SpMV calls)."""
        self._check_vectors(b, x)
        res = (ctypes.c_double * (maxit + 1))()
        it, calls = ctypes.c_int(0), ctypes.c_int64(0)
        _check(_L.amgt_pcg(self.h, b.data_ptr(), x.data_ptr(), int(maxit), float(rtol), res, ctypes.byref(it),
                           ctypes.byref(calls), _stream(stream)))
        return list(res)[:it.value + 1], int(it.value), int(calls.value)

    def close(self):
        if self.h:
            _L.amgt_hierarchy_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------------------------ instrumentation
TIMER_CLASSES = ("spmv_l1", "spmv", "spgemm_symbolic", "spgemm_numeric", "csr2mbsr", "mbsr2csr", "cast", "vector")


def timing_enable(on=True):
    """True = all classes, False = off, or an int bitmask over TIMER_CLASSES."""
    _check(_L.amgt_timing_enable(-1 if on is True else (0 if on is False else int(on))))


def timing_reset():
    _check(_L.amgt_timing_reset())


def timing_sample(every: int = 1):
    """Time one call in `every` of each enabled class (amgt_timing_sample)."""
    _check(_L.amgt_timing_sample(int(every)))


def timing_read() -> dict:
    ms = (ctypes.c_double * 8)()
    n = (ctypes.c_int64 * 8)()
    by = (ctypes.c_double * 8)()
    _check(_L.amgt_timing_read(ms, n, by))
    return {TIMER_CLASSES[i]: {"ms": ms[i], "launches": n[i], "bytes": by[i]} for i in range(8)}


def launch_count() -> int:
    return int(_L.amgt_launch_count())
