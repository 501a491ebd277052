"""Row-partitioned multi-GPU path (the paper's 8-GPU runs, L363-365) — the
ctypes binding of libamgt's distributed ABI (include/amgt.h, "distributed path").  Argument
marshalling only: partition plans, halo exchanges, the row gathers of the distributed RAP, the
agglomerated coarse levels and the V-cycle all run inside libamgt (csrc/dist.cu).

Transports:
  * NCCL — one process per GPU (torchrun); the 128-byte NCCL id is broadcast over an existing
    torch.distributed group (`DistComm.nccl`).
  * loopback — G virtual ranks in one process on one GPU, one host thread each (`run_loopback`);
    the same code paths with device-to-device copies instead of NVLink transfers.

A rank's matrices hold its own rows with global column indices (e.g. `from_csr` of the rows
`gen.partition.slab_inputs` generates); its vectors hold its own rows.
"""
from __future__ import annotations

import ctypes
import threading

import torch

from . import _lib
from ._lib import _AL, _L, Mbsr, _check, _stream, c_dist_hier_info, c_dist_piece, c_mbsr, c_vcycle_opts, PREC

_P = ctypes.POINTER


class DistComm:
    """An amgt_dist communicator (one rank)."""

    def __init__(self, handle: ctypes.c_void_p, rank: int, size: int, rows: tuple):
        self.h, self.rank, self.size, self.rows = handle, rank, size, rows
        self._keep = []

    @staticmethod
    def nccl(rank: int, size: int, rows: tuple, group=None) -> "DistComm":
        """NCCL communicator; `group` (torch.distributed) carries the unique id from rank 0."""
        import torch.distributed as dist
        uid = ctypes.create_string_buffer(128)
        if rank == 0:
            _check(_L.amgt_nccl_unique_id(uid))
        t = torch.frombuffer(bytearray(uid.raw), dtype=torch.uint8).clone()
        if size > 1:
            if dist.get_backend(group) == "nccl":
                t = t.cuda()
            dist.broadcast(t, 0, group=group)
        raw = bytes(t.cpu().tolist())
        h = ctypes.c_void_p()
        _check(_L.amgt_dist_create(ctypes.create_string_buffer(raw, 128), rank, size, int(rows[0]), int(rows[1]),
                                   ctypes.byref(h)))
        return DistComm(h, rank, size, rows)

    def spmv(self, A: Mbsr, x: torch.Tensor, y: torch.Tensor, stream=None) -> torch.Tensor:
        """amgt_dist_spmv: y = own rows of A x (collective)."""
        _check(_L.amgt_dist_spmv(self.h, ctypes.byref(A.c), x.data_ptr(), y.data_ptr(), _stream(stream)))
        return y

    def rap(self, R: Mbsr, A: Mbsr, P: Mbsr, stream=None) -> Mbsr:
        """amgt_dist_rap: own coarse rows of R (A P) (collective)."""
        out = Mbsr()
        _check(_L.amgt_dist_rap(self.h, ctypes.byref(R.c), ctypes.byref(A.c), ctypes.byref(P.c), ctypes.byref(out.c),
                                _AL, _stream(stream)))
        return out

    def allgather(self, M: Mbsr, stream=None) -> Mbsr:
        """amgt_dist_allgather_mbsr: every rank's rows in rank order (collective)."""
        out = Mbsr()
        _check(_L.amgt_dist_allgather_mbsr(self.h, ctypes.byref(M.c), ctypes.byref(out.c), _AL, _stream(stream)))
        return out

    def allreduce_sum(self, t: torch.Tensor, stream=None) -> torch.Tensor:
        assert t.dtype == torch.float64 and t.is_cuda and t.is_contiguous()
        _check(_L.amgt_dist_allreduce_sum(self.h, t.data_ptr(), t.numel(), _stream(stream)))
        return t

    def close(self):
        if self.h:
            _L.amgt_dist_destroy(self.h)
            self.h = None


class LoopGroup:
    """amgt_dist_group: `size` virtual ranks sharing this process and GPU."""

    def __init__(self, size: int):
        h = ctypes.c_void_p()
        _check(_L.amgt_dist_group_create(int(size), ctypes.byref(h)))
        self.h, self.size = h, size

    def member(self, rank: int, rows: tuple) -> DistComm:
        h = ctypes.c_void_p()
        _check(_L.amgt_dist_create_loopback(self.h, int(rank), int(rows[0]), int(rows[1]), ctypes.byref(h)))
        return DistComm(h, rank, self.size, rows)

    def close(self):
        if self.h:
            _L.amgt_dist_group_destroy(self.h)
            self.h = None


def run_loopback(size: int, rows_of, fn, device: int = 0):
    """Run fn(rank, comm, stream) for `size` virtual ranks, one host thread each (its own CUDA
    stream); rows_of(rank) -> (row_begin, row_end).  Returns the per-rank results in rank order;
    re-raises the first exception."""
    G = LoopGroup(size)
    out, errs = [None] * size, [None] * size

    def body(r):
        torch.cuda.set_device(device)
        comm = None
        try:
            comm = G.member(r, rows_of(r))
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                out[r] = fn(r, comm, st)
            st.synchronize()
        except BaseException as e:  # noqa: BLE001 - reported to the caller
            errs[r] = e
            _L.amgt_dist_group_abort(G.h)  # the other ranks stop waiting for this one
        finally:
            if comm is not None:
                comm.close()

    th = [threading.Thread(target=body, args=(r,), daemon=True) for r in range(size)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    G.close()
    first = [e for e in errs if e is not None and "group aborted" not in str(e)] or [e for e in errs if e is not None]
    if first:
        raise first[0]
    return out


class DistHierarchy:
    """amgt_dist_hierarchy_create / amgt_dist_vcycle (collective)."""

    def __init__(self, comm: DistComm, A: Mbsr, Ps: list, level_prec=("f64", "f32", "f16", "f16", "f16", "f16", "f16",
                 "f16"), nu1=1, nu2=1, omega=2.0 / 3.0, smoother="jacobi", agg_rows: int = 32768, stream=None):
        self.comm, self.nlev = comm, len(Ps) + 1
        o = c_vcycle_opts()
        o.max_levels = self.nlev
        o.nu1, o.nu2, o.omega = int(nu1), int(nu2), float(omega)
        o.smoother = {"jacobi": 0, "l1_jacobi": 1}[smoother]
        o.interp = 0
        o.theta, o.omega_p = 0.25, 2.0 / 3.0
        lp = list(level_prec) + ["f16"] * 8
        for k in range(8):
            o.level_prec[k] = PREC[lp[k]]
        self._keep = [A, *Ps]  # A_l is borrowed by the library
        self.npad = 4 * A.blc_row
        arr = (_P(c_mbsr) * max(len(Ps), 1))(*[ctypes.pointer(p.c) for p in Ps])
        h = ctypes.c_void_p()
        _check(_L.amgt_dist_hierarchy_create(comm.h, ctypes.byref(A.c), arr, self.nlev, ctypes.byref(o), int(agg_rows),
                                             _AL, _stream(stream), ctypes.byref(h)))
        self.h = h

    def vcycle(self, b: torch.Tensor, x: torch.Tensor, ncycles: int, stream=None):
        for name, t in (("b", b), ("x", x)):
            if t.dtype != torch.float64 or not t.is_cuda or not t.is_contiguous() or t.numel() < self.npad:
                raise ValueError(f"{name}: contiguous CUDA float64 with >= {self.npad} elements expected")
        res = (ctypes.c_double * (ncycles + 1))()
        calls = ctypes.c_int64(0)
        _check(_L.amgt_dist_vcycle(self.h, b.data_ptr(), x.data_ptr(), int(ncycles), res, ctypes.byref(calls),
                                   _stream(stream)))
        return list(res), int(calls.value)

    def info(self) -> dict:
        i = c_dist_hier_info()
        _check(_L.amgt_dist_hierarchy_info(self.h, ctypes.byref(i)))
        n = i.nlev
        return {"nlev": n, "agg_level": i.agg_level, "rows": list(i.rows)[:n], "tiles": list(i.tiles)[:n],
                "row_begin": list(i.row_begin)[:i.agg_level], "ext": [(i.ext_begin[k], i.ext_end[k])
                                                                     for k in range(i.agg_level)],
                "halo_recv": list(i.halo_recv)[:i.agg_level], "halo_send": list(i.halo_send)[:i.agg_level],
                "interior": [tuple(i.interior[k]) for k in range(i.agg_level)]}

    def close(self):
        if self.h:
            _L.amgt_dist_hierarchy_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def plan_host(rank: int, rows, colmin, colmax, cap: int = 64):
    """amgt_dist_plan_host (no GPU): ((eb, ee), [(peer, begin, end) received], [... sent]) in block
    rows, from every rank's own row count and min / max tile column."""
    import numpy as np
    size = len(rows)
    r = np.ascontiguousarray(rows, dtype=np.int64)
    lo = np.ascontiguousarray(colmin, dtype=np.int64)
    hi = np.ascontiguousarray(colmax, dtype=np.int64)
    ext = (ctypes.c_int64 * 2)()
    rv, sd = (c_dist_piece * cap)(), (c_dist_piece * cap)()
    nr, ns = ctypes.c_int(0), ctypes.c_int(0)
    _check(_L.amgt_dist_plan_host(int(rank), size, r.ctypes.data, lo.ctypes.data, hi.ctypes.data, ext, rv,
                                  ctypes.byref(nr), sd, ctypes.byref(ns), cap))
    return ((ext[0], ext[1]), [(p.peer, p.begin, p.end) for p in rv[:nr.value]],
            [(p.peer, p.begin, p.end) for p in sd[:ns.value]])
