"""Row-slab distributed AmgT hot path (the paper runs 8 GPUs through
HYPRE/MPI, L363-365 — this is the NCCL re-design).

Partition: every rank owns a contiguous, 4-row-aligned range [rb, re) of the rows of each
level (z-slabs of the lexicographic grid; 2x2x2 aggregates never straddle slabs, so the
coarse ranges are contiguous too).  A rank stores its rows with columns remapped to its
extended range [eb, ee) = [own rows] + the halo its rows touch, eb aligned to 4 so tile
columns shift by whole tiles.  Vectors that SpMV reads live in extended buffers
[halo_lo | own | halo_hi].

  SpMV       halo exchange of x (point-to-point, NCCL over NVLink on GPUs) overlapped with
             the interior block rows (rows whose columns stay inside the own range, from the
             matrix bandwidth), then the boundary block rows (amgt_spmv_fused_range).
  RAP        the P rows of the halo range are gathered from the neighbours (P_ext); A_loc P_ext
             and R_loc (A P) are then local (R_loc = P_own^T: aggregates are rank-local).
  V-cycle    Alg. 2 with halo SpMVs per level, all-reduce of the residual norm, all-gather of
             the coarsest right-hand side and a redundant dense solve on every rank.

All arithmetic runs in libamgt's kernels (LibOps).  Communication uses torch.distributed:
device tensors with NCCL; host-staged tensors with gloo (CPU tests, or several ranks
sharing one GPU).  The compute backend is injectable so the partition / halo / remap logic
is testable on CPU (tests supply an oracle-backed backend).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np
import torch
import torch.distributed as dist

EPI_NAMES = ("y", "jacobi", "residual", "accum")


# ------------------------------------------------------------------ communication
class Comm:
    """torch.distributed wrapper: point-to-point batches, all-reduce, all-gather."""

    def __init__(self, group=None):
        self.group = group
        self.rank = dist.get_rank(group)
        self.size = dist.get_world_size(group)
        self.backend = dist.get_backend(group)
        self.nccl = self.backend == "nccl"

    def exchange(self, sends, recvs):
        """sends/recvs: lists of (peer, tensor).  Returns an object with wait()."""
        if not sends and not recvs:
            return _Done()
        if self.nccl:
            ops = [dist.P2POp(dist.isend, t, p, self.group) for p, t in sends]
            ops += [dist.P2POp(dist.irecv, t, p, self.group) for p, t in recvs]
            return _Works(dist.batch_isend_irecv(ops))
        # gloo: stage through host memory
        hs = [(p, t.detach().cpu()) for p, t in sends]
        hr = [(p, torch.empty(t.shape, dtype=t.dtype)) for p, t in recvs]
        works = [dist.isend(t, p, self.group) for p, t in hs] + [dist.irecv(t, p, self.group) for p, t in hr]
        return _Staged(works, hr, recvs, hs)

    def allreduce_sum(self, t: torch.Tensor) -> torch.Tensor:
        if self.nccl:
            dist.all_reduce(t, group=self.group)
            return t
        h = t.detach().cpu()
        dist.all_reduce(h, group=self.group)
        t.copy_(h)
        return t

    def allgather_obj(self, obj):
        """All-gather a small Python value.  Integers and tuples of integers (every use in the
        setup: row ranges, extended ranges, counts) go through one int64 tensor all-gather;
        anything else through all_gather_object (pickled)."""
        if self.size == 1:
            return [obj]
        ints = isinstance(obj, int) or (isinstance(obj, tuple) and all(isinstance(v, int) for v in obj))
        if ints:
            vals = [obj] if isinstance(obj, int) else list(obj)
            dev = torch.device("cuda", torch.cuda.current_device()) if self.nccl else torch.device("cpu")
            t = torch.tensor(vals, dtype=torch.int64, device=dev)
            outs = [torch.empty_like(t) for _ in range(self.size)]
            dist.all_gather(outs, t, group=self.group)
            host = torch.stack(outs).cpu().tolist()
            return [h[0] if isinstance(obj, int) else tuple(h) for h in host]
        out = [None] * self.size
        dist.all_gather_object(out, obj, group=self.group)
        return out

    def allgather_var(self, t: torch.Tensor) -> list:
        """All-gather 1-D tensors of different lengths (padded to the max)."""
        n = self.allgather_obj(int(t.numel()))
        mx = max(n) if n else 0
        buf = torch.zeros(mx, dtype=t.dtype, device=t.device)
        buf[:t.numel()] = t
        if self.nccl:
            outs = [torch.empty_like(buf) for _ in range(self.size)]
            dist.all_gather(outs, buf, group=self.group)
        else:
            hb = buf.cpu()
            outs = [torch.empty_like(hb) for _ in range(self.size)]
            dist.all_gather(outs, hb, group=self.group)
            outs = [o.to(t.device) for o in outs]
        return [o[:k] for o, k in zip(outs, n)]


class _Done:
    def wait(self):
        pass


class _Works:
    def __init__(self, w):
        self.w = w

    def wait(self):
        for w in self.w:
            w.wait()


class _Staged:
    def __init__(self, works, hr, recvs, hs):
        self.works, self.hr, self.recvs, self.hs = works, hr, recvs, hs

    def wait(self):
        for w in self.works:
            w.wait()
        for (_, h), (_, t) in zip(self.hr, self.recvs):
            t.copy_(h)


# ------------------------------------------------------------------ compute backend
class LibOps:
    """The product backend: libamgt kernels on the current CUDA device."""

    device = "cuda"

    def __init__(self):
        from . import _lib
        self.L = _lib

    def csr_to_local(self, rp, col, val, m, n_cols, col_offset, prec):
        return self.L.csr_to_mbsr_ex(m, n_cols, rp, col, val, col_offset, prec)

    def csr_col_range(self, rp, col, m, row_offset):
        return self.L.csr_col_range(m, rp, col, row_offset)

    def col_range_tiles(self, A, blk_row_offset):
        return self.L.mbsr_col_range(A, blk_row_offset)

    def shift_cols(self, A, delta_tiles, new_n):
        return self.L.shift_cols(A, delta_tiles, new_n)

    def spgemm(self, A, B):
        return self.L.spgemm(A, B)

    def transpose(self, A):
        return self.L.Mbsr.transpose(A)

    def cast(self, A, prec):
        if self.L.PREC[prec] == A.prec:
            return A
        C = A.cast(prec)
        return C

    def to_csr(self, A):
        return A.to_csr()

    def rows(self, A):
        return A.m

    def cols(self, A):
        return A.n

    def blc_row(self, A):
        return A.blc_row

    def spmv_range(self, A, i0, i1, x, y, mode, b=None, dinv=None, xs=None, omega=2.0 / 3.0):
        return self.L.spmv_range(A, i0, i1, x, y, mode, b, dinv, xs, omega)

    def dinv(self, A, diag_tile_offset, dtype):
        return self.L.dinv(A, diag_tile_offset, dtype)

    def dense_inverse(self, a):
        return self.L.dense_spd_inverse(a)

    def dense_matvec(self, n, Ainv, b, x):
        return self.L.dense_matvec(n, Ainv, b, x)

    def norm2sq(self, r):
        return self.L.norm2sq(r)


# ------------------------------------------------------------------ partition / halo plan
def slab_ranges(n_planes: int, plane: int, size: int):
    """Contiguous z-slab row ranges: rank r owns planes [r*np/size, (r+1)*np/size)."""
    out = []
    for r in range(size):
        z0 = (r * n_planes) // size
        z1 = ((r + 1) * n_planes) // size
        out.append((z0 * plane, z1 * plane))
    return out


def _overlap(a0, a1, b0, b1):
    lo, hi = max(a0, b0), min(a1, b1)
    return (lo, hi) if lo < hi else None


@dataclass
class HaloPlan:
    rb: int
    re: int
    eb: int
    ee: int
    recvs: list = field(default_factory=list)  # (peer, g0, g1) into my ext buffer
    sends: list = field(default_factory=list)  # (peer, g0, g1) from my own rows

    @staticmethod
    def build(me: int, ranges, exts):
        """ranges[q] = (rb_q, re_q) owned rows; exts[q] = (eb_q, ee_q) extended ranges."""
        rb, re_ = ranges[me]
        eb, ee = exts[me]
        plan = HaloPlan(rb, re_, eb, ee)
        for q, (qb, qe) in enumerate(ranges):
            if q == me:
                continue
            for h0, h1 in ((eb, rb), (re_, ee)):  # my halo pieces owned by q
                o = _overlap(h0, h1, qb, qe)
                if o:
                    plan.recvs.append((q, o[0], o[1]))
            qeb, qee = exts[q]
            for h0, h1 in ((qeb, qb), (qe, qee)):  # q's halo pieces that I own
                o = _overlap(h0, h1, rb, re_)
                if o:
                    plan.sends.append((q, o[0], o[1]))
        plan.recvs.sort()
        plan.sends.sort()
        return plan

    def ops_for(self, xe: torch.Tensor):
        """(sends, recvs) tensor views of an extended buffer for Comm.exchange."""
        sends = [(q, xe[g0 - self.eb:g1 - self.eb]) for q, g0, g1 in self.sends]
        recvs = [(q, xe[g0 - self.eb:g1 - self.eb]) for q, g0, g1 in self.recvs]
        return sends, recvs


def _vdtype(prec: str):
    return torch.float64 if prec == "f64" else torch.float32


def _ceil4(v: int) -> int:
    return 4 * ((v + 3) // 4)


# ------------------------------------------------------------------ one distributed level
class DistLevel:
    def __init__(self, comm: Comm, ops, A_loc, ranges, plan: HaloPlan, bw: int, n_global: int, prec: str):
        self.comm, self.ops, self.A, self.ranges, self.plan = comm, ops, A_loc, ranges, plan
        self.prec, self.n_global = prec, n_global
        self.vdt = _vdtype(prec)
        self.rb, self.re, self.eb, self.ee = plan.rb, plan.re, plan.eb, plan.ee
        self.m = self.re - self.rb
        self.BR = (self.m + 3) // 4
        self.next = _ceil4(self.ee - self.eb)
        self.off = self.rb - self.eb  # own segment offset in the extended buffer (multiple of 4)
        # interior block rows: rows within `bw` of the slab edges may touch the halo
        lo = (bw + 3) // 4
        hi = (self.m - bw) // 4
        self.int0, self.int1 = (lo, hi) if lo < hi else (0, 0)
        dev = ops.device
        self.xe = [torch.zeros(max(self.next, self.off + 4 * self.BR), dtype=self.vdt, device=dev) for _ in range(2)]
        self.cur = 0
        self.b = torch.zeros(4 * self.BR, dtype=self.vdt, device=dev)
        self.r = torch.zeros(4 * self.BR, dtype=self.vdt, device=dev)
        self.dinv = ops.dinv(A_loc, self.off // 4, self.vdt) if self.m > 0 else torch.zeros(0, dtype=self.vdt, device=dev)
        self.P = None  # P_k own rows x own coarse rows (local indices), level-k precision
        self.R = None  # R_k = P_k^T
        self.spmv_calls = 0

    def own(self, i: int):
        return self.xe[i][self.off:self.off + 4 * self.BR]

    def spmv(self, xe_idx: int, y: torch.Tensor, mode: str, b=None, xs=None, omega=2.0 / 3.0):
        """y = epilogue(A x) with x the extended buffer xe[xe_idx]; halo exchange overlapped
        with the interior block rows."""
        self.spmv_calls += 1
        xe = self.xe[xe_idx]
        sends, recvs = self.plan.ops_for(xe)
        h = self.comm.exchange(sends, recvs)
        d = self.dinv if mode == "jacobi" else None
        if self.int1 > self.int0:
            self.ops.spmv_range(self.A, self.int0, self.int1, xe, y, mode, b, d, xs, omega)
        h.wait()
        if self.int0 > 0:
            self.ops.spmv_range(self.A, 0, self.int0, xe, y, mode, b, d, xs, omega)
        if self.BR > self.int1:
            self.ops.spmv_range(self.A, max(self.int1, self.int0 if self.int1 > self.int0 else 0), self.BR, xe, y, mode,
                                b, d, xs, omega)
        return y


def _extended_range(rb, re_, mn, mx, n):
    eb = min(rb, 4 * (mn // 4)) if mn <= mx else rb
    ee = max(re_, min(n, _ceil4(mx + 1))) if mn <= mx else re_
    return eb, ee


# ------------------------------------------------------------------ distributed hierarchy
class DistHierarchy:
    """Setup (Alg. 1 with fixed P, RAP per level) and V-cycles (Alg. 2) over slabs.

    A_rows: this rank's rows of A_1 (gen.CSR, global columns), row range `rows0`;
    P_rows: per level, this rank's rows of P_k (gen.CSR, global coarse columns) — the rows
    of P_k it owns on level k (P_k rows are fine rows of level k).
    """

    def __init__(self, comm: Comm, A_rows, rows0, n0: int, P_rows: list, level_prec=("f64", "f32", "f16", "f16", "f16",
                 "f16", "f16", "f16"), omega=2.0 / 3.0, nu1=1, nu2=1, ops=None):
        self.comm = comm
        self.ops = ops or LibOps()
        self.omega, self.nu1, self.nu2 = omega, nu1, nu2
        self.nlev = len(P_rows) + 1
        self.prec = list(level_prec)[:self.nlev]
        ops, dev = self.ops, self.ops.device
        rb, re_ = rows0
        ranges = comm.allgather_obj((rb, re_))
        A = A_rows.to(dev)
        mn, mx, bw = ops.csr_col_range(A.row_ptr, A.col, A.m, rb)
        self.levels = []
        n = n0
        A_loc = None
        for k in range(self.nlev):
            prec = self.prec[k]
            if k == 0:
                eb, ee = _extended_range(rb, re_, mn, mx, n)
                exts = comm.allgather_obj((eb, ee))
                plan = HaloPlan.build(comm.rank, ranges, exts)
                A_loc = ops.csr_to_local(A.row_ptr, A.col, A.val, A.m, ee - eb, eb, prec)
            else:
                mn_t, mx_t, bw_t = ops.col_range_tiles(A_glob, rb // 4)
                mn, mx, bw = 4 * mn_t, 4 * mx_t + 3, 4 * bw_t + 3
                eb, ee = _extended_range(rb, re_, mn, mx, n)
                exts = comm.allgather_obj((eb, ee))
                plan = HaloPlan.build(comm.rank, ranges, exts)
                A_loc = ops.shift_cols(A_glob, -(eb // 4), ee - eb)
            L = DistLevel(comm, ops, A_loc, ranges, plan, bw, n, prec)
            self.levels.append(L)
            if k + 1 == self.nlev:
                break
            # ---- RAP for level k+1 (Alg. 1 line 5) in level-k precision
            P = P_rows[k].to(dev)
            nc = P.n
            cmn, cmx, _ = ops.csr_col_range(P.row_ptr, P.col, P.m, 0)
            crb, cre = (cmn, cmx + 1) if P.m > 0 else (0, 0)
            cranges = comm.allgather_obj((crb, cre))
            self._check_tiling(cranges, nc)
            P_ext = self._gather_P_ext(plan, P, nc, prec)
            AP = ops.spgemm(A_loc, P_ext)
            L.P = ops.csr_to_local(P.row_ptr, P.col, P.val, P.m, cre - crb, crb, prec)
            L.R = ops.transpose(L.P)
            A_next = ops.spgemm(L.R, AP)  # own coarse rows (local), global coarse columns
            A_glob = ops.cast(A_next, self.prec[k + 1])
            rb, re_, ranges, n = crb, cre, cranges, nc
        self._setup_coarsest()

    @staticmethod
    def _check_tiling(ranges, n):
        pos = 0
        for b, e in ranges:
            if b != pos or e < b or b % 4:
                raise ValueError(f"coarse row ranges {ranges} do not tile [0, {n}) in 4-aligned slabs")
            pos = e
        if pos != n:
            raise ValueError(f"coarse row ranges {ranges} do not cover [0, {n})")

    def _gather_P_ext(self, plan: HaloPlan, P, nc, prec):
        """P rows for the extended range [eb, ee): own rows + rows received from the owners
        of the halo (two-phase exchange: row lengths, then columns and values)."""
        ops, comm = self.ops, self.comm
        dev = ops.device
        rp = P.row_ptr
        lens_send = [(q, (rp[g1 - plan.rb] - rp[g0 - plan.rb]).reshape(1).to(torch.int64).clone())
                     for q, g0, g1 in plan.sends]
        rowlen_send = [(q, (rp[g0 - plan.rb + 1:g1 - plan.rb + 1] - rp[g0 - plan.rb:g1 - plan.rb]).contiguous())
                       for q, g0, g1 in plan.sends]
        rowlen_recv = [(q, torch.empty(g1 - g0, dtype=torch.int64, device=dev)) for q, g0, g1 in plan.recvs]
        comm.exchange(rowlen_send, rowlen_recv).wait()
        del lens_send
        col_send, val_send = [], []
        for q, g0, g1 in plan.sends:
            a, b = int(rp[g0 - plan.rb]), int(rp[g1 - plan.rb])
            col_send.append((q, P.col[a:b].contiguous()))
            val_send.append((q, P.val[a:b].contiguous()))
        col_recv = [(q, torch.empty(int(t.sum()), dtype=torch.int32, device=dev)) for q, t in rowlen_recv]
        val_recv = [(q, torch.empty(int(t.sum()), dtype=torch.float64, device=dev)) for q, t in rowlen_recv]
        comm.exchange(col_send + val_send, col_recv + val_recv).wait()
        # assemble rows in global order: [eb, rb) halo, own [rb, re), [re, ee) halo
        pieces = []  # (g0, rowlens, cols, vals)
        for (q, g0, g1), (_, rl), (_, c), (_, v) in zip(plan.recvs, rowlen_recv, col_recv, val_recv):
            pieces.append((g0, rl, c, v))
        pieces.append((plan.rb, (rp[1:] - rp[:-1]).to(torch.int64), P.col, P.val))
        pieces.sort(key=lambda p: p[0])
        n_ext = plan.ee - plan.eb
        lens = torch.zeros(n_ext, dtype=torch.int64, device=dev)
        cols, vals = [], []
        for g0, rl, c, v in pieces:
            lens[g0 - plan.eb:g0 - plan.eb + rl.numel()] = rl
            cols.append(c)
            vals.append(v)
        row_ptr = torch.zeros(n_ext + 1, dtype=torch.int64, device=dev)
        row_ptr[1:] = torch.cumsum(lens, 0)
        col = torch.cat(cols) if cols else torch.zeros(0, dtype=torch.int32, device=dev)
        val = torch.cat(vals) if vals else torch.zeros(0, dtype=torch.float64, device=dev)
        return ops.csr_to_local(row_ptr, col.contiguous(), val.contiguous(), n_ext, nc, 0, prec)

    def _setup_coarsest(self):
        """Gather A_M on every rank, factorise on the host (R22), keep A_M^{-1} on the device."""
        ops, comm = self.ops, self.comm
        C = self.levels[-1]
        rp, ci, v = ops.to_csr(C.A)
        rows = torch.repeat_interleave(torch.arange(C.m, dtype=torch.int64, device=rp.device) + C.rb,
                                       (rp[1:] - rp[:-1]).to(torch.int64))
        cols = ci.to(torch.int64) + C.eb
        R = torch.cat(comm.allgather_var(rows))
        K = torch.cat(comm.allgather_var(cols))
        V = torch.cat(comm.allgather_var(v))
        n = C.n_global
        dense = np.zeros((n, n))
        dense[R.cpu().numpy(), K.cpu().numpy()] = V.cpu().numpy()
        self.nM = n
        self.Ainv = torch.from_numpy(ops.dense_inverse(dense)).to(ops.device)
        self.coarse_ranges = comm.allgather_obj((C.rb, C.re))

    # ---------------------------------------------------------------- solve
    def _smooth(self, L: DistLevel, b, sweeps):
        for _ in range(sweeps):
            src, dst = L.cur, 1 - L.cur
            L.spmv(src, L.own(dst), "jacobi", b=b, xs=L.own(src), omega=self.omega)
            L.cur = dst

    def vcycle(self, b_own: torch.Tensor, x_own: torch.Tensor, ncycles: int):
        """b_own, x_own: this rank's rows of b and x (level 1, FP64, length 4*BR_own).
        Returns (global residual norms [ncycles+1], SpMV calls on this rank)."""
        Ls, M = self.levels, self.nlev - 1
        for L in Ls:
            L.spmv_calls = 0
        L0 = Ls[0]
        L0.cur = 0
        L0.own(0).copy_(x_own)
        norms = []

        def resnorm():
            L0.spmv(L0.cur, L0.r, "residual", b=b_own)
            s = self.ops.norm2sq(L0.r)
            self.comm.allreduce_sum(s)
            norms.append(s)

        resnorm()
        for _ in range(ncycles):
            for k in range(M):  # Alg. 2 lines 1-5
                L = Ls[k]
                bk = b_own if k == 0 else L.b
                if k > 0:
                    L.cur = 0
                    L.own(0).zero_()
                self._smooth(L, bk, self.nu1)
                L.spmv(L.cur, L.r, "residual", b=bk)
                N = Ls[k + 1]
                self.ops.spmv_range(L.R, 0, L.R.blc_row if hasattr(L.R, "blc_row") else self.ops.blc_row(L.R), L.r, N.b,
                                    "y")
                L.spmv_calls += 1
            C = Ls[M]  # line 6: all-gather the RHS, redundant dense solve
            bfull = torch.cat(self.comm.allgather_var(C.b[:C.m]))
            xfull = torch.zeros(self.nM, dtype=C.vdt, device=self.ops.device)
            self.ops.dense_matvec(self.nM, self.Ainv, bfull.contiguous(), xfull)
            C.cur = 0
            C.own(0)[:C.m].copy_(xfull[C.rb:C.re])
            for k in range(M - 1, -1, -1):  # lines 7-11
                L, N = Ls[k], Ls[k + 1]
                bk = b_own if k == 0 else L.b
                self.ops.spmv_range(L.P, 0, self.ops.blc_row(L.P), N.own(N.cur), L.own(L.cur), "accum")
                L.spmv_calls += 1
                self._smooth(L, bk, self.nu2)
            resnorm()
        x_own.copy_(L0.own(L0.cur))
        res = torch.stack([n.reshape(()) for n in norms]).double().sqrt().cpu().tolist()
        return res, sum(L.spmv_calls for L in Ls)


# ------------------------------------------------------------------ native V-cycle (libamgt + NCCL)
class NativeComm:
    """libamgt-owned NCCL communicator (amgt_dist_create); unique id shared over `comm`."""

    def __init__(self, comm: Comm):
        import ctypes
        from . import _lib
        self.L = _lib
        uid = ctypes.create_string_buffer(128)
        if comm.rank == 0:
            _lib._check(_lib._L.amgt_dist_unique_id(uid))
        raw = comm.allgather_obj(bytes(uid.raw) if comm.rank == 0 else None)[0]
        uid = ctypes.create_string_buffer(raw, 128)
        h = ctypes.c_void_p()
        _lib._check(_lib._L.amgt_dist_create(uid, comm.rank, comm.size, ctypes.byref(h)))
        self.h = h
        self.rank, self.size = comm.rank, comm.size

    def close(self):
        if self.h:
            self.L._L.amgt_dist_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _native_vcycle(self, native: NativeComm, b_own: torch.Tensor, x_own: torch.Tensor, ncycles: int):
    """Alg. 2 over the slabs inside libamgt (amgt_dist_vcycle): halo exchanges with NCCL on a
    side stream overlapped with the interior rows, device-side norms and coarse gather."""
    import ctypes
    from . import _lib
    keep = []
    levels = (_lib.c_dist_level * self.nlev)()
    for k, L in enumerate(self.levels):
        d = levels[k]
        d.A = ctypes.addressof(L.A.c)
        d.P = ctypes.addressof(L.P.c) if L.P is not None else None
        d.R = ctypes.addressof(L.R.c) if L.R is not None else None
        d.m, d.off, d.int0, d.int1 = L.m, L.off, L.int0, L.int1
        d.xe[0], d.xe[1] = L.xe[0].data_ptr(), L.xe[1].data_ptr()
        d.b, d.r = L.b.data_ptr(), L.r.data_ptr()
        d.dinv = L.dinv.data_ptr() if L.dinv.numel() else None
        d.vprec = 0 if L.vdt == torch.float64 else 1
        sp = np.array([q for q, _, _ in L.plan.sends], dtype=np.int32)
        so = np.array([g0 - L.eb for _, g0, _ in L.plan.sends], dtype=np.int64)
        sc = np.array([g1 - g0 for _, g0, g1 in L.plan.sends], dtype=np.int64)
        rp = np.array([q for q, _, _ in L.plan.recvs], dtype=np.int32)
        ro = np.array([g0 - L.eb for _, g0, _ in L.plan.recvs], dtype=np.int64)
        rc = np.array([g1 - g0 for _, g0, g1 in L.plan.recvs], dtype=np.int64)
        keep += [sp, so, sc, rp, ro, rc]
        d.nsend, d.nrecv = len(sp), len(rp)
        d.send_peer, d.send_off, d.send_cnt = sp.ctypes.data, so.ctypes.data, sc.ctypes.data
        d.recv_peer, d.recv_off, d.recv_cnt = rp.ctypes.data, ro.ctypes.data, rc.ctypes.data
    C = self.levels[-1]
    counts = np.array([e - b for b, e in self.coarse_ranges], dtype=np.int64)
    displs = np.array([b for b, _ in self.coarse_ranges], dtype=np.int64)
    bfull = torch.zeros(self.nM, dtype=C.vdt, device=self.ops.device)
    xfull = torch.zeros(self.nM, dtype=C.vdt, device=self.ops.device)
    keep += [counts, displs, bfull, xfull]
    co = _lib.c_dist_coarse(self.nM, self.Ainv.data_ptr(), counts.ctypes.data, displs.ctypes.data, bfull.data_ptr(),
                            xfull.data_ptr())
    res = (ctypes.c_double * (ncycles + 1))()
    calls = ctypes.c_int64(0)
    _lib._check(_lib._L.amgt_dist_vcycle(native.h, self.nlev, levels, ctypes.byref(co), float(self.omega), int(self.nu1),
                                         int(self.nu2), b_own.data_ptr(), x_own.data_ptr(), int(ncycles), res,
                                         ctypes.byref(calls), _lib._stream()))
    del keep
    return list(res), int(calls.value)


DistHierarchy.native_vcycle = _native_vcycle
