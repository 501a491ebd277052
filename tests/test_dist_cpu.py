"""Distributed path on CPU, world size 2 and 3 over gloo.

The native library computes every rank's halo plan from the all-gathered (rows, min tile column,
max tile column) metadata (`amgt_dist_plan_host`, host-only C code — the same function the CUDA
path calls).  Each rank here builds its row slab, all-gathers the metadata over gloo, asks the
library for its plan and then executes the plan with gloo point-to-point transfers and the
oracle as the compute backend:
  * the distributed SpMV (halo of x per the plan, own rows of A x) equals the global oracle's
    rows bit for bit (integer x);
  * the distributed RAP (P rows of the halo gathered per the plan, A_l P_ext, then
    R_loc (AP) with R_loc = P_own^T) equals the global oracle's R (A P) rows bit for bit;
  * the send / receive pieces of all ranks match pairwise, and a rank's received pieces plus its
    own rows tile its extended range exactly.
"""
import os
import queue
import socket
import time

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tile_range(rp, col):
    return (int(col.min()) // 4, int(col.max()) // 4) if col.size else (1, 0)


def _send_recv(sends, recvs):
    """sends/recvs: [(peer, numpy array)] exchanged with gloo (recv arrays filled in place)."""
    works = []
    hs = []
    for p, a in sends:
        t = torch.from_numpy(np.ascontiguousarray(a))
        hs.append(t)
        works.append(dist.isend(t, p))
    hr = []
    for p, a in recvs:
        t = torch.from_numpy(a)
        hr.append(t)
        works.append(dist.irecv(t, p))
    for w in works:
        w.wait()


def _worker(rank, size, port, kind, dims, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=size)
    try:
        from paper_conf_sc_luzwflcy0c024_b200.dist import plan_host
        A, rows, n, Ps = gen.partition.slab_inputs(kind, dims, 2, rank, size)
        Ao = oracle.as_csr(A)
        Po = oracle.as_csr(Ps[0])
        m = rows[1] - rows[0]
        lo, hi = _tile_range(Ao.row_ptr, Ao.col)
        meta = [None] * size
        dist.all_gather_object(meta, (m, lo, hi))
        (eb, ee), recv, send = plan_host(rank, [t[0] for t in meta], [t[1] for t in meta], [t[2] for t in meta])
        rb, re_ = rows[0] // 4, (rows[1] + 3) // 4
        # ---- distributed SpMV: x = global row index (integers)
        xe = np.zeros(4 * (ee - eb))
        xe[4 * (rb - eb):4 * (rb - eb) + m] = np.arange(rows[0], rows[1], dtype=np.float64)
        _send_recv([(p, xe[4 * (g0 - eb):4 * (g1 - eb)].copy()) for p, g0, g1 in send],
                   [(p, xe[4 * (g0 - eb):4 * (g1 - eb)]) for p, g0, g1 in recv])
        A_ext = oracle.Csr(m, 4 * (ee - eb), Ao.row_ptr, (Ao.col.astype(np.int64) - 4 * eb).astype(np.int32), Ao.val)
        y = oracle.spmv(A_ext, xe)
        # ---- distributed RAP: gather the P rows of [eb, ee) per the plan (row lengths, then rows)
        prp = Po.row_ptr
        lens_send = [(p, np.diff(prp[4 * (g0 - rb):4 * (g1 - rb) + 1]).astype(np.int64)) for p, g0, g1 in send]
        lens_recv = [(p, np.zeros(4 * (g1 - g0), dtype=np.int64)) for p, g0, g1 in recv]
        _send_recv(lens_send, lens_recv)
        cs, vs = [], []
        for (p, g0, g1) in send:
            a, b = prp[4 * (g0 - rb)], prp[4 * (g1 - rb)]
            cs.append((p, Po.col[a:b].astype(np.int32)))
            vs.append((p, Po.val[a:b].astype(np.float64)))
        cr = [(p, np.zeros(int(l.sum()), dtype=np.int32)) for p, l in lens_recv]
        vr = [(p, np.zeros(int(l.sum()), dtype=np.float64)) for p, l in lens_recv]
        _send_recv(cs, cr)
        _send_recv(vs, vr)
        nrows_ext = min(4 * ee, n) - 4 * eb
        lens = np.zeros(nrows_ext, dtype=np.int64)
        cols = [None] * nrows_ext
        vals = [None] * nrows_ext
        pieces = [(g0, l, c, v) for (p, g0, g1), (_, l), (_, c), (_, v) in zip(recv, lens_recv, cr, vr)]
        pieces.append((rb, np.diff(prp).astype(np.int64), Po.col, Po.val))
        for g0, l, c, v in pieces:
            off = np.concatenate([[0], np.cumsum(l)])
            for i in range(l.size):
                r = 4 * (g0 - eb) + i
                if r < nrows_ext:
                    lens[r] = l[i]
                    cols[r] = c[off[i]:off[i + 1]]
                    vals[r] = v[off[i]:off[i + 1]]
        Pext = oracle.Csr(nrows_ext, Po.n, np.concatenate([[0], np.cumsum(lens)]).astype(np.int64),
                          np.concatenate([c for c in cols if c is not None]).astype(np.int32),
                          np.concatenate([v for v in vals if v is not None]).astype(np.float64))
        A_ext2 = oracle.Csr(m, nrows_ext, Ao.row_ptr, (Ao.col.astype(np.int64) - 4 * eb).astype(np.int32), Ao.val)
        AP = oracle.spgemm(A_ext2, Pext)
        cb = int(Po.col.min()) // 4
        ce = int(Po.col.max()) // 4 + 1
        Ploc = oracle.Csr(m, min(4 * ce, Po.n) - 4 * cb, Po.row_ptr, (Po.col.astype(np.int64) - 4 * cb).astype(np.int32),
                          Po.val)
        Ac = oracle.spgemm(oracle.transpose(Ploc), AP)
        q.put((rank, rows, (eb, ee), recv, send, y, (Ac.row_ptr, Ac.col, Ac.val), (cb, ce)))
    finally:
        dist.destroy_process_group()


def _run(kind, dims, size):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, size, port, kind, dims, q)) for r in range(size)]
    for p in procs:
        p.start()
    out, t0 = [], time.time()
    while len(out) < size:
        try:
            out.append(q.get(timeout=2))
        except queue.Empty:
            if any(p.exitcode not in (None, 0) for p in procs) or time.time() - t0 > 300:
                for p in procs:
                    p.kill()
                raise AssertionError(f"worker failed: {[p.exitcode for p in procs]}")
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return sorted(out, key=lambda t: t[0])


@pytest.mark.parametrize("kind,dims,size", [("7pt", (8, 8, 16), 2), ("27pt", (8, 8, 8), 2), ("7pt", (8, 8, 24), 3)])
def test_dist_plan_spmv_rap_match_oracle(kind, dims, size):
    out = _run(kind, dims, size)
    offs, center = gen.partition.STENCILS[kind]
    A = oracle.as_csr(gen.stencil(dims, offs, center, -1.0))
    P = oracle.as_csr(gen.aggregation_P(dims))
    y_glob = oracle.spmv(A, np.arange(A.n, dtype=np.float64))
    Ac = oracle.rap(oracle.transpose(P), A, P)
    plane = dims[0] * dims[1]
    for rank, rows, (eb, ee), recv, send, y, (rp, ci, v), (cb, ce) in out:
        # SpMV rows bit-exact
        assert np.array_equal(y, y_glob[rows[0]:rows[1]])
        # halo = one grid plane per neighbour (z-slabs): 7-point and 27-point reach +-1 plane
        rb, re_ = rows[0] // 4, rows[1] // 4
        assert eb == max(0, rb - plane // 4) and ee == min(A.m // 4, re_ + plane // 4)
        # received pieces + own rows tile [eb, ee)
        cover = sorted([(g0, g1) for _, g0, g1 in recv] + [(rb, re_)])
        pos = eb
        for g0, g1 in cover:
            assert g0 == pos
            pos = g1
        assert pos == ee
        # RAP rows bit-exact (structure and values)
        r0, r1 = 4 * cb, min(4 * ce, Ac.m)
        ref_rp = Ac.row_ptr[r0:r1 + 1] - Ac.row_ptr[r0]
        assert np.array_equal(rp, ref_rp)
        assert np.array_equal(ci, Ac.col[Ac.row_ptr[r0]:Ac.row_ptr[r1]])
        assert np.array_equal(v, Ac.val[Ac.row_ptr[r0]:Ac.row_ptr[r1]])
    # pairwise: what q receives from r is exactly what r sends to q
    for rank, _, _, recv, _, _, _, _ in out:
        for p, g0, g1 in recv:
            assert (rank, g0, g1) in [(pp, a, b) for pp, a, b in out[p][4]]
    for rank, _, _, _, send, _, _, _ in out:
        for p, g0, g1 in send:
            assert (rank, g0, g1) in [(pp, a, b) for pp, a, b in out[p][3]]


def test_plan_host_edge_cases():
    from paper_conf_sc_luzwflcy0c024_b200 import AmgtError
    from paper_conf_sc_luzwflcy0c024_b200.dist import plan_host
    # one rank: no pieces, extended range = own rows
    assert plan_host(0, [16], [0], [3]) == ((0, 4), [], [])
    # a rank with no tiles (colmin > colmax) needs no halo but may still be sent nothing
    (e, r, s) = plan_host(1, [8, 8, 8], [0, 1, 0], [3, 0, 5])
    assert e == (2, 4) and r == [] and s == [(0, 2, 4), (2, 2, 4)]
    # wide halo spanning two ranks
    (e, r, s) = plan_host(2, [4, 4, 4, 4], [0, 0, 0, 3], [1, 2, 3, 3])
    assert e == (0, 4) and r == [(0, 0, 1), (1, 1, 2), (3, 3, 4)] and s == [(1, 2, 3)]
    # ragged row counts are only allowed on the last rank
    with pytest.raises(AmgtError):
        plan_host(0, [6, 8], [0, 0], [1, 3])
    plan_host(0, [8, 6], [0, 0], [1, 3])
