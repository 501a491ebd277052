"""Distributed driver on CPU: world size 2 over gloo, oracle-backed compute.
Checks the slab partition, extended column ranges, halo plans, the P-row gather of the
distributed RAP, the all-gathered coarsest solve and the all-reduced norms: the
distributed V-cycle must reproduce the global oracle's residual history (FP64)."""
import os
import socket

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


def _worker(rank, size, port, kind, dims, nlev, ncyc, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=size)
    try:
        from dist_oracle_ops import OracleOps
        from paper_conf_sc_luzwflcy0c024_b200.dist import Comm, DistHierarchy
        A, rows, n, Ps = gen.partition.slab_inputs(kind, dims, nlev, rank, size)
        comm = Comm()
        H = DistHierarchy(comm, A, rows, n, Ps, level_prec=("f64",) * nlev, ops=OracleOps())
        b = gen.uniform_vector(n, 3)[rows[0]:rows[1]].clone()
        x = torch.zeros(rows[1] - rows[0], dtype=torch.float64)
        res, calls = H.vcycle(b, x, ncyc)
        # distributed SpMV alone: y = A x for x = (1..n)
        L0 = H.levels[0]
        L0.own(0).copy_(torch.arange(rows[0], rows[1], dtype=torch.float64))
        y = torch.zeros(4 * L0.BR, dtype=torch.float64)
        L0.spmv(0, y, "y")
        q.put((rank, res, calls, x.numpy(), y[:rows[1] - rows[0]].numpy(), rows,
               [(Lk.rb, Lk.re, Lk.eb, Lk.ee) for Lk in H.levels]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("kind,dims,nlev", [("7pt", (8, 8, 16), 3), ("27pt", (8, 8, 8), 3)])
def test_dist_vcycle_world2_matches_oracle(kind, dims, nlev):
    size, ncyc = 2, 4
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, size, port, kind, dims, nlev, ncyc, q)) for r in range(size)]
    for p in procs:
        p.start()
    out = []
    import queue as _queue
    import time as _time
    t0 = _time.time()
    while len(out) < size:
        try:
            out.append(q.get(timeout=2))
        except _queue.Empty:
            if any(p.exitcode not in (None, 0) for p in procs) or _time.time() - t0 > 300:
                for p in procs:
                    p.kill()
                raise AssertionError(f"distributed worker failed: exit codes {[p.exitcode for p in procs]}")
    out.sort(key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # global oracle on the same problem
    offs, center = gen.partition.STENCILS[kind]
    A = gen.stencil(dims, offs, center, -1.0)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3).numpy()
    xo, res_o, calls_o = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=ncyc)
    for rank, res, calls, x, y, rows, lv in out:
        np.testing.assert_allclose(res, res_o, rtol=1e-10)
        np.testing.assert_allclose(x, xo[rows[0]:rows[1]], rtol=0, atol=1e-10 * np.abs(xo).max())
        assert calls == calls_o  # every rank issues every SpMV of Alg. 2
        yo = oracle.spmv(A, np.arange(A.n, dtype=np.float64))[rows[0]:rows[1]]
        assert np.array_equal(y, yo)
        for (rb, re_, eb, ee) in lv:  # extended ranges are 4-aligned and contain the own rows
            assert eb % 4 == 0 and eb <= rb < re_ <= ee
    # halos are exactly one plane on the 7-point level 1 (z-slab partition)
    if kind == "7pt":
        plane = dims[0] * dims[1]
        r0 = out[0][6][0]
        assert r0[3] - r0[1] == plane and out[1][6][0][0] - out[1][6][0][2] == plane
