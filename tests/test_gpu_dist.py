"""Distributed path with the CUDA kernels: 2 ranks sharing cuda:0 (gloo,
host-staged halos — NCCL refuses two ranks on one device).  Same parity bar as the single-
GPU V-cycle: FP64 hierarchy reproduces the oracle's residual history; mixed precision keeps
the per-cycle reduction within 1%; the distributed SpMV equals the oracle's bit for bit on
integer data."""
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

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, size, port, kind, dims, nlev, prec, ncyc, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=size)
    try:
        from paper_conf_sc_luzwflcy0c024_b200.dist import Comm, DistHierarchy
        A, rows, n, Ps = gen.partition.slab_inputs(kind, dims, nlev, rank, size, device="cuda")
        H = DistHierarchy(Comm(), A, rows, n, Ps, level_prec=prec)
        m = rows[1] - rows[0]
        b = gen.uniform_vector(n, 3)[rows[0]:rows[1]].cuda()
        x = torch.zeros(m, dtype=torch.float64, device="cuda")
        res, calls = H.vcycle(b, x, ncyc)
        L0 = H.levels[0]
        L0.own(0).copy_(torch.arange(rows[0], rows[1], dtype=torch.float64, device="cuda"))
        y = torch.zeros(4 * L0.BR, dtype=torch.float64, device="cuda")
        L0.spmv(0, y, "y")
        q.put((rank, res, calls, x.cpu().numpy(), y[:m].cpu().numpy(), rows))
    finally:
        dist.destroy_process_group()


def _run(kind, dims, nlev, prec, ncyc, size=2):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, size, port, kind, dims, nlev, prec, ncyc, q)) for r in range(size)]
    for p in procs:
        p.start()
    out, t0 = [], time.time()
    while len(out) < size:
        try:
            out.append(q.get(timeout=2))
        except queue.Empty:
            if any(p.exitcode not in (None, 0) for p in procs) or time.time() - t0 > 600:
                for p in procs:
                    p.kill()
                raise AssertionError(f"worker failed: {[p.exitcode for p in procs]}")
    for p in procs:
        p.join(timeout=60)
    return sorted(out, key=lambda t: t[0])


@pytest.mark.parametrize("kind,dims,nlev,size", [("7pt", (16, 16, 32), 4, 2), ("27pt", (16, 16, 16), 3, 2),
                                                 ("7pt", (16, 16, 64), 4, 4)])
def test_dist_gpu_fp64_matches_oracle(kind, dims, nlev, size):
    ncyc = 5
    out = _run(kind, dims, nlev, ("f64",) * nlev, ncyc, size)
    offs, center = gen.partition.STENCILS[kind]
    A = gen.stencil(dims, offs, center, -1.0)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3).numpy()
    xo, res_o, calls_o = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=ncyc)
    yo = oracle.spmv(A, np.arange(A.n, dtype=np.float64))
    for rank, res, calls, x, y, rows in out:
        np.testing.assert_allclose(res, res_o, rtol=1e-9)
        np.testing.assert_allclose(x, xo[rows[0]:rows[1]], rtol=0, atol=1e-10 * np.abs(xo).max())
        assert calls == calls_o
        assert np.array_equal(y, yo[rows[0]:rows[1]])


def test_dist_gpu_mixed_precision_rho():
    kind, dims, nlev, ncyc = "27pt", (32, 32, 32), 4, 8
    out = _run(kind, dims, nlev, ("f64", "f32", "f16", "f16"), ncyc)
    offs, center = gen.partition.STENCILS[kind]
    A = gen.stencil(dims, offs, center, -1.0)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3).numpy()
    _, res_o, _ = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=ncyc)
    res_o = np.array(res_o)
    rho_o = res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    for rank, res, calls, x, y, rows in out:
        res = np.array(res)
        rho = res[1:] / res[:-1]
        assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)


def _native_worker(port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        import paper_conf_sc_luzwflcy0c024_b200 as amgt
        from paper_conf_sc_luzwflcy0c024_b200.dist import Comm, DistHierarchy, NativeComm
        comm = Comm()
        dims, nlev, prec = (32, 32, 32), 5, ("f64", "f32", "f16", "f16", "f16")
        A, rows, n, Ps = gen.partition.slab_inputs("7pt", dims, nlev, 0, 1, device="cuda")
        H = DistHierarchy(comm, A, rows, n, Ps, level_prec=prec)
        nat = NativeComm(comm)
        b = gen.uniform_vector(n, 3).cuda()
        x1 = torch.zeros(n, dtype=torch.float64, device="cuda")
        res_nat, calls_nat = H.native_vcycle(nat, b, x1, 6)
        x2 = torch.zeros(n, dtype=torch.float64, device="cuda")
        res_py, calls_py = H.vcycle(b, x2, 6)
        # the single-GPU library V-cycle on the same problem
        PR = gen.aggregation_hierarchy(dims, nlev)
        Hs = amgt.Hierarchy(amgt.from_csr(gen.laplacian_7pt(32, device="cuda")), [amgt.from_csr(P) for P, _ in PR],
                            level_prec=prec)
        x3 = torch.zeros(n, dtype=torch.float64, device="cuda")
        res_s, calls_s = Hs.vcycle(b, x3, 6)
        nat.close()
        q.put((res_nat, calls_nat, res_py, calls_py, res_s, calls_s, float((x1 - x3).abs().max()),
               float((x1 - x2).abs().max())))
    finally:
        dist.destroy_process_group()


def test_dist_native_single_rank_matches_single_gpu():
    """amgt_dist_vcycle (NCCL communicator, 1 rank) == the Python distributed driver == the
    single-GPU amgt_vcycle (same kernels, same per-row order)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_native_worker, args=(_free_port(), q))
    p.start()
    try:
        out = q.get(timeout=600)
    finally:
        p.join(timeout=60)
    res_nat, calls_nat, res_py, calls_py, res_s, calls_s, dx_s, dx_py = out
    assert calls_nat == calls_py == calls_s
    np.testing.assert_allclose(res_nat, res_s, rtol=1e-12)
    np.testing.assert_allclose(res_nat, res_py, rtol=1e-12)
    assert dx_s <= 1e-12 and dx_py <= 1e-12
