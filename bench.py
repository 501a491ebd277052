#!/usr/bin/env python
"""bench.py — one JSON line for the driver.

A step = one pass of the whole hot path over BASELINE config 2
(3D 7-point Laplacian 128^3, 2x2x2 aggregation P, 7 levels 128^3 -> 2^3):
  a1 CSR->mBSR of A and of every P_k; a2 per-level casts (FP64 / FP32 / FP16, L266);
  a3-a7 RAP per level (two SpGEMM calls each: binning, two-step hash symbolic, TC/CUDA-core
  numeric); R_k = P_k^T; a8 mBSR->CSR of the coarsest level + dense factorisation;
  a9/a10 50 V-cycles (L308) of weighted-Jacobi smoothing with load-balanced SpMV.
Inputs (CSR A, P_k, b) are resident in HBM when the timed region starts.

value = algorithmic bytes of the step (SURVEY §8(d) byte model per kernel, summed) / step
time, i.e. whole-job GB/s; the components (SpMV GB/s, SpGEMM GFLOP/s, setup / solve ms)
are reported beside it.  `--impl reference` runs the CPU oracle on a bounded sample of
the same workload (setup + a few cycles) in the same unit.
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMV GB/s, SpGEMM GFLOP/s (mBSR, 1–8 B200); AMG setup+solve s"
LEVEL_PREC = ("f64", "f32", "f16", "f16", "f16", "f16", "f16")


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        mode = os.environ.get("AMGT_BENCH_CLOCKS", "smi")  # smi | nvml (in-process) | off (testing only)
        if mode == "off":
            return self
        if mode == "nvml":
            try:
                import pynvml
                pynvml.nvmlInit()
                h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
                mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
                bits = (pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                        pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap)
                self.stop = threading.Event()

                def poll():
                    while not self.stop.is_set():
                        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                        r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                        self.lines.append(", ".join([str(sm), str(mx)] +
                                                    ["Active" if r & b else "Not Active" for b in bits]))
                        self.stop.wait(0.1)

                self.t = threading.Thread(target=poll, daemon=True)
                self.t.start()
            except Exception:
                self.stop = None
            return self
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            # nvidia-smi's start-up (driver queries) stalls CUDA calls of this process for
            # milliseconds: wait for its first sample so that happens before the timed region
            t0 = time.time()
            while not self.lines and time.time() - t0 < 5.0:
                time.sleep(0.02)
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if getattr(self, "stop", None) is not None:
            self.stop.set()
            self.t.join(timeout=5)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[2:6]):
                if v.lower() == "active":
                    reasons.add(n)
        busy = [s for s in sm if s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(busy) if busy else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ byte model
S_BYTES = {"f64": 8, "f32": 4, "f16": 2}


def byte_model(sz, cycles):
    """Algorithmic bytes of one step from structure sizes (identical for both arms).
    sz: {"A_nnz", "P_nnz": [..], "P_m": [..], "lev": [{"m","BR","BC","T"}], "P_T", "R_T", "AP_T": [..],
         "prec": [..]}.  Tiles count 16 s + 4 + 2 bytes (values, blc_idx, blc_map)."""
    L = len(sz["lev"])
    s = [S_BYTES[p] for p in sz["prec"]]
    vs = [8 if p == "f64" else 4 for p in sz["prec"]]
    tb = lambda T, sk: T * (16 * sk + 6)
    lev = sz["lev"]
    out = {}
    # a1: CSR -> mBSR of A (FP64) and of every P_k (FP64)
    c = sz["A_nnz"] * 12 + (lev[0]["m"] + 1) * 8 + tb(lev[0]["T"], 8) + (lev[0]["BR"] + 1) * 8
    for k in range(L - 1):
        c += sz["P_nnz"][k] * 12 + (sz["P_m"][k] + 1) * 8 + tb(sz["P_T"][k], 8) + (lev[k]["BR"] + 1) * 8
    out["csr2mbsr"] = c
    # a2: casts (A_{k+1} from level-k precision to level-(k+1); P_k from FP64 to level k)
    c = 0
    for k in range(L - 1):
        if s[k] != 8:
            c += 16 * sz["P_T"][k] * (8 + s[k])
        if s[k + 1] != s[k]:
            c += 16 * lev[k + 1]["T"] * (s[k] + s[k + 1])
    out["cast"] = c
    # a3-a7: two SpGEMMs per level; symbolic reads structure twice, writes C's; numeric
    # reads operands once and writes C once
    sym = num = 0
    for k in range(L - 1):
        TA, TP, TR, TAP, TC = lev[k]["T"], sz["P_T"][k], sz["R_T"][k], sz["AP_T"][k], lev[k + 1]["T"]
        sym += 2 * (TA + TP) * 6 + TAP * 6 + 2 * (TR + TAP) * 6 + TC * 6
        num += tb(TA, s[k]) + tb(TP, s[k]) + tb(TAP, s[k]) + tb(TR, s[k]) + tb(TAP, s[k]) + tb(TC, s[k])
        num += 2 * TP * (16 * s[k] + 6)  # R = P^T (tile transpose: read + write)
    out["spgemm_symbolic"], out["spgemm_numeric"] = sym, num
    out["mbsr2csr"] = tb(lev[-1]["T"], s[-1]) + lev[-1]["m"] * 20
    # a9/a10: the SpMV operations of Alg. 2, each counted with its own operand bytes (the
    # paper's SpMV GB/s convention; independent of how kernels fuse them): per cycle and level
    # k < L: pre-smoothing, residual, post-smoothing with A_k, restriction R_k, interpolation
    # P_k, plus on level 1 the residual reported after every cycle (L308) and the initial one.
    # Fused kernels serve several of these from one HBM pass (the level-1 sweeps read A_1 once
    # for three of them), so whole-step GB/s can exceed the HBM peak; the roofline object
    # reports the physical fraction of the dominant kernel.
    def spmv_b(T, BR, BC, sk, xs, ys):
        return tb(T, sk) + (BR + 1) * 8 + 4 * BC * xs + 4 * BR * ys
    sp1 = spmv_b(lev[0]["T"], lev[0]["BR"], lev[0]["BC"], s[0], vs[0], vs[0])
    l1 = sp1 * (4 if L > 1 else 1)
    other, vec = 0, 0
    for k in range(L - 1):
        if k > 0:
            other += 3 * spmv_b(lev[k]["T"], lev[k]["BR"], lev[k]["BC"], s[k], vs[k], vs[k])
        other += spmv_b(sz["R_T"][k], lev[k + 1]["BR"], lev[k]["BR"], s[k], vs[k], vs[k + 1])
        other += spmv_b(sz["P_T"][k], lev[k]["BR"], lev[k + 1]["BR"], s[k], vs[k + 1], vs[k])
        # vector operands of the Alg. 2 steps beyond the SpMV's own x/y: each Jacobi sweep
        # reads b and D^-1, the residual reads b, the correction reads x (6 vectors)
        vec += 6 * 4 * lev[k]["BR"] * vs[k]
    # coarse solve; residual b + norm read; the fused pre-smoothing pass also writes r
    vec += lev[-1]["m"] ** 2 * 8 + (3 if L > 1 else 2) * 4 * lev[0]["BR"] * 8
    out["spmv_l1"] = l1 * cycles + sp1
    out["spmv"] = other * cycles
    out["vector"] = vec * cycles
    return out


def sample_bytes_model(bm, cycles, total_cycles):
    setup = sum(bm[k] for k in ("spgemm_symbolic", "spgemm_numeric", "csr2mbsr", "mbsr2csr", "cast"))
    solve = sum(bm[k] for k in ("spmv_l1", "spmv", "vector"))
    return setup + solve * cycles / max(total_cycles, 1)


def gpu_sizes(amgt, A, Ps):
    """Structure sizes of the hierarchy built by the CUDA path (for the byte model)."""
    MA = amgt.from_csr(A)
    H = amgt.Hierarchy(MA, [amgt.from_csr(P) for P in Ps], level_prec=LEVEL_PREC[:len(Ps) + 1])
    sz = {"A_nnz": A.nnz, "P_nnz": [P.nnz for P in Ps], "P_m": [P.m for P in Ps], "lev": [], "P_T": [], "R_T": [],
          "AP_T": [], "prec": list(LEVEL_PREC[:len(Ps) + 1])}
    flops = 0
    for k in range(H.nlev):
        Ak, Pk, Rk = H.level(k)
        sz["lev"].append({"m": Ak.m, "BR": Ak.blc_row, "BC": Ak.blc_col, "T": Ak.blc_num})
        if Pk is not None:
            AP, i1 = amgt.spgemm_symbolic(Ak, Pk, info=True)
            _, i2 = amgt.spgemm_symbolic(Rk, AP, info=True)
            flops += 2 * (i1["scalar_products"] + i2["scalar_products"])
            sz["P_T"].append(Pk.blc_num)
            sz["R_T"].append(Rk.blc_num)
            sz["AP_T"].append(AP.blc_num)
            AP.free()
    H.close()
    MA.free()
    return sz, flops


def oracle_sizes(A, PR):
    import oracle
    Ao = oracle.as_csr(A.to("cpu"))
    PRo = [(oracle.as_csr(P.to("cpu")), oracle.as_csr(R.to("cpu"))) for P, R in PR]
    As = oracle.build_hierarchy(Ao, PRo)
    sz = {"A_nnz": Ao.nnz, "P_nnz": [P.nnz for P, _ in PRo], "P_m": [P.m for P, _ in PRo], "lev": [], "P_T": [],
          "R_T": [], "AP_T": [], "prec": list(LEVEL_PREC[:len(As)])}
    for k, Ak in enumerate(As):
        T = oracle.csr_to_mbsr(Ak).blc_num
        sz["lev"].append({"m": Ak.m, "BR": (Ak.m + 3) // 4, "BC": (Ak.n + 3) // 4, "T": T})
        if k + 1 < len(As):
            P, R = PRo[k]
            sz["P_T"].append(oracle.csr_to_mbsr(P).blc_num)
            sz["R_T"].append(oracle.csr_to_mbsr(R).blc_num)
            sz["AP_T"].append(oracle.csr_to_mbsr(oracle.spgemm(Ak, P)).blc_num)
    return sz


# ------------------------------------------------------------------ workload
L1_SAMPLE = 10  # live events on every 10th level-1 SpMV of the timed steps


def make_inputs(cfg, device):
    import gen
    N = cfg.N
    A = gen.configs.build_matrix(cfg, device=device)
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device=device)
    Ps = [P for P, _ in PR]
    b = gen.uniform_vector(A.m, cfg.seed).to(device)
    return A, Ps, b, PR, N


def gpu_step(amgt, A, Ps, b, x, ncycles, torch, after_setup=None):
    """The whole hot path once (inputs on the device).  after_setup: called once the
    hierarchy exists (the e2e leg enqueues the next step's upload there)."""
    MA = amgt.from_csr(A)                       # a1
    MPs = [amgt.from_csr(P) for P in Ps]        # a1 (P_k)
    H = amgt.Hierarchy(MA, MPs, level_prec=LEVEL_PREC[:len(Ps) + 1])  # a2-a8
    if after_setup is not None:
        after_setup()
    x.zero_()
    res, calls = H.vcycle(b, x, ncycles)        # a9-a10
    H.close()
    MA.free()
    for M in MPs:
        M.free()
    return res, calls


def run_dist(args, rank, world, local):
    """N > 1: the row-slab partitioned path, weak scaling — every rank owns a
    128^3 slab of a 128 x 128 x (128 N) 7-point grid (N = 1 would be config 2 exactly);
    halo exchanges over NCCL, all-reduced norms, all-gathered coarsest RHS."""
    import torch
    import torch.distributed as dist

    import gen
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    from paper_conf_sc_luzwflcy0c024_b200.dist import Comm, DistHierarchy

    # stdout carries the one JSON line: library banners printed from C (the NCCL version line)
    # go to stderr while the run is set up and measured
    sys.stdout.flush()
    json_fd = os.dup(1)
    os.dup2(2, 1)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    comm = Comm()
    cfg = gen.configs.CONFIGS["cfg2"]
    dims = (cfg.N, cfg.N, cfg.N * world)
    nlev = cfg.nlev
    A, rows, n, Ps = gen.partition.slab_inputs("7pt", dims, nlev, rank, world, alpha=cfg.alpha, device="cuda")
    m = rows[1] - rows[0]
    b = gen.uniform_vector(n, cfg.seed)[rows[0]:rows[1]].cuda()
    x = torch.zeros(m, dtype=torch.float64, device="cuda")
    # per-rank algorithmic bytes: the config-2 byte model (each rank's slab is a 128^3 block)
    A2, Ps2, _, _, _ = make_inputs(cfg, "cuda")
    sz, flops = gpu_sizes(amgt, A2, Ps2)
    bm = byte_model(sz, args.cycles)
    bytes_rank = sum(bm.values())
    del A2, Ps2

    from paper_conf_sc_luzwflcy0c024_b200.dist import NativeComm
    native = NativeComm(comm)  # libamgt-owned NCCL communicator for the native V-cycle

    def step():
        H = DistHierarchy(comm, A, rows, n, Ps, level_prec=LEVEL_PREC[:nlev])
        x.zero_()
        res, calls = H.native_vcycle(native, b, x, args.cycles)
        return H, res, calls

    for _ in range(args.warmup):
        step()
    stream = torch.cuda.current_stream()
    dist.barrier()
    torch.cuda.synchronize()
    launches0 = amgt.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gc.collect()
    gc.disable()  # no collector pause inside the timed region (host stalls starve the GPU queue)
    with ClockSampler(local) as clk:
        e0.record(stream)
        host_ms = []
        for _ in range(args.steps):
            t_h = time.perf_counter()
            H, res, calls = step()
            host_ms.append(round((time.perf_counter() - t_h) * 1e3, 2))
        e1.record(stream)
        dist.barrier()
        torch.cuda.synchronize()
    gc.enable()
    print(f"[bench] host ms per timed step (enqueue + host syncs): {host_ms}", file=sys.stderr)
    ms = torch.tensor([e0.elapsed_time(e1) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_step = float(ms.item())
    launches = amgt.launch_count() - launches0
    # distributed level-1 SpMV (halo exchange + interior/boundary kernels), timed with events
    L0 = H.levels[0]
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(20)]
    y = torch.empty_like(L0.r)
    for a_, b_ in ev:
        a_.record(stream)
        L0.spmv(L0.cur, y, "y")
        b_.record(stream)
    torch.cuda.synchronize()
    spmv_ms = sum(a_.elapsed_time(b_) for a_, b_ in ev) / len(ev)
    # e2e: the same step with this rank's inputs (slab CSR of A, the P_k rows, b) uploaded from
    # pinned host memory every step and x read back, max over ranks
    CSR = type(A)
    hA = CSR(A.m, A.n, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(), A.val.cpu().pin_memory())
    hPs = [CSR(P.m, P.n, P.row_ptr.cpu().pin_memory(), P.col.cpu().pin_memory(), P.val.cpu().pin_memory()) for P in Ps]
    hb = b.cpu().pin_memory()
    hx = torch.empty(x.numel(), dtype=torch.float64).pin_memory()
    h2d = sum(t.numel() * t.element_size() for M in [hA, *hPs] for t in (M.row_ptr, M.col, M.val)) + hb.numel() * 8
    d2h = hx.numel() * 8 + (args.cycles + 1) * 8

    # as the single-GPU leg: uploads on a copy stream into two buffer sets, step i+1's upload
    # enqueued once step i's hierarchy exists (it overlaps step i's V-cycles)
    host_in = [hA.row_ptr, hA.col, hA.val] + [t for P in hPs for t in (P.row_ptr, P.col, P.val)] + [hb]
    dev_in = [[torch.empty(t.shape, dtype=t.dtype, device="cuda") for t in host_in] for _ in range(2)]
    cs = torch.cuda.Stream()
    ev_in = [torch.cuda.Event(), torch.cuda.Event()]

    def upload(k):
        with torch.cuda.stream(cs):
            for d, h in zip(dev_in[k], host_in):
                d.copy_(h, non_blocking=True)
            ev_in[k].record(cs)

    def e2e_step(k, nxt):
        stream.wait_event(ev_in[k])
        d = dev_in[k]
        dA = CSR(hA.m, hA.n, d[0], d[1], d[2])
        dPs = [CSR(P.m, P.n, d[3 + 3 * i], d[4 + 3 * i], d[5 + 3 * i]) for i, P in enumerate(hPs)]
        H_ = DistHierarchy(comm, dA, rows, n, dPs, level_prec=LEVEL_PREC[:nlev])
        if nxt is not None:
            upload(nxt)
        x.zero_()
        H_.native_vcycle(native, d[-1], x, args.cycles)
        hx.copy_(x, non_blocking=True)

    upload(0)
    e2e_step(0, None)
    dist.barrier()
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    cs.wait_event(f0)
    upload(0)
    for i in range(args.steps):
        e2e_step(i % 2, (i + 1) % 2 if i + 1 < args.steps else None)
    f1.record(stream)
    dist.barrier()
    torch.cuda.synchronize()
    e2e_t = torch.tensor([f0.elapsed_time(f1) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_ms = float(e2e_t.item())
    l0 = sz["lev"][0]
    sp_bytes = l0["T"] * (16 * 8 + 6) + (l0["BR"] + 1) * 8 + 8 * 4 * l0["BC"] + 8 * 4 * l0["BR"]
    peak, peak_kind = _peaks()
    achieved = sp_bytes / (spmv_ms * 1e-3) / 1e9
    sys.stdout.flush()
    os.dup2(json_fd, 1)
    os.close(json_fd)
    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": round(bytes_rank * world / (ms_step * 1e-3) / 1e9, 2), "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64/f32/f16 (per AMG level, L266)",
            "data": "synthetic",
            "config": {"workload": f"7-point Laplacian {dims[0]}x{dims[1]}x{dims[2]} row-slab partitioned over {world} GPUs "
                                   f"(128^3 per rank; N=1 is config 2)", "levels": nlev, "vcycles_per_step": args.cycles,
                       "parallelism": f"row-slab x{world} (NCCL halo exchange overlapped with interior rows, all-reduce, all-gather)",
                       "l2": "inputs larger than L2; no flush", "spmv_calls_per_step": calls},
            "roofline": {"kernel": "distributed level-1 FP64 SpMV (halo exchange + k_spmv_rows interior/boundary)",
                         "bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "peak_source": peak_kind, "bytes_per_launch": sp_bytes,
                         "avg_launch_us": round(spmv_ms * 1e3, 2), "traffic": None},
            "components": {"final_rel_residual": res[-1] / res[0], "bytes_per_rank_step": bytes_rank},
            "e2e": {"value": round(bytes_rank * world / (e2e_ms * 1e-3) / 1e9, 2), "unit": "GB/s",
                    "ms_per_step": round(e2e_ms, 3), "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world,
                    "copies": "each rank uploads its slab inputs from pinned host memory every step (copy stream, "
                              "double-buffered, overlapping the previous step's V-cycles) and reads x back"},
            "gpu_launches": launches, "clocks": clk.summary(),
        }), flush=True)
    dist.destroy_process_group()


def run_gpu(args):
    import numpy as np
    import torch

    import gen
    import paper_conf_sc_luzwflcy0c024_b200 as amgt

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dist = None
    if world > 1 or args.force_dist:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if "MASTER_PORT" not in os.environ:
            import socket
            with socket.socket() as so:
                so.bind(("127.0.0.1", 0))
                os.environ["MASTER_PORT"] = str(so.getsockname()[1])
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
        return run_dist(args, rank, world, local)
    cfg = gen.configs.CONFIGS[args.config]
    A, Ps, b, PR, N = make_inputs(cfg, "cuda")
    x = torch.zeros(4 * ((A.m + 3) // 4), dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    # ---- warm-up
    for _ in range(args.warmup):
        gpu_step(amgt, A, Ps, b, x, args.cycles, torch)
    # ---- one instrumented step (after warm-up: warm allocator): per-class device times
    amgt.timing_reset()
    amgt.timing_enable(True)
    res, calls = gpu_step(amgt, A, Ps, b, x, args.cycles, torch)
    torch.cuda.synchronize()
    prof = amgt.timing_read()
    amgt.timing_enable(False)
    sz, flops = gpu_sizes(amgt, A, Ps)
    bm = byte_model(sz, args.cycles)
    bytes_step = sum(bm.values())
    l0 = sz["lev"][0]
    spmv_l1_bytes = l0["T"] * (16 * 8 + 6) + (l0["BR"] + 1) * 8 + 4 * l0["BC"] * 8 + 4 * l0["BR"] * 8

    barrier()

    # ---- timed region: K steps, live events around every level-1 SpMV (dominant kernel)
    amgt.timing_reset()
    amgt.timing_enable(1)  # only the dominant kernel class (level-1 SpMV) records events,
    amgt.timing_sample(L1_SAMPLE)  # on one launch in L1_SAMPLE (an event pair breaks the PDL overlap)
    launches0 = amgt.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gc.collect()
    gc.disable()  # no collector pause inside the timed region (host stalls starve the GPU queue)
    with ClockSampler(local) as clk:
        barrier()
        ev0.record(stream)
        host_ms = []
        for _ in range(args.steps):
            t_h = time.perf_counter()
            gpu_step(amgt, A, Ps, b, x, args.cycles, torch)
            host_ms.append(round((time.perf_counter() - t_h) * 1e3, 2))
        ev1.record(stream)
        barrier()
    gc.enable()
    print(f"[bench] host ms per timed step (enqueue + host syncs): {host_ms}", file=sys.stderr)
    launches = amgt.launch_count() - launches0
    live = amgt.timing_read()
    amgt.timing_enable(False)
    amgt.timing_sample(1)
    ms_total = ev0.elapsed_time(ev1)
    if dist:
        t = torch.tensor([ms_total], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
    ms_step = ms_total / args.steps
    value = bytes_step * world / (ms_step * 1e-3) / 1e9

    spmv_l1 = live["spmv_l1"]
    n_l1 = max(spmv_l1["launches"], 1)
    spmv_avg_ms = spmv_l1["ms"] / n_l1
    l1_bytes_per_launch = spmv_l1["bytes"] / n_l1  # SpMV bytes + fused epilogue vectors, per launch
    achieved = l1_bytes_per_launch / (spmv_avg_ms * 1e-3) / 1e9
    peak, peak_kind = _peaks()
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_spmv_l1_traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    setup_ms = sum(prof[k]["ms"] for k in ("spgemm_symbolic", "spgemm_numeric", "csr2mbsr", "mbsr2csr", "cast"))
    spgemm_ms = prof["spgemm_symbolic"]["ms"] + prof["spgemm_numeric"]["ms"]

    # ---- e2e: same step through the public API with host (pinned) inputs and outputs
    hA = type(A)(A.m, A.n, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(), A.val.cpu().pin_memory())
    hPs = [type(P)(P.m, P.n, P.row_ptr.cpu().pin_memory(), P.col.cpu().pin_memory(), P.val.cpu().pin_memory())
           for P in Ps]
    hb = b.cpu().pin_memory()
    hx = torch.empty(x.numel(), dtype=torch.float64).pin_memory()
    h2d = sum(t.numel() * t.element_size() for M in [hA, *hPs] for t in (M.row_ptr, M.col, M.val)) + hb.numel() * 8
    d2h = hx.numel() * 8 + (args.cycles + 1) * 8
    e2e_steps = args.steps

    def to_dev(t):
        d = torch.empty(t.shape, dtype=t.dtype, device="cuda")
        d.copy_(t, non_blocking=True)
        return d

    def to_dev_csr(M):
        return type(M)(M.m, M.n, to_dev(M.row_ptr), to_dev(M.col), to_dev(M.val))

    for _ in range(args.warmup):  # warm the allocator for the copied-input pattern
        gpu_step(amgt, to_dev_csr(hA), [to_dev_csr(P) for P in hPs], to_dev(hb), x, args.cycles, torch)
    # Every step copies its own inputs (A, the P_k, b) from pinned host memory and reads x
    # back; the copies run on a second stream into two buffer sets, so step i+1's upload
    # overlaps step i's compute (its buffers were last used by step i-1, finished: the
    # V-cycle call returns its residual norms to the host).
    host_in = [hA.row_ptr, hA.col, hA.val] + [t for P in hPs for t in (P.row_ptr, P.col, P.val)] + [hb]
    dev_in = [[torch.empty(t.shape, dtype=t.dtype, device="cuda") for t in host_in] for _ in range(2)]
    cs = torch.cuda.Stream()
    ev_in = [torch.cuda.Event(), torch.cuda.Event()]

    def upload(k):
        with torch.cuda.stream(cs):
            for d, h in zip(dev_in[k], host_in):
                d.copy_(h, non_blocking=True)
            ev_in[k].record(cs)

    def unpack(k):
        d = dev_in[k]
        dA = type(hA)(hA.m, hA.n, d[0], d[1], d[2])
        dPs = [type(P)(P.m, P.n, d[3 + 3 * i], d[4 + 3 * i], d[5 + 3 * i]) for i, P in enumerate(hPs)]
        return dA, dPs, d[-1]

    # x alternates between two device buffers so that step i's read-back (on the copy stream)
    # overlaps step i+1
    xs = [x, torch.empty_like(x)]
    ev_out = torch.cuda.Event()
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    cs.wait_event(e0)
    upload(0)
    for i in range(e2e_steps):
        stream.wait_event(ev_in[i % 2])
        dA, dPs, db = unpack(i % 2)
        # step i+1's upload is enqueued once step i's hierarchy exists: it then overlaps the
        # V-cycles instead of competing with the setup's small synchronised read-backs
        nxt = (lambda k=(i + 1) % 2: upload(k)) if i + 1 < e2e_steps else None
        gpu_step(amgt, dA, dPs, db, xs[i % 2], args.cycles, torch, after_setup=nxt)  # norms come back here
        ev_out.record(stream)
        cs.wait_event(ev_out)
        with torch.cuda.stream(cs):
            hx.copy_(xs[i % 2], non_blocking=True)
    stream.wait_stream(cs)
    e1.record(stream)
    barrier()
    e2e_ms = e0.elapsed_time(e1) / e2e_steps
    if dist:
        t = torch.tensor([e2e_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t.item())
    e2e_val = bytes_step * world / (e2e_ms * 1e-3) / 1e9

    line = {
        "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64/f32/f16 (per AMG level, L266)", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg.description}", "grid": f"{N}^3", "levels": len(Ps) + 1,
                   "level_prec": list(LEVEL_PREC[:len(Ps) + 1]), "vcycles_per_step": args.cycles,
                   "smoother": "weighted Jacobi w=2/3, nu1=nu2=1", "parallelism": f"replicas x{world}",
                   "l2": "inputs larger than L2 (level-1 mBSR A = %.0f MB vs 126 MB L2); no flush" %
                         (A1_bytes_mb(A)), "spmv_calls_per_step": calls},
        "roofline": {"kernel": ("k_sweep (level-1 FP64 A_1: post-smoothing, pre-smoothing + residual norm, residual "
                                "as one wavefront pass over HBM; achieved = A_1 once + stage vectors per launch)"
                                if os.environ.get("AMGT_SWEEP", "0") == "1" else
                                "k_spmv_rows<double,double,double> (level-1 FP64 SpMV of A_1, fused Alg. 2 epilogues)"),
                     "bound": "hbm",
                     "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "peak_source": peak_kind,
                     "bytes_per_launch": round(l1_bytes_per_launch), "plain_spmv_bytes": spmv_l1_bytes,
                     "avg_launch_us": round(spmv_avg_ms * 1e3, 2),
                     "launches_timed": spmv_l1["launches"], "launch_sampling": f"1 in {L1_SAMPLE}",
                     "traffic": traffic},
        "components": {"setup_ms": round(setup_ms, 3), "solve_ms": round(ms_step - setup_ms, 3),
                       "spmv_l1_gbs": round(achieved, 1),
                       "spgemm_gflops": round(flops / (spgemm_ms * 1e-3) / 1e9, 2) if spgemm_ms else None,
                       "spgemm_roofline": {
                           "bound": "hbm", "unit": "GB/s", "peak": peak,
                           "achieved": round((bm["spgemm_symbolic"] + bm["spgemm_numeric"]) / (spgemm_ms * 1e-3) / 1e9, 1)
                           if spgemm_ms else None,
                           "frac": round((bm["spgemm_symbolic"] + bm["spgemm_numeric"]) / (spgemm_ms * 1e-3) / 1e9 / peak, 4)
                           if spgemm_ms else None,
                           "scope": "every SpGEMM call of the setup (symbolic + numeric, all levels; instrumented step), "
                                    "algorithmic bytes of SURVEY 8(d)"},
                       "rap_flops": flops, "bytes_per_step": bytes_step,
                       "bytes_by_phase": {k: int(v) for k, v in bm.items()},
                       "per_class_ms": {k: round(v["ms"], 3) for k, v in prof.items()},
                       "final_rel_residual": res[-1] / res[0]},
        "e2e": {"value": round(e2e_val, 2), "unit": "GB/s", "ms_per_step": round(e2e_ms, 3),
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "copies": "pinned host inputs uploaded every step on a copy stream, double-buffered "
                          "(step i+1's upload overlaps step i's V-cycles); x (double-buffered, read back on the "
                          "copy stream) and the residual norms read back every step"},
        "gpu_launches": launches,
        "clocks": clk.summary(),
    }
    if rank == 0 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(args, bm, A, PR)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def A1_bytes_mb(A):
    # rough level-1 mBSR footprint (FP64 tiles) from the CSR size: reported in config only
    return A.nnz * 134.0 / 4.0 / 1e6


# ------------------------------------------------------------------ oracle (CPU) legs
def oracle_sample(args, A, PR, cycles):
    """The oracle's version of a step, on a bounded number of V-cycles."""
    import gen
    import oracle
    t0 = time.perf_counter()
    Ao = oracle.as_csr(A.to("cpu"))
    oracle.csr_to_mbsr(Ao)                     # a1 (level 1)
    PRo = [(oracle.as_csr(P.to("cpu")), oracle.as_csr(R.to("cpu"))) for P, R in PR]
    As = oracle.build_hierarchy(Ao, PRo)       # a7 (RAP chain)
    for Ak in As[1:]:
        oracle.mbsr_to_csr(oracle.csr_to_mbsr(Ak))  # a8 round trips (2L-1 conversions)
    b = gen.uniform_vector(Ao.m, gen.configs.CONFIGS[args.config].seed).numpy()
    t1 = time.perf_counter()
    oracle.vcycle(As, PRo, b, ncycles=cycles)
    t2 = time.perf_counter()
    return t1 - t0, t2 - t1


def cpu_baseline(args, bm, A, PR):
    import oracle
    cycles = args.cpu_cycles
    ts, tv = oracle_sample(args, A, PR, cycles)
    by = sample_bytes_model(bm, cycles, args.cycles)
    return {"value": round(by / (ts + tv) / 1e9, 4), "unit": "GB/s", "cores": oracle.max_threads(), "kind": "oracle",
            "sample": f"{args.config}: CSR->mBSR + full RAP hierarchy + {cycles} of {args.cycles} V-cycles "
                      f"(FP64 C oracle, OpenMP rows); setup {ts:.2f}s, solve {tv:.2f}s"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import gen
    import oracle
    cfg = gen.configs.CONFIGS[args.config]
    A, Ps, b, PR, N = make_inputs(cfg, "cpu")
    bm = byte_model(oracle_sizes(A, PR), args.cycles)  # same byte model as the GPU arm
    cycles = args.cpu_cycles
    for _ in range(args.warmup):
        oracle_sample(args, A, PR, cycles)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle_sample(args, A, PR, cycles)
    dt = (time.perf_counter() - t0) / args.steps
    val = sample_bytes_model(bm, cycles, args.cycles) / dt / 1e9
    sample = f"{args.config}: CSR->mBSR + full RAP hierarchy + {cycles} of {args.cycles} V-cycles per step (FP64 C oracle)"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(val, 4), "unit": "GB/s", "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 2), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg.description}", "levels": cfg.nlev},
        "cpu_baseline": {"value": round(val, 4), "unit": "GB/s", "cores": oracle.max_threads(), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(val, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="amgt", choices=["amgt", "reference"])
    ap.add_argument("--config", default="cfg2", choices=["cfg2", "cfg3", "cfg5"])
    ap.add_argument("--cycles", type=int, default=50, help="V-cycles per step (paper: 50, L308)")
    ap.add_argument("--cpu-cycles", type=int, default=10, help="V-cycles in the oracle's bounded sample")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--force-dist", action="store_true", help="use the partitioned path even at N = 1 (testing)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "amgt" else args.warmup
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
