#!/usr/bin/env python
"""bench.py — one JSON line for the driver.

A step = one pass of the whole hot path over one BASELINE workload:
  a1 CSR->mBSR of A and of every P_k; a2 per-level casts (FP64 / FP32 / FP16, L266);
  a3-a7 RAP per level (two SpGEMM calls each: binning, two-step hash symbolic, numeric);
  R_k = P_k^T; a8 mBSR->CSR of the coarsest level + dense factorisation;
  a9/a10 50 V-cycles (L308) of weighted-Jacobi smoothing with load-balanced SpMV.
Inputs (CSR A, P_k, b) are resident in HBM when the timed region starts.

Workload: N = 1 runs config 3 (27-point 256^3, 449M nonzeros, mixed FP64/FP32/FP16 levels) — the
largest single-GPU configuration; N > 1 (torchrun, NCCL) runs config 5 (7-point 512^3)
STRONG-scaled over the N ranks as z-slabs; `--config cfg5` at N = 1 is its G = 1
point (the single-GPU hierarchy).

value = physical algorithmic bytes of the step / step time: the SURVEY §8(d) byte figure of every
kernel launch the step makes (each SpMV / SpGEMM / conversion / cast / vector kernel counts its
own operands once — a fused kernel that serves two of Alg. 2's operations from one pass over A
counts that pass once), summed from one instrumented step.  `components.value_ops` is the
operation count convention (every one of Alg. 2's 1,551 SpMV operations with its own bytes).
The line also carries config 4's A*A SpGEMM (GFLOP/s and byte-roofline fraction).
`--impl reference` runs the CPU oracle on a bounded sample of the same workload.
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
AGG_ROWS = 262144  # distributed path: levels with <= 64^3 global rows agglomerated on every rank (DESIGN 9)
FLUSH_BYTES = 512 << 20  # > 2x the 126 MB L2


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region (nvidia-smi every 100 ms, or
    in-process NVML with AMGT_BENCH_CLOCKS=nvml; falls back to nvidia-smi when NVML fails)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []
        self.source = None
        self.stop = None

    def _nvml(self):
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
        mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        bits = (pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap)
        pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)  # fails here rather than in the thread
        self.stop = threading.Event()

        def poll():
            try:
                while not self.stop.is_set():
                    sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                    r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                    self.lines.append(", ".join([str(sm), str(mx)] + ["Active" if r & b else "Not Active" for b in bits]))
                    self.stop.wait(0.1)
            finally:
                try:
                    pynvml.nvmlShutdown()
                except Exception:
                    pass

        self.t = threading.Thread(target=poll, daemon=True)
        self.t.start()
        self.source = "nvml"

    def _smi(self):
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
        self.source = "nvidia-smi"

    def __enter__(self):
        mode = os.environ.get("AMGT_BENCH_CLOCKS", "smi")  # smi | nvml | off (testing only)
        if mode == "off":
            self.source = "off"
            return self
        if mode == "nvml":
            try:
                self._nvml()
                return self
            except Exception:
                self.stop = None
        try:
            self._smi()
        except Exception:
            self.proc = None
            self.source = "unavailable"
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.stop is not None:
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
        if not sm:  # unmeasured, not "no throttling"
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": None, "samples": 0, "source": self.source}
        busy = [s for s in sm if s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(busy), "sm_max_mhz": mx or None, "reasons": sorted(reasons),
                "samples": len(sm), "source": self.source}


# ------------------------------------------------------------------ byte model
S_BYTES = {"f64": 8, "f32": 4, "f16": 2}


def byte_model(sz, cycles):
    """Operation-count bytes of one step from structure sizes (identical for both arms): every
    SpMV operation of Alg. 2 counted with its own operand bytes (the paper's SpMV
    convention), whether or not a kernel serves two operations from one pass.
    sz: {"A_nnz", "P_nnz": [..], "P_m": [..], "lev": [{"m","BR","BC","T"}], "P_T", "R_T", "AP_T": [..],
         "prec": [..]}.  Tiles count 16 s + 4 + 2 bytes (values, blc_idx, blc_map)."""
    L = len(sz["lev"])
    s = [S_BYTES[p] for p in sz["prec"]]
    vs = [8 if p == "f64" else 4 for p in sz["prec"]]
    tb = lambda T, sk: T * (16 * sk + 6)
    lev = sz["lev"]
    out = {}
    c = sz["A_nnz"] * 12 + (lev[0]["m"] + 1) * 8 + tb(lev[0]["T"], 8) + (lev[0]["BR"] + 1) * 8
    for k in range(L - 1):
        c += sz["P_nnz"][k] * 12 + (sz["P_m"][k] + 1) * 8 + tb(sz["P_T"][k], 8) + (lev[k]["BR"] + 1) * 8
    out["csr2mbsr"] = c
    c = 0
    for k in range(L - 1):
        if s[k] != 8:
            c += 16 * sz["P_T"][k] * (8 + s[k])
        if s[k + 1] != s[k]:
            c += 16 * lev[k + 1]["T"] * (s[k] + s[k + 1])
    out["cast"] = c
    sym = num = 0
    for k in range(L - 1):
        TA, TP, TR, TAP, TC = lev[k]["T"], sz["P_T"][k], sz["R_T"][k], sz["AP_T"][k], lev[k + 1]["T"]
        sym += 2 * (TA + TP) * 6 + TAP * 6 + 2 * (TR + TAP) * 6 + TC * 6
        num += tb(TA, s[k]) + tb(TP, s[k]) + tb(TAP, s[k]) + tb(TR, s[k]) + tb(TAP, s[k]) + tb(TC, s[k])
        num += 2 * TP * (16 * s[k] + 6)  # R = P^T (tile transpose: read + write)
    out["spgemm_symbolic"], out["spgemm_numeric"] = sym, num
    out["mbsr2csr"] = tb(lev[-1]["T"], s[-1]) + lev[-1]["m"] * 20

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
        vec += 6 * 4 * lev[k]["BR"] * vs[k]
    vec += lev[-1]["m"] ** 2 * 8 + (3 if L > 1 else 2) * 4 * lev[0]["BR"] * 8
    out["spmv_l1"] = l1 * cycles + sp1
    out["spmv"] = other * cycles
    out["vector"] = vec * cycles
    return out


SETUP_KEYS = ("spgemm_symbolic", "spgemm_numeric", "csr2mbsr", "mbsr2csr", "cast")
SOLVE_KEYS = ("spmv_l1", "spmv", "vector")


def gpu_sizes(amgt, A, Ps, level_prec):
    """Structure sizes of the hierarchy built by the CUDA path (for the byte model)."""
    MA = amgt.from_csr(A)
    H = amgt.Hierarchy(MA, [amgt.from_csr(P) for P in Ps], level_prec=level_prec)
    sz = {"A_nnz": A.nnz, "P_nnz": [P.nnz for P in Ps], "P_m": [P.m for P in Ps], "lev": [], "P_T": [], "R_T": [],
          "AP_T": [], "prec": list(level_prec)}
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


def oracle_sizes(As, PRo, level_prec):
    import oracle
    sz = {"A_nnz": As[0].nnz, "P_nnz": [P.nnz for P, _ in PRo], "P_m": [P.m for P, _ in PRo], "lev": [], "P_T": [],
          "R_T": [], "AP_T": [], "prec": list(level_prec)}
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
    A = gen.configs.build_matrix(cfg, device=device)
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device=device)
    Ps = [P for P, _ in PR]
    b = gen.uniform_vector(A.m, cfg.seed).to(device)
    return A, Ps, b, PR


def gpu_step(amgt, A, Ps, b, x, ncycles, level_prec, after_setup=None):
    """The whole hot path once (inputs on the device).  after_setup: called once the
    hierarchy exists (the e2e leg enqueues the next step's upload there)."""
    MA = amgt.from_csr(A)                       # a1
    MPs = [amgt.from_csr(P) for P in Ps]        # a1 (P_k)
    H = amgt.Hierarchy(MA, MPs, level_prec=level_prec)  # a2-a8
    if after_setup is not None:
        after_setup()
    x.zero_()
    res, calls = H.vcycle(b, x, ncycles)        # a9-a10
    H.close()
    MA.free()
    for M in MPs:
        M.free()
    return res, calls


def _traffic(config: str):
    """ncu DRAM bytes per launch of the level-1 SpMV for this config (profiles/, one ncu --set full
    capture per config), or None."""
    p = os.path.join(ROOT, "profiles", f"ncu_traffic_{config}.json")
    if not os.path.exists(p):
        return None, None
    try:
        d = json.load(open(p))
        return d.get("spmv_l1", {}).get("dram_bytes_per_launch"), d
    except Exception:
        return None, None


def spgemm_cfg4(amgt, torch, peak, reps=5):
    """Config 4 (power-law block-sparse, 2^18 block rows): C = A*A through the public SpGEMM calls,
    L2 flushed before every repetition; GFLOP/s (2 x scalar products) and the byte roofline
    (A read twice + C written once)."""
    import gen
    cfg = gen.configs.CONFIGS["cfg4"]
    A = gen.configs.build_matrix(cfg, device="cuda")
    M = amgt.from_csr(A)
    del A
    C, info = amgt.spgemm_symbolic(M, M, info=True)
    amgt.spgemm_numeric(M, M, C)
    TC = C.blc_num
    C.free()
    flush = torch.empty(FLUSH_BYTES // 4, dtype=torch.float32, device="cuda")
    st = torch.cuda.current_stream()
    for _ in range(2):
        amgt.spgemm(M, M).free()
    sym_ms, num_ms = [], []
    for _ in range(reps):
        flush.fill_(1.0)
        e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        e0.record(st)
        C = amgt.spgemm_symbolic(M, M)
        e1.record(st)
        amgt.spgemm_numeric(M, M, C)
        e2.record(st)
        torch.cuda.synchronize()
        sym_ms.append(e0.elapsed_time(e1))
        num_ms.append(e1.elapsed_time(e2))
        C.free()
    tb = lambda T: T * (16 * 8 + 6)
    bytes_alg = 2 * tb(M.blc_num) + tb(TC) + 3 * (M.blc_row + 1) * 8
    flops = 2 * info["scalar_products"]
    ms = statistics.median([a + b for a, b in zip(sym_ms, num_ms)])
    gbs = bytes_alg / (ms * 1e-3) / 1e9
    out = {"workload": "cfg4: irregular power-law block-sparse 2^18 block rows, C = A*A FP64",
           "A_tiles": M.blc_num, "C_tiles": TC, "bins": info["bin_rows"], "pairs_nonzero": info["pairs_nonzero"],
           "flops": flops, "ms": round(ms, 4), "symbolic_ms": round(statistics.median(sym_ms), 4),
           "numeric_ms": round(statistics.median(num_ms), 4), "gflops": round(flops / (ms * 1e-3) / 1e9, 2),
           "roofline": {"bound": "hbm", "algorithmic_bytes": bytes_alg, "achieved": round(gbs, 1), "peak": peak,
                        "unit": "GB/s", "frac": round(gbs / peak, 4)},
           "l2": f"flushed before every repetition ({FLUSH_BYTES >> 20} MB write)", "reps": reps}
    _, tr = _traffic("cfg4")
    if tr and "spgemm" in tr:
        out["ncu"] = tr["spgemm"]
    M.free()
    del flush
    torch.cuda.empty_cache()
    return out


def _level_prec(cfg):
    return tuple(cfg.level_prec[:cfg.nlev])


def run_gpu(args):
    import torch

    import gen
    import paper_conf_sc_luzwflcy0c024_b200 as amgt

    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    cfg = gen.configs.CONFIGS[args.config]
    lp = _level_prec(cfg)
    A, Ps, b, PR = make_inputs(cfg, "cuda")
    npad = 4 * ((A.m + 3) // 4)
    x = torch.zeros(npad, dtype=torch.float64, device="cuda")
    stream = torch.cuda.current_stream()

    for _ in range(args.warmup):
        gpu_step(amgt, A, Ps, b, x, args.cycles, lp)
    # ---- one instrumented step (after warm-up): per-class device time and algorithmic bytes of
    # every kernel launched (the sub-cycle runs as direct launches so each is counted)
    amgt.timing_reset()
    amgt.timing_enable(True)
    res, calls = gpu_step(amgt, A, Ps, b, x, args.cycles, lp)
    torch.cuda.synchronize()
    prof = amgt.timing_read()
    amgt.timing_enable(False)
    bytes_phys = sum(v["bytes"] for v in prof.values())
    sz, flops = gpu_sizes(amgt, A, Ps, lp)
    bm = byte_model(sz, args.cycles)
    bytes_ops = sum(bm.values())
    l0 = sz["lev"][0]
    spmv_l1_bytes = l0["T"] * (16 * 8 + 6) + (l0["BR"] + 1) * 8 + 4 * l0["BC"] * 8 + 4 * l0["BR"] * 8
    torch.cuda.synchronize()

    # ---- timed region: K steps, live events around 1 in L1_SAMPLE level-1 SpMVs (dominant kernel)
    amgt.timing_reset()
    amgt.timing_enable(1)
    amgt.timing_sample(L1_SAMPLE)
    launches0 = amgt.launch_count()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gc.collect()
    gc.disable()  # no collector pause inside the timed region (host stalls starve the GPU queue)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        ev0.record(stream)
        host_ms = []
        for _ in range(args.steps):
            t_h = time.perf_counter()
            gpu_step(amgt, A, Ps, b, x, args.cycles, lp)
            host_ms.append(round((time.perf_counter() - t_h) * 1e3, 2))
        ev1.record(stream)
        torch.cuda.synchronize()
    gc.enable()
    print(f"[bench] host ms per timed step (enqueue + host syncs): {host_ms}", file=sys.stderr)
    launches = amgt.launch_count() - launches0
    live = amgt.timing_read()
    amgt.timing_enable(False)
    amgt.timing_sample(1)
    ms_step = ev0.elapsed_time(ev1) / args.steps
    peak, peak_kind = _peaks()
    value = bytes_phys / (ms_step * 1e-3) / 1e9

    spmv_l1 = live["spmv_l1"]
    n_l1 = max(spmv_l1["launches"], 1)
    spmv_avg_ms = spmv_l1["ms"] / n_l1
    l1_bytes_per_launch = spmv_l1["bytes"] / n_l1  # SpMV bytes + fused epilogue vectors, per launch
    achieved = l1_bytes_per_launch / (spmv_avg_ms * 1e-3) / 1e9
    traffic, _ = _traffic(args.config)
    setup_ms = sum(prof[k]["ms"] for k in SETUP_KEYS)
    spgemm_ms = prof["spgemm_symbolic"]["ms"] + prof["spgemm_numeric"]["ms"]
    spgemm_bytes = prof["spgemm_symbolic"]["bytes"] + prof["spgemm_numeric"]["bytes"]

    # ---- e2e: the same step through the public API with host (pinned) inputs and outputs
    hA = type(A)(A.m, A.n, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(), A.val.cpu().pin_memory())
    hPs = [type(P)(P.m, P.n, P.row_ptr.cpu().pin_memory(), P.col.cpu().pin_memory(), P.val.cpu().pin_memory())
           for P in Ps]
    hb = b.cpu().pin_memory()
    hx = torch.empty(x.numel(), dtype=torch.float64).pin_memory()
    h2d = sum(t.numel() * t.element_size() for M in [hA, *hPs] for t in (M.row_ptr, M.col, M.val)) + hb.numel() * 8
    d2h = hx.numel() * 8 + (args.cycles + 1) * 8
    host_in = [hA.row_ptr, hA.col, hA.val] + [t for P in hPs for t in (P.row_ptr, P.col, P.val)] + [hb]
    del A, Ps
    torch.cuda.empty_cache()
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

    upload(0)
    stream.wait_event(ev_in[0])
    dA, dPs, db = unpack(0)
    gpu_step(amgt, dA, dPs, db, x, args.cycles, lp)  # warm the allocator for this input pattern
    # Every step copies its own inputs (A, the P_k, b) from pinned host memory on a copy stream
    # into two buffer sets (step i+1's upload overlaps step i's V-cycles) and reads x back
    xs = [x, torch.empty_like(x)]
    ev_out = torch.cuda.Event()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    cs.wait_event(e0)
    upload(0)
    for i in range(args.steps):
        stream.wait_event(ev_in[i % 2])
        dA, dPs, db = unpack(i % 2)
        nxt = (lambda k=(i + 1) % 2: upload(k)) if i + 1 < args.steps else None
        gpu_step(amgt, dA, dPs, db, xs[i % 2], args.cycles, lp, after_setup=nxt)
        ev_out.record(stream)
        cs.wait_event(ev_out)
        with torch.cuda.stream(cs):
            hx.copy_(xs[i % 2], non_blocking=True)
    stream.wait_stream(cs)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1) / args.steps
    del dev_in, dA, dPs, db
    torch.cuda.empty_cache()

    components = {
        "setup_ms": round(setup_ms, 3), "solve_ms": round(ms_step - setup_ms, 3),
        "setup_solve_s": round(ms_step * 1e-3, 5),
        "spmv_l1_gbs": round(achieved, 1),
        "value_ops": round(bytes_ops / (ms_step * 1e-3) / 1e9, 2),
        "value_ops_note": "every SpMV operation of Alg. 2 with its own operand bytes (the fused level-1 "
                          "pre-smoothing sweep delivers the previous cycle's residual: 4 operations, 3 passes)",
        "bytes_per_step": bytes_phys, "bytes_ops_per_step": bytes_ops,
        "spgemm_gflops": round(flops / (spgemm_ms * 1e-3) / 1e9, 2) if spgemm_ms else None,
        "spgemm_roofline": {
            "bound": "hbm", "unit": "GB/s", "peak": peak,
            "achieved": round(spgemm_bytes / (spgemm_ms * 1e-3) / 1e9, 1) if spgemm_ms else None,
            "frac": round(spgemm_bytes / (spgemm_ms * 1e-3) / 1e9 / peak, 4) if spgemm_ms else None,
            "scope": "every SpGEMM call of the setup (symbolic + numeric, all levels; instrumented step)"},
        "rap_flops": flops,
        "bytes_by_class": {k: int(v["bytes"]) for k, v in prof.items()},
        "per_class_ms": {k: round(v["ms"], 3) for k, v in prof.items()},
        "final_rel_residual": res[-1] / res[0],
    }
    if not args.no_cfg4:
        components["spgemm_cfg4"] = spgemm_cfg4(amgt, torch, peak)
    line = {
        "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64/f32/f16 (per AMG level, L266)", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg.description}", "levels": cfg.nlev, "level_prec": list(lp),
                   "vcycles_per_step": args.cycles, "smoother": "weighted Jacobi w=2/3, nu1=nu2=1",
                   "parallelism": "single GPU",
                   "l2": "inputs larger than L2 (level-1 mBSR A = %.0f MB vs 126 MB L2); no flush" %
                         (l0["T"] * 134 / 1e6), "spmv_calls_per_step": calls},
        "roofline": {"kernel": "k_spmv_rows<double,double,double> (level-1 FP64 SpMV of A_1, fused Alg. 2 epilogues)",
                     "bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "peak_source": peak_kind,
                     "bytes_per_launch": round(l1_bytes_per_launch), "plain_spmv_bytes": spmv_l1_bytes,
                     "avg_launch_us": round(spmv_avg_ms * 1e3, 2), "launches_timed": spmv_l1["launches"],
                     "launch_sampling": f"1 in {L1_SAMPLE}", "traffic": traffic,
                     "traffic_source": f"profiles/ncu_traffic_{args.config}.json" if traffic else None},
        "components": components,
        "e2e": {"value": round(bytes_phys / (e2e_ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(e2e_ms, 3),
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "copies": "pinned host inputs uploaded every step on a copy stream, double-buffered "
                          "(step i+1's upload overlaps step i's V-cycles); x (double-buffered, read back on the "
                          "copy stream) and the residual norms read back every step"},
        "gpu_launches": launches,
        "clocks": clk.summary(),
    }
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(args, hA, hPs, hb)
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ N > 1: config 5 strong-scaled
def run_dist(args, rank, world, local):
    """The row-slab partitioned path: config 5 (7-point 512^3, 7 levels) split into
    `world` z-slabs, one rank per GPU over NCCL; levels with <= 32^3 rows agglomerated."""
    import torch
    import torch.distributed as dist

    import gen
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    from paper_conf_sc_luzwflcy0c024_b200.dist import DistComm, DistHierarchy

    sys.stdout.flush()
    json_fd = os.dup(1)
    os.dup2(2, 1)  # library banners (NCCL) to stderr; stdout carries the one JSON line
    torch.cuda.set_device(local)
    dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    cfg = gen.configs.CONFIGS[args.config]
    lp = _level_prec(cfg)
    dims = gen.configs.grid_dims(cfg)
    A, rows, n, Ps = gen.partition.slab_inputs(cfg.kind, dims, cfg.nlev, rank, world, alpha=cfg.alpha, device="cuda")
    m = rows[1] - rows[0]
    b = gen.uniform_vector(n, cfg.seed)[rows[0]:rows[1]].cuda()
    x = torch.zeros(m, dtype=torch.float64, device="cuda")
    comm = DistComm.nccl(rank, world, rows)
    stream = torch.cuda.current_stream()

    def step(xv=x, A_=A, Ps_=Ps, b_=b, after_setup=None):
        MA = amgt.from_csr(A_)
        MPs = [amgt.from_csr(P) for P in Ps_]
        H = DistHierarchy(comm, MA, MPs, level_prec=lp, agg_rows=AGG_ROWS)
        if after_setup is not None:
            after_setup()
        xv.zero_()
        res, calls = H.vcycle(b_, xv, args.cycles)
        info = H.info()
        H.close()
        MA.free()
        for M in MPs:
            M.free()
        return res, calls, info

    for _ in range(args.warmup):
        step()
    amgt.timing_reset()
    amgt.timing_enable(True)
    res, calls, info = step()
    torch.cuda.synchronize()
    prof = amgt.timing_read()
    amgt.timing_enable(False)
    by = torch.tensor([sum(v["bytes"] for v in prof.values())], dtype=torch.float64, device="cuda")
    dist.all_reduce(by)  # whole-job bytes
    bytes_job = float(by.item())
    setup_ms = sum(prof[k]["ms"] for k in SETUP_KEYS)

    dist.barrier()
    torch.cuda.synchronize()
    launches0 = amgt.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gc.collect()
    gc.disable()
    host_ms = []
    with ClockSampler(local) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            t_h = time.perf_counter()
            step()
            host_ms.append(round((time.perf_counter() - t_h) * 1e3, 2))
        e1.record(stream)
        dist.barrier()
        torch.cuda.synchronize()
    gc.enable()
    print(f"[bench] rank {rank} host ms per timed step (enqueue + host syncs): {host_ms}", file=sys.stderr)
    t = torch.tensor([e0.elapsed_time(e1) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_step = float(t.item())
    launches = amgt.launch_count() - launches0
    # distributed level-1 SpMV (halo exchange overlapped with the interior rows), events
    MA = amgt.from_csr(A)
    y = torch.empty(m, dtype=torch.float64, device="cuda")
    comm.spmv(MA, b, y)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(20)]
    dist.barrier()
    for a_, b_ in ev:
        a_.record(stream)
        comm.spmv(MA, b, y)
        b_.record(stream)
    torch.cuda.synchronize()
    spmv_ms = statistics.median(a_.elapsed_time(b_) for a_, b_ in ev)
    sp_bytes = MA.blc_num * (16 * 8 + 6) + (MA.blc_row + 1) * 8 + 8 * 4 * MA.blc_row * 2
    MA.free()
    peak, peak_kind = _peaks()
    achieved = sp_bytes / (spmv_ms * 1e-3) / 1e9
    ach = torch.tensor([achieved], dtype=torch.float64, device="cuda")
    dist.all_reduce(ach, op=dist.ReduceOp.MIN)
    # e2e: every rank uploads its slab inputs from pinned host memory each step, x read back
    CSR = type(A)
    hA = CSR(A.m, A.n, A.row_ptr.cpu().pin_memory(), A.col.cpu().pin_memory(), A.val.cpu().pin_memory())
    hPs = [CSR(P.m, P.n, P.row_ptr.cpu().pin_memory(), P.col.cpu().pin_memory(), P.val.cpu().pin_memory()) for P in Ps]
    hb = b.cpu().pin_memory()
    hx = torch.empty(x.numel(), dtype=torch.float64).pin_memory()
    h2d = sum(t_.numel() * t_.element_size() for M in [hA, *hPs] for t_ in (M.row_ptr, M.col, M.val)) + hb.numel() * 8
    d2h = hx.numel() * 8 + (args.cycles + 1) * 8
    host_in = [hA.row_ptr, hA.col, hA.val] + [t_ for P in hPs for t_ in (P.row_ptr, P.col, P.val)] + [hb]
    dev_in = [[torch.empty(t_.shape, dtype=t_.dtype, device="cuda") for t_ in host_in] for _ in range(2)]
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
        step(x, dA, dPs, d[-1], after_setup=(lambda: upload(nxt)) if nxt is not None else None)
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
    te = torch.tensor([f0.elapsed_time(f1) / args.steps], dtype=torch.float64, device="cuda")
    dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_ms = float(te.item())
    sys.stdout.flush()
    os.dup2(json_fd, 1)
    os.close(json_fd)
    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": round(bytes_job / (ms_step * 1e-3) / 1e9, 2), "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f64/f32/f16 (per AMG level, L266)", "data": "synthetic",
            "config": {"workload": f"{args.config}: {cfg.description}, strong-scaled over {world} ranks (z-slabs)",
                       "levels": cfg.nlev, "level_prec": list(lp), "vcycles_per_step": args.cycles,
                       "parallelism": f"row-slab x{world} (NCCL halo exchange overlapped with interior rows; levels "
                                      f"<= {AGG_ROWS} rows agglomerated on every rank)",
                       "agg_level": info["agg_level"], "l2": "inputs larger than L2; no flush",
                       "spmv_calls_per_step": calls},
            "roofline": {"kernel": "amgt_dist_spmv level-1 FP64 (halo exchange + k_spmv_rows interior/boundary), "
                                   "slowest rank", "bound": "hbm", "achieved": round(float(ach.item()), 1),
                         "peak": peak, "unit": "GB/s", "frac": round(float(ach.item()) / peak, 4),
                         "peak_source": peak_kind, "bytes_per_launch": sp_bytes,
                         "avg_launch_us": round(spmv_ms * 1e3, 2), "traffic": None},
            "components": {"setup_ms_rank0": round(setup_ms, 3), "bytes_per_step": bytes_job,
                           "final_rel_residual": res[-1] / res[0], "host_ms_per_step_rank0": host_ms},
            "e2e": {"value": round(bytes_job / (e2e_ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(e2e_ms, 3),
                    "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world,
                    "copies": "each rank uploads its slab inputs from pinned host memory every step (copy stream, "
                              "double-buffered, overlapping the previous step's V-cycles) and reads x back"},
            "gpu_launches": launches, "clocks": clk.summary(),
        }), flush=True)
    comm.close()
    dist.destroy_process_group()


# ------------------------------------------------------------------ oracle (CPU) legs
SLAB_FRACTION = 16  # the setup sample: the level-1 conversion + RAP of 1/16 of the fine grid


class OracleSample:
    """The oracle's version of a step on a bounded sample of the same workload (hierarchy built
    once at construction): (a) setup — CSR->mBSR of A_1's rows and the level-1 RAP (A P, then
    R (A P)) restricted to one z-slab of 1/SLAB_FRACTION of the grid; (b) solve — `cycles` full
    V-cycles on the whole hierarchy.  Its bytes: that fraction of the setup's and cycles/50 of the
    solve's byte model."""

    def __init__(self, config, A, PR, b):
        import gen
        import oracle
        self.cfg = gen.configs.CONFIGS[config]
        self.lp = _level_prec(self.cfg)
        self.Ao = oracle.as_csr(A)
        self.PRo = [(oracle.as_csr(P), oracle.as_csr(R)) for P, R in PR]
        self.As = oracle.build_hierarchy(self.Ao, self.PRo)
        self.b = b
        dims = gen.configs.grid_dims(self.cfg)
        plane = dims[0] * dims[1]
        nz = dims[-1] // SLAB_FRACTION
        r0, r1 = 0, nz * plane
        self.A_slab = gen.stencil(dims, *gen.partition.STENCILS[self.cfg.kind], -1.0, rows=(r0, r1)) \
            if self.cfg.kind in gen.partition.STENCILS else None
        P, R = self.PRo[0]
        self.P = P
        c1 = (nz // 2) * (plane // 4)
        # the slab's aggregates reach only the slab's fine rows: columns index AP's rows
        self.R_slab = oracle.Csr(c1, r1 - r0, R.row_ptr[:c1 + 1].copy(), R.col[:R.row_ptr[c1]].copy(),
                                 R.val[:R.row_ptr[c1]].copy())
        assert self.R_slab.col.size == 0 or int(self.R_slab.col.max()) < r1 - r0

    def run(self, cycles):
        import oracle
        t0 = time.perf_counter()
        As = oracle.as_csr(self.A_slab)
        oracle.csr_to_mbsr(As)                   # a1 on the slab's rows
        AP = oracle.spgemm(As, self.P)           # a7: A P restricted to the slab
        oracle.spgemm(self.R_slab, AP)           # a7: R (A P) of the slab's aggregates
        t1 = time.perf_counter()
        oracle.vcycle(self.As, self.PRo, self.b, ncycles=cycles)  # a9-a10
        t2 = time.perf_counter()
        return t1 - t0, t2 - t1

    def sample_bytes(self, bm, cycles, total_cycles):
        return sum(bm[k] for k in SETUP_KEYS) / SLAB_FRACTION + sum(bm[k] for k in SOLVE_KEYS) * cycles / total_cycles

    def describe(self, cycles, total_cycles):
        return (f"{self.cfg.key}: level-1 CSR->mBSR + RAP of 1/{SLAB_FRACTION} of the grid (one z-slab) + {cycles} of "
                f"{total_cycles} V-cycles on the full hierarchy (FP64 C oracle, OpenMP rows); bytes = the same fractions "
                "of the step's byte model")


def cpu_baseline(args, hA, hPs, hb):
    import gen
    import oracle
    cfg = gen.configs.CONFIGS[args.config]
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha)
    S = OracleSample(args.config, hA, PR, hb.numpy())
    bm = byte_model(oracle_sizes(S.As, S.PRo, S.lp), args.cycles)
    ts, tv = S.run(args.cpu_cycles)
    by = S.sample_bytes(bm, args.cpu_cycles, args.cycles)
    return {"value": round(by / (ts + tv) / 1e9, 4), "unit": "GB/s", "cores": oracle.max_threads(), "kind": "oracle",
            "sample": S.describe(args.cpu_cycles, args.cycles) + f"; setup {ts:.2f}s, solve {tv:.2f}s",
            "note": "operation-count bytes (value_ops convention)"}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import gen
    import oracle
    cfg = gen.configs.CONFIGS[args.config]
    A, Ps, b, PR = make_inputs(cfg, "cpu")
    S = OracleSample(args.config, A, PR, b.numpy())
    bm = byte_model(oracle_sizes(S.As, S.PRo, S.lp), args.cycles)
    cycles = args.cpu_cycles
    for _ in range(args.warmup):
        S.run(cycles)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        S.run(cycles)
    dt = (time.perf_counter() - t0) / args.steps
    val = S.sample_bytes(bm, cycles, args.cycles) / dt / 1e9
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(val, 4), "unit": "GB/s", "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 2), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg.description}", "levels": cfg.nlev},
        "cpu_baseline": {"value": round(val, 4), "unit": "GB/s", "cores": oracle.max_threads(), "kind": "oracle",
                         "sample": S.describe(cycles, args.cycles)},
        "e2e": {"value": round(val, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="amgt", choices=["amgt", "reference"])
    ap.add_argument("--config", default=None, choices=["cfg2", "cfg3", "cfg5"],
                    help="default: cfg3 at N = 1, cfg5 (strong scaling) at N > 1")
    ap.add_argument("--cycles", type=int, default=50, help="V-cycles per step (paper: 50, L308)")
    ap.add_argument("--cpu-cycles", type=int, default=1, help="V-cycles in the oracle's bounded sample")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cfg4", action="store_true", help="skip the config-4 SpGEMM component")
    ap.add_argument("--force-dist", action="store_true", help="the partitioned (NCCL) path even at N = 1 (testing)")
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.config is None:
        args.config = "cfg5" if world > 1 else "cfg3"
    if args.impl == "reference":
        run_reference(args)
        return
    args.warmup = max(args.warmup, 3)
    if world > 1 or args.force_dist:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if "MASTER_PORT" not in os.environ:
            import socket
            with socket.socket() as so:
                so.bind(("127.0.0.1", 0))
                os.environ["MASTER_PORT"] = str(so.getsockname()[1])
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
        return run_dist(args, int(os.environ["RANK"]), world, int(os.environ.get("LOCAL_RANK", "0")))
    run_gpu(args)


if __name__ == "__main__":
    main()
