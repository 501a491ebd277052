"""Per-call timeline of the AMG hierarchy (§8(f) NEXT-4; the paper's Fig. 8 / Fig. 10 analogs,
L337-339, L353-357, L367-381): every SpGEMM (symbolic, numeric) of the setup and every SpMV of
one V-cycle, level by level, timed with CUDA events through the public C ABI, plus CSR->mBSR
against cuSPARSE csr2bsr (block size 4) on the level-1 operator as an optional comparator.

Measurement only: it rebuilds the hierarchy step by step through the same entry points that
amgt_hierarchy_create uses (cast, transpose, spgemm_symbolic/numeric, spmv_fused), so the
times are those of the library calls; nothing here is on the product path.

usage: python tools/timeline.py [cfg2|cfg3] [--interp sa] [--out profiles/r01_timeline_cfg2.json]
"""
import argparse
import ctypes
import glob
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_sc_luzwflcy0c024_b200 as amgt  # noqa: E402

S = {"f64": 8, "f32": 4, "f16": 2}


def timed(fn, reps=3):
    """Median over reps of a CUDA-event-timed call (ms); returns (ms, last result)."""
    st = torch.cuda.current_stream()
    ts, out = [], None
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(st)
        out = fn()
        e1.record(st)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2], out


def tile_bytes(M, s):
    return M.blc_num * (16 * s + 6) + (M.blc_row + 1) * 8


def cusparse_csr2bsr(A, reps=5):
    """cuSPARSE csr2bsr (legacy API, int32 indices, block 4) time in ms, or None."""
    cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cusparse", "lib", "libcusparse.so*"))
    cands += ["libcusparse.so.12", "libcusparse.so"]
    lib = None
    for c in cands:
        try:
            lib = ctypes.CDLL(c)
            break
        except OSError:
            continue
    if lib is None or A.nnz >= 2 ** 31:
        return None
    h, da, dc = ctypes.c_void_p(), ctypes.c_void_p(), ctypes.c_void_p()
    if lib.cusparseCreate(ctypes.byref(h)) != 0:
        return None
    lib.cusparseSetStream(h, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    lib.cusparseCreateMatDescr(ctypes.byref(da))
    lib.cusparseCreateMatDescr(ctypes.byref(dc))
    m, n, bd = A.m, A.n, 4
    mb, nb = (m + 3) // 4, (n + 3) // 4
    rp = A.row_ptr.to(torch.int32).contiguous()
    ci = A.col.to(torch.int32).contiguous()
    val = A.val.contiguous()
    brp = torch.empty(mb + 1, dtype=torch.int32, device="cuda")
    nnzb = ctypes.c_int(0)

    def run():
        lib.cusparseXcsr2bsrNnz(h, 0, m, n, da, ctypes.c_void_p(rp.data_ptr()), ctypes.c_void_p(ci.data_ptr()), bd, dc,
                                ctypes.c_void_p(brp.data_ptr()), ctypes.byref(nnzb))
        bci = torch.empty(max(nnzb.value, 1), dtype=torch.int32, device="cuda")
        bval = torch.empty(max(nnzb.value, 1) * 16, dtype=torch.float64, device="cuda")
        lib.cusparseDcsr2bsr(h, 0, m, n, da, ctypes.c_void_p(val.data_ptr()), ctypes.c_void_p(rp.data_ptr()),
                             ctypes.c_void_p(ci.data_ptr()), bd, dc, ctypes.c_void_p(bval.data_ptr()),
                             ctypes.c_void_p(brp.data_ptr()), ctypes.c_void_p(bci.data_ptr()))
        return nnzb.value

    run()
    ms, blocks = timed(run, reps)
    lib.cusparseDestroy(h)
    return {"ms": round(ms, 4), "blocks": blocks}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="cfg2")
    ap.add_argument("--interp", default="given", choices=["given", "sa"])
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    cfg = gen.configs.CONFIGS[args.config]
    prec = list(cfg.level_prec[:cfg.nlev])
    A = gen.configs.build_matrix(cfg, device="cuda")
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
    out = {"config": args.config, "interp": args.interp, "level_prec": prec, "setup": [], "solve": []}

    timed(lambda: amgt.from_csr(A), 2)
    ms, MA = timed(lambda: amgt.from_csr(A), 3)
    out["csr2mbsr_l1"] = {"ms": round(ms, 4), "tiles": MA.blc_num,
                          "GBps": round((A.nnz * 12 + (A.m + 1) * 8 + tile_bytes(MA, 8)) / (ms * 1e-3) / 1e9, 1),
                          "cusparse_csr2bsr": cusparse_csr2bsr(A)}

    for warm in (True, False):  # first pass loads every kernel (lazy module loading) and warms the allocator
        levels, ops = setup(args, MA, PR, prec, out, warm)
    solve(levels, ops, prec, out)
    line = json.dumps(out)
    print(line)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(out, f, indent=1)


def setup(args, MA, PR, prec, out, warm):
    """Alg. 1 level by level: [SA interpolation], R = P^T, AP, R(AP), cast; records into out."""
    out["setup"] = []
    Ak = MA if prec[0] == "f64" else MA.cast(prec[0])
    levels = [Ak]
    ops = []
    for k, (P, _) in enumerate(PR):
        MP = amgt.from_csr(P)
        if prec[k] != "f64":
            MP = MP.cast(prec[k])
        rec = {"level": k + 1, "prec": prec[k], "A_tiles": Ak.blc_num}
        if args.interp == "sa":
            ms, MP = timed(lambda: amgt.sa_interp(Ak, MP), 3)
            rec["sa_interp_ms"] = round(ms, 4)
        ms, MR = timed(lambda: MP.transpose(), 3)
        rec["transpose_ms"] = round(ms, 4)
        for name, X, Y in (("AP", Ak, MP), ("RAP", MR, None)):
            if name == "RAP":
                X, Y = MR, AP
            ms_s, (C, info) = timed(lambda: amgt.spgemm_symbolic(X, Y, info=True), 3)
            ms_n, _ = timed(lambda: amgt.spgemm_numeric(X, Y, C), 3)
            flops = 2 * info["scalar_products"]
            s = S[prec[k]]
            byts = tile_bytes(X, s) + tile_bytes(Y, s) + tile_bytes(C, s)
            rec[name] = {"symbolic_ms": round(ms_s, 4), "numeric_ms": round(ms_n, 4), "C_tiles": C.blc_num,
                         "flops": flops, "GFLOPs": round(flops / ((ms_s + ms_n) * 1e-3) / 1e9, 2),
                         "numeric_GBps": round(byts / (ms_n * 1e-3) / 1e9, 1), "bins": info["bin_rows"]}
            if name == "AP":
                AP = C
            else:
                Ac = C
        if k + 1 < len(prec) and prec[k + 1] != prec[k]:
            ms, Ac = timed(lambda: Ac.cast(prec[k + 1]), 3)
            rec["cast_ms"] = round(ms, 4)
        out["setup"].append(rec)
        ops.append((Ak, MP, MR))
        Ak = Ac
        levels.append(Ak)

    return levels, ops


def solve(levels, ops, prec, out):
    """Every SpMV kind of one V-cycle per level (A_k Jacobi, R_k, P_k)."""
    for k, Ak in enumerate(levels):
        Ak.analyze()  # the SpMV plan the hierarchy builds for every A_k, P_k, R_k
        if k < len(ops):
            ops[k][1].analyze()
            ops[k][2].analyze()
        vd = torch.float64 if prec[k] == "f64" else torch.float32
        n = 4 * Ak.blc_row
        x = torch.rand(4 * Ak.blc_col, dtype=vd, device="cuda")
        y = torch.empty(n, dtype=vd, device="cuda")
        b = torch.rand(n, dtype=vd, device="cuda")
        d = torch.full((n,), 0.1, dtype=vd, device="cuda")
        s, sv = S[prec[k]], (8 if vd == torch.float64 else 4)
        byts = tile_bytes(Ak, s) + 4 * Ak.blc_col * sv + 4 * Ak.blc_row * sv
        ms, _ = timed(lambda: amgt.spmv_fused(Ak, x, y, "jacobi", b=b, dinv=d), 5)
        rec = {"level": k + 1, "prec": prec[k], "tiles": Ak.blc_num, "A_jacobi_us": round(ms * 1e3, 2),
               "A_GBps": round((byts + 2 * n * sv) / (ms * 1e-3) / 1e9, 1)}
        if k < len(ops):
            _, MP, MR = ops[k]
            vdn = torch.float64 if prec[k + 1] == "f64" else torch.float32
            bn = torch.empty(4 * MR.blc_row, dtype=vdn, device="cuda")
            ms, _ = timed(lambda: amgt.spmv_fused(MR, y, bn, "y"), 5)
            rec["R_us"] = round(ms * 1e3, 2)
            xc = torch.rand(4 * MP.blc_col, dtype=vdn, device="cuda")
            ms, _ = timed(lambda: amgt.spmv_fused(MP, xc, y, "accum"), 5)
            rec["P_us"] = round(ms * 1e3, 2)
        out["solve"].append(rec)


if __name__ == "__main__":
    main()
