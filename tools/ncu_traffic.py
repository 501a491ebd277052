"""ncu DRAM traffic of the bench's dominant kernels, per config (bench.py reads
profiles/ncu_traffic_<cfg>.json for the roofline `traffic` field).

  python tools/ncu_traffic.py run cfg3        # workload to run UNDER ncu (see below)
  python tools/ncu_traffic.py summarize cfg3 report.ncu-rep   # -> profiles/ncu_traffic_cfg3.json

cfg2 / cfg3 / cfg5: hierarchy setup, then one V-cycle; capture the level-1 FP64 SpMV launches
  ncu --set full --clock-control none -k regex:'k_spmv_rows<double' -c 4 -o rep python tools/ncu_traffic.py run cfg3
cfg4: one C = A*A SpGEMM after a warm-up; capture every launch of the second call
  ncu --set full --clock-control none --nvtx --nvtx-include 'amgt_spgemm/' -o rep python tools/ncu_traffic.py run cfg4
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(cfg_name):
    import torch
    import gen
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    cfg = gen.configs.CONFIGS[cfg_name]
    side = os.path.join(ROOT, "gpurun_out", f"ncu_traffic_{cfg_name}_sizes.json")
    os.makedirs(os.path.dirname(side), exist_ok=True)
    if cfg.kind == "irregular":
        A = gen.configs.build_matrix(cfg, device="cuda")
        M = amgt.from_csr(A)
        C, info = amgt.spgemm(M, M, info=True)
        TC = C.blc_num
        C.free()
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_push("amgt_spgemm")
        C = amgt.spgemm(M, M)
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_pop()
        json.dump({"A_tiles": M.blc_num, "C_tiles": TC, "BR": M.blc_row, "scalar_products": info["scalar_products"]},
                  open(side, "w"))
        return
    A = gen.configs.build_matrix(cfg, device="cuda")
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha, device="cuda")
    MA = amgt.from_csr(A)
    del A
    H = amgt.Hierarchy(MA, [amgt.from_csr(P) for P, _ in PR], level_prec=cfg.level_prec[:cfg.nlev])
    b = gen.uniform_vector(MA.m, cfg.seed).cuda()
    x = torch.zeros(4 * MA.blc_row, dtype=torch.float64, device="cuda")
    json.dump({"T": MA.blc_num, "BR": MA.blc_row, "BC": MA.blc_col}, open(side, "w"))
    torch.cuda.synchronize()
    H.vcycle(b, x, 1)
    torch.cuda.synchronize()


def _raw(rep, metrics):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(metrics)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        res.append(d)
    return res, dict(zip(h, units))


def _num(v, unit):
    v = float(str(v).replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
             "msecond": 1e-3, "second": 1, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1}[unit]
    return v * scale


def summarize(cfg_name, rep):
    side = json.load(open(os.path.join(ROOT, "gpurun_out", f"ncu_traffic_{cfg_name}_sizes.json")))
    mets = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"]
    rows, units = _raw(rep, mets)
    launches = []
    for d in rows:
        rd = _num(d["dram__bytes_read.sum"], units["dram__bytes_read.sum"])
        wr = _num(d["dram__bytes_write.sum"], units["dram__bytes_write.sum"])
        t = _num(d["gpu__time_duration.sum"], units["gpu__time_duration.sum"])
        launches.append({"kernel": d.get("Kernel Name", "")[:160], "dram_read": rd, "dram_write": wr,
                         "dram_bytes": rd + wr, "us": t * 1e6})
    out = {"config": cfg_name, "report": os.path.basename(rep),
           "capture": "ncu --set full --clock-control none (cold caches, serialised)", "launches": launches}
    if "A_tiles" in side:  # config 4 SpGEMM
        tb = lambda T: T * (16 * 8 + 6)
        alg = 2 * tb(side["A_tiles"]) + tb(side["C_tiles"]) + 3 * (side["BR"] + 1) * 8
        tot = sum(l["dram_bytes"] for l in launches)
        out["spgemm"] = {"dram_bytes": tot, "algorithmic_bytes": alg, "ratio": round(tot / alg, 3),
                         "kernel_us": round(sum(l["us"] for l in launches), 1), "launches": len(launches)}
    else:
        T, BR, BC = side["T"], side["BR"], side["BC"]
        plain = T * (16 * 8 + 6) + (BR + 1) * 8 + 4 * BC * 8 + 4 * BR * 8
        n = max(len(launches), 1)
        out["spmv_l1"] = {"dram_bytes_per_launch": sum(l["dram_bytes"] for l in launches) / n,
                          "plain_spmv_bytes": plain, "us_per_launch": sum(l["us"] for l in launches) / n,
                          "launches": len(launches)}
    dst = os.path.join(ROOT, "profiles", f"ncu_traffic_{cfg_name}.json")
    json.dump(out, open(dst, "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k != "launches"}, indent=1))


if __name__ == "__main__":
    if sys.argv[1] == "run":
        run(sys.argv[2])
    else:
        summarize(sys.argv[2], sys.argv[3])
