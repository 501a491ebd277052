"""Key metrics of an ncu --set full report, one block per captured kernel (for profiles/).

usage: python tools/ncu_brief.py report.ncu-rep [more.ncu-rep ...]
"""
import csv
import io
import subprocess
import sys

KEYS = ("Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Cache Throughput", "L2 Cache Throughput",
        "L1/TEX Hit Rate", "L2 Hit Rate", "Registers Per Thread", "Theoretical Active Warps per SM",
        "Achieved Active Warps Per SM", "Eligible Warps Per Scheduler", "Issued Warp Per Scheduler",
        "Warp Cycles Per Issued Instruction", "Grid Size", "Block Size", "Dynamic Shared Memory Per Block")


def main():
    for rep in sys.argv[1:]:
        out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        h = rows[0]
        seen = {}
        for r in rows[1:]:
            d = dict(zip(h, r))
            k = (d["ID"], d["Kernel Name"])
            if d["Metric Name"] in KEYS:
                seen.setdefault(k, []).append(f'{d["Metric Name"]} = {d["Metric Value"]} {d["Metric Unit"]}'.rstrip())
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                              "dram__bytes_read.sum,dram__bytes_write.sum"], capture_output=True, text=True).stdout
        rr = list(csv.reader(io.StringIO(raw)))
        by = {}
        if len(rr) > 2:
            hh = rr[0]
            for r in rr[2:]:
                d = dict(zip(hh, r))
                by[d.get("ID")] = (d.get("dram__bytes_read.sum"), d.get("dram__bytes_write.sum"), rr[1][hh.index("dram__bytes_read.sum")])
        print(f"# {rep}")
        for (i, name), items in seen.items():
            print(f"[{i}] {name[:150]}")
            for it in items:
                print("    " + it)
            if i in by:
                print(f"    dram bytes read = {by[i][0]} {by[i][2]}, write = {by[i][1]} {by[i][2]}")
        print()


if __name__ == "__main__":
    main()
