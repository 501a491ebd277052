"""Per-kernel summary of an ncu --csv launch list (gpu__time_duration / dram bytes):
python tools/ncu_sum_launches.py launches.csv [--per-launch]"""
import collections
import csv
import sys

SCALE = {"ns": 1e-3, "us": 1.0, "ms": 1e3, "s": 1e6, "nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3,
         "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main():
    rows = [r for r in csv.reader(open(sys.argv[1])) if r and not r[0].startswith("==")]
    h = rows[0]
    iK, iM, iU, iV = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
    iID = h.index("ID")
    per = collections.OrderedDict()
    for r in rows[1:]:
        d = per.setdefault(r[iID], {"k": r[iK]})
        d[r[iM]] = float(r[iV].replace(",", "")) * SCALE.get(r[iU], 1.0)
    agg = collections.OrderedDict()
    tot = 0.0
    for i, d in per.items():
        us = d.get("gpu__time_duration.sum", 0.0)
        by = d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
        tot += us
        if "--per-launch" in sys.argv:
            print(f"{i:>5} {us:9.1f} us {by / 1e6:9.1f} MB {by / max(us, 1e-9) / 1e3:7.0f} GB/s  {d['k'][:110]}")
        a = agg.setdefault(d["k"][:110], [0, 0.0, 0.0])
        a[0] += 1
        a[1] += us
        a[2] += by
    print(f"# {len(per)} launches, {tot:.1f} us total")
    for k, (n, us, by) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{n:5d} x {us / n:9.1f} us = {us:9.1f} us ({100 * us / tot:5.1f}%) {by / max(us, 1e-9) / 1e3:7.0f} GB/s  {k}")


if __name__ == "__main__":
    main()
