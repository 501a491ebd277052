"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): total time per kernel.

usage: python tools/ncu_sum.py launches.csv [--last-frac F] [--top N]
  --last-frac F  only the last fraction F of launches (e.g. 0.5 = the second of two identical runs)
"""
import argparse
import collections
import csv
import io


def load(path):
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    rows = list(csv.DictReader(io.StringIO("".join(lines))))
    out = []
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "ns")
        us = v / 1e3 if unit == "ns" else v * 1e3 if unit == "msecond" else v if unit == "usecond" else v / 1e3
        name = r["Kernel Name"]
        out.append((int(r["ID"]), name, us, r.get("Grid Size", ""), r.get("Block Size", "")))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--last-frac", type=float, default=1.0)
    ap.add_argument("--top", type=int, default=25)
    a = ap.parse_args()
    L = load(a.csv)
    L = L[int(len(L) * (1 - a.last_frac)):]
    agg = collections.OrderedDict()
    for _, name, us, g, b in L:
        key = name[:110]
        t, n = agg.get(key, (0.0, 0))
        agg[key] = (t + us, n + 1)
    tot = sum(t for t, _ in agg.values())
    print(f"launches {len(L)}  total {tot:.1f} us")
    for k, (t, n) in sorted(agg.items(), key=lambda kv: -kv[1][0])[: a.top]:
        print(f"{t:10.1f} us {100 * t / tot:5.1f}%  x{n:<5d} {k}")


if __name__ == "__main__":
    main()
