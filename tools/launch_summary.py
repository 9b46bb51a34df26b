#!/usr/bin/env python
"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into per-launch and
per-kernel tables (ms and share of the step).

usage: python tools/launch_summary.py gpurun_out/launches.csv "<header line>" > profiles/rNN_ncu_launches.txt
"""
import csv
import sys
from collections import OrderedDict


def main():
    path = sys.argv[1]
    header = sys.argv[2] if len(sys.argv) > 2 else path
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    launches = []
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "ns")
        ms = v / 1e6 if unit == "ns" else (v / 1e3 if unit in ("us", "usecond") else v)
        name = r["Kernel Name"].split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "")
        name = name.replace("<unnamed>::", "").replace("unnamed>::", "").replace("gpa::", "")
        launches.append((name, ms))
    total = sum(ms for _, ms in launches)
    print(f"# {header}")
    print(f"# {len(launches)} launches, {total:.3f} ms of kernel time (cold-cache, serialised: compare shares)")
    agg = OrderedDict()
    for n, ms in launches:
        a = agg.setdefault(n, [0, 0.0])
        a[0] += 1
        a[1] += ms
    print("\n## per kernel")
    print(f"{'kernel':60s} {'launches':>8s} {'ms':>9s} {'share':>7s}")
    for n, (c, ms) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{n[:60]:60s} {c:8d} {ms:9.3f} {100 * ms / total:6.1f}%")
    print("\n## per launch (in order)")
    for n, ms in launches:
        print(f"{n[:60]:60s} {ms:9.3f} {100 * ms / total:6.1f}%")


if __name__ == "__main__":
    main()
