"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV): per-kernel totals and shares.
python tools/launch_summary.py launches.csv [skip_name_regex]"""
import csv
import re
import sys
from collections import defaultdict

UNIT = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}


def main(path, skip=None):
    rows = list(csv.reader(open(path)))
    hdr = None
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr is None or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"]
        if skip and re.search(skip, name):
            continue
        ms = float(d["Metric Value"].replace(",", "")) * UNIT.get(d["Metric Unit"], 1.0)
        short = re.sub(r"\(.*", "", name)[:70]
        agg[short][0] += 1
        agg[short][1] += ms
    tot = sum(v[1] for v in agg.values()) or 1
    print(f"{'ms total':>10} {'launches':>8} {'share':>6}  kernel")
    for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{t:10.3f} {c:8d} {100 * t / tot:5.1f}%  {n}")
    print(f"{tot:10.3f} total")


if __name__ == "__main__":
    main(*sys.argv[1:])
