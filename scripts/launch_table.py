#!/usr/bin/env python
"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: per kernel (short
name) launches and total / mean us, in launch order of first appearance; --seq prints every
launch in order."""
import csv
import re
import sys
from collections import OrderedDict


def short(name):
    name = re.sub(r"\(.*", "", name)
    name = name.replace("void ", "").replace("inl::", "").replace("<unnamed>::", "")
    return name[:60]


def rows(path):
    hdr = None
    for r in csv.reader(open(path)):
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name", "gpu__time_duration.sum") == "gpu__time_duration.sum":
                v = float(d["Metric Value"].replace(",", ""))
                unit = d.get("Metric Unit", "nsecond")
                us = v / 1000 if unit.startswith("ns") or unit == "nsecond" else v if unit.startswith("us") else v * 1000
                yield short(d["Kernel Name"]), us


def main():
    path = sys.argv[1]
    if "--seq" in sys.argv:
        for k, us in rows(path):
            print(f"{us:10.1f} us  {k}")
        return
    agg = OrderedDict()
    for k, us in rows(path):
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += us
    tot = sum(v[1] for v in agg.values())
    for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{k:60s} {n:6d} launches {us:12.1f} us total {us / n:10.1f} us mean {100 * us / tot:5.1f}%")


if __name__ == "__main__":
    main()
