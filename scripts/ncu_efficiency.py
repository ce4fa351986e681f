#!/usr/bin/env python
"""The paper's Table I / II metrics from an ncu metrics-only launch list:

  ncu --metrics gpu__time_duration.sum,smsp__thread_inst_executed_per_inst_executed.ratio,\
smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct,\
smsp__sass_average_data_bytes_per_sector_mem_global_op_st.pct --clock-control none --csv \
      --log-file X.csv <cmd>
  python scripts/ncu_efficiency.py X.csv [kernel-regex] [label]

warp_eff = thread instructions per warp instruction / 32 (the paper's "warp execution
efficiency"); gld_eff / gst_eff = bytes used per sector moved for global loads / stores (its
"gld / gst efficiency").  Launches matching the regex are combined weighted by their device
time.  Prints one line: label, launches, kernel us, warp_eff, gld_eff, gst_eff.
"""
import csv
import re
import sys
from collections import defaultdict


def main():
    path = sys.argv[1]
    rx = re.compile(sys.argv[2]) if len(sys.argv) > 2 else re.compile(".")
    label = sys.argv[3] if len(sys.argv) > 3 else path
    hdr, launches = None, defaultdict(dict)
    names = {}
    for r in csv.reader(open(path)):
        if "Kernel Name" in r and "Metric Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if not rx.search(d["Kernel Name"]):
            continue
        key = d.get("ID", "") + "|" + d["Kernel Name"]
        names[key] = d["Kernel Name"]
        v = d["Metric Value"].replace(",", "")
        try:
            launches[key][d["Metric Name"]] = float(v)
        except ValueError:
            pass
    tw = sum(m.get("gpu__time_duration.sum", 0.0) for m in launches.values())
    def wavg(metric):
        num = sum(m.get("gpu__time_duration.sum", 0.0) * m.get(metric, 0.0) for m in launches.values())
        return num / tw if tw else 0.0
    we = wavg("smsp__thread_inst_executed_per_inst_executed.ratio") / 32.0
    ld = wavg("smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct")
    st = wavg("smsp__sass_average_data_bytes_per_sector_mem_global_op_st.pct")
    print(f"{label:28s} {len(launches):8d} {tw / 1000.0:12.1f} {we:9.3f} {ld:8.1f} {st:8.1f}")


if __name__ == "__main__":
    main()
