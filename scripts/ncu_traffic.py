"""Per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) of the profiled
kernel in an .ncu-rep -> profiles/traffic.json[key] (bench.py reports it as roofline.traffic).
usage: ncu_traffic.py <rep> <key> [<rep> <key> ...]"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
out = os.path.join(ROOT, "profiles", "traffic.json")
d = json.load(open(out)) if os.path.exists(out) else {}
args = sys.argv[1:]
for rep, key in zip(args[0::2], args[1::2]):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(raw.splitlines()))
    h, u = r[0], r[1]
    vals = []
    for row in r[2:]:
        tot = 0.0
        for name in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = h.index(name)
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u[i]]
            tot += float(row[i]) * scale
        vals.append(tot)
    d[key] = int(sum(vals) / len(vals))
    print(key, d[key], f"({len(vals)} launch(es) of {rep})")
d["_note"] = ("dram__bytes_read.sum + dram__bytes_write.sum per launch of the dominant kernel, "
              "ncu --set full --clock-control none (scripts/ncu_traffic.py; reports under profiles/)")
json.dump(d, open(out, "w"), indent=1)
