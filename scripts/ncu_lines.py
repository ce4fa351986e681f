"""Attribute ncu per-SASS metrics (instructions executed, stall samples) to CUDA source lines
using nvdisasm -g line info of the same binary.  usage: ncu_lines.py <rep> <cubin> <mangled fn>"""
import csv
import re
import subprocess
import sys
from collections import defaultdict

rep, cubin, fn = sys.argv[1:4]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(src.splitlines()))
h = r[1]
rows = [dict(zip(h, x)) for x in r[2:] if len(x) == len(h)]
base = int(rows[0]["Address"], 16)
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
sec = dis.split("//--------------------- .text." + fn + " ")[1].split("//---------------------")[0]
line_of = {}
cur = None
for ln in sec.splitlines():
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        line_of[int(m.group(1), 16)] = cur
agg = defaultdict(lambda: [0, 0])
for x in rows:
    off = int(x["Address"], 16) - base
    key = line_of.get(off, ("?", 0))
    agg[key][0] += int(x["Instructions Executed"] or 0)
    agg[key][1] += int(x["Warp Stall Sampling (All Samples)"] or 0)
tot = sum(v[0] for v in agg.values())
tots = sum(v[1] for v in agg.values())
print(f"total warp instructions {tot/1e6:.1f}M, stall samples {tots}")
files = {}
for (f, l), (c, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:int(sys.argv[4]) if len(sys.argv) > 4 else 40]:
    if f not in files:
        try:
            files[f] = open(next(p for p in [f"paper_conf_icpp_liwb15_b200/csrc/{f}"] )).read().splitlines()
        except Exception:
            files[f] = []
    text = files[f][l - 1].strip()[:80] if 0 < l <= len(files[f]) else ""
    print(f"{c/1e6:7.2f}M {100*c/tot:5.1f}%  stalls {st:6d} {f}:{l:<5d} {text}")
