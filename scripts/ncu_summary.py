"""Summarise an .ncu-rep (raw metrics + top stall sites) for profiles/."""
import csv
import re
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
h, units = r[0], r[1]
pat = re.compile(r"gpu__time_duration.sum$|dram__bytes_(read|write)\.sum$|lts__t_sectors_srcunit_tex_op_read.sum$|"
                 r"lts__t_sector_hit_rate.pct$|dram__throughput.avg.pct_of_peak_sustained_elapsed$|"
                 r"sm__warps_active.avg.pct_of_peak_sustained_active$|launch__grid_size$|launch__block_size$|"
                 r"launch__occupancy_limit_(registers|shared_mem|warps)$|launch__registers_per_thread$|"
                 r"lts__throughput.avg.pct_of_peak_sustained_elapsed$|l1tex__t_sector_hit_rate.pct$|"
                 r"smsp__inst_executed.sum$|smsp__thread_inst_executed_per_inst_executed.ratio$|"
                 r"smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct$|"
                 r"smsp__average_warps_issue_stalled_(long_scoreboard|barrier|short_scoreboard|wait|lg_throttle|mio_throttle|no_instruction|math_pipe_throttle|branch_resolving|membar|sleeping)_per_issue_active.ratio$|"
                 r"sm__throughput.avg.pct_of_peak_sustained_elapsed$|l1tex__throughput.avg.pct_of_peak_sustained_elapsed$")
for row in r[2:]:
    name = row[h.index("Kernel Name")] if "Kernel Name" in h else "?"
    print("kernel:", name[:120])
    for k, u, v in zip(h, units, row):
        if pat.search(k):
            print(f"  {k:90s} {v:>16s} {u}")
if len(sys.argv) > 2:
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rr = list(csv.reader(src.splitlines()))
    hh = rr[1]
    rows = [dict(zip(hh, x)) for x in rr[2:] if len(x) == len(hh)]
    tot = sum(int(x["Warp Stall Sampling (All Samples)"]) for x in rows)
    print("stall samples:", tot)
    top = sorted(range(len(rows)), key=lambda i: -int(rows[i]["Warp Stall Sampling (All Samples)"]))[: int(sys.argv[2])]
    for i in top:
        x = rows[i]
        print(f"----- {x['Address'][-5:]} {x['Warp Stall Sampling (All Samples)']}")
        for y in rows[max(0, i - 3): i + 1]:
            print(f"    {y['Address'][-5:]} {y['Warp Stall Sampling (All Samples)']:>6s} {y['Instructions Executed']:>9s} {y['Source'][:90]}")
