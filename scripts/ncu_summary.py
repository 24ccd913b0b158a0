"""Summarise one ncu report: headline metrics + SASS instruction mix per edge + top stall lines."""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
edges = float(sys.argv[2]) if len(sys.argv) > 2 else 61859140
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
for w in ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
          "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
          "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__t_sector_hit_rate.pct"]:
    if w in hdr:
        i = hdr.index(w)
        print(f"{w:55s} {vals[i][:60]:>20s} {units[i]}")
sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                      text=True).stdout
rows = list(csv.reader(io.StringIO(sass)))
hdr, data = rows[1], rows[2:]
ie, ws, src = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source")
tot = sum(float(r[ie] or 0) for r in data)
tots = sum(float(r[ws] or 0) for r in data)
by = collections.defaultdict(lambda: [0.0, 0.0])
for r in data:
    t = r[src].split()
    op = t[1] if t and t[0].startswith("@") else (t[0] if t else "?")
    by[op.split(".")[0]][0] += float(r[ie] or 0)
    by[op.split(".")[0]][1] += float(r[ws] or 0)
print(f"warp-instructions per edge: {tot / edges:.1f}")
print("  " + " ".join(f"{k}={v[0] / edges:.1f}({v[1] / tots:.0%})" for k, v in sorted(by.items(), key=lambda x: -x[1][0])[:16]))
