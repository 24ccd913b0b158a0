"""Instruction mix and hot runs of one kernel from an ncu report (--page source --csv).
Usage: python scripts/ncu_src_summary.py report.ncu-rep kernel_regex edges [nruns]"""
import collections
import csv
import io
import subprocess
import sys

rep, kre, E = sys.argv[1], sys.argv[2], float(sys.argv[3])
nruns = int(sys.argv[4]) if len(sys.argv) > 4 else 12
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", "regex:" + kre],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
ie = h.index("Instructions Executed")
d = [r for r in rows[2:] if len(r) == len(h) and r[ie].isdigit()]
seen, dd = set(), []
for r in d:          # the export repeats the listing; keep the first copy of each address
    if r[0] in seen:
        break
    seen.add(r[0])
    dd.append(r)
d = dd
si, ist = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
tot = sum(int(r[ie]) for r in d)
print(f"{kre}: {tot / E:.1f} warp instructions per edge, {len(d)} SASS lines")
c, s = collections.Counter(), collections.Counter()
for r in d:
    t = r[si].strip().split()
    if not t:
        continue
    op = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
    c[op] += int(r[ie])
    s[op] += int(r[ist] or 0)
print(" ".join(f"{op}={n / E:.1f}" for op, n in c.most_common(18)))
runs, cur = [], None
for i, r in enumerate(d):
    n = int(r[ie])
    if cur and abs(n - cur[1]) <= 0.02 * max(n, 1):
        cur[2] += 1; cur[3] += n; cur[4] += int(r[ist] or 0)
    else:
        cur = [i, n, 1, n, int(r[ist] or 0)]
        runs.append(cur)
runs.sort(key=lambda x: -x[3])
for st, n, cnt, tt, stall in runs[:nruns]:
    print(f"  @{st:5d} len {cnt:4d} x {n / E:.3f}/edge = {tt / E:6.2f}/edge  stall {stall:7d}  {d[st][si].strip()[:50]}")
