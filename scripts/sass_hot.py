"""Top SASS instructions by warp-stall samples from `ncu --page source --csv --print-source sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
ci = hdr.index("Source")
si = hdr.index("Warp Stall Sampling (All Samples)")
cols = [c for c in hdr if c.startswith("stall_") and "Not Issued" not in c]
tot = sum(float(r[si] or 0) for r in data if len(r) > si)
top = sorted(data, key=lambda r: -float(r[si] or 0) if len(r) > si else 0)[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]
print(f"total samples {tot:.0f}")
for r in top:
    s = float(r[si] or 0)
    br = sorted(((c, float(r[hdr.index(c)] or 0)) for c in cols), key=lambda x: -x[1])[:3]
    print(f"{s / tot:6.1%} {r[0]:>6s} {r[ci][:70]:70s} " + " ".join(f"{c[6:]}={v:.0f}" for c, v in br))
