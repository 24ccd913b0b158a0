"""From an ncu launch list with gpu__time_duration / dram bytes per launch, derive
per-kernel shares and per-call DRAM traffic (bench.py's `traffic` field).

usage: launch_traffic.py launches.csv steps_run layers out_prefix
The launch list holds `steps_run` identical steps (warm-up + timed); the last
one is used."""
import collections
import csv
import io
import json
import sys

path, steps, layers, out = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
lines = open(path).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
hdr, data = rows[0], rows[1:]
ki, mi, vi, ii = (hdr.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "ID"))
launch = collections.OrderedDict()
for r in data:
    d = launch.setdefault(r[ii], {"name": r[ki]})
    d[r[mi]] = float(r[vi].replace(",", ""))


def short(n):
    n = n.split("(")[0].replace("void ", "")
    return n.replace("mega::", "").replace("kern::", "") if "mega::" in n else "[lib] " + n[:48]


L = list(launch.values())
sel = L[len(L) * (steps - 1) // steps:]
tot = collections.defaultdict(lambda: [0, 0.0, 0.0])
for d in sel:
    k = short(d["name"])
    t = tot[k]
    t[0] += 1
    t[1] += d.get("gpu__time_duration.sum", 0)
    t[2] += d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
T = sum(v[1] for v in tot.values())
rows_out = []
for k, (n, t, b) in sorted(tot.items(), key=lambda x: -x[1][1]):
    rows_out.append({"kernel": k, "launches": n, "time_ns": t, "share": t / T, "dram_bytes": b,
                     "dram_bytes_per_launch": b / n})
    print(f"{k[:60]:60s} n={n:3d} share={t / T:6.1%} dram/launch={b / n / 1e9:8.3f} GB")
json.dump(rows_out, open(out + "_launches.json", "w"), indent=1)


def per_launch(pred):
    return sum(r["dram_bytes"] for r in rows_out if pred(r["kernel"])) / layers


traffic = {
    "gat_fwd": per_launch(lambda k: k.startswith(("gat_fwd", "fwd_stats"))),
    "gat_bwd": per_launch(lambda k: k.startswith(("dlt_kernel", "gat_bwd_src", "gat_bwd_dst", "param_reduce"))),
    "gat_bwd_src": per_launch(lambda k: k.startswith(("dlt_kernel", "gat_bwd_src"))),
    "gat_bwd_dst": per_launch(lambda k: k.startswith(("gat_bwd_dst", "param_reduce"))),
    "note": "ncu DRAM read+write bytes per layer-launch of the call's kernels (cold-cache, serialised replay)",
}
json.dump(traffic, open(out + "_traffic.json", "w"), indent=1)
print(json.dumps(traffic))
