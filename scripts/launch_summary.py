"""Summarise an ncu launch list (gpu__time_duration.sum per launch) into per-kernel shares."""
import collections
import csv
import io
import json
import sys


def summarise(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
    hdr, data = rows[0], rows[1:]
    ki, vi, mi, ui = (hdr.index(k) for k in ("Kernel Name", "Metric Value", "Metric Name", "Metric Unit"))
    tot, cnt, unit = collections.defaultdict(float), collections.Counter(), None
    for r in data:
        if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki]
        short = name.split("(")[0]
        if "mega::kern::" in short:
            short = short.replace("void ", "").split("mega::kern::")[1]
        else:
            short = "[lib] " + short.replace("void ", "")[:50]
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        tot[short] += v
        cnt[short] += 1
    T = sum(tot.values())
    out = [{"kernel": k, "launches": cnt[k], "total": v, "unit": unit, "share": v / T}
           for k, v in sorted(tot.items(), key=lambda x: -x[1])]
    return out


if __name__ == "__main__":
    res = summarise(sys.argv[1])
    for r in res:
        print(f"{r['kernel'][:70]:70s} n={r['launches']:4d} {r['total']:14.1f} {r['unit']} {r['share']:6.1%}")
    if len(sys.argv) > 2:
        json.dump(res, open(sys.argv[2], "w"), indent=1)
