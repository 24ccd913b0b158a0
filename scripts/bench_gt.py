"""Time the NEXT-3 Graph Transformer kernels (mega_gt_fwd / mega_gt_bwd, bf16 and fp32) on
BASELINE-shaped synthetic graphs with CUDA events on the launching stream.
Prints one JSON line per config: ms per fwd / bwd call, layer-edges/s and the
requested-bytes rate of the per-edge row gathers (fwd: K_j and V_j rows, 2 D 4
bytes per edge; bwd dst pass: K_j, V_j; src pass: Q_i, g_i -> 4 D 4 bytes per
edge) against the measured HBM peak.  Usage: python scripts/bench_gt.py [cfg ...]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_icdcs_dengr24_b200 import mega as M  # noqa: E402


def run(name, steps=10, dtype="bf16"):
    cfg = synth.get_config(name)
    ip, ix, _ = synth.make_graph(cfg)
    lay = M.mega_preprocess(ip, ix)
    lay.bind(0)
    n, H, F = cfg.n, cfg.heads, cfg.head_dim
    D = H * F
    gen = torch.Generator(device="cuda").manual_seed(cfg.seed & 0xFFFFFFFF)
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    q, k, v, g = (torch.randn(n, D, device="cuda", generator=gen).to(tdt) for _ in range(4))
    out = torch.empty(n, D, device="cuda", dtype=tdt)
    lse = torch.empty(n, H, device="cuda")
    gq, gk, gv = (torch.empty(n, D, device="cuda") for _ in range(3))
    ws = torch.empty(M.mega_gt_workspace_bytes(lay, 0, H, F, M._dtype_code(q)), dtype=torch.uint8, device="cuda")

    def fwd():
        M.mega_gt_fwd(lay, 0, q, k, v, H, F, out, lse, ws)

    def bwd():
        M.mega_gt_bwd(lay, 0, q, k, v, H, F, out, lse, g, gq, gk, gv, ws)

    for _ in range(3):
        fwd()
        bwd()
    torch.cuda.synchronize()
    res = {}
    for nm, fn in (("fwd", fwd), ("bwd", bwd)):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        for _ in range(steps):
            fn()
        e.record()
        torch.cuda.synchronize()
        res[nm] = s.elapsed_time(e) / steps
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    m = cfg.m
    sb = 2 if dtype == "bf16" else 4
    line = {"workload": f"{name}-shaped GT attention ({dtype})", "nodes": n, "edges": m, "heads": H, "head_dim": F,
            "fwd_ms": res["fwd"], "bwd_ms": res["bwd"],
            "edges_per_s_fwd_bwd": m / ((res["fwd"] + res["bwd"]) * 1e-3),
            "fwd_gather_gbs": m * 2 * D * sb / (res["fwd"] * 1e-3) / 1e9,
            "bwd_gather_gbs": m * 4 * D * sb / (res["bwd"] * 1e-3) / 1e9,
            "peaks": {k: v for k, v in peak.items() if "hbm" in k.lower()}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    for dt in ("bf16", "fp32"):
        for c in sys.argv[1:] or ["zinc-b256", "reddit", "products"]:
            run(c, dtype=dt)
