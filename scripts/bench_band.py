"""NEXT-2 measurement: GAT forward and backward over the faithful path-band layout
next to the exact-layout forward (mega_gat_fwd over mega_preprocess's layout) on the
same graph, features and parameters; CUDA events, 10 calls after warm-up.  Prints one
JSON line per config with |P| / n, the band's bytes, and both forward times.
Usage: python scripts/bench_band.py [config ...]"""
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_icdcs_dengr24_b200 import mega as M  # noqa: E402

CASES = {   # name -> (config, scaled n, scaled m, dtype)
    "zinc-b256": ("zinc-b256", 0, 0, "fp32"),
    "cycles-b128": ("cycles-b128", 0, 0, "fp32"),
    "csl-b128": ("csl-b128", 0, 0, "fp32"),
    "products-200k": ("products", 200000, 5000000, "bf16"),
    "reddit-50k": ("reddit", 50000, 25000000, "bf16"),
}


def timed(fn, reps=10):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    return float(np.median(ts))


def main():
    names = sys.argv[1:] or list(CASES)
    for name in names:
        cname, sn, sm, dtype = CASES[name]
        cfg = synth.get_config(cname)
        if sn:
            cfg = synth.scaled(cfg, sn, sm)
        ip, ix, _ = synth.make_graph(cfg)
        n, H, F = cfg.n, cfg.heads, cfg.head_dim
        D = H * F
        if dtype == "bf16" and D % 256:
            dtype = "fp32"
        tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
        rng = np.random.default_rng(1)
        Wh = torch.tensor(rng.standard_normal((n, D)).astype(np.float32), device="cuda").to(tdt)
        a_l = torch.tensor((rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32), device="cuda")
        a_r = torch.tensor((rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32), device="cuda")
        t = time.time()
        band = M.mega_band_build(ip, ix)
        tb = time.time() - t
        band.bind()
        v = band.view()
        out = torch.empty_like(Wh)
        ctx = torch.zeros(M.MEGA_CTX_PLANES, n, H, dtype=torch.float32, device="cuda")
        ws = torch.empty(max(M.mega_band_gat_workspace_bytes(band, H, F, M._dtype_code(Wh)), 256), dtype=torch.uint8,
                         device="cuda")
        ms_band = timed(lambda: M.mega_band_gat_fwd(band, Wh, a_l, a_r, H, F, out, ctx, ws))
        g = torch.tensor(rng.standard_normal((n, D)).astype(np.float32), device="cuda").to(tdt)
        gf = torch.empty(n, D, dtype=torch.float32, device="cuda")
        gal, gar = torch.empty(D, device="cuda"), torch.empty(D, device="cuda")
        ms_band_bwd = timed(lambda: M.mega_band_gat_bwd(band, Wh, a_l, a_r, H, F, out, g, ctx, gf, gal, gar, ws))
        # the exact layout's forward on the same graph (features permuted into its order)
        lay = M.mega_preprocess(ip, ix)
        lay.bind(0)
        perm = torch.tensor(lay.view(0)["perm"].astype(np.int64), device="cuda")
        Wn = Wh[perm].contiguous()
        out2 = torch.empty_like(Wn)
        ctx2 = torch.zeros(M.MEGA_CTX_PLANES, n, H, dtype=torch.float32, device="cuda")
        fw, _ = M.mega_gat_workspace_bytes(lay, 0, H, F, M._dtype_code(Wn))
        ws2 = torch.empty(max(fw, 256), dtype=torch.uint8, device="cuda")
        ms_csr = timed(lambda: M.mega_gat_fwd(lay, 0, Wn, a_l, a_r, H, F, out2, ctx2, ws2))
        _, bw = M.mega_gat_workspace_bytes(lay, 0, H, F, M._dtype_code(Wn))
        wsb = torch.empty(max(bw, 256), dtype=torch.uint8, device="cuda")
        gn = g[perm].contiguous()
        gf2 = torch.empty(n, D, dtype=torch.float32, device="cuda")
        ms_csr_bwd = timed(lambda: M.mega_gat_bwd(lay, 0, Wn, a_l, a_r, H, F, out2, gn, ctx2, gf2, gal, gar, wsb))
        # both compute graph attention of the same multiset: compare (band in input order)
        inv = torch.empty_like(perm)
        inv[perm] = torch.arange(n, device="cuda")
        diff = float((out.float() - out2.float()[inv]).abs().max())
        L = int(v["length"])
        band_bytes = 4 * L + 16 * L + 4 * (L + 1) + 2 * len(v["cnt"]) + 4 * L + 12 * int(v["num_merges"])
        print(json.dumps({"config": name, "n": n, "m": cfg.m, "dtype": dtype, "heads": H, "head_dim": F,
                          "window": int(v["window"]), "path_length": L, "appearances_per_node": L / n,
                          "edges_u": int(v["edges_u"]), "edges_u_per_appearance": int(v["edges_u"]) / max(L, 1),
                          "virtual_edges": int(v["virtual_edges"]), "jumps": int(v["jumps"]),
                          "multi_appearance_nodes": int(v["num_merges"]), "partial_slots": int(v["num_slots"]),
                          "band_bytes": band_bytes, "csr_index_bytes": 4 * cfg.m, "build_s": tb,
                          "band_fwd_ms": ms_band, "layout_fwd_ms": ms_csr,
                          "band_bwd_ms": ms_band_bwd, "layout_bwd_ms": ms_csr_bwd,
                          "band_edges_per_s": cfg.m / (ms_band * 1e-3), "layout_edges_per_s": cfg.m / (ms_csr * 1e-3),
                          "max_abs_diff_band_vs_layout": diff}), flush=True)


if __name__ == "__main__":
    main()
