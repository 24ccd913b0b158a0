"""Row-gather bandwidth calibration on the GPU: how fast can
rows be gathered by index for the access patterns the attention kernels see?
Writes profiles/calib_gather.json when --out is given."""
import argparse
import ctypes
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_icdcs_dengr24_b200 import mega as M  # noqa: E402


def timed_gather(table, row_bytes, idx, reps=5):
    L = M.lib()
    L.mega_calib_gather.restype = ctypes.c_int
    L.mega_calib_gather.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_int64,
                                    ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
    sink = torch.empty(1 << 16, dtype=torch.float32, device="cuda")
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    args = (ctypes.c_void_p(table.data_ptr()), table.shape[0], row_bytes, ctypes.c_void_p(idx.data_ptr()),
            idx.numel(), ctypes.c_void_p(sink.data_ptr()), sink.numel(), st)
    assert L.mega_calib_gather(*args) == 0, M.lib().mega_last_error()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        L.mega_calib_gather(*args)
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    ms = float(np.median(ts))
    return {"ms": ms, "GBps": idx.numel() * row_bytes / (ms * 1e-3) / 1e9}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out")
    args = ap.parse_args()
    res = {}
    for name, rb in (("products", 1024), ("reddit", 512)):
        cfg = synth.CONFIGS[name]
        ip, ix, _ = synth.make_graph(cfg)
        table = torch.zeros(cfg.n, rb // 2, dtype=torch.bfloat16, device="cuda")
        n = cfg.m
        rng = np.random.default_rng(0)
        pats = {"random": rng.integers(0, cfg.n, n, dtype=np.int32)}
        for order in ("traversal", "identity"):
            lay = M.mega_preprocess(ip, ix, order=order)
            pats[f"csr_src_{order}"] = lay.view(0)["src"]
        lay = M.mega_preprocess(ip, ix, block_rows=M.auto_block_rows(rb))
        pats["csr_src_traversal_l2blocked"] = lay.view(0)["src"]
        # L2-resident table: random rows of the first 24 MB (the L2 gather ceiling)
        pats["random_l2_resident"] = rng.integers(0, (24 << 20) // rb, n, dtype=np.int32)
        pats["sequential"] = (np.arange(n, dtype=np.int64) % cfg.n).astype(np.int32)
        for k, v in pats.items():
            idx = torch.tensor(v, device="cuda")
            r = timed_gather(table, rb, idx)
            res[f"{name}/{k}"] = {"rows": cfg.n, "row_bytes": rb, "table_MB": cfg.n * rb / 1e6, "n": n, **r}
            print(name, k, r, flush=True)
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
