"""Bare row-gather over the forward source stream of several node orders
(analysis only): how much L2 reuse does each order buy on the real chip?
Prints requested GB/s per order; run under ncu for DRAM bytes per launch.
Usage: python scripts/calib_orders.py [config] [reps]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import synth  # noqa: E402
from calib import timed_gather  # noqa: E402
from order_sim import communities, stream_of  # noqa: E402
from paper_conf_icdcs_dengr24_b200 import mega as M  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "products"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    cfg = synth.CONFIGS[name]
    rb = cfg.dim * 2
    ip, ix, _ = synth.make_graph(cfg)
    orders = {}
    lay = M.mega_preprocess(ip, ix)
    orders["traversal"] = lay.view(0)["perm"].astype(np.int64)
    lay = M.mega_preprocess(ip, ix, block_rows=M.auto_block_rows(rb))
    orders["blocked"] = lay.view(0)["perm"].astype(np.int64)
    comm = communities(cfg)
    pos = np.empty(cfg.n, np.int64)
    pos[orders["traversal"]] = np.arange(cfg.n)
    orders["community"] = np.lexsort((pos, comm))
    extra = os.environ.get("ORDER_NPY")
    if extra:
        orders["extra"] = np.load(extra)
    table = torch.zeros(cfg.n, rb // 2, dtype=torch.bfloat16, device="cuda")
    for k, perm in orders.items():
        idx = torch.tensor(stream_of(perm, ip, ix), device="cuda")
        r = timed_gather(table, rb, idx, reps)
        print(f"{name} {k}: {r['ms']:.2f} ms  {r['GBps']:.0f} GB/s requested", flush=True)


if __name__ == "__main__":
    main()
