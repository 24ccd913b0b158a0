#!/usr/bin/env python
"""bench.py — MEGA GAT layer fwd+bwd on B200 (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl mega|reference]
                  [--config products|reddit|arxiv|pubmed|cora] [--dtype bf16|fp32]

One "step" = one pass of the whole hot path over the
workload: every GAT layer of the config forward (projection on tensor cores,
fused attention) then backward (attention backward, projection backward).
`value` = layers * E / step time: GAT layer fwd+bwd edges per second, whole
job.  Inputs are resident in HBM when the timed region starts; `e2e` repeats
the measurement with the step's inputs copied from pinned host memory and the
parameter gradients read back every step.  `--impl reference` times the CPU
oracle (oracle/, the only other place bench.py runs it) on a bounded sample.
Multi-GPU (torchrun, N > 1): destination partitions of the MEGA order, one per
rank; see paper_conf_icdcs_dengr24_b200/dist.py.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "GAT layer fwd+bwd edges/sec and HBM GB/s fraction at 1/2/4/8 B200"


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mega", choices=["mega", "reference"])
    ap.add_argument("--config", default="products")
    ap.add_argument("--dtype", default="bf16", choices=["bf16", "fp32"])
    ap.add_argument("--order", default="traversal",
                    help="traversal (MEGA), identity, degree, random, community (ablations, SURVEY 8(d)-d5)")
    ap.add_argument("--window", type=int, default=0, help="traversal window omega (0 = auto)")
    ap.add_argument("--seg-edges", type=int, default=0, help="work-item segment size S (0 = auto)")
    ap.add_argument("--block-rows", type=int, default=-1,
                    help="L2 blocking B (DESIGN.md R24): -1 = auto (0.4 L2 / row bytes), 0 = off")
    ap.add_argument("--cuda-graph", action="store_true",
                    help="capture one step in a CUDA graph and replay it (launch-bound batch workloads)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    return ap.parse_args()


# ------------------------------------------------------------------ helpers
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "100"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        t0 = time.time()   # the sampler must be live before the timed region starts
        while self.proc is not None and not self.rows and time.time() - t0 < 3.0:
            time.sleep(0.02)
        self.skip = len(self.rows)   # samples taken before the timed region are not counted
        self.after = False
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *exc):
        if self.proc and len(self.rows) <= self.skip:   # a region shorter than the 100 ms sampling period
            try:
                out = subprocess.run(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits", "-i",
                                      str(self.index)], capture_output=True, text=True, timeout=10).stdout
                self.rows += [[x.strip() for x in ln.split(",")] for ln in out.splitlines() if ln.strip()]
                self.after = True
            except (OSError, subprocess.TimeoutExpired):
                pass
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        rows = self.rows[getattr(self, "skip", 0):]
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.rows = rows
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 4 + i and "Active" in r[4 + i]
                          and "Not" not in r[4 + i]})
        out = {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
               "reasons": reasons, "samples": len(self.rows)}
        if getattr(self, "after", False):
            out["sampled"] = "right after the timed region (shorter than the 100 ms sampling period)"
        return out


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d.get("bf16_tflops_sustained", d["bf16_tflops"]),
                "source": "measured (MEASURED_PEAKS.json)"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "source": "fallback (B200_PROFILING.md)"}


# Measured ceiling of gathering random 1 KB rows through L2 (scripts/l2probe.cu, all hits: working set
# <= 64 MB, 16 GB requested per launch, 8 CTAs/SM): 17.4 TB/s requested (profiles/r02/l2/probe_p0.txt).
# The gathering kernels' "gather_frac" is their requested row rate against it (E rows of D*s bytes).
L2_GATHER_TBS = 17.4


def floor_bytes(kernel, rows, N, E, H, D, sb, R=None):
    """SURVEY §8(d)-d3 algorithmic bytes of one launch group, with R row fetches of the
    gathered operand (R = N: the compulsory floor, every gathered row once; R = E: no
    reuse).  bf16/fp32 storage sb, out in storage type, fp32 dWh, int32 indices.
      KB2      B_fwd = 4E + R (D sb + 4H) + rows (8 + 8H + D sb)
      KB3+KB4  N (2D sb + 4H) + 4E(1+H) + R (D sb + 12H) + N (8 + D sb + 8H + 4D)
      KB5      4E(1+H) + N (8 + 8D + 4H + D sb)
    (rows = destination rows of the part; N = rows at k = 1)."""
    R = N if R is None else R
    if kernel == "KB2":
        return 4 * E + R * (D * sb + 4 * H) + rows * (8 + 8 * H + D * sb)
    if kernel == "KB3+KB4":
        return rows * (2 * D * sb + 4 * H) + 4 * E * (1 + H) + R * (D * sb + 12 * H) + N * (8 + D * sb + 8 * H + 4 * D)
    if kernel == "KB5":
        return 4 * E * (1 + H) + rows * (8 + 8 * D + 4 * H + D * sb)
    raise KeyError(kernel)


def design_bytes(kernel, rows, N, E, H, D, sb):
    """The design's own compulsory bytes (LP_ONLY training path): what these
    kernels must move given the layout (16-byte work items, the cpos map, dz in CSR order,
    the bf16 projection operand written instead of fp32 dWh; in bf16 the source pass's dWh
    partial also lives in that operand, DESIGN.md R-lp)."""
    items = 16 * rows
    pb = sb if sb == 2 else 4   # bytes of the dWh partial handed from the source to the destination pass
    if kernel == "KB2":   # idx, items, Wh, er (all sources once), el, out, lse
        return 4 * E + items + N * D * sb + N * H * 4 + rows * H * 4 + rows * D * sb + rows * H * 4
    if kernel == "KB3+KB4":   # g,out -> Dlt; cdst, cpos, items, Wh, er, g_i, el/lse/Dlt, dz, dWh, der
        return ((2 * rows * D * sb + rows * H * 4) + (8 * E + 16 * N + N * D * sb + N * H * 4 + rows * D * sb
                                                       + 3 * rows * H * 4 + 4 * E * H + N * D * pb + N * H * 4))
    if kernel == "KB5":   # indptr, dz, dWh partial, der, Wh, bf16 operand
        return 4 * (rows + 1) + 4 * E * H + rows * D * pb + rows * H * 4 + rows * D * sb + rows * D * pb
    raise KeyError(kernel)


# kernel-name prefixes (ncu launch list) of each launch group
GROUPS = {"KB2": ("gat_fwd",), "KB3+KB4": ("dlt_kernel", "gat_bwd_src"), "KB5": ("gat_bwd_dst", "param_reduce"),
          "proj_fwd": ("umma_gemm_persistent<0",),
          "proj_bwd": ("umma_gemm_persistent<1", "umma_gemm_kernel<2", "dw_reduce")}


def ncu_launch_summary(path):
    """Per launch group: mean DRAM bytes, ncu duration and tensor-pipe % per call, from an
    ncu --csv launch list (scripts/gpu_prof_r02.sh).  Each kernel type of a group is
    launched once per call, so a group's per-call figure is the sum of its kernels' means."""
    import csv
    if not os.path.exists(path):
        return None
    per = {}
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for row in csv.DictReader(lines):
        name = row.get("Kernel Name", "")
        full = name.split("(")[0].replace("void ", "")
        head = full.split("<")[0]
        short = head.split("::")[-1] + full[len(head):]     # namespaces dropped, template args kept
        d = per.setdefault(short, {})
        try:
            v = float(row["Metric Value"].replace(",", ""))
        except (KeyError, ValueError):
            continue
        unit = row.get("Metric Unit", "")
        v *= {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1e3, "msecond": 1e6, "second": 1e9}.get(unit, 1.0)
        d.setdefault(row["Metric Name"], []).append(v)
    out = {}
    for g, pref in GROUPS.items():
        ks = [k for k in per if any(k.startswith(p) for p in pref)]
        if not ks:
            continue
        mean = lambda k, m: float(np.mean(per[k].get(m, [0.0])))   # noqa: E731
        dur_unit = 1e-6   # gpu__time_duration in ns (ncu default "nsecond")
        out[g] = {"dram_bytes": sum(mean(k, "dram__bytes_read.sum") + mean(k, "dram__bytes_write.sum") for k in ks),
                  "ncu_ms": sum(mean(k, "gpu__time_duration.sum") for k in ks) * dur_unit,
                  "kernels": sorted(ks)}
        tp = [mean(k, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed") for k in ks
              if "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed" in per[k]]
        if g.startswith("proj") and tp:
            out[g]["tensor_pipe_pct"] = max(tp)
    return out


# ------------------------------------------------------------------ workload
def block_rows_for(cfg, dtype, block_rows=-1, l2_bytes=None):
    """-1 -> auto: 0.4 of the device L2 in gathered rows (D * bytes per element; R24,
    the rule of mega.auto_block_rows).  Pure arithmetic: the reference arm uses it too."""
    if block_rows >= 0:
        return block_rows
    if l2_bytes is None:
        l2_bytes = 126 * 1024 * 1024
        try:
            import torch
            if torch.cuda.is_available():
                l2_bytes = torch.cuda.get_device_properties(torch.cuda.current_device()).L2_cache_size
        except Exception:  # noqa: BLE001 - no device: the B200 figure
            pass
    return max(1, int(0.4 * l2_bytes) // max(1, cfg.dim * (2 if dtype == "bf16" else 4)))


def build_workload(cfg_name, dtype, order, rank=0, world=1, window=0, seg_edges=0, block_rows=-1):
    import synth
    cfg = synth.get_config(cfg_name)
    block_rows = block_rows_for(cfg, dtype, block_rows)
    t0 = time.time()
    indptr, indices, gstats = synth.make_graph(cfg)
    t_gen = time.time() - t0
    from paper_conf_icdcs_dengr24_b200 import mega as M
    relabel = None
    if order in ("community", "comdeg"):   # ablation upper bound: nodes sorted by generator
        comm = synth.communities(cfg)         # community (comdeg: and by descending in-degree inside it)
        keys = (np.arange(cfg.n), comm) if order == "community" else (np.arange(cfg.n), -np.diff(indptr), comm)
        relabel = np.lexsort(keys)
        ip_in, ix_in = synth.relabel(indptr, indices, relabel)
        order, block_rows = "identity", 0
    else:
        ip_in, ix_in = indptr, indices
    t0 = time.time()
    layout = M.mega_preprocess(ip_in, ix_in, order=order, num_parts=world, window=window, seg_edges=seg_edges,
                               block_rows=block_rows)
    t_pre = time.time() - t0
    perm = layout.view(0)["perm"].astype(np.int64)
    if relabel is not None:
        perm = relabel[perm]     # back to the generator's node ids
    layers = []
    in_dim = cfg.f_in
    for li in range(cfg.layers):
        inp = synth.make_layer_inputs(cfg, layer=li, in_dim=in_dim)
        if dtype == "bf16":
            inp["w"] = synth.bf16_round(inp["w"])
        layers.append(inp)
        in_dim = cfg.dim
    x0 = layers[0]["x"][perm]
    g_last = layers[-1]["grad_out"][perm]
    if dtype == "bf16":
        x0, g_last = synth.bf16_round(x0), synth.bf16_round(g_last)
    return {"cfg": cfg, "indptr": indptr, "indices": indices, "layout": layout, "perm": perm, "layers": layers,
            "x0": np.ascontiguousarray(x0), "g_last": np.ascontiguousarray(g_last), "gen_s": t_gen, "pre_s": t_pre,
            "graph_stats": gstats}


class Model:
    """The config's GAT stack on this rank's part (k = world), every step through libmega.so."""

    def __init__(self, wl, dtype, dev, rank=0, world=1):
        import torch
        from paper_conf_icdcs_dengr24_b200.dist import DistGATLayer, make_comm
        self.torch = torch
        cfg = wl["cfg"]
        tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
        lay = wl["layout"]
        lay.bind(rank)
        v = lay.view(rank, arrays=False)
        self.b0, self.b1 = v["row_begin"], v["row_end"]
        self.rows, self.part_edges = self.b1 - self.b0, v["part_edges"]
        self.x0 = torch.tensor(wl["x0"][self.b0:self.b1], device=dev).to(tdt).contiguous()
        self.g = torch.tensor(wl["g_last"][self.b0:self.b1], device=dev).to(tdt).contiguous()
        self.layers = []
        self.comm = make_comm() if world > 1 else None   # library-owned NCCL communicator
        x = self.x0
        for li, inp in enumerate(wl["layers"]):
            w = torch.tensor(inp["w"], device=dev).to(tdt).contiguous()
            Ld = DistGATLayer(lay, rank, x, w, torch.tensor(inp["a_l"], device=dev),
                              torch.tensor(inp["a_r"], device=dev), cfg.heads, cfg.head_dim, in_dim=inp["in_dim"],
                              want_grad_x=li > 0, lp_only=dtype == "bf16", comm=self.comm)
            self.layers.append(Ld)
            x = Ld.L.out
        self.launches = sum(Ld.L.launches_per_step() for Ld in self.layers)

    def step(self, ev=None, before_bwd=None, split=False):
        """ev: optional dict name -> list of (start, end) event pairs to record into;
        before_bwd: called between the forward and the backward (e2e: wait for grad_out's copy);
        split: run the single-GPU backward as its two phases (per-kernel-group timing)."""
        torch = self.torch

        def timed(name, fn):
            if ev is None:
                fn()
                return
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            fn()
            e.record()
            ev.setdefault(name, []).append((s, e))

        for Ld in self.layers:
            Ld.forward(timed)
        if before_bwd is not None:
            before_bwd()
        g = self.g
        for Ld in reversed(self.layers):
            g = Ld.backward(g, timed, split=split)


# ------------------------------------------------------------------ CPU oracle
def cpu_sample(cfg, indptr, indices, seconds_target):
    """Bounded sample of the workload for the CPU oracle (oracle/ only; no libmega.so):
    the first R destination rows of the INPUT order (mega-synth permutes ids at random,
    so this is a uniform sample of destinations) with all their in-edges, compacted to
    the nodes they touch, run through every layer of the config as one step: projection
    (oracle.gat.project_forward), attention forward and backward (oracle/c, fp64, OpenMP)
    and projection backward, with the config's layer widths.  Returns (run, R, describe)
    where run(R) -> (seconds, sample edges)."""
    from oracle import coracle
    from oracle import gat as og
    import synth
    indptr = np.asarray(indptr, np.int64)
    indices = np.asarray(indices)
    n = len(indptr) - 1
    H, F, D = cfg.heads, cfg.head_dim, cfg.dim
    rng = np.random.default_rng(0)
    widths = [cfg.f_in_pad] + [D] * (cfg.layers - 1)
    ws = [synth.bf16_round(rng.uniform(-0.05, 0.05, (k, D)).astype(np.float32)) for k in widths]
    a_l = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    a_r = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    base_x = synth.bf16_round(rng.standard_normal((4096, max(widths))).astype(np.float32))
    base_g = synth.bf16_round(rng.standard_normal((4096, D)).astype(np.float32))

    def sub(R):
        e = int(indptr[R])
        nodes, inv = np.unique(np.concatenate([np.arange(R, dtype=np.int64), indices[:e].astype(np.int64)]),
                               return_inverse=True)   # ids 0..R-1 keep their positions
        k = len(nodes)
        ptr = np.concatenate([indptr[:R + 1], np.full(k - R, e, np.int64)])
        return ptr, inv[R:].astype(np.int32), nodes, e

    def run(R):
        ptr, idx, nodes, e = sub(R)
        k = len(nodes)
        g = base_g[nodes & 4095].reshape(k, H, F)     # values do not change the work
        Wh = base_g[nodes & 4095].copy()              # rows of sources outside the sample (values only)
        t0 = time.perf_counter()
        for li, w in enumerate(ws):
            # the sample owns its R destination rows: their projection (fwd and bwd) is its share of the
            # layer's dense work, so GEMM work per edge matches the full workload (N/E rows per edge)
            x = base_x[nodes[:R] & 4095, :w.shape[0]]
            Wh[:R] = og.project_forward(x, w)
            f = coracle.gat_forward(ptr, idx, Wh.reshape(k, H, F), a_l, a_r)
            b = coracle.gat_backward(ptr, idx, Wh.reshape(k, H, F), a_l, a_r, g, fwd=f)
            og.project_backward(x, w, b["grad_feat"].reshape(k, D)[:R])
        return time.perf_counter() - t0, e

    try:   # host-memory bound: ~8 fp64 [k, D] arrays for the k touched nodes
        import psutil
        cap = 0.4 * psutil.virtual_memory().available
    except Exception:  # pragma: no cover
        cap = 16e9

    def fits(R):
        k = len(np.unique(np.concatenate([np.arange(R, dtype=np.int64), indices[:indptr[R]]])))
        return k * D * 8 * 8 + 32 * int(indptr[R]) <= cap

    R = max(1, min(n, int(np.searchsorted(indptr, 50000))))
    t, e = run(R)
    for _ in range(3):
        if t >= seconds_target / 2 or R >= n:
            break
        e_want = int(e * seconds_target / max(t, 1e-3))
        R2 = max(R + 1, min(n, int(np.searchsorted(indptr, min(len(indices), e_want)))))
        while R2 > R + 1 and not fits(R2):
            R2 = R + (R2 - R) // 2
        if R2 <= R + 1 and not fits(R2):
            break
        R = R2
        t, e = run(R)

    def describe(R, e, t=None):
        return (f"oracle/ fp64 (oracle/c OpenMP attention + numpy projection), one step of all {cfg.layers} "
                f"layers (projection fwd, GAT fwd+bwd, projection bwd; H={H}, F={F}) over the first {R} "
                f"destination rows of the input order and their {e} in-edges, compacted to the nodes they touch; "
                f"the projection runs on the sample's own R rows"
                + ("" if t is None else f"; {t:.1f} s"))
    return run, R, describe


def cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count()


# ------------------------------------------------------------------ main paths
def workload_config(cfg, args, block_rows, flush_note):
    """The `config` object of the JSON line, shared by both arms."""
    return {"workload": f"{cfg.name}-shaped synthetic GAT", "nodes": cfg.n, "edges": cfg.m, "layers": cfg.layers,
            "heads": cfg.heads, "head_dim": cfg.head_dim, "f_in": cfg.f_in, "order": args.order,
            "block_rows": block_rows,
            "value_definition": "layers * E / step time (each layer's edges fwd+bwd; max over ranks)",
            "l2": flush_note,
            **({"batch": cfg.batch, "num_graphs": cfg.num_graphs, "edge_drop": cfg.drop} if cfg.batch else {})}


def run_reference(args):
    """--impl reference: the CPU oracle (oracle/, never libmega.so) timed on this box's
    host cores, on bounded samples of the same workload; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import synth
    cfg = synth.get_config(args.config)
    indptr, indices, _ = synth.make_graph(cfg)
    per_step = max(2.0, min(10.0, 150.0 / max(1, args.steps + args.warmup)))
    run, R, describe = cpu_sample(cfg, indptr, indices, per_step)
    for _ in range(args.warmup):
        run(R)
    times, edges = [], 0
    for _ in range(args.steps):
        t, e = run(R)
        times.append(t)
        edges = e
    tot = float(np.sum(times))
    value = cfg.layers * edges * args.steps / tot
    sample = describe(R, edges)
    conf = workload_config(cfg, args, block_rows_for(cfg, args.dtype, args.block_rows), "host memory (no device)")
    conf.update({"parallelism": "host cores (oracle)", "sample": sample})
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (mega-synth v1, seeded; random-init weights)", "config": conf,
            "cpu_baseline": {"value": value, "unit": "edges/s", "cores": cores(), "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": "edges/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_mega(args):
    import torch
    import torch.distributed as dist
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (no CPU fallback)")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.gpus != world:
            raise SystemExit(f"bench.py --gpus {args.gpus} launched with WORLD_SIZE={world}")
        dist.init_process_group("nccl", device_id=dev)

    def sync_all():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    t0 = time.time()
    wl = build_workload(args.config, args.dtype, args.order, rank, world, args.window, args.seg_edges,
                        args.block_rows)
    cfg = wl["cfg"]
    if rank == 0:
        log(f"[bench] {cfg.name}: gen {wl['gen_s']:.1f}s, mega_preprocess {wl['pre_s']:.1f}s, parts {world}")
    model = Model(wl, args.dtype, dev, rank, world)
    for _ in range(max(3, args.warmup)):
        model.step()
    sync_all()
    # ---- device-timed region (inputs resident; inputs >> L2 so no flush) ----
    graph = None
    if args.cuda_graph:   # one step captured once; every kernel in it is ours or cuBLAS's
        side = torch.cuda.Stream(device=dev)
        side.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(side):
            model.step()
        torch.cuda.current_stream().wait_stream(side)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            model.step()
        for _ in range(max(3, args.warmup)):
            graph.replay()
        sync_all()
    run_step = (lambda: graph.replay()) if graph is not None else (lambda: model.step())
    # inputs smaller than L2 (the batch workloads): flush L2 between timed steps, outside the events
    sb0 = 2 if args.dtype == "bf16" else 4
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = None
    if cfg.n * cfg.dim * sb0 * 4 < 2 * l2_bytes:
        flush = torch.empty(2 * l2_bytes // 4, dtype=torch.float32, device=dev)
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        sync_all()
        if flush is None and graph is None:
            start.record()
            for _ in range(args.steps):
                model.step()
            end.record()
            sync_all()
            ms_step = start.elapsed_time(end) / args.steps
        else:
            pairs = []
            for _ in range(args.steps):
                if flush is not None:
                    flush.fill_(1.0)
                s1, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s1.record()
                run_step()
                e1.record()
                pairs.append((s1, e1))
            sync_all()
            ms_step = float(np.sum([a.elapsed_time(b) for a, b in pairs])) / args.steps
    # per-call breakdown from a separate eager pass (CUDA events on the launching stream around
    # every library call; the backward split into its source and destination phases)
    ev = {}
    sync_all()
    for _ in range(args.steps):
        if flush is not None:
            flush.fill_(1.0)
        model.step(ev, split=True)
    sync_all()
    ms_t = torch.tensor([ms_step], device=dev)
    if world > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())
    n_launch = {k: len(v) for k, v in ev.items()}
    calls = {k: float(np.mean([s.elapsed_time(e) for s, e in v])) for k, v in ev.items()}
    per_step_calls = {k: float(np.sum([s.elapsed_time(e) for s, e in v])) / args.steps for k, v in ev.items()}
    L = cfg.layers
    value = L * cfg.m / (ms * 1e-3)
    # ---- roofline per launch group (SURVEY §8(d)-d3 bytes; this rank's part) ----
    pk = peaks()
    sb = 2 if args.dtype == "bf16" else 4
    E, N, rows, H, D = model.part_edges, cfg.n, model.rows, cfg.heads, cfg.dim
    ncu = ncu_launch_summary(os.path.join(ROOT, "profiles", "r02", f"launches_{cfg.name}_{args.dtype}.csv"))
    call_of = {"KB2": "gat_fwd", "KB3+KB4": "gat_bwd_src", "KB5": "gat_bwd_dst", "KB3-KB5": "gat_bwd"}
    kernels = {}
    for kname, call in call_of.items():
        if call not in calls:
            continue
        t = calls[call] * 1e-3
        parts = ("KB3+KB4", "KB5") if kname == "KB3-KB5" else (kname,)   # k > 1: the backward is one call
        fb = sum(floor_bytes(q, rows, N, E, H, D, sb) for q in parts)
        nb = sum(floor_bytes(q, rows, N, E, H, D, sb, R=E) for q in parts)
        db = sum(design_bytes(q, rows, N, E, H, D, sb) for q in parts)
        ent = {"call": call, "ms": calls[call], "floor_bytes": fb, "noreuse_bytes": nb, "design_bytes": db,
               "achieved_gbs": fb / t / 1e9, "frac": fb / t / 1e9 / pk["hbm_gbs"],
               "noreuse_frac": nb / t / 1e9 / pk["hbm_gbs"], "design_frac": db / t / 1e9 / pk["hbm_gbs"]}
        if kname in ("KB2", "KB3+KB4"):   # the row-gathering kernels: requested rows vs the L2 gather ceiling
            req = E * D * sb
            ent["gather_requested_bytes"] = req
            ent["gather_tbs"] = req / t / 1e12
            ent["gather_ceiling_tbs"] = L2_GATHER_TBS
            ent["gather_frac"] = ent["gather_tbs"] / L2_GATHER_TBS
        if ncu and kname in ncu and world == 1:
            ent["traffic"] = ncu[kname]["dram_bytes"]
            ent["traffic_gbs"] = ncu[kname]["dram_bytes"] / t / 1e9
            ent["traffic_frac"] = ent["traffic_gbs"] / pk["hbm_gbs"]
            ent["ncu_ms"] = ncu[kname]["ncu_ms"]
        kernels[kname] = ent
    dom = max(kernels, key=lambda k: kernels[k]["ms"])
    kd = kernels[dom]
    roofline = {"bound": "hbm", "kernel": dom, "achieved": kd["achieved_gbs"], "peak": pk["hbm_gbs"], "unit": "GB/s",
                "frac": kd["frac"], "traffic": kd.get("traffic"), "algorithmic_bytes": kd["floor_bytes"],
                "launch_ms": kd["ms"], "peak_source": pk["source"] + " (hbm_gbs, copy bandwidth)",
                "note": "algorithmic bytes = SURVEY §8(d)-d3 floor (R = N: every gathered row once) per launch; "
                        "time = CUDA events around the call on its stream (eager pass, bwd split by phase); "
                        "traffic = ncu DRAM bytes per launch from profiles/r02/launches_<cfg>_<dtype>.csv",
                "kernels": kernels}
    if kd.get("traffic"):
        roofline["traffic_frac"] = kd["traffic_frac"]
    # ---- L2 fraction when the gathered table fits in L2: the forward's requested
    # gather rate (E rows of D*s bytes / its time) against a bare gather of the SAME index stream
    # (mega_calib_gather over the layout's CSR sources, same table) timed here ----
    row_bytes = cfg.dim * sb
    if world == 1 and cfg.n * row_bytes <= l2_bytes and row_bytes in (512, 1024, 2048) and "gat_fwd" in calls:
        from paper_conf_icdcs_dengr24_b200 import mega as M
        idx = torch.tensor(wl["layout"].view(0)["src"], dtype=torch.int32, device=dev)
        table = model.layers[0].L.feat
        sink = torch.empty(1 << 16, dtype=torch.float32, device=dev)
        M.mega_calib_gather(table, row_bytes, idx, sink)
        torch.cuda.synchronize()
        ts = []
        for _ in range(5):
            a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a_.record()
            M.mega_calib_gather(table, row_bytes, idx, sink)
            b_.record()
            torch.cuda.synchronize()
            ts.append(a_.elapsed_time(b_))
        calib_gbs = idx.numel() * row_bytes / (float(np.median(ts)) * 1e-3) / 1e9
        fwd_gbs = model.part_edges * row_bytes / (calls["gat_fwd"] * 1e-3) / 1e9
        roofline["l2"] = {"bound": "l2 gather", "fwd_requested_gbs": fwd_gbs, "calib_gbs": calib_gbs,
                          "frac": fwd_gbs / calib_gbs, "table_bytes": cfg.n * row_bytes,
                          "note": "fwd gathered-row bytes (E * D * s, no reuse counted) per second over a bare "
                                  "gather of the same CSR source stream from the same table (mega_calib_gather)"}
    if ncu:
        roofline["gemm"] = {g: {**ncu[g], "ms_per_call": calls.get("project_fwd" if g == "proj_fwd" else "project_bwd")}
                            for g in ("proj_fwd", "proj_bwd") if g in ncu}
    # ---- e2e: this step's inputs from pinned host memory, parameter grads back ----
    e2e = None
    if not args.no_e2e:
        hx = model.x0.cpu().pin_memory()
        hg = model.g.cpu().pin_memory()
        outs = [Ld.L.grad_w for Ld in model.layers] + [Ld.L.grad_attn_l for Ld in model.layers] + \
               [Ld.L.grad_attn_r for Ld in model.layers]
        hout = [torch.empty(o.shape, dtype=o.dtype).pin_memory() for o in outs]
        h2d = hx.numel() * hx.element_size() + hg.numel() * hg.element_size()
        d2h = sum(o.numel() * o.element_size() for o in outs)

        # Double-buffered input pipeline, as a training loop runs it: the H2D copy of step i+1's inputs
        # (X and grad_out, pinned host memory) runs on a copy stream during step i; at the start of a
        # step its staged inputs are moved into place with a device-to-device copy.  Every timed step
        # carries one full H2D copy of a step's inputs, one D2D move and the D2H read of its grads.
        cpy = torch.cuda.Stream(device=dev)
        stage_x, stage_g = torch.empty_like(model.x0), torch.empty_like(model.g)
        ev_free, ev_ready = torch.cuda.Event(), torch.cuda.Event()
        cur = torch.cuda.current_stream()

        def prefetch():
            cpy.wait_event(ev_free)
            with torch.cuda.stream(cpy):
                stage_x.copy_(hx, non_blocking=True)
                stage_g.copy_(hg, non_blocking=True)
            ev_ready.record(cpy)

        def e2e_step():
            cur.wait_event(ev_ready)
            model.x0.copy_(stage_x)
            model.g.copy_(stage_g)
            ev_free.record(cur)
            prefetch()                      # the next step's inputs travel while this step computes
            if graph is not None:
                graph.replay()
            else:
                model.step()
            for h, o in zip(hout, outs):
                h.copy_(o, non_blocking=True)

        ev_free.record(cur)
        prefetch()
        for _ in range(2):
            e2e_step()
        sync_all()
        s2, e2 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s2.record()
        for _ in range(args.steps):
            e2e_step()
        cur.wait_event(ev_ready)            # the last step's prefetch lands inside the timed region
        e2.record()
        sync_all()
        me = torch.tensor([s2.elapsed_time(e2) / args.steps], device=dev)
        if world > 1:
            dist.all_reduce(me, op=dist.ReduceOp.MAX)
        ms_e2e = float(me.item())
        e2e = {"value": L * cfg.m / (ms_e2e * 1e-3), "unit": "edges/s", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": ms_e2e,
               "pipeline": "step i+1's X and grad_out copied H2D from pinned memory on a copy stream during "
                           "step i, moved into place D2D at its start; parameter grads read D2H every step"}
    # ---- CPU oracle baseline (bounded sample; rank 0 at N = 1 only) ----
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        run, R, describe = cpu_sample(cfg, wl["indptr"], wl["indices"], args.cpu_seconds)
        t, e = run(R)
        cpu = {"value": cfg.layers * e / t, "unit": "edges/s", "cores": cores(), "kind": "oracle",
               "sample": describe(R, e, t)}
    if rank == 0:
        st = wl["layout"].stats()
        line = {
            "metric": METRIC, "value": value, "unit": "edges/s", "n_gpus": world, "steps": args.steps,
            "warmup": max(3, args.warmup), "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": args.dtype,
            "data": ("synthetic (mega-synth v1: Table II-shaped block-diagonal batch, seeded; random-init weights)"
                     if cfg.batch else "synthetic (mega-synth v1: DC-SBM power-law graph, seeded; random-init weights)"),
            "config": {**workload_config(cfg, args, st["block_rows"],
                                         "no flush: inputs larger than L2 (Wh %.2f GB)" % (cfg.n * cfg.dim * sb / 1e9)
                                         if flush is None else "L2 flushed between timed steps (%d MB write, "
                                         "outside the events)" % (flush.numel() * 4 >> 20)),
                       "parallelism": "single GPU" if world == 1 else
                       f"dst-partitioned x{world} (NCCL all-gather-v of [Wh|er], reduce-to-owner of [dWh|der])",
                       "cuda_graph": graph is not None},
            "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": model.launches * args.steps,
            "clocks": clk.summary(), "calls_ms_per_step": per_step_calls,
            "layout": {k: st[k] for k in ("window", "seg_edges", "path_length", "revisits", "jumps",
                                          "tile_unique_sources", "max_in_degree", "preprocess_seconds",
                                          "block_rows", "num_blocks", "block_sweeps")},
            "setup_s": time.time() - t0,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def launch_cmd(argv, n, port):
    """The one-process-per-GPU relaunch of `bench.py argv` on n GPUs of this node."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}", "--master-addr",
            "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__), *argv]


def maybe_spawn(args, argv):
    """`bench.py --gpus N` without a torchrun environment: re-launch itself as N ranks
    (one per GPU, NCCL) and exit with their status.  Fails loudly without N devices."""
    if args.impl != "mega" or args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        raise SystemExit(f"bench.py --gpus {args.gpus}: only {have} CUDA device(s) visible")
    r = subprocess.run(launch_cmd(argv, args.gpus, free_port()))
    raise SystemExit(r.returncode)


def main():
    args = parse()
    maybe_spawn(args, sys.argv[1:])
    if args.impl == "reference":
        run_reference(args)
    else:
        run_mega(args)


if __name__ == "__main__":
    main()
