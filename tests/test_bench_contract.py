"""bench.py contract: the reference arm (the CPU oracle) prints one
JSON line with the driver's keys, on a small config; the GPU arm's line is checked on
the B200 (marked gpu)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config"}


def _run(args, timeout):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--config", "pubmed", "--steps", "2", "--warmup", "1"], 600)
    assert KEYS <= set(d) and d["impl"] == "reference"
    assert d["value"] > 0 and d["unit"] == "edges/s" and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


@pytest.mark.gpu
def test_gpu_arm_line():
    d = _run(["--config", "pubmed", "--steps", "3", "--warmup", "3", "--cpu-seconds", "2"], 900)
    assert KEYS <= set(d)
    assert d["gpu_launches"] > 0 and d["value"] > 0
    r = d["roofline"]
    assert r["bound"] == "hbm" and 0 < r["frac"] and r["peak"] > 0 and r["achieved"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])


def test_reference_arm_runs_no_product_code():
    """The reference arm is the oracle alone: it must not import the package or load libmega.so."""
    code = ("import sys, json; sys.argv = ['bench.py', '--impl', 'reference', '--config', 'cora', '--steps', '1', "
            "'--warmup', '0']; import bench; bench.main(); "
            "maps = open('/proc/self/maps').read(); "
            "print(json.dumps({'pkg': any(m.startswith('paper_conf_icdcs_dengr24_b200') for m in sys.modules), "
            "'so': 'libmega.so' in maps}))")
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    res = json.loads(r.stdout.strip().splitlines()[-1])
    assert res == {"pkg": False, "so": False}


def test_reference_arm_batch_config():
    d = _run(["--impl", "reference", "--config", "aqsol-b128-drop20", "--steps", "2", "--warmup", "1"], 600)
    assert KEYS <= set(d) and d["impl"] == "reference" and d["value"] > 0
    assert "aqsol-b128-drop20" in d["config"]["workload"]


@pytest.mark.gpu
def test_gpu_arm_batch_cuda_graph():
    d = _run(["--config", "zinc-b64", "--steps", "5", "--warmup", "3", "--cuda-graph", "--cpu-seconds", "1"], 900)
    assert KEYS <= set(d) and d["value"] > 0 and d["gpu_launches"] > 0
    c = d["config"]
    assert c["cuda_graph"] is True and c["batch"] == "zinc" and c["num_graphs"] == 64
    assert c["l2"].startswith("L2 flushed")


def test_gpus_n_relaunches_as_n_ranks(monkeypatch):
    """--gpus N outside torchrun re-launches bench.py as N ranks (one per GPU), and
    refuses loudly when fewer than N devices are visible."""
    import bench
    cmd = bench.launch_cmd(["--gpus", "2", "--steps", "3"], 2, 29999)
    assert cmd[1:3] == ["-m", "torch.distributed.run"] and "--nproc-per-node=2" in cmd
    assert cmd[-4:] == [os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3"][-4:]
    assert "127.0.0.1" in cmd
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    import torch
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 1)
    import argparse
    ns = argparse.Namespace(impl="mega", gpus=2)
    with pytest.raises(SystemExit) as e:
        bench.maybe_spawn(ns, ["--gpus", "2"])
    assert "only 1 CUDA device" in str(e.value)
    calls = []
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 2)
    monkeypatch.setattr(bench.subprocess, "run", lambda c: calls.append(c) or type("R", (), {"returncode": 0})())
    with pytest.raises(SystemExit) as e:
        bench.maybe_spawn(ns, ["--gpus", "2"])
    assert e.value.code == 0 and "--nproc-per-node=2" in calls[0]
