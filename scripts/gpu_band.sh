#!/bin/bash
# NEXT-2 band forward: GPU parity, then timing next to the exact-layout forward.
O=gpurun_out/band
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_band.py -q -x -m gpu 2>&1 | tail -15 > $O/pytest.log
timeout 1200 python scripts/bench_band.py > $O/bench_band.jsonl 2> $O/bench_band.err
