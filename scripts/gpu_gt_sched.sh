#!/bin/bash
O=gpurun_out/gt_sched
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_gt.py -q -x -m gpu 2>&1 | tail -3 > $O/pytest.log
timeout 1200 python scripts/bench_gt.py > $O/bench_gt.jsonl 2> $O/bench_gt.err
