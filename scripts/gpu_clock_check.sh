#!/bin/bash
O=gpurun_out/clock
mkdir -p $O
export PYTHONPATH=$PWD
timeout 600 python bench.py --config zinc-b64 --steps 20 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_zinc-b64.json 2> $O/bench_zinc.err
timeout 600 python bench.py --config reddit --steps 10 --warmup 3 > $O/bench_reddit.json 2> $O/bench_reddit.err
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err
