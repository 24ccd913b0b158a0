#!/bin/bash
O=gpurun_out/zinc
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --print-units base -s 200 -c 120 --csv \
  --log-file $O/launches_zinc-b64.csv python bench.py --config zinc-b64 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
