#!/bin/bash
# L2 block size B under the claimed schedule (products), then the launch lists at HEAD.
O=gpurun_out/blocks
mkdir -p $O
export PYTHONPATH=$PWD
for B in ${BS:-16384 26000 100000 200000}; do
  timeout 900 python bench.py --block-rows $B --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products_B$B.json 2> $O/bench_products_B$B.err
done
bash scripts/gpu_launches_r02.sh
