#!/bin/bash
# interleaved A/B of the L2 block size (auto = 0.4 L2 / row bytes vs 0.8)
O=gpurun_out/blocks_ab
mkdir -p $O
export PYTHONPATH=$PWD
for rep in 1 2; do
  for B in 51814 100000; do
    timeout 900 python bench.py --block-rows $B --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products_B${B}_r$rep.json 2> /dev/null
  done
  for B in 103628 207000; do
    timeout 900 python bench.py --config reddit --block-rows $B --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_reddit_B${B}_r$rep.json 2> /dev/null
  done
done
