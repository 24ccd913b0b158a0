#!/bin/bash
# interleaved A/B of the chunk quantum (MEGA_SCHED_Q / QB)
O=gpurun_out/q_ab
mkdir -p $O
export PYTHONPATH=$PWD
for rep in 1 2; do
  for q in 256 128 512; do
    MEGA_SCHED_Q=$q MEGA_SCHED_QB=$q timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products_q${q}_r$rep.json 2> /dev/null
  done
done
