#!/bin/bash
O=gpurun_out/q_ab2
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -q -x -m gpu -k "not schedule_variants" 2>&1 | tail -3 > $O/pytest.log
for rep in 1 2; do
  for q in 128 64; do
    MEGA_SCHED_Q=$q MEGA_SCHED_QB=$q timeout 900 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products_q${q}_r$rep.json 2> /dev/null
  done
done
timeout 900 python bench.py --config reddit --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_reddit_q128.json 2> /dev/null
