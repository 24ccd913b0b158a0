#!/bin/bash
# Work-item segment size S (load balance of the static grid stride) on products and reddit, and with degree order.
O=gpurun_out/r02/seg
mkdir -p $O
export PYTHONPATH=$PWD
for CFG in ${CFGS:-products reddit}; do
  for S in ${SEGS:-512 256 128}; do
    timeout 900 python bench.py --config $CFG --seg-edges $S --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
      > $O/bench_${CFG}_s$S.json 2> $O/bench_${CFG}_s$S.err
  done
  timeout 900 python bench.py --config $CFG --order degree --block-rows 0 --seg-edges 256 --steps 5 --warmup 3 \
    --no-e2e --no-cpu-baseline > $O/bench_${CFG}_degree_s256.json 2> $O/bench_${CFG}_degree_s256.err
done
