#!/bin/bash
# Locality / L2-policy sweep on products (same kernels): L2 block size B and the gathered-row cache hints.
O=gpurun_out/r02/sweep
mkdir -p $O
export PYTHONPATH=$PWD
CFG=${CFG:-products}
for BR in ${BRS:-8192 16384 32768}; do
  timeout 900 python bench.py --config $CFG --block-rows $BR --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    > $O/bench_${CFG}_br$BR.json 2> $O/bench_${CFG}_br$BR.err
done
for V in ${VARS:-"MEGA_L2_POLICY=1" "MEGA_L2_POLICY=2" "MEGA_L2_HOT_MB=0" "MEGA_L2_HOT_MB=24" "MEGA_L2_HOT_MB=96"}; do
  env $V timeout 900 python bench.py --config $CFG --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    > $O/bench_${CFG}_${V}.json 2> $O/bench_${CFG}_${V}.err
done
