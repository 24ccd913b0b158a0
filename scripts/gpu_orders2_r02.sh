#!/bin/bash
O=gpurun_out/r02/ablation
mkdir -p $O
export PYTHONPATH=$PWD
for CFG in products reddit; do
  timeout 900 python bench.py --config $CFG --order comdeg --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    > $O/bench_${CFG}_comdeg.json 2> $O/bench_${CFG}_comdeg.err
done
