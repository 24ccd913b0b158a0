#!/bin/bash
# GT parity, full GPU suite, batch + products bench after the one-launch param reduce.
set -u
O=gpurun_out/r01c
mkdir -p $O
timeout 300 python -m pytest tests/test_gpu_gt.py -m gpu -q > $O/pytest_gt.log 2>&1; echo "PYTEST_RC=$?" >> $O/pytest_gt.log
timeout 600 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "PYTEST_RC=$?" >> $O/pytest_gpu.log
for c in zinc-b64 zinc-b256 csl-b128; do
  timeout 200 python bench.py --config $c --steps 50 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_${c}_graph.json 2> $O/bench_${c}_graph.err
done
timeout 400 python bench.py > $O/bench_products.json 2> $O/bench_products.err
tail -3 $O/pytest_gt.log $O/pytest_gpu.log
for f in $O/bench_*.json; do echo "$f"; head -c 300 "$f"; echo; done
