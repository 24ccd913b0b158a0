#!/bin/bash
# bench lines for every BASELINE config (and an fp32 products line); L2-resident ones get the L2 fraction.
O=gpurun_out/r02/configs
mkdir -p $O
export PYTHONPATH=$PWD
for C in cora pubmed arxiv reddit products; do
  timeout 900 python bench.py --config $C --steps 10 --warmup 3 > $O/bench_$C.json 2> $O/bench_$C.err
done
timeout 900 python bench.py --config products --dtype fp32 --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_products_fp32.json 2> $O/bench_products_fp32.err
for C in zinc-b64 zinc-b256 csl-b128; do
  timeout 900 python bench.py --config $C --steps 20 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_$C.json 2> $O/bench_$C.err
done
