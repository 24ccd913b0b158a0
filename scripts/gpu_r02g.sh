#!/bin/bash
# small-graph schedule fix + band backward: tests, batch / arxiv / products bench lines, band bench.
O=gpurun_out/r02g
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_band.py -q -x -m gpu 2>&1 | tail -8 > $O/pytest_band.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "not schedule_variants" 2>&1 | tail -4 > $O/pytest_parity.log
for C in zinc-b64 zinc-b256 csl-b128; do
  timeout 900 python bench.py --config $C --steps 20 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_$C.json 2> $O/bench_$C.err
done
timeout 900 python bench.py --config arxiv --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_arxiv.json 2> $O/bench_arxiv.err
timeout 900 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products.json 2> $O/bench_products.err
timeout 1200 python scripts/bench_band.py > $O/bench_band.jsonl 2> $O/bench_band.err
