#!/bin/bash
O=gpurun_out/r02k
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "random_multigraph or whole_layer or edge_cases" 2>&1 | tail -3 > $O/pytest.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products.json 2> $O/bench_products.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
  --clock-control none --print-units base -k regex:"gat_bwd_dst" -s 1 -c 2 --csv --log-file $O/launches_dst.csv \
  python bench.py --config products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
