#!/bin/bash
# Pipelined source pass: full GPU suite, smoke, bench lines, launch list.
O=gpurun_out/r02e
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "random_multigraph or edge_cases or whole_layer" 2>&1 | tail -5 > $O/pytest_quick.log
if grep -q failed $O/pytest_quick.log; then exit 1; fi
timeout 600 python bench.py --config products --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products.json 2> $O/bench_products.err
timeout 600 python bench.py --config reddit --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_reddit.json 2> $O/bench_reddit.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
  --clock-control none --print-units base -k regex:"gat_|dlt" -s 16 -c 8 --csv --log-file $O/launches_products.csv \
  python bench.py --config products --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
timeout 1800 python -m pytest tests -q -rf -m gpu 2>&1 | tail -15 > $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
