#!/bin/bash
# no-hint gathers; bwd ring (U, NBF) variants; parity subset first.
O=gpurun_out/r02d
mkdir -p $O
export PYTHONPATH=$PWD
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist_loopback.py -q -x -m gpu 2>&1 | tail -15 > $O/pytest.log
for r in ${RINGS:-0 1 2 3}; do
  MEGA_BWD_RING=$r timeout 600 python bench.py --config products --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    > $O/bench_products_ring$r.json 2> $O/bench_products_ring$r.err
done
for r in ${RRINGS:-0 1 3}; do
  MEGA_BWD_RING=$r timeout 600 python bench.py --config reddit --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
    > $O/bench_reddit_ring$r.json 2> $O/bench_reddit_ring$r.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
  --clock-control none --print-units base -k regex:"gat_|dlt" -s 16 -c 16 --csv --log-file $O/launches_products.csv \
  python bench.py --config products --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
