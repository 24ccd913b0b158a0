#!/bin/bash
# TMA-ring forward vs the pipe kernel; bf16 LP partial; parity subset first.
O=gpurun_out/r02c
mkdir -p $O
export PYTHONPATH=$PWD
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist_loopback.py tests/test_gpu_fullsize.py -q -x -m gpu 2>&1 | tail -15 > $O/pytest.log
for v in ${VARS:-"tma:1" "pipe:0"}; do
  IFS=: read name t <<< "$v"
  for cfg in products reddit; do
    MEGA_FWD_TMA=$t timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
      > $O/bench_${cfg}_$name.json 2> $O/bench_${cfg}_$name.err
  done
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
  --clock-control none --print-units base -k regex:"gat_" -s 12 -c 12 --csv --log-file $O/launches_products_tma.csv \
  python bench.py --config products --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_tma.err
