#!/bin/bash
# Analysis: effective L2 capacity (uniform random 1 KB rows over W MB) and the bare gather of the products
# forward stream under grid-size / policy variants (ncu DRAM bytes per launch).
O=gpurun_out/l2
mkdir -p $O
export PYTHONPATH=$PWD
M=gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct
[ -x scripts/l2probe ] || nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/l2probe scripts/l2probe.cu
for pol in 0 1; do
  ./scripts/l2probe $pol 8 > $O/probe_p${pol}.txt 2>&1
  timeout 600 ncu --metrics $M --cache-control none --clock-control none --print-units base --csv \
    --log-file $O/probe_p${pol}_ncu.csv ./scripts/l2probe $pol 8 > /dev/null 2>&1
done
for v in "8 0" "1 0" "2 0" "8 1"; do
  set -- $v
  MEGA_CALIB_BPS=$1 MEGA_CALIB_POL=$2 timeout 900 ncu --metrics $M --cache-control none --clock-control none \
    --print-units base --csv --log-file $O/orders_b$1_p$2_ncu.csv python scripts/calib_orders.py products 1 \
    > $O/orders_b$1_p$2.txt 2>&1
done
