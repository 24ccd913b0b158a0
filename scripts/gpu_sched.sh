#!/bin/bash
# Work-schedule / L2-policy variants of the gathering kernels: parity subset under the default, then
# bench per variant and ncu DRAM bytes of the attention launches.
# Variant = "name DYN Q POL": MEGA_SCHED_DYN (claimed vs static chunks), MEGA_SCHED_Q(B) chunk quantum
# (0 = one item per chunk), MEGA_L2_POLICY (0 hot evict_last + cold evict_first, 1 all normal, 2 hot last + cold normal)
O=gpurun_out/sched
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist_loopback.py -q -x -m gpu 2>&1 | tail -5 > $O/pytest.log
VARS=${VARS:-"old:0:0:0 dyn:1:256:0 dynpol2:1:256:2 dynpol1:1:256:1 statq:0:256:2"}
for cfg in ${CFGS:-products}; do
  for v in $VARS; do
    IFS=: read name dyn q pol <<< "$v"
    MEGA_SCHED_DYN=$dyn MEGA_SCHED_Q=$q MEGA_SCHED_QB=$q MEGA_L2_POLICY=$pol timeout 600 python bench.py --config $cfg \
      --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_${cfg}_$name.json 2> $O/bench_${cfg}_$name.err
  done
done
for v in ${NCU_VARS:-old:0:0:0 dynpol2:1:256:2}; do
  IFS=: read name dyn q pol <<< "$v"
  MEGA_SCHED_DYN=$dyn MEGA_SCHED_Q=$q MEGA_SCHED_QB=$q MEGA_L2_POLICY=$pol timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct \
    --clock-control none --print-units base -k regex:"gat_" -s 12 -c 12 --csv --log-file $O/launches_products_$name.csv \
    python bench.py --config products --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_$name.err
done
