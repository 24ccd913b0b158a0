#!/bin/bash
# Order ablation at HEAD: same kernels, different node orders.
O=${OUT:-gpurun_out/r02/ablation}
mkdir -p $O
export PYTHONPATH=$PWD
for CFG in ${CFGS:-products reddit}; do
  for V in "traversal" "traversal:--block-rows,0" "identity:--block-rows,0" "degree:--block-rows,0" "random:--block-rows,0" "community"; do
    ORD=${V%%:*}; EXTRA=""; [ "$V" != "$ORD" ] && EXTRA=${V#*:}; EXTRA=${EXTRA//,/ }
    TAG=${CFG}_${ORD}$( [ -n "$EXTRA" ] && echo _noblock )
    timeout 900 python bench.py --config $CFG --order $ORD $EXTRA --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
      > $O/bench_$TAG.json 2> $O/bench_$TAG.err
    timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --print-units base \
      --clock-control none -k regex:"gat_fwd_pipe|gat_bwd_src_ring" -s 2 -c 2 --csv --log-file $O/ncu_$TAG.csv \
      python bench.py --config $CFG --order $ORD $EXTRA --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  done
done
