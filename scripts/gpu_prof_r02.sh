#!/bin/bash
# ncu evidence at HEAD (one GPU): per-launch time + DRAM bytes of one products step, and a full-set
# capture of the tcgen05 GEMMs and (optionally) the attention kernels.
O=gpurun_out/r02
export PYTHONPATH=$PWD
CFG=${CFG:-products}
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
  --clock-control none --print-units base -s ${SKIP:-60} -c ${COUNT:-40} --csv --log-file $O/launches_${CFG}_bf16.csv \
  python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/launches_${CFG}_bf16.err
if [ -n "$FULL_K" ]; then
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$FULL_K" -s ${FULL_S:-6} -c ${FULL_C:-3} \
    -o $O/ncu_full_${CFG} python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_full_${CFG}.err
fi
