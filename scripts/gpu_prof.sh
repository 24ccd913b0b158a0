#!/bin/bash
# ncu launch list + full-set captures of the attention kernels (1 GPU).
set -x
mkdir -p gpurun_out
CFG=${CFG:-products}
ARGS="--config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${CFG}.csv python bench.py $ARGS > gpurun_out/ncu_launch_bench.json 2> gpurun_out/ncu_launch.err
tail -2 gpurun_out/ncu_launch.err
for K in ${KERNELS:-gat_fwd_kernel gat_bwd_src_kernel gat_bwd_dst_kernel}; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s ${SKIP:-3} -c 1 -o gpurun_out/prof_${CFG}_$K python bench.py $ARGS > /dev/null 2> gpurun_out/prof_$K.err
  tail -2 gpurun_out/prof_$K.err
done
ls -la gpurun_out
