#!/bin/bash
# Evidence for profiles/: launch list (gpu__time_duration) and per-kernel DRAM bytes of one bench step,
# plus full-set captures of the top attention kernels.  Never a bench value (runs under ncu).
mkdir -p gpurun_out
CFG=${CFG:-products}
ARGS="--config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${CFG}.csv python bench.py $ARGS > /dev/null 2> gpurun_out/ncu_launch.err
echo "launch list rc=$?"
for K in ${KERNELS:-gat_fwd_kernel gat_bwd_src_kernel gat_bwd_dst_kernel}; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s ${SKIP:-3} -c 1 \
      -o gpurun_out/prof_${CFG}_$K python bench.py $ARGS > /dev/null 2>&1
  echo "$K rc=$?"
done
