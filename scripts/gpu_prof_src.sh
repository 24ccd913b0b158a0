#!/bin/bash
# Full ncu capture (source-level) of the two gathering kernels of one products step.
O=gpurun_out/prof
mkdir -p $O
export PYTHONPATH=$PWD
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"${KRE:-gat_fwd_pipe|gat_bwd_src_ring|gat_bwd_dst}" -s ${S:-3} -c ${C:-3} \
  -o $O/ncu_full_${TAG:-head} python bench.py --config ${CFG:-products} --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_full.err
