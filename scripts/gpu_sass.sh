#!/bin/bash
# Per-SASS-instruction execution counts and stall samples of selected kernels
# (ncu source page), for instruction-budget work.  Never a bench value.
# Env: CFG, KERNELS, BARGS, TAG.
mkdir -p gpurun_out
CFG=${CFG:-products}; TAG=${TAG:-sass}
ARGS="--config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline $BARGS"
for K in ${KERNELS}; do
  timeout 900 ncu --section SourceCounters --section WarpStateStats --section SchedulerStats --section LaunchStats \
      --section Occupancy --section SpeedOfLight --clock-control none --import-source on -k regex:$K -s ${SKIP:-3} -c 1 \
      -o /tmp/sass_$K python bench.py $ARGS > /dev/null 2>&1
  echo "== $K rc=$?"
  ncu -i /tmp/sass_$K.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_src_$K.csv 2>/dev/null
  ncu -i /tmp/sass_$K.ncu-rep --page details --csv > gpurun_out/${TAG}_details_$K.csv 2>/dev/null
  python scripts/sass_hot.py gpurun_out/${TAG}_src_$K.csv 20
done
