#!/bin/bash
# Launch list (time + DRAM bytes per launch) of one bench step and full-set ncu
# summaries of selected kernels, summarised ON THE BOX (reports stay in /tmp).
# Never a bench value (runs under ncu).  Env: CFG, KERNELS, BARGS, TAG.
mkdir -p gpurun_out
CFG=${CFG:-products}; TAG=${TAG:-prof}
ARGS="--config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline $BARGS"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file /tmp/launches.csv python bench.py $ARGS > /dev/null 2> gpurun_out/${TAG}_launch.err
echo "launch list rc=$?"
python scripts/launch_summary.py /tmp/launches.csv gpurun_out/${TAG}_launches.json | head -30 | tee gpurun_out/${TAG}_launches.txt
python scripts/launch_traffic.py /tmp/launches.csv 4 3 gpurun_out/${TAG} > gpurun_out/${TAG}_traffic.txt 2>&1; head -30 gpurun_out/${TAG}_traffic.txt
cp /tmp/launches.csv gpurun_out/${TAG}_launches.csv
for K in ${KERNELS}; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$K -s ${SKIP:-3} -c 1 \
      -o /tmp/prof_$K python bench.py $ARGS > /dev/null 2>&1
  echo "== $K rc=$?" | tee -a gpurun_out/${TAG}_ncu.txt
  python scripts/ncu_summary.py /tmp/prof_$K.ncu-rep 2>&1 | tee -a gpurun_out/${TAG}_ncu.txt
  ncu -i /tmp/prof_$K.ncu-rep --page details --csv > gpurun_out/${TAG}_details_$K.csv 2>/dev/null
done
