#!/bin/bash
# Batch workloads (NEXT-4) on one B200: parity, bench lines (eager and CUDA graph), launch list.
set -u
O=gpurun_out/batch
mkdir -p $O
timeout 600 python -m pytest tests/test_batch_workload.py "tests/test_gpu_parity.py::test_whole_layer" -m gpu -q \
  > $O/pytest_batch.log 2>&1; echo "PYTEST_RC=$?" >> $O/pytest_batch.log
for c in zinc-b64 zinc-b128 zinc-b256 aqsol-b128 aqsol-b128-drop20 csl-b128 cycles-b128; do
  timeout 240 python bench.py --config $c --steps 50 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_${c}_graph.json 2> $O/bench_${c}_graph.err
done
for c in zinc-b64 zinc-b256; do
  timeout 240 python bench.py --config $c --steps 50 --warmup 5 --cpu-seconds 3 > $O/bench_${c}_eager.json 2> $O/bench_${c}_eager.err
done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file $O/launches_zinc-b64.csv python bench.py --config zinc-b64 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e \
  > $O/ncu_run.log 2>&1
tail -2 $O/pytest_batch.log
for f in $O/bench_*.json; do echo "$f"; head -c 400 "$f"; echo; done
