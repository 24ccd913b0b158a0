#!/bin/bash
# row element offsets staged once per edge: parity, bench, launch list with instruction counts.
O=gpurun_out/r02j
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist_loopback.py tests/test_gpu_fullsize.py -q -x -m gpu -k "not schedule_variants" 2>&1 | tail -4 > $O/pytest.log
if grep -q failed $O/pytest.log; then exit 1; fi
for cfg in products reddit; do
  timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_$cfg.json 2> $O/bench_$cfg.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
  --clock-control none --print-units base -k regex:"gat_fwd_pipe|gat_bwd_src_ring" -s 3 -c 3 --csv --log-file $O/launches.csv \
  python bench.py --config products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
