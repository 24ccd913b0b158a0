#!/bin/bash
# last check at HEAD: GPU suite, smoke, default bench line, reddit, GT timing, launch lists.
O=gpurun_out/final2
mkdir -p $O
export PYTHONPATH=$PWD
cat .git_head > $O/head.txt 2>/dev/null
timeout 1800 python -m pytest tests -q -rf -m gpu 2>&1 | tail -15 > $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for cfg in products reddit; do
  timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
    --clock-control none --print-units base -s 60 -c 40 --csv --log-file $O/launches_${cfg}_bf16.csv \
    python bench.py --config $cfg --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/launches_${cfg}.err
  cp $O/launches_${cfg}_bf16.csv profiles/r02/launches_${cfg}_bf16.csv
done
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --config reddit > $O/bench_reddit.json 2> $O/bench_reddit.err
timeout 1200 python scripts/bench_gt.py > $O/bench_gt.jsonl 2> $O/bench_gt.err
