#!/bin/bash
# Round 2, claimed chunk schedule: GPU suite, bench lines, Q sweep, launch lists and full ncu captures.
O=gpurun_out/r02b
mkdir -p $O
export PYTHONPATH=$PWD
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt
if [ -z "$SKIP_TESTS" ]; then
  timeout 1500 python -m pytest tests -q -rf -m gpu 2>&1 | tail -30 > $O/pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
fi
for cfg in products reddit; do
  timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 ${BENCH_ARGS} > $O/bench_$cfg.json 2> $O/bench_$cfg.err
done
for q in ${QS:-128 512}; do
  MEGA_SCHED_Q=$q MEGA_SCHED_QB=$q timeout 600 python bench.py --config products --steps 5 --warmup 3 --no-e2e \
    --no-cpu-baseline > $O/bench_products_q$q.json 2> $O/bench_products_q$q.err
done
MEGA_SCHED_DYN=0 MEGA_SCHED_Q=0 MEGA_SCHED_QB=0 MEGA_L2_POLICY=0 timeout 600 python bench.py --config reddit --steps 5 \
  --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_reddit_old.json 2> $O/bench_reddit_old.err
for cfg in products reddit; do
  timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
    --clock-control none --print-units base -s ${SKIP:-60} -c ${COUNT:-40} --csv --log-file $O/launches_${cfg}_bf16.csv \
    python bench.py --config $cfg --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/launches_${cfg}.err
done
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"gat_fwd_pipe|gat_bwd_src_ring" -s 2 -c 2 \
  -o $O/ncu_full_products python bench.py --config products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_full.err
