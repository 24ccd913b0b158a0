#!/bin/bash
# Round-2 evidence at HEAD: launch lists (the bench roofline's traffic source) first, then the GPU
# suite and smoke, bench lines for every config, the reference arm, and full ncu captures.
O=gpurun_out/final
mkdir -p $O
export PYTHONPATH=$PWD
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/gpu.txt
git_head=$(cat .git_head 2>/dev/null); echo "$git_head" > $O/head.txt
for cfg in products reddit; do
  timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active \
    --clock-control none --print-units base -s ${SKIP:-60} -c ${COUNT:-40} --csv --log-file $O/launches_${cfg}_bf16.csv \
    python bench.py --config $cfg --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2> $O/launches_${cfg}.err
  mkdir -p profiles/r02 && cp $O/launches_${cfg}_bf16.csv profiles/r02/launches_${cfg}_bf16.csv
done
timeout 1800 python -m pytest tests -q -rf -m gpu 2>&1 | tail -15 > $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench_default.json 2> $O/bench_default.err
for C in reddit arxiv pubmed cora; do
  timeout 900 python bench.py --config $C --steps 10 --warmup 3 > $O/bench_$C.json 2> $O/bench_$C.err
done
timeout 900 python bench.py --config products --dtype fp32 --steps 5 --warmup 3 --no-cpu-baseline > $O/bench_products_fp32.json 2> $O/bench_products_fp32.err
for C in zinc-b64 zinc-b256 csl-b128 cycles-b128; do
  timeout 900 python bench.py --config $C --steps 20 --warmup 5 --cuda-graph --cpu-seconds 3 > $O/bench_$C.json 2> $O/bench_$C.err
done
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"gat_fwd_pipe|gat_bwd_src_ring|gat_bwd_dst" -s 3 -c 3 \
  -o $O/ncu_full_products python bench.py --config products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu_full.err
