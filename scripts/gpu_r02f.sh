#!/bin/bash
# Resident-B GEMMs: projection parity, whole-layer parity, A/B bench, GEMM launch list.
O=gpurun_out/r02f
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_project.py tests/test_gpu_parity.py -q -x -m gpu -k "project or whole_layer or lp_only" 2>&1 | tail -5 > $O/pytest.log
if grep -q failed $O/pytest.log; then exit 1; fi
for r in 1 0; do
  MEGA_GEMM_RESB=$r timeout 600 python bench.py --config products --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/bench_products_resb$r.json 2> $O/bench_products_resb$r.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed \
  --clock-control none --print-units base -k regex:"umma|dw_reduce" -s 8 -c 8 --csv --log-file $O/launches_gemm.csv \
  python bench.py --config products --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2> $O/ncu.err
