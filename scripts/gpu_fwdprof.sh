#!/bin/bash
# quick: GPU tests (parity subset), bench, and one ncu capture of the fwd kernel with SASS instruction mix
mkdir -p gpurun_out
MEGA_DEBUG_SYNC=1 timeout 900 python -m pytest tests -x -q -m gpu ${PYTEST_ARGS} 2>&1 | tail -25
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/bench.json'));print(d['ms_per_step'], d['value'], {k: round(v,2) for k,v in d['calls_ms_per_step'].items()})"
K=${KERNEL:-gat_fwd_kernel}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 -o gpurun_out/prof_q python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
echo "ncu rc=$?"
