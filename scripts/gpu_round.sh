#!/bin/bash
# One gpurun session: smoke, GPU tests, bench variants.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -5 | tee gpurun_out/smoke.log
if [ -z "$SKIP_TESTS" ]; then
MEGA_DEBUG_SYNC=1 timeout 900 python -m pytest tests -x -q -m gpu ${PYTEST_ARGS} 2>&1 | tail -30 | tee gpurun_out/pytest_gpu.log
fi
timeout 900 python bench.py --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
for V in ${VARIANTS}; do   # e.g. VARIANTS="MEGA_L2_HOT_MB=0:--no-e2e ..."
  ENVS=${V%%:*}; ARGS=${V#*:}
  env $ENVS timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e ${ARGS//,/ } > gpurun_out/bench_var.json 2>/dev/null
  echo "VARIANT $V"; python -c "import json;d=json.load(open('gpurun_out/bench_var.json'));print(d['ms_per_step'], {k: round(v,2) for k,v in d['calls_ms_per_step'].items()})"
done
