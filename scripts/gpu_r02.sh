#!/bin/bash
# One gpurun session of round 2: projection GEMM tests first (short timeout), then the GPU suite, smoke, bench.
mkdir -p gpurun_out/r02
O=gpurun_out/r02
export PYTHONPATH=$PWD
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/gpu.txt
if [ -n "$FIRST" ]; then
  timeout ${FIRST_TIMEOUT:-300} python -m pytest $FIRST -q -rf 2>&1 | tail -40 > $O/first.log; echo "first rc=$?" >> $O/first.log
fi
if [ -z "$SKIP_SMOKE" ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
fi
if [ -z "$SKIP_TESTS" ]; then
  timeout ${TEST_TIMEOUT:-1500} python -m pytest tests -q -rf -m gpu ${PYTEST_ARGS} 2>&1 | tail -40 > $O/pytest_gpu.log
fi
if [ -z "$SKIP_BENCH" ]; then
  timeout 900 python bench.py --steps 10 --warmup 3 ${BENCH_ARGS} > $O/bench.json 2> $O/bench.err; echo "bench rc=$?" >> $O/bench.err
fi
if [ -n "$EXTRA" ]; then bash -c "$EXTRA" > $O/extra.log 2>&1; fi
