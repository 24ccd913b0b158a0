#!/bin/bash
# One gpurun session: smoke, GPU tests, short bench, launch list.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv | tee gpurun_out/gpu.txt
python -c "import torch;print(torch.cuda.get_device_properties(0))" | tee -a gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -20 | tee gpurun_out/smoke.log
MEGA_DEBUG_SYNC=1 timeout 900 python -m pytest tests -x -q -m gpu ${PYTEST_ARGS} 2>&1 | tail -40 | tee gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
