#!/bin/bash
# unsplit dW threshold for the batch regime: projection parity, zinc / csl lines at thresholds 8 and 32.
O=gpurun_out/r02i
mkdir -p $O
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests/test_gpu_project.py tests/test_gpu_parity.py -q -x -m gpu -k "project or whole_layer" 2>&1 | tail -3 > $O/pytest.log
for kb in 8 32 128; do
  for C in zinc-b64 zinc-b256 csl-b128; do
    MEGA_DW_UNSPLIT_KB=$kb timeout 900 python bench.py --config $C --steps 20 --warmup 5 --cuda-graph --no-e2e --no-cpu-baseline > $O/bench_${C}_kb$kb.json 2> $O/bench_${C}_kb$kb.err
  done
done
