#!/bin/bash
# calibration + ncu evidence for the L2-blocked order (1 GPU)
mkdir -p gpurun_out
python scripts/calib.py --out gpurun_out/calib_gather.json > gpurun_out/calib.log 2>&1; echo "calib rc=$?"
cat gpurun_out/calib.log | grep -v Warn | tail -12
KERNELS="gat_fwd_kernel gat_bwd_src_kernel" bash scripts/gpu_evidence.sh
ls gpurun_out
