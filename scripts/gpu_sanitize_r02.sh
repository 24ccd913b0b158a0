#!/bin/bash
# compute-sanitizer at HEAD on the new code paths (tcgen05 GEMMs, k-GPU loopback) and a parity subset.
O=gpurun_out/r02/sanitize
mkdir -p $O
export PYTHONPATH=$PWD
SEL_PROJ='tests/test_gpu_project.py -k "1000-100 or 777-512 or 300-128"'
SEL_DIST='tests/test_gpu_dist_loopback.py -k "random_multigraph or whole_layer_bf16"'
SEL_PAR='tests/test_gpu_parity.py -k "random_multigraph and 4-128 or edge_cases"'
for TOOL in memcheck racecheck synccheck initcheck; do
  for SEL in "$SEL_PROJ" "$SEL_DIST" "$SEL_PAR"; do
    NAME=$(echo "$SEL" | cut -d' ' -f1 | xargs basename .py)
    eval timeout 1200 compute-sanitizer --tool $TOOL --print-limit 10 python -m pytest -q -x $SEL \
      >> $O/${TOOL}.txt 2>&1
    echo "== $TOOL $NAME rc=$?" >> $O/${TOOL}.txt
  done
  grep -E "ERROR SUMMARY|== $TOOL|passed|failed" $O/${TOOL}.txt > $O/${TOOL}_summary.txt
done
