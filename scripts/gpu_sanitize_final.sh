#!/bin/bash
# compute-sanitizer on this session's new code: the claimed chunk schedule and bf16 partial (parity
# subset on a graph with > kChunkMinItems items would be too slow; the schedule-variant test runs the
# static paths), the band forward / backward, and the loopback k-GPU path.
O=gpurun_out/sanitize_final
mkdir -p $O
export PYTHONPATH=$PWD
SEL_BAND='tests/test_gpu_band.py -k "window and 1 and fp32-4-32 or bf16-4-64 or batch"'
SEL_PAR='tests/test_gpu_parity.py -k "random_multigraph and 4-128 or edge_cases or lp_only"'
SEL_DIST='tests/test_gpu_dist_loopback.py -k "random_multigraph"'
for TOOL in memcheck racecheck synccheck; do
  for SEL in "$SEL_BAND" "$SEL_PAR" "$SEL_DIST"; do
    NAME=$(echo "$SEL" | cut -d' ' -f1 | xargs basename .py)
    eval timeout 900 compute-sanitizer --tool $TOOL --print-limit 10 python -m pytest -q -x -m gpu $SEL \
      >> $O/${TOOL}.txt 2>&1
    echo "== $TOOL $NAME rc=$?" >> $O/${TOOL}.txt
  done
  grep -E "ERROR SUMMARY|== $TOOL|passed|failed" $O/${TOOL}.txt > $O/${TOOL}_summary.txt
done
