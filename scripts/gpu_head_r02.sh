#!/bin/bash
# final check at HEAD: GPU suite, smoke, default bench line.
O=gpurun_out/head
mkdir -p $O
export PYTHONPATH=$PWD
cat .git_head > $O/head.txt 2>/dev/null
timeout 1800 python -m pytest tests -q -rf -m gpu 2>&1 | tail -15 > $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --config reddit > $O/bench_reddit.json 2> $O/bench_reddit.err
