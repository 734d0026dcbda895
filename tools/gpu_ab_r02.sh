#!/bin/bash
# usage (via gpurun): bash tools/gpu_ab_r02.sh TAG "variants" [tests]
# A/B timing of library variants (tools/ab_time.sh: cfgs 5 4 3, schedule 0), then the bench
# line of the main library; with "tests" also the full GPU test suite first.
TAG=${1:-ab}; VARS=${2:-main}
O=gpurun_out/$TAG
mkdir -p $O
if [ "$3" = "tests" ]; then
  timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log
fi
bash tools/ab_time.sh $TAG "$VARS" "5 4 3" > /dev/null 2>&1
cat $O/ab.txt
timeout 1200 python bench.py --no-direct-count > $O/bench.json 2> $O/bench.err; echo "bench exit $?"
tail -c 600 $O/bench.json
