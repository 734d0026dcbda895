#!/bin/bash
# A/B timing of library variants plus their GPU parity suites:
# bash tools/ab_session.sh TAG "main v1 v2 ..." [cfgs]
TAG=$1; VARS=$2; CFGS=${3:-"5 4 3 2 1"}
O=gpurun_out/$TAG; mkdir -p $O
bash tools/ab_time.sh $TAG "$VARS" "$CFGS" > /dev/null 2>&1
for v in $VARS; do
  [ "$v" = main ] && continue
  SIAC_LIB_VARIANT=$v timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_$v.log 2>&1; echo "exit $?" >> $O/pytest_$v.log
done
