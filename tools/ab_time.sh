#!/bin/bash
# A/B timing of library variants on the GPU: bash tools/ab_time.sh OUT "variant1 variant2 ..." [cfgs]
# ("main" = the default library).  Each variant: cfg-5 full workload + other cfgs, schedule 0.
OUT=gpurun_out/$1; mkdir -p $OUT
CFGS=${3:-"5 4 3"}
for v in $2; do
  if [ "$v" = main ]; then vv=""; else vv=$v; fi
  echo "== $v" >> $OUT/ab.txt
  SIAC_LIB_VARIANT=$vv QT_FULL=1 QT_SCHED=${QT_SCHED:-0} timeout 600 python tools/quick_time.py $CFGS >> $OUT/ab.txt 2>&1
done
cat $OUT/ab.txt
