# 2D A/B: main vs a variant ($1), 2 reps interleaved, then the variant's 2D parity tests
V=${1:-mb5}; O=gpurun_out/ab2d_$V; mkdir -p $O; rm -f $O/ab.txt
for rep in 1 2; do for v in main $V; do
  if [ $v = main ]; then vv=""; else vv=$v; fi
  echo "== $v rep $rep" >> $O/ab.txt
  SIAC_LIB_VARIANT=$vv QT_FULL=1 QT_SCHED=0 timeout 600 python tools/quick_time.py 5 4 3 >> $O/ab.txt 2>&1
done; done
SIAC_LIB_VARIANT=$V timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_$V.log 2>&1; echo "exit $?" >> $O/pytest_$V.log
grep -E '==|sched=0' $O/ab.txt; tail -2 $O/pytest_$V.log
