# 2D A/B: main vs cut2 (x2 interleaved), then cut2's 2D parity tests
O=gpurun_out/ab2d; mkdir -p $O; rm -f $O/ab.txt
for rep in 1 2; do for v in main cut2; do
  if [ $v = main ]; then vv=""; else vv=$v; fi
  echo "== $v rep $rep" >> $O/ab.txt
  SIAC_LIB_VARIANT=$vv QT_FULL=1 QT_SCHED=0 timeout 600 python tools/quick_time.py 5 4 3 >> $O/ab.txt 2>&1
done; done
SIAC_LIB_VARIANT=cut2 timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_cut2.log 2>&1; echo "exit $?" >> $O/pytest_cut2.log
cat $O/ab.txt; tail -3 $O/pytest_cut2.log
