# 3D: shared work queue for the splitting -- tests, then timing (k = 1 at 3 / 4 blocks per SM, k = 2)
O=gpurun_out/wq3; mkdir -p $O; rm -f $O/ab.txt
timeout 1500 python -m pytest tests/test_gpu3d.py -x -q > $O/pytest3d.log 2>&1; echo "exit $?" >> $O/pytest3d.log
tail -3 $O/pytest3d.log
for mb in 4 3; do
  SIAC3_MINB=$mb timeout 600 python tools/bench3d.py 8000 1 3 8 $O/b_1_$mb.json 0 > /dev/null 2>&1
  python -c "import json;d=json.load(open('$O/b_1_$mb.json'));print('k=1 minb $mb', round(d['ms_per_eval'],1), d['parity']['max_normwise'], d['pieces'])" >> $O/ab.txt
done
timeout 600 python tools/bench3d.py 8000 2 3 8 $O/b_2.json 0 > /dev/null 2>&1
python -c "import json;d=json.load(open('$O/b_2.json'));print('k=2', round(d['ms_per_eval'],1), d['parity']['max_normwise'], d['pieces'])" >> $O/ab.txt
cat $O/ab.txt
