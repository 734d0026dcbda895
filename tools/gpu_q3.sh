O=gpurun_out/q3$1; mkdir -p $O; rm -f $O/ab.txt
timeout 1500 python -m pytest tests/test_gpu3d.py -x -q > $O/pytest3d.log 2>&1; echo "exit $?" >> $O/pytest3d.log; tail -2 $O/pytest3d.log >> $O/ab.txt
for cfg in "8000 1" "8000 2" "2000 3"; do set -- $cfg
  timeout 600 python tools/bench3d.py $1 $2 2 4 $O/b_$2.json 0 > /dev/null 2>&1
  python -c "import json;d=json.load(open('$O/b_$2.json'));print('k=$2', round(d['ms_per_eval'],1), round(d['model_frac_of_fp64_peak'],4), d['parity']['max_normwise'])" >> $O/ab.txt
done
cat $O/ab.txt
