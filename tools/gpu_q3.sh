O=gpurun_out/q3$1; mkdir -p $O; rm -f $O/ab.txt
for cfg in "8000 1" "8000 2"; do set -- $cfg
  timeout 600 python tools/bench3d.py $1 $2 3 2 $O/b_$2.json 0 > /dev/null 2>&1
  python -c "import json;d=json.load(open('$O/b_$2.json'));print('k=$2', round(d['ms_per_eval'],1), d['parity']['max_normwise'])" >> $O/ab.txt
done
cat $O/ab.txt
