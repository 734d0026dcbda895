# A/B on one box: 3D warp-tile kernel with / without dropping the outside side of support-end cuts
O=gpurun_out/ab3; mkdir -p $O
for rep in 1 2; do for v in main nodrop; do
  if [ $v = main ]; then vv=""; else vv=$v; fi
  for cfg in "8000 1" "8000 2"; do set -- $cfg
    SIAC_LIB_VARIANT=$vv timeout 600 python tools/bench3d.py $1 $2 3 2 $O/b_${v}_$2_$rep.json 0 > /dev/null 2>&1
    python -c "import json;d=json.load(open('$O/b_${v}_$2_$rep.json'));print('$v k=$2 rep $rep', round(d['ms_per_eval'],1))" >> $O/ab.txt
  done
done; done
cat $O/ab.txt
