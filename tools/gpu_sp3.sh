# 3D small problem (8K tets, 1,121 point tiles): tile split 1 / 2 / 4 at k = 1 and 2
O=gpurun_out/sp3; mkdir -p $O; rm -f $O/ab.txt
for k in 1 2; do for sp in 1 2 4; do
  SIAC3_SPLIT=$sp timeout 600 python tools/bench3d.py 8000 $k 2 4 $O/b_${k}_$sp.json 0 > /dev/null 2>&1
  python -c "import json;d=json.load(open('$O/b_${k}_$sp.json'));print('k=$k split $sp', round(d['ms_per_eval'],1), d['parity']['max_normwise'])" >> $O/ab.txt
done; done
cat $O/ab.txt
