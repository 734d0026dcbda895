# 3D measurement refresh: bench (both mappings at k = 1, 2; default at 64K tets k = 1 and at k = 3),
# ncu full capture of the default kernel at k = 1 and k = 2.
O=gpurun_out/f3d; mkdir -p $O
timeout 900 python tools/bench3d.py 8000 1 3 16 $O/bench3d_k1.json 1 > $O/b1.log 2>&1
timeout 900 python tools/bench3d.py 8000 2 3 8 $O/bench3d_k2.json 1 > $O/b2.log 2>&1
timeout 900 python tools/bench3d.py 64000 1 3 8 $O/bench3d_k1_64k.json 0 > $O/b1b.log 2>&1
timeout 900 python tools/bench3d.py 2000 3 2 4 $O/bench3d_k3.json 0 > $O/b3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_eval3w -c 1 -o $O/k3w_k1 python tools/profile3d.py 8000 1 > $O/ncu1.log 2>&1
python tools/ncu_summary.py $O/k3w_k1.ncu-rep > $O/summary_k1.txt 2>&1
for f in $O/bench3d_*.json; do python -c "import json;d=json.load(open('$f'));t=d['thread_per_point'] or {};print('$f', round(d['ms_per_eval'],1), round(d['model_frac_of_fp64_peak'],4), d['parity']['max_normwise'], t.get('ms_per_eval'))"; done
