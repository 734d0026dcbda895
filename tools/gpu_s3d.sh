# 3D warp-tile kernel after the centroid-check fix: tests + bench at k = 1, 2, 3 (both schedules where affordable)
O=gpurun_out/s3d; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu3d.py -x -q --durations=8 > $O/pytest3d.log 2>&1; echo "exit $?" >> $O/pytest3d.log
timeout 600 python tools/bench3d.py 8000 1 3 16 $O/bench3d_k1.json 1 > $O/b1.log 2>&1
timeout 600 python tools/bench3d.py 64000 1 3 8 $O/bench3d_k1_64k.json 0 > $O/b1b.log 2>&1
timeout 900 python tools/bench3d.py 8000 2 3 8 $O/bench3d_k2.json 1 > $O/b2.log 2>&1
timeout 900 python tools/bench3d.py 2000 3 2 4 $O/bench3d_k3.json 1 > $O/b3.log 2>&1
for f in $O/bench3d_*.json; do python -c "import json;d=json.load(open('$f'));t=d['thread_per_point'] or {};print('$f', round(d['ms_per_eval'],1), round(d['model_frac_of_fp64_peak'],4), d['parity']['max_normwise'], t.get('ms_per_eval'), t.get('same_counts'), t.get('max_rel_diff_vs_schedule0'))"; done
tail -14 $O/pytest3d.log
