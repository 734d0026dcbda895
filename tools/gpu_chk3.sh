# 3D: the device-check build (SIAC_DEVICE_CHECKS=1: queue / cell / split bounds asserted) through
# the 3D GPU tests, then the default build's 3D bench after dropping the outside side of
# support-end cuts.  (compute-sanitizer is not available on this pool.)
O=gpurun_out/chk3; mkdir -p $O
SIAC_LIB_VARIANT=chk timeout 1500 python -m pytest tests/test_gpu3d.py -x -q > $O/pytest3d_chk.log 2>&1; echo "exit $?" >> $O/pytest3d_chk.log
SIAC_LIB_VARIANT=chk timeout 600 python tools/sanitize_run3d.py > $O/run3d_chk.log 2>&1; echo "exit $?" >> $O/run3d_chk.log
timeout 900 python tools/bench3d.py 8000 1 3 16 $O/bench3d_k1.json 0 > $O/b1.log 2>&1
timeout 900 python tools/bench3d.py 8000 2 3 8 $O/bench3d_k2.json 0 > $O/b2.log 2>&1
timeout 900 python tools/bench3d.py 64000 1 3 8 $O/bench3d_k1_64k.json 0 > $O/b1b.log 2>&1
tail -3 $O/pytest3d_chk.log; cat $O/run3d_chk.log
for f in $O/bench3d_*.json; do python -c "import json;d=json.load(open('$f'));print('$f', round(d['ms_per_eval'],1), round(d['model_frac_of_fp64_peak'],4), d['parity']['max_normwise'], d['pieces'])"; done
