#!/bin/bash
# Final round-2 GPU session: full GPU test suite, smoke, bench (N=1), launch list, sanitizer on
# the 3D warp-tile kernel, 3D bench k = 1 / 2.
TAG=${1:-r02d}
O=gpurun_out/$TAG; mkdir -p $O
timeout 2700 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $O/pytest_gpu.log
tail -n 3 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke exit $?" >> $O/smoke.log
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench exit $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --no-direct-count --no-oneshot > $O/bench_ncu.log 2>&1
timeout 900 python tools/bench3d.py 8000 1 3 16 $O/bench3d_k1.json 1 > $O/b3d1.log 2>&1
timeout 900 python tools/bench3d.py 8000 2 3 8 $O/bench3d_k2.json 0 > $O/b3d2.log 2>&1
ls -la $O
