#!/bin/bash
# Round-2 refresh at HEAD: the r02 session (parity tests, smoke, bench, launch list, full-launch
# ncu capture, survey-sized cfg-5 parity sample, 2-rank functional run) plus the NEXT-4 3D bench.
# usage (via gpurun): bash tools/gpu_session_r02b.sh TAG
TAG=${1:-r02b}
bash tools/gpu_session_r02.sh $TAG
O=gpurun_out/$TAG
timeout 900 python tools/bench3d.py 8000 1 5 16 $O/bench3d_k1.json > $O/bench3d.log 2>&1; echo "bench3d exit $?" >> $O/bench3d.log
