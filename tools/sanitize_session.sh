#!/bin/bash
# compute-sanitizer session: memcheck, racecheck, synccheck, initcheck on
# configs 1-2 for the jump schedules (0 = default JUMPX, 4 = JUMP, 6 = ELEM), the direct
# schedules (1, 2, 3), the split-warp partial-sum path (active on these small configs) and
# CUDA-graph replay.  usage (via gpurun): bash tools/sanitize_session.sh TAG
TAG=${1:-san}
O=gpurun_out/$TAG
mkdir -p $O
CS=compute-sanitizer
run() {   # tool cfg schedules [graphs]
    local tool=$1 cfg=$2 sch=$3 g=$4
    local f=$O/${tool}_cfg${cfg}_s${sch//,/-}${g:+_graphs}.log
    timeout 1500 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_run.py $cfg $sch $g > $f 2>&1
    echo "exit $?" >> $f
    tail -n 3 $f | sed "s|^|$tool cfg$cfg s$sch $g: |"
}
run memcheck 1 0,4,5,6,1,2,3 graphs
run memcheck 2 0,4,6,2,3
run synccheck 1 0,4,6,3 graphs
run synccheck 2 0,4,6
run racecheck 1 0,4,6,3
run racecheck 2 0
run initcheck 1 0,4,6
ls -la $O
