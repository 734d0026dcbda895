#!/bin/bash
# One GPU session: parity tests, bench, launch list, one full ncu capture of the top kernel.
# usage (via gpurun): bash tools/gpu_session.sh TAG [NCU_POINTS]
TAG=${1:-run}
NPTS=${2:-200000}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke exit $?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --no-direct-count > $O/bench_ncu.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_eval -c 1 -o $O/k_eval_full python tools/profile_eval.py 5 $NPTS 1 > $O/ncu_full.log 2>&1
ls -la $O
# multi-rank functional check of the N>1 bench path (2 ranks on one GPU, gloo) and context lines
SIAC_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 2 --warmup 3 --config 4 --e2e-steps 1 --no-cpu-baseline > $O/bench_2rank_gloo_cfg4.json 2> $O/bench_2rank.err
timeout 900 python bench.py --schedule 6 --steps 3 --no-cpu-baseline --no-direct-count > $O/bench_elem.json 2> $O/bench_elem.err
ls -la $O
