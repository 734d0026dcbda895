#!/bin/bash
# Round-2 GPU session: parity tests, smoke, bench (N=1), launch list, one ncu --set full capture
# of the FULL config-5 k_eval launch (the bench's own launch), the survey-sized cfg-5 parity
# sample, and the 2-rank functional run of the N>1 path.
# usage (via gpurun): bash tools/gpu_session_r02.sh TAG [skip_tests]
TAG=${1:-r02}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
if [ "$2" != "skip_tests" ]; then
  timeout 2400 python -m pytest tests -m gpu -x -q -s > $O/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $O/pytest_gpu.log
  tail -n 3 $O/pytest_gpu.log
fi
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke exit $?" >> $O/smoke.log
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench exit $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --no-direct-count --no-oneshot > $O/bench_ncu.log 2>&1
NP=12594264
timeout 1500 ncu --set full --metrics smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum --clock-control none --import-source on -k regex:k_eval -c 1 -o $O/k_eval_full python tools/profile_eval.py 5 $NP 1 > $O/ncu_full.log 2>&1
python tools/ncu_summary.py $O/k_eval_full.ncu-rep > $O/ncu_summary.txt 2>&1
python tools/ncu_traffic.py $O/k_eval_full.ncu-rep $NP "ncu --set full, tools/profile_eval.py 5 $NP 1 (the whole config-5 launch)" $O/ncu_traffic_cfg5.json > /dev/null 2>&1
timeout 900 python tools/parity_cfg5.py sinsin $O/parity_cfg5_sinsin.json > $O/parity_cfg5.log 2>&1; echo "parity exit $?" >> $O/parity_cfg5.log
SIAC_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 2 --warmup 3 --config 4 --e2e-steps 1 > $O/bench_2rank_gloo_cfg4.json 2> $O/bench_2rank.err
ls -la $O
