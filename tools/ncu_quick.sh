#!/bin/bash
# Quick ncu counters of the k_eval launch for library variants on a cfg-5 subset:
# bash tools/ncu_quick.sh TAG "variants" [npts]
TAG=$1; VARS=$2; NP=${3:-2000000}
O=gpurun_out/$TAG; mkdir -p $O
M=gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed,sass__inst_executed_local_loads,sass__inst_executed_local_stores,sm__warps_active.avg.pct_of_peak_sustained_active,l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed,smsp__inst_executed_op_shared_ld.sum
for v in $VARS; do
  if [ "$v" = main ]; then vv=""; else vv=$v; fi
  SIAC_LIB_VARIANT=$vv timeout 600 ncu --metrics $M --clock-control none -k regex:k_eval -c 1 --csv python tools/profile_eval.py 5 $NP 1 > $O/ncu_$v.csv 2>&1
  echo "== $v"; grep -E '"(gpu__|smsp__|sm__|l1tex__|sass__)' $O/ncu_$v.csv | awk -F'","' '{print $(NF-2), $NF}' | tr -d '"'
done
