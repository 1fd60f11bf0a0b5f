#!/bin/bash
# Instruction-issue evidence for every decode configuration (SURVEY.md 8(d) issue roof):
# one ncu capture per (config, mode) with the instruction / pipe / stall / occupancy counters,
# exported to CSV and folded into profiles/r02_issue.json by scripts/ncu_issue_json.py.
#   gpurun -- 'bash scripts/issue_profile.sh'
set -x
R=gpurun_out/issue
mkdir -p $R
CFGS=${CFGS:-"for_b0 for_b1 for_b4 for_b8 for_b12 for_b16 dfor_d1_2^28 dfor_sorted_uniform dfor_near_sorted dfor_consecutive rfor_runs4 rfor_runs8 rfor_runs16 rfor_runs64"}
MET=smsp__inst_executed.sum,smsp__inst_executed_pipe_alu.sum,smsp__inst_executed_pipe_fma.sum,smsp__inst_executed_pipe_lsu.sum,smsp__inst_executed_pipe_uniform.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,sm__cycles_elapsed.avg.per_second
for c in $CFGS; do
  for m in sum global; do
    f=$R/${c//^/}_$m
    timeout 300 ncu --metrics $MET --section WarpStateStats --section Occupancy --clock-control none \
      -k regex:k_decode -s 2 -c 1 --csv --page raw --log-file $f.csv python scripts/profile_one.py "$c" $m > $f.log 2>&1
  done
done
python scripts/ncu_issue_json.py $R > $R/summary.log 2>&1
