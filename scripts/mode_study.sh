# ncu metrics for scripts/mode_study.py: every nest_kernel launch (warm + profiled per run).
mkdir -p gpurun_out/modes
M=sass__inst_executed_per_opcode,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,smsp__thread_inst_executed_per_inst_executed.ratio,smsp__sass_branch_targets.sum,smsp__sass_branch_targets_threads_divergent.sum,sm__sass_inst_executed_op_shared_ld.sum,sm__sass_inst_executed_op_shared_st.sum,smsp__warps_issue_stalled_barrier.sum,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,smsp__issue_active.avg.pct_of_peak_sustained_active
ncu --metrics $M --print-metric-instances details --clock-control none -k regex:nest_kernel --csv python scripts/mode_study.py > gpurun_out/modes/ncu.csv 2> gpurun_out/modes/ncu.err
python scripts/mode_study_table.py gpurun_out/modes/ncu.csv > gpurun_out/modes/table.md
