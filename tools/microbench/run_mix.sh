cd $GRAFT_REPO_ROOT
./tools/microbench/mix_pipes > gpurun_out/mix.txt 2>&1
ncu --clock-control none --metrics sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.per_cycle_active,smsp__inst_executed.sum --csv ./tools/microbench/mix_pipes > gpurun_out/mix_ncu.csv 2>&1
