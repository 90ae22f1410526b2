set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
./tools/microbench/int_peaks | tee gpurun_out/int_peaks.json
ncu --clock-control none --metrics sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_fmalite.sum,sm__inst_executed.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed.avg.per_cycle_active,smsp__inst_executed.avg.per_cycle_active,sm__cycles_elapsed.avg.per_second --csv ./tools/microbench/int_peaks > gpurun_out/int_peaks_ncu.csv 2>&1
tail -5 gpurun_out/int_peaks_ncu.csv
