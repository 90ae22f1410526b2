cd $GRAFT_REPO_ROOT
./tools/microbench/l1_gather > gpurun_out/l1_gather.txt 2>&1
ncu --clock-control none --metrics l1tex__data_pipe_lsu_wavefronts_mem_lgds.sum,smsp__inst_executed_op_global_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,gpu__time_duration.sum,l1tex__data_pipe_tex_wavefronts.sum,l1tex__data_pipe_lsu_wavefronts.sum,smsp__inst_executed_op_texture.sum --csv ./tools/microbench/l1_gather > gpurun_out/l1_gather_ncu.csv 2>&1
