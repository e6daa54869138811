# r02 ncu evidence for config 5 (a full call takes ~55 s per replay pass): the roofline counters
# on rank 0's shard of an 8-way split (the same LPT-dealt points an 8-GPU rank integrates), and
# the DRAM bytes of one whole-mesh call (2 passes).
set -x
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__inst_executed_pipe_fp64.sum,smsp__inst_executed.sum,smsp__sass_average_branch_targets_threads_uniform.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,smsp__thread_inst_executed_per_inst_executed.ratio,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,launch__registers_per_thread
timeout 2400 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_cfg5.csv python tools/ncu_cfg.py 5 1 8 subregion > gpurun_out/ncu_cfg5.log 2>&1
tail -1 gpurun_out/ncu_cfg5.log | cut -c1-200
timeout 1500 ncu --profile-from-start off --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:k_integrate --csv --log-file gpurun_out/ncu_cfg5_dram.csv python tools/ncu_cfg.py 5 1 1 subregion > gpurun_out/ncu_cfg5_dram.log 2>&1
tail -1 gpurun_out/ncu_cfg5_dram.log | cut -c1-200
