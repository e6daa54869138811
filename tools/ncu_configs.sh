# r02 ncu evidence for every BASELINE config: one whole integrator call (rp_compute_potentials on
# the full mesh, after warm-up steps) of configs 1..5 with the roofline counters, plus a
# `--set full` capture with source of config 3.  Summarised by tools/ncu_config_summary.py.
set -x
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__inst_executed_pipe_fp64.sum,smsp__inst_executed.sum,smsp__sass_average_branch_targets_threads_uniform.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,smsp__thread_inst_executed_per_inst_executed.ratio,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,launch__registers_per_thread
for c in 1 2 3 4 5; do
  w=2; [ $c = 5 ] && w=1
  timeout 1800 ncu --profile-from-start off --clock-control none --metrics $M --csv --log-file gpurun_out/ncu_cfg$c.csv python tools/ncu_cfg.py $c $w 1 subregion > gpurun_out/ncu_cfg$c.log 2>&1
  tail -1 gpurun_out/ncu_cfg$c.log | cut -c1-200
done
timeout 1200 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:k_integrate -o gpurun_out/prof_cfg3 -f python tools/ncu_cfg.py 3 2 1 subregion > gpurun_out/ncu_full_cfg3.log 2>&1
tail -2 gpurun_out/ncu_full_cfg3.log
