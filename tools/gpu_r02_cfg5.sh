# r02: cfg5 baseline (persistence vs subregion-major schedule) + targeted ncu of one integrator
# call on an 8-way shard of cfg5 (DRAM traffic, FP64 pipe, branch uniformity, sectors/request)
set -x
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__average_branch_targets_threads_uniform.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,smsp__thread_inst_executed_per_inst_executed.ratio,sm__warps_active.avg.pct_of_peak_sustained_active,l1tex__t_sector_hit_rate.pct
python bench.py --config 5 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/c5_pers.json 2> gpurun_out/c5_pers.err; cat gpurun_out/c5_pers.json
python bench.py --config 5 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --schedule subregion > gpurun_out/c5_sub.json 2> gpurun_out/c5_sub.err; cat gpurun_out/c5_sub.json
for s in persistence subregion; do
timeout 1200 ncu --profile-from-start off --clock-control none --metrics $M -k regex:k_integrate --csv --log-file gpurun_out/ncu_c5_$s.csv python tools/ncu_cfg.py 5 1 8 $s > gpurun_out/ncu_c5_$s.log 2>&1
tail -2 gpurun_out/ncu_c5_$s.log
done
