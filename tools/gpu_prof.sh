# ncu --set full of the integrator (one launch after warm-up) + launch list
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_integrate -s 2 -c 1 -o gpurun_out/prof_integrate -f python bench.py --steps 1 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
