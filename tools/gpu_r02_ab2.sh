set -x
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -8 gpurun_out/pytest_gpu.log
for v in base pf1 pf2; do
  timeout 600 python variants/$v/tools/ncu_cfg.py 5 0 8 subregion > gpurun_out/ab_c5_$v.json 2>&1; tail -1 gpurun_out/ab_c5_$v.json | cut -c1-300
done
python bench.py --config 2 --steps 3 --warmup 3 > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; cat gpurun_out/bench_c2.json; tail -3 gpurun_out/bench_c2.err
