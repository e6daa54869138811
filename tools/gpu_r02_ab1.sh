# r02: GPU tests + smoke on the new boundary, then the L1-prefetch A/B (variants/) on cfg5/cfg3/cfg2
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -5 gpurun_out/pytest_gpu.log
for v in base pf1 pf2; do
  timeout 600 python variants/$v/tools/ncu_cfg.py 5 0 8 subregion > gpurun_out/ab_c5_$v.json 2>&1; tail -1 gpurun_out/ab_c5_$v.json
  timeout 600 python variants/$v/bench.py --config 3 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ab_c3_$v.json 2>&1; tail -1 gpurun_out/ab_c3_$v.json | cut -c1-400
  timeout 600 python variants/$v/bench.py --config 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ab_c2_$v.json 2>&1; tail -1 gpurun_out/ab_c2_$v.json | cut -c1-400
done
