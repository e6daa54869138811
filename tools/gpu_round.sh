# Full round evidence: GPU tests, smoke, bench (default args), ncu launch list, ncu --set full of
# the integrator.  Outputs under gpurun_out/ (summaries are copied to profiles/ by hand).
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; cat gpurun_out/bench_ref.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_integrate -s 6 -c 2 -o gpurun_out/prof_integrate -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -2 gpurun_out/ncu_full.log
# multi-GPU projection from one GPU (shards of N = 1, 2, 4, 8 timed through the product call)
timeout 600 python tools/shard_balance.py 2 3 > gpurun_out/shard_cfg2.json 2>&1
timeout 900 python tools/shard_balance.py 4 2 > gpurun_out/shard_cfg4.json 2>&1
