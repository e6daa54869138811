# r02 round evidence on one B200: smoke, the GPU tests, the driver's bench command (config 5,
# 20 + 5 steps) and its reference arm, the FP64 peak clock record, an ncu launch list of a short
# config-5 bench.  Outputs under gpurun_out/.
set -x
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
bash tools/fp64_peak_clocks.sh
( time timeout 1800 python bench.py --impl reference --steps 20 --warmup 5 ) > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; cat gpurun_out/bench_ref.json | cut -c1-600; tail -3 gpurun_out/bench_ref.err
( time timeout 1800 python bench.py --gpus 1 --steps 20 --warmup 5 ) > gpurun_out/bench_cfg5.json 2> gpurun_out/bench_cfg5.err; cat gpurun_out/bench_cfg5.json; tail -3 gpurun_out/bench_cfg5.err
