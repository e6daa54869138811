# quick GPU check: parity tests (per-test timeout, durations), short bench
timeout 1500 python -m pytest tests -m gpu -q --timeout=400 --durations=12 > gpurun_out/pytest_gpu.log 2>&1; tail -22 gpurun_out/pytest_gpu.log
python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
python -c "
import json; d=json.load(open('gpurun_out/bench_quick.json')); print(d['ms_per_step'], d['roofline']['frac'], d['kernel_ms_per_step'])"
tail -3 gpurun_out/bench_quick.err
