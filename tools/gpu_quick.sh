# quick GPU check: parity tests + a short bench (no profiler)
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
python bench.py --steps 3 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
python - <<'PY'
import json
d = json.load(open("gpurun_out/bench_quick.json"))
print("value", d["value"], "ms/step", d["ms_per_step"], "gflops", d["fp64_gflops"], "frac", d["roofline"]["frac"])
print("kernels", d["kernel_ms_per_step"])
print("work", d["work_per_step"], "clocks", d["clocks"], "e2e", d["e2e"] and d["e2e"]["ms_per_step"])
PY
tail -3 gpurun_out/bench_quick.err
