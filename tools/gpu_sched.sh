# scheduling-forecast ablation (results are bit-identical; only the integrator time changes)
for s in index persistence knn5 knn9 knn25 persistence; do
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --schedule $s > gpurun_out/sched.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/sched.json')); print('$s', round(d['ms_per_step'],2), 'ms/step', round(d['kernel_ms_per_step']['integrate_ms'],2), 'ms integrate')"
done
