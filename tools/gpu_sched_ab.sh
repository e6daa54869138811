# schedule A/B on one build: persistence vs subregion-major (cfg2, cfg3), result bytes must match
set -x
for s in persistence subregion; do
  for c in 2 3; do
    timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --schedule $s > gpurun_out/sched_c${c}_$s.json 2>&1
    tail -1 gpurun_out/sched_c${c}_$s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$s', 'cfg$c', round(d['ms_per_step'],2), d['result_sha256'])"
  done
done
