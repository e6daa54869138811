# development A/B of build variants (tools/variant.sh): cfg5 8-way shard integrator time, cfg3 and
# cfg2 bench lines (result_sha256 must match across variants: bit-identical results)
#   bash tools/gpu_ab.sh base tp ...
set -x
for v in "$@"; do
  timeout 600 python variants/$v/tools/ncu_cfg.py 5 0 8 subregion > gpurun_out/ab_c5_$v.json 2>&1; tail -1 gpurun_out/ab_c5_$v.json | cut -c1-200
  timeout 600 python variants/$v/bench.py --config 3 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ab_c3_$v.json 2>&1
  timeout 600 python variants/$v/bench.py --config 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ab_c2_$v.json 2>&1
done
python - "$@" <<'PY'
import json, sys
for v in sys.argv[1:]:
    try:
        d = json.loads(open(f"gpurun_out/ab_c5_{v}.json").read().strip().splitlines()[-1])
        ev = d["info"]["evals"] - d["info"]["skipped"]
        print(v, "cfg5/8", round(d["integrate_ms"], 1), "ms", round(1e9 * d["integrate_ms"] / ev, 3), "ps/eval")
    except Exception as e:
        print(v, 5, "ERR", e)
    for c in (3, 2):
        try:
            d = json.loads(open(f"gpurun_out/ab_c{c}_{v}.json").read().strip().splitlines()[-1])
            w = d["work_per_step"]
            ms = d["kernel_ms_per_step"]["integrate_ms"]
            print(v, f"cfg{c}", round(d["ms_per_step"], 2), "ms", "frac", round(d["roofline"]["frac"], 4),
                  round(1e9 * ms / (w["evals"] - w["skipped"]), 3), "ps/eval", d["result_sha256"])
        except Exception as e:
            print(v, c, "ERR", e)
PY
