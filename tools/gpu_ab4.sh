# development A/B of build variants on the full configs 4, 3, 2 (bench.py; result_sha256 equal
# unless the variant changes values): bash tools/gpu_ab4.sh base v1 ...
for v in "$@"; do
  for c in 4 3 2; do
    timeout 900 python variants/$v/bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ab4_c${c}_$v.json 2>&1
  done
done
python - "$@" <<'PY'
import json, sys
for v in sys.argv[1:]:
    for c in (4, 3, 2):
        try:
            d = json.loads(open(f"gpurun_out/ab4_c{c}_{v}.json").read().strip().splitlines()[-1])
            w = d["work_per_step"]
            ms = d["kernel_ms_per_step"]["integrate_ms"]
            print(v, f"cfg{c}", round(d["ms_per_step"], 2), "ms", "frac", round(d["roofline"]["frac"], 4),
                  round(1e9 * ms / (w["evals"] - w["skipped"]), 3), "ps/eval", d["result_sha256"])
        except Exception as e:
            print(v, c, "ERR", e)
PY
