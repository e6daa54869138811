# FP64 DFMA/DMMA peak microbenchmark (tools/mix_peak.cu) repeated for ~10 s with nvidia-smi
# sampling the SM clock and throttle reasons during the runs -> gpurun_out/r02_fp64_peak_clocks.json
set -e
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mix_peak tools/mix_peak.cu
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active,power.draw --format=csv,noheader,nounits -lms 50 > /tmp/clk.csv &
SMI=$!
/tmp/mix_peak 1500 > /tmp/mix.jsonl
kill $SMI
python - <<'PY'
import json, statistics
runs = [json.loads(l) for l in open("/tmp/mix.jsonl") if l.startswith("{")]
dfma = [r["dfma_tf"] for r in runs if r["dmma_per_iter"] == 0]
dmma = [r["dmma_tf"] for r in runs if r["dfma_rounds"] == 0]
clk = []
for l in open("/tmp/clk.csv"):
    p = [x.strip() for x in l.split(",")]
    try:
        clk.append((float(p[0]), float(p[1]), p[2], float(p[3])))
    except Exception:
        pass
busy = [c for c in clk if c[3] > 250]  # samples under load (idle ~ 140 W)
out = {"tool": "tools/mix_peak.cu 1500 (8 interleaved DFMA chains / 8 DMMA per iteration, 148 SMs; the pure DFMA and DMMA runs repeated 1500 times, ~8 s of load)",
       "dfma_tf_median": statistics.median(dfma), "dfma_tf_max": max(dfma),
       "dmma_tf_median": statistics.median(dmma), "dmma_tf_max": max(dmma),
       "clock_samples_under_load": len(busy),
       "sm_mhz_median_under_load": statistics.median([c[0] for c in busy]) if busy else None,
       "sm_max_mhz": max(c[1] for c in clk) if clk else None,
       "event_reasons_under_load": sorted({c[2] for c in busy}),
       "power_w_max": max(c[3] for c in clk) if clk else None}
json.dump(out, open("gpurun_out/r02_fp64_peak_clocks.json", "w"), indent=1)
print(json.dumps(out))
PY
