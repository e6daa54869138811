# Predictive-RP ablation on config 2 (one B200): merged clusters (m = max(nx, ny)) and
# per-point partitions (m = nx*ny, the forecast-as-initial-partition alone)
timeout 300 python tools/predictive_ablation.py 2 2 9 0 > gpurun_out/pred_ablation_m64.jsonl 2>&1; tail -1 gpurun_out/pred_ablation_m64.jsonl
timeout 600 python tools/predictive_ablation.py 2 5 9 4096 > gpurun_out/pred_ablation_m4096.jsonl 2>&1; tail -2 gpurun_out/pred_ablation_m4096.jsonl
timeout 600 python tools/predictive_ablation.py 2 5 1 4096 > gpurun_out/pred_ablation_m4096_k1.jsonl 2>&1; tail -1 gpurun_out/pred_ablation_m4096_k1.jsonl
