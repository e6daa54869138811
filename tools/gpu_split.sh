# subtree units: shard projection (near-field-only split vs all subregions), full-size parity
timeout 300 python tools/shard_balance.py 2 3 > gpurun_out/shard_cfg2_j1.json 2>&1
RP_SPLITJ=100000 timeout 300 python tools/shard_balance.py 2 3 > gpurun_out/shard_cfg2_jall.json 2>&1
timeout 600 python tools/shard_balance.py 4 2 > gpurun_out/shard_cfg4_j1.json 2>&1
for f in gpurun_out/shard_cfg2_j1.json gpurun_out/shard_cfg2_jall.json gpurun_out/shard_cfg4_j1.json; do python -c "
import json,sys
d=json.load(open('$f'))
print('$f', [(n, round(v['max_ms'],1), round(v['projected_speedup'],2)) for n,v in d['per_n'].items()])"; done
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x --timeout=600 -k "units or full_size" 2>&1 | tail -2
