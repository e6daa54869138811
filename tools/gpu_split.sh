timeout 300 python tools/ab_eval.py 2 5 4 RP_SPLIT=0,RP_EVAL=4 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -q -x --timeout=400 2>&1 | tail -3
timeout 300 python tools/shard_balance.py 2 3 2>&1 | tail -c 1600
