timeout 900 python -m pytest tests/test_gpu_predictive.py -q -x --timeout=400 2>&1 | tail -15
timeout 900 python -m pytest tests -m gpu -q -x --timeout=400 --deselect tests/test_gpu_predictive.py 2>&1 | tail -3
(cd variants/head && python tools/ab_eval.py 2 5 4 2>&1 | tail -1 | sed 's/^/HEAD /')
python tools/ab_eval.py 2 5 4 2>&1 | tail -1
timeout 600 python tools/predictive_ablation.py 2 4 9 0 2>&1 | tail -5
