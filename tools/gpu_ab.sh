python tools/ab_eval.py 2 5 ${AB_VARIANTS:-0 1 2 3} 2>&1 | tail -6
if [ -n "$AB_TESTS" ]; then timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3; fi
