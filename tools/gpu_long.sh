# work per step over a long config-2 trajectory (is the bench window representative?)
python tools/ab_eval.py 2 40 4 2>&1 | grep variant
