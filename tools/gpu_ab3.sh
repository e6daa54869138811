# integrator A/B: variants/head (a saved tree) against the working tree's variants
(cd variants/head && python tools/ab_eval.py 2 5 4 2>&1 | tail -1 | sed 's/^/HEAD /')
python tools/ab_eval.py 2 5 ${AB_VARIANTS:-4} 2>&1 | tail -4
