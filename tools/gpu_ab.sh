# integrator A/B: a saved variant tree (variants/$AB_DIR) against the working tree
(cd variants/${AB_DIR:-head} && python tools/ab_eval.py 2 5 4 2>&1 | tail -1 | sed "s/^/${AB_DIR:-head} /")
python tools/ab_eval.py 2 5 ${AB_VARIANTS:-4} 2>&1 | tail -4
