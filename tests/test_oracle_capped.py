"""P:106 ("always achieves the required error tolerance") at the capped leaves of the canonical
tree (R-12: accepted at D_max with err > tol): on config 2's steady state, the true error at the
points with the most capped leaves -- against the same integral refined to tau/100 with
D_max = 45 -- stays far inside tau, and the splits chasing them are a small share of the work.
Full 200-point analysis: profiles/r02/capped_cfg2.json (tests/capped_analysis.py)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))


def test_capped_leaves_meet_the_tolerance():
    import capped_analysis
    out = capped_analysis.analyse(2, 60, worst=3)
    assert out["capped_leaves"] > 0  # the case exists on this workload
    assert out["max_true_error_over_tau"] < 1e-2
    assert out["chase_eval_share"] < 0.10
