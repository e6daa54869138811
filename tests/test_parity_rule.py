"""The parity rule of the GPU tests (tests/gpu_util.compare_potentials, reading
R-28) on hand-made records: strict 1e-11 values and equal counts, except at points whose oracle
run flags a rounding-determined decision (relative margin < 1e-9: `ties`; within 4 ulp of
|K| + |G|: `noise_ties`), whose values must agree within 4 tau per flagged decision."""
import numpy as np

import oracle
from tests import gpu_util as G


def _records(n):
    r = np.zeros(n, dtype=np.ctypeslib.as_array((oracle.Result * 1)()).dtype)
    r["phi"] = 100.0
    r["ax"] = 50.0
    r["ay"] = -5.0
    r["err"] = 1e-3
    r["nseg"] = 40
    r["nleaf"] = 21
    return r


def _gpu(orc):
    return {k: orc[k].astype(float if k in ("phi", "ax", "ay", "err") else np.int32).copy()
            for k in ("phi", "ax", "ay", "err", "nseg", "nleaf", "capped")}


def test_strict_points():
    orc = _records(4)
    pts = np.arange(4)
    gpu = _gpu(orc)
    gpu["phi"][1] += 1e-8          # 1e-10 relative: fails the 1e-11 bar
    gpu["nseg"][2] += 2            # a different tree
    gpu["ax"][3] += 5e-10          # 5e-12 relative: passes
    fail, worst, nflag = G.compare_potentials(gpu, orc, pts, tau=0.01)
    assert fail.tolist() == [False, True, True, False] and nflag == 0
    assert 9e-11 < worst < 1.1e-10


def test_flagged_points_compare_values_within_tau():
    orc = _records(5)
    orc["noise_ties"][[0, 1, 2]] = [1, 1, 2]
    orc["ties"][3] = 1
    pts = np.arange(5)
    gpu = _gpu(orc)
    tau = 0.01
    gpu["nseg"][:4] += 6           # the other branch at the flagged decision: counts differ
    gpu["phi"][0] += 3.9 * tau     # within 4 tau (one flagged decision)
    gpu["phi"][1] += 4.1 * tau     # beyond 4 tau
    gpu["ay"][2] += 7.9 * tau      # within 4 tau x 2 flagged decisions
    gpu["err"][3] += 1e-3 * tau    # relative-margin tie, values close
    gpu["nseg"][4] += 1            # unflagged: strict
    fail, _, nflag = G.compare_potentials(gpu, orc, pts, tau=tau)
    assert fail.tolist() == [False, True, False, False, True] and nflag == 4
    # without tau the flagged points are only reported (round 1's rule)
    fail, _, _ = G.compare_potentials(gpu, orc, pts)
    assert fail.tolist() == [False, False, False, False, True]
