"""Development A/B of integrator evaluation loops (RP_EVAL=<v> selects one at rp_create; a
variant may also be a comma list of environment settings read at rp_create, e.g. RP_COEF=0).

Runs `steps` steps of a config per variant in one process, checks that every variant's
potentials / segment counts are bit-identical to the first one's, and prints the integrator's
CUDA-event time per step.  usage: python tools/ab_eval.py [config] [steps] [variants...]
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation  # noqa: E402

cfgn = int(sys.argv[1]) if len(sys.argv) > 1 else 2
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
variants = sys.argv[3:] or ["4", "RP_COEF=0"]
cfg = W.config(cfgn)
ref = None
for v in variants:
    for key in ("RP_EVAL", "RP_COEF"):
        os.environ.pop(key, None)
    if "=" in v:
        for kv in v.split(","):
            key, val = kv.split("=")
            os.environ[key] = val
    else:
        os.environ["RP_EVAL"] = v
    sim = Simulation(cfg)
    rp.rp_profile_enable(sim.ctx, True)
    outs, ms, ev, last = [], [], [], 0.0
    for s in range(steps):
        info = sim.step(info=True)
        torch.cuda.synchronize()
        prof = rp.rp_profile_read(sim.ctx)
        ms.append(prof.integrate_ms - last)
        last = prof.integrate_ms
        ev.append(info.evals)
        outs.append([t.cpu().numpy().copy() for t in (sim.phi, sim.ax, sim.ay, sim.nseg)])
    if v == "7":
        import ctypes
        buf = (ctypes.c_ulonglong * 6)()
        rp._lib.rp_dev_phase_cycles(buf, 1)
        tot = sum(buf)
        names = ["item", "nodes", "scan", "rounds", "leftover", "tail"]
        print("phase cycles (all steps, warp-summed):",
              {n: f"{100 * b / tot:.1f}%" for n, b in zip(names, buf)}, flush=True)
    sim.close()
    same = None
    if ref is None:
        ref = outs
    else:
        same = all(np.array_equal(a.view(np.uint8) if a.dtype != np.int32 else a,
                                  b.view(np.uint8) if b.dtype != np.int32 else b)
                   for oa, ob in zip(outs, ref) for a, b in zip(oa, ob))
        if not same:  # rounding-level differences: report the relative size and nseg equality
            rel = max(float(np.max(np.abs(a - b))) / max(float(np.max(np.abs(b))), 1e-300)
                      for oa, ob in zip(outs, ref) for a, b in zip(oa[:3], ob[:3]))
            nseg_eq = all(np.array_equal(oa[3], ob[3]) for oa, ob in zip(outs, ref))
            same = f"no (max rel diff {rel:.2e}, nseg equal {nseg_eq})"
    print(f"variant {v}: integrate ms/step {[round(x, 2) for x in ms]} "
          f"(steps 2+: {np.mean(ms[2:]) if len(ms) > 2 else np.mean(ms):.2f}); "
          f"ps/eval {[round(1e9 * m / e, 2) for m, e in zip(ms, ev)]}; "
          f"evals/step (1e9) {[round(e / 1e9, 3) for e in ev]}; bit-identical to first: {same}", flush=True)
