"""One integrator call of a config, bracketed by cudaProfilerStart/Stop for ncu.

    ncu --profile-from-start off ... python tools/ncu_cfg.py <config> <warm steps> [world] [schedule]

Runs `warm` full steps of the config (sim.Simulation through the C ABI), deposits the next
step, then calls the integrator once inside the profiler range: the whole mesh
(rp_compute_potentials) for world = 1, else rank 0's shard of `world` (the same LPT-dealt
sample of points a rank of an N-GPU run integrates), which bounds the time a full ncu replay
takes on the large configs.  Prints one JSON line with the call's event time and work.
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation  # noqa: E402

cfgn = int(sys.argv[1]) if len(sys.argv) > 1 else 2
warm = int(sys.argv[2]) if len(sys.argv) > 2 else 3
world = int(sys.argv[3]) if len(sys.argv) > 3 else 1
sched = sys.argv[4] if len(sys.argv) > 4 else "persistence"
cfg = W.config(cfgn)
sim = Simulation(cfg)
if sched == "subregion":
    rp.rp_set_schedule(sim.ctx, rp.RP_SCHED_SUBREGION, 1)
for _ in range(warm):
    sim.step()
rp.rp_deposit_step(sim.ctx, sim.x, sim.y, sim.ux, sim.uy, sim.q, W.frame(cfg, sim.k))
npts = cfg.nx * cfg.ny
f64 = dict(dtype=torch.float64, device="cuda")
torch.cuda.synchronize()
rp.rp_profile_enable(sim.ctx, True)
torch.cuda.profiler.start()
if world == 1:
    out = [torch.zeros(npts, **f64) for _ in range(4)]
    nseg = torch.zeros(npts, dtype=torch.int32, device="cuda")
    inf = rp.rp_compute_potentials(sim.ctx, *out, nseg, info=True)
    n = npts
else:
    cap = rp.rp_shard_capacity(sim.ctx, world)
    shard = torch.zeros((cap, 6), **f64)
    n, inf = rp.rp_compute_potentials_shard(sim.ctx, 0, world, shard, info=True)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
pr = rp.rp_profile_read(sim.ctx).as_dict()
print(json.dumps({"config": cfg.name, "step": sim.k, "world": world, "points": n,
                  "schedule": sched, "integrate_ms": pr["integrate_ms"],
                  "units_ms": pr["units_ms"], "info": inf.as_dict()}), flush=True)
sim.close()
