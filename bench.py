#!/usr/bin/env python
"""Benchmark of the retarded-potential step (BASELINE.json metric: mesh-point potentials/s
and FP64 GFLOP/s per step at 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 5] [--impl ours|reference]

One step = the whole hot path of the paper's loop: deposit -> retarded potentials at
every mesh point -> self-fields -> push.  Default workload: BASELINE.json configs[4] (config 5:
512x512 mesh, 1e8 particles, LCLS bend, full retarded history kappa = 2000), the strong-scaling
configuration the metric is quoted on; `--config 1..4` runs the others.  Inputs are seeded
synthetic (workloads/).

One timed pass serves both numbers.  Every step goes through the C ABI's end-to-end call
rp_step_host with PINNED HOST buffers (H2D of this rank's particles, the step, D2H of the pushed
particles and the six mesh outputs): CUDA events around the call give `e2e`; librp's own
events around the step's device part (deposit through push, between the copies) give `value`,
the throughput with inputs resident in HBM.  N > 1: one process per GPU (torchrun, or
self-spawned when WORLD_SIZE is unset); librp owns an NCCL communicator (unique id broadcast
over torch.distributed) and all-gathers inside its calls; mesh points are sharded, the history
replicated (strong scaling: the same mesh and bunch for every N); times are the max over ranks.
RP_DIST_BACKEND=gloo instead runs the caller-side transport (torch gloo all-gathers around
librp's shard calls) so several ranks can share one GPU.

--impl reference times the CPU oracle (oracle/, test infrastructure; the one other place
bench.py may execute it) on the same workload, a bounded sample of mesh points per step.
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import socket
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

# Algorithmic FP64 flop census (FMA = 2), DESIGN.md sec. 6 / SURVEY 8(d):
F_EVAL = 210   # one integrand evaluation f(r', theta', t'): 27-point TSC x Lagrange-3 gather
F_NODE = 100   # one r' node: retarded frame, circle centre, arcs
F_SEG = 60     # one GK15 segment: K15/G7 sums, error, decision
METRIC = "mesh-point potentials/sec (and FP64 GFLOP/s per step)"
UNIT = "mesh-point potentials/s"
L2_BYTES = 126 * 2 ** 20


def algorithmic_flops(info: dict) -> float:
    # evaluations performed: the rules' integrand nodes minus the arc end nodes on the support
    # boundary, where the integrand vanishes and the GPU path skips them (DESIGN R-24)
    performed = info["evals"] - info.get("skipped", 0)
    return performed * F_EVAL + info["nodes"] * F_NODE + info["segments"] * F_SEG


def measured_peaks():
    out = {"hbm_gbs": 6544.3, "fp64_tflops": 34.1, "source": "fallback"}
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            mp = json.load(f)
        out["hbm_gbs"] = mp.get("hbm_gbs", out["hbm_gbs"])
        out["source"] = "MEASURED_PEAKS.json"
    except Exception:
        pass
    # FP64 DFMA peak: the best of the committed microbenchmarks (tools/fp64_peak.cu,
    # tools/mix_peak.cu); DMMA shares the same FP64 pipe (profiles/r01_fp64_dmma_mix.json)
    best, src = 0.0, None
    for name in ("r01_fp64_peak.json", "r01_fp64_dmma_mix.json"):
        try:
            with open(os.path.join(ROOT, "profiles", name)) as f:
                for line in f:
                    d = json.loads(line)
                    for key in ("fp64_tflops_sustained", "fp64_tflops_burst", "dfma_tf"):
                        if d.get(key, 0.0) > best:
                            best, src = d[key], f"profiles/{name} ({key})"
        except Exception:
            pass
    if best > 0:
        out["fp64_tflops"], out["fp64_source"] = best, src + ", measured DFMA peak"
    else:
        out["fp64_source"] = "fallback 34.1 TF/s (DESIGN.md)"
    return out


def ncu_traffic(cfg_number: int):
    """DRAM bytes (read + write) of one integrator call of THIS config, from the committed ncu
    capture of the same workload (profiles/ncu_traffic_cfg<N>.json); None if there is none."""
    try:
        with open(os.path.join(ROOT, "profiles", f"ncu_traffic_cfg{cfg_number}.json")) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_call"), d.get("source")
    except Exception:
        return None, None


class ClockSampler:
    QUERY = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = None

    def start(self):
        try:
            fd, self.path = tempfile.mkstemp(suffix=".csv")
            os.close(fd)
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.QUERY}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        time.sleep(0.15)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        os.unlink(self.path)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def _free_port() -> int:
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def self_spawn(argv, n) -> int:
    """`--gpus N` without torchrun: relaunch this script as N ranks (one per GPU)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node",
           str(n), "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.abspath(__file__), *argv]
    return subprocess.call(cmd)


def _cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def _set_schedule(rp, ctx, sched):
    if sched == "index":
        rp.rp_set_schedule(ctx, rp.RP_SCHED_INDEX, 1)
    elif sched == "persistence":
        rp.rp_set_schedule(ctx, rp.RP_SCHED_PERSISTENCE, 1)
    elif sched == "subregion":
        rp.rp_set_schedule(ctx, rp.RP_SCHED_SUBREGION, 1)
    elif sched.startswith("knn"):
        rp.rp_set_schedule(ctx, rp.RP_SCHED_KNN, int(sched[3:]))
    else:
        raise SystemExit(f"unknown schedule {sched}")


# ---------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_arumugamrztgi17_b200 import rp

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    backend = os.environ.get("RP_DIST_BACKEND", "nccl")
    ngpu = max(1, torch.cuda.device_count())
    dev_index = local % ngpu
    torch.cuda.set_device(dev_index)
    dev = torch.device("cuda", dev_index)
    if world > 1:
        if backend == "nccl":
            os.environ.setdefault("NCCL_DEBUG", "INFO")  # rank count visible on stderr
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    cfg = W.config(args.config)
    cfg.rule = 1 if args.rule == "simpson" else 0
    cfg.interp = 1 if args.interp == "lagrange3" else 0
    npts = cfg.nx * cfg.ny
    ring_bytes = cfg.H * (cfg.nx + 6) * (cfg.ny + 6) * 32
    flush_l2 = ring_bytes <= 4 * L2_BYTES
    flush = torch.empty(512 * 1024 * 1024 // 8, dtype=torch.float64, device=dev) if flush_l2 else None

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(d):
        if world == 1:
            return d
        t = torch.tensor(list(d.values()), dtype=torch.float64, device=dev)
        dist.all_reduce(t)
        return {k: int(v) for k, v in zip(d, t.tolist())}

    x, y, ux, uy = W.particles(cfg)
    n_all = len(x)
    lo, hi = (n_all * rank) // world, (n_all * (rank + 1)) // world
    host = [torch.from_numpy(np.ascontiguousarray(a[lo:hi])).pin_memory() for a in (x, y, ux, uy)]
    del x, y, ux, uy
    q = 1.0 / n_all
    mesh = torch.zeros((6, npts), dtype=torch.float64).pin_memory()
    stream = torch.cuda.current_stream(dev)
    totals = {"evals": 0, "skipped": 0, "nodes": 0, "segments": 0, "capped": 0, "items": 0,
              "units": 0}
    e2e_ms = []
    sim = ctx = None
    in_lib = world == 1 or backend == "nccl"
    if in_lib:
        # the product path: librp owns the exchange (an NCCL communicator when world > 1)
        dist_arg = None
        if world > 1:
            obj = [rp.rp_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            dist_arg = (rank, world, obj[0])
        ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau,
                           cfg.n_theta, cfg.max_depth, cfg.n_root, dev_index, cfg.rule, cfg.interp,
                           dist=dist_arg)
        rp.rp_set_stream(ctx, stream)
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
    else:
        from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
        sim = Simulation(cfg, group=dist.group.WORLD, transport="host")
        ctx = sim.ctx
    _set_schedule(rp, ctx, args.schedule)
    dev_events = []

    def one_step(k, info):
        if in_lib:
            return rp.rp_step_host(ctx, *host, q, W.frame(cfg, k), cfg.q_over_mc, cfg.bz_ext, mesh,
                                   info=info)
        # caller-side transport: the same host copies around Simulation.step (torch copies)
        for d, h in zip((sim.x, sim.y, sim.ux, sim.uy), host):
            d.copy_(h, non_blocking=True)
        m0 = torch.cuda.Event(enable_timing=True)
        m1 = torch.cuda.Event(enable_timing=True)
        m0.record(stream)
        inf = sim.step(info=info)
        m1.record(stream)
        for i, t in enumerate((sim.phi, sim.ax, sim.ay, sim.ex, sim.ey, sim.bz)):
            mesh[i].copy_(t, non_blocking=True)
        for d, h in zip((sim.x, sim.y, sim.ux, sim.uy), host):
            h.copy_(d, non_blocking=True)
        dev_events.append((m0, m1))
        return inf

    k = 0
    for _ in range(args.warmup):
        one_step(k, False)
        k += 1
    barrier()
    dev_events.clear()
    launches0 = rp.rp_launch_count(ctx)
    rp.rp_profile_enable(ctx, True)
    clocks = ClockSampler(dev_index)
    clocks.start()
    barrier()
    for _ in range(args.steps):
        if flush is not None:
            flush.fill_(1.0)  # evict L2 between timed steps (outside the events)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        inf = one_step(k, True)
        e1.record(stream)
        e1.synchronize()
        e2e_ms.append(e0.elapsed_time(e1))
        for key in totals:
            totals[key] += getattr(inf, key)
        k += 1
    barrier()
    clk = clocks.stop()
    prof = rp.rp_profile_read(ctx).as_dict()
    rp.rp_profile_enable(ctx, False)
    launches = rp.rp_launch_count(ctx) - launches0
    if in_lib:
        dev_ms = prof["step_ms"]
    else:
        dev_ms = sum(a.elapsed_time(b) for a, b in dev_events)
    total_ms = max_over_ranks(dev_ms)
    total_e2e = max_over_ranks(sum(e2e_ms))
    integ_max = max_over_ranks(prof["integrate_ms"])
    totals = sum_over_ranks(totals)
    value = npts * args.steps / (total_ms * 1e-3)
    flops_total = algorithmic_flops(totals)
    gflops = flops_total / (total_ms * 1e-3) / 1e9
    digest = hashlib.sha256(mesh.numpy().tobytes()).hexdigest()[:16]
    pbytes = 4 * host[0].numel() * 8
    e2e = {"value": npts * args.steps / (total_e2e * 1e-3), "unit": UNIT,
           "h2d_bytes_per_step": pbytes, "d2h_bytes_per_step": pbytes + 6 * npts * 8,
           "ms_per_step": total_e2e / args.steps,
           "bytes_per": "rank 0 (its particle shard)" if world > 1 else "the whole job",
           "api": ("rp_step_host (C ABI, pinned host buffers)" if in_lib else
                   "sim.Simulation.step with pinned host copies (torch, gloo transport)")}
    peaks = measured_peaks()
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, args, rp, ctx, dev, value, totals)
    if rank == 0:
        integ_ms_avg = integ_max / max(1, prof["integrate_launches"])
        flops_per_launch = flops_total / args.steps / max(1, world)
        achieved = flops_per_launch / (integ_ms_avg * 1e-3) / 1e12 if integ_ms_avg > 0 else 0.0
        traffic, tsrc = ncu_traffic(cfg.number)
        line = {
            "metric": METRIC,
            "value": value,
            "unit": UNIT,
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": total_ms / args.steps,
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "f64",
            "data": "synthetic (seeded Gaussian bunch in the LCLS bend, workloads/)",
            "config": {"workload": cfg.name, "mesh": f"{cfg.nx}x{cfg.ny}",
                       "particles": cfg.n_particles, "history_depth": cfg.kappa_max,
                       "tau": cfg.tau, "n_theta": cfg.n_theta, "n_root": cfg.n_root,
                       "parallelism": f"mesh-point shards x{world}, history replicated",
                       "transport": ("none" if world == 1 else "librp NCCL all-gathers" if in_lib
                                     else f"caller-side {backend} all-gathers"),
                       "l2": ("flushed between timed steps (512 MB write)" if flush_l2 else
                              f"inputs larger than L2 (ring {ring_bytes / 2 ** 30:.1f} GiB)"),
                       "schedule": args.schedule, "outer_rule": args.rule,
                       "interp": args.interp},
            "fp64_gflops": gflops,
            "evals_per_s": totals["evals"] / (total_ms * 1e-3),
            "work_per_step": {k2: v / args.steps for k2, v in totals.items()},
            "roofline": {"kernel": "k_integrate (GK15 tree integrator)", "bound": "alu",
                         "achieved": achieved, "peak": peaks["fp64_tflops"], "unit": "TFLOP/s",
                         "frac": achieved / peaks["fp64_tflops"], "traffic": traffic,
                         "traffic_source": tsrc,
                         "peak_source": peaks["fp64_source"],
                         "share_of_step": prof["integrate_ms"] / dev_ms if dev_ms else None,
                         "avg_launch_ms": integ_ms_avg,
                         "algorithmic_flops_per_launch": flops_per_launch},
            "kernel_ms_per_step": {k2: v / args.steps for k2, v in prof.items() if k2.endswith("_ms")},
            "gpu_launches": launches,
            "clocks": clk,
            "e2e": e2e,
            "result_sha256": digest,
            "paper_context": "485 DP GFLOP/s and 2.5x on one Tesla K40 (PAPER.md P:11, P:255)",
        }
        if cpu is not None:
            line["cpu_baseline"] = cpu
        print(json.dumps(line), flush=True)
    if sim is not None:
        sim.close()
    else:
        rp.rp_destroy(ctx)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


# ---------------------------------------------------------------------------- oracle arm
def _problem(cfg, ring, frames, k):
    import oracle
    return oracle.Problem(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt,
                          tau=cfg.tau, kappa_max=cfg.kappa_max, k=k, n_pre=cfg.n_pre, ring=ring,
                          frames=frames, n_theta=cfg.n_theta, max_depth=cfg.max_depth,
                          n_root=cfg.n_root, rule=cfg.rule, interp=cfg.interp)


def _oracle_rigid_state(cfg):
    """The oracle's own step-0 state: its deposit of the seeded bunch + the rigid pre-history."""
    import oracle
    oracle.set_threads(_cores())  # all host cores, whatever OMP_NUM_THREADS torchrun set
    x, y, ux, uy = W.particles(cfg)
    q = 1.0 / len(x)
    M, _, _ = oracle.deposit(x, y, ux, uy, q, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    del x, y, ux, uy
    ring = oracle.rigid_ring(M, W.ring_frames(cfg, 0))
    return _problem(cfg, ring, W.ring_frames(cfg, 0), 0)


def _time_sample(P, order, budget_s, chunk):
    done, t, evals = 0, 0.0, 0
    while done < len(order) and t < budget_s:
        pts = order[done:done + chunk]
        t0 = time.perf_counter()
        res = P.potentials(pts)
        t += time.perf_counter() - t0
        evals += int(res["evals"].sum())
        done += len(pts)
    return done, t, evals


def cpu_baseline(cfg, args, rp, ctx, dev, gpu_value, gpu_totals, budget_s: float = 15.0):
    """The oracle as it stands, all host cores (OpenMP), on a bounded random sample of the mesh
    points of the LAST TIMED STEP: the GPU's history ring and frames at that step are copied out
    (rp_save_state), so both arms integrate the same state; reported per point and per
    integrand evaluation (the work per point varies along the trajectory)."""
    import oracle
    import torch
    oracle.set_threads(_cores())
    ring = torch.zeros((cfg.H, cfg.ny, cfg.nx, 4), dtype=torch.float64, device=dev)
    k, frames = rp.rp_save_state(ctx, ring, cfg.H)
    ring_h = ring.cpu().numpy()
    del ring
    P = _problem(cfg, ring_h, frames, k)
    npts = cfg.nx * cfg.ny
    order = np.random.default_rng(2).permutation(npts).astype(np.int32)
    chunk = max(4, min(64, 4 * _cores()))
    done, t, evals = _time_sample(P, order, budget_s, chunk)
    gpu_eps = gpu_totals["evals"] / args.steps * gpu_value / npts
    return {"value": done / t, "unit": UNIT, "cores": _cores(), "kind": "oracle",
            "evals_per_s": evals / t, "gpu_evals_per_s_same_steps": gpu_eps,
            "sample": f"{done} random mesh points of {cfg.name} at step {k} (the last timed GPU "
                      f"step: the GPU's ring and frames copied out), {t:.1f} s wall, "
                      f"{evals / max(done, 1):.3g} integrand evaluations per point"}


REF_SAMPLE = {1: 256, 2: 256, 3: 128, 4: 64, 5: 64}  # points per reference step (~seconds each)


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cfg = W.config(args.config)
    P = _oracle_rigid_state(cfg)
    sample = REF_SAMPLE.get(cfg.number, 64)
    order = np.random.default_rng(3).permutation(cfg.nx * cfg.ny).astype(np.int32)
    for w in range(args.warmup):
        P.potentials(order[w * 4:(w + 1) * 4])
    t, evals = 0.0, 0
    for s in range(args.steps):
        pts = order[(s * sample) % len(order):][:sample]
        t0 = time.perf_counter()
        res = P.potentials(pts)
        t += time.perf_counter() - t0
        evals += int(res["evals"].sum())
    value = sample * args.steps / t
    print(json.dumps({
        "impl": "reference", "metric": METRIC,
        "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded Gaussian bunch in the LCLS bend, workloads/)",
        "config": {"workload": cfg.name, "mesh": f"{cfg.nx}x{cfg.ny}",
                   "particles": cfg.n_particles, "history_depth": cfg.kappa_max},
        "evals_per_s": evals / t,
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": _cores(), "kind": "oracle",
                         "evals_per_s": evals / t,
                         "sample": f"{sample} random mesh points per step of {cfg.name} at step 0 "
                                   f"(the oracle's own deposit + rigid steady-state pre-history; "
                                   f"{evals / (sample * args.steps):.3g} integrand evaluations "
                                   f"per point)"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=int(os.environ.get("WORLD_SIZE", "1")))
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--rule", default="gk15", choices=["gk15", "simpson"],
                    help="outer segment rule (simpson = the paper's RP-QUADRULE, a variant)")
    ap.add_argument("--interp", default="tsc", choices=["tsc", "lagrange3"],
                    help="spatial part of the 27-point stencil (lagrange3 = variant R-25)")
    ap.add_argument("--schedule", default="subregion",
                    help="work-order forecast: index | persistence | subregion | knn5 | knn9 | knn25")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        raise SystemExit(self_spawn(sys.argv[1:], args.gpus))
    if args.warmup < 3 and args.impl == "ours":
        print("warning: fewer than 3 warm-up steps", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
