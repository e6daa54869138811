#!/usr/bin/env python
"""Benchmark of the retarded-potential step (BASELINE.json metric: mesh-point potentials/s
and FP64 GFLOP/s per step at 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--impl ours|reference]

One step = the whole hot path of the paper's loop on BASELINE.json configs[1]
(config 2: 64x64 mesh, 1e6 particles, LCLS bend, full retarded history kappa = 100):
deposit -> retarded potentials at every mesh point -> self-fields -> push.  Inputs are
seeded synthetic (workloads/); the timed region starts with everything resident in HBM.
For N > 1 run under torchrun: mesh points are sharded and the history replicated (strong
scaling: the same mesh and bunch for every N).  Rank 0 prints ONE JSON line.

--impl reference times the CPU oracle (oracle/, test infrastructure; the one other place
bench.py may execute it) on the same workload, a bounded sample of mesh points per step.
"""
from __future__ import annotations

import argparse
import json
import math
import os
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


def ncu_traffic():
    """Per-launch DRAM bytes of the integrator from the committed ncu --set full summary."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_integrate.json")) as f:
            d = json.load(f)
        return d.get("dram_bytes_per_launch")
    except Exception:
        return None


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


# ---------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, __import__("torch").cuda.device_count())
    if args.gpus != world:
        if world == 1 and args.gpus > 1:
            raise SystemExit("--gpus N > 1 must be launched with torchrun (one rank per GPU)")
    torch.cuda.set_device(local % max(1, torch.cuda.device_count()))
    group = None
    if world > 1:
        backend = os.environ.get("RP_DIST_BACKEND", "nccl")  # gloo: 2 ranks on 1 GPU (tests)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        group = dist.group.WORLD
    cfg = W.config(args.config)
    cfg.rule = 1 if args.rule == "simpson" else 0
    cfg.interp = 1 if args.interp == "lagrange3" else 0
    sim = Simulation(cfg, group=group)
    sched = args.schedule
    if sched == "index":
        rp.rp_set_schedule(sim.ctx, rp.RP_SCHED_INDEX, 1)
    elif sched == "subregion":
        rp.rp_set_schedule(sim.ctx, rp.RP_SCHED_SUBREGION, 1)
    elif sched.startswith("knn"):
        rp.rp_set_schedule(sim.ctx, rp.RP_SCHED_KNN, int(sched[3:]))
    dev = torch.device("cuda", local)
    flush = torch.empty(512 * 1024 * 1024 // 8, dtype=torch.float64, device=dev)  # 512 MB > L2

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        sim.step()
    barrier()
    launches0 = rp.rp_launch_count(sim.ctx)
    rp.rp_profile_enable(sim.ctx, True)
    stream = torch.cuda.current_stream()
    clocks = ClockSampler(local)
    clocks.start()
    barrier()
    step_ms = []
    totals = {"evals": 0, "skipped": 0, "nodes": 0, "segments": 0, "capped": 0, "items": 0,
              "units": 0, "unit_overflow": 0}
    for _ in range(args.steps):
        flush.fill_(1.0)  # evict L2 between timed steps (outside the events)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        inf = sim.step(info=True)
        e1.record(stream)
        e1.synchronize()
        step_ms.append(e0.elapsed_time(e1))
        for k2 in totals:
            totals[k2] += getattr(inf, k2)
    barrier()
    clk = clocks.stop()
    prof = rp.rp_profile_read(sim.ctx).as_dict()
    rp.rp_profile_enable(sim.ctx, False)
    launches = rp.rp_launch_count(sim.ctx) - launches0
    local_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([local_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
        c = torch.tensor([totals[k2] for k2 in totals], dtype=torch.float64, device=dev)
        dist.all_reduce(c)
        totals = {k2: int(v) for k2, v in zip(totals, c.tolist())}
        p = torch.tensor([prof["integrate_ms"]], dtype=torch.float64, device=dev)
        dist.all_reduce(p, op=dist.ReduceOp.MAX)
        prof["integrate_ms"] = float(p.item())
    else:
        total_ms = local_ms
    npts = cfg.nx * cfg.ny
    value = npts * args.steps / (total_ms * 1e-3)
    flops_total = algorithmic_flops(totals)
    gflops = flops_total / (total_ms * 1e-3) / 1e9

    # ---- end-to-end through the C ABI with host buffers (pinned), every step:
    # H2D of the particles, the whole step, D2H of the pushed particles + six mesh outputs.
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(cfg, args, dev) if world == 1 else run_e2e_dist(cfg, args, dev, group)

    peaks = measured_peaks()
    if rank == 0:
        integ_ms_avg = prof["integrate_ms"] / max(1, prof["integrate_launches"])
        flops_per_launch = flops_total / args.steps / max(1, world)
        achieved = flops_per_launch / (integ_ms_avg * 1e-3) / 1e12 if integ_ms_avg > 0 else 0.0
        traffic = ncu_traffic()
        line = {
            "metric": "mesh-point potentials/sec (and FP64 GFLOP/s per step)",
            "value": value,
            "unit": "mesh-point potentials/s",
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
                       "l2": "flushed between timed steps (512 MB write)",
                       "schedule": args.schedule, "outer_rule": args.rule,
                       "interp": args.interp},
            "fp64_gflops": gflops,
            "work_per_step": {k2: v / args.steps for k2, v in totals.items()},
            "roofline": {"kernel": "k_integrate (GK15 tree integrator)", "bound": "alu",
                         "achieved": achieved, "peak": peaks["fp64_tflops"], "unit": "TFLOP/s",
                         "frac": achieved / peaks["fp64_tflops"], "traffic": traffic,
                         "peak_source": peaks["fp64_source"],
                         "share_of_step": prof["integrate_ms"] / total_ms if world == 1 else None,
                         "avg_launch_ms": integ_ms_avg},
            "kernel_ms_per_step": {k2: v / args.steps for k2, v in prof.items() if k2.endswith("_ms")},
            "gpu_launches": launches,
            "clocks": clk,
            "e2e": e2e,
            "paper_context": "485 DP GFLOP/s and 2.5x on one Tesla K40 (PAPER.md P:11, P:255)",
        }
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(cfg, args)
        print(json.dumps(line), flush=True)
    sim.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def run_e2e_dist(cfg, args, dev, group):
    """N > 1: each rank copies its particle shard from pinned host memory, runs the sharded
    step, and copies the full-mesh potentials and fields (and its pushed shard) back.  Time is
    the max over ranks of the CUDA-event time on the step's stream."""
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
    sim = Simulation(cfg, group=group)
    host = [t.detach().cpu().pin_memory() for t in (sim.x, sim.y, sim.ux, sim.uy)]
    npts = cfg.nx * cfg.ny
    mesh = torch.zeros((6, npts), dtype=torch.float64).pin_memory()
    stream = torch.cuda.current_stream()
    for _ in range(args.warmup):
        sim.step()
    dist.barrier()
    torch.cuda.synchronize()
    ms = 0.0
    for _ in range(args.steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for d, h in zip((sim.x, sim.y, sim.ux, sim.uy), host):
            d.copy_(h, non_blocking=True)
        sim.step()
        for i, t in enumerate((sim.phi, sim.ax, sim.ay, sim.ex, sim.ey, sim.bz)):
            mesh[i].copy_(t, non_blocking=True)
        for d, h in zip((sim.x, sim.y, sim.ux, sim.uy), host):
            h.copy_(d, non_blocking=True)
        e1.record(stream)
        e1.synchronize()
        ms += e0.elapsed_time(e1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    sim.close()
    pbytes = 4 * sim.x.numel() * 8
    return {"value": npts * args.steps / (ms * 1e-3), "unit": "mesh-point potentials/s",
            "h2d_bytes_per_step": pbytes, "d2h_bytes_per_step": pbytes + 6 * npts * 8,
            "ms_per_step": ms / args.steps, "bytes_per": "rank 0 (particle shard)",
            "api": "sim.Simulation.step with pinned host copies (torch) around the C-ABI calls"}


def run_e2e(cfg, args, dev):
    import torch

    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    x, y, ux, uy = W.particles(cfg)
    hx, hy, hux, huy = (torch.tensor(a).pin_memory() for a in (x, y, ux, uy))
    npts = cfg.nx * cfg.ny
    mesh = torch.zeros((6, npts), dtype=torch.float64).pin_memory()
    ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau,
                       cfg.n_theta, cfg.max_depth, cfg.n_root, dev.index or 0, cfg.rule,
                       cfg.interp)
    try:
        stream = torch.cuda.current_stream()
        rp.rp_set_stream(ctx, stream)
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        k = 0
        for _ in range(args.warmup):
            rp.rp_step_host(ctx, hx, hy, hux, huy, 1.0 / len(x), W.frame(cfg, k), cfg.q_over_mc,
                            cfg.bz_ext, mesh)
            k += 1
        torch.cuda.synchronize()
        ms = 0.0
        for _ in range(args.steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            rp.rp_step_host(ctx, hx, hy, hux, huy, 1.0 / len(x), W.frame(cfg, k), cfg.q_over_mc,
                            cfg.bz_ext, mesh)
            e1.record(stream)
            e1.synchronize()
            ms += e0.elapsed_time(e1)
            k += 1
        pbytes = 4 * len(x) * 8
        return {"value": npts * args.steps / (ms * 1e-3), "unit": "mesh-point potentials/s",
                "h2d_bytes_per_step": pbytes, "d2h_bytes_per_step": pbytes + 6 * npts * 8,
                "ms_per_step": ms / args.steps, "api": "rp_step_host (C ABI, pinned host buffers)"}
    finally:
        rp.rp_destroy(ctx)


# ---------------------------------------------------------------------------- oracle arm
def _oracle_state(cfg):
    import oracle
    oracle.set_threads(_cores())  # all host cores, whatever OMP_NUM_THREADS torchrun set
    x, y, ux, uy = W.particles(cfg)
    q = 1.0 / len(x)
    t0 = time.perf_counter()
    M, _, _ = oracle.deposit(x, y, ux, uy, q, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    t_dep = time.perf_counter() - t0
    ring = oracle.rigid_ring(M, W.ring_frames(cfg, 0))
    P = oracle.Problem(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt, tau=cfg.tau,
                       kappa_max=cfg.kappa_max, k=0, n_pre=cfg.n_pre, ring=ring,
                       frames=W.ring_frames(cfg, 0), n_theta=cfg.n_theta, max_depth=cfg.max_depth,
                       n_root=cfg.n_root)
    return P, t_dep


def _cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_baseline(cfg, args, budget_s: float = 15.0):
    """The oracle as it stands, all host cores (OpenMP), on a bounded stratified sample of
    the mesh points of step 0 of the same workload."""
    P, t_dep = _oracle_state(cfg)
    npts = cfg.nx * cfg.ny
    order = W.sample_points(cfg.nx, cfg.ny, npts, seed=0)
    rng = np.random.default_rng(2)
    order = rng.permutation(order).astype(np.int32)
    done, t = 0, 0.0
    while done < npts and t < budget_s:
        chunk = order[done:done + 64]
        t0 = time.perf_counter()
        P.potentials(chunk)
        t += time.perf_counter() - t0
        done += len(chunk)
    return {"value": done / t, "unit": "mesh-point potentials/s", "cores": _cores(),
            "kind": "oracle",
            "sample": f"{done} random mesh points of {cfg.name} step 0 (rigid history), "
                      f"{t:.1f} s wall; oracle deposit of all particles {t_dep:.2f} s not included"}


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cfg = W.config(args.config)
    P, _ = _oracle_state(cfg)
    sample = 256
    order = np.random.default_rng(3).permutation(cfg.nx * cfg.ny).astype(np.int32)
    for w in range(args.warmup):
        P.potentials(order[w * 16:(w + 1) * 16])
    t = 0.0
    for s in range(args.steps):
        pts = order[(s * sample) % len(order):][:sample]
        t0 = time.perf_counter()
        P.potentials(pts)
        t += time.perf_counter() - t0
    value = sample * args.steps / t
    print(json.dumps({
        "impl": "reference", "metric": "mesh-point potentials/sec (and FP64 GFLOP/s per step)",
        "value": value, "unit": "mesh-point potentials/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded Gaussian bunch in the LCLS bend, workloads/)",
        "config": {"workload": cfg.name, "mesh": f"{cfg.nx}x{cfg.ny}",
                   "particles": cfg.n_particles, "history_depth": cfg.kappa_max},
        "cpu_baseline": {"value": value, "unit": "mesh-point potentials/s", "cores": _cores(),
                         "kind": "oracle",
                         "sample": f"{sample} random mesh points per step of {cfg.name} step 0"},
        "e2e": {"value": value, "unit": "mesh-point potentials/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=int(os.environ.get("WORLD_SIZE", "1")))
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--rule", default="gk15", choices=["gk15", "simpson"],
                    help="outer segment rule (simpson = the paper's RP-QUADRULE, a variant)")
    ap.add_argument("--interp", default="tsc", choices=["tsc", "lagrange3"],
                    help="spatial part of the 27-point stencil (lagrange3 = variant R-25)")
    ap.add_argument("--schedule", default="persistence",
                    help="work-order forecast: index | persistence | knn5 | knn9 | knn25")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        print("warning: fewer than 3 warm-up steps", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
