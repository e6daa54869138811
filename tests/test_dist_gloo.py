"""The N > 1 plumbing of the step driver (paper_conf_icpp_arumugamrztgi17_b200/sim.py) on CPU:
two processes, torch.distributed gloo backend, world_size 2 (mesh points sharded,
history replicated, partial moment grids and potential shards all-gathered).

librp needs a GPU, so the ops the driver calls are replaced by a stand-in that implements
the same C-ABI contract (include/rp.h) with the CPU oracle: rank-ordered sum of partials,
snake deal of points longest-predicted-first from the previous step's counts, shard rows.
The sharded 2-rank run must reproduce the 1-rank run (to rounding of the partial sums).
"""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W


def _cfg():
    return W.Config(number=0, name="gloo-12x12", nx=12, ny=12, n_particles=600, steps=3,
                    kappa_max=4, geometry="static", sigma=1.0, cdt=2.2, q_over_mc=1e-3,
                    seed=17_099)


class _Ctx:
    pass


class OracleOps:
    """CPU stand-in for the librp binding with the C-ABI semantics of include/rp.h."""

    def rp_create(self, nx, ny, hx, hy, kap, c, dt, tau, n_theta, max_depth, n_root, dev, rule=0,
                  interp=0, dist=None):
        assert dist is None  # the stand-in has no NCCL: the host (gloo) transport only
        x = _Ctx()
        x.rule, x.interp = rule, interp
        x.nx, x.ny, x.hx, x.hy, x.kap, x.c, x.dt, x.tau = nx, ny, hx, hy, kap, c, dt, tau
        x.n_theta, x.max_depth, x.n_root = n_theta, max_depth, n_root
        x.H = kap + 2
        x.ring = np.zeros((x.H, ny, nx, 4))
        x.frames = np.tile([0.0, 0.0, 1.0, 0.0], (x.H, 1))
        x.k, x.n_pre, x.rigid = -1, 0, False
        x.nseg_prev = None
        return x

    def rp_destroy(self, ctx):
        pass

    def rp_history_init(self, ctx, n_pre, frames, grids, rigid):
        for i, f in enumerate(np.asarray(frames)):
            ctx.frames[(-n_pre + i) % ctx.H] = f
        ctx.n_pre, ctx.rigid = n_pre, rigid

    def rp_partial_bytes(self, ctx):
        return ctx.ny * ctx.nx * 4 * 8  # the stand-in keeps FP64 partials

    def rp_deposit(self, ctx, x, y, ux, uy, q, fk, partial, info=False):
        M, _, _ = oracle.deposit(x.numpy(), y.numpy(), ux.numpy(), uy.numpy(), q, fk, ctx.nx, ctx.ny,
                                 ctx.hx, ctx.hy)
        partial.view(torch.float64).copy_(torch.from_numpy(M).view(-1))

    def rp_history_append(self, ctx, partials, n_parts, fk):
        tot = np.zeros((ctx.ny, ctx.nx, 4))
        parts = partials.view(torch.float64).view(n_parts, ctx.ny, ctx.nx, 4)
        for i in range(n_parts):  # rank order
            tot = tot + parts[i].numpy()
        ctx.k += 1
        ctx.ring[ctx.k % ctx.H] = tot
        ctx.frames[ctx.k % ctx.H] = fk
        if ctx.k == 0 and ctx.rigid:
            for l in range(-ctx.n_pre, 0):
                ctx.ring[l % ctx.H] = oracle.rigid_level(tot, fk, ctx.frames[l % ctx.H])

    def rp_deposit_step(self, ctx, x, y, ux, uy, q, fk, info=False):
        part = torch.zeros(self.rp_partial_bytes(ctx), dtype=torch.uint8)
        self.rp_deposit(ctx, x, y, ux, uy, q, fk, part)
        self.rp_history_append(ctx, part, 1, fk)

    def _problem(self, ctx):
        return oracle.Problem(nx=ctx.nx, ny=ctx.ny, hx=ctx.hx, hy=ctx.hy, c=ctx.c, dt=ctx.dt,
                              tau=ctx.tau, kappa_max=ctx.kap, k=ctx.k, n_pre=ctx.n_pre,
                              ring=ctx.ring, frames=ctx.frames, n_theta=ctx.n_theta,
                              max_depth=ctx.max_depth, n_root=ctx.n_root, rule=ctx.rule,
                              interp=ctx.interp)

    def rp_compute_potentials(self, ctx, phi, ax, ay, err=None, nseg=None, info=False):
        r = self._problem(ctx).potentials(np.arange(ctx.nx * ctx.ny))
        phi.copy_(torch.from_numpy(r["phi"]))
        ax.copy_(torch.from_numpy(r["ax"]))
        ay.copy_(torch.from_numpy(r["ay"]))
        if err is not None:
            err.copy_(torch.from_numpy(r["err"]))
        if nseg is not None:
            nseg.copy_(torch.from_numpy(r["nseg"].astype(np.int32)))
        ctx.nseg_prev = r["nseg"].astype(np.int64)
        return None

    def rp_shard_capacity(self, ctx, world):
        return -(-(ctx.nx * ctx.ny) // world)

    def _owner(self, ctx, world):
        npts = ctx.nx * ctx.ny
        w = ctx.nseg_prev if ctx.nseg_prev is not None else np.zeros(npts, dtype=np.int64)
        order = np.argsort(-w, kind="stable")  # longest predicted first, ties by point id
        owner, row = np.zeros(npts, int), np.zeros(npts, int)
        for i, p in enumerate(order):
            b, r = divmod(i, world)
            owner[p] = world - 1 - r if b % 2 else r  # snake deal
            row[p] = b
        return owner, row

    def rp_compute_potentials_shard(self, ctx, rank, world, shard, info=False):
        owner, row = self._owner(ctx, world)
        pts = np.nonzero(owner == rank)[0].astype(np.int32)
        r = self._problem(ctx).potentials(pts)
        shard.zero_()
        for p, rr in zip(pts, r):
            shard[row[p]] = torch.tensor([p, rr["phi"], rr["ax"], rr["ay"], rr["err"], rr["nseg"]],
                                         dtype=torch.float64)
        return len(pts), None

    def rp_shard_scatter(self, ctx, shards, world, phi, ax, ay, err=None, nseg=None):
        npts = ctx.nx * ctx.ny
        cap = shards.shape[1]
        ns = np.zeros(npts, dtype=np.int64)
        for r in range(world):
            for b in range(cap):
                i = b * world + (world - 1 - r if b % 2 else r)
                if i >= npts:
                    continue
                rec = shards[r, b]
                p = int(rec[0])
                phi[p], ax[p], ay[p] = rec[1], rec[2], rec[3]
                if err is not None:
                    err[p] = rec[4]
                ns[p] = int(rec[5])
                if nseg is not None:
                    nseg[p] = int(rec[5])
        ctx.nseg_prev = ns

    def rp_compute_fields(self, ctx, phi, ax, ay, a_prev, ex, ey, bz):
        sh = (ctx.ny, ctx.nx)
        m = 0 if a_prev is None else a_prev.shape[0]
        m = min(m, ctx.H - 1, ctx.k + ctx.n_pre)  # the frames the ring holds (rp.h)
        frames = [ctx.frames[(ctx.k - j) % ctx.H] for j in range(m + 1)]
        prev = [(a_prev[j, 0].numpy().reshape(sh), a_prev[j, 1].numpy().reshape(sh)) for j in range(m)]
        a, b, c = oracle.fields(ctx.nx, ctx.ny, ctx.hx, ctx.hy, ctx.c, ctx.dt, frames,
                                phi.numpy().reshape(sh), ax.numpy().reshape(sh), ay.numpy().reshape(sh),
                                prev)
        ex.copy_(torch.from_numpy(a.ravel()))
        ey.copy_(torch.from_numpy(b.ravel()))
        bz.copy_(torch.from_numpy(c.ravel()))

    def rp_kick_external(self, ctx, ux, uy, qmc, bz_ext, frac, ox, oy):
        a, b = oracle.kick_external(ctx.dt, ux.numpy(), uy.numpy(), qmc, bz_ext, frac)
        ox.copy_(torch.from_numpy(a))
        oy.copy_(torch.from_numpy(b))

    def rp_push_particles(self, ctx, x, y, ux, uy, qmc, bz_ext, ex, ey, bz):
        fk = ctx.frames[ctx.k % ctx.H]
        sh = (ctx.ny, ctx.nx)
        nx_, ny_, nux, nuy = oracle.push(ctx.nx, ctx.ny, ctx.hx, ctx.hy, ctx.c, ctx.dt, fk,
                                         x.numpy(), y.numpy(), ux.numpy(), uy.numpy(), qmc, bz_ext,
                                         ex.numpy().reshape(sh), ey.numpy().reshape(sh),
                                         bz.numpy().reshape(sh))
        for t, v in zip((x, y, ux, uy), (nx_, ny_, nux, nuy)):
            t.copy_(torch.from_numpy(v))


def _run(world, rank, port, out):
    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
    group = None
    if world > 1:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        group = dist.group.WORLD
    cfg = _cfg()
    sim = Simulation(cfg, device="cpu", group=group, ops=OracleOps())
    res = []
    for _ in range(cfg.steps):
        sim.step()
        res.append(np.stack([sim.phi.numpy().copy(), sim.ax.numpy().copy(),
                             sim.nseg.numpy().astype(np.float64)]))
    parts = [sim.x.numpy().copy(), sim.ux.numpy().copy()]
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    out[rank] = (np.stack(res), parts)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    out = {}
    _run(world, rank, port, out)
    q.put((rank, out[rank]))


@pytest.mark.slow
def test_two_rank_gloo_matches_single_rank():
    single = {}
    _run(1, 0, 0, single)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = {}
    import queue as _q
    while len(got) < 2:
        try:
            r, v = q.get(timeout=5)
            got[r] = v
        except _q.Empty:
            assert all(p.is_alive() for p in procs), "a rank died"
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    ref = single[0][0]
    for r in range(2):
        res = got[r][0]
        # every rank ends each step with the full mesh (post all-gather), equal to 1 rank
        scale = np.abs(ref[:, 0]).max()
        assert np.abs(res[:, :2] - ref[:, :2]).max() <= 1e-12 * scale
        np.testing.assert_array_equal(res[:, 2], ref[:, 2])
    # particles are sharded by index: rank r pushed particles [r*n/2, (r+1)*n/2)
    n = _cfg().n_particles
    x_all = np.concatenate([got[0][1][0], got[1][1][0]])
    assert len(x_all) == n
    assert np.abs(x_all - single[0][1][0]).max() < 1e-12


def test_snake_shard_map_balances_and_covers():
    ops = OracleOps()
    ctx = ops.rp_create(10, 7, 1.0, 1.0, 3, 1.0, 1.0, 1e-6, 64, 30, 2, 0)
    rng = np.random.default_rng(0)
    ctx.nseg_prev = rng.integers(1, 400, size=70)
    for world in (2, 3, 4, 8):
        owner, row = ops._owner(ctx, world)
        counts = np.bincount(owner, minlength=world)
        assert counts.max() - counts.min() <= 1
        assert row.max() < ops.rp_shard_capacity(ctx, world)
        work = np.bincount(owner, weights=ctx.nseg_prev, minlength=world)
        assert work.max() / work.mean() < 1.1  # LPT snake deal keeps predicted work balanced
