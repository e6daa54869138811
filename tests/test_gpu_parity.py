"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element,
on the same seeded inputs.

Bars: deposition bins bit-exact; moment grids within 1e-12 of max|M|; potentials within
1e-11 * max(|phi|,|A|) per point with equal segment counts (oracle tie-flagged points are
reported, not failed); fields within 1e-11 relative; push within 1e-13.
"""
import math

import numpy as np
import pytest

import oracle
import workloads as W
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    assert t.cuda.is_available()
    return t


def _dev_arrays(torch, *arrs):
    return [torch.tensor(np.ascontiguousarray(a), dtype=torch.float64, device="cuda") for a in arrs]


# ------------------------------------------------------------------ deposition
def _partial(torch, ctx, n=1):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    return torch.zeros(n * rp.rp_partial_bytes(ctx), dtype=torch.uint8, device="cuda")


def _slot_moments(torch, ctx, cfg, slot):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    ring = torch.zeros((cfg.H, cfg.ny, cfg.nx, 4), dtype=torch.float64, device="cuda")
    rp.rp_save_state(ctx, ring)
    return ring[slot].cpu().numpy()


@pytest.mark.parametrize("cfgno", [1, 2])
def test_deposit_bins_bit_exact_and_moments(torch, cfgno):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(cfgno)
    x, y, ux, uy = W.particles(cfg)
    x = x.copy()
    x[:3] += 30 * cfg.sigma  # some lost particles
    M, bins, ql = oracle.deposit(x, y, ux, uy, cfg.q_particle, W.frame(cfg, 0), cfg.nx, cfg.ny,
                                 cfg.hx, cfg.hy)
    ctx = G.make_ctx(cfg)
    try:
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        part = _partial(torch, ctx)
        info = rp.rp_deposit(ctx, xd, yd, uxd, uyd, cfg.q_particle, W.frame(cfg, 0), part, info=True)
        b = torch.zeros(len(x), dtype=torch.int32, device="cuda")
        rp.rp_debug_bins(ctx, b)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(b.cpu().numpy(), bins)
        rp.rp_history_append(ctx, part, 1, W.frame(cfg, 0))
        Mg = _slot_moments(torch, ctx, cfg, 0)
        scale = np.abs(M).max()
        assert np.abs(Mg - M).max() <= 1e-12 * scale
        assert info.n_lost == int((bins < 0).sum())
        assert abs(info.q_lost - ql) < 1e-15
        tot = Mg[..., 0].sum() * cfg.hx * cfg.hy + info.q_lost
        assert abs(tot - 1.0) < 1e-12
    finally:
        rp.rp_destroy(ctx)


def test_rigid_prehistory_rotates_the_current(torch):
    """rp_history_init(rigid=1) on the bend (R-23): every pre-history level is the step-0
    deposit as the same comoving bunch in that level's frame (oracle.rigid_ring)."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    x, y, ux, uy = W.particles(cfg, n=20_000, seed=11)
    q = 1.0 / len(x)
    M, _, _ = oracle.deposit(x, y, ux, uy, q, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    want = oracle.rigid_ring(M, W.ring_frames(cfg, 0))
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, q, W.frame(cfg, 0))
        ring = torch.zeros((cfg.H, cfg.ny, cfg.nx, 4), dtype=torch.float64, device="cuda")
        rp.rp_save_state(ctx, ring)
        got = ring.cpu().numpy()
    finally:
        rp.rp_destroy(ctx)
    scale = np.abs(M).max()
    assert np.abs(got - want).max() <= 1e-12 * scale
    for l in range(-cfg.n_pre, 0):  # rho is a copy of slot 0 bit for bit
        np.testing.assert_array_equal(got[l % cfg.H, ..., 0], got[0, ..., 0])
    assert np.abs(got[1, ..., 2] - got[0, ..., 2]).max() > 0.05 * np.abs(got[0, ..., 1]).max()


def test_deposit_exact_for_any_particle_split(torch):
    """Exact fixed-point partial sums: depositing the bunch in one piece or
    split into 3 unequal rank shards and appending the partials gives a bit-identical D_k."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    x, y, ux, uy = W.particles(cfg, n=200_000, seed=11)
    q = 1.0 / len(x)
    fk = W.frame(cfg, 0)
    ctx1, ctx3 = G.make_ctx(cfg), G.make_ctx(cfg)
    try:
        d = _dev_arrays(torch, x, y, ux, uy)
        p1 = _partial(torch, ctx1)
        rp.rp_deposit(ctx1, *d, q, fk, p1)
        rp.rp_history_append(ctx1, p1, 1, fk)
        pb = rp.rp_partial_bytes(ctx3)
        p3 = _partial(torch, ctx3, 3)
        cuts = [0, 31_337, 150_001, len(x)]
        for r in range(3):
            sl = [t[cuts[r]:cuts[r + 1]].contiguous() for t in d]
            rp.rp_deposit(ctx3, *sl, q, fk, p3[r * pb:(r + 1) * pb])
        rp.rp_history_append(ctx3, p3, 3, fk)
        a, b = _slot_moments(torch, ctx1, cfg, 0), _slot_moments(torch, ctx3, cfg, 0)
        np.testing.assert_array_equal(a, b)
        assert np.abs(a).max() > 0
    finally:
        rp.rp_destroy(ctx1)
        rp.rp_destroy(ctx3)


def test_deposit_golden_ties(torch):
    import json, os
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "bins_ties.json")))
    x = np.array([c["x"] for c in g["cases"]])
    y = np.array([c["y"] for c in g["cases"]])
    z = np.zeros_like(x)
    ctx = rp.rp_create(g["nx"], g["ny"], g["hx"], g["hy"], 2, 1.0, 1.0, 1e-6)
    try:
        xd, yd, zd, zd2 = _dev_arrays(torch, x, y, z, z)
        part = _partial(torch, ctx)
        rp.rp_deposit(ctx, xd, yd, zd, zd2, 1.0, g["frame"], part)
        b = torch.zeros(len(x), dtype=torch.int32, device="cuda")
        rp.rp_debug_bins(ctx, b)
        np.testing.assert_array_equal(b.cpu().numpy(), [c["bin"] for c in g["cases"]])
    finally:
        rp.rp_destroy(ctx)


# ------------------------------------------------------------------ potentials
def _deposit_rigid_ring(cfg, n=None, seed=None):
    x, y, ux, uy = W.particles(cfg, n=n, seed=seed)
    q = 1.0 / len(x)
    M, _, _ = oracle.deposit(x, y, ux, uy, q, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    return oracle.rigid_ring(M, W.ring_frames(cfg, 0)), (x, y, ux, uy, q)


def test_potentials_static_cfg1_full_mesh(torch):
    """Config 1 (BASELINE.json configs[0]), step 0 with rigid pre-history, every mesh point."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    ring, _ = _deposit_rigid_ring(cfg)
    frames = W.ring_frames(cfg, 0)
    pts = np.arange(cfg.nx * cfg.ny)
    orc = G.oracle_problem(cfg, ring, frames, 0, cfg.n_pre).potentials(pts)
    ctx = G.make_ctx(cfg)
    try:
        G.load_state(ctx, cfg, 0, cfg.n_pre, ring, frames)
        gpu, info = G.gpu_potentials(ctx, len(pts))
        fail, worst, nties = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (np.nonzero(fail)[0][:10], worst)
        assert worst < G.REL
        assert info.segments == int(orc["nseg"].sum())
        assert info.capped == int(orc["capped"].sum())
        assert info.evals == int(orc["evals"].sum())
        assert info.kappa == cfg.kappa_max
    finally:
        rp.rp_destroy(ctx)


def test_potentials_bend_cfg2_full_size_sampled(torch):
    """Config 2 (the bench workload) at full size through the product path: GPU deposit of
    1e6 particles + rigid pre-history + potentials on the whole 64x64 mesh in the bench's
    launch configuration; the oracle computes a stratified sample of points."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    ring, (x, y, ux, uy, q) = _deposit_rigid_ring(cfg)
    pts = W.sample_points(cfg.nx, cfg.ny, 128, seed=5)
    orc = G.oracle_problem(cfg, ring, W.ring_frames(cfg, 0), 0, cfg.n_pre).potentials(pts)
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_schedule(ctx, rp.RP_SCHED_SUBREGION, 1)  # bench.py's launch configuration
        pre = W.frames(cfg, range(-cfg.n_pre, 0))
        rp.rp_history_init(ctx, cfg.n_pre, pre, None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, q, W.frame(cfg, 0))
        gpu, info = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        fail, worst, nties = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (pts[fail][:10], worst)
        assert np.isfinite(gpu["phi"]).all()
    finally:
        rp.rp_destroy(ctx)


def _bend_small(n=24, kap=60):
    c = W.config(2)
    return W.Config(number=2, name="bend-small", nx=n, ny=n, n_particles=1, steps=kap,
                    kappa_max=kap, geometry="bend", sigma=c.sigma, cdt=c.cdt, gamma0=c.gamma0,
                    r0=c.r0, sigma_xp=c.sigma_xp, q_over_mc=c.q_over_mc)


@pytest.mark.parametrize("rule,interp", [(0, 0), (1, 0), (0, 1)])
def test_potentials_bend_small_full_mesh_two_steps(torch, rule, interp):
    """Moving frames, node-sampled history with a time-varying amplitude, two consecutive
    steps (the second uses the first step's counts as the schedule forecast); GK15, the
    paper's Simpson rule (R-22) and the Lagrange-3 spatial stencil (R-25)."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    # Lagrange-3 is discontinuous (R-25): its trees chase the jumps to D_max, so the oracle
    # needs a smaller mesh and cap to finish in seconds (D_max = 30 at 24^2: > 20 min)
    cfg = _bend_small(12, 20) if interp else _bend_small()
    cfg.rule = rule
    cfg.interp = interp
    if interp:
        cfg.max_depth = 14
    ctx = G.make_ctx(cfg)
    try:
        for k in (5, 6):
            ring = W.node_gaussian_ring(cfg, k=k, beta=(cfg.beta0, 0.01),
                                        amp_of_level=lambda l: 1.0 + 0.01 * l)
            frames = W.ring_frames(cfg, k)
            pts = np.arange(cfg.nx * cfg.ny)
            orc = G.oracle_problem(cfg, ring, frames, k, cfg.n_pre).potentials(pts)
            G.load_state(ctx, cfg, k, cfg.n_pre, ring, frames)
            gpu, info = G.gpu_potentials(ctx, len(pts))
            fail, worst, nties = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
            assert not fail.any(), (np.nonzero(fail)[0][:10], worst)
    finally:
        rp.rp_destroy(ctx)


def test_subtree_units_match_the_unsplit_walk(torch):
    """Deep trees split into subtree work units walk the same canonical tree:
    equal segment counts per point and values equal to the single-warp walk up to the
    summation grouping (config 2 at full size, the bench workload).  With a per-item budget
    of 2 units every further level-11 split of a near-field item descends in place (the
    budget-full path): same tree, fewer units."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    ring, _ = _deposit_rigid_ring(cfg)
    frames = W.ring_frames(cfg, 0)
    out = {}
    for split, budget in ((12, 0), (12, 2), (0, 0)):
        ctx = G.make_ctx(cfg)
        try:
            rp.rp_set_work_split(ctx, split, budget)
            G.load_state(ctx, cfg, 0, cfg.n_pre, ring, frames)
            out[(split, budget)] = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        finally:
            rp.rp_destroy(ctx)
    b, ib = out[(0, 0)]
    assert ib.units == 0
    for key in ((12, 0), (12, 2)):
        a, ia = out[key]
        assert ia.units > 1000
        for k in ("nseg", "nleaf", "capped"):
            np.testing.assert_array_equal(a[k], b[k])
        assert ia.evals == ib.evals and ia.leaves == ib.leaves and ia.capped == ib.capped
        scale = max(np.abs(b["phi"]).max(), np.abs(b["ax"]).max(), np.abs(b["ay"]).max())
        # the leaf error estimate eps is merged from the units like the values
        for k in ("phi", "ax", "ay", "err"):
            assert np.abs(a[k] - b[k]).max() <= 1e-13 * scale, (key, k)
    # the budget binds: at most 2 units per near-field item, fewer than the default budget's
    assert out[(12, 2)][1].units < out[(12, 0)][1].units
    assert out[(12, 2)][1].units <= 2 * cfg.nx * cfg.ny


@pytest.mark.parametrize("which", ["bend_small", "cfg2_sampled"])
def test_support_clip_bit_exact(torch, which):
    """Step a5 (R-5): the GPU's per-(point, subregion) support [A, B] equals the oracle's clip
    bit for bit (both follow the same operation order in IEEE round-to-nearest), including
    which items are empty."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    if which == "bend_small":
        cfg = _bend_small()
        k = 5
        ring = W.node_gaussian_ring(cfg, k=k, beta=(cfg.beta0, 0.01),
                                    amp_of_level=lambda l: 1.0 + 0.01 * l)
        frames = W.ring_frames(cfg, k)
    else:
        cfg = W.config(2)
        k = 0
        ring, _ = _deposit_rigid_ring(cfg, n=20_000, seed=3)
        frames = W.ring_frames(cfg, 0)
    ctx = G.make_ctx(cfg)
    try:
        G.load_state(ctx, cfg, k, cfg.n_pre, ring, frames)
        gpu, info = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        ab = torch.zeros(cfg.nx * cfg.ny * cfg.kappa_max * 2, dtype=torch.float64, device="cuda")
        rp.rp_debug_clip(ctx, ab)
        ab = ab.cpu().numpy().reshape(cfg.nx * cfg.ny, cfg.kappa_max, 2)
    finally:
        rp.rp_destroy(ctx)
    P = G.oracle_problem(cfg, ring, frames, k, cfg.n_pre)
    kap = P.kappa()
    assert kap == info.kappa and kap > 0
    rng = np.random.default_rng(1)
    items = [(p, j) for p in range(cfg.nx * cfg.ny) for j in range(kap)]
    if len(items) > 30_000:
        items = [items[i] for i in rng.choice(len(items), 30_000, replace=False)]
    nonempty = 0
    for p, j in items:
        c = P.clip(*P.mesh_point(p % cfg.nx, p // cfg.nx), j)
        want = (0.0, 0.0) if c is None else c
        assert ab[p, j, 0] == want[0] and ab[p, j, 1] == want[1], (p, j, ab[p, j], c)
        nonempty += c is not None
    assert nonempty > 100


@pytest.mark.parametrize("variant", [dict(n_root=1), dict(max_depth=5), dict(n_theta=16),
                                     dict(rule=1), dict(rule=1, n_root=1),
                                     dict(interp=1, max_depth=12),
                                     dict(interp=1, n_theta=16, max_depth=12)])
def test_potentials_variants(torch, variant):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.Config(number=0, name="v", nx=20, ny=13, n_particles=4000, steps=4, kappa_max=7,
                   geometry="static", sigma=1.0, cdt=1.9, **variant)
    ring, _ = _deposit_rigid_ring(cfg, n=4000, seed=9)
    frames = W.ring_frames(cfg, 3)
    pts = np.arange(cfg.nx * cfg.ny)
    orc = G.oracle_problem(cfg, ring, frames, 3, 0).potentials(pts)
    ctx = G.make_ctx(cfg)
    try:
        G.load_state(ctx, cfg, 3, 0, ring, frames)
        gpu, info = G.gpu_potentials(ctx, len(pts))
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (np.nonzero(fail)[0][:10], worst)
        if "max_depth" in variant:
            assert info.capped > 0 and info.capped == int(orc["capped"].sum())
    finally:
        rp.rp_destroy(ctx)


def test_potentials_degenerate_kappa_zero_and_min_grid(torch):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.Config(number=0, name="min", nx=4, ny=4, n_particles=50, steps=3, kappa_max=2,
                   geometry="static", sigma=0.3, cdt=0.5)
    x, y, ux, uy = W.particles(cfg, n=50, seed=1)
    ctx = G.make_ctx(cfg)
    try:
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        for k in range(3):
            rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, 1.0 / 50, W.frame(cfg, k))
            gpu, info = G.gpu_potentials(ctx, 16)
            if k < 2:  # no pre-history: kappa(k) = k - 1 <= 0 -> nothing to integrate (R-3)
                assert info.kappa == 0 and (gpu["phi"] == 0).all() and (gpu["nseg"] == 0).all()
        # k = 2: kappa = 1, compare with the oracle on the ring the GPU was given
        ring = np.zeros((cfg.H, 4, 4, 4))
        M, _, _ = oracle.deposit(x, y, ux, uy, 1.0 / 50, W.frame(cfg, 0), 4, 4, cfg.hx, cfg.hy)
        for l in range(3):
            ring[l % cfg.H] = M
        orc = G.oracle_problem(cfg, ring, W.ring_frames(cfg, 2), 2, 0).potentials(np.arange(16))
        fail, worst, _ = G.compare_potentials(gpu, orc, np.arange(16), tau=cfg.tau)
        assert not fail.any(), worst
    finally:
        rp.rp_destroy(ctx)


# ------------------------------------------------------------------ analytic sources
@pytest.mark.parametrize("kind", ["gauss", "disk"])
def test_analytic_sources_closed_form_on_gpu(torch, kind):
    import scipy.special as sp
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    sq = math.sqrt(math.pi / 2)
    if kind == "gauss":
        cfg = W.Config(number=0, name="g", nx=9, ny=9, n_particles=1, steps=1, kappa_max=12,
                       geometry="static", sigma=1.0, cdt=1.6)
        src = dict(kind=rp.RP_SRC_GAUSS, x0=0.0, y0=0.0, width=1.0, q=1.0, bx=0.3, by=-0.2)
        okind = oracle.SRC_GAUSS
    else:
        cfg = W.Config(number=0, name="d", nx=9, ny=9, n_particles=1, steps=1, kappa_max=12,
                       geometry="static", sigma=1.0, cdt=0.8)
        src = dict(kind=rp.RP_SRC_DISK, x0=0.0, y0=0.0, width=1.0, q=1.0, bx=0.0, by=0.0)
        okind = oracle.SRC_DISK
    # mesh nodes at (ix*h - 5, iy*h - 5) with h = 10/8: the source at the origin
    ring = np.zeros((cfg.H, cfg.ny, cfg.nx, 4))
    frames = W.ring_frames(cfg, 20)
    ctx = G.make_ctx(cfg, tau=1e-6 * sq if kind == "gauss" else 1e-6)
    try:
        G.load_state(ctx, cfg, 20, 0, ring, frames)
        d = {k: torch.zeros(81, dtype=torch.float64, device="cuda") for k in ("phi", "ax", "ay", "err")}
        nseg = torch.zeros(81, dtype=torch.int32, device="cuda")
        # analytic source centre in frame-local coordinates: the lab origin = local (5, 5)
        rp.rp_debug_potentials_analytic(ctx, src["kind"], 5.0, 5.0, src["width"], src["q"],
                                        src["bx"], src["by"], None, d["phi"], d["ax"], d["ay"],
                                        d["err"], nseg)
        gpu = {k: v.cpu().numpy() for k, v in d.items()}
        gpu["nseg"] = nseg.cpu().numpy()
        P = G.oracle_problem(cfg, None, frames, 20, 0, source=okind, x0=5.0, y0=5.0,
                             width=src["width"], q=src["q"], bx=src["bx"], by=src["by"],
                             tau=1e-6 * sq if kind == "gauss" else 1e-6)
        pts = np.arange(81)
        orc = P.potentials(pts)
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=P.params.tau)
        assert not fail.any(), worst
        for p in pts:
            px, py = P.mesh_point(p % 9, p // 9)
            s = math.hypot(px, py)
            if kind == "gauss":
                exact = sq * sp.i0e(s * s / 4)
            elif s < 1:
                exact = 4 * sp.ellipe(s * s)
            elif s == 1:
                exact = 4.0
            else:
                exact = 4 * s * (sp.ellipe(1 / s ** 2) - (1 - 1 / s ** 2) * sp.ellipk(1 / s ** 2))
            assert abs(gpu["phi"][p] - exact) < 1e-6
    finally:
        rp.rp_destroy(ctx)


# ------------------------------------------------------------------ fields and push
def test_fields_parity(torch):
    """k_fields vs orc_fields from common inputs (R-15b: order-m backward differences of the node
    values and positions, m = 0..4), 1e-11 relative."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = _bend_small(n=17, kap=6)
    rng = np.random.default_rng(21)
    npts = cfg.nx * cfg.ny
    sh = (cfg.ny, cfg.nx)
    phi, ax, ay = (rng.standard_normal(npts) for _ in range(3))
    prev = rng.standard_normal((4, 2, npts))
    k = 5
    ctx = G.make_ctx(cfg)
    try:
        ring = np.zeros((cfg.H, cfg.ny, cfg.nx, 4))
        G.load_state(ctx, cfg, k, 0, ring, W.ring_frames(cfg, k))
        d = _dev_arrays(torch, phi, ax, ay, prev)
        out = [torch.zeros(npts, dtype=torch.float64, device="cuda") for _ in range(3)]
        for m in range(5):
            frames = [W.frame(cfg, k - j) for j in range(m + 1)]
            want = oracle.fields(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.c, cfg.dt, frames,
                                 phi.reshape(sh), ax.reshape(sh), ay.reshape(sh),
                                 [(prev[j, 0].reshape(sh), prev[j, 1].reshape(sh)) for j in range(m)])
            rp.rp_compute_fields(ctx, d[0], d[1], d[2], d[3][:m].contiguous() if m else None, *out)
            for got, w in zip(out, want):
                g = got.cpu().numpy().reshape(sh)
                assert np.abs(g - w).max() <= 1e-11 * np.abs(w).max(), m
    finally:
        rp.rp_destroy(ctx)


def test_push_parity(torch):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    x, y, ux, uy = W.particles(cfg, n=200_000, seed=3)
    rng = np.random.default_rng(4)
    npts = cfg.nx * cfg.ny
    scale = 1e8
    ex, ey, bz = (scale * rng.standard_normal(npts) for _ in range(3))
    fk = W.frame(cfg, 0)
    want = oracle.push(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.c, cfg.dt, fk, x, y, ux, uy,
                       cfg.q_over_mc, cfg.bz_ext, ex, ey, bz)
    ctx = G.make_ctx(cfg)
    try:
        ring = np.zeros((cfg.H, cfg.ny, cfg.nx, 4))
        G.load_state(ctx, cfg, 0, 0, ring, W.ring_frames(cfg, 0))
        xd, yd, uxd, uyd, exd, eyd, bzd = _dev_arrays(torch, x, y, ux, uy, ex, ey, bz)
        rp.rp_push_particles(ctx, xd, yd, uxd, uyd, cfg.q_over_mc, cfg.bz_ext, exd, eyd, bzd)
        got = [t.cpu().numpy() for t in (xd, yd, uxd, uyd)]
        # positions: absolute 1e-13 of the orbit scale; momenta: 1e-13 relative
        assert np.abs(got[0] - want[0]).max() < 1e-13 * cfg.r0 * 1e-2 + 1e-15
        assert np.abs(got[1] - want[1]).max() < 1e-13 * cfg.r0 * 1e-2 + 1e-15
        assert np.abs(got[2] - want[2]).max() < 1e-13 * np.abs(want[2]).max()
        assert np.abs(got[3] - want[3]).max() < 1e-13 * np.abs(want[2]).max()
    finally:
        rp.rp_destroy(ctx)


def test_particle_forces_parity(torch):
    """rp_particle_forces (E + beta x B gathered at the particles) against orc_forces, the
    particle-level force of the paper's validation; 1e-13 relative."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    x, y, ux, uy = W.particles(cfg, n=200_000, seed=3)
    rng = np.random.default_rng(6)
    npts = cfg.nx * cfg.ny
    ex, ey, bz = (1e3 * rng.standard_normal(npts) for _ in range(3))
    fk = W.frame(cfg, 0)
    want = oracle.forces(cfg.nx, cfg.ny, cfg.hx, cfg.hy, fk, x, y, ux, uy, cfg.bz_ext, ex, ey, bz)
    ctx = G.make_ctx(cfg)
    try:
        ring = np.zeros((cfg.H, cfg.ny, cfg.nx, 4))
        G.load_state(ctx, cfg, 0, 0, ring, W.ring_frames(cfg, 0))
        xd, yd, uxd, uyd, exd, eyd, bzd = _dev_arrays(torch, x, y, ux, uy, ex, ey, bz)
        fx, fy = (torch.zeros(len(x), dtype=torch.float64, device="cuda") for _ in range(2))
        rp.rp_particle_forces(ctx, xd, yd, uxd, uyd, cfg.bz_ext, exd, eyd, bzd, fx, fy)
        for g, w in zip((fx, fy), want):
            g = g.cpu().numpy()
            assert np.abs(g - w).max() <= 1e-13 * np.abs(w).max()
    finally:
        rp.rp_destroy(ctx)


def test_kick_external_parity(torch):
    """rp_kick_external (the deposit's time-centred momenta, R-27) against orc_kick_external on
    the bend bunch with its dipole field; 1e-13 relative."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    _, _, ux, uy = W.particles(cfg, n=100_000, seed=3)
    want = oracle.kick_external(cfg.dt, ux, uy, cfg.q_over_mc, cfg.bz_ext, 0.5)
    ctx = G.make_ctx(cfg)
    try:
        uxd, uyd = _dev_arrays(torch, ux, uy)
        ox, oy = torch.empty_like(uxd), torch.empty_like(uyd)
        rp.rp_kick_external(ctx, uxd, uyd, cfg.q_over_mc, cfg.bz_ext, 0.5, ox, oy)
        for g, w in zip((ox, oy), want):
            assert np.abs(g.cpu().numpy() - w).max() <= 1e-13 * np.abs(want[0]).max()
        # it turns the momenta from the tangent at -dt/2 onto the tangent at 0 (R-21, R-27)
        ang = np.arctan2(oy.cpu().numpy(), ox.cpu().numpy())
        assert abs(np.median(ang)) < 1e-6 < abs(np.median(np.arctan2(uy, ux)))
    finally:
        rp.rp_destroy(ctx)


# ------------------------------------------------------------------ sharding, e2e, loop
def test_shard_path_equals_full_mesh(torch):
    """Mesh-point sharding simulated on one GPU: ranks 0..W-1 each compute
    their shard; the scattered result is bit-identical to the single-call result."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    ring, _ = _deposit_rigid_ring(cfg)
    frames = W.ring_frames(cfg, 0)
    ctx = G.make_ctx(cfg)
    try:
        G.load_state(ctx, cfg, 0, cfg.n_pre, ring, frames)
        full, _ = G.gpu_potentials(ctx, 1024)
        for world in (2, 3, 8):
            for step in range(2):  # second pass uses the counts as the shard forecast
                cap = rp.rp_shard_capacity(ctx, world)
                shards = torch.zeros((world, cap, 6), dtype=torch.float64, device="cuda")
                tot = 0
                for r in range(world):
                    n, _ = rp.rp_compute_potentials_shard(ctx, r, world, shards[r])
                    tot += n
                assert tot == 1024
                out = {k: torch.zeros(1024, dtype=torch.float64, device="cuda") for k in ("phi", "ax", "ay", "err")}
                nseg = torch.zeros(1024, dtype=torch.int32, device="cuda")
                rp.rp_shard_scatter(ctx, shards, world, out["phi"], out["ax"], out["ay"], out["err"], nseg)
                for k in ("phi", "ax", "ay", "err"):
                    np.testing.assert_array_equal(out[k].cpu().numpy(), full[k])
                np.testing.assert_array_equal(nseg.cpu().numpy(), full["nseg"])
    finally:
        rp.rp_destroy(ctx)


def test_step_host_matches_device_path(torch):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    x, y, ux, uy = W.particles(cfg)
    q = cfg.q_particle
    pre = W.frames(cfg, range(-cfg.n_pre, 0))
    # device path
    ctx = G.make_ctx(cfg)
    ctx2 = G.make_ctx(cfg)
    try:
        rp.rp_history_init(ctx, cfg.n_pre, pre, None, True)
        rp.rp_history_init(ctx2, cfg.n_pre, pre, None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        n = cfg.nx * cfg.ny
        phi, ax, ay, ex, ey, bz = (torch.zeros(n, dtype=torch.float64, device="cuda") for _ in range(6))
        ahist = torch.zeros((4, 2, n), dtype=torch.float64, device="cuda")
        hx, hy, hux, huy = (torch.tensor(a).pin_memory() for a in (x, y, ux, uy))
        mesh = torch.zeros((6, n), dtype=torch.float64).pin_memory()
        for k in range(6):
            cux, cuy = torch.empty_like(uxd), torch.empty_like(uyd)
            rp.rp_kick_external(ctx, uxd, uyd, cfg.q_over_mc, 0.0, 0.5, cux, cuy)
            rp.rp_deposit_step(ctx, xd, yd, cux, cuy, q, W.frame(cfg, k))
            rp.rp_compute_potentials(ctx, phi, ax, ay)
            rp.rp_compute_fields(ctx, phi, ax, ay, ahist[:min(k, 4)].contiguous() if k else None,
                                 ex, ey, bz)
            ahist[1:] = ahist[:-1].clone()
            ahist[0, 0].copy_(ax); ahist[0, 1].copy_(ay)
            rp.rp_push_particles(ctx, xd, yd, uxd, uyd, cfg.q_over_mc, 0.0, ex, ey, bz)
            rp.rp_step_host(ctx2, hx, hy, hux, huy, q, W.frame(cfg, k), cfg.q_over_mc, 0.0, mesh)
            torch.cuda.synchronize()
            for i, t in enumerate((phi, ax, ay, ex, ey, bz)):
                np.testing.assert_array_equal(mesh[i].numpy(), t.cpu().numpy())
            np.testing.assert_array_equal(hx.numpy(), xd.cpu().numpy())
        assert rp.rp_launch_count(ctx) > 0
    finally:
        rp.rp_destroy(ctx)
        rp.rp_destroy(ctx2)


def test_call_order_errors(torch):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    ctx = G.make_ctx(cfg)
    try:
        z = torch.zeros(1024, dtype=torch.float64, device="cuda")
        with pytest.raises(rp.RpError) as e:
            rp.rp_compute_potentials(ctx, z, z, z)
        assert e.value.code == -5
        x = torch.zeros(10, dtype=torch.float64, device="cuda")
        rp.rp_deposit_step(ctx, x, x, x, x, 0.1, W.frame(cfg, 0))
        with pytest.raises(rp.RpError) as e:
            rp.rp_history_init(ctx, 2, W.frames(cfg, [-2, -1]), None, True)
        assert e.value.code == -5
    finally:
        rp.rp_destroy(ctx)


# ------------------------------------------------------------------ more product-path cases
def test_history_init_explicit_grids_and_empty_deposit(torch):
    """rp_history_init with explicit pre-history grids (rigid = 0), then a step whose local
    deposit is empty (0 particles): the potentials come from the pre-history alone."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = _bend_small(n=20, kap=12)
    ring = W.node_gaussian_ring(cfg, k=0, beta=(cfg.beta0, 0.0), amp_of_level=lambda l: 1.0 + 0.02 * l)
    n_pre = cfg.kappa_max + 1
    pre_levels = list(range(-n_pre, 0))
    grids = np.stack([ring[l % cfg.H] for l in pre_levels])
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_history_init(ctx, n_pre, W.frames(cfg, pre_levels),
                           torch.tensor(grids, dtype=torch.float64, device="cuda"), False)
        z = torch.zeros(0, dtype=torch.float64, device="cuda")
        info = rp.rp_deposit_step(ctx, z, z, z, z, 1.0, W.frame(cfg, 0), info=True)
        assert info.n_lost == 0 and info.q_total == 0.0
        gpu, _ = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        full = ring.copy()
        full[0 % cfg.H] = 0.0  # step 0 grid is empty
        pts = np.arange(cfg.nx * cfg.ny)
        orc = G.oracle_problem(cfg, full, W.ring_frames(cfg, 0), 0, n_pre).potentials(pts)
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), worst
    finally:
        rp.rp_destroy(ctx)


@pytest.mark.slow
def test_potentials_bend_cfg3_full_size_sampled(torch):
    """Config 3 (128x128, 1e7 particles, full history kappa = 500) through the product path;
    the oracle computes a stratified sample of 128 points from its own deposit."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(3)
    ring, (x, y, ux, uy, q) = _deposit_rigid_ring(cfg)
    pts = W.sample_points(cfg.nx, cfg.ny, 128, seed=9)
    orc = G.oracle_problem(cfg, ring, W.ring_frames(cfg, 0), 0, cfg.n_pre).potentials(pts)
    del ring
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_schedule(ctx, rp.RP_SCHED_SUBREGION, 1)  # bench.py's launch configuration
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, q, W.frame(cfg, 0))
        gpu, info = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (pts[fail][:10], worst)
        assert info.kappa == cfg.kappa_max
        assert info.units > 0
    finally:
        rp.rp_destroy(ctx)


@pytest.mark.slow
def test_potentials_bend_cfg4_full_size_sampled(torch):
    """Config 4 (256x256, 1e8 particles, full history kappa = 1000: BASELINE.json configs[3])
    through the product path on one GPU; the oracle computes 64 stratified points from its own
    deposit of the same 1e8 particles (2.1 GB ring on the host)."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(4)
    ring, (x, y, ux, uy, q) = _deposit_rigid_ring(cfg)
    pts = W.sample_points(cfg.nx, cfg.ny, 64, seed=13)
    orc = G.oracle_problem(cfg, ring, W.ring_frames(cfg, 0), 0, cfg.n_pre).potentials(pts)
    del ring
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_schedule(ctx, rp.RP_SCHED_SUBREGION, 1)  # bench.py's launch configuration
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        del x, y, ux, uy
        rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, q, W.frame(cfg, 0))
        del xd, yd, uxd, uyd
        gpu, info = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (pts[fail][:10], worst)
        assert info.kappa == cfg.kappa_max
        assert info.units > 0
    finally:
        rp.rp_destroy(ctx)


@pytest.mark.slow
def test_potentials_bend_cfg5_full_size_sampled(torch):
    """Config 5 (512x512, 1e8 particles, kappa = 2000: BASELINE.json configs[4]) on one GPU
    (76 GB of HBM), the oracle on 48 stratified points with a 16.8 GB host ring."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(5)
    ring, (x, y, ux, uy, q) = _deposit_rigid_ring(cfg)
    pts = W.sample_points(cfg.nx, cfg.ny, 48, seed=17)
    orc = G.oracle_problem(cfg, ring, W.ring_frames(cfg, 0), 0, cfg.n_pre).potentials(pts)
    del ring
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_schedule(ctx, rp.RP_SCHED_SUBREGION, 1)  # bench.py's launch configuration
        rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        xd, yd, uxd, uyd = _dev_arrays(torch, x, y, ux, uy)
        del x, y, ux, uy
        rp.rp_deposit_step(ctx, xd, yd, uxd, uyd, q, W.frame(cfg, 0))
        del xd, yd, uxd, uyd
        gpu, info = G.gpu_potentials(ctx, cfg.nx * cfg.ny)
        fail, worst, _ = G.compare_potentials(gpu, orc, pts, tau=cfg.tau)
        assert not fail.any(), (pts[fail][:10], worst)
        assert info.kappa == cfg.kappa_max
        assert info.units > 0
    finally:
        rp.rp_destroy(ctx)


@pytest.mark.parametrize("policy,k", [(0, 1), (2, 9), (2, 25), (2, 5), (3, 1)])
def test_schedule_policies_bit_identical(torch, policy, k):
    """The forecast (paper's predictor g) only orders the work: every policy gives
    bit-identical results to the default persistence forecast over several steps."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
    cfg = W.config(1)
    a, b = Simulation(cfg), Simulation(cfg)
    try:
        rp.rp_set_schedule(b.ctx, policy, k)
        for _ in range(3):
            a.step()
            b.step()
            for t1, t2 in ((a.phi, b.phi), (a.ax, b.ax), (a.ay, b.ay), (a.nseg, b.nseg), (a.ex, b.ex)):
                assert torch.equal(t1, t2)
    finally:
        a.close()
        b.close()


def _bench(args, env=None, timeout=900):
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    e = dict(os.environ)
    e.update(env or {})
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args],
                         capture_output=True, text=True, timeout=timeout, env=e)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.strip().startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_json_contract(torch):
    """bench.py prints one JSON line with the keys the driver and the judge read; with
    RP_DIST_BACKEND=gloo, `--gpus 2` (self-spawned, two ranks sharing the test GPU) gives the
    same result bytes as one GPU."""
    d = _bench(["--config", "1", "--steps", "2", "--warmup", "3"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "gpu_launches", "clocks",
              "e2e", "cpu_baseline", "evals_per_s", "result_sha256"):
        assert k in d, k
    assert d["value"] > 0 and d["steps"] == 2 and d["warmup"] == 3 and d["dtype"] == "f64"
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1.2 and r["peak"] > 30
    assert d["gpu_launches"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and 0 < d["e2e"]["value"] <= d["value"] * 1.001
    assert d["config"]["workload"] == "cfg1-32x32-static"
    c = d["cpu_baseline"]
    assert c["kind"] == "oracle" and c["evals_per_s"] > 0 and "step 4" in c["sample"]
    d2 = _bench(["--config", "1", "--steps", "2", "--warmup", "3", "--gpus", "2"],
                env={"RP_DIST_BACKEND": "gloo"})
    assert d2["n_gpus"] == 2 and d2["result_sha256"] == d["result_sha256"]
    assert "gloo" in d2["config"]["transport"]
