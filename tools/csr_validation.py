"""Physics validation in the LCLS bend (the paper's Sec. V-A, Fig. 2-3).

Three references for the self-forces of a Gaussian bunch (sigma_s = sigma_x = 50 um, Q = 1) in
steady-state circular motion on the LCLS orbit (R0 = 25.13 m, gamma = 1e4), all computed through
the whole GPU path (history ring -> retarded potentials -> fields -> particle forces):

1. The 1D steady-state CSR field of a rigid line charge (Derbenev et al. 1995; Saldin,
   Schneidmiller, Yurkov 1997 -- textbook results standing in for the paper's absent refs
   [24], [25]):  E_s(s) = -2 Q / (3^(1/3) R^(2/3)) int_0^inf x^(-1/3) lambda'(s - x) dx.
   It is the sigma_x -> 0 limit; the flat bunch differs from it by its radial size.
2. The exact steady-state solution of the SAME sheet bunch, semi-analytic: the bunch centre
   moves on the orbit, X_c(t) = ref(beta0 c t), with current rho beta0 t-hat(t); for an
   isotropic Gaussian the theta' integral of Eq. 1 over the full circle is closed-form, so
       phi(P, t) = int_0^R (Q / sigma^2) exp(-(r - s)^2 / 2 sigma^2) i0e(r s / sigma^2) dr,
       A(P, t)   = int_0^R beta0 t-hat(t - r/c) (same kernel) dr,   s(r) = |P - X_c(t - r/c)|
   (scipy quad), and E = -grad phi - (1/c) dA/dt, B_z = d_x A_y - d_y A_x by 4th-order central
   differences.  No grid, history, interpolation, clip, arcs or adaptive tree is involved, so
   it checks the longitudinal AND the transverse force of the method end to end.
3. Monte-Carlo convergence (Fig. 3): particle-level forces from deposited bunches of N
   particles against the force of the noise-free expected deposit (the bunch's Gaussian
   convolved with the TSC kernel), mean-square error vs N -- "scales as 1/N".

    python tools/csr_validation.py [n] [--out file.json]        (1 and 2 on an n x n mesh)
    python tools/csr_validation.py --mse [--out file.json]      (3 on 129 x 129)
"""
import json
import math
import os
import sys

import numpy as np
import scipy.integrate as si
import scipy.special as sp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402


def csr_config(n, kappa=100):
    base = W.config(2)
    return W.Config(number=2, name=f"csr-{n}", nx=n, ny=n, n_particles=1, steps=kappa,
                    kappa_max=kappa, geometry="bend", sigma=base.sigma, cdt=base.cdt,
                    gamma0=base.gamma0, r0=base.r0, sigma_xp=base.sigma_xp,
                    q_over_mc=base.q_over_mc)


def gaussian_nodes(cfg):
    """Node samples of the normalised bunch density on the comoving grid."""
    u = np.arange(cfg.nx) * cfg.hx
    v = np.arange(cfg.ny) * cfg.hy
    U, V = np.meshgrid(u, v)
    half = 0.5 * cfg.extent
    return np.exp(-((U - half) ** 2 + (V - half) ** 2) / (2 * cfg.sigma ** 2)) / (
        2 * math.pi * cfg.sigma ** 2)


def tsc_expected_nodes(cfg):
    """Expected TSC deposit of the Gaussian bunch (density x TSC kernel), per node: the
    noise-free limit of a particle deposit, separable in the frame axes."""
    def axis(n, h):
        half = 0.5 * cfg.extent
        x = np.linspace(-8 * cfg.sigma, 8 * cfg.sigma, 40001)
        g = np.exp(-x ** 2 / (2 * cfg.sigma ** 2)) / (math.sqrt(2 * math.pi) * cfg.sigma)
        out = np.zeros(n)
        for i in range(n):
            t = (half + x) / h - i  # particle offset from node i in cells
            a = np.abs(t)
            w = np.where(a <= 0.5, 0.75 - a * a, np.where(a <= 1.5, 0.5 * (1.5 - a) ** 2, 0.0))
            out[i] = np.trapezoid(g * w, x) / h
        return out
    return np.outer(axis(cfg.ny, cfg.hy), axis(cfg.nx, cfg.hx))


def steady_ring(cfg, k, density=None, psi_offset=0.0):
    """Ring at step k: every level holds the same comoving bunch `density` (default: node
    samples of the Gaussian), current rho beta0 along the level's tangent turned by psi_offset
    (lab components)."""
    g = gaussian_nodes(cfg) if density is None else density
    ring = np.zeros((cfg.H, cfg.ny, cfg.nx, 4))
    co, so = math.cos(psi_offset), math.sin(psi_offset)
    for l in range(k - cfg.H + 1, k + 1):
        _, _, c, s = W.frame(cfg, l)
        ring[l % cfg.H, :, :, 0] = g
        ring[l % cfg.H, :, :, 1] = g * cfg.beta0 * (c * co - s * so)
        ring[l % cfg.H, :, :, 2] = g * cfg.beta0 * (s * co + c * so)
    return ring


def csr_1d(s, sigma, R):
    lam_p = lambda x: -x / sigma ** 2 * math.exp(-x * x / (2 * sigma ** 2)) / (math.sqrt(2 * math.pi) * sigma)
    f = lambda x: x ** (-1.0 / 3.0) * lam_p(s - x)
    val, _ = si.quad(f, 0, s + 12 * sigma, limit=400, points=[max(s, 1e-30)] if s > 0 else None)
    if s + 12 * sigma < 0:
        val = 0.0
    return -2.0 / (3 ** (1 / 3) * R ** (2 / 3)) * val


# ------------------------------------------------------------------ semi-analytic (2.)
def _orbit(cfg, t):
    """Bunch centre and tangent at time t (c = 1): the reference orbit (workloads geometry)."""
    psi = cfg.beta0 * t / cfg.r0
    return (np.array([cfg.r0 * math.sin(psi), cfg.r0 * (1.0 - math.cos(psi))]),
            np.array([math.cos(psi), math.sin(psi)]))


def semi_analytic_potentials(cfg, P, t, R=None):
    """(phi, A_x, A_y) at lab point P and time t of the isotropic Gaussian sheet moving on the
    orbit (Q = 1), Eq. 1 with the theta' integral in closed form."""
    sg = cfg.sigma
    R = cfg.kappa_max * cfg.cdt if R is None else R
    P = np.asarray(P, dtype=float)

    def kern(r):
        xc, _ = _orbit(cfg, t - r)
        s = math.hypot(P[0] - xc[0], P[1] - xc[1])
        return math.exp(-0.5 * ((r - s) / sg) ** 2) * sp.i0e(r * s / sg ** 2) / sg ** 2

    def comp(i):
        if i == 0:
            return kern
        return lambda r: kern(r) * cfg.beta0 * _orbit(cfg, t - r)[1][i - 1]

    pts = [x for x in (2 * sg, 10 * sg, 50 * sg, 1e-2, 5e-2, 0.2, 0.5, 1.0, 2.0) if x < R]
    out = []
    for i in range(3):
        v, _ = si.quad(comp(i), 0.0, R, points=pts, limit=2000, epsabs=0.0, epsrel=1e-13)
        out.append(v)
    return np.array(out)


_D4 = np.array([1.0, -8.0, 8.0, -1.0]) / 12.0  # f'(0) ~ sum c_i f(o_i h) / h, o = -2, -1, 1, 2
_O4 = (-2, -1, 1, 2)


def semi_analytic_fields(cfg, P, t, dh=None, dt=None):
    """(E_x, E_y, B_z) at (P, t): E = -grad phi - (1/c) dA/dt, B_z = d_x A_y - d_y A_x."""
    dh = 0.02 * cfg.sigma if dh is None else dh
    dt = 0.02 * cfg.sigma if dt is None else dt
    P = np.asarray(P, dtype=float)
    gx = sum(c * semi_analytic_potentials(cfg, P + [o * dh, 0.0], t) for c, o in zip(_D4, _O4)) / dh
    gy = sum(c * semi_analytic_potentials(cfg, P + [0.0, o * dh], t) for c, o in zip(_D4, _O4)) / dh
    gt = sum(c * semi_analytic_potentials(cfg, P, t + o * dt) for c, o in zip(_D4, _O4)) / dt
    ex = -gx[0] - gt[1]
    ey = -gy[0] - gt[2]
    bz = gx[2] - gy[1]
    return np.array([ex, ey, bz])


def semi_analytic_forces(cfg, P, t):
    """(F_s, F_n) per unit charge on a particle at P moving with beta0 t-hat(t):
    F = E + beta x B_z z-hat, resolved on the orbit tangent / normal at t."""
    ex, ey, bz = semi_analytic_fields(cfg, P, t)
    _, th = _orbit(cfg, t)
    nh = np.array([-th[1], th[0]])
    b = cfg.beta0 * th
    f = np.array([ex + b[1] * bz, ey - b[0] * bz])
    return float(f @ th), float(f @ nh)


def axis_points(cfg, k, offsets_sigma, v_sigma=0.0):
    """Lab points at comoving (u, v) = (5 sigma + o sigma, 5 sigma + v sigma) of frame k."""
    ox, oy, c, s = W.frame(cfg, k)
    half = 0.5 * cfg.extent
    u = half + np.asarray(offsets_sigma) * cfg.sigma
    v = half + v_sigma * cfg.sigma + 0 * u
    return np.stack([ox + u * c - v * s, oy + u * s + v * c], axis=1)


# ------------------------------------------------------------------ GPU path
def gpu_steady_fields(rp, torch, cfg, k, density=None, psi_offset=0.0, n_prev=4):
    """Potentials at steps k-n_prev .. k of the steady-state ring, then the fields at step k
    (dA/dt from the n_prev previous steps, R-15b)."""
    n = cfg.nx * cfg.ny
    dev = torch.device("cuda:0")
    ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau)
    try:
        pot = {}
        for kk in range(k - n_prev, k + 1):
            rp.rp_load_state(ctx, kk, cfg.n_pre, W.ring_frames(cfg, kk),
                             torch.tensor(steady_ring(cfg, kk, density, psi_offset), device=dev))
            t3 = [torch.zeros(n, dtype=torch.float64, device=dev) for _ in range(3)]
            rp.rp_compute_potentials(ctx, *t3)
            pot[kk] = t3
        prev = None
        if n_prev:
            prev = torch.stack([torch.stack([pot[k - j][1], pot[k - j][2]]) for j in range(1, n_prev + 1)])
        out = [torch.zeros(n, dtype=torch.float64, device=dev) for _ in range(3)]
        rp.rp_compute_fields(ctx, *pot[k], prev, *out)
        torch.cuda.synchronize()
        return ctx, out
    except Exception:
        rp.rp_destroy(ctx)
        raise


def gpu_particle_forces(rp, torch, ctx, cfg, k, fields, P):
    """(F_s, F_n) from rp_particle_forces at lab points P (particles moving with gamma0 beta0
    along the tangent of frame k), self-fields only (no external dipole)."""
    dev = torch.device("cuda:0")
    _, _, c, s = W.frame(cfg, k)
    g = cfg.gamma0 * cfg.beta0
    t = lambda a: torch.tensor(np.ascontiguousarray(a, dtype=np.float64), device=dev)
    n = len(P)
    fx, fy = (torch.zeros(n, dtype=torch.float64, device=dev) for _ in range(2))
    rp.rp_particle_forces(ctx, t(P[:, 0]), t(P[:, 1]), t(np.full(n, g * c)), t(np.full(n, g * s)),
                          0.0, *fields, fx, fy)
    fx, fy = fx.cpu().numpy(), fy.cpu().numpy()
    return fx * c + fy * s, -fx * s + fy * c


def validate_forces(n=129, k=201, offsets=None):
    """References 1 and 2 against the GPU on the bunch axis (and 1 sigma off it for F_n)."""
    import torch
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = csr_config(n)
    offsets = np.linspace(-3.0, 3.0, 25) if offsets is None else np.asarray(offsets)
    ctx, fields = gpu_steady_fields(rp, torch, cfg, k)
    rec = {"mesh": n, "sigma": cfg.sigma, "R0": cfg.r0, "gamma0": cfg.gamma0, "step": k,
           "s_over_sigma": offsets.tolist()}
    try:
        for vs in (0.0, 1.0):
            P = axis_points(cfg, k, offsets, vs)
            fs, fn = gpu_particle_forces(rp, torch, ctx, cfg, k, fields, P)
            ref = np.array([semi_analytic_forces(cfg, p, k * cfg.dt) for p in P])
            tag = "axis" if vs == 0 else "v+1sigma"
            rec[f"gpu_Fs_{tag}"], rec[f"gpu_Fn_{tag}"] = fs.tolist(), fn.tolist()
            rec[f"exact_Fs_{tag}"], rec[f"exact_Fn_{tag}"] = ref[:, 0].tolist(), ref[:, 1].tolist()
            rec[f"max_rel_dev_Fs_{tag}"] = float(np.abs(fs - ref[:, 0]).max() / np.abs(ref[:, 0]).max())
            rec[f"max_rel_dev_Fn_{tag}"] = float(np.abs(fn - ref[:, 1]).max() / np.abs(ref[:, 1]).max())
        line = np.array([csr_1d(o * cfg.sigma, cfg.sigma, cfg.r0) for o in offsets])
        rec["csr_1d_Es"] = line.tolist()
        rec["max_rel_dev_Fs_axis_vs_1d_line"] = float(
            np.abs(np.array(rec["gpu_Fs_axis"]) - line).max() / np.abs(line).max())
        rec["max_rel_dev_exact_sheet_vs_1d_line"] = float(
            np.abs(np.array(rec["exact_Fs_axis"]) - line).max() / np.abs(line).max())
    finally:
        rp.rp_destroy(ctx)
    return rec


# ------------------------------------------------------------------ Monte-Carlo MSE (3.)
def _bunch_particles(cfg, n, seed, k):
    """n particles of the comoving Gaussian at step k: the workloads recipe drawn in frame 0
    and carried rigidly to frame k (same local coordinates; momenta rotated with the frame)."""
    x, y, ux, uy = W.particles(cfg, n=n, seed=seed)
    f0, fk = W.frame(cfg, 0), W.frame(cfg, k)
    du = (x - f0[0]) * f0[2] + (y - f0[1]) * f0[3]
    dv = (y - f0[1]) * f0[2] - (x - f0[0]) * f0[3]
    X = fk[0] + du * fk[2] - dv * fk[3]
    Y = fk[1] + du * fk[3] + dv * fk[2]
    cd = fk[2] * f0[2] + fk[3] * f0[3]
    sd = fk[3] * f0[2] - fk[2] * f0[3]
    return X, Y, cd * ux - sd * uy, sd * ux + cd * uy


def mse_study(ns=(10_000, 100_000, 1_000_000, 10_000_000), n=129, k=4, seed=17_129):
    """Fig. 3: mean-square error of the longitudinal force on the particles vs N on a fixed
    129^2 grid.  Each run: rigid pre-history + GPU deposit of the bunch at steps 0..k (the
    particles carried rigidly along the orbit), potentials at every step, fields at step k from
    the k previous potentials (R-15b), forces at the step-k particles.  The exact force of each
    particle: the same path fed the noise-free expected deposit (the Gaussian convolved with the
    TSC kernel) with the particles' mean current -- along the tangent half a step back, where
    the leap-frog momenta live (R-21) -- gathered at the same positions."""
    import torch
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = csr_config(n)
    dev = torch.device("cuda:0")
    npts = n * n
    t = lambda a: torch.tensor(np.ascontiguousarray(a, dtype=np.float64), device=dev)
    ref_ctx, ref_fields = gpu_steady_fields(rp, torch, cfg, k, tsc_expected_nodes(cfg))
    out = {"mesh": n, "step": k, "ns": list(ns), "mse_Fs": [], "mse_Fn": [], "mean_Fs2": [],
           "mean_Fn2": [], "n_ppc": []}
    try:
        for N in ns:
            ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau)
            try:
                rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
                pot = []
                for kk in range(k + 1):
                    X, Y, UX, UY = _bunch_particles(cfg, N, seed, kk)
                    # the current with the momenta of t_k (R-27), as the simulation loop does
                    cu = [torch.empty(N, dtype=torch.float64, device=dev) for _ in range(2)]
                    rp.rp_kick_external(ctx, t(UX), t(UY), cfg.q_over_mc, cfg.bz_ext, 0.5, *cu)
                    rp.rp_deposit_step(ctx, t(X), t(Y), *cu, 1.0 / N, W.frame(cfg, kk))
                    p3 = [torch.zeros(npts, dtype=torch.float64, device=dev) for _ in range(3)]
                    rp.rp_compute_potentials(ctx, *p3)
                    pot.append(p3)
                prev = torch.stack([torch.stack([pot[k - j][1], pot[k - j][2]]) for j in range(1, k + 1)])
                fld = [torch.zeros(npts, dtype=torch.float64, device=dev) for _ in range(3)]
                rp.rp_compute_fields(ctx, *pot[k], prev, *fld)
                xs, ys, uxs, uys = t(X), t(Y), cu[0], cu[1]
                f = [torch.zeros(N, dtype=torch.float64, device=dev) for _ in range(4)]
                rp.rp_particle_forces(ctx, xs, ys, uxs, uys, 0.0, *fld, f[0], f[1])
                rp.rp_particle_forces(ref_ctx, xs, ys, uxs, uys, 0.0, *ref_fields, f[2], f[3])
            finally:
                rp.rp_destroy(ctx)
            _, _, c, s = W.frame(cfg, k)
            fs = (f[0] * c + f[1] * s).cpu().numpy()
            fn = (-f[0] * s + f[1] * c).cpu().numpy()
            rs = (f[2] * c + f[3] * s).cpu().numpy()
            rn = (-f[2] * s + f[3] * c).cpu().numpy()
            out["mse_Fs"].append(float(np.mean((fs - rs) ** 2)))
            out["mse_Fn"].append(float(np.mean((fn - rn) ** 2)))
            out["mean_Fs2"].append(float(np.mean(rs ** 2)))
            out["mean_Fn2"].append(float(np.mean(rn ** 2)))
            out["n_ppc"].append(N / npts)
            if N == max(ns):  # absolute forces on a sample of particles vs the exact solution
                # particles in the bunch core (|u|, |v| <= 3 sigma of the centre): the mesh ends at
                # 5 sigma, where the zero-padded stencils and one-sided differences take over
                fk = W.frame(cfg, k)
                du = (X - fk[0]) * fk[2] + (Y - fk[1]) * fk[3] - 0.5 * cfg.extent
                dv = (Y - fk[1]) * fk[2] - (X - fk[0]) * fk[3] - 0.5 * cfg.extent
                core = np.nonzero((np.abs(du) <= 3 * cfg.sigma) & (np.abs(dv) <= 3 * cfg.sigma))[0]
                rng = np.random.default_rng(5)
                idx = rng.choice(core, 60, replace=False)
                # the exact force on each sampled particle with its own velocity (its transverse
                # beta ~ 2e-5 times the space-charge B_z is of the size of the CSR force)
                cux, cuy = cu[0].cpu().numpy(), cu[1].cpu().numpy()
                ex_ = []
                for i in idx:
                    exf, eyf, bzf = semi_analytic_fields(cfg, (X[i], Y[i]), k * cfg.dt)
                    g = math.sqrt(1.0 + cux[i] ** 2 + cuy[i] ** 2)
                    fx_, fy_ = exf + cuy[i] / g * bzf, eyf - cux[i] / g * bzf
                    ex_.append((fx_ * c + fy_ * s, -fx_ * s + fy_ * c))
                ex_ = np.array(ex_)
                peak = np.abs(ex_[:, 0]).max()
                out["sample_particles"] = 60
                out["exact_Fs_peak_in_sample"] = float(peak)
                out["ref_vs_exact_Fs_max_over_peak"] = float(np.abs(rs[idx] - ex_[:, 0]).max() / peak)
                out["ref_vs_exact_Fn_max_over_peak"] = float(
                    np.abs(rn[idx] - ex_[:, 1]).max() / np.abs(ex_[:, 1]).max())
                out["noisy_vs_exact_Fs_rms_over_peak"] = float(
                    np.sqrt(np.mean((fs[idx] - ex_[:, 0]) ** 2)) / peak)
    finally:
        rp.rp_destroy(ref_ctx)
    ln = np.log(np.array(ns, dtype=float))
    out["slope_Fs"] = float(np.polyfit(ln, np.log(np.array(out["mse_Fs"])), 1)[0])
    out["slope_Fn"] = float(np.polyfit(ln, np.log(np.array(out["mse_Fn"])), 1)[0])
    return out


def main():
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    if "--mse" in sys.argv:
        rec = mse_study()
    else:
        n = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 129
        rec = validate_forces(n)
    print(json.dumps({k: v for k, v in rec.items() if not isinstance(v, list) or len(v) < 8}))
    if out:
        json.dump(rec, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
