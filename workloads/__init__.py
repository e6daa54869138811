"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NO arithmetic of the method (no deposition, quadrature,
interpolation, fields or push).  It only draws seeded random numbers and
lays out the geometry the paper's workloads are quoted on:

* PAPER.md P:170  -- Q = 1 nC bunches sampled by Monte Carlo, tau = 1e-6.
* LCLS bend: R0 = 25.13 m, theta_b = 11.4 deg,
  sigma_s = 50 um, emittance 1 nm, Q = 1 nC (configs 2-5).
* BASELINE.json ``configs`` -- mesh, particle count, steps, history depth.

Recipe (DESIGN.md sec. 2 "Inputs"): numpy PCG64 with seed 17_000 + config
number; Gaussian bunch in the comoving frame; frames on the reference orbit;
rigid steady-state pre-history (n_pre = kappa_max + 1 levels of the step-0 bunch, R-23).
Units: lengths in metres for the bend (sigma = 50e-6), sigma = 1 for the
static config; c = 1 (time in length units); bunch charge Q = 1.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

R_E = 2.8179403262e-15       # classical electron radius [m]
N_E_PER_NC = 6.241509074e9   # electrons in 1 nC


@dataclasses.dataclass
class Config:
    number: int
    name: str
    nx: int
    ny: int
    n_particles: int
    steps: int
    kappa_max: int
    geometry: str            # "static" | "bend"
    sigma: float             # bunch rms size (both planes)
    cdt: float               # subregion width c*dt
    c: float = 1.0
    gamma0: float = 1.0
    r0: float = 0.0          # bend radius
    sigma_xp: float = 0.0    # rms angle spread
    q_over_mc: float = 0.0   # coupling of the self-fields in the push
    n_theta: int = 64
    max_depth: int = 30
    n_root: int = 2
    rule: int = 0            # outer segment rule: 0 = GK15, 1 = Simpson/Boole (the paper's)
    interp: int = 0          # spatial weights: 0 = TSC (R-6), 1 = quadratic Lagrange (R-25)
    tau_rel: float = 1e-6    # tau = tau_rel * (Q/sigma) sqrt(pi/2)
    seed: int = 0

    @property
    def H(self) -> int:
        return self.kappa_max + 2

    @property
    def n_pre(self) -> int:
        return self.kappa_max + 1

    @property
    def extent(self) -> float:
        return 10.0 * self.sigma              # +-5 sigma

    @property
    def hx(self) -> float:
        return self.extent / (self.nx - 1)

    @property
    def hy(self) -> float:
        return self.extent / (self.ny - 1)

    @property
    def dt(self) -> float:
        return self.cdt / self.c

    @property
    def tau(self) -> float:
        return self.tau_rel * (1.0 / self.sigma) * math.sqrt(math.pi / 2.0)

    @property
    def beta0(self) -> float:
        return math.sqrt(max(0.0, 1.0 - 1.0 / (self.gamma0 * self.gamma0)))

    @property
    def q_particle(self) -> float:
        return 1.0 / self.n_particles

    @property
    def bz_ext(self) -> float:
        """Uniform dipole field that keeps the reference particle on radius R0
        (counter-clockwise), in the push's units: du/dt = q/mc (E + beta x B)."""
        if self.geometry != "bend":
            return 0.0
        return -self.gamma0 * self.beta0 / (self.r0 * self.q_over_mc) * self.c

    def summary(self) -> dict:
        return {"workload": self.name, "config": self.number, "mesh": f"{self.nx}x{self.ny}",
                "particles": self.n_particles, "steps": self.steps,
                "history_depth": self.kappa_max, "geometry": self.geometry,
                "cdt": self.cdt, "tau": self.tau, "n_theta": self.n_theta,
                "max_depth": self.max_depth, "n_root": self.n_root}


_BEND_R0 = 25.13
_BEND_ANGLE = 11.4 * math.pi / 180.0
_BEND_LEN = _BEND_R0 * _BEND_ANGLE          # ~5.0 m
_SIGMA = 50e-6
_EPS = 1e-9


def _bend(number, n, npart, steps):
    return Config(number=number, name=f"cfg{number}-{n}x{n}-bend", nx=n, ny=n,
                  n_particles=npart, steps=steps, kappa_max=steps, geometry="bend",
                  sigma=_SIGMA, cdt=_BEND_LEN / steps, gamma0=1e4, r0=_BEND_R0,
                  sigma_xp=_EPS / _SIGMA, q_over_mc=R_E * N_E_PER_NC,
                  seed=17_000 + number)


def config(number: int) -> Config:
    """BASELINE.json configs[number-1]."""
    if number == 1:
        return Config(number=1, name="cfg1-32x32-static", nx=32, ny=32, n_particles=10_000,
                      steps=10, kappa_max=10, geometry="static", sigma=1.0, cdt=1.6,
                      q_over_mc=1e-3, seed=17_001)
    if number == 2:
        return _bend(2, 64, 1_000_000, 100)
    if number == 3:
        return _bend(3, 128, 10_000_000, 500)
    if number == 4:
        return _bend(4, 256, 100_000_000, 1000)
    if number == 5:
        return _bend(5, 512, 100_000_000, 2000)
    raise ValueError(number)


# ------------------------------------------------------------------ geometry
def frame(cfg: Config, level: float) -> np.ndarray:
    """(ox, oy, cos psi, sin psi) of the mesh at step ``level`` (may be < 0).

    static: lower-left node at (-5 sigma, -5 sigma), axes = lab axes.
    bend: reference orbit = counter-clockwise circle of radius R0 centred at
    (0, R0); s_l = beta0 * l * c dt; the mesh is centred on ref(s_l) with its
    u axis along the tangent (SURVEY 8(d) "Bend geometry").
    """
    half = 0.5 * cfg.extent
    if cfg.geometry == "static":
        return np.array([-half, -half, 1.0, 0.0])
    s = cfg.beta0 * level * cfg.cdt
    psi = s / cfg.r0
    cp, sp = math.cos(psi), math.sin(psi)
    rx, ry = cfg.r0 * math.sin(psi), cfg.r0 * (1.0 - math.cos(psi))
    ox = rx - half * cp + half * sp
    oy = ry - half * sp - half * cp
    return np.array([ox, oy, cp, sp])


def frames(cfg: Config, levels) -> np.ndarray:
    return np.stack([frame(cfg, l) for l in levels])


def ring_frames(cfg: Config, k: int) -> np.ndarray:
    """Frames as stored in a ring of H slots at step k: slot(l) = l mod H
    holds the frame of level l for l in k-H+1 .. k."""
    H = cfg.H
    out = np.zeros((H, 4))
    for l in range(k - H + 1, k + 1):
        out[l % H] = frame(cfg, l)
    return out


def particles(cfg: Config, n: int | None = None, seed: int | None = None):
    """Step-0 particles (x, y, ux, uy), u = gamma*beta, float64 SoA."""
    n = cfg.n_particles if n is None else n
    rng = np.random.default_rng(cfg.seed if seed is None else seed)
    half = 0.5 * cfg.extent
    u = half + cfg.sigma * rng.standard_normal(n)
    v = half + cfg.sigma * rng.standard_normal(n)
    ox, oy, c, s = frame(cfg, 0)
    x = ox + u * c - v * s
    y = oy + u * s + v * c
    if cfg.geometry == "static":
        return x, y, np.zeros(n), np.zeros(n)
    xp = cfg.sigma_xp * rng.standard_normal(n)
    # leap-frog momenta live at t = -dt/2: tangent of the orbit half a step back
    psi = -0.5 * cfg.beta0 * cfg.cdt / cfg.r0
    tx, ty = math.cos(psi), math.sin(psi)
    g = cfg.gamma0 * cfg.beta0
    ux = g * (tx - xp * ty)
    uy = g * (ty + xp * tx)
    return x, y, ux, uy


def node_gaussian_ring(cfg: Config, k: int, amp_of_level=None, beta=(0.0, 0.0),
                       centre=None, sigma=None) -> np.ndarray:
    """A ring [H, ny, nx, 4] whose grids are node samples of a Gaussian
    (rho, rho*bx, rho*by, 0) with a per-level amplitude: a synthetic history
    that needs no deposition (used to test potentials from a known state)."""
    H = cfg.H
    sg = cfg.sigma if sigma is None else sigma
    cx, cy = (0.5 * cfg.extent, 0.5 * cfg.extent) if centre is None else centre
    u = np.arange(cfg.nx) * cfg.hx
    v = np.arange(cfg.ny) * cfg.hy
    U, V = np.meshgrid(u, v)
    g = np.exp(-((U - cx) ** 2 + (V - cy) ** 2) / (2 * sg * sg)) / (2 * math.pi * sg * sg)
    ring = np.zeros((H, cfg.ny, cfg.nx, 4))
    for l in range(k - H + 1, k + 1):
        a = 1.0 if amp_of_level is None else amp_of_level(l)
        ring[l % H, :, :, 0] = a * g
        ring[l % H, :, :, 1] = a * g * beta[0]
        ring[l % H, :, :, 2] = a * g * beta[1]
    return ring


def sample_points(nx: int, ny: int, m: int, seed: int = 1) -> np.ndarray:
    """Stratified sample of m flattened mesh points (raster stride + jitter)."""
    n = nx * ny
    if m >= n:
        return np.arange(n, dtype=np.int32)
    rng = np.random.default_rng(seed)
    base = (np.arange(m) * n) // m
    step = max(1, n // m)
    pts = base + rng.integers(0, step, size=m)
    return np.unique(np.minimum(pts, n - 1)).astype(np.int32)
