"""CPU oracle for the retarded-potential step (Arumugam et al., ICPP'17).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
module.  The product package never imports it and it imports nothing from the
product package.

This module is argument marshalling (ctypes) around ``rp_oracle.c``; every
arithmetic step of the method lives in that C file, which cites PAPER.md
(``/root/reference/PAPER.md``) line by line.  ``build()`` compiles it with
``gcc -O2 -ffp-contract=off -fopenmp`` (no FMA contraction, plain IEEE FP64).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rp_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

SRC_GRID, SRC_GAUSS, SRC_DISK = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile rp_oracle.c into liboracle.so (in-tree)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-std=c11", "-shared", "-fPIC", "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class Frame(C.Structure):
    _fields_ = [("ox", C.c_double), ("oy", C.c_double), ("c", C.c_double), ("s", C.c_double)]


class Params(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("hx", C.c_double), ("hy", C.c_double),
                ("c", C.c_double), ("dt", C.c_double), ("tau", C.c_double),
                ("n_theta", C.c_int32), ("max_depth", C.c_int32), ("n_root", C.c_int32),
                ("kappa_max", C.c_int32), ("rule", C.c_int32), ("interp", C.c_int32)]


class Hist(C.Structure):
    _fields_ = [("ring", C.POINTER(C.c_double)), ("frames", C.POINTER(Frame)),
                ("H", C.c_int32), ("k", C.c_int32), ("n_pre", C.c_int32)]


class Source(C.Structure):
    _fields_ = [("kind", C.c_int32), ("x0", C.c_double), ("y0", C.c_double),
                ("width", C.c_double), ("q", C.c_double), ("bx", C.c_double),
                ("by", C.c_double), ("amp", C.POINTER(C.c_double))]


class Result(C.Structure):
    _fields_ = [("phi", C.c_double), ("ax", C.c_double), ("ay", C.c_double), ("err", C.c_double),
                ("nseg", C.c_int32), ("nleaf", C.c_int32), ("capped", C.c_int32),
                ("ties", C.c_int32), ("max_level", C.c_int32), ("noise_ties", C.c_int32),
                ("evals", C.c_int64), ("nodes", C.c_int64), ("min_margin", C.c_double),
                ("chase_segs", C.c_int64), ("chase_evals", C.c_int64), ("min_noise", C.c_double)]


_lib = None


def set_threads(n: int) -> int:
    """Set the OpenMP thread count of the oracle's parallel loops (the calling thread's
    nthreads ICV).  torchrun exports OMP_NUM_THREADS=1 and torch loads libgomp.so.1 before
    the oracle, so the environment cannot be changed after the fact; bench.py calls this with
    the host cores it reports.  Returns the count in effect."""
    lib()
    gomp = C.CDLL("libgomp.so.1")  # the instance already loaded (shared by soname)
    gomp.omp_set_num_threads(C.c_int(int(n)))
    return int(gomp.omp_get_max_threads())


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.POINTER
        d, i32, i64 = C.c_double, C.c_int32, C.c_int64
        pd, pi32 = P(d), P(i32)
        pu16, pi64 = P(C.c_uint16), P(i64)
        sig = {
            "orc_gk15_constants": (None, [pd, pd, pd]),
            "orc_tsc_weights": (None, [d, pd]),
            "orc_lagrange3_weights": (None, [d, pd]),
            "orc_bin_of": (i32, [d, d, P(Frame), d, d, i32, i32, pi32, pi32, pd, pd]),
            "orc_deposit": (d, [i64, pd, pd, pd, pd, d, P(Frame), i32, i32, d, d, pd, pi32]),
            "orc_rigid_level": (None, [pd, P(Frame), P(Frame), i32, i32, pd]),
            "orc_arcs_rect": (i32, [d, d, d, d, d, d, d, pd]),
            "orc_arcs_disk": (i32, [d, d, d, d, d, d, pd]),
            "orc_kappa": (i32, [P(Params), P(Hist)]),
            "orc_mesh_point": (None, [P(Params), P(Frame), i32, i32, pd, pd]),
            "orc_point_lab": (None, [P(Params), P(Hist), P(Source), d, d, P(Result)]),
            "orc_potentials": (None, [P(Params), P(Hist), P(Source), pi32, i32, P(Result)]),
            "orc_potentials_ex": (None, [P(Params), P(Hist), P(Source), pi32, i32, pu16, P(Result)]),
            "orc_potentials_predictive": (i32, [P(Params), P(Hist), P(Source), pu16, i32, i32, i32,
                                                pi32, i32, pi32, pu16, P(Result)]),
            "orc_knn_pattern": (i32, [pu16, i32, i32, i32, i32, i32, i32]),
            "orc_kmeans": (i32, [pu16, i32, i32, i32, i32, pi32]),
            "orc_merge_partitions": (i64, [P(Params), pu16, pi32, i32, i32, pi64, pd]),
            "orc_merge_partitions_mode": (i64, [P(Params), pu16, pi32, i32, i32, i32, pi64, pi32,
                                                pd, pi64, pd]),
            "orc_potentials_parts": (None, [P(Params), P(Hist), P(Source), pi32, i32, pi64, pd,
                                            P(Result)]),
            "orc_potentials_predictive2": (i32, [P(Params), P(Hist), P(Source), pu16, i32, i32,
                                                 i32, i32, pi64, pi32, pd, pi32, i32, pi32, pu16,
                                                 P(Result)]),
            "orc_clip_at": (i32, [P(Params), P(Hist), P(Source), d, d, i32, pd, pd]),
            "orc_dists_at": (None, [P(Params), P(Hist), P(Source), d, d, i32, d, pd, pd]),
            "orc_centre_at": (None, [P(Params), P(Hist), P(Source), d, d, i32, d, pd, pd, pd]),
            "orc_inner_at": (i64, [P(Params), P(Hist), P(Source), d, d, i32, d, pd]),
            "orc_integrand_at": (None, [P(Params), P(Hist), P(Source), i32, d, d, d, pd]),
            "orc_gk15_at": (None, [P(Params), P(Hist), P(Source), d, d, i32, d, d, pd, pd, pd]),
            "orc_fields": (None, [P(Params), P(Frame), i32, pd, pd, pd, pd, pd, pd, pd]),
            "orc_kick_external": (None, [P(Params), i64, pd, pd, d, d, d, pd, pd]),
            "orc_forces": (None, [P(Params), P(Frame), i64, pd, pd, pd, pd, d, pd, pd, pd, pd, pd]),
            "orc_push": (None, [P(Params), P(Frame), i64, pd, pd, pd, pd, d, d, pd, pd, pd]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(_lib, name)
            fn.restype = res
            fn.argtypes = args
    return _lib


# ---------------------------------------------------------------- helpers
def _pd(a):
    if a is None:
        return None
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _pi(a):
    assert a.dtype == np.int32 and a.flags.c_contiguous
    return a.ctypes.data_as(C.POINTER(C.c_int32))


def _pu16(a):
    assert a.dtype == np.uint16 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(C.POINTER(C.c_uint16))


def knn_pattern(prev, nx, ny, p, j, knn):
    prev = np.ascontiguousarray(prev, dtype=np.uint16)
    return lib().orc_knn_pattern(_pu16(prev), nx, ny, prev.shape[1], p, j, knn)


def kmeans(pattern, m, max_iters=20):
    """RP-CLUSTERING (R-26): (assignment, passes)."""
    pattern = np.ascontiguousarray(pattern, dtype=np.uint16)
    assign = np.zeros(pattern.shape[0], dtype=np.int32)
    it = lib().orc_kmeans(_pu16(pattern), pattern.shape[0], pattern.shape[1], m, max_iters,
                          _pi(assign))
    return assign, it


def frame(f) -> Frame:
    return Frame(*[float(v) for v in f])


class Problem:
    """Bundles (params, history, source) with the numpy buffers kept alive.

    ``ring``: float64 [H, ny, nx, 4]; ``frames``: float64 [H, 4] (ox, oy, c, s);
    ``amp``: optional float64 [H] amplitudes for analytic sources.
    """

    def __init__(self, *, nx, ny, hx, hy, c, dt, tau, kappa_max, k, n_pre,
                 ring=None, frames=None, n_theta=64, max_depth=30, n_root=2,
                 source=SRC_GRID, x0=0.0, y0=0.0, width=1.0, q=1.0, bx=0.0, by=0.0, amp=None,
                 rule=0, interp=0):
        H = kappa_max + 2
        self.params = Params(nx, ny, hx, hy, c, dt, tau, n_theta, max_depth, n_root, kappa_max,
                             rule, interp)
        self.ring = None if ring is None else np.ascontiguousarray(ring, dtype=np.float64)
        if self.ring is not None:
            assert self.ring.shape == (H, ny, nx, 4), self.ring.shape
        fr = np.zeros((H, 4)) if frames is None else np.asarray(frames, dtype=np.float64)
        if frames is None:
            fr[:, 2] = 1.0
        self.frames_np = np.ascontiguousarray(fr)
        assert self.frames_np.shape == (H, 4)
        self.frames = (Frame * H)(*[Frame(*row) for row in self.frames_np])
        self.amp = None if amp is None else np.ascontiguousarray(amp, dtype=np.float64)
        self.hist = Hist(_pd(self.ring) if self.ring is not None else None,
                         C.cast(self.frames, C.POINTER(Frame)), H, k, n_pre)
        self.source = Source(source, x0, y0, width, q, bx, by,
                             _pd(self.amp) if self.amp is not None else None)

    # -------------------------------------------------------------- calls
    def kappa(self) -> int:
        return lib().orc_kappa(C.byref(self.params), C.byref(self.hist))

    def mesh_point(self, ix, iy):
        px, py = C.c_double(), C.c_double()
        H = self.hist.H
        lib().orc_mesh_point(C.byref(self.params), C.byref(self.frames[self.hist.k % H]),
                             ix, iy, C.byref(px), C.byref(py))
        return px.value, py.value

    def point_lab(self, px, py) -> Result:
        r = Result()
        lib().orc_point_lab(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                            px, py, C.byref(r))
        return r

    def potentials(self, pts) -> np.ndarray:
        """Potentials at flattened mesh points; returns a structured array."""
        pts = np.ascontiguousarray(pts, dtype=np.int32)
        out = (Result * len(pts))()
        lib().orc_potentials(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                             _pi(pts), len(pts), out)
        return np.ctypeslib.as_array(out).copy() if len(pts) else np.zeros(0)

    def potentials_items(self, pts):
        """Potentials at flattened mesh points plus the observed access pattern: accepted
        segments per (point, subregion), uint16 [len(pts), kappa_max]."""
        pts = np.ascontiguousarray(pts, dtype=np.int32)
        out = (Result * len(pts))()
        leaves = np.zeros((len(pts), self.params.kappa_max), dtype=np.uint16)
        lib().orc_potentials_ex(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                                _pi(pts), len(pts), _pu16(leaves), out)
        return np.ctypeslib.as_array(out).copy(), leaves

    def potentials_predictive(self, prev, pts, knn=9, m=0, max_iters=20):
        """Predictive-RP variant (Algorithm 1, reading R-26) at step k from the previous
        step's pattern prev [nx*ny, kappa_max] (uint16).  Returns (results, clusters [nx*ny],
        leaves [len(pts), kappa_max], k-means passes)."""
        prev = np.ascontiguousarray(prev, dtype=np.uint16)
        nall = self.params.nx * self.params.ny
        assert prev.shape == (nall, self.params.kappa_max)
        pts = np.ascontiguousarray(pts, dtype=np.int32)
        out = (Result * max(len(pts), 1))()
        clusters = np.zeros(nall, dtype=np.int32)
        leaves = np.zeros((len(pts), self.params.kappa_max), dtype=np.uint16)
        it = lib().orc_potentials_predictive(C.byref(self.params), C.byref(self.hist),
                                             C.byref(self.source), _pu16(prev), knn, m, max_iters,
                                             _pi(pts), len(pts), _pi(clusters), _pu16(leaves), out)
        res = np.ctypeslib.as_array(out).copy()[:len(pts)]
        return res, clusters, leaves, it

    def potentials_parts(self, pts):
        """The accepted partition of every item (P:104's partition of an earlier step): for
        point i and subregion j, the leaves' left ends in r' order and the last right end
        (count + 1 doubles; none without leaves).  Returns (results, leaves [len(pts), kmax],
        off [len(pts) * kmax] int64, plen [len(pts) * kmax] int32, parts float64)."""
        pts = np.ascontiguousarray(pts, dtype=np.int32)
        res, leaves = self.potentials_items(pts)
        plen = np.where(leaves > 0, leaves.astype(np.int64) + 1, 0).reshape(-1)
        off = np.zeros(plen.size, dtype=np.int64)
        off[1:] = np.cumsum(plen)[:-1]
        parts = np.zeros(max(int(plen.sum()), 1))
        out = (Result * max(len(pts), 1))()
        lib().orc_potentials_parts(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                                   _pi(pts), len(pts), off.ctypes.data_as(C.POINTER(C.c_int64)),
                                   _pd(parts), out)
        return res, leaves, off, plen.astype(np.int32), parts

    def potentials_predictive_adaptive(self, prev, prev_off, prev_len, prev_parts, pts, knn=9,
                                       m=0, max_iters=20):
        """Predictive-RP with adaptive partitioning (reading R-26b): line 4 refines the
        earlier step's accepted partitions of all nx*ny points (potentials_parts over every
        point, in point order) by the forecast.  Same returns as potentials_predictive."""
        prev = np.ascontiguousarray(prev, dtype=np.uint16)
        nall = self.params.nx * self.params.ny
        assert prev.shape == (nall, self.params.kappa_max)
        prev_off = np.ascontiguousarray(prev_off, dtype=np.int64)
        prev_len = np.ascontiguousarray(prev_len, dtype=np.int32)
        prev_parts = np.ascontiguousarray(prev_parts, dtype=np.float64)
        assert prev_off.size == nall * self.params.kappa_max == prev_len.size
        pts = np.ascontiguousarray(pts, dtype=np.int32)
        out = (Result * max(len(pts), 1))()
        clusters = np.zeros(nall, dtype=np.int32)
        leaves = np.zeros((len(pts), self.params.kappa_max), dtype=np.uint16)
        it = lib().orc_potentials_predictive2(
            C.byref(self.params), C.byref(self.hist), C.byref(self.source), _pu16(prev), knn, m,
            max_iters, 1, prev_off.ctypes.data_as(C.POINTER(C.c_int64)), _pi(prev_len),
            _pd(prev_parts), _pi(pts), len(pts), _pi(clusters), _pu16(leaves), out)
        res = np.ctypeslib.as_array(out).copy()[:len(pts)]
        return res, clusters, leaves, it

    def merge_partitions_adaptive(self, pattern, assign, m, prev_off, prev_len, prev_parts):
        """Per-cluster merged adaptive partitions (R-26b; lines 4, 9-12)."""
        pattern = np.ascontiguousarray(pattern, dtype=np.uint16)
        assign = np.ascontiguousarray(assign, dtype=np.int32)
        prev_off = np.ascontiguousarray(prev_off, dtype=np.int64)
        prev_len = np.ascontiguousarray(prev_len, dtype=np.int32)
        prev_parts = np.ascontiguousarray(prev_parts, dtype=np.float64)
        off = np.zeros(m * self.params.kappa_max + 1, dtype=np.int64)
        args = (C.byref(self.params), _pu16(pattern), _pi(assign), len(assign), m, 1,
                prev_off.ctypes.data_as(C.POINTER(C.c_int64)), _pi(prev_len), _pd(prev_parts),
                off.ctypes.data_as(C.POINTER(C.c_int64)))
        n = lib().orc_merge_partitions_mode(*args, None)
        bp = np.zeros(max(n, 1))
        lib().orc_merge_partitions_mode(*args, _pd(bp))
        return off, bp[:n]

    def merge_partitions(self, pattern, assign, m):
        """Per-cluster merged uniform partitions of S_j (lines 4, 9-12): (off, breakpoints)."""
        pattern = np.ascontiguousarray(pattern, dtype=np.uint16)
        assign = np.ascontiguousarray(assign, dtype=np.int32)
        off = np.zeros(m * self.params.kappa_max + 1, dtype=np.int64)
        n = lib().orc_merge_partitions(C.byref(self.params), _pu16(pattern), _pi(assign),
                                       len(assign), m, off.ctypes.data_as(C.POINTER(C.c_int64)), None)
        bp = np.zeros(max(n, 1))
        lib().orc_merge_partitions(C.byref(self.params), _pu16(pattern), _pi(assign), len(assign),
                                   m, off.ctypes.data_as(C.POINTER(C.c_int64)), _pd(bp))
        return off, bp[:n]

    def clip(self, px, py, j):
        A, B = C.c_double(), C.c_double()
        ok = lib().orc_clip_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                               px, py, j, C.byref(A), C.byref(B))
        return (A.value, B.value) if ok else None

    def dists(self, px, py, j, r):
        a, b = C.c_double(), C.c_double()
        lib().orc_dists_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                           px, py, j, r, C.byref(a), C.byref(b))
        return a.value, b.value

    def centre(self, px, py, j, r):
        """Frame-local circle centre at radius r of subregion j and the time weights."""
        cu, cv, w = C.c_double(), C.c_double(), np.zeros(3)
        lib().orc_centre_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                            px, py, j, r, C.byref(cu), C.byref(cv), _pd(w))
        return cu.value, cv.value, w

    def inner(self, px, py, j, r):
        out = np.zeros(3)
        n = lib().orc_inner_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                               px, py, j, r, _pd(out))
        return out, n

    def integrand(self, j, u, v, tau_t):
        out = np.zeros(3)
        lib().orc_integrand_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                               j, u, v, tau_t, _pd(out))
        return out

    def gk15(self, px, py, j, a, b):
        K, G, e = np.zeros(3), np.zeros(3), C.c_double()
        lib().orc_gk15_at(C.byref(self.params), C.byref(self.hist), C.byref(self.source),
                          px, py, j, a, b, _pd(K), _pd(G), C.byref(e))
        return K, G, e.value


# ---------------------------------------------------------------- free functions
def gk15_constants():
    x, wk, wg = np.zeros(8), np.zeros(8), np.zeros(4)
    lib().orc_gk15_constants(_pd(x), _pd(wk), _pd(wg))
    return x, wk, wg


def tsc_weights(d):
    w = np.zeros(3)
    lib().orc_tsc_weights(float(d), _pd(w))
    return w


def lagrange3_weights(t):
    w = np.zeros(3)
    lib().orc_lagrange3_weights(float(t), _pd(w))
    return w


def bin_of(x, y, fr, hx, hy, nx, ny):
    ix, iy, dx, dy = C.c_int32(), C.c_int32(), C.c_double(), C.c_double()
    b = lib().orc_bin_of(x, y, C.byref(frame(fr)), hx, hy, nx, ny, C.byref(ix), C.byref(iy),
                         C.byref(dx), C.byref(dy))
    return b, ix.value, iy.value, dx.value, dy.value


def deposit(x, y, ux, uy, q, fr, nx, ny, hx, hy):
    """Returns (M [ny,nx,4], bins int32[n], q_lost)."""
    x, y, ux, uy = (np.ascontiguousarray(a, dtype=np.float64) for a in (x, y, ux, uy))
    M = np.zeros((ny, nx, 4))
    bins = np.zeros(len(x), dtype=np.int32)
    ql = lib().orc_deposit(len(x), _pd(x), _pd(y), _pd(ux), _pd(uy), q, C.byref(frame(fr)),
                           nx, ny, hx, hy, _pd(M), _pi(bins))
    return M, bins, ql


def rigid_level(M0, f0, fl):
    """Step-0 moments M0 [ny,nx,4] as the same comoving bunch in frame fl (R-23)."""
    M0 = np.ascontiguousarray(M0, dtype=np.float64)
    ny, nx = M0.shape[:2]
    out = np.zeros_like(M0)
    lib().orc_rigid_level(_pd(M0), C.byref(frame(f0)), C.byref(frame(fl)), nx, ny, _pd(out))
    return out


def rigid_ring(M0, ring_frames, k=0, n_pre=None):
    """Ring [H,ny,nx,4] at step k = 0 of a rigid pre-history: slot(0) = M0, slot(l) for the
    n_pre levels l = -n_pre..-1 = rigid_level(M0, frame 0, frame l).  ``ring_frames`` as
    stored in the ring (slot(l) = l mod H)."""
    H = len(ring_frames)
    n_pre = H - 1 if n_pre is None else n_pre
    ring = np.zeros((H,) + np.shape(M0))
    ring[0] = M0
    for l in range(-n_pre, 0):
        ring[l % H] = rigid_level(M0, ring_frames[0], ring_frames[l % H])
    return ring


def arcs_rect(cu, cv, r, U0, U1, V0, V1):
    out = np.zeros(16)
    n = lib().orc_arcs_rect(cu, cv, r, U0, U1, V0, V1, _pd(out))
    return n, out[: 2 * max(n, 0)].reshape(-1, 2)


def arcs_disk(cu, cv, r, x0, y0, a):
    out = np.zeros(16)
    n = lib().orc_arcs_disk(cu, cv, r, x0, y0, a, _pd(out))
    return n, out[: 2 * max(n, 0)].reshape(-1, 2)


def fields(nx, ny, hx, hy, c, dt, frames, phi, ax, ay, a_prev=()):
    """frames: of levels k, k-1, ..., k-m; a_prev: the m previous (A_x, A_y) pairs, most recent
    first (m <= 4; order-m backward differences, R-15b).  m = 0: no dA/dt term."""
    P = Params(nx, ny, hx, hy, c, dt, 1.0, 64, 30, 2, 1, 0)
    phi, ax, ay = (np.ascontiguousarray(a, dtype=np.float64) for a in (phi, ax, ay))
    m = len(a_prev)
    fr = np.asarray(frames, dtype=np.float64).reshape(-1, 4)
    assert m <= 4 and len(fr) >= m + 1
    fa = (Frame * len(fr))(*[frame(f) for f in fr])
    prev = None
    if m:
        prev = np.ascontiguousarray(np.stack([np.stack([np.ravel(a), np.ravel(b)]) for a, b in a_prev]),
                                    dtype=np.float64)
    ex, ey, bz = np.zeros_like(phi), np.zeros_like(phi), np.zeros_like(phi)
    lib().orc_fields(C.byref(P), fa, m, _pd(phi), _pd(ax), _pd(ay), _pd(prev), _pd(ex), _pd(ey),
                     _pd(bz))
    return ex, ey, bz


def push(nx, ny, hx, hy, c, dt, fk, x, y, ux, uy, q_over_mc, bz_ext, ex, ey, bz):
    """In-place Boris push on copies; returns (x, y, ux, uy)."""
    P = Params(nx, ny, hx, hy, c, dt, 1.0, 64, 30, 2, 1, 0)
    x, y, ux, uy = (np.array(a, dtype=np.float64, copy=True) for a in (x, y, ux, uy))
    ex, ey, bz = (np.ascontiguousarray(a, dtype=np.float64) for a in (ex, ey, bz))
    lib().orc_push(C.byref(P), C.byref(frame(fk)), len(x), _pd(x), _pd(y), _pd(ux), _pd(uy),
                   q_over_mc, bz_ext, _pd(ex), _pd(ey), _pd(bz))
    return x, y, ux, uy


def forces(nx, ny, hx, hy, fk, x, y, ux, uy, bz_ext, ex, ey, bz):
    """Lorentz force per unit charge E + beta x B at each particle: (fx, fy)."""
    P = Params(nx, ny, hx, hy, 1.0, 1.0, 1.0, 64, 30, 2, 1, 0)
    x, y, ux, uy, ex, ey, bz = (np.ascontiguousarray(a, dtype=np.float64)
                                for a in (x, y, ux, uy, ex, ey, bz))
    fx, fy = np.zeros(len(x)), np.zeros(len(x))
    lib().orc_forces(C.byref(P), C.byref(frame(fk)), len(x), _pd(x), _pd(y), _pd(ux), _pd(uy),
                     bz_ext, _pd(ex), _pd(ey), _pd(bz), _pd(fx), _pd(fy))
    return fx, fy


def kick_external(dt, ux, uy, q_over_mc, bz_ext, frac=0.5):
    """Momenta advanced by frac * dt in the uniform external B_z (R-27): (ux, uy)."""
    P = Params(4, 4, 1.0, 1.0, 1.0, dt, 1.0, 64, 30, 2, 1, 0)
    ux, uy = (np.ascontiguousarray(a, dtype=np.float64) for a in (ux, uy))
    ox, oy = np.zeros(len(ux)), np.zeros(len(ux))
    lib().orc_kick_external(C.byref(P), len(ux), _pd(ux), _pd(uy), q_over_mc, bz_ext, frac,
                            _pd(ox), _pd(oy))
    return ox, oy
