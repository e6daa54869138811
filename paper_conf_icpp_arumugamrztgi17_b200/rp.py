"""Thin Python binding of librp (include/rp.h): argument marshalling only.

Every function here has the name of the C entry point it calls and does nothing but
check/convert arguments (torch CUDA tensors -> device pointers, numpy -> host pointers)
and raise ``RpError`` on a non-zero return code.  All arithmetic of the method runs in
the CUDA kernels of ``csrc/``.  There is no CPU fallback: if ``librp.so`` is missing or
cannot be loaded, importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "librp.so")

RP_SRC_GRID, RP_SRC_GAUSS, RP_SRC_DISK = 0, 1, 2
RP_SCHED_INDEX, RP_SCHED_PERSISTENCE, RP_SCHED_KNN, RP_SCHED_SUBREGION = 0, 1, 2, 3
RP_RULE_GK15, RP_RULE_SIMPSON = 0, 1


class RpError(RuntimeError):
    def __init__(self, code: int, where: str, detail: str):
        super().__init__(f"{where}: {rp_strerror(code)} ({code}): {detail}")
        self.code = code


class rp_frame(C.Structure):
    _fields_ = [("ox", C.c_double), ("oy", C.c_double), ("cos_psi", C.c_double),
                ("sin_psi", C.c_double)]


class rp_config(C.Structure):
    _fields_ = [("nx", C.c_int32), ("ny", C.c_int32), ("hx", C.c_double), ("hy", C.c_double),
                ("history_depth", C.c_int32), ("c", C.c_double), ("dt", C.c_double),
                ("tau", C.c_double), ("n_theta", C.c_int32), ("max_depth", C.c_int32),
                ("n_root", C.c_int32), ("device", C.c_int32), ("outer_rule", C.c_int32),
                ("interp", C.c_int32)]


class rp_deposit_info(C.Structure):
    _fields_ = [("n_lost", C.c_int64), ("q_lost", C.c_double), ("q_total", C.c_double)]


class rp_profile(C.Structure):
    _fields_ = [("deposit_ms", C.c_double), ("append_ms", C.c_double), ("clip_ms", C.c_double),
                ("sort_ms", C.c_double), ("integrate_ms", C.c_double), ("reduce_ms", C.c_double),
                ("fields_ms", C.c_double), ("push_ms", C.c_double),
                ("integrate_launches", C.c_int64), ("units_ms", C.c_double),
                ("step_ms", C.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class rp_potential_info(C.Structure):
    _fields_ = [("evals", C.c_int64), ("nodes", C.c_int64), ("segments", C.c_int64),
                ("leaves", C.c_int64), ("capped", C.c_int64), ("ties", C.c_int64),
                ("items", C.c_int64), ("max_level", C.c_int32), ("kappa", C.c_int32),
                ("skipped", C.c_int64), ("units", C.c_int64)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


RP_NCCL_ID_BYTES = 128


class rp_dist(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("nccl_comm", C.c_void_p),
                ("nccl_id", C.c_ubyte * RP_NCCL_ID_BYTES)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class rp_predictive_info(C.Structure):
    _fields_ = [("active", C.c_int32), ("clusters", C.c_int32), ("kmeans_passes", C.c_int32),
                ("partition", C.c_int32), ("breakpoints", C.c_int64), ("host_ms", C.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


if not os.path.exists(LIB_PATH):
    raise ImportError(f"librp.so not built at {LIB_PATH}: run "
                      "`python -m paper_conf_icpp_arumugamrztgi17_b200.build` (no CPU fallback)")
_lib = C.CDLL(LIB_PATH)

_P = C.POINTER
_vp, _d, _i32, _i64 = C.c_void_p, C.c_double, C.c_int32, C.c_int64
_SIG = {
    "rp_version": (C.c_int, []),
    "rp_strerror": (C.c_char_p, [C.c_int]),
    "rp_last_error": (C.c_char_p, [_vp]),
    "rp_launch_count": (_i64, [_vp]),
    "rp_profile_enable": (C.c_int, [_vp, _i32]),
    "rp_set_schedule": (C.c_int, [_vp, _i32, _i32]),
    "rp_set_predictive": (C.c_int, [_vp, _i32, _i32, _i32, _i32]),
    "rp_predictive_info_read": (C.c_int, [_vp, _P(rp_predictive_info), _vp]),
    "rp_profile_read": (C.c_int, [_vp, _P(rp_profile)]),
    "rp_create": (C.c_int, [_P(rp_config), _P(rp_dist), _P(_vp)]),
    "rp_nccl_unique_id": (C.c_int, [_vp]),
    "rp_set_work_split": (C.c_int, [_vp, _i32, _i32]),
    "rp_set_predictive_partition": (C.c_int, [_vp, _i32]),
    "rp_predictive_lists_read": (C.c_int, [_vp, _vp, _vp]),
    "rp_destroy": (None, [_vp]),
    "rp_set_stream": (C.c_int, [_vp, _vp]),
    "rp_history_init": (C.c_int, [_vp, _i32, _P(rp_frame), _vp, _i32]),
    "rp_deposit": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _d, _i64, _P(rp_frame), _vp,
                             _P(rp_deposit_info)]),
    "rp_history_append": (C.c_int, [_vp, _vp, _i32, _P(rp_frame)]),
    "rp_partial_bytes": (_i64, [_vp]),
    "rp_deposit_step": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _d, _i64, _P(rp_frame),
                                  _P(rp_deposit_info)]),
    "rp_compute_potentials": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _vp, _P(rp_potential_info)]),
    "rp_compute_potentials_shard": (C.c_int, [_vp, _i32, _i32, _vp, _i64, _P(_i64),
                                              _P(rp_potential_info)]),
    "rp_shard_capacity": (_i64, [_vp, _i32]),
    "rp_shard_scatter": (C.c_int, [_vp, _vp, _i32, _i64, _vp, _vp, _vp, _vp, _vp]),
    "rp_compute_fields": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _i32, _vp, _vp, _vp]),
    "rp_push_particles": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _i64, _d, _d, _vp, _vp, _vp]),
    "rp_particle_forces": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _i64, _d, _vp, _vp, _vp, _vp, _vp]),
    "rp_kick_external": (C.c_int, [_vp, _vp, _vp, _i64, _d, _d, _d, _vp, _vp]),
    "rp_step_host": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _i64, _d, _P(rp_frame), _d, _d, _vp,
                               _P(rp_potential_info)]),
    "rp_load_state": (C.c_int, [_vp, _i32, _i32, _P(rp_frame), _vp]),
    "rp_save_state": (C.c_int, [_vp, _P(_i32), _vp, _P(rp_frame)]),
    "rp_debug_bins": (C.c_int, [_vp, _vp, _i64]),
    "rp_debug_clip": (C.c_int, [_vp, _vp, _i64]),
    "rp_debug_point_counts": (C.c_int, [_vp, _vp, _vp, _i64]),
    "rp_debug_item_leaves": (C.c_int, [_vp, _vp, _i64]),
    "rp_debug_potentials_analytic": (C.c_int, [_vp, _i32, _d, _d, _d, _d, _d, _d, _vp, _vp, _vp,
                                               _vp, _vp, _vp, _P(rp_potential_info)]),
}
for _name, (_res, _args) in _SIG.items():
    _fn = getattr(_lib, _name)
    _fn.restype = _res
    _fn.argtypes = _args

EXPORTED = tuple(_SIG)


# ---------------------------------------------------------------- marshalling helpers
def _dev(t, dtype=None, name="array"):
    """Device pointer of a contiguous CUDA tensor (or None -> NULL)."""
    if t is None:
        return None
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name}: expected a CUDA torch tensor")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"{name}: expected {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    return C.c_void_p(t.data_ptr())


def _f64(t, name="array"):
    import torch
    return _dev(t, torch.float64, name)


def _i32t(t, name="array"):
    import torch
    return _dev(t, torch.int32, name)


def _host(a, dtype=np.float64, name="array"):
    if a is None:
        return None
    if hasattr(a, "data_ptr"):  # pinned torch CPU tensor
        if a.is_cuda or not a.is_contiguous():
            raise TypeError(f"{name}: expected a contiguous CPU tensor")
        return C.c_void_p(a.data_ptr())
    if a.dtype != dtype or not a.flags.c_contiguous:
        raise TypeError(f"{name}: expected contiguous {dtype}")
    return C.c_void_p(a.ctypes.data)


def frame(f) -> rp_frame:
    if isinstance(f, rp_frame):
        return f
    return rp_frame(*[float(v) for v in f])


def frames_array(fr):
    fr = np.asarray(fr, dtype=np.float64).reshape(-1, 4)
    return (rp_frame * len(fr))(*[rp_frame(*row) for row in fr])


def _check(rc: int, ctx, where: str):
    if rc != 0:
        detail = _lib.rp_last_error(ctx).decode() if ctx else ""
        raise RpError(rc, where, detail)


# ---------------------------------------------------------------- API (same names as the C ABI)
def rp_version() -> int:
    return _lib.rp_version()


def rp_strerror(code: int) -> str:
    return _lib.rp_strerror(code).decode()


def rp_last_error(ctx) -> str:
    return _lib.rp_last_error(ctx).decode()


def rp_launch_count(ctx) -> int:
    return _lib.rp_launch_count(ctx)


def rp_set_schedule(ctx, policy, k=9) -> None:
    _check(_lib.rp_set_schedule(ctx, int(policy), int(k)), ctx, "rp_set_schedule")


def rp_set_predictive(ctx, enable=True, knn=9, n_clusters=0, max_iters=20) -> None:
    _check(_lib.rp_set_predictive(ctx, int(bool(enable)), int(knn), int(n_clusters),
                                  int(max_iters)), ctx, "rp_set_predictive")


RP_PART_UNIFORM, RP_PART_ADAPTIVE = 0, 1


def rp_set_predictive_partition(ctx, mode) -> None:
    """Line 4 of the Predictive-RP variant: RP_PART_UNIFORM or RP_PART_ADAPTIVE
    (reading R-26b)."""
    _check(_lib.rp_set_predictive_partition(ctx, int(mode)), ctx, "rp_set_predictive_partition")


def rp_predictive_lists_read(ctx, n_lists, n_bp):
    """The last merged partition lists: (off int64 [n_lists + 1], bp float64 [n_bp]) with
    n_lists = clusters * history_depth and n_bp = rp_predictive_info.breakpoints."""
    off = np.zeros(int(n_lists) + 1, dtype=np.int64)
    bp = np.zeros(max(int(n_bp), 1), dtype=np.float64)
    _check(_lib.rp_predictive_lists_read(ctx, off.ctypes.data_as(_vp), bp.ctypes.data_as(_vp)),
           ctx, "rp_predictive_lists_read")
    return off, bp[:int(n_bp)]


def rp_predictive_info_read(ctx, npts=None):
    """Returns rp_predictive_info; with npts = nx * ny also the int32 [npts] point clusters."""
    info = rp_predictive_info()
    if npts is None:
        _check(_lib.rp_predictive_info_read(ctx, C.byref(info), None), ctx, "rp_predictive_info_read")
        return info
    out = np.zeros(int(npts), dtype=np.int32)
    _check(_lib.rp_predictive_info_read(ctx, C.byref(info), out.ctypes.data_as(_vp)), ctx,
           "rp_predictive_info_read")
    return info, out


def rp_profile_enable(ctx, enable=True) -> None:
    _check(_lib.rp_profile_enable(ctx, int(bool(enable))), ctx, "rp_profile_enable")


def rp_profile_read(ctx) -> rp_profile:
    out = rp_profile()
    _check(_lib.rp_profile_read(ctx, C.byref(out)), ctx, "rp_profile_read")
    return out


def rp_nccl_unique_id() -> bytes:
    """A fresh ncclUniqueId (128 bytes) for rp_create's rp_dist (call on rank 0, broadcast)."""
    buf = (C.c_ubyte * RP_NCCL_ID_BYTES)()
    _check(_lib.rp_nccl_unique_id(C.cast(buf, _vp)), None, "rp_nccl_unique_id")
    return bytes(buf)


def rp_create(nx, ny, hx, hy, history_depth, c, dt, tau, n_theta=64, max_depth=30, n_root=2,
              device=0, outer_rule=0, interp=0, dist=None):
    """dist: None (single GPU) or (rank, world, nccl_id bytes) -- librp then creates the
    NCCL communicator (collective over the ranks) and exchanges inside its calls."""
    cfg = rp_config(nx, ny, hx, hy, history_depth, c, dt, tau, n_theta, max_depth, n_root, device,
                    outer_rule, interp)
    d = None
    if dist is not None:
        rank, world, nid = dist
        if len(nid) != RP_NCCL_ID_BYTES:
            raise ValueError("nccl_id: expected 128 bytes")
        d = rp_dist(int(rank), int(world), None, (C.c_ubyte * RP_NCCL_ID_BYTES)(*nid))
    out = C.c_void_p()
    _check(_lib.rp_create(C.byref(cfg), C.byref(d) if d is not None else None, C.byref(out)),
           None, "rp_create")
    return out


def rp_set_work_split(ctx, level, budget=0) -> None:
    _check(_lib.rp_set_work_split(ctx, int(level), int(budget)), ctx, "rp_set_work_split")


def rp_destroy(ctx) -> None:
    _lib.rp_destroy(ctx)


def rp_set_stream(ctx, stream) -> None:
    """stream: a torch.cuda.Stream (or None for the legacy default stream)."""
    ptr = None if stream is None else C.c_void_p(stream.cuda_stream)
    _check(_lib.rp_set_stream(ctx, ptr), ctx, "rp_set_stream")


def rp_history_init(ctx, n_pre, frames, grids=None, rigid=True) -> None:
    fa = frames_array(frames)
    assert len(fa) == n_pre
    _check(_lib.rp_history_init(ctx, n_pre, fa, _f64(grids, "grids"), int(bool(rigid))), ctx,
           "rp_history_init")


def rp_partial_bytes(ctx) -> int:
    return _lib.rp_partial_bytes(ctx)


def rp_deposit(ctx, x, y, ux, uy, q, frame_k, partial, info=False):
    """partial: uint8 CUDA tensor of rp_partial_bytes(ctx) bytes (opaque exact sums)."""
    inf = rp_deposit_info() if info else None
    if partial.numel() * partial.element_size() < rp_partial_bytes(ctx):
        raise ValueError("partial: smaller than rp_partial_bytes(ctx)")
    _check(_lib.rp_deposit(ctx, _f64(x, "x"), _f64(y, "y"), _f64(ux, "ux"), _f64(uy, "uy"),
                           float(q), x.numel(), C.byref(frame(frame_k)), _dev(partial, None, "partial"),
                           C.byref(inf) if inf is not None else None), ctx, "rp_deposit")
    return inf


def rp_history_append(ctx, partials, n_parts, frame_k) -> None:
    """partials: n_parts consecutive partial buffers (uint8 CUDA tensor)."""
    _check(_lib.rp_history_append(ctx, _dev(partials, None, "partials"), n_parts,
                                  C.byref(frame(frame_k))),
           ctx, "rp_history_append")


def rp_deposit_step(ctx, x, y, ux, uy, q, frame_k, info=False):
    inf = rp_deposit_info() if info else None
    _check(_lib.rp_deposit_step(ctx, _f64(x, "x"), _f64(y, "y"), _f64(ux, "ux"), _f64(uy, "uy"),
                                float(q), x.numel(), C.byref(frame(frame_k)),
                                C.byref(inf) if inf is not None else None), ctx, "rp_deposit_step")
    return inf


def rp_compute_potentials(ctx, phi, ax, ay, err=None, nseg=None, info=False):
    inf = rp_potential_info() if info else None
    _check(_lib.rp_compute_potentials(ctx, _f64(phi, "phi"), _f64(ax, "ax"), _f64(ay, "ay"),
                                      _f64(err, "err"), _i32t(nseg, "nseg"),
                                      C.byref(inf) if inf is not None else None), ctx,
           "rp_compute_potentials")
    return inf


def rp_shard_capacity(ctx, world) -> int:
    return _lib.rp_shard_capacity(ctx, world)


def rp_compute_potentials_shard(ctx, rank, world, shard_out, info=False):
    inf = rp_potential_info() if info else None
    n = C.c_int64()
    cap = shard_out.shape[0]
    _check(_lib.rp_compute_potentials_shard(ctx, rank, world, _f64(shard_out, "shard_out"), cap,
                                            C.byref(n), C.byref(inf) if inf is not None else None),
           ctx, "rp_compute_potentials_shard")
    return n.value, inf


def rp_shard_scatter(ctx, shards, world, phi, ax, ay, err=None, nseg=None) -> None:
    cap = shards.shape[-2]
    _check(_lib.rp_shard_scatter(ctx, _f64(shards, "shards"), world, cap, _f64(phi, "phi"),
                                 _f64(ax, "ax"), _f64(ay, "ay"), _f64(err, "err"),
                                 _i32t(nseg, "nseg")), ctx, "rp_shard_scatter")


def rp_compute_fields(ctx, phi, ax, ay, a_prev, ex, ey, bz, n_prev=None) -> None:
    """a_prev: None, or a float64 CUDA tensor [n_prev][2][npts] of (A_x, A_y) at steps k-1, ...
    (most recent first); n_prev defaults to its first dimension (0..4)."""
    if a_prev is None:
        n = 0
    else:
        n = a_prev.shape[0] if n_prev is None else int(n_prev)
    _check(_lib.rp_compute_fields(ctx, _f64(phi), _f64(ax), _f64(ay), _f64(a_prev, "a_prev"), n,
                                  _f64(ex), _f64(ey), _f64(bz)), ctx, "rp_compute_fields")


def rp_push_particles(ctx, x, y, ux, uy, q_over_mc, bz_ext, ex, ey, bz) -> None:
    _check(_lib.rp_push_particles(ctx, _f64(x), _f64(y), _f64(ux), _f64(uy), x.numel(),
                                  float(q_over_mc), float(bz_ext), _f64(ex), _f64(ey), _f64(bz)),
           ctx, "rp_push_particles")


def rp_particle_forces(ctx, x, y, ux, uy, bz_ext, ex, ey, bz, fx, fy) -> None:
    _check(_lib.rp_particle_forces(ctx, _f64(x, "x"), _f64(y, "y"), _f64(ux, "ux"), _f64(uy, "uy"),
                                   x.numel(), float(bz_ext), _f64(ex, "ex"), _f64(ey, "ey"),
                                   _f64(bz, "bz"), _f64(fx, "fx"), _f64(fy, "fy")), ctx,
           "rp_particle_forces")


def rp_kick_external(ctx, ux, uy, q_over_mc, bz_ext, frac, ux_out, uy_out) -> None:
    _check(_lib.rp_kick_external(ctx, _f64(ux, "ux"), _f64(uy, "uy"), ux.numel(), float(q_over_mc),
                                 float(bz_ext), float(frac), _f64(ux_out, "ux_out"),
                                 _f64(uy_out, "uy_out")), ctx, "rp_kick_external")


def rp_step_host(ctx, x, y, ux, uy, q, frame_k, q_over_mc, bz_ext, mesh_out, info=False):
    """x..uy and mesh_out ([6, npts]) are host buffers (pinned torch CPU tensors or numpy)."""
    n = x.numel() if hasattr(x, "numel") else len(x)
    inf = rp_potential_info() if info else None
    _check(_lib.rp_step_host(ctx, _host(x), _host(y), _host(ux), _host(uy), n, float(q),
                             C.byref(frame(frame_k)), float(q_over_mc), float(bz_ext),
                             _host(mesh_out), C.byref(inf) if inf is not None else None), ctx,
           "rp_step_host")
    return inf


def rp_load_state(ctx, k, n_pre, frames, ring) -> None:
    fa = frames_array(frames)
    _check(_lib.rp_load_state(ctx, k, n_pre, fa, _f64(ring, "ring")), ctx, "rp_load_state")


def rp_save_state(ctx, ring=None, H=None):
    k = C.c_int32()
    fa = (rp_frame * H)() if H else None
    _check(_lib.rp_save_state(ctx, C.byref(k), _f64(ring, "ring"), fa), ctx, "rp_save_state")
    frames = None
    if fa is not None:
        frames = np.array([[f.ox, f.oy, f.cos_psi, f.sin_psi] for f in fa])
    return k.value, frames


def rp_debug_clip(ctx, ab) -> None:
    """ab: float64 CUDA tensor of nx*ny*history_depth*2 elements ((A, B) per item)."""
    _check(_lib.rp_debug_clip(ctx, _f64(ab, "ab"), ab.numel() // 2), ctx, "rp_debug_clip")


def rp_debug_item_leaves(ctx, out) -> None:
    """out: torch.int16 tensor of nx * ny * history_depth elements (the uint16 counts)."""
    _check(_lib.rp_debug_item_leaves(ctx, C.c_void_p(out.data_ptr()), out.numel()), ctx,
           "rp_debug_item_leaves")


def rp_debug_point_counts(ctx, nleaf=None, capped=None) -> None:
    """nleaf / capped: int32 CUDA tensors of nx*ny elements (either may be None)."""
    n = (nleaf if nleaf is not None else capped).numel()
    _check(_lib.rp_debug_point_counts(ctx, _i32t(nleaf, "nleaf"), _i32t(capped, "capped"), n),
           ctx, "rp_debug_point_counts")


def rp_debug_bins(ctx, bins) -> None:
    _check(_lib.rp_debug_bins(ctx, _i32t(bins, "bins"), bins.numel()), ctx, "rp_debug_bins")


def rp_debug_potentials_analytic(ctx, kind, x0, y0, width, q, bx, by, amp, phi, ax, ay,
                                 err=None, nseg=None, info=False):
    inf = rp_potential_info() if info else None
    amp_p = None
    if amp is not None:
        amp = np.ascontiguousarray(amp, dtype=np.float64)
        amp_p = C.c_void_p(amp.ctypes.data)
    _check(_lib.rp_debug_potentials_analytic(ctx, kind, x0, y0, width, q, bx, by, amp_p,
                                             _f64(phi), _f64(ax), _f64(ay), _f64(err),
                                             _i32t(nseg), C.byref(inf) if inf is not None else None),
           ctx, "rp_debug_potentials_analytic")
    return inf
