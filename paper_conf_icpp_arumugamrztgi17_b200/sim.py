"""One time step of the paper's loop on one GPU per process, optionally sharded
over ranks (mesh points sharded, history replicated).

Per step k on every rank (torch.distributed is plumbing only; every arithmetic step
runs in librp's kernels):

  world == 1, or world > 1 with transport "nccl" (the product path: librp owns an NCCL
  communicator made from a unique id broadcast over the process group, and exchanges inside
  its calls):
               rp_deposit_step -> rp_compute_potentials                  [full mesh]
  world > 1 with transport "host" (a caller-side transport, e.g. gloo for the CPU tests
  and for two ranks sharing one GPU, where NCCL refuses duplicate devices):
               rp_deposit(local particle shard) -> all_gather(partial grids)
               -> rp_history_append(partials in rank order)              [replicated ring]
               -> rp_compute_potentials_shard(rank)                      [owned points]
               -> all_gather(shards) -> rp_shard_scatter                 [full mesh]
  then         rp_compute_fields (replicated) -> rp_push_particles (local shard)

Both transports give bit-identical results for any number of ranks (exact deposition, the
same shard map).  ``ops`` defaults to the librp binding; tests substitute a CPU stand-in to
exercise the multi-process plumbing with the gloo backend.
"""
from __future__ import annotations

import numpy as np
import torch

import workloads as W


class Simulation:
    def __init__(self, cfg: W.Config, device=None, group=None, ops=None, particles=None,
                 transport: str = "host", nccl_id: bytes | None = None):
        """nccl_id (transport "nccl"): a unique id already agreed on by the ranks (else rank 0
        makes one and broadcasts it over `group`); with one process it gives a one-rank
        communicator -- the N > 1 code path on one GPU."""
        if ops is None:
            from . import rp as ops
        self.ops = ops
        self.cfg = cfg
        self.group = group
        if group is not None:
            import torch.distributed as dist
            self.rank, self.world = dist.get_rank(group), dist.get_world_size(group)
        else:
            self.rank, self.world = 0, 1
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        dev_index = self.device.index if self.device.type == "cuda" else 0
        if transport not in ("host", "nccl"):
            raise ValueError(transport)
        # librp exchanges over its own NCCL communicator (world > 1, transport "nccl")
        self.in_lib = self.world == 1 or transport == "nccl"
        dist_arg = None
        if transport == "nccl" and (self.world > 1 or nccl_id is not None):
            if nccl_id is None:
                import torch.distributed as dist
                obj = [ops.rp_nccl_unique_id() if self.rank == 0 else None]
                dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0), group=group)
                nccl_id = obj[0]
            dist_arg = (self.rank, self.world, nccl_id)
        self.ctx = ops.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt,
                                 cfg.tau, cfg.n_theta, cfg.max_depth, cfg.n_root, dev_index or 0,
                                 cfg.rule, cfg.interp, dist=dist_arg)
        if self.device.type == "cuda":
            ops.rp_set_stream(self.ctx, torch.cuda.current_stream(self.device))
        ops.rp_history_init(self.ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
        x, y, ux, uy = W.particles(cfg) if particles is None else particles
        n = len(x)
        lo, hi = (n * self.rank) // self.world, (n * (self.rank + 1)) // self.world
        f64 = dict(dtype=torch.float64, device=self.device)
        self.x, self.y, self.ux, self.uy = (torch.tensor(np.ascontiguousarray(a[lo:hi]), **f64)
                                            for a in (x, y, ux, uy))
        # time-centred momenta of the deposit (R-27)
        self.cux, self.cuy = torch.empty_like(self.ux), torch.empty_like(self.uy)
        self.q = 1.0 / n
        npts = cfg.nx * cfg.ny
        self.npts = npts
        self.phi, self.err, self.ex, self.ey, self.bz = (torch.zeros(npts, **f64) for _ in range(5))
        # A of the current step and of the 4 before, for the fields' dA/dt (R-15b)
        self.Ahist = torch.zeros((5, 2, npts), **f64)
        self.n_prev = 0
        self.nseg = torch.zeros(npts, dtype=torch.int32, device=self.device)
        self.k = 0
        if not self.in_lib:
            pb = ops.rp_partial_bytes(self.ctx)  # opaque exact partial sums
            self.partial = torch.zeros(pb, dtype=torch.uint8, device=self.device)
            self.partials = torch.zeros(self.world * pb, dtype=torch.uint8, device=self.device)
            cap = ops.rp_shard_capacity(self.ctx, self.world)
            self.shard = torch.zeros((cap, 6), **f64)
            self.shards = torch.zeros((self.world, cap, 6), **f64)

    # ------------------------------------------------------------------
    @property
    def ax(self):
        """A_x of the last completed step."""
        return self.Ahist[0, 0]

    @property
    def ay(self):
        return self.Ahist[0, 1]

    def step(self, info: bool = False):
        """Advance one step; returns rp_potential_info (syncs) when info=True."""
        import torch.distributed as dist
        ops, cfg = self.ops, self.cfg
        fk = W.frame(cfg, self.k)
        # shift the A history: slot 0 receives this step's A, slots 1.. hold steps k-1, k-2, ...
        self.Ahist[1:] = self.Ahist[:-1].clone()
        ax, ay = self.Ahist[0, 0], self.Ahist[0, 1]
        # the current of step k with the momenta of t_k: leap-frog momenta + half a step (R-27)
        ops.rp_kick_external(self.ctx, self.ux, self.uy, cfg.q_over_mc, cfg.bz_ext, 0.5, self.cux,
                             self.cuy)
        if self.in_lib:
            ops.rp_deposit_step(self.ctx, self.x, self.y, self.cux, self.cuy, self.q, fk)
            inf = ops.rp_compute_potentials(self.ctx, self.phi, ax, ay, self.err, self.nseg, info=info)
        else:
            ops.rp_deposit(self.ctx, self.x, self.y, self.cux, self.cuy, self.q, fk, self.partial)
            dist.all_gather_into_tensor(self.partials.view(-1), self.partial.view(-1), group=self.group)
            ops.rp_history_append(self.ctx, self.partials, self.world, fk)
            _, inf = ops.rp_compute_potentials_shard(self.ctx, self.rank, self.world, self.shard, info=info)
            dist.all_gather_into_tensor(self.shards.view(-1), self.shard.view(-1), group=self.group)
            ops.rp_shard_scatter(self.ctx, self.shards, self.world, self.phi, ax, ay, self.err, self.nseg)
        prev = self.Ahist[1:1 + self.n_prev] if self.n_prev else None
        ops.rp_compute_fields(self.ctx, self.phi, ax, ay, prev, self.ex, self.ey, self.bz)
        self.n_prev = min(self.n_prev + 1, 4)
        ops.rp_push_particles(self.ctx, self.x, self.y, self.ux, self.uy, cfg.q_over_mc, cfg.bz_ext,
                              self.ex, self.ey, self.bz)
        self.k += 1
        return inf

    def close(self):
        if self.ctx is not None:
            self.ops.rp_destroy(self.ctx)
            self.ctx = None

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass
