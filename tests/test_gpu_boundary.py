"""The C-ABI contract of include/rp.h on the GPU: stream-ordered, enqueue-only
calls (no host synchronisation inside rp_compute_potentials), CUDA-graph capture of a whole
potentials call, and the multi-GPU path through librp's own NCCL communicator (a one-rank
communicator on the one-GPU test box: the same calls and code path as N > 1, exchanges
included, bit-identical to the single-GPU context).  Alg. 1's single COMPUTE-POTENTIALS call
per step is what rp_compute_potentials implements."""
import time

import numpy as np
import pytest

import workloads as W
from tests import gpu_util as G

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch():
    import torch as t
    assert t.cuda.is_available()
    return t


def _state_cfg2(torch, ctx, cfg):
    """Rigid pre-history + the GPU deposit of config 2's bunch (the bench state at step 0)."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    x, y, ux, uy = W.particles(cfg)
    dev = [torch.tensor(a, dtype=torch.float64, device="cuda") for a in (x, y, ux, uy)]
    rp.rp_history_init(ctx, cfg.n_pre, W.frames(cfg, range(-cfg.n_pre, 0)), None, True)
    rp.rp_deposit_step(ctx, *dev, 1.0 / len(x), W.frame(cfg, 0))
    return dev


def _outs(torch, n):
    f = dict(dtype=torch.float64, device="cuda")
    return ([torch.zeros(n, **f) for _ in range(4)], torch.zeros(n, dtype=torch.int32, device="cuda"))


def test_compute_potentials_returns_before_its_kernels_finish(torch):
    """rp.h: calls return after enqueueing unless 'syncs' is stated -- the unit launch reads its
    count on the device, so there is no host round trip in the integrator."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(2)
    ctx = G.make_ctx(cfg)
    try:
        stream = torch.cuda.current_stream()
        rp.rp_set_stream(ctx, stream)
        _state_cfg2(torch, ctx, cfg)
        (phi, ax, ay, err), nseg = _outs(torch, cfg.nx * cfg.ny)
        rp.rp_compute_potentials(ctx, phi, ax, ay, err, nseg)  # warm-up: sizes the scratch
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rp.rp_compute_potentials(ctx, phi, ax, ay, err, nseg)
        host_ms = 1e3 * (time.perf_counter() - t0)
        ev = torch.cuda.Event()
        ev.record(stream)
        pending = not ev.query()
        t1 = time.perf_counter()
        ev.synchronize()
        wait_ms = 1e3 * (time.perf_counter() - t1)
        assert pending, "the device work had already finished when the call returned"
        assert wait_ms > 5 * host_ms, (host_ms, wait_ms)
    finally:
        rp.rp_destroy(ctx)


def test_cuda_graph_capture_of_compute_potentials(torch):
    """One rp_compute_potentials call captured in a CUDA graph and replayed gives the results
    of a direct call bit for bit (the schedule forecast only orders the work)."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    ctx = G.make_ctx(cfg)
    try:
        s = torch.cuda.Stream()
        rp.rp_set_stream(ctx, s)
        n = cfg.nx * cfg.ny
        with torch.cuda.stream(s):
            _state_cfg2(torch, ctx, cfg)
            (phi, ax, ay, err), nseg = _outs(torch, n)
            rp.rp_compute_potentials(ctx, phi, ax, ay, err, nseg)  # direct call (and warm-up)
        s.synchronize()
        ref = [t.clone() for t in (phi, ax, ay, err, nseg)]
        for t in (phi, ax, ay, err):
            t.zero_()
        nseg.zero_()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            rp.rp_compute_potentials(ctx, phi, ax, ay, err, nseg)
        g.replay()
        g.replay()
        torch.cuda.synchronize()
        for a, b in zip((phi, ax, ay, err, nseg), ref):
            assert torch.equal(a, b)
        assert float(phi.abs().max()) > 0
    finally:
        rp.rp_destroy(ctx)


def test_nccl_one_rank_communicator_matches_single_gpu(torch):
    """rp_create with an rp_dist (librp creates the NCCL communicator from a unique id):
    deposit_step / compute_potentials then run the sharded path with NCCL all-gathers inside
    the library.  With one rank the results equal the plain single-GPU context bit for bit
    over three full steps."""
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
    cfg = W.config(1)
    a = Simulation(cfg)
    b = Simulation(cfg, transport="nccl", nccl_id=rp.rp_nccl_unique_id())
    try:
        for _ in range(3):
            a.step()
            inf = b.step(info=True)
            assert inf.segments > 0
            for t1, t2 in ((a.phi, b.phi), (a.ax, b.ax), (a.ay, b.ay), (a.err, b.err),
                           (a.nseg, b.nseg), (a.ex, b.ex), (a.bz, b.bz), (a.x, b.x), (a.uy, b.uy)):
                assert torch.equal(t1, t2)
    finally:
        a.close()
        b.close()
