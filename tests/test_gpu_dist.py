"""The sharded multi-rank step through the real CUDA library: two processes share the one GPU
of the test box and talk through torch.distributed's gloo backend (CUDA tensors), so every
rank runs librp's kernels in the sharded mode (partial deposit -> all-gather -> rank-ordered
append -> owned-point potentials -> all-gather -> scatter -> fields -> local push).  The
result must equal the single-rank run BIT FOR BIT: the partial deposits are exact fixed-point
sums, so the history ring does not depend on how the particles are split over ranks.  On the 8-GPU driver box the same code
path runs with NCCL (bench.py under torchrun)."""
import os
import queue
import socket

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu


def _cfg():
    return W.config(1)


def _run(world, rank, port, q):
    import torch
    import torch.distributed as dist
    from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation
    torch.cuda.set_device(0)
    group = None
    if world > 1:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        group = dist.group.WORLD
    cfg = _cfg()
    sim = Simulation(cfg, group=group)
    out = []
    for _ in range(3):
        sim.step()
        out.append(np.stack([sim.phi.cpu().numpy(), sim.ax.cpu().numpy(), sim.ay.cpu().numpy(),
                             sim.ex.cpu().numpy(), sim.nseg.cpu().numpy().astype(np.float64)]))
    x = sim.x.cpu().numpy()
    sim.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    q.put((rank, np.stack(out), x))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_two_ranks_on_one_gpu_match_one_rank():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q1 = ctx.Queue()
    p = ctx.Process(target=_run, args=(1, 0, 0, q1))
    p.start()
    _, ref, xref = q1.get(timeout=300)
    p.join(60)
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_run, args=(2, r, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    got = {}
    while len(got) < 2:
        try:
            r, v, x = q.get(timeout=5)
            got[r] = (v, x)
        except queue.Empty:
            assert all(pr.is_alive() for pr in procs), "a rank died"
    for pr in procs:
        pr.join(60)
        assert pr.exitcode == 0
    for r in range(2):
        np.testing.assert_array_equal(got[r][0], ref)
    np.testing.assert_array_equal(np.concatenate([got[0][1], got[1][1]]), xref)
