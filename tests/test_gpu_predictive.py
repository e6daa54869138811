"""GPU parity of the Predictive-RP variant (the paper's Algorithm 1 COMPUTE-POTENTIALS,
P:110-166; DESIGN reading R-26) through the C ABI: the previous step runs the canonical
tree on both sides (each side records its own observed access pattern n_j(p)); the next step
forecasts, clusters, merges and integrates over the merged partitions on both sides.

Bars: k-means clusters identical; potentials within 1e-11 * max(|phi|, |A|) per point with
equal segment counts; the results stay within tau of the canonical tree's.
"""
import numpy as np
import pytest

import oracle
import workloads as W
from tests import gpu_util as G
from tests.test_gpu_parity import _bend_small, _deposit_rigid_ring

pytestmark = pytest.mark.gpu


def _two_steps(cfg, rings, n_pre, knn, m, pts=None, part=0):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    (k0, ring0, fr0), (k1, ring1, fr1) = rings
    npts = cfg.nx * cfg.ny
    allp = np.arange(npts)
    pts = allp if pts is None else pts
    o0 = G.oracle_problem(cfg, ring0, fr0, k0, n_pre)
    o1 = G.oracle_problem(cfg, ring1, fr1, k1, n_pre)
    if part == 0:  # uniform partitioning
        canon0, leaves0 = o0.potentials_items(allp)
        pred1, clusters1, _, passes = o1.potentials_predictive(leaves0, pts, knn=knn, m=m)
    else:  # adaptive partitioning (R-26b) from step 0's accepted partitions
        canon0, leaves0, off0, plen0, parts0 = o0.potentials_parts(allp)
        pred1, clusters1, _, passes = o1.potentials_predictive_adaptive(
            leaves0, off0, plen0, parts0, pts, knn=knn, m=m)
    canon1 = o1.potentials(pts)
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_predictive(ctx, True, knn, m, 20)
        rp.rp_set_predictive_partition(ctx, part)
        G.load_state(ctx, cfg, k0, n_pre, ring0, fr0)
        gpu0, _ = G.gpu_potentials(ctx, npts)  # no previous pattern yet: canonical tree
        assert rp.rp_predictive_info_read(ctx).active == 0
        fail, worst, _ = G.compare_potentials(gpu0, canon0, allp, tau=cfg.tau)
        assert not fail.any(), worst
        G.load_state(ctx, cfg, k1, n_pre, ring1, fr1)
        gpu1, info = G.gpu_potentials(ctx, npts)
        pinfo, clusters = rp.rp_predictive_info_read(ctx, npts)
        goff, gbp = rp.rp_predictive_lists_read(ctx, pinfo.clusters * cfg.kappa_max,
                                                pinfo.breakpoints)
    finally:
        rp.rp_destroy(ctx)
    assert pinfo.active == 1 and pinfo.kmeans_passes == passes and pinfo.partition == part
    np.testing.assert_array_equal(clusters, clusters1)
    # lines 3, 4 and 9-12 are host arithmetic on both sides: the merged lists agree exactly
    kap = o1.kappa()
    pat = np.zeros((npts, cfg.kappa_max), dtype=np.uint16)
    for p in range(npts):
        for j in range(kap):
            pat[p, j] = oracle.knn_pattern(leaves0, cfg.nx, cfg.ny, p, j, knn)
    if part == 0:
        ooff, obp = o1.merge_partitions(pat, clusters1, pinfo.clusters)
    else:
        ooff, obp = o1.merge_partitions_adaptive(pat, clusters1, pinfo.clusters, off0, plen0,
                                                 parts0)
    np.testing.assert_array_equal(goff, ooff)
    np.testing.assert_array_equal(gbp, obp)
    fail, worst, nties = G.compare_potentials(gpu1, pred1, pts, tau=cfg.tau)
    assert not fail.any(), (np.nonzero(fail)[0][:10], worst)
    assert info.segments == int(pred1["nseg"].sum()) or len(pts) < npts
    # forecast-dependent, but within the tolerance of the canonical result
    scale = np.abs(canon1["phi"]).max()
    assert np.abs(pred1["phi"] - canon1["phi"]).max() <= 2 * cfg.tau
    assert np.abs(gpu1["phi"][pts] - canon1["phi"]).max() <= 2 * cfg.tau
    assert (pred1["nseg"] != canon1["nseg"]).any()
    return pinfo, scale


@pytest.mark.parametrize("part", [0, 1])
def test_predictive_static_cfg1_full_mesh(part):
    """Config 1 (32x32, static frame, rigid history): two consecutive steps; uniform
    and adaptive partitioning."""
    cfg = W.config(1)
    ring, _ = _deposit_rigid_ring(cfg)
    fr = W.ring_frames(cfg, 0)
    fr1 = W.ring_frames(cfg, 1)
    _two_steps(cfg, [(0, ring, fr), (1, ring, fr1)], cfg.n_pre, knn=9, m=0, part=part)


@pytest.mark.parametrize("knn,m,rule,part", [(9, 0, 0, 0), (1, 12, 0, 0), (25, 40, 0, 0),
                                             (9, 0, 1, 0), (9, 0, 0, 1), (1, 12, 0, 1),
                                             (9, 0, 1, 1)])
def test_predictive_bend_small_full_mesh(knn, m, rule, part):
    """Moving frames (bend), node-sampled history with a time-varying amplitude; GK15 and the
    paper's own Simpson rule (R-22), which Algorithm 1's RP-QUADRULE names."""
    cfg = _bend_small(16, 24)
    cfg.rule = rule
    rings = []
    for k in (5, 6):
        ring = W.node_gaussian_ring(cfg, k=k, beta=(cfg.beta0, 0.01),
                                    amp_of_level=lambda l: 1.0 + 0.01 * l)
        rings.append((k, ring, W.ring_frames(cfg, k)))
    _two_steps(cfg, rings, cfg.n_pre, knn=knn, m=m, part=part)


def test_predictive_refuses_the_shard_path():
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    cfg = W.config(1)
    ctx = G.make_ctx(cfg)
    try:
        rp.rp_set_predictive(ctx, True)
        with pytest.raises(rp.RpError):
            rp.rp_set_predictive(ctx, True, knn=4)
        import torch
        ring, _ = _deposit_rigid_ring(cfg)
        G.load_state(ctx, cfg, 0, cfg.n_pre, ring, W.ring_frames(cfg, 0))
        sh = torch.zeros((rp.rp_shard_capacity(ctx, 2), 6), dtype=torch.float64, device="cuda")
        with pytest.raises(rp.RpError) as e:
            rp.rp_compute_potentials_shard(ctx, 0, 2, sh)
        assert e.value.code == -1
    finally:
        rp.rp_destroy(ctx)
