"""The u16 per-source SSSP (Phase II as the paper states it, Alg. 1 lines 4-7) at its
edges, bit-exact against the CPU oracle (Dijkstra per source): distances that do not fit 16 bits (the
route must fall back to int32), a heavy first arrival whose final distance does fit (it must not), arc
weights >= 0xFFFF, frontier lists that overflow their shared-memory capacity (the bitmap-scan rounds),
and D from the u16 kernel equal to the FW's D."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
from paper_conf_ipps_duttackb17_b200.graphgen import Graph

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_ipps_duttackb17_b200 as p
    p.lib()
    return p


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def full(pkg, g, flags):
    out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def exact(got, ref, what):
    bad = np.argwhere(got != ref)
    assert bad.size == 0, f"{what}: {len(bad)} mismatches, first {bad[:3].tolist()}"


def reduced_equal(pkg, g):
    p1 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    p2 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_SSSP)
    D1, D2 = pkg.alloc_D(p1), pkg.alloc_D(p2)
    pkg.apsp_reduced(p1, D1)
    pkg.apsp_reduced(p2, D2)
    torch.cuda.synchronize()
    assert torch.equal(D1, D2)


@pytest.mark.parametrize("scale", [1, 40, 400])
def test_heavy_weights(pkg, scale):
    """scale 400: most distances exceed 0xFFFF -- the u16 rows saturate and both routes fall back"""
    g0 = gg.torus(12, 12, 150, seed=3)
    g = Graph(g0.n, g0.src, g0.dst, (g0.w.astype(np.int64) * scale).astype(np.int32))
    ref = oracle.apsp(g.n, g.src, g.dst, g.w)
    if scale == 400:
        assert ref[ref < 2**31 - 1].max() >= 0xFFFF
    exact(full(pkg, g, pkg.FLAG_SSSP), ref, f"scale {scale}")
    reduced_equal(pkg, g)


def test_heavy_first_arrival(pkg):
    """Direct arcs of weight 70,000 from vertex 0 reach far vertices in round 1 (a candidate >= 0xFFFF for
    an unreached vertex) while every true distance is small: the row must be kept, and exact."""
    g0 = gg.grid(30, 30, 1500, seed=4)
    rng = np.random.default_rng(0)
    far = rng.choice(np.arange(1, g0.n), 12, replace=False)
    src = np.r_[g0.src, np.zeros(12, np.int32)]
    dst = np.r_[g0.dst, far.astype(np.int32)]
    w = np.r_[g0.w, np.full(12, 70000, np.int32)]
    g = Graph(g0.n, src.astype(np.int32), dst.astype(np.int32), w.astype(np.int32))
    ref = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert ref.max() < 0xFFFF
    exact(full(pkg, g, pkg.FLAG_SSSP), ref, "heavy first arrival")
    reduced_equal(pkg, g)


def test_bridge_heavier_than_u16(pkg):
    """two grids joined by one arc of weight 100,000: half of D is >= 0xFFFF"""
    a = gg.grid(10, 10, 200, seed=5)
    b = gg.grid(10, 10, 200, seed=6)
    src = np.r_[a.src, b.src + a.n, [3]]
    dst = np.r_[a.dst, b.dst + a.n, [a.n + 7]]
    w = np.r_[a.w, b.w, [100000]]
    g = Graph(a.n + b.n, src.astype(np.int32), dst.astype(np.int32), w.astype(np.int32))
    ref = oracle.apsp(g.n, g.src, g.dst, g.w)
    exact(full(pkg, g, pkg.FLAG_SSSP), ref, "bridge")
    reduced_equal(pkg, g)


def test_two_components(pkg):
    """unreachable vertices stay INF (0xFFFF in the u16 rows) without a saturation"""
    a = gg.grid(10, 10, 200, seed=7)
    b = gg.torus(6, 6, 90, seed=8)
    g = Graph(a.n + b.n, np.r_[a.src, b.src + a.n].astype(np.int32), np.r_[a.dst, b.dst + a.n].astype(np.int32),
              np.r_[a.w, b.w].astype(np.int32))
    exact(full(pkg, g, pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w), "two components")


@pytest.mark.parametrize("cap", [8, 64])
def test_list_overflow(pkg, monkeypatch, cap):
    """a list capacity far below the frontier: most rounds run the bitmap-scan branch"""
    monkeypatch.setenv("EAR_SSSP16_CAP", str(cap))
    for g in [gg.config("cfg1"), gg.corner_cases(11, n_target=400), gg.torus(12, 12, 150, seed=9)]:
        exact(full(pkg, g, pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w), f"cap {cap} n {g.n}")


def test_high_degree_falls_back(pkg):
    """a vertex of degree > 16 in G^r: the ELL rows do not apply, the int32 kernels run"""
    g0 = gg.grid(12, 12, 300, seed=10)
    hub_to = np.random.default_rng(1).choice(np.arange(1, g0.n), 24, replace=False)
    g = Graph(g0.n, np.r_[g0.src, np.zeros(24)].astype(np.int32), np.r_[g0.dst, hub_to].astype(np.int32),
              np.r_[g0.w, np.full(24, 50)].astype(np.int32))
    exact(full(pkg, g, pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w), "hub")


def test_cfg3_sampled_rows(pkg):
    """the largest single-row-block config the oracle checks row by row, through the u16 route"""
    g = gg.config("cfg3_f60")
    out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_SSSP)
    rows = np.unique(np.r_[[0, g.n - 1], np.random.default_rng(2).choice(g.n, 24, replace=False)])
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    exact(out[torch.as_tensor(rows).cuda().long()].cpu().numpy(), ref, "cfg3_f60 rows")
