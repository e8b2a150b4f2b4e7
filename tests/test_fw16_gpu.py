"""GPU: the packed 16-bit FW path against the oracle and against the int32 FW.

The 16-bit FW computes min(d, 0x7FFF) exactly; its result is kept only when no pair of the same
component reached the cap, otherwise the int32 FW re-runs.  These tests pin both branches: graphs
whose reduced distances stay below the cap (16-bit result kept, bit-exact), graphs that exceed it
(fallback taken, still bit-exact), the boundary on both sides, disconnected graphs (the cap stands for
EAR_INF across components), and equality with EAR_FLAG_FW32 (int32 throughout) on the configs.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu
CAP = 0x7FFF


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_ipps_duttackb17_b200 as p
    p.lib()
    return p


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def ladder(L, rail_w, rung_w=1, seed=None):
    """2 x L ladder: rails (i, i+1), (L+i, L+i+1) of weight rail_w, rungs (i, L+i) of weight rung_w.
    Every vertex but the 4 corners has degree 3, so almost all of it survives Reduce(G)."""
    i = np.arange(L - 1)
    src = np.concatenate([i, L + i, np.arange(L)])
    dst = np.concatenate([i + 1, L + i + 1, L + np.arange(L)])
    w = np.concatenate([np.full(2 * (L - 1), rail_w), np.full(L, rung_w)])
    if seed is not None:   # jitter the rails a little
        w[: 2 * (L - 1)] += np.random.default_rng(seed).integers(0, 3, 2 * (L - 1))
    return gg.Graph(2 * L, src.astype(np.int32), dst.astype(np.int32), w.astype(np.int32))


def reduced(pkg, g, flags=0):
    """D from apsp_reduced with profiling on: (D on V^r, profile)."""
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
    D = pkg.alloc_D(plan)
    pkg.profile_reset()
    pkg.profile_enable(True)
    pkg.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    prof = pkg.profile_read()
    pkg.profile_enable(False)
    nr = plan.info().n_reduced
    out = D[:nr, :nr].cpu().numpy()
    plan.destroy()
    return out, prof


def oracle_on_terminals(g):
    r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    T = np.nonzero(r.term)[0]
    return oracle.apsp_rows(g.n, g.src, g.dst, g.w, T)[:, T]


def assert_exact(got, ref, what):
    bad = np.argwhere(got != ref)
    assert bad.size == 0, f"{what}: {len(bad)} mismatches, first {bad[:5].tolist()}"


def test_short_distances_keep_the_16bit_result(pkg):
    g = ladder(400, 20, seed=1)                 # max distance ~ 400 * 21 << cap
    ref = oracle_on_terminals(g)
    assert ref[ref < oracle.INF].max() < CAP
    got, prof = reduced(pkg, g)
    assert prof["fw16_used"] == 1 and prof["fw16_fallbacks"] == 0
    assert prof["fw_phase3_16_minplus"] > 0
    assert_exact(got, ref, "ladder, 16-bit kept")


def test_long_distances_fall_back_to_int32(pkg):
    g = ladder(700, 100, seed=2)                # max distance ~ 70,000 > cap
    ref = oracle_on_terminals(g)
    assert ref[ref < oracle.INF].max() > CAP
    got, prof = reduced(pkg, g)
    assert prof["fw16_used"] == 0 and prof["fw16_fallbacks"] == 1
    assert_exact(got, ref, "ladder, int32 fallback")


@pytest.mark.parametrize("delta", [-1, 0])
def test_cap_boundary(pkg, delta):
    """Largest reduced distance exactly CAP - 1 (16-bit kept) or exactly CAP (fallback).  In a 2 x L
    ladder with rails a and rungs b (b < 2a + b via the corner chains), the farthest terminals are the
    top of column 1 and the bottom of column L-2: (L - 3) a + b."""
    L, a = 300, 100
    target = CAP - 1 if delta == -1 else CAP
    g = ladder(L, a, rung_w=target - (L - 3) * a)
    ref = oracle_on_terminals(g)
    assert ref[ref < oracle.INF].max() == target
    got, prof = reduced(pkg, g)
    assert prof["fw16_used"] == (1 if delta == -1 else 0)
    assert prof["fw16_fallbacks"] == (0 if delta == -1 else 1)
    assert_exact(got, ref, f"boundary {target}")


def test_disconnected_components_cap_means_unreachable(pkg):
    a, b = ladder(200, 30, seed=3), ladder(150, 40, seed=4)
    g = gg.Graph(a.n + b.n, np.concatenate([a.src, b.src + a.n]).astype(np.int32),
                 np.concatenate([a.dst, b.dst + a.n]).astype(np.int32), np.concatenate([a.w, b.w]).astype(np.int32))
    ref = oracle_on_terminals(g)
    assert (ref == oracle.INF).any()
    got, prof = reduced(pkg, g)
    assert prof["fw16_used"] == 1
    assert_exact(got, ref, "two components")


def test_one_component_long_other_short(pkg):
    """A long component forces the fallback even though the short one alone would fit."""
    a, b = ladder(700, 100, seed=5), ladder(150, 10, seed=6)
    g = gg.Graph(a.n + b.n, np.concatenate([a.src, b.src + a.n]).astype(np.int32),
                 np.concatenate([a.dst, b.dst + a.n]).astype(np.int32), np.concatenate([a.w, b.w]).astype(np.int32))
    got, prof = reduced(pkg, g)
    assert prof["fw16_fallbacks"] == 1
    assert_exact(got, oracle_on_terminals(g), "long + short components")


@pytest.mark.parametrize("name", ["cfg1", "cfg2"])
def test_default_equals_fw32(pkg, name):
    g = gg.config(name)
    d16, p16 = reduced(pkg, g)
    d32, p32 = reduced(pkg, g, flags=pkg.FLAG_FW32)
    assert p16["fw16_used"] == 1 and p32["fw16_used"] == 0 and p32["fw16_fallbacks"] == 0
    assert np.array_equal(d16, d32)


@pytest.mark.parametrize("seed", range(4))
def test_bcc_pieces_16bit(pkg, seed):
    """The big biconnected pieces run the 16-bit FW too (a piece is connected)."""
    g = gg.corner_cases(3000 + seed, n_target=1500 + 200 * seed)
    ref = oracle_on_terminals(g)
    got, prof = reduced(pkg, g, flags=pkg.FLAG_BCC)
    assert_exact(got, ref, f"bcc corner seed {seed}")


# ------------------------------------------------------------- the 16-bit row-block sharded schedule
def emulated(pkg, g, P, flags=0):
    """D on V^r from the P-rank sharded schedule emulated on this GPU, with its profile."""
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
    pkg.profile_reset()
    pkg.profile_enable(True)
    D = pkg.apsp_reduced_emulated(plan, P)
    torch.cuda.synchronize()
    prof = pkg.profile_read()
    pkg.profile_enable(False)
    nr = plan.info().n_reduced
    out = D[:nr, :nr].cpu().numpy()
    plan.destroy()
    return out, prof


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_sharded16_kept(pkg, P):
    """Every virtual rank runs the packed kernel on its owned rows (MODE_LIST) and the result is kept."""
    g = gg.config("cfg1")
    got, prof = emulated(pkg, g, P)
    assert prof["fw16_used"] == 1 and prof["fw16_fallbacks"] == 0 and prof["fw_phase3_16_minplus"] > 0
    assert_exact(got, oracle_on_terminals(g), f"sharded16 P={P}")


@pytest.mark.parametrize("P", [2, 5])
def test_sharded16_fallback(pkg, P):
    g = ladder(700, 100, seed=7)
    got, prof = emulated(pkg, g, P)
    assert prof["fw16_used"] == 0 and prof["fw16_fallbacks"] == 1
    assert_exact(got, oracle_on_terminals(g), f"sharded16 fallback P={P}")


@pytest.mark.parametrize("delta", [-1, 0])
def test_sharded16_cap_boundary(pkg, delta):
    L, a = 300, 100
    target = CAP - 1 if delta == -1 else CAP
    g = ladder(L, a, rung_w=target - (L - 3) * a)
    got, prof = emulated(pkg, g, 3)
    assert prof["fw16_used"] == (1 if delta == -1 else 0)
    assert_exact(got, oracle_on_terminals(g), f"sharded16 boundary {target}")


def test_sharded16_disconnected(pkg):
    a, b = ladder(200, 30, seed=8), ladder(150, 40, seed=9)
    g = gg.Graph(a.n + b.n, np.concatenate([a.src, b.src + a.n]).astype(np.int32),
                 np.concatenate([a.dst, b.dst + a.n]).astype(np.int32), np.concatenate([a.w, b.w]).astype(np.int32))
    got, prof = emulated(pkg, g, 4)
    assert prof["fw16_used"] == 1
    assert_exact(got, oracle_on_terminals(g), "sharded16 two components")


@pytest.mark.parametrize("seed", range(3))
def test_sharded16_corner_equals_fw32(pkg, seed):
    g = gg.corner_cases(4100 + seed, n_target=900 + 300 * seed)
    d16, p16 = emulated(pkg, g, 3)
    d32, p32 = emulated(pkg, g, 3, flags=pkg.FLAG_FW32)
    assert p32["fw16_used"] == 0 and p32["fw16_fallbacks"] == 0
    assert np.array_equal(d16, d32)
    assert_exact(d16, oracle_on_terminals(g), f"sharded16 corner seed {seed}")


@pytest.mark.parametrize("P", [1, 3, 8])
def test_sharded16_without_lookahead(pkg, P, monkeypatch):
    """The sharded packed schedule with its lookahead off (serial pivot chains) gives the same D."""
    g = gg.corner_cases(4200 + P, n_target=1400)
    d_la, _ = emulated(pkg, g, P)
    monkeypatch.setenv("EAR_FW16_LOOKAHEAD", "0")
    d_serial, prof = emulated(pkg, g, P)
    assert prof["fw16_used"] == 1
    assert np.array_equal(d_la, d_serial)
    assert_exact(d_serial, oracle_on_terminals(g), f"sharded16 serial P={P}")


def test_cap_precheck_abandons_hopeless_fw16(pkg):
    """A reduced graph large enough for the cap precheck (>= 64 tiles) whose corner vertex is already
    farther than the cap from something: the packed FW is abandoned after round 3 and the int32 FW
    gives the exact result (sampled rows against the oracle)."""
    g = ladder(4200, 100, seed=11)              # 8,400 vertices in a 2 x 4,200 ladder, distances ~420k
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    D = pkg.alloc_D(plan)
    pkg.profile_reset()
    pkg.profile_enable(True)
    pkg.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    prof = pkg.profile_read()
    pkg.profile_enable(False)
    assert plan.info().n_reduced_padded // 128 >= 64
    assert prof["fw16_prechecked"] == 1 and prof["fw16_fallbacks"] == 1 and prof["fw16_used"] == 0
    r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    T = np.nonzero(r.term)[0]
    rows = np.random.default_rng(2).choice(len(T), 12, replace=False)
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, T[rows])[:, T]
    assert_exact(D[torch.as_tensor(rows).cuda().long()][:, :len(T)].cpu().numpy(), ref, "precheck fallback")


def test_cap_precheck_keeps_short_fw16(pkg):
    """cfg2 (20k vertices, 7,917 reduced: 62 tiles -> no precheck) and a large short-distance ladder
    (precheck passes): the packed result is kept."""
    g = ladder(4200, 3, seed=12)                # distances ~12.6k < cap
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    D = pkg.alloc_D(plan)
    pkg.profile_reset()
    pkg.profile_enable(True)
    pkg.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    prof = pkg.profile_read()
    pkg.profile_enable(False)
    assert prof["fw16_prechecked"] == 0 and prof["fw16_used"] == 1


def test_cap_precheck_sharded(pkg):
    """The sharded packed schedule takes the same precheck (every rank decides alike): abandoned after
    round 3 for the long ladder, the int32 schedule's result exact (sampled rows)."""
    g = ladder(4200, 100, seed=13)
    d, prof = emulated(pkg, g, 3)
    assert prof["fw16_prechecked"] == 1 and prof["fw16_used"] == 0
    r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    T = np.nonzero(r.term)[0]
    rows = np.random.default_rng(3).choice(len(T), 10, replace=False)
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, T[rows])[:, T]
    assert_exact(d[rows], ref, "sharded precheck fallback")
