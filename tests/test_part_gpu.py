"""Phase II by regions (EAR_FLAG_PART, csrc/part.cu, reading C24): G^r cut into
connected regions, distances inside each region, the boundary graph's FW, and the two min-plus products
through the region boundaries -- sec. 2.2's composition through articulation points with
boundary sets as separators.  Every test compares with the CPU oracle (Dijkstra per source on the
ORIGINAL graph, the definition of S at P:109) element by element, and checks that the route actually
ran (its product launches are counted) or, where it must not apply, that the fallback is exact."""
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


def exact(got, ref, what):
    bad = np.argwhere(got != ref)
    assert bad.size == 0, f"{what}: {len(bad)} mismatches, first {bad[:3].tolist()}"


def run(pkg, g, flags=None, rows=None):
    """apsp_full on the region route; returns (rows of S, whether the products ran)"""
    flags = pkg.FLAG_PART if flags is None else flags
    pkg.profile_reset()
    pkg.profile_enable(True)
    try:
        if rows is None:
            out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
        else:
            out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags, row_begin=rows[0],
                                row_end=rows[1])
        torch.cuda.synchronize()
        prof = pkg.profile_read()
    finally:
        pkg.profile_enable(False)
    return out, prof["part_mp_launches"] > 0


def part_info(pkg, g):
    p = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_PART)
    return p.part_info(), p.info()


@pytest.mark.parametrize("seed", range(12))
def test_corner_cases(pkg, seed):
    """self-loops, parallel edges, pendant paths, closed ears, pure cycles, isolated vertices, several
    components (cross-component pairs must come out INF although their u16 sums wrap)"""
    g = gg.corner_cases(seed, n_target=400 + 100 * seed)
    out, ran = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"corner case {seed}")
    assert ran


@pytest.mark.parametrize("seed", range(4))
def test_block_trees(pkg, seed):
    g = gg.block_tree(seed, n_target=1500, big=600)
    out, ran = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"block tree {seed}")
    assert ran


def test_cfg1_full(pkg):
    g = gg.config("cfg1")
    out, ran = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), "cfg1")
    assert ran


@pytest.mark.parametrize("labels", ["morton", "random"])
def test_cfg2_full(pkg, labels):
    """20k vertices, 7.9k reduced; random labels: the regions do not depend on the labelling (BFS)"""
    g = gg.config("cfg2", labels=labels)
    out, ran = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"cfg2 {labels}")
    assert ran


def test_partition_shape(pkg):
    """regions <= 256 vertices (one CTA's registers), boundary a small share of G^r on the paper's
    sparse graphs, and the product work (N_r + |B|) sum |R_i||B_i| far below the FW's N_r^3 / 2"""
    g = gg.config("cfg2")
    pi, info = part_info(pkg, g)
    nr = info.n_reduced
    assert 0 < pi["max_region"] <= 256
    assert pi["n_regions"] >= nr // 256
    assert pi["n_boundary"] < 0.5 * nr
    assert pi["max_boundary"] <= pi["max_region"]
    assert pi["multi_component"] == 0
    assert (nr + pi["n_boundary"]) * pi["sum_region_boundary"] < 0.05 * nr ** 3 / 2


def test_reduced_D_equals_fw(pkg):
    """apsp_reduced: the int32 D of G^r (padding isolated) equals the blocked FW's, bit for bit"""
    for g in (gg.config("cfg1"), gg.torus(30, 30, 700, seed=2), gg.corner_cases(3, n_target=900)):
        p1 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
        p2 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_PART)
        D1, D2 = pkg.alloc_D(p1), pkg.alloc_D(p2)
        pkg.apsp_reduced(p1, D1)
        pkg.apsp_reduced(p2, D2)
        torch.cuda.synchronize()
        assert torch.equal(D1, D2)


@pytest.mark.parametrize("scale", [1, 20, 40, 100, 400])
def test_heavy_weights_fallback(pkg, scale):
    """scale 20 / 40: boundary distances past the 64-tile FW's 0x7FFF cap (its int32 fallback) with the
    products still in range; scale 100: distances up to ~0xFFFF -- the u16 sum bound fails and another
    route runs; scale 400: distances beyond 0xFFFF.  Either way S is exact."""
    g0 = gg.torus(12, 12, 150, seed=3)
    g = Graph(g0.n, g0.src, g0.dst, (g0.w.astype(np.int64) * scale).astype(np.int32))
    out, ran = run(pkg, g, flags=pkg.FLAG_PART | pkg.FLAG_SSSP)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"scale {scale}")
    if scale == 1:
        assert ran


def test_heavy_arc_inside_region(pkg):
    """one arc of weight 40,000 (>= the region FW's 0x7FFF cap): the route must decline, S stays exact"""
    g0 = gg.grid(20, 20, 800, seed=7)
    w = g0.w.copy()
    w[5] = 40000
    g = Graph(g0.n, g0.src, g0.dst, w)
    out, _ = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), "heavy arc")


@pytest.mark.parametrize("n", [1, 2, 3, 7, 255, 256, 257, 600])
def test_small_paths_and_cycles(pkg, n):
    for g in (gg.path(n, seed=n), gg.cycle(max(n, 3), seed=n)):
        out, _ = run(pkg, g)
        exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"n={g.n}")


def test_no_contract_grid(pkg):
    """every vertex a terminal (FLAG_NO_CONTRACT): regions on the uncontracted grid"""
    g = gg.grid(40, 40, 1600, seed=9)
    out, ran = run(pkg, g, flags=pkg.FLAG_PART | pkg.FLAG_NO_CONTRACT)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), "grid")
    assert ran


@pytest.mark.parametrize("labels", ["morton", "random"])
def test_cfg4_sampled_rows(pkg, labels):
    """cfg4 at full size (100k vertices, ~30k reduced, 40 GB output) in the bench's launch
    configuration; 40 sampled rows against the oracle, and the columns of those rows (symmetry)"""
    g = gg.config("cfg4", labels=labels)
    out, ran = run(pkg, g)
    assert ran
    rng = np.random.default_rng(11)
    rows = np.unique(np.concatenate([[0, g.n - 1], rng.choice(g.n, 38, replace=False)]))
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    idx = torch.as_tensor(rows).cuda().long()
    exact(out[idx].cpu().numpy(), ref, f"cfg4 {labels} rows")
    exact(out[:, idx].t().cpu().numpy(), ref, f"cfg4 {labels} columns")
    del out
    torch.cuda.empty_cache()


def test_row_range(pkg):
    g = gg.config("cfg2")
    out, ran = run(pkg, g, rows=(1234, 5678))
    assert ran
    exact(out.cpu().numpy(), oracle.apsp_rows(g.n, g.src, g.dst, g.w, np.arange(1234, 5678)), "rows")


@pytest.mark.parametrize("n,deg", [(1500, 3), (3000, 4)])
def test_expander_big_boundaries(pkg, n, deg):
    """a random sparse graph (an expander: most region vertices are boundary vertices, |B_i| > 32, so the
    general product kernel runs beside the persistent one)"""
    rng = np.random.default_rng(n)
    m = n * deg // 2
    src = rng.integers(0, n, m).astype(np.int32)
    dst = rng.integers(0, n, m).astype(np.int32)
    ring = np.arange(n, dtype=np.int32)   # connected
    g = Graph(n, np.r_[src, ring], np.r_[dst, (ring + 1) % n].astype(np.int32),
              rng.integers(1, 101, m + n).astype(np.int32))
    pi, _ = part_info(pkg, g)
    assert pi["max_boundary"] > 32
    out, ran = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"expander n={n}")
    assert ran


def _g(n, edges, w=None):
    s, d = (np.array(c, np.int32) for c in zip(*edges))
    w = np.ones(len(s), np.int32) if w is None else np.asarray(w, np.int32)
    return Graph(n, s, d, w)


@pytest.mark.parametrize("case", ["star", "complete", "two_complete", "long_path", "unit_grid", "ladder"])
def test_adversarial_shapes(pkg, case):
    """shapes the Voronoi regions handle badly or trivially: a star (every leaf one hop from the hub: the
    cell splitting runs down to one-vertex regions), complete graphs (every vertex a boundary vertex),
    a 5,000-vertex path, a grid of unit weights (all ties), a ladder (two long parallel paths)"""
    rng = np.random.default_rng(7)
    if case == "star":
        g = _g(701, [(0, i) for i in range(1, 701)], rng.integers(1, 50, 700))
    elif case == "complete":
        e = [(i, j) for i in range(300) for j in range(i + 1, 300)]
        g = _g(300, e, rng.integers(1, 100, len(e)))
    elif case == "two_complete":
        e = [(i, j) for i in range(120) for j in range(i + 1, 120)]
        e += [(120 + i, 120 + j) for i, j in e]
        g = _g(240, e, rng.integers(1, 100, len(e)))
    elif case == "long_path":
        g = gg.path(5000, seed=3)
    elif case == "unit_grid":
        e = [(r * 40 + c, r * 40 + c + 1) for r in range(40) for c in range(39)]
        e += [(r * 40 + c, (r + 1) * 40 + c) for r in range(39) for c in range(40)]
        g = _g(1600, e)
    else:
        e = [(i, i + 1) for i in range(999)] + [(1000 + i, 1001 + i) for i in range(999)]
        e += [(i, 1000 + i) for i in range(0, 1000, 7)]
        g = _g(2000, e, rng.integers(1, 100, len(e)))
    out, _ = run(pkg, g)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), case)


@pytest.mark.parametrize("rng_rows", [(0, 1), (17, 18), (300, 700), (1499, 1500)])
def test_row_ranges_need_only_their_regions(pkg, rng_rows):
    """a strict row range computes only the regions Phase III stages for it (the chain ends of its rows):
    several components, pendant paths and closed ears around the range edges"""
    g = gg.corner_cases(5, n_target=1500)
    a, b = rng_rows
    b = min(b, g.n)
    a = min(a, b - 1)
    out, ran = run(pkg, g, rows=(a, b))
    exact(out.cpu().numpy(), oracle.apsp_rows(g.n, g.src, g.dst, g.w, np.arange(a, b)), f"rows {a}:{b}")
    assert ran


@pytest.mark.parametrize("variant", ["0", "1", "2"])
@pytest.mark.parametrize("case", ["cfg2", "corner", "cfg2_random"])
def test_expansion_variants(pkg, case, variant, monkeypatch):
    """the pair-major expansion's three variants, forced by EAR_XP_GP: 0 the partners' rows staged beside the
    item's (chosen by default when the labels lack locality and D16 exceeds L2), 1 only the item's row
    staged and the partners' gathered from global memory by lane-consecutive columns with two 512-thread
    CTAs per SM (the default for cfg1-cfg4), 2 the same with one 1024-thread CTA (cfg5's 120 KB rows)"""
    monkeypatch.setenv("EAR_XP_GP", variant)
    g = {"cfg2": lambda: gg.config("cfg2"), "corner": lambda: gg.corner_cases(17, n_target=1800),
         "cfg2_random": lambda: gg.config("cfg2", labels="random")}[case]()
    for flags in (pkg.FLAG_PART, pkg.FLAG_BCC):
        out, _ = run(pkg, g, flags=flags)
        exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"{case} flags={flags}")


@pytest.mark.parametrize("split", ["0", "1"])
@pytest.mark.parametrize("case", ["cfg2", "corner", "heavy20"])
def test_boundary_fw_schedules(pkg, case, split, monkeypatch):
    """the dense boundary FW (64-tile, one cooperative launch) under both schedules, forced by
    EAR_FW64_SPLIT: 1 the split barriers (block 0 runs the next pivot while the others finish the round;
    the default), 0 two grid barriers per round; heavy20: distances past the u16 cap (the int32 twin)"""
    monkeypatch.setenv("EAR_FW64_SPLIT", split)
    if case == "heavy20":
        g0 = gg.torus(12, 12, 150, seed=3)
        g = Graph(g0.n, g0.src, g0.dst, (g0.w.astype(np.int64) * 20).astype(np.int32))
    else:
        g = {"cfg2": lambda: gg.config("cfg2"), "corner": lambda: gg.corner_cases(5, n_target=1800)}[case]()
    out, ran = run(pkg, g, flags=pkg.FLAG_PART | pkg.FLAG_SSSP)
    exact(out.cpu().numpy(), oracle.apsp(g.n, g.src, g.dst, g.w), f"{case} split={split}")
