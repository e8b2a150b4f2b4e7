"""GPU parity of Phase II by biconnected pieces (EAR_FLAG_BCC; paper sec. 2.2; SURVEY 8.f
NEXT 3) against the CPU oracle, bit-exact, and of the block structure it finds against a plain
sequential Tarjan block count on the oracle's reduced graph (test code, not the oracle).

Graphs: the chain corner cases, block trees (cycles / grids / wheels / thetas glued at articulation
points, bridges, pendant trees, several components, isolated vertices -- the shape of P:121), a block
tree with a dominant multi-tile block, cfg1 / cfg2 / cfg4 (sampled rows at full size).
"""
import sys

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_ipps_duttackb17_b200 as p
    p.lib()
    return p


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def run_full(pkg, g, flags):
    out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
    torch.cuda.synchronize()
    return out.cpu().numpy()


def assert_exact(got, ref, what):
    bad = np.argwhere(got != ref)
    assert bad.size == 0, f"{what}: {len(bad)} mismatches, first {bad[:5].tolist()}"


def tarjan_blocks(nv, edges):
    """(components, blocks with >= 1 edge, articulation points) of a simple undirected graph,
    iterative Hopcroft-Tarjan DFS."""
    adj = [[] for _ in range(nv)]
    for a, b in edges:
        adj[a].append(b)
        adj[b].append(a)
    disc = [-1] * nv
    low = [0] * nv
    t = 0
    comps = blocks = 0
    art = [False] * nv
    for r in range(nv):
        if disc[r] >= 0:
            continue
        comps += 1
        disc[r] = low[r] = t
        t += 1
        root_children = 0
        stack = [(r, -1, iter(adj[r]))]
        while stack:
            v, p, it = stack[-1]
            nxt = next(it, None)
            if nxt is None:
                stack.pop()
                if p >= 0:
                    low[p] = min(low[p], low[v])
                    if low[v] >= disc[p]:
                        blocks += 1             # (p, v) closes a block
                        if stack[-1][1] >= 0:
                            art[p] = True
                        else:
                            root_children += 1
                continue
            if nxt == p:
                continue
            if disc[nxt] >= 0:
                low[v] = min(low[v], disc[nxt])
            else:
                disc[nxt] = low[nxt] = t
                t += 1
                stack.append((nxt, v, iter(adj[nxt])))
        if root_children >= 2:
            art[r] = True
    return comps, blocks, sum(art)


def reduced_simple_graph(g):
    red = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    terms = np.flatnonzero(red.term)
    idx = -np.ones(g.n, dtype=np.int64)
    idx[terms] = np.arange(len(terms))
    e = {(min(a, b), max(a, b)) for a, b in zip(idx[red.re_u].tolist(), idx[red.re_v].tolist()) if a != b}
    return len(terms), sorted(e)


# ------------------------------------------------------------------------------ parity
@pytest.mark.parametrize("seed", range(30))
def test_bcc_corner_cases(pkg, seed):
    g = gg.corner_cases(5000 + seed, n_target=20 + 11 * seed)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC), oracle.apsp(g.n, g.src, g.dst, g.w), f"bcc corner {seed}")


@pytest.mark.parametrize("seed", range(24))
def test_bcc_block_trees(pkg, seed):
    g = gg.block_tree(seed, n_target=40 + 60 * seed)
    ref = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC), ref, f"block tree {seed}")
    # blocks of the uncontracted graph too (every vertex a terminal)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC | pkg.FLAG_NO_CONTRACT), ref, f"block tree {seed} no-contract")


@pytest.mark.parametrize("seed", range(3))
def test_bcc_dominant_multi_tile_block(pkg, seed):
    """A root piece of several 128-tiles (blocked TMA FW) with small pieces hanging off it."""
    g = gg.block_tree(100 + seed, n_target=6000, big=900 + 400 * seed)
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
    info = plan.bcc_info()
    assert info["largest_piece"] > 128
    assert info["n_pieces"] > 10
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC), oracle.apsp(g.n, g.src, g.dst, g.w), f"dominant {seed}")


def decorated_grid(side, frac, seed):
    """A side x side grid block whose edges are, with probability frac, subdivided by a vertex x that
    also carries a pendant triangle: x has degree 3 in G (a terminal of G^r) but degree 2 inside the
    grid block, so the block reduces again (some edges get a second subdivision of plain degree-two
    vertices, some pendants get a pendant path).  Random weights 1-100, random relabelling."""
    rng = np.random.default_rng(seed)
    us, vs = [], []
    n = side * side
    for y in range(side):
        for x in range(side):
            i = y * side + x
            for j in ([i + 1] if x + 1 < side else []) + ([i + side] if y + 1 < side else []):
                if rng.random() < frac:
                    xv, a, b = n, n + 1, n + 2
                    n += 3
                    us += [i, xv, xv, a, b]
                    vs += [xv, j, a, b, xv]
                    if rng.random() < 0.3:   # a plain chain vertex on the other half-edge too
                        us[-4] = n
                        us.append(n); vs.append(xv)
                        n += 1
                else:
                    us.append(i); vs.append(j)
    perm = rng.permutation(n)
    src = perm[np.array(us)].astype(np.int32)
    dst = perm[np.array(vs)].astype(np.int32)
    w = rng.integers(1, 101, len(src)).astype(np.int32)
    return gg.Graph(n, src, dst, w)


@pytest.mark.parametrize("seed", range(3))
def test_bcc_rereduce_big_pieces(pkg, seed, monkeypatch):
    """P:123's order -- G split into blocks, then EACH block reduced: a subdividing vertex with a
    hanging triangle is a terminal of G^r but has degree two inside its block, so the big piece is
    reduced again (possibly twice) and expanded back.  The composed D equals the FW on the whole piece
    (EAR_NO_REREDUCE) bit for bit, and the full S equals the oracle."""
    g = decorated_grid(24 + 4 * seed, 0.3 + 0.1 * seed, seed)
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
    D = pkg.alloc_D(plan)
    pkg.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    info = plan.bcc_info()
    assert info["rereduced_pieces"] >= 1 and 0 < info["largest_reduced"] < info["largest_piece"] - 128, info
    assert info["rereduce_levels"] >= 1
    with monkeypatch.context() as m:
        m.setenv("EAR_NO_REREDUCE", "1")
        p2 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
        D2 = pkg.alloc_D(p2)
        pkg.apsp_reduced(p2, D2)
        torch.cuda.synchronize()
        assert p2.bcc_info()["rereduced_pieces"] == 0
    assert torch.equal(D, D2)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC), oracle.apsp(g.n, g.src, g.dst, g.w), f"rereduce {seed}")


@pytest.mark.parametrize("name", ["cfg1", "cfg2", "block"])
def test_bcc_D_equals_fw_D(pkg, name):
    """Composed S^r (pieces + P:131 join) equals the blocked-FW S^r bit for bit, padding included."""
    g = gg.block_tree(7, n_target=8000, big=1500) if name == "block" else gg.config(name)
    p1 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    p2 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
    D1, D2 = pkg.alloc_D(p1), pkg.alloc_D(p2)
    pkg.apsp_reduced(p1, D1)
    pkg.apsp_reduced(p2, D2)
    torch.cuda.synchronize()
    assert torch.equal(D1, D2)


def test_bcc_cfg4_sampled_rows(pkg):
    g = gg.config("cfg4")
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
    info = plan.bcc_info()
    nr = plan.info().n_reduced
    assert info["largest_piece"] < nr and info["sum_cubes"] < 0.7 * float(nr) ** 3
    print("cfg4 bcc", info, file=sys.stderr)
    D = pkg.alloc_D(plan)
    pkg.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    info = plan.bcc_info()
    print("cfg4 bcc after solve", info, file=sys.stderr)
    assert info["rereduced_pieces"] >= 1 and info["largest_reduced"] < info["largest_piece"]
    rows = np.unique(np.concatenate([[0, g.n - 1], np.random.default_rng(9).choice(g.n, 24, replace=False)]))
    out = torch.empty((len(rows), g.n), dtype=torch.int32, device="cuda")
    for i, r in enumerate(rows):
        pkg.expand_ears(plan, D, int(r), int(r) + 1, out=out[i:i + 1])
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    assert_exact(out.cpu().numpy(), ref, "cfg4 bcc rows")


def _graph(n, edges):
    from paper_conf_ipps_duttackb17_b200.graphgen import Graph
    if edges:
        s, d, w = (np.array(c, np.int32) for c in zip(*edges))
    else:
        s = d = w = np.zeros(0, np.int32)
    return Graph(n, s, d, w)


@pytest.mark.parametrize("case", ["n1", "m0", "cycle", "path", "star", "two_triangles", "bowtie_chain", "k4"])
def test_bcc_degenerate(pkg, case):
    g = {"n1": _graph(1, []), "m0": _graph(6, []), "cycle": gg.cycle(11, seed=5), "path": gg.path(30, seed=6),
         "star": _graph(50, [(0, i, i) for i in range(1, 50)]),
         "two_triangles": _graph(7, [(0, 1, 1), (1, 2, 2), (2, 0, 3), (4, 5, 1), (5, 6, 1), (6, 4, 5)]),
         "bowtie_chain": _graph(9, [(0, 1, 2), (1, 2, 2), (2, 0, 2), (2, 3, 7), (3, 4, 1), (4, 2, 1),
                                    (4, 5, 3), (5, 6, 3), (6, 7, 3), (7, 4, 3), (7, 8, 9)]),
         "k4": _graph(4, [(a, b, a + b + 1) for a in range(4) for b in range(a + 1, 4)])}[case]
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC), oracle.apsp(g.n, g.src, g.dst, g.w), case)


# ------------------------------------------------------------------------------ blocks solved by SSSP
# EAR_FLAG_BCC | EAR_FLAG_SSSP: the block structure of sec. 2.2 with every big piece reduced
# again and its reduced graph solved by the paper's per-source SSSP instead of the FW.
@pytest.mark.parametrize("seed", range(10))
def test_bcc_sssp_block_trees(pkg, seed):
    g = gg.block_tree(40 + seed, n_target=300 + 500 * seed, big=200 * (seed % 4))
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC | pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w),
                 f"bcc+sssp block tree {seed}")


@pytest.mark.parametrize("seed", range(8))
def test_bcc_sssp_corner_cases(pkg, seed):
    g = gg.corner_cases(7000 + seed, n_target=30 + 25 * seed)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC | pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w),
                 f"bcc+sssp corner {seed}")


@pytest.mark.parametrize("seed", range(2))
def test_bcc_sssp_rereduced_pieces(pkg, seed):
    g = decorated_grid(24 + 4 * seed, 0.3 + 0.1 * seed, seed)
    assert_exact(run_full(pkg, g, pkg.FLAG_BCC | pkg.FLAG_SSSP), oracle.apsp(g.n, g.src, g.dst, g.w),
                 f"bcc+sssp rereduce {seed}")


@pytest.mark.parametrize("name", ["cfg2", "block"])
def test_bcc_sssp_D_equals_fw_D(pkg, name):
    g = gg.block_tree(7, n_target=8000, big=1500) if name == "block" else gg.config(name)
    p1 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    p2 = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC | pkg.FLAG_SSSP)
    D1, D2 = pkg.alloc_D(p1), pkg.alloc_D(p2)
    pkg.apsp_reduced(p1, D1)
    pkg.apsp_reduced(p2, D2)
    torch.cuda.synchronize()
    assert torch.equal(D1, D2)


def test_bcc_sssp_cfg4_sampled_rows(pkg):
    """the bench's route at its size: full N x N through apsp_full (u16 compose), sampled rows"""
    g = gg.config("cfg4")
    out = pkg.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC | pkg.FLAG_SSSP)
    rows = np.unique(np.concatenate([[0, g.n - 1], np.random.default_rng(10).choice(g.n, 24, replace=False)]))
    ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    assert_exact(out[torch.as_tensor(rows).cuda().long()].cpu().numpy(), ref, "cfg4 bcc+sssp rows")
    del out
    torch.cuda.empty_cache()


# ------------------------------------------------------------------------------ structure
@pytest.mark.parametrize("seed", range(12))
def test_bcc_structure_matches_tarjan(pkg, seed):
    g = gg.block_tree(200 + seed, n_target=100 + 150 * seed) if seed % 3 else gg.corner_cases(300 + seed, 80 + 30 * seed)
    nv, edges = reduced_simple_graph(g)
    comps, blocks, arts = tarjan_blocks(nv, edges)
    plan = pkg.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=pkg.FLAG_BCC)
    assert plan.info().n_reduced == nv
    info = plan.bcc_info()
    assert (info["n_components"], info["n_blocks"], info["n_articulation"]) == (comps, blocks, arts)
