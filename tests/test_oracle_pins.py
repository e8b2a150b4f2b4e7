"""Pins for the CPU oracle.  CPU only (``-m "not gpu"``).

The oracle (oracle/apsp_oracle.c) is a Dijkstra-per-source; every check here comes from something
other than itself: brute-force Floyd-Warshall [9] on tiny inputs, exhaustive enumeration of all small
labelled graphs, closed forms, union-find, the Bellman certificate, scipy's Dijkstra, and the
paper's own identities (P:109 distance preservation, P:111/P:115 expansion formulas, Lemma 3.1's
edge count P:289-293, Fig. 4's chains P:312).
"""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
from tests import pins

INF = oracle.INF


# ------------------------------------------------------------------------------ P1 brute force
@pytest.mark.parametrize("seed", range(40))
def test_oracle_matches_bruteforce_fw_corner_cases(seed):
    g = gg.corner_cases(seed, n_target=int(10 + seed * 1.5))
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert np.array_equal(S, pins.brute_fw(g.n, g.src, g.dst, g.w))


def _stack_graphs(graph_list, n):
    """Disjoint union of many n-vertex graphs: returns (N, src, dst, w)."""
    src, dst, w = [], [], []
    for i, edges in enumerate(graph_list):
        for (a, b, x) in edges:
            src.append(i * n + a); dst.append(i * n + b); w.append(x)
    return len(graph_list) * n, np.array(src, np.int32), np.array(dst, np.int32), np.array(w, np.int32)


def _exhaustive(n, weights, chunk=1500):
    pairs = list(itertools.combinations(range(n), 2))
    choices = [0] + list(weights)             # 0 = edge absent
    all_graphs = []
    for assign in itertools.product(choices, repeat=len(pairs)):
        all_graphs.append([(a, b, x) for (a, b), x in zip(pairs, assign) if x])
    big = np.iinfo(np.int64).max // 8
    for c0 in range(0, len(all_graphs), chunk):
        part = all_graphs[c0:c0 + chunk]
        N, src, dst, w = _stack_graphs(part, n)
        # oracle on the disjoint union, rows of every vertex
        S = oracle.apsp(N, src, dst, w)
        # brute force per graph, batched
        D = np.full((len(part), n, n), big, dtype=np.int64)
        D[:, np.arange(n), np.arange(n)] = 0
        for gi, edges in enumerate(part):
            for (a, b, x) in edges:
                D[gi, a, b] = min(D[gi, a, b], x)
                D[gi, b, a] = min(D[gi, b, a], x)
        D = pins.batched_fw(D)
        D[D >= big] = INF
        for gi in range(len(part)):
            blk = S[gi * n:(gi + 1) * n, gi * n:(gi + 1) * n]
            assert np.array_equal(blk, D[gi]), (n, part[gi])
            # nothing leaks across the disjoint union
            assert np.all(S[gi * n:(gi + 1) * n, :gi * n] == INF)
    return len(all_graphs)


def test_oracle_exhaustive_weighted_n4():
    # every graph on 4 labelled vertices, each edge absent or weight 1, 2 or 3: 4^6 = 4096 graphs
    assert _exhaustive(4, (1, 2, 3)) == 4 ** 6


def test_oracle_exhaustive_weighted_n5():
    # every graph on 5 labelled vertices, each edge absent or weight 1 or 2: 3^10 = 59049 graphs
    assert _exhaustive(5, (1, 2), chunk=4000) == 3 ** 10


def test_oracle_exhaustive_unweighted_n6():
    # every unweighted graph on 6 labelled vertices: 2^15 = 32768 graphs
    assert _exhaustive(6, (1,), chunk=3000) == 2 ** 15


# ------------------------------------------------------------------------------ P2 closed forms
@pytest.mark.parametrize("n", [1, 2, 3, 17, 200])
def test_oracle_path_closed_form(n):
    g = gg.path(n, seed=n)
    pre = np.concatenate([[0], np.cumsum(g.w.astype(np.int64))])
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert np.array_equal(S, np.abs(pre[:, None] - pre[None, :]))


@pytest.mark.parametrize("n", [3, 4, 9, 150])
def test_oracle_cycle_closed_form(n):
    g = gg.cycle(n, seed=n)
    pre = np.concatenate([[0], np.cumsum(g.w.astype(np.int64))])[:n]
    W = int(g.w.astype(np.int64).sum())
    d = np.abs(pre[:, None] - pre[None, :])
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert np.array_equal(S, np.minimum(d, W - d))


@pytest.mark.parametrize("n", [3, 10, 101])
def test_oracle_uniform_cycle(n):
    w = 7
    src = np.arange(n, dtype=np.int32)
    S = oracle.apsp(n, src, (src + 1) % n, np.full(n, w, np.int32))
    i = np.arange(n)
    d = np.abs(i[:, None] - i[None, :])
    assert np.array_equal(S, w * np.minimum(d, n - d))


def _subdivided_lattice(gx, gy, s, wrap):
    """g x h grid / torus whose every base edge is subdivided into s+1 unit edges."""
    vid = lambda x, y: x * gy + y  # noqa: E731
    src, dst = [], []
    nxt = gx * gy
    for x in range(gx):
        for y in range(gy):
            for dx, dy in ((1, 0), (0, 1)):
                X, Y = x + dx, y + dy
                if wrap:
                    X, Y = X % gx, Y % gy
                elif X >= gx or Y >= gy:
                    continue
                prev = vid(x, y)
                for _ in range(s):
                    src.append(prev); dst.append(nxt); prev = nxt; nxt += 1
                src.append(prev); dst.append(vid(X, Y))
    m = len(src)
    return nxt, np.array(src, np.int32), np.array(dst, np.int32), np.ones(m, np.int32)


@pytest.mark.parametrize("gx,gy,s", [(4, 5, 0), (6, 3, 2), (5, 5, 3)])
def test_oracle_subdivided_grid_closed_form(gx, gy, s):
    n, src, dst, w = _subdivided_lattice(gx, gy, s, wrap=False)
    base = np.arange(gx * gy)
    S = oracle.apsp_rows(n, src, dst, w, base)[:, :gx * gy]
    x, y = base // gy, base % gy
    exp = (s + 1) * (np.abs(x[:, None] - x[None, :]) + np.abs(y[:, None] - y[None, :]))
    assert np.array_equal(S, exp)


@pytest.mark.parametrize("gx,gy,s", [(4, 6, 1), (5, 5, 2), (3, 7, 0)])
def test_oracle_subdivided_torus_closed_form(gx, gy, s):
    n, src, dst, w = _subdivided_lattice(gx, gy, s, wrap=True)
    base = np.arange(gx * gy)
    S = oracle.apsp_rows(n, src, dst, w, base)[:, :gx * gy]
    x, y = base // gy, base % gy
    dx = np.abs(x[:, None] - x[None, :]); dy = np.abs(y[:, None] - y[None, :])
    exp = (s + 1) * (np.minimum(dx, gx - dx) + np.minimum(dy, gy - dy))
    assert np.array_equal(S, exp)


@pytest.mark.parametrize("n,w", [(2, 5), (7, 3), (30, 11)])
def test_oracle_complete_graph(n, w):
    a, b = np.triu_indices(n, 1)
    S = oracle.apsp(n, a.astype(np.int32), b.astype(np.int32), np.full(len(a), w, np.int32))
    exp = np.full((n, n), w); np.fill_diagonal(exp, 0)
    assert np.array_equal(S, exp)


@pytest.mark.parametrize("seed", range(5))
def test_oracle_random_tree_path_sums(seed):
    rng = np.random.default_rng(seed)
    n = 120
    parent = np.array([-1] + [int(rng.integers(0, i)) for i in range(1, n)])
    wt = rng.integers(1, 101, size=n)
    # root distance and depth by walking parent pointers (tree: the unique path)
    depth_w = np.zeros(n, np.int64)
    for v in range(1, n):
        depth_w[v] = depth_w[parent[v]] + wt[v]
    anc = [set() for _ in range(n)]
    for v in range(n):
        x = v
        while x >= 0:
            anc[v].add(x); x = parent[x]
    exp = np.zeros((n, n), np.int64)
    for s in range(n):
        for t in range(n):
            common = anc[s] & anc[t]
            # the deepest common ancestor: largest root distance among common ancestors
            lca = max(common, key=lambda z: (depth_w[z], z))
            exp[s, t] = depth_w[s] + depth_w[t] - 2 * depth_w[lca]
    S = oracle.apsp(n, np.arange(1, n, dtype=np.int32), parent[1:].astype(np.int32), wt[1:].astype(np.int32))
    assert np.array_equal(S, exp)


# ------------------------------------------------------------------------------ P3 invariants
@pytest.mark.parametrize("seed", range(10))
def test_oracle_invariants(seed):
    g = gg.corner_cases(100 + seed, n_target=80)
    S = oracle.apsp(g.n, g.src, g.dst, g.w).astype(np.int64)
    assert np.array_equal(S, S.T)
    assert np.all(np.diag(S) == 0)
    fin = S < INF
    # triangle inequality (exhaustive), among finite entries
    tri = S[:, :, None] + S[None, :, :]
    assert np.all(S[:, None, :] <= np.where(fin[:, :, None] & fin[None, :, :], tri, np.iinfo(np.int64).max))
    comp = pins.components(g.n, g.src, g.dst)
    assert np.array_equal(S == INF, comp[:, None] != comp[None, :])


def test_oracle_triangle_sampled_cfg2():
    g = gg.config("cfg2")
    rng = np.random.default_rng(0)
    rows = rng.choice(g.n, 64, replace=False)
    S = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows).astype(np.int64)
    # d(a,t) <= d(a,b) + d(b,t) for sampled rows a, b among the computed rows
    for i in range(len(rows)):
        for j in range(len(rows)):
            assert np.all(S[i] <= S[i, rows[j]] + S[j])


# ------------------------------------------------------------------------------ P4 certificate
@pytest.mark.parametrize("name", ["cfg1"])
def test_oracle_bellman_certificate(name):
    g = gg.config(name)
    rows = np.arange(g.n)
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert pins.bellman_certificate(S, rows, g.n, g.src, g.dst, g.w)


def test_certificate_catches_perturbations():
    g = gg.corner_cases(7, n_target=50)
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    rows = np.arange(g.n)
    assert pins.bellman_certificate(S, rows, g.n, g.src, g.dst, g.w)
    rng = np.random.default_rng(1)
    for _ in range(60):
        s, t = rng.integers(0, g.n, 2)
        P = S.copy()
        P[s, t] = P[s, t] - 1 if P[s, t] > 0 else P[s, t] + 1
        if P[s, t] > INF:
            continue
        assert not pins.bellman_certificate(P, rows, g.n, g.src, g.dst, g.w)


# ------------------------------------------------------------------------------ P4, the C checker
# oracle.certify_rows (oracle/apsp_oracle.c) is what certifies the full cfg4 / cfg5 matrices
# (tests/test_full_verify_gpu.py).  Pinned here: it accepts the oracle's rows, it agrees with the numpy
# certificate on perturbed rows, and -- exhaustively on small graphs -- the true row is the ONLY row it
# accepts (uniqueness of the Bellman fixed point with weights >= 1).
@pytest.mark.parametrize("seed", range(12))
def test_c_certificate_accepts_oracle_rows(seed):
    g = gg.corner_cases(seed, n_target=30 + 40 * seed)
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    assert oracle.certify_rows(g.n, g.src, g.dst, g.w, np.arange(g.n), S) == (0, None)


def test_c_certificate_accepts_cfg_rows():
    for name, rows in (("cfg1", np.arange(2000)), ("cfg2", np.arange(0, 20000, 97))):
        g = gg.config(name)
        S = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
        assert oracle.certify_rows(g.n, g.src, g.dst, g.w, rows, S) == (0, None)


def test_c_certificate_agrees_with_numpy_on_perturbations():
    g = gg.corner_cases(7, n_target=50)
    S = oracle.apsp(g.n, g.src, g.dst, g.w)
    rows = np.arange(g.n)
    rng = np.random.default_rng(3)
    for trial in range(200):
        P = S.copy()
        s, t = (int(x) for x in rng.integers(0, g.n, 2))
        kind = trial % 4
        if kind == 0:
            P[s, t] += 1 if P[s, t] < INF else -1
        elif kind == 1:
            P[s, t] = P[s, t] - 1 if P[s, t] > 0 else 1
        elif kind == 2:
            P[s, t] = INF if P[s, t] != INF else 0
        else:   # swap two different entries of a row
            u = (t + 1 + int(rng.integers(0, g.n - 1))) % g.n
            if P[s, t] == P[s, u]:
                continue
            P[s, t], P[s, u] = P[s, u], P[s, t]
        bad, first = oracle.certify_rows(g.n, g.src, g.dst, g.w, rows, P)
        assert bad > 0 and first[0] == s
        assert not pins.bellman_certificate(P, rows, g.n, g.src, g.dst, g.w)


def test_c_certificate_unique_fixed_point_exhaustive_n4():
    # every graph on 4 labelled vertices, each edge absent or weight 1 or 2 (3^6 = 729 graphs); for every
    # source, all 8^4 candidate rows over {0..6, INF}: exactly one is accepted, the brute-force FW row
    n = 4
    vals = np.array(list(range(7)) + [INF], dtype=np.int32)
    cand = np.array(list(itertools.product(vals, repeat=n)), dtype=np.int32)   # (4096, 4)
    pairs = list(itertools.combinations(range(n), 2))
    graphs = 0
    for assign in itertools.product((0, 1, 2), repeat=len(pairs)):
        edges = [(a, b, x) for (a, b), x in zip(pairs, assign) if x]
        src = np.array([e[0] for e in edges], np.int32)
        dst = np.array([e[1] for e in edges], np.int32)
        w = np.array([e[2] for e in edges], np.int32)
        truth = pins.brute_fw(n, src, dst, w)
        for s in range(n):
            _, _, per = oracle.certify_rows(n, src, dst, w, np.full(len(cand), s), cand, per_row=True)
            ok = np.flatnonzero(per == 0)
            assert len(ok) == 1 and np.array_equal(cand[ok[0]], truth[s]), (edges, s)
        graphs += 1
    assert graphs == 3 ** 6


# ------------------------------------------------------------------------------ P5 library routine
@pytest.mark.parametrize("name,nrows", [("cfg1", None), ("cfg2", 200), ("cfg4", 24)])
def test_oracle_matches_scipy(name, nrows):
    from scipy.sparse import coo_matrix
    from scipy.sparse.csgraph import dijkstra

    g = gg.config(name)
    rows = np.arange(g.n) if nrows is None else np.random.default_rng(0).choice(g.n, nrows, replace=False)
    # scipy's csgraph sums duplicates in coo -> keep the min weight per pair explicitly
    keep = g.src != g.dst
    a = np.minimum(g.src[keep], g.dst[keep]).astype(np.int64)
    b = np.maximum(g.src[keep], g.dst[keep]).astype(np.int64)
    key = a * g.n + b
    order = np.lexsort((g.w[keep], key))
    key, wv = key[order], g.w[keep][order]
    first = np.r_[True, key[1:] != key[:-1]]
    A = coo_matrix((wv[first].astype(np.float64), (key[first] // g.n, key[first] % g.n)), shape=(g.n, g.n))
    ref = dijkstra(A.tocsr(), directed=False, indices=rows)
    ref = np.where(np.isinf(ref), INF, ref).astype(np.int64)
    S = oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    assert np.array_equal(S, ref)


# ------------------------------------------------------------------------------ P6 paper identities
def _reduced_fw(r, n):
    """Brute-force FW on G^r (P:88 edges, P:90 keep-the-shortest) indexed by original vertex id."""
    keep = r.re_u != r.re_v                       # closed-ear self-loops never shorten a path (C6)
    return pins.brute_fw(n, r.re_u[keep], r.re_v[keep], r.re_w[keep])


@pytest.mark.parametrize("seed", range(25))
def test_reduce_preserves_distances_and_expansion_formulas(seed):
    """S[u,v] = S^r[u,v] on V^r; P:111 2-term rule; P:115 4-term rule; P:107 same-ear rule
    (with the ear-id reading C8 and the along-ear distance C9)."""
    g = gg.corner_cases(200 + seed, n_target=50)
    S = oracle.apsp(g.n, g.src, g.dst, g.w).astype(np.int64)
    r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    T = np.nonzero(r.term)[0]
    Sr = _reduced_fw(r, g.n)
    assert np.array_equal(S[np.ix_(T, T)], Sr[np.ix_(T, T)])
    Sr = np.where(Sr >= INF, 1 << 40, Sr)
    X = np.nonzero(r.term == 0)[0]
    for x in X:
        two = np.minimum(r.d0[x] + Sr[r.end0[x], T], r.d1[x] + Sr[r.end1[x], T])
        assert np.array_equal(np.minimum(two, INF), S[x, T])
        for y in X:
            four = min(r.d0[x] + Sr[r.end0[x], r.end0[y]] + r.d0[y],
                       r.d0[x] + Sr[r.end0[x], r.end1[y]] + r.d1[y],
                       r.d1[x] + Sr[r.end1[x], r.end0[y]] + r.d0[y],
                       r.d1[x] + Sr[r.end1[x], r.end1[y]] + r.d1[y])
            if r.chain[x] == r.chain[y]:                                           # P:107, C8/C9
                four = min(four, abs(r.d0[x] - r.d0[y]))
            assert min(four, INF) == S[x, y], (x, y)


@pytest.mark.parametrize("seed", range(30))
def test_reduce_cyclomatic_identity(seed):
    """Lemma 3.1 proof: replacing a chain with k degree-two nodes removes k nodes and
    k edges, so |E| - |V| is preserved (E = simple edge set after C3, E^r before the P:90 rule)."""
    g = gg.corner_cases(300 + seed, n_target=70)
    r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
    keep = g.src != g.dst
    key = np.unique(np.minimum(g.src[keep], g.dst[keep]).astype(np.int64) * g.n
                    + np.maximum(g.src[keep], g.dst[keep]))
    assert len(key) - g.n == len(r.re_u) - r.n_reduced
    assert g.n - r.n_reduced == int(np.sum(r.deg == 2)) - r.n_promoted


def test_reduce_figure4_chains():
    """Fig. 4 (fixture tests/golden/fig4_chains.json): nodes 4, 5, 6 have degree two; chains
    {1,4,3} and {2,5,6,3} become G^r edges {1,3} and {2,3}.  The figure's other edges are completed
    with 1-2, 1-3 and 2-3 (its weights are only in the image; vertex 0 is an isolated filler so ids
    match the figure)."""
    import json
    import os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig4_chains.json")))
    E = [(1, 4, 2), (4, 3, 3), (2, 5, 1), (5, 6, 4), (6, 3, 2), (1, 2, 5), (1, 3, 9), (2, 3, 6)]
    src, dst, w = (np.array(c, np.int32) for c in zip(*E))
    r = oracle.reduce_graph(7, src, dst, w)
    assert list(np.nonzero(r.term == 0)[0]) == gold["degree_two_nodes"]
    for ch, (a, b) in zip(gold["chains"], gold["reduced_edges_from_chains"]):
        inner = ch[1:-1]
        assert len({int(r.chain[x]) for x in inner}) == 1
        for x in inner:
            assert {int(r.end0[x]), int(r.end1[x])} == {a, b}
    assert r.chain[4] != r.chain[5]
    red = sorted((int(min(a, b)), int(max(a, b)), int(x)) for a, b, x in zip(r.re_u, r.re_v, r.re_w))
    assert (1, 3, 5) in red and (2, 3, 7) in red and (1, 3, 9) in red
    S = oracle.apsp(7, src, dst, w)
    assert S[1, 3] == 5 and S[2, 3] == 6


def test_table1_max_memory_is_4_bytes_per_entry():
    """Table 1: Max Memory = 4 |V|^2 bytes, i.e. int32 distance entries (reading C1)."""
    import os
    rows = [l.split(",") for l in open(os.path.join(os.path.dirname(__file__), "golden", "table1_memory.csv"))
            if l.strip() and not l.startswith("#") and not l.startswith("graph")]
    for name, vk, mb in rows:
        n_implied = (int(mb) * 2 ** 20 / 4) ** 0.5
        assert int(n_implied // 1000) == int(vk), name


def test_config_sizes_match_survey():
    """The generated workloads have the sizes quoted for them."""
    for name, n, nr in [("cfg1", 2000, 1089), ("cfg2", 20000, 7917), ("cfg4", 100000, 29925)]:
        g = gg.config(name)
        r = oracle.reduce_graph(g.n, g.src, g.dst, g.w)
        assert g.n == n and r.n_reduced == nr


# ------------------------------------------------------------------------------ MCB oracle pins
# (paper sec. 3).  oracle.mcb_horton (Horton [18]) and oracle.mcb_depina (Algorithm 2 with the
# signed-graph search of sec. 3.2.1) are pinned against a brute force over the WHOLE cycle space of tiny
# multigraphs, closed forms, and Lemma 3.1 (W(MCB(G)) = W(MCB(G^r)), equal dimensions).
def _brute_mcb(n, src, dst, w):
    """Enumerate all 2^f elements of the cycle space (xor of fundamental cycles of a BFS spanning
    forest), keep the simple cycles (every vertex of degree 0 or 2, one connected piece), and run the
    matroid greedy over them by weight."""
    m = len(src)
    adj = [[] for _ in range(n)]
    for e in range(m):
        adj[src[e]].append((dst[e], e))
        adj[dst[e]].append((src[e], e))
    par, pe, seen = [-1] * n, [-1] * n, [False] * n
    intree = [False] * m
    for r in range(n):
        if seen[r]:
            continue
        seen[r] = True
        q = [r]
        for a in q:
            for b, e in adj[a]:
                if not seen[b]:
                    seen[b] = True
                    par[b], pe[b] = a, e
                    intree[e] = True
                    q.append(b)

    def path_bits(a):
        bits = 0
        while par[a] >= 0:
            bits ^= 1 << pe[a]
            a = par[a]
        return bits

    fund = [path_bits(src[e]) ^ path_bits(dst[e]) ^ (1 << e) for e in range(m) if not intree[e]]
    f = len(fund)
    cycles = []
    for mask in range(1, 1 << f):
        v = 0
        for i in range(f):
            if mask >> i & 1:
                v ^= fund[i]
        es = [e for e in range(m) if v >> e & 1]
        deg = [0] * n
        for e in es:
            deg[src[e]] += 1
            deg[dst[e]] += 1
        if any(d not in (0, 2) for d in deg):
            continue
        # connected: walk the edge set from one vertex
        verts = {x for e in es for x in (src[e], dst[e])}
        start = next(iter(verts))
        reach, stack = {start}, [start]
        while stack:
            a = stack.pop()
            for e in es:
                for x, y in ((src[e], dst[e]), (dst[e], src[e])):
                    if x == a and y not in reach:
                        reach.add(y)
                        stack.append(y)
        if reach != verts:
            continue
        cycles.append((sum(w[e] for e in es), v))
    cycles.sort(key=lambda c: c[0])
    basis, total = {}, 0     # pivot bit -> vector (echelon form)
    for wt, v in cycles:
        while v:
            p = v & -v
            if p in basis:
                v ^= basis[p]
            else:
                basis[p] = v
                total += wt
                break
        if len(basis) == f:
            break
    assert len(basis) == f
    return total, f


def _rand_multigraph(rng):
    n = int(rng.integers(2, 7))
    m = int(rng.integers(n - 1, n + 6))
    src, dst = [], []
    for _ in range(m):
        a = int(rng.integers(0, n))
        b = a if rng.random() < 0.08 else int(rng.integers(0, n))   # some self-loops, many parallel edges
        src.append(a)
        dst.append(b)
    w = [int(x) for x in rng.integers(1, 4, m)]                      # weights 1-3: many ties
    return n, src, dst, w


def test_mcb_oracles_match_brute_force_cycle_space():
    rng = np.random.default_rng(11)
    checked = 0
    while checked < 250:
        n, src, dst, w = _rand_multigraph(rng)
        k = len({pins_find(n, src, dst, v) for v in range(n)})
        if len(src) - n + k > 11:   # keep 2^f small
            continue
        bw, bf = _brute_mcb(n, src, dst, w)
        hw, hf, cyc = oracle.mcb_horton(n, src, dst, w)
        dw, df, _ = oracle.mcb_depina(n, src, dst, w)
        assert (hw, hf) == (bw, bf) == (dw, df), (n, src, dst, w)
        assert sum(int(sum(w[e] for e in c)) for c in cyc) == hw
        checked += 1


def pins_find(n, src, dst, v):
    """component representative of v (union-find over the edge list)"""
    p = list(range(n))

    def f(x):
        while p[x] != x:
            x = p[x]
        return x
    for a, b in zip(src, dst):
        ra, rb = f(a), f(b)
        if ra != rb:
            p[ra] = rb
    return f(v)


def _grid(gx, gy, s=0):
    """gx x gy grid, every base edge subdivided by s unit-weight vertices (unit weights)"""
    n = gx * gy
    src, dst = [], []
    for y in range(gy):
        for x in range(gx):
            i = y * gx + x
            for j in ([i + 1] if x + 1 < gx else []) + ([i + gx] if y + 1 < gy else []):
                prev = i
                for _ in range(s):
                    src.append(prev); dst.append(n); prev = n; n += 1
                src.append(prev); dst.append(j)
    return n, src, dst, [1] * len(src)


@pytest.mark.parametrize("gx,gy,s", [(2, 2, 0), (3, 4, 0), (5, 5, 0), (4, 3, 2), (6, 2, 1)])
def test_mcb_grid_closed_form(gx, gy, s):
    # a grid's faces: (gx-1)(gy-1) cycles of weight 4(s+1) each, the girth -> MCB weight 4(s+1)(gx-1)(gy-1)
    n, src, dst, w = _grid(gx, gy, s)
    f = (gx - 1) * (gy - 1)
    assert oracle.mcb_horton(n, src, dst, w)[:2] == (4 * (s + 1) * f, f)
    if n <= 40:
        assert oracle.mcb_depina(n, src, dst, w)[:2] == (4 * (s + 1) * f, f)


@pytest.mark.parametrize("lens", [(1, 2, 3), (2, 2, 2), (1, 1, 5), (3, 4, 7)])
def test_mcb_theta_closed_form(lens):
    # two vertices joined by three paths of lengths a <= b <= c: MCB = {a+b, a+c}
    a, b, c = sorted(lens)
    n, src, dst = 2, [], []
    for L in lens:
        prev = 0
        for _ in range(L - 1):
            src.append(prev); dst.append(n); prev = n; n += 1
        src.append(prev); dst.append(1)
    w = [1] * len(src)
    assert oracle.mcb_horton(n, src, dst, w)[:2] == (2 * a + b + c, 2)
    assert oracle.mcb_depina(n, src, dst, w)[:2] == (2 * a + b + c, 2)


@pytest.mark.parametrize("k", [3, 4, 5, 6])
def test_mcb_complete_graph(k):
    # K_k, unit weights: girth 3 and the triangles span the cycle space -> 3 * (m - n + 1)
    src, dst = zip(*itertools.combinations(range(k), 2))
    f = len(src) - k + 1
    assert oracle.mcb_horton(k, src, dst, [1] * len(src))[:2] == (3 * f, f)
    assert oracle.mcb_depina(k, src, dst, [1] * len(src))[:2] == (3 * f, f)


@pytest.mark.parametrize("n", [3, 10, 57])
def test_mcb_cycle_is_its_own_basis(n):
    g = gg.cycle(n, seed=n)
    assert oracle.mcb_horton(g.n, g.src, g.dst, g.w)[:2] == (int(g.w.sum()), 1)


def _canonical(g):
    """reading C3: drop self-loops, parallel edges -> the lightest"""
    best = {}
    for a, b, x in zip(g.src.tolist(), g.dst.tolist(), g.w.tolist()):
        if a == b:
            continue
        key = (min(a, b), max(a, b))
        best[key] = min(best.get(key, x), x)
    ks = sorted(best)
    return (np.array([k[0] for k in ks], np.int32), np.array([k[1] for k in ks], np.int32),
            np.array([best[k] for k in ks], np.int32))


@pytest.mark.parametrize("seed", range(15))
def test_mcb_lemma_3_1_reduced_graph(seed):
    # Lemma 3.1: the MCB of G and of its reduced multigraph G^r (chains -> weighted edges,
    # closed ears -> self-loops, parallel chains -> parallel edges) have the same weight and dimension
    g = gg.corner_cases(seed, n_target=25 + 6 * seed)
    s, d, w = _canonical(g)
    red = oracle.reduce_graph(g.n, s, d, w)
    terms = np.flatnonzero(red.term)
    idx = -np.ones(g.n, np.int64)
    idx[terms] = np.arange(len(terms))
    ru, rv = idx[red.re_u], idx[red.re_v]
    assert np.all(ru >= 0) and np.all(rv >= 0)
    wg, fg, _ = oracle.mcb_horton(g.n, s, d, w)
    wr, fr, _ = oracle.mcb_horton(len(terms), ru.astype(np.int32), rv.astype(np.int32), red.re_w.astype(np.int32))
    assert (wg, fg) == (wr, fr)
    if len(terms) <= 60 and fr <= 60:
        assert oracle.mcb_depina(len(terms), ru.astype(np.int32), rv.astype(np.int32), red.re_w.astype(np.int32))[:2] == (wr, fr)
