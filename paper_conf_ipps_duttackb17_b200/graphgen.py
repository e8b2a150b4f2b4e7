"""Seeded synthetic graph generators (inputs only -- no shortest-path arithmetic lives here).

This module is the ONLY code shared by the product path, the oracle-based tests and ``bench.py``: it
builds edge lists ``(src, dst, w)`` with the shapes of the paper's workloads and nothing else.

Workload recipes:

* weights are i.i.d. uniform integers in [1, 100] (``numpy.random.default_rng(seed)``);
* sparse graphs with a high share of degree-two vertices, as in Table 1 ("Nodes Removed"
  0 .. 77.6 %): a base graph whose edges are subdivided by degree-two vertices dropped
  multinomially onto the base edges;
* vertex ids are spatially coherent like real road / power datasets: every vertex has a 2-D position
  (chain vertices interpolated along their base edge) and ids follow the Morton order of positions;
* cfg1 ``torus`` 33x33 + 911 subdivisions (N = 2000, ~45 % degree two);
  cfg2 ``grid`` 89x89 open grid + subdivisions to N = 20,000 (road-like, ~60 %);
  cfg3 ``torus`` with N_r = 50k (1 - f) base vertices + f * 50k subdivisions (f-sweep);
  cfg4 ``power_grid`` 28,500 uniform points joined to their 3 nearest neighbours, +5 % pendant leaves,
  components chained, N = 100,000 (~30k reduced vertices);
  cfg5 the same generator with 57,000 base points and N = 200,000.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

WMAX = 100


@dataclass
class Graph:
    n: int
    src: np.ndarray  # int32 [m]
    dst: np.ndarray  # int32 [m]
    w: np.ndarray    # int32 [m]
    meta: dict = field(default_factory=dict)

    @property
    def m(self) -> int:
        return int(self.src.shape[0])


# ----------------------------------------------------------------------------------- helpers
def _morton_codes(pos: np.ndarray) -> np.ndarray:
    """64-bit Morton (Z-order) codes of 2-D positions normalised to [0, 1)."""
    lo = pos.min(axis=0)
    span = np.maximum(pos.max(axis=0) - lo, 1e-12)
    q = np.minimum(((pos - lo) / span * (1 << 20)).astype(np.uint64), (1 << 20) - 1)

    def spread(x):
        x = x & np.uint64(0xFFFFF)
        x = (x | (x << np.uint64(16))) & np.uint64(0x0000FFFF0000FFFF)
        x = (x | (x << np.uint64(8))) & np.uint64(0x00FF00FF00FF00FF)
        x = (x | (x << np.uint64(4))) & np.uint64(0x0F0F0F0F0F0F0F0F)
        x = (x | (x << np.uint64(2))) & np.uint64(0x3333333333333333)
        x = (x | (x << np.uint64(1))) & np.uint64(0x5555555555555555)
        return x

    return spread(q[:, 0]) | (spread(q[:, 1]) << np.uint64(1))


def _finish(n, u, v, pos, rng, meta, labels="morton") -> Graph:
    """Relabel (Morton / random / identity), draw weights, shuffle edge order and direction."""
    u = np.asarray(u, dtype=np.int64)
    v = np.asarray(v, dtype=np.int64)
    if labels == "morton":
        order = np.argsort(_morton_codes(pos), kind="stable")
        perm = np.empty(n, dtype=np.int64)
        perm[order] = np.arange(n)
    elif labels == "random":
        perm = rng.permutation(n)
    else:
        perm = np.arange(n)
    u, v = perm[u], perm[v]
    m = len(u)
    w = rng.integers(1, WMAX + 1, size=m)
    eo = rng.permutation(m)
    u, v, w = u[eo], v[eo], w[eo]
    flip = rng.random(m) < 0.5
    u, v = np.where(flip, v, u), np.where(flip, u, v)
    meta = dict(meta)
    meta["labels"] = labels
    return Graph(n, u.astype(np.int32), v.astype(np.int32), w.astype(np.int32), meta)


def _subdivide(nb, bu, bv, bpos, n_sub, rng, wrap=None):
    """Drop ``n_sub`` degree-two vertices multinomially onto base edges (bu[i], bv[i]).

    Returns (n, u, v, pos): edge endpoint arrays of the subdivided graph and vertex positions
    (new vertices interpolated along their base edge; ``wrap`` = torus period for interpolation).
    """
    k = len(bu)
    cnt = rng.multinomial(n_sub, np.full(k, 1.0 / k)) if n_sub > 0 else np.zeros(k, dtype=np.int64)
    n = nb + n_sub
    # vertex ids of the new vertices: contiguous per base edge
    first = nb + np.concatenate([[0], np.cumsum(cnt)[:-1]])
    e_of = np.repeat(np.arange(k), cnt)                      # base edge of each new vertex
    idx = np.arange(n_sub) - (first[e_of] - nb)              # 0..c-1 position along the edge
    # positions
    pu, pv = bpos[bu[e_of]], bpos[bv[e_of]]
    d = pv - pu
    if wrap is not None:
        d = (d + wrap / 2) % wrap - wrap / 2
    t = (idx + 1) / (cnt[e_of] + 1)
    npos = pu + d * t[:, None]
    if wrap is not None:
        npos = npos % wrap
    pos = np.concatenate([bpos, npos], axis=0) if n_sub else bpos.copy()
    # edges: for a base edge with c new vertices x0..x_{c-1}: u-x0, x0-x1, ..., x_{c-1}-v
    new_ids = np.arange(nb, n)
    # chain-internal and last edges
    has = cnt > 0
    eu = [bu[~has]]
    ev = [bv[~has]]
    # u -> first new vertex
    eu.append(bu[has]); ev.append(first[has])
    # consecutive new vertices on the same base edge
    same = np.zeros(n_sub, dtype=bool)
    if n_sub > 1:
        same[1:] = e_of[1:] == e_of[:-1]
    eu.append(new_ids[np.nonzero(same)[0] - 1]); ev.append(new_ids[same])
    # last new vertex -> v
    last = first[has] + cnt[has] - 1
    eu.append(last); ev.append(bv[has])
    return n, np.concatenate(eu), np.concatenate(ev), pos


# ----------------------------------------------------------------------------------- families
def torus(gx: int, gy: int, n_sub: int, seed: int = 0, labels: str = "morton") -> Graph:
    """gx x gy torus (every base vertex degree 4) + ``n_sub`` subdivision vertices."""
    rng = np.random.default_rng(seed)
    ix, iy = np.meshgrid(np.arange(gx), np.arange(gy), indexing="ij")
    ix, iy = ix.ravel(), iy.ravel()
    vid = lambda x, y: (x % gx) * gy + (y % gy)  # noqa: E731
    bu = np.concatenate([vid(ix, iy), vid(ix, iy)])
    bv = np.concatenate([vid(ix + 1, iy), vid(ix, iy + 1)])
    bpos = np.stack([ix, iy], axis=1).astype(np.float64)
    n, u, v, pos = _subdivide(gx * gy, bu, bv, bpos, n_sub, rng, wrap=np.array([gx, gy], dtype=np.float64))
    return _finish(n, u, v, pos, rng, dict(family="torus", gx=gx, gy=gy, n_sub=n_sub, seed=seed), labels)


def grid(gx: int, gy: int, n_total: int, seed: int = 0, labels: str = "morton") -> Graph:
    """Open gx x gy grid (road-like; corners have degree 2) subdivided up to ``n_total`` vertices."""
    rng = np.random.default_rng(seed)
    nb = gx * gy
    ix, iy = np.meshgrid(np.arange(gx), np.arange(gy), indexing="ij")
    vid = ix * gy + iy
    bu = np.concatenate([vid[:-1, :].ravel(), vid[:, :-1].ravel()])
    bv = np.concatenate([vid[1:, :].ravel(), vid[:, 1:].ravel()])
    bpos = np.stack([ix.ravel(), iy.ravel()], axis=1).astype(np.float64)
    n, u, v, pos = _subdivide(nb, bu, bv, bpos, max(0, n_total - nb), rng)
    return _finish(n, u, v, pos, rng, dict(family="grid", gx=gx, gy=gy, seed=seed), labels)


def power_grid(n_base: int, n_total: int, seed: int = 0, pendant_frac: float = 0.05,
               labels: str = "morton") -> Graph:
    """Power-grid-like graph: 3-nearest-neighbour geometric base graph + pendant leaves, base
    components chained by one edge each, then degree-two vertices dropped onto the base edges."""
    from scipy.sparse import coo_matrix
    from scipy.sparse.csgraph import connected_components
    from scipy.spatial import cKDTree

    rng = np.random.default_rng(seed)
    pts = rng.random((n_base, 2))
    _, nn = cKDTree(pts).query(pts, k=4)
    a = np.repeat(np.arange(n_base), 3)
    b = nn[:, 1:].ravel()
    lo, hi = np.minimum(a, b), np.maximum(a, b)
    key = np.unique(lo.astype(np.int64) * n_base + hi)
    bu, bv = (key // n_base), (key % n_base)
    # pendant leaves
    n_p = int(round(pendant_frac * n_base))
    anchors = rng.integers(0, n_base, size=n_p)
    leaf = np.arange(n_base, n_base + n_p)
    ppos = pts[anchors] + rng.normal(scale=0.3 / np.sqrt(n_base), size=(n_p, 2))
    bu = np.concatenate([bu, anchors]); bv = np.concatenate([bv, leaf])
    nb = n_base + n_p
    bpos = np.concatenate([pts, ppos], axis=0)
    # chain the base components
    adj = coo_matrix((np.ones(len(bu)), (bu, bv)), shape=(nb, nb))
    ncomp, lab = connected_components(adj, directed=False)
    if ncomp > 1:
        rep = np.full(ncomp, -1, dtype=np.int64)
        order = np.argsort(lab, kind="stable")
        first_idx = np.searchsorted(lab[order], np.arange(ncomp))
        rep = order[first_idx]
        bu = np.concatenate([bu, rep[:-1]]); bv = np.concatenate([bv, rep[1:]])
    n, u, v, pos = _subdivide(nb, bu, bv, bpos, max(0, n_total - nb), rng)
    return _finish(n, u, v, pos, rng, dict(family="power_grid", n_base=n_base, n_pendant=n_p,
                                           base_components=int(ncomp), seed=seed), labels)


def path(n: int, seed: int = 0, wmax: int = WMAX) -> Graph:
    """Simple path 0-1-...-(n-1) with random weights (ids in path order)."""
    rng = np.random.default_rng(seed)
    u = np.arange(n - 1)
    w = rng.integers(1, wmax + 1, size=n - 1)
    return Graph(n, u.astype(np.int32), (u + 1).astype(np.int32), w.astype(np.int32), dict(family="path"))


def cycle(n: int, seed: int = 0, wmax: int = WMAX) -> Graph:
    """Simple cycle 0-1-...-(n-1)-0 with random weights (edge i joins i and i+1 mod n)."""
    rng = np.random.default_rng(seed)
    u = np.arange(n)
    w = rng.integers(1, wmax + 1, size=n)
    return Graph(n, u.astype(np.int32), ((u + 1) % n).astype(np.int32), w.astype(np.int32),
                 dict(family="cycle"))


def corner_cases(seed: int, n_target: int = 60) -> Graph:
    """Small random multigraph exercising every chain corner case of DESIGN.md readings C3-C8:
    self-loops, parallel edges (also given in both directions with different weights), pendant
    paths, closed ears, parallel chains between the same ends, pure-cycle components, isolated
    vertices and path components.  Ids are randomly relabelled."""
    rng = np.random.default_rng(seed)
    us, vs = [], []
    n = 0

    def new(k):
        nonlocal n
        ids = np.arange(n, n + k)
        n += k
        return ids

    def chain_between(a, b, k):
        xs = new(k)
        seq = [a, *xs.tolist(), b]
        for i in range(len(seq) - 1):
            us.append(seq[i]); vs.append(seq[i + 1])

    # a random core on a few vertices
    core = new(int(rng.integers(3, 9)))
    for _ in range(int(rng.integers(len(core), 3 * len(core)))):
        a, b = rng.choice(core, 2)
        us.append(a); vs.append(b)          # may be a self-loop or a parallel edge
    while n < n_target:
        kind = int(rng.integers(0, 8))
        a, b = rng.choice(core, 2)
        k = int(rng.integers(1, 6))
        if kind == 0:                       # chain between two core vertices (maybe a == b)
            chain_between(a, b, k)
        elif kind == 1:                     # parallel chains between the same ends
            chain_between(a, b, k); chain_between(a, b, int(rng.integers(1, 6)))
        elif kind == 2:                     # closed ear at a
            chain_between(a, a, max(k, 2))
        elif kind == 3:                     # pendant path
            xs = new(k)
            seq = [a, *xs.tolist()]
            for i in range(len(seq) - 1):
                us.append(seq[i]); vs.append(seq[i + 1])
        elif kind == 4:                     # pure-cycle component
            xs = new(max(k, 3))
            for i in range(len(xs)):
                us.append(xs[i]); vs.append(xs[(i + 1) % len(xs)])
        elif kind == 5:                     # isolated vertex / path component
            xs = new(k)
            for i in range(len(xs) - 1):
                us.append(xs[i]); vs.append(xs[i + 1])
        elif kind == 6:                     # duplicated edge in reverse direction
            if us:
                j = int(rng.integers(0, len(us)))
                us.append(vs[j]); vs.append(us[j])
        else:                               # self-loop on a chain vertex / new core vertex
            if n > 0:
                x = int(rng.integers(0, n))
                us.append(x); vs.append(x)
            core = np.concatenate([core, new(1)])
            us.append(core[-1]); vs.append(a)
    u = np.array(us, dtype=np.int64)
    v = np.array(vs, dtype=np.int64)
    return _finish(n, u, v, None, rng, dict(family="corner_cases", seed=seed), labels="random")


def block_tree(seed: int, n_target: int = 200, big: int = 0, chains: bool = True) -> Graph:
    """Sparse graph made of many biconnected blocks glued at articulation points -- the shape sec. 2.2
    of the paper is about (real sparse graphs are not 2-connected): cycles, small grids, wheels
    and theta graphs hung off each other at single vertices, bridges and pendant trees, 1-3 connected
    components plus isolated vertices.  ``big`` > 0 makes the first block a grid of about ``big``
    vertices (a dominant block, like the largest BCC of cfg4); ``chains`` subdivides some block
    edges by degree-two vertices.  Ids are randomly relabelled."""
    rng = np.random.default_rng(seed)
    us, vs = [], []
    n = 0

    def new(k):
        nonlocal n
        ids = list(range(n, n + k))
        n += k
        return ids

    def edge(a, b):
        if chains and rng.random() < 0.3:   # subdivide by 1-3 degree-two vertices
            xs = new(int(rng.integers(1, 4)))
            seq = [a, *xs, b]
        else:
            seq = [a, b]
        for i in range(len(seq) - 1):
            us.append(seq[i]); vs.append(seq[i + 1])

    def grid_block(a, gx, gy):
        ids = [a] + new(gx * gy - 1)
        for y in range(gy):
            for x in range(gx):
                i = y * gx + x
                if x + 1 < gx:
                    edge(ids[i], ids[i + 1])
                if y + 1 < gy:
                    edge(ids[i], ids[i + gx])
        return ids

    ncomp = int(rng.integers(1, 4))
    for c in range(ncomp):
        goal = n_target * (c + 1) // ncomp
        if big and c == 0:
            side = max(2, int(round(big ** 0.5)))
            pool = grid_block(new(1)[0], side, side)
        else:
            pool = new(int(rng.integers(3, 7)))
            for i in range(len(pool)):
                edge(pool[i], pool[(i + 1) % len(pool)])
        while n < goal:
            a = int(rng.choice(pool))
            kind = int(rng.integers(0, 6))
            if kind == 0:                       # cycle through a
                xs = new(int(rng.integers(2, 7)))
                seq = [a, *xs, a]
                for i in range(len(seq) - 1):
                    edge(seq[i], seq[i + 1])
                pool += xs
            elif kind == 1:                     # bridge to a pendant tree
                xs = new(int(rng.integers(1, 5)))
                prev = [a]
                for x in xs:
                    edge(int(rng.choice(prev)), x)
                    prev.append(x)
                pool += xs
            elif kind == 2:                     # small grid sharing its corner with a
                pool += grid_block(a, int(rng.integers(2, 4)), int(rng.integers(2, 5)))[1:]
            elif kind == 3:                     # theta: three internally disjoint a-b paths
                b = new(1)[0]
                for _ in range(3):
                    xs = new(int(rng.integers(0, 3)))
                    seq = [a, *xs, b]
                    for i in range(len(seq) - 1):
                        edge(seq[i], seq[i + 1])
                    pool += xs
                pool.append(b)
            elif kind == 4:                     # wheel with hub a
                xs = new(int(rng.integers(3, 7)))
                for i in range(len(xs)):
                    edge(xs[i], xs[(i + 1) % len(xs)])
                    edge(a, xs[i])
                pool += xs
            else:                               # a chord inside the current component
                b = int(rng.choice(pool))
                if b != a and rng.random() < 0.3:
                    edge(a, b)
    new(int(rng.integers(0, 4)))               # isolated vertices
    u = np.array(us, dtype=np.int64)
    v = np.array(vs, dtype=np.int64)
    return _finish(n, u, v, None, rng, dict(family="block_tree", seed=seed, big=big), labels="random")


# ----------------------------------------------------------------------------------- configs
# cfg3 torus shapes for the degree-two fraction sweep f (N = 50,000, N_r = 50k (1 - f)).
CFG3_SHAPES = {0: (200, 250), 20: (200, 200), 40: (150, 200), 60: (100, 200), 80: (100, 100)}


def config(name: str, seed: int = 0, labels: str = "morton") -> Graph:
    """BASELINE.json configs: cfg1, cfg2, cfg3_f{0,20,40,60,80}, cfg4, cfg5."""
    if name == "cfg1":
        return torus(33, 33, 911, seed, labels)
    if name == "cfg2":
        return grid(89, 89, 20000, seed, labels)
    if name.startswith("cfg3"):
        f = int(name.split("_f")[1]) if "_f" in name else 60
        gx, gy = CFG3_SHAPES[f]
        return torus(gx, gy, 50000 - gx * gy, seed, labels)
    if name == "cfg4":
        return power_grid(28500, 100000, seed, labels=labels)
    if name == "cfg5":
        return power_grid(57000, 200000, seed, labels=labels)
    raise ValueError(f"unknown config {name!r}")


def stats(g: Graph) -> dict:
    """Measured N, M, degree-two fraction and degree histogram of a generated graph (reported by
    bench.py; pure counting, no path arithmetic)."""
    u, v = g.src.astype(np.int64), g.dst.astype(np.int64)
    keep = u != v
    lo, hi = np.minimum(u[keep], v[keep]), np.maximum(u[keep], v[keep])
    key = np.unique(lo * g.n + hi)
    deg = np.bincount(np.concatenate([key // g.n, key % g.n]), minlength=g.n)
    return dict(n=g.n, m=g.m, deg2_frac=float(np.mean(deg == 2)), deg1_frac=float(np.mean(deg == 1)),
                max_deg=int(deg.max()) if g.n else 0)
