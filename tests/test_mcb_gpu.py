"""GPU minimum cycle basis (paper sec. 3) against the CPU oracle.

The MCB WEIGHT is unique, so it is compared exactly with oracle.mcb_horton (Horton's algorithm on the
canonical G; pinned in test_oracle_pins.py by brute force, closed forms and Lemma 3.1), together with the
dimension f = m - n + k.  WHICH basis is returned is not unique, so every returned cycle is checked for
validity instead: expanded to G (post-processing, sec. 3.3.3) it is a simple closed walk of G whose
weight is the reported one, and the f cycles are linearly independent over GF(2).
"""
import itertools

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ea():
    import paper_conf_ipps_duttackb17_b200 as p
    p.lib()
    return p


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def canonical(n, src, dst, w):
    """reading C3: self-loops dropped, parallel edges -> the lightest; edge index by (min, max)"""
    best = {}
    for a, b, x in zip(np.asarray(src).tolist(), np.asarray(dst).tolist(), np.asarray(w).tolist()):
        if a != b:
            k = (min(a, b), max(a, b))
            best[k] = min(best.get(k, x), x)
    keys = sorted(best)
    index = {k: i for i, k in enumerate(keys)}
    s = np.array([k[0] for k in keys], np.int32)
    d = np.array([k[1] for k in keys], np.int32)
    ww = np.array([best[k] for k in keys], np.int32)
    return s, d, ww, index


def check_mcb(ea, n, src, dst, w):
    s, d, ww, index = canonical(n, src, dst, w)
    ref_w, ref_f, _ = oracle.mcb_horton(n, s, d, ww)
    res = ea.mcb(n, dev(src), dev(dst), dev(w))
    try:
        info = res.info()
        assert (info["weight"], info["dim"]) == (ref_w, ref_f), (info, ref_w, ref_f)
        cw = res.weights().cpu().numpy()
        assert int(cw.sum()) == ref_w
        basis = {}
        for i in range(info["dim"]):
            cyc = res.cycle(i).cpu().numpy().tolist()
            assert len(cyc) >= 1 and len(set(cyc)) == len(cyc), f"cycle {i} repeats a vertex: {cyc}"
            if len(cyc) < 3:
                raise AssertionError(f"cycle {i} has {len(cyc)} vertices in a simple graph: {cyc}")
            vec, tot = 0, 0
            for a, b in zip(cyc, cyc[1:] + cyc[:1]):
                k = (min(a, b), max(a, b))
                assert k in index, f"cycle {i}: {a}-{b} is not an edge of G"
                vec ^= 1 << index[k]
                tot += int(ww[index[k]])
            assert tot == int(cw[i]), (i, tot, int(cw[i]))
            while vec:   # GF(2) independence of the f cycles
                p = vec & -vec
                if p in basis:
                    vec ^= basis[p]
                else:
                    basis[p] = vec
                    break
            assert vec, f"cycle {i} depends on the earlier ones"
        return info
    finally:
        res.destroy()


@pytest.mark.parametrize("seed", range(20))
def test_mcb_corner_cases(ea, seed):
    g = gg.corner_cases(seed, n_target=30 + 15 * seed)
    check_mcb(ea, g.n, g.src, g.dst, g.w)


def test_mcb_cfg1(ea):
    g = gg.config("cfg1")
    info = check_mcb(ea, g.n, g.src, g.dst, g.w)
    assert info["n_reduced"] == 1089 and info["dim"] == g.m - g.n + 1


@pytest.mark.parametrize("gx,gy,s", [(4, 4, 0), (7, 5, 2), (12, 9, 1)])
def test_mcb_grid_closed_form(ea, gx, gy, s):
    # subdivided grid, unit weights: (gx-1)(gy-1) faces of weight 4(s+1) -- the girth -- form an MCB
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
    w = [1] * len(src)
    info = check_mcb(ea, n, src, dst, w)
    f = (gx - 1) * (gy - 1)
    assert (info["weight"], info["dim"]) == (4 * (s + 1) * f, f)


@pytest.mark.parametrize("case", ["tree", "cycle", "two_cycles", "theta", "k5", "pendants", "ties"])
def test_mcb_degenerate(ea, case):
    if case == "tree":
        g = gg.corner_cases(3, n_target=40)
        rng = np.random.default_rng(0)
        n = 50
        src = np.arange(1, n)
        dst = np.array([rng.integers(0, v) for v in range(1, n)])
        w = rng.integers(1, 100, n - 1)
        res = ea.mcb(n, dev(src), dev(dst), dev(w))
        assert res.info()["dim"] == 0 and res.info()["weight"] == 0
        res.destroy()
        return
    if case == "cycle":
        g = gg.cycle(300, seed=2)
        n, src, dst, w = g.n, g.src, g.dst, g.w
    elif case == "two_cycles":     # two components, each a pure cycle (closed ears at promoted vertices)
        a, b = gg.cycle(40, seed=1), gg.cycle(25, seed=3)
        n = a.n + b.n
        src, dst, w = np.concatenate([a.src, b.src + a.n]), np.concatenate([a.dst, b.dst + a.n]), np.concatenate([a.w, b.w])
    elif case == "theta":          # two vertices and three chains: parallel edges of G^r
        n, src, dst = 2, [], []
        for L in (3, 5, 8):
            prev = 0
            for _ in range(L - 1):
                src.append(prev); dst.append(n); prev = n; n += 1
            src.append(prev); dst.append(1)
        w = list(range(1, len(src) + 1))
    elif case == "k5":
        src, dst = map(list, zip(*itertools.combinations(range(5), 2)))
        n, w = 5, [7] * 10
    elif case == "pendants":       # a grid with pendant paths and isolated vertices
        g = gg.corner_cases(5, n_target=200)
        n, src, dst, w = g.n, g.src, g.dst, g.w
    else:                          # all weights equal: maximal ties between candidate cycles
        g = gg.torus(6, 7, 10, seed=9)
        n, src, dst, w = g.n, g.src, g.dst, np.ones_like(g.w)
    check_mcb(ea, n, src, dst, w)


def test_mcb_deterministic(ea):
    """Two builds of the same graph choose the same trees, candidates and basis (the perturbation of
    reading M3 is a fixed hash; every tie is broken by the edge id)."""
    g = gg.config("cfg1")
    runs = []
    for _ in range(2):
        r = ea.mcb(g.n, dev(g.src), dev(g.dst), dev(g.w))
        runs.append((r.info(), r.weights().cpu().numpy(), [r.cycle(i).cpu().numpy().tolist() for i in (0, 7, 500)]))
        r.destroy()
    assert runs[0][0] == runs[1][0]
    assert np.array_equal(runs[0][1], runs[1][1])
    assert runs[0][2] == runs[1][2]
