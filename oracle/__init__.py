"""CPU oracle for the ear-reduced APSP hot path.  TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package.  The product package ``paper_conf_ipps_duttackb17_b200`` never imports,
links or executes anything here, and the two share no code (the seeded graph generators in
``paper_conf_ipps_duttackb17_b200/graphgen.py`` hold none of the method's arithmetic and are the only
thing both sides use).

Functions (paper = /root/reference/PAPER.md, ``P:NN`` = line NN):

* :func:`apsp_rows` -- rows of ``S[s, t]``, the shortest-path weight in the ORIGINAL undirected graph
  (P:41), by Dijkstra from each requested source (the paper's SSSP primitive) on
  plain C/OpenMP (``apsp_oracle.c``).  Unreachable -> ``INF`` (reading C11).
* :func:`apsp` -- all rows.
* :func:`reduce_graph` -- ``G^r = Reduce(G)`` by a sequential chain walk as defined
  (readings C3-C7 in DESIGN.md).
* :func:`certify_rows` -- a CHECKER: how many entries of candidate rows violate the Bellman optimality
  equations of S on the original graph (P:41, P:109 restated as a fixed point; SURVEY 8.c pin P4).
  Its only solution with integer weights >= 1 is S itself, and it costs O(N + M) per row, so it
  certifies whole N x N matrices (cfg4, cfg5) where Dijkstra from every source would take minutes.

* :func:`mcb_horton` / :func:`mcb_depina` -- minimum cycle basis (paper sec. 3) of a
  multigraph (self-loops and parallel edges allowed, as in G^r): Horton's algorithm [18] (the
  Horton set + a GF(2) greedy) and de Pina's Algorithm 2 with the signed-graph search of sec. 3.2.1
  (``mcb_oracle.c``).  Two independent routes to the unique MCB weight.

Pinned by ``tests/test_oracle_pins.py``: brute-force Floyd-Warshall and exhaustive enumeration of
all small graphs (P1), closed forms (P2), invariants (P3), the Bellman certificate (P4), scipy's
Dijkstra (P5) and the paper's own identities / Fig. 4 chains (P6).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

INF = 0x3FFFFFFF
_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "apsp_oracle.c")
_SRCS = [_SRC, os.path.join(_HERE, "mcb_oracle.c")]
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile ``liboracle.so`` with gcc (plain C + OpenMP)."""
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(s) for s in _SRCS):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", tmp, *_SRCS])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        lib.oracle_apsp_rows.argtypes = [ctypes.c_int32, ctypes.c_int64, P, P, P, ctypes.c_int32, P, P,
                                         ctypes.c_int32]
        lib.oracle_apsp_rows.restype = ctypes.c_int
        lib.oracle_num_threads.argtypes = [ctypes.c_int32]
        lib.oracle_num_threads.restype = ctypes.c_int
        lib.oracle_reduce.argtypes = [ctypes.c_int32, ctypes.c_int64, P, P, P] + [P] * 10 + [ctypes.c_int64, P]
        lib.oracle_reduce.restype = ctypes.c_int
        lib.oracle_certify_rows.argtypes = [ctypes.c_int32, ctypes.c_int64, P, P, P, ctypes.c_int32, P, P,
                                            ctypes.c_int64, ctypes.c_int32, P, P]
        lib.oracle_certify_rows.restype = ctypes.c_int64
        lib.oracle_mcb_horton.argtypes = [ctypes.c_int32, ctypes.c_int64, P, P, P, P, P, P, P, ctypes.c_int64]
        lib.oracle_mcb_horton.restype = ctypes.c_int
        lib.oracle_mcb_depina.argtypes = [ctypes.c_int32, ctypes.c_int64, P, P, P, P, P, P]
        lib.oracle_mcb_depina.restype = ctypes.c_int
        _lib = lib
    return _lib


def _edges(src, dst, w):
    src = np.ascontiguousarray(src, dtype=np.int32)
    dst = np.ascontiguousarray(dst, dtype=np.int32)
    w = np.ascontiguousarray(w, dtype=np.int32)
    assert src.shape == dst.shape == w.shape
    return src, dst, w


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def num_threads(nthreads: int = 0) -> int:
    return int(_load().oracle_num_threads(nthreads))


def apsp_rows(n: int, src, dst, w, rows, nthreads: int = 0) -> np.ndarray:
    """``S[rows, :]`` as an int32 array of shape (len(rows), n)."""
    src, dst, w = _edges(src, dst, w)
    rows = np.ascontiguousarray(rows, dtype=np.int32)
    out = np.empty((len(rows), n), dtype=np.int32)
    st = _load().oracle_apsp_rows(n, len(src), _ptr(src), _ptr(dst), _ptr(w), len(rows), _ptr(rows),
                                  _ptr(out), nthreads)
    if st != 0:
        raise ValueError(f"oracle_apsp_rows failed with status {st}")
    return out


def apsp(n: int, src, dst, w, nthreads: int = 0) -> np.ndarray:
    """The full ``S`` (n x n int32)."""
    return apsp_rows(n, src, dst, w, np.arange(n, dtype=np.int32), nthreads)


def certify_rows(n: int, src, dst, w, rows, D: np.ndarray, nthreads: int = 0, per_row: bool = False):
    """Check candidate rows ``D[i] == S[rows[i], :]`` through the Bellman optimality equations (see the
    module docstring).  ``D``: int32, shape (len(rows), >= n), C-contiguous rows.  Returns
    ``(violations, (i, t) of the first one or None)`` -- plus the per-row violation counts with
    ``per_row``."""
    src, dst, w = _edges(src, dst, w)
    rows = np.ascontiguousarray(rows, dtype=np.int32)
    if D.dtype != np.int32 or D.ndim != 2 or D.shape[0] < len(rows) or D.shape[1] < n or D.strides[1] != 4:
        raise ValueError("D must be an int32 (rows, >= n) array with unit column stride")
    first = np.full(2, -1, dtype=np.int64)
    rb = np.zeros(len(rows), dtype=np.int64) if per_row else None
    bad = _load().oracle_certify_rows(n, len(src), _ptr(src), _ptr(dst), _ptr(w), len(rows), _ptr(rows),
                                      D.ctypes.data_as(ctypes.c_void_p), D.strides[0] // 4, nthreads, _ptr(first),
                                      _ptr(rb) if per_row else None)
    if bad < 0:
        raise ValueError(f"oracle_certify_rows failed with status {bad}")
    res = (int(bad), (None if first[0] < 0 else (int(first[0]), int(first[1]))))
    return res + (rb,) if per_row else res


def mcb_horton(n: int, src, dst, w):
    """MCB by Horton's algorithm: ``(weight, dim, cycles)`` with every kept cycle as an int32 array of
    edge indices (into src/dst/w), in the order the greedy kept them (non-decreasing weight)."""
    src, dst, w = _edges(src, dst, w)
    m = len(src)
    weight = np.zeros(1, np.int64)
    dim = np.zeros(1, np.int32)
    off = np.zeros(m + 2, np.int64)
    cap = max(1, 2 * (m + 1) * (n + 1))
    cap = min(cap, 1 << 26)
    edges = np.zeros(cap, np.int32)
    st = _load().oracle_mcb_horton(n, m, _ptr(src), _ptr(dst), _ptr(w), _ptr(weight), _ptr(dim), _ptr(off),
                                   _ptr(edges), cap)
    if st != 0:
        raise ValueError(f"oracle_mcb_horton failed with status {st}")
    f = int(dim[0])
    return int(weight[0]), f, [edges[off[i]:off[i + 1]].copy() for i in range(f)]


def mcb_depina(n: int, src, dst, w):
    """MCB by de Pina's Algorithm 2 (signed-graph search): ``(weight, dim, phase_weights)``."""
    src, dst, w = _edges(src, dst, w)
    m = len(src)
    weight = np.zeros(1, np.int64)
    dim = np.zeros(1, np.int32)
    wts = np.zeros(max(m, 1), np.int64)
    st = _load().oracle_mcb_depina(n, m, _ptr(src), _ptr(dst), _ptr(w), _ptr(weight), _ptr(dim), _ptr(wts))
    if st != 0:
        raise ValueError(f"oracle_mcb_depina failed with status {st}")
    return int(weight[0]), int(dim[0]), wts[:int(dim[0])].copy()


@dataclass
class Reduced:
    deg: np.ndarray      # distinct-neighbour degree (C3)
    term: np.ndarray     # 1 for V^r (C4, C5)
    end0: np.ndarray     # chain ends (vertex ids); V^r vertices: itself
    end1: np.ndarray
    d0: np.ndarray       # along-chain distance to end0 / end1 (C7)
    d1: np.ndarray
    chain: np.ndarray    # chain index, -1 for V^r vertices
    re_u: np.ndarray     # G^r edges before the parallel-edge rule (closed ears as a == a)
    re_v: np.ndarray
    re_w: np.ndarray
    n_reduced: int
    n_chains: int
    n_promoted: int


def reduce_graph(n: int, src, dst, w) -> Reduced:
    src, dst, w = _edges(src, dst, w)
    m = len(src)
    i32 = lambda: np.empty(n, dtype=np.int32)  # noqa: E731
    i64 = lambda: np.empty(n, dtype=np.int64)  # noqa: E731
    deg, term, end0, end1, chain = i32(), i32(), i32(), i32(), i32()
    d0, d1 = i64(), i64()
    cap = m + n + 1
    re_u = np.empty(cap, dtype=np.int32)
    re_v = np.empty(cap, dtype=np.int32)
    re_w = np.empty(cap, dtype=np.int64)
    counts = np.zeros(4, dtype=np.int64)
    st = _load().oracle_reduce(n, m, _ptr(src), _ptr(dst), _ptr(w), _ptr(deg), _ptr(term), _ptr(end0),
                               _ptr(end1), _ptr(d0), _ptr(d1), _ptr(chain), _ptr(re_u), _ptr(re_v),
                               _ptr(re_w), cap, _ptr(counts))
    if st != 0:
        raise ValueError(f"oracle_reduce failed with status {st}")
    k = int(counts[1])
    return Reduced(deg, term, end0, end1, d0, d1, chain, re_u[:k].copy(), re_v[:k].copy(), re_w[:k].copy(),
                   int(counts[0]), int(counts[2]), int(counts[3]))
