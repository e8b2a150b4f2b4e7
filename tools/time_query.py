#!/usr/bin/env python
"""Compact / query mode (UPDATE_DISTANCE per pair; memory P:137) measured:
Phases I-II once (D of G^r kept, O(N_r^2 + N) memory instead of N^2), then ear_query_pairs on batches
of uniformly random (s, t) pairs.  Each pair reads two 16-byte descriptors, two chain ids and four D
entries at random addresses, plus 12 streamed bytes (s, t, result).  The descriptors and chain ids
(20 bytes per vertex: 2 MB at cfg4, 4 MB at cfg5) stay in L2; D (3.6 / 14.4 GB) does not, so the DRAM
traffic is 4 random 32-byte D sectors + 12 bytes per pair, reported as dram_GBps against the copy
bandwidth (random sectors cannot reach the streaming rate).  Parity of the query path: tests/test_parity_gpu.py.

    python tools/time_query.py [cfg4|cfg5] [--pairs 67108864] [--reps 5]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="cfg4")
    ap.add_argument("--pairs", type=int, default=1 << 26)
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()

    g = gg.config(args.config)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    gen = torch.Generator(device="cuda").manual_seed(7)
    s = torch.randint(0, g.n, (args.pairs,), device="cuda", dtype=torch.int32, generator=gen)
    t = torch.randint(0, g.n, (args.pairs,), device="cuda", dtype=torch.int32, generator=gen)
    out = torch.empty(args.pairs, dtype=torch.int32, device="cuda")
    ea.query_pairs(plan, D, s, t, out=out)   # warm-up
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.reps):
        ea.query_pairs(plan, D, s, t, out=out)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.reps
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    dram_bytes = (4 * 32 + 12) * args.pairs
    print(json.dumps({"config": args.config, "n": g.n, "n_reduced": plan.info().n_reduced,
                      "D_bytes": int(D.numel()) * 4, "full_matrix_bytes": 4 * g.n * g.n,
                      "pairs": args.pairs, "ms_per_batch": ms, "pairs_per_s": args.pairs / (ms / 1e3),
                      "dram_GBps": dram_bytes / (ms / 1e3) / 1e9, "hbm_copy_GBps": peaks["hbm_gbs"]}))


if __name__ == "__main__":
    main()
