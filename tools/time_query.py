"""Query mode throughput (S[s,t] for arbitrary pairs from D + descriptors, no N x N
matrix): 2^26 pairs per batch on cfg4 (or the given config), uniformly random and source-grouped
(1,024 random targets per random source), through ear_query_pairs.  Parity of the query path:
tests/test_parity_gpu.py.

    python tools/time_query.py [cfg4] [--pairs N] [--out profiles/...jsonl]
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
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    g = gg.config(args.config)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    gen = torch.Generator(device="cuda").manual_seed(7)
    P = args.pairs
    workloads = {
        "uniform": (torch.randint(0, g.n, (P,), device="cuda", dtype=torch.int32, generator=gen),
                    torch.randint(0, g.n, (P,), device="cuda", dtype=torch.int32, generator=gen)),
        "source_grouped_1024": (torch.randint(0, g.n, (P // 1024,), device="cuda", dtype=torch.int32,
                                              generator=gen).repeat_interleave(1024),
                                torch.randint(0, g.n, (P,), device="cuda", dtype=torch.int32, generator=gen)),
    }
    out = torch.empty(P, dtype=torch.int32, device="cuda")
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    lines = []
    for name, (s, t) in workloads.items():
        ea.query_pairs(plan, D, s, t, out=out)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.reps):
            ea.query_pairs(plan, D, s, t, out=out)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.reps
        rec = {"config": args.config, "workload": name, "pairs": P, "n": g.n, "n_reduced": plan.info().n_reduced,
               "D_bytes": int(D.numel()) * 4, "full_matrix_bytes": 4 * g.n * g.n, "ms_per_batch": ms,
               "pairs_per_s": P / (ms / 1e3), "hbm_copy_GBps": peaks.get("hbm_gbs")}
        print(json.dumps(rec), flush=True)
        lines.append(rec)
    if args.out:
        with open(args.out, "w") as f:
            for r in lines:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
