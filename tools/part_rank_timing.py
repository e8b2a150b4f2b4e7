#!/usr/bin/env python
"""Per-rank work of the region route at P ranks, measured on one B200: rank r of P runs apsp_full for its
row block only (ea.row_block), which is everything that rank does -- the region route has no exchange
(every rank computes the D rows its Phase III stages: the regions of its rows' chain ends, then expands
its rows).  Device time per call (CUDA events, median of 5 after a warm-up) for every rank of
P = 1, 2, 4, 8; the job's time at P is the slowest rank's.

    python tools/part_rank_timing.py [cfg4] [--out file.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="cfg4")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    g = gg.config(args.config)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
    base = None
    for P in (1, 2, 4, 8):
        ranks = []
        for r in range(P):
            r0, r1 = ea.row_block(g.n, P, r)
            o = out[: r1 - r0]
            ea.apsp_full(g.n, src, dst, w, out=o, row_begin=r0, row_end=r1, flags=ea.FLAG_PART)
            ts = []
            for _ in range(5):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                ea.apsp_full(g.n, src, dst, w, out=o, row_begin=r0, row_end=r1, flags=ea.FLAG_PART)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ranks.append(statistics.median(ts))
        job = max(ranks)
        base = base or job
        rec = {"config": args.config, "P": P, "rank_ms": ranks, "job_ms": job, "speedup": base / job,
               "entries_per_s": g.n * g.n / (job / 1e3),
               "note": "each rank's whole apsp_full (no exchange on the region route), measured alone on one B200"}
        line = json.dumps(rec)
        print(line, flush=True)
        if args.out:
            with open(args.out, "a") as f:
                f.write(line + "\n")


if __name__ == "__main__":
    main()
