"""Per-rank compute of the packed 16-bit row-block sharded FW for P = 1, 2, 4, 8 ranks, measured on ONE
B200 (apsp_reduced_rank_timing: one rank's kernels without the other ranks and without the NCCL
exchange; min-plus work is data-independent).  Reported beside the single-GPU FW on the same reduced
graph and the exchange volume per round (4 * 128 * Np bytes all-reduced), which is not measured here.

    python tools/rank_timing.py [cfg4] [--out profiles/...jsonl]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402


def timed(fn, reps=1):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="cfg4")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    g = gg.config(args.config)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w)
    nr = plan.info().n_reduced
    D = ea.alloc_D(plan)
    single = timed(lambda: ea.apsp_reduced(plan, D))
    del D
    torch.cuda.empty_cache()
    lines = [{"config": args.config, "n_reduced": nr, "what": "single-GPU packed FW (apsp_reduced, lookahead)",
              "ms": single}]
    for P in (1, 2, 4, 8):
        np_ = plan.info(P).n_reduced_padded
        ranks = sorted({0, P - 1})
        ms = {r: timed(lambda: ea.apsp_reduced_rank_timing(plan, P, r)) for r in ranks}
        rounds = np_ // 128
        rec = {"config": args.config, "P": P, "Np": np_, "rank_ms": {str(r): v for r, v in ms.items()},
               "max_rank_ms": max(ms.values()), "speedup_vs_single": single / max(ms.values()),
               "exchange_bytes_per_round": 4 * 128 * np_, "rounds": rounds,
               "exchange_bytes_total": 4 * 128 * np_ * rounds,
               "note": "per-rank compute only (no NCCL all-reduce of the pivot row block, no final gather)"}
        lines.append(rec)
    for r in lines:
        print(json.dumps(r), flush=True)
    if args.out:
        with open(args.out, "w") as fh:
            for r in lines:
                fh.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
