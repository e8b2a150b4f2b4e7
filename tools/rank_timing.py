"""Per-rank compute of the row-block sharded FW for P = 1, 2, 4, 8 ranks, measured on ONE B200
(apsp_reduced_rank_timing: one rank's kernels without the other ranks and without the exchange; min-plus
work is data-independent), packed u16x2 by default, int32 with --fw32 (cfg5's path: its reduced
diameter exceeds the 16-bit cap).  Reported beside the single-GPU FW on the same reduced graph and the
exchange volume per round (the pivot row block, received once per rank), not measured here.

    python tools/rank_timing.py [cfg4] [--fw32] [--out profiles/...jsonl]
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
    ap.add_argument("--fw32", action="store_true", help="int32 FW throughout (EAR_FLAG_FW32)")
    args = ap.parse_args()
    g = gg.config(args.config)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    fl = ea.FLAG_FW32 if args.fw32 else 0
    elem = "int32" if args.fw32 else "packed u16x2"
    esz = 4 if args.fw32 else 2
    plan = ea.ear_decompose(g.n, src, dst, w, flags=fl)
    nr = plan.info().n_reduced
    D = ea.alloc_D(plan)
    single = timed(lambda: ea.apsp_reduced(plan, D))
    del D
    torch.cuda.empty_cache()
    np1 = plan.info(1).n_reduced_padded
    peak = 148 * (64 if args.fw32 else 128) * 1.965e9
    rate = (np1 ** 3 / 2) / (single / 1e3)
    lines = [{"config": args.config, "n_reduced": nr, "Np": np1, "element": elem,
              "what": "single-GPU FW (apsp_reduced: init + dynamic tiles + lookahead)", "ms": single,
              "minplus_per_s": rate, "frac_of_peak_at_1965MHz": rate / peak}]
    for P in (1, 2, 4, 8):
        np_ = plan.info(P).n_reduced_padded
        ranks = sorted({0, P - 1})
        ms = {r: timed(lambda: ea.apsp_reduced_rank_timing(plan, P, r)) for r in ranks}
        rounds = np_ // 128
        rec = {"config": args.config, "P": P, "Np": np_, "rank_ms": {str(r): v for r, v in ms.items()},
               "max_rank_ms": max(ms.values()), "speedup_vs_single": single / max(ms.values()),
               "element": elem, "exchange_bytes_received_per_round": esz * 128 * np_ * (P - 1) // P, "rounds": rounds,
               "note": "per-rank compute only (no peer pushes of the pivot pieces, no final gather)"}
        lines.append(rec)
    for r in lines:
        print(json.dumps(r), flush=True)
    if args.out:
        with open(args.out, "w") as fh:
            for r in lines:
                fh.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
