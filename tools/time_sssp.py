"""Time Phase II routes on the paper's configs: apsp_reduced (int32 D) by per-source SSSP and by the
blocked FW, and apsp_full (the full N x N int32 output) with EAR_FLAG_SSSP against EAR_FLAG_BCC, CUDA
events on the current stream, median of `--reps`.  Set EAR_SSSP_STATS=1 for round / improvement counts;
EAR_SSSP16=0 times the round-1 int32 kernels instead of the u16 route.

usage: python tools/time_sssp.py cfg1 cfg2 cfg4 [--reps 5] [--out file.jsonl] [--no-full] [--no-fw]"""
import argparse
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402


def timed(fn, reps):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out")
    ap.add_argument("--no-full", action="store_true")
    ap.add_argument("--no-fw", action="store_true")
    a = ap.parse_args()
    for name in a.configs:
        g = gg.config(name)
        src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
        rec = {"config": name, "n": g.n}
        p = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_SSSP)
        rec["n_reduced"] = p.info().n_reduced
        D = ea.alloc_D(p)
        rec["reduced_sssp_ms"] = timed(lambda: ea.apsp_reduced(p, D), a.reps)
        if not a.no_fw:
            p2 = ea.ear_decompose(g.n, src, dst, w)
            D2 = ea.alloc_D(p2)
            rec["reduced_fw_ms"] = timed(lambda: ea.apsp_reduced(p2, D2), max(1, a.reps // 2))
            torch.cuda.synchronize()
            rec["D_equal"] = bool(torch.equal(D, D2))
            del D2, p2
        del D, p
        p3 = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC | ea.FLAG_SSSP)
        D3 = ea.alloc_D(p3)
        rec["reduced_bcc_sssp_ms"] = timed(lambda: ea.apsp_reduced(p3, D3), a.reps)
        del D3, p3
        torch.cuda.empty_cache()
        if not a.no_full:
            out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
            for fl, key in ((ea.FLAG_SSSP, "full_sssp_ms"), (ea.FLAG_BCC | ea.FLAG_SSSP, "full_bcc_sssp_ms"),
                            (ea.FLAG_BCC, "full_bcc_ms")):
                rec[key] = timed(lambda: ea.apsp_full(g.n, src, dst, w, out=out, flags=fl), a.reps)
            rec["full_sssp_entries_per_s"] = g.n * g.n / (rec["full_sssp_ms"] * 1e-3)
            rec["full_bcc_sssp_entries_per_s"] = g.n * g.n / (rec["full_bcc_sssp_ms"] * 1e-3)
            del out
            torch.cuda.empty_cache()
        print(json.dumps(rec), flush=True)
        if a.out:
            with open(a.out, "a") as f:
                f.write(json.dumps(rec) + "\n")


if __name__ == "__main__":
    main()
