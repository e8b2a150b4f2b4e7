"""Full N x N verification at the north-star sizes (S defined at P:109; SURVEY 8.c pin P4).

Every entry of cfg4's matrix (100k vertices, 40 GB) in the bench's launch configuration (apsp_full,
Phase II by regions, EAR_FLAG_PART), by biconnected pieces solved by per-source SSSP and by the blocked-FW route, and -- with EAR_VERIFY_CFG5=1 -- every entry of cfg5's (200k vertices,
160 GB: Phase II once, the expansion in row blocks) is checked by the oracle's Bellman certificate
(oracle.certify_rows: the definition of S restated as a fixed point whose only solution is S) on the
host's cores, streaming row blocks device -> pinned host while the previous block is being certified.
EAR_VERIFY_OUT=<path> appends a JSON summary line (entries, violations, timings, threads).
"""
import json
import os
import threading
import time
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def certify_stream(g, produce, block_rows):
    """produce(r0, r1) -> device int32 tensor of rows [r0, r1) (may be a view); returns the summary."""
    bufs = [torch.empty((block_rows, g.n), dtype=torch.int32, pin_memory=True) for _ in range(2)]
    pool = ThreadPoolExecutor(max_workers=1)
    pending, violations, first = [None, None], 0, None
    t_copy = t_cert = 0.0
    lock = threading.Lock()

    def cert(buf, r0, r1):
        nonlocal violations, first, t_cert
        t = time.perf_counter()
        bad, fb = oracle.certify_rows(g.n, g.src, g.dst, g.w, np.arange(r0, r1), buf[: r1 - r0].numpy())
        with lock:
            t_cert += time.perf_counter() - t
            violations += bad
            if fb is not None and first is None:
                first = (r0 + fb[0], fb[1])

    t0 = time.perf_counter()
    for i, r0 in enumerate(range(0, g.n, block_rows)):
        r1 = min(g.n, r0 + block_rows)
        b = i & 1
        if pending[b] is not None:
            pending[b].result()           # the buffer is free again
        blk = produce(r0, r1)
        t = time.perf_counter()
        bufs[b][: r1 - r0].copy_(blk)     # device -> pinned host (synchronous)
        t_copy += time.perf_counter() - t
        pending[b] = pool.submit(cert, bufs[b], r0, r1)
    for p in pending:
        if p is not None:
            p.result()
    pool.shutdown()
    return {"entries": g.n * g.n, "violations": violations, "first_violation": first,
            "copy_s": t_copy, "certify_cpu_s": t_cert, "wall_s": time.perf_counter() - t0,
            "threads": oracle.num_threads(), "block_rows": block_rows}


def report(summary):
    path = os.environ.get("EAR_VERIFY_OUT")
    if path:
        with open(path, "a") as f:
            f.write(json.dumps(summary) + "\n")
    print(json.dumps(summary))


ROUTES = {"part": ("FLAG_PART (regions; bench default)", lambda ea: ea.FLAG_PART | ea.FLAG_BCC | ea.FLAG_SSSP),
          "bcc_sssp": ("FLAG_BCC | FLAG_SSSP", lambda ea: ea.FLAG_BCC | ea.FLAG_SSSP),
          "bcc_fw": ("FLAG_BCC (pieces by the blocked FW)", lambda ea: ea.FLAG_BCC)}


@pytest.mark.parametrize("route", list(ROUTES))
def test_cfg4_full_matrix_certified(route):
    import paper_conf_ipps_duttackb17_b200 as ea
    g = gg.config("cfg4")
    name, fl = ROUTES[route]
    flags = fl(ea)
    out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
    src, dst, w = dev(g.src), dev(g.dst), dev(g.w)
    ea.apsp_full(g.n, src, dst, w, out=out, flags=flags)   # warm-up
    torch.cuda.synchronize()
    t = time.perf_counter()
    ea.apsp_full(g.n, src, dst, w, out=out, flags=flags)
    torch.cuda.synchronize()
    gpu_s = time.perf_counter() - t
    s = certify_stream(g, lambda r0, r1: out[r0:r1], 5000)
    s.update({"config": "cfg4", "n": g.n, "m": g.m, "path": f"apsp_full {name}, one call", "gpu_apsp_full_s": gpu_s})
    del out
    torch.cuda.empty_cache()
    report(s)
    assert s["violations"] == 0, s


@pytest.mark.skipif(os.environ.get("EAR_VERIFY_CFG5") != "1", reason="cfg5 full check: EAR_VERIFY_CFG5=1 (~3 min)")
@pytest.mark.parametrize("route", list(ROUTES))
def test_cfg5_full_matrix_certified(route):
    import paper_conf_ipps_duttackb17_b200 as ea
    g = gg.config("cfg5")
    name, fl = ROUTES[route]
    src, dst, w = dev(g.src), dev(g.dst), dev(g.w)
    plan = ea.ear_decompose(g.n, src, dst, w, flags=fl(ea))
    D = ea.alloc_D(plan)
    t = time.perf_counter()
    ea.apsp_reduced(plan, D)
    torch.cuda.synchronize()
    phase2_s = time.perf_counter() - t
    rows = 10000
    out = torch.empty((rows, g.n), dtype=torch.int32, device="cuda")
    t_exp = [0.0]

    def produce(r0, r1):
        t1 = time.perf_counter()
        ea.expand_ears(plan, D, r0, r1, out=out)
        torch.cuda.synchronize()
        t_exp[0] += time.perf_counter() - t1
        return out[: r1 - r0]

    s = certify_stream(g, produce, rows)
    s.update({"config": "cfg5", "n": g.n, "m": g.m, "n_reduced": plan.info().n_reduced,
              "path": f"ear_decompose {name} + apsp_reduced once + expand_ears by 10,000-row blocks (one B200)",
              "gpu_phase2_s": phase2_s, "gpu_expand_s": t_exp[0]})
    plan.destroy()
    del D, out
    torch.cuda.empty_cache()
    report(s)
    assert s["violations"] == 0, s


@pytest.mark.skipif(os.environ.get("EAR_VERIFY_CFG5") != "1", reason="cfg5 full check: EAR_VERIFY_CFG5=1 (~3 min)")
def test_cfg5_one_call_one_gpu_certified():
    """The north-star size in ONE apsp_full call on ONE B200: cfg5's whole 200k x 200k int32 matrix (160 GB)
    resident in HBM beside the region route's working set, timed, then every entry certified."""
    import paper_conf_ipps_duttackb17_b200 as ea
    g = gg.config("cfg5")
    free, total = torch.cuda.mem_get_info()
    need = 4 * g.n * g.n
    if free < need + 12 * 2**30:
        pytest.skip(f"{free / 2**30:.0f} GiB free of {total / 2**30:.0f}: the 149 GiB output does not fit beside the rest")
    src, dst, w = dev(g.src), dev(g.dst), dev(g.w)
    out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
    fl = ea.FLAG_PART | ea.FLAG_BCC | ea.FLAG_SSSP
    ea.apsp_full(g.n, src, dst, w, out=out, flags=fl)   # warm-up (module load, pools)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ea.apsp_full(g.n, src, dst, w, out=out, flags=fl)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    s = certify_stream(g, lambda r0, r1: out[r0:r1], 10000)
    s.update({"config": "cfg5", "n": g.n, "m": g.m, "path": "apsp_full FLAG_PART, ONE call, 160 GB output on one B200",
              "gpu_apsp_full_ms": ms, "entries_per_s": g.n * g.n / (ms / 1e3),
              "hbm_free_gib_before": free / 2**30, "hbm_total_gib": total / 2**30})
    del out
    torch.cuda.empty_cache()
    report(s)
    assert s["violations"] == 0, s
