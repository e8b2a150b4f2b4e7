"""Time the expansion-kernel candidates of microbench/expand_lab.cu against the library's k_expand
(bit-exact check + CUDA-event timing on the same D and descriptors).

    python tools/expand_lab.py [cfg4] [variants...]
"""
import ctypes
import json
import os
import subprocess
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

LAB = os.path.join(ROOT, "microbench", "libexpandlab.so")


def build():
    src = os.path.join(ROOT, "microbench", "expand_lab.cu")
    if os.path.exists(LAB) and os.path.getmtime(LAB) > os.path.getmtime(src):
        return
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
                           "-shared", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include"), "-I",
                           os.path.join(ROOT, "paper_conf_ipps_duttackb17_b200", "csrc"), src, "-o", LAB])


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
    variants = [int(v) for v in sys.argv[2:]] or [9, 1, 6, 7, 8, 10]
    build()
    lab = ctypes.CDLL(LAB)
    lab.lab_expand.restype = ctypes.c_int
    lab.lab_expand.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32,
                               ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
    g = gg.config(cfg)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)
    out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()
    gb = (4.0 * g.n * g.n + 4.0 * plan.info().n_reduced ** 2 + 16.0 * g.n) / 1e9

    def timeit(fn, reps=5):
        fn()
        fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps

    ms = timeit(lambda: ea.expand_ears(plan, D, 0, g.n, out=out))
    print(json.dumps({"variant": 0, "name": "library k_expand", "ms": ms, "GBps": gb / ms * 1e3}), flush=True)
    # reference rows (sampled, to keep host memory small): every 97th row
    rows = torch.arange(0, g.n, 97, device="cuda")
    ref = out[rows].clone()
    for v in variants:
        out.fill_(-7)
        rc = lab.lab_expand(v, plan.handle, D.data_ptr(), D.stride(0), 0, g.n, out.data_ptr(), out.stride(0),
                            stream.cuda_stream)
        torch.cuda.synchronize()
        if rc != 0:
            print(json.dumps({"variant": v, "error": rc}), flush=True)
            continue
        ok = bool(torch.equal(out[rows], ref)) if v != 9 else None
        if v != 9 and ok:
            # full check of a contiguous block and the tail too
            blk = ea.expand_ears(plan, D, g.n - 777, g.n)
            ok = bool(torch.equal(out[g.n - 777:], blk))
        ms = timeit(lambda: lab.lab_expand(v, plan.handle, D.data_ptr(), D.stride(0), 0, g.n, out.data_ptr(),
                                           out.stride(0), stream.cuda_stream))
        print(json.dumps({"variant": v, "ms": ms, "GBps": gb / ms * 1e3, "exact": ok}), flush=True)


if __name__ == "__main__":
    main()
