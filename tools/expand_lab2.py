"""Round-2 expansion lab: time microbench/expand_lab2.cu variants of k_expand against the library kernel
on cfg4's D (Phase II by blocks, as the bench) -- full-output bit-exact comparison, CUDA-event timing.

    python tools/expand_lab2.py [cfg4] [variants...]
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

LAB = os.path.join(ROOT, "microbench", "libexpandlab2.so")
NAMES = {1: "prefetch.L2 exact addresses, 1 chunk ahead", 2: "prefetch.L2 exact, 2 ahead", 3: "evict_last gathers",
         4: "u16 D gathers", 5: "u16 D + prefetch 1 ahead", 6: "prefetch 1 ahead + evict_last gathers",
         7: "u16 D + prefetch 2 ahead", 10: "baseline (copy of the library kernel)"}


def build():
    src = os.path.join(ROOT, "microbench", "expand_lab2.cu")
    if os.path.exists(LAB) and os.path.getmtime(LAB) > os.path.getmtime(src):
        return
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
                           "-shared", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include"), "-I",
                           os.path.join(ROOT, "paper_conf_ipps_duttackb17_b200", "csrc"), src, "-o", LAB])


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
    variants = [int(v) for v in sys.argv[2:]] or [10, 1, 2, 3, 4, 5, 6, 7]
    build()
    lab = ctypes.CDLL(LAB)
    lab.lab2_expand.restype = ctypes.c_int
    lab.lab2_expand.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32,
                                ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p]
    g = gg.config(cfg)
    src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
    plan = ea.ear_decompose(g.n, src, dst, w, flags=ea.FLAG_BCC)
    D = ea.alloc_D(plan)
    ea.apsp_reduced(plan, D)
    Dc = torch.clamp(D, max=65535)
    D16 = (Dc - 65536 * (Dc >= 32768).to(torch.int32)).to(torch.int16).contiguous()
    del Dc
    ref = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
    out = torch.empty_like(ref)
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

    ms = timeit(lambda: ea.expand_ears(plan, D, 0, g.n, out=ref))
    print(json.dumps({"variant": 0, "name": "library k_expand", "ms": ms, "GBps": gb / ms * 1e3}), flush=True)
    for v in variants:
        Dv, ldd = (D16, D16.stride(0)) if v in (4, 5, 7) else (D, D.stride(0))
        call = lambda: lab.lab2_expand(v, plan.handle, Dv.data_ptr(), ldd, 0, g.n, out.data_ptr(),  # noqa: E731
                                       out.stride(0), stream.cuda_stream)
        out.fill_(-7)
        rc = call()
        torch.cuda.synchronize()
        if rc != 0:
            print(json.dumps({"variant": v, "error": rc}), flush=True)
            continue
        ok = bool(torch.equal(out, ref))
        ms = timeit(call)
        print(json.dumps({"variant": v, "name": NAMES.get(v), "ms": ms, "GBps": gb / ms * 1e3, "exact": ok}), flush=True)


if __name__ == "__main__":
    main()
