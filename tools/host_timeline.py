"""Host-side timeline of one apsp_full-equivalent step (diagnostics): each stage synchronised and
timed on the host, to find time outside the kernels."""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
g = gg.config(cfg)
src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
for it in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ea.apsp_full(g.n, src, dst, w, out=out)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    plan = ea.ear_decompose(g.n, src, dst, w)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    D = ea.alloc_D(plan)
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    ea.apsp_reduced(plan, D)
    t3b = time.perf_counter()
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    ea.expand_ears(plan, D, 0, g.n, out=out)
    torch.cuda.synchronize()
    t5 = time.perf_counter()
    plan.destroy()
    del D
    torch.cuda.synchronize()
    t6 = time.perf_counter()
    print(f"iter {it}: apsp_full {1e3*(t1-t0):.1f} ms | decompose {1e3*(t2-t1):.1f} alloc {1e3*(t3-t2):.1f} "
          f"fw {1e3*(t4-t3):.1f} (enqueue {1e3*(t3b-t3):.1f}) expand {1e3*(t5-t4):.1f} destroy {1e3*(t6-t5):.1f}",
          flush=True)
ea.profile_enable(True)
ea.profile_reset()
t0 = time.perf_counter()
ea.apsp_full(g.n, src, dst, w, out=out)
torch.cuda.synchronize()
print(f"profiled apsp_full {1e3*(time.perf_counter()-t0):.1f} ms", ea.profile_read())
