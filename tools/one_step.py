"""One apsp_full call on a config (for ncu launch lists): python tools/one_step.py cfg4 [part|bcc_sssp|bcc|sssp|fw]"""
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg4"
route = sys.argv[2] if len(sys.argv) > 2 else "bcc_sssp"
flags = {"bcc_sssp": ea.FLAG_BCC | ea.FLAG_SSSP, "bcc": ea.FLAG_BCC, "sssp": ea.FLAG_SSSP, "fw": 0,
         "part": ea.FLAG_PART | ea.FLAG_BCC | ea.FLAG_SSSP}[route]
g = gg.config(cfg)
src, dst, w = (torch.as_tensor(x).cuda() for x in (g.src, g.dst, g.w))
out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
for i in range(int(sys.argv[3]) if len(sys.argv) > 3 else 1):
    torch.cuda.synchronize()
    t = time.perf_counter()
    ea.apsp_full(g.n, src, dst, w, out=out, flags=flags)
    torch.cuda.synchronize()
    print(f"step {i}: {(time.perf_counter() - t) * 1e3:.1f} ms wall", flush=True)
