"""Small end-to-end runs for compute-sanitizer (memcheck / racecheck / synccheck): every kernel of the
library on graphs small enough for the instrumented run -- packed and int32 FW (single, emulated
sharding with the owner-side phase 2 and lookahead, and a one-rank communicator: window pushes, flags,
the pull gather), blocks with a re-reduced piece (u16 compose route), SSSP, expansion (pair-major on
aligned rows, row-group on unaligned rows), query mode, Phase I with pure cycles, the MCB (trees,
candidates, phases, cycle expansion), the host-buffer entry points (two async jobs in flight, pinned
and pageable inputs)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402

dev = lambda a: torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()  # noqa: E731
from tests.test_bcc_gpu import decorated_grid  # noqa: E402  (a big block that is reduced again)

for g in [gg.corner_cases(5, n_target=300), gg.torus(12, 12, 150, seed=1), gg.cycle(40, seed=2),
          decorated_grid(18, 0.35, 1)]:
    for flags in (0, ea.FLAG_SSSP, ea.FLAG_BCC, ea.FLAG_FW32):
        out = ea.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags)
    plan = ea.ear_decompose(g.n, dev(g.src), dev(g.dst), dev(g.w))
    D = ea.apsp_reduced_emulated(plan, 2)
    D3 = ea.apsp_reduced_emulated(plan, 3)   # packed sharded FW: owner-side phase 2, lookahead
    ea.apsp_reduced_rank_timing(plan, 2, 1)
    big = torch.zeros((g.n, g.n + 3), dtype=torch.int32, device="cuda")
    ea.expand_ears(plan, D, 0, g.n, out=big[:, 1:1 + g.n])
    s = dev(np.arange(g.n)); t = dev(np.arange(g.n)[::-1].copy())
    ea.query_pairs(plan, D, s, t)
    aligned = torch.zeros((g.n, (g.n + 3) // 4 * 4), dtype=torch.int32, device="cuda")
    ea.expand_ears(plan, D, 0, g.n, out=aligned[:, :g.n])          # pair-major kernel (aligned rows)
    mc = ea.mcb(g.n, dev(g.src), dev(g.dst), dev(g.w))
    for i in range(min(3, mc.info()["dim"])):
        mc.cycle(i)
    mc.destroy()
comm = ea.Comm.single()   # the sharded schedule through its window: pushes, flags, pull gather
for g in [gg.corner_cases(5, n_target=300), gg.torus(12, 12, 150, seed=1)]:
    for flags in (0, ea.FLAG_FW32, ea.FLAG_BCC):
        ea.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), flags=flags, comm=comm)
comm.destroy()
# host-buffer entry points, two async jobs in flight (mapped-pinned readbacks, kernel memsets)
g = gg.corner_cases(5, n_target=300)
hs, hd, hw = (torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).pin_memory() for a in (g.src, g.dst, g.w))
outs = [torch.empty((g.n, g.n), dtype=torch.int32, pin_memory=True) for _ in range(2)]
j0 = ea.apsp_full_host_async(g.n, hs, hd, hw, out=outs[0], flags=ea.FLAG_BCC)
j1 = ea.apsp_full_host_async(g.n, hs, hd, hw, out=outs[1], flags=ea.FLAG_BCC)
j0.wait(); j1.wait()
ea.apsp_full_host(g.n, g.src, g.dst, g.w)   # pageable inputs: the copy-in branch
torch.cuda.synchronize()
print("sanitize run ok")
