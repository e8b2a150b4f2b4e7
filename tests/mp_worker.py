"""Worker of tests/test_multiprocess_gpu.py, launched with torch.distributed.run: every rank is a
separate process and ALL ranks share cuda:0 (one GPU reachable here).  The communicator's windows are
mapped between the processes by CUDA IPC exactly as between the GPUs of a node, so the sharded FW's
per-round pushes and flags, the pivot-tile push, the range-check agreement and the final gather run for
real across processes.  Each rank checks its caller row block of S against the CPU oracle, bit for bit
(P:109 defines S), for every Phase II mode; prints MP-OK on success."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_ipps_duttackb17_b200 as ea  # noqa: E402
from paper_conf_ipps_duttackb17_b200 import graphgen as gg  # noqa: E402
from tests.test_bcc_gpu import decorated_grid  # noqa: E402


def heavy_torus():
    """A torus whose weights are scaled so that the reduced diameter exceeds the packed FW's 16-bit
    cap: the sharded packed schedule must detect it on some rank and every rank must fall back."""
    g = gg.torus(24, 24, 400, seed=3)
    return gg.Graph(g.n, g.src, g.dst, (g.w.astype(np.int64) * 60).astype(np.int32))


def main():
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    comm = ea.Comm.from_torch_distributed()
    dev = lambda a: torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()  # noqa: E731
    graphs = [("cfg1", gg.config("cfg1")), ("multi-tile", gg.corner_cases(1003, n_target=1311)),
              ("decorated", decorated_grid(24, 0.3, 0)), ("heavy-torus", heavy_torus())]
    for name, g in graphs:
        r0, r1 = ea.row_block(g.n, world, rank)
        ref = oracle.apsp_rows(g.n, g.src, g.dst, g.w, np.arange(r0, r1))
        for flags in (0, ea.FLAG_FW32, ea.FLAG_BCC, ea.FLAG_SSSP, ea.FLAG_BCC | ea.FLAG_FW32,
                      ea.FLAG_BCC | ea.FLAG_SSSP, ea.FLAG_PART | ea.FLAG_BCC | ea.FLAG_SSSP):
            out = ea.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), row_begin=r0, row_end=r1, flags=flags,
                               comm=comm)
            torch.cuda.synchronize()
            bad = int((out.cpu().numpy() != ref).sum())
            assert bad == 0, f"rank {rank}/{world}: {name} flags={flags}: {bad} mismatches"
        print(f"rank {rank}: {name} ok", flush=True)
    comm.destroy()
    dist.destroy_process_group()
    print(f"MP-OK rank {rank}", flush=True)


if __name__ == "__main__":
    main()
