"""The communicator path on one GPU with ONE rank: the sharded schedule with its exchange window
(pieces pushed into the stage buffer, flags raised and awaited every round, the final D gathered
from the window region) and the sharded SSSP Phase II, then the expansion -- bit-exact against the
oracle; default flags run the packed sharded FW, FLAG_FW32 the int32 one, FLAG_BCC shards the largest
biconnected piece.  Several ranks as separate processes: tests/test_multiprocess_gpu.py."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def test_one_rank_comm_path():
    import paper_conf_ipps_duttackb17_b200 as ea
    from tests.test_bcc_gpu import decorated_grid   # a big piece that FLAG_BCC reduces again
    comm = ea.Comm.single()
    try:
        for g in [gg.config("cfg1"), gg.corner_cases(12, n_target=500), decorated_grid(24, 0.3, 0)]:
            ref = oracle.apsp(g.n, g.src, g.dst, g.w)
            for flags in (0, ea.FLAG_SSSP, ea.FLAG_BCC, ea.FLAG_FW32, ea.FLAG_BCC | ea.FLAG_FW32,
                          ea.FLAG_BCC | ea.FLAG_SSSP):
                out = ea.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), comm=comm, flags=flags)
                torch.cuda.synchronize()
                assert np.array_equal(out.cpu().numpy(), ref), f"comm path mismatch (flags={flags})"
            host = ea.apsp_full_host(g.n, g.src, g.dst, g.w, comm=comm)
            assert np.array_equal(host.numpy(), ref), "comm host path mismatch"
    finally:
        comm.destroy()
