"""The NCCL path on one GPU: a communicator of ONE rank (torch.distributed nccl process group, NCCL
unique id from the library) runs the sharded schedule with its real ncclAllReduce(MIN) of the pivot
row block every FW round and of the final D (and the sharded SSSP Phase II), then the expansion --
bit-exact against the oracle; with the default flags the packed 16-bit sharded FW runs, FLAG_FW32 the
int32 one, FLAG_BCC shards the largest biconnected piece.  (The multi-rank schedule
itself is checked on one GPU by test_parity_gpu.py::test_sharded_schedule_emulated.)"""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r'''
import os, sys, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, ROOT)
import oracle, paper_conf_ipps_duttackb17_b200 as ea
from paper_conf_ipps_duttackb17_b200 import graphgen as gg
torch.cuda.set_device(0)
dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
comm = ea.Comm.from_torch_distributed()
dev = lambda a: torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()
from tests.test_bcc_gpu import decorated_grid   # a big piece that FLAG_BCC reduces again
for g in [gg.config("cfg1"), gg.corner_cases(12, n_target=500), decorated_grid(24, 0.3, 0)]:
    ref = oracle.apsp(g.n, g.src, g.dst, g.w)
    for flags in (0, ea.FLAG_SSSP, ea.FLAG_BCC, ea.FLAG_FW32, ea.FLAG_BCC | ea.FLAG_FW32):
        out = ea.apsp_full(g.n, dev(g.src), dev(g.dst), dev(g.w), comm=comm, flags=flags)
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy(), ref), f"nccl path mismatch (flags={flags})"
    host = ea.apsp_full_host(g.n, g.src, g.dst, g.w, comm=comm)
    assert np.array_equal(host.numpy(), ref), "nccl host path mismatch"
comm.destroy()
dist.destroy_process_group()
print("NCCL-PATH-OK")
'''


def test_one_rank_nccl_path():
    s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    r = subprocess.run([sys.executable, "-c", SCRIPT.replace("ROOT", repr(ROOT))], env=env, capture_output=True,
                       text=True, timeout=600)
    assert "NCCL-PATH-OK" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]
