"""The sharded path with several REAL ranks: 2 and 4 processes (torch.distributed.run, gloo for the
host plumbing) share the one GPU, each owning its rows of D and its exchange window, mapped into the
other processes by CUDA IPC -- the same transport as across the GPUs of a node.  Every rank checks its
row block of S against the oracle (tests/mp_worker.py)."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("nranks", [2, 4])
def test_ranks_as_processes_on_one_gpu(nranks):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(nranks),
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()),
           os.path.join(ROOT, "tests", "mp_worker.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    out = r.stdout + r.stderr
    assert r.returncode == 0, out[-6000:]
    for k in range(nranks):
        assert f"MP-OK rank {k}" in r.stdout, out[-6000:]
