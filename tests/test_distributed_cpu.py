"""Multi-process host logic of the N>1 path on CPU (gloo, world_size 2, 127.0.0.1).

The GPU-side sharded schedule runs for real with 2 and 4 ranks as separate processes sharing one GPU
(tests/test_multiprocess_gpu.py) and emulated in one process (test_parity_gpu.py); here the host
plumbing: the communicator's all-gather callback over torch.distributed (the IPC-handle exchange
path), row blocks and the max-over-ranks timing rule.
"""
import json
import os
import socket
import subprocess
import sys

import pytest
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from paper_conf_ipps_duttackb17_b200 import ear_apsp
    comm = ear_apsp.Comm.from_torch_distributed()     # ear_comm_init agrees on the layout via the callback
    uid = (comm.nranks, comm.rank)
    comm.destroy()
    blocks = [ear_apsp.row_block(100000, world, r) for r in range(world)]
    mx = bench.max_over_ranks(float(rank + 1) * 1.5, world, torch.device("cpu"))
    q.put((rank, uid, blocks, mx))
    dist.destroy_process_group()


def test_two_rank_host_logic():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, uid0, b0, m0), (r1, uid1, b1, m1) = res
    assert uid0 == (2, 0) and uid1 == (2, 1)
    assert b0 == b1 == [(0, 50000), (50000, 100000)]
    assert m0 == m1 == 3.0                                 # max over ranks, as the bench times


def test_reference_arm_under_torchrun_prints_one_line():
    port = free_port()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "bench.py"),
           "--impl", "reference", "--gpus", "2", "--config", "cfg1", "--steps", "1", "--warmup", "0"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["n"] == 2000
