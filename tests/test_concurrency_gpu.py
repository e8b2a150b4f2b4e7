"""Concurrent FW calls on one device (the header's "distinct plans are thread-safe" contract).

Two host threads, each on its own stream, run the packed FW with its lookahead (the pivot chain of
round k+1 on a side stream, ordered after round k's cross tiles by an event) on a cfg2-size reduced
graph (62 tiles) at the same time.  EAR_DEBUG_RACE_US makes the library sleep between recording the
cross-tile event and the side stream's wait on it -- the window in which a shared (per-device) event or
side stream would let one call's pivot chain wait on the OTHER call's work and read tiles still being
updated.  Every result is compared with the CPU oracle (P:109 definition of S), bit for bit.
Round 1's library (per-device statics) fails this test; per-call lookahead state passes it.
"""
import threading

import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_duttackb17_b200 import graphgen as gg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pkg():
    import paper_conf_ipps_duttackb17_b200 as p
    p.lib()
    return p


@pytest.fixture(scope="module")
def cfg2_ref():
    g = gg.config("cfg2")
    return g, oracle.apsp(g.n, g.src, g.dst, g.w)


def dev(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.int32)).cuda()


@pytest.mark.parametrize("flags", ["fw", "fw32"])
def test_concurrent_fw_lookahead_race(pkg, cfg2_ref, monkeypatch, flags):
    monkeypatch.setenv("EAR_DEBUG_RACE_US", "300")
    g, ref = cfg2_ref
    fl = pkg.FLAG_FW32 if flags == "fw32" else 0
    src, dst, w = dev(g.src), dev(g.dst), dev(g.w)
    iters = 4
    bad = []
    errs = []
    barrier = threading.Barrier(2)

    def work(k):
        try:
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                out = torch.empty((g.n, g.n), dtype=torch.int32, device="cuda")
                barrier.wait()
                for it in range(iters):
                    pkg.apsp_full(g.n, src, dst, w, out=out, flags=fl, stream=st)
                    st.synchronize()
                    nb = int((out.cpu().numpy() != ref).sum())
                    if nb:
                        bad.append((k, it, nb))
        except Exception as e:  # noqa: BLE001  (reported below)
            errs.append(e)

    ts = [threading.Thread(target=work, args=(k,)) for k in range(2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not errs, errs
    assert not bad, f"(thread, iteration, mismatching entries): {bad}"
