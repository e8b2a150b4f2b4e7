"""Raw device -> host copy bandwidth into pinned host memory (the e2e roofline of the host-buffer API):
40 GB in 256 MB chunks on one stream, into (a) one torch pinned tensor, (b) a second one; repeated."""
import json
import time

import torch

n = 10_000_000_000   # int32 entries = 40 GB
chunk = 64 << 20     # entries (256 MB)
src = torch.empty(chunk, dtype=torch.int32, device="cuda").fill_(1)
res = []
bufs = [torch.empty(n, dtype=torch.int32, pin_memory=True) for _ in range(2)]
for rep in range(3):
    for b, h in enumerate(bufs):
        torch.cuda.synchronize()
        t = time.perf_counter()
        for off in range(0, n, chunk):
            m = min(chunk, n - off)
            h[off:off + m].copy_(src[:m], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
        res.append({"rep": rep, "buf": b, "GBps": 4 * n / dt / 1e9})
print(json.dumps(res))
