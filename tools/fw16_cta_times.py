"""Per-CTA start/end times of one rest-of-round k_fw_tiles16 launch (EAR_FW16_DBG=N), summarised:
how long each SM slot is occupied relative to the launch."""
import collections
import os
import subprocess
import sys

N = sys.argv[1] if len(sys.argv) > 1 else "99"
env = dict(os.environ, EAR_FW16_DBG=N)
r = subprocess.run([sys.executable, "tools/sweep_fw16.py", "--one", "cfg4"], env=env, capture_output=True, text=True)
rows = [l.split()[1:] for l in r.stderr.splitlines() if l.startswith("FW16DBG ") and not l.startswith("FW16DBG launch")]
head = [l for l in r.stderr.splitlines() if l.startswith("FW16DBG launch")]
print(head[0] if head else r.stderr[-2000:])
t = [(int(b), int(s), int(e), int(sm)) for b, s, e, sm in rows]
end = max(e for _, _, e, _ in t)
starts = sorted(s for _, s, _, _ in t)
ends = sorted(e for _, _, e, _ in t)
print(f"launch span {end/1e3:.1f} us; CTA starts: min {starts[0]/1e3:.1f} median {starts[len(starts)//2]/1e3:.1f} "
      f"max {starts[-1]/1e3:.1f} us; ends: min {ends[0]/1e3:.1f} median {ends[len(ends)//2]/1e3:.1f} max {ends[-1]/1e3:.1f} us")
occ = sum(e - s for _, s, e, _ in t) / (end * 148)
print(f"average resident CTAs per SM over the launch: {occ:.2f}")
per_sm = collections.Counter(sm for *_, sm in t)
print("CTAs per SM histogram:", collections.Counter(per_sm.values()))
# start-time clusters
buckets = collections.Counter(int(s // 50000) for s in starts)
print("starts per 50 us bucket:", sorted(buckets.items())[:20])
