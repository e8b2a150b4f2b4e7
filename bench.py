#!/usr/bin/env python
"""Benchmark: full APSP distance entries/s of the ear-reduced B200 path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config cfg4] [--impl ours|reference]

One step = one pass of the whole hot path over the workload: apsp_full =
Reduce(G) chain contraction -> Phase II on G^r -> ear expansion of this rank's rows of the N x N int32
matrix, graph already resident in HBM.  By default (--phase2 part) Phase II cuts G^r into connected
regions of <= 256 vertices and composes every row of D through the region boundaries (sec. 2.2's
composition through articulation points, with boundary sets as separators):
region distances by one CTA each, a blocked FW on the boundary graph, two min-plus products with a
region boundary as the inner dimension.  --phase2 bcc_sssp splits G^r into its biconnected pieces
(P:119-131), reduces every big piece again and solves it by the paper's own per-source SSSP
(P:101); --phase2 bcc solves the pieces by the blocked min-plus FW, --phase2 fw runs one FW over all of
G^r, --phase2 sssp the SSSP over all of G^r.  For N > 1 GPUs (torchrun, one process per GPU) every rank
computes D (a few ms) and expands its own row block; the total work is fixed (strong scaling).  Timing:
W untimed warm-up steps, then exactly K steps between barrier + synchronize, CUDA events on the
launching stream, max over ranks.  The output (40 GB) is far larger than L2, so no flush is needed
between steps.

Rank 0 prints one JSON line.  Extra keys: roofline (the kernel with the largest share of the step: the
expansion k_expand_pairs, HBM bound, on the region route; else the Phase II kernel), roofline_phase2 /
roofline_expand (the other one), cpu_baseline (the CPU oracle on a bounded sample,
rank 0 at N = 1 only), e2e (the same metric through the host-buffer C-ABI calls with every step's
H2D edge upload and D2H copy of the output rows: by default K jobs of apsp_full_host_async pipelined one
deep -- job i+1's Phases I-II overlap job i's expansion and row copies -- into two pinned output buffers;
--e2e-mode sync times the synchronous apsp_full_host), clocks, gpu_launches, phases_ms.

--impl reference runs the CPU oracle (Dijkstra from every source of a bounded sample of sources on
all host cores) as the reference arm; under torchrun only rank 0 runs it.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import psutil

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "full APSP distance entries/sec at 1/2/4/8 B200; min-plus GOPS & HBM GB/s"
UNIT = "entries/s"
SM_COUNT = 148
ALU_LANES_PER_SM = 64          # VIADDMNMX issue rate measured by microbench/minplus_peak.cu
WORKLOADS = {
    "cfg1": "cfg1: 33x33 torus + 911 degree-two subdivisions (N=2,000, 45.6% degree two)",
    "cfg2": "cfg2: 89x89 open grid subdivided to N=20,000 (road-like, 60% degree two)",
    "cfg3_f0": "cfg3 f=0%: 200x250 torus, N=50,000 (no degree-two vertices)",
    "cfg3_f20": "cfg3 f=20%: 200x200 torus + 10,000 subdivisions, N=50,000",
    "cfg3_f40": "cfg3 f=40%: 150x200 torus + 20,000 subdivisions, N=50,000",
    "cfg3_f60": "cfg3 f=60%: 100x200 torus + 30,000 subdivisions, N=50,000",
    "cfg3_f80": "cfg3 f=80%: 100x100 torus + 40,000 subdivisions, N=50,000",
    "cfg4": "cfg4: power-grid-like (28,500-point 3-NN geometric graph + 5% pendants, chained components, "
            "degree-two subdivisions), N=100,000, ~30k reduced vertices, 40 GB int32 distance matrix",
    "cfg5": "cfg5: power-grid-like, N=200,000, ~60k reduced vertices, 160 GB int32 distance matrix",
}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def max_over_ranks(x: float, world: int, device) -> float:
    """Max of a per-rank time over all ranks (the contract's multi-GPU timing rule)."""
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# ------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ["clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, gpu_id: str):
        self.gpu_id, self.lines, self.proc = gpu_id, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", self.gpu_id, "--query-gpu=" + ",".join(self.FIELDS),
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception as e:  # pragma: no cover
            log("clock sampler unavailable:", e)
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, pw, reasons = [], [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) != len(self.FIELDS):
                continue
            try:
                sm.append(float(p[0])); mx.append(float(p[1])); pw.append(float(p[2]))
            except ValueError:
                continue
            for nm, v in zip(names, p[3:]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "power_w_max": max(pw) if pw else None, "reasons": sorted(reasons), "samples": len(sm)}


def gpu_id_for(dev_index: int) -> str:
    import torch
    try:
        u = str(torch.cuda.get_device_properties(dev_index).uuid)
        return u if u.startswith("GPU-") else "GPU-" + u
    except Exception:
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        return vis.split(",")[dev_index] if vis else str(dev_index)


def measured_peaks() -> dict:
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def ncu_traffic(kernel_key: str, workload: str):
    """Per-launch DRAM bytes of a kernel from the committed ncu --set full summary (or None)."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(path))
        e = d.get(workload, {}).get(kernel_key)
        return None if e is None else float(e["dram_bytes_per_launch"])
    except Exception:
        return None


# ------------------------------------------------------------------------------------ CPU oracle
def oracle_sample(g, target_s: float, rows_hint: int | None = None):
    """Time the CPU oracle (as it stands) on a bounded sample of source rows: returns
    (entries_per_s, rows, seconds, threads)."""
    import numpy as np

    import oracle
    threads = oracle.num_threads()
    if rows_hint is None:
        probe = min(g.n, max(threads * 2, 32))
        t = time.perf_counter()
        oracle.apsp_rows(g.n, g.src, g.dst, g.w, np.arange(probe))
        dt = time.perf_counter() - t
        rows_hint = int(min(g.n, max(probe, probe * target_s / max(dt, 1e-6))))
    rows = np.arange(rows_hint) % g.n
    t = time.perf_counter()
    oracle.apsp_rows(g.n, g.src, g.dst, g.w, rows)
    dt = time.perf_counter() - t
    return rows_hint * g.n / dt, rows_hint, dt, threads


def host_info() -> dict:
    """CPU model, nproc and the affinity count of this process."""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity": len(os.sched_getaffinity(0))}


def cfg1_one_core() -> dict:
    """The oracle on ONE core over all of cfg1 (2,000 sources x 2,000 columns), SURVEY 8.d."""
    import oracle
    from paper_conf_ipps_duttackb17_b200 import graphgen as gg
    g = gg.config("cfg1")
    t = time.perf_counter()
    oracle.apsp(g.n, g.src, g.dst, g.w, nthreads=1)
    dt = time.perf_counter() - t
    oracle.num_threads(len(os.sched_getaffinity(0)))   # back to every core this process may use
    return {"seconds": dt, "entries_per_s": g.n * g.n / dt, "threads": 1}


def run_reference(args, rank, world):
    """The reference arm for this tier: the CPU oracle, timed on the box's host cores."""
    if rank != 0:
        return
    import numpy as np

    import oracle
    from paper_conf_ipps_duttackb17_b200 import graphgen as gg
    g = gg.config(args.config, args.seed)
    threads = oracle.num_threads()
    # size one step to ~2-3 s of all-core CPU work
    probe = max(threads * 2, 32)
    t = time.perf_counter()
    oracle.apsp_rows(g.n, g.src, g.dst, g.w, np.arange(probe))
    per_row = (time.perf_counter() - t) / probe
    rows_per_step = int(min(g.n, max(threads, 2.5 / max(per_row, 1e-9))))
    for i in range(args.warmup):
        oracle.apsp_rows(g.n, g.src, g.dst, g.w, (np.arange(rows_per_step) + i * rows_per_step) % g.n)
    t = time.perf_counter()
    for i in range(args.steps):
        oracle.apsp_rows(g.n, g.src, g.dst, g.w, (np.arange(rows_per_step) + i * rows_per_step) % g.n)
    dt = time.perf_counter() - t
    value = rows_per_step * g.n * args.steps / dt
    sample = (f"{rows_per_step} Dijkstra sources per step on the uncontracted {args.config} graph "
              f"(N={g.n}); entries = sources x N")
    line = {"metric": METRIC, "value": value, "unit": UNIT, "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int64 (int32 output)",
            "data": "synthetic (seeded generator)",
            "config": {"workload": WORKLOADS.get(args.config, args.config), "name": args.config, "n": g.n,
                       "m": g.m, "seed": args.seed},
            "cpu_baseline": dict({"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
                                 **host_info()),
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------ our arm
def run_ours(args, rank, world, local_rank):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_duttackb17_b200 as ea
    from paper_conf_ipps_duttackb17_b200 import graphgen as gg

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    comm = None
    if world > 1:
        comm = ea.Comm.from_torch_distributed()

    def barrier():
        if world > 1:
            dist.barrier()

    t0 = time.perf_counter()
    g = gg.config(args.config, args.seed)
    stats = gg.stats(g)
    log(f"[rank {rank}] generated {args.config}: n={g.n} m={g.m} in {time.perf_counter() - t0:.1f}s")
    src = torch.as_tensor(g.src).to(dev)
    dst = torch.as_tensor(g.dst).to(dev)
    w = torch.as_tensor(g.w).to(dev)
    r0, r1 = ea.row_block(g.n, world, rank)
    rows = r1 - r0
    out = torch.empty((rows, g.n), dtype=torch.int32, device=dev)
    plan = ea.ear_decompose(g.n, src, dst, w)
    info = plan.info(world)
    plan.destroy()
    stream = torch.cuda.current_stream(dev)

    flags = {"fw": 0, "sssp": ea.FLAG_SSSP, "bcc": ea.FLAG_BCC, "bcc_sssp": ea.FLAG_BCC | ea.FLAG_SSSP,
             "part": ea.FLAG_PART | ea.FLAG_BCC | ea.FLAG_SSSP}[args.phase2] \
        | (ea.FLAG_FW32 if args.fw32 else 0)
    bcc = part = None
    if args.phase2 == "part":
        pp = ea.ear_decompose(g.n, src, dst, w, flags=flags)
        part = pp.part_info()
        pp.destroy()
    if args.phase2 in ("bcc", "bcc_sssp"):
        pb = ea.ear_decompose(g.n, src, dst, w, flags=flags)
        if world == 1 and not args.no_alt:   # one untimed Phase II: the re-reduction counts of a solve
            Dp = ea.alloc_D(pb)
            ea.apsp_reduced(pb, Dp)
            torch.cuda.synchronize()
            del Dp
        bcc = pb.bcc_info()
        bcc["sum_cubes_over_nr3"] = bcc["sum_cubes"] / float(max(info.n_reduced, 1)) ** 3
        pb.destroy()

    def step():
        ea.apsp_full(g.n, src, dst, w, out=out, row_begin=r0, row_end=r1, flags=flags, comm=comm, stream=stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()

    # the headline: K steps with the library's per-launch profiling OFF (only its launch counter runs)
    sampler = ClockSampler(gpu_id_for(local_rank))
    sampler.start()
    time.sleep(0.3)
    ea.profile_enable(False)
    ea.profile_reset()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    evs[0].record(stream)
    for i in range(args.steps):
        step()
        evs[i + 1].record(stream)
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    clocks = sampler.stop()
    launches = int(ea.profile_read()["launches"])
    ms = evs[0].elapsed_time(evs[-1])
    step_ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(args.steps)]
    ms_max = max_over_ranks(ms, world, dev)
    value = float(g.n) * float(g.n) * args.steps / (ms_max / 1e3)

    # a separate profiled pass of the same K steps: CUDA events around every library launch on the
    # stream it runs on -> per-kernel-class device times for phases_ms and the roofline objects
    ea.profile_reset()
    ea.profile_enable(True)
    p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p0.record(stream)
    for _ in range(args.steps):
        step()
    p1.record(stream)
    torch.cuda.synchronize()
    prof = ea.profile_read()
    ea.profile_enable(False)
    profiled_ms = p0.elapsed_time(p1) / args.steps

    # roofline of the dominant kernel: FW phase-3 min-plus tiles (ALU bound)
    peaks = measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    peak_alu = SM_COUNT * ALU_LANES_PER_SM * sm_max * 1e6 / 1e12     # T min-plus / s
    p3_ms = prof["fw_phase3_ms"]
    ach = prof["fw_phase3_minplus"] / (p3_ms / 1e3) / 1e12 if p3_ms > 0 else 0.0
    n_p3 = max(prof["fw_phase3_launches"], 1)
    roofline = {"bound": "alu", "kernel": "k_fw_tiles<Frag32> (FW phase 3, int32)", "achieved": ach, "peak": peak_alu,
                "unit": "Tminplus/s", "frac": ach / peak_alu if peak_alu else None,
                "traffic": ncu_traffic("k_fw_tiles<Frag32>", args.config),
                "avg_launch_ms": p3_ms / n_p3, "minplus_per_launch": prof["fw_phase3_minplus"] / n_p3,
                "peak_basis": f"{SM_COUNT} SMs x {ALU_LANES_PER_SM} VIADDMNMX/clk/SM x {sm_max:.0f} MHz "
                              "(sm_max_mhz of MEASURED_PEAKS.json; issue rate from microbench/minplus_peak.cu)"}
    lanes = ALU_LANES_PER_SM
    if prof["fw_phase3_16_minplus"] > 0:
        # the packed 16-bit FW ran: two min-plus per VIADDMNMX.U16x2 at the same issue
        # rate (microbench/minplus_peak.cu: 37.15 T/s), so its roofline peak is twice the int32 one
        lanes = 2 * ALU_LANES_PER_SM
        p16 = prof["fw_phase3_16_ms"]
        n16 = max(int(prof["fw_phase3_launches"]), 1)
        ach = prof["fw_phase3_16_minplus"] / (p16 / 1e3) / 1e12
        peak_alu = SM_COUNT * lanes * sm_max * 1e6 / 1e12
        roofline.update({"kernel": "k_fw_tiles<Frag16> (FW phase 3, packed u16x2)", "achieved": ach, "peak": peak_alu,
                         "frac": ach / peak_alu, "traffic": ncu_traffic("k_fw_tiles<Frag16>", args.config),
                         "avg_launch_ms": p16 / n16, "minplus_per_launch": prof["fw_phase3_16_minplus"] / n16,
                         "peak_basis": f"{SM_COUNT} SMs x {lanes} min-plus/clk/SM (64 VIADDMNMX.U16x2, two lanes "
                                       f"each) x {sm_max:.0f} MHz (sm_max_mhz of MEASURED_PEAKS.json; issue rate "
                                       "from microbench/minplus_peak.cu)"})
    if clocks.get("sm_mhz"):
        roofline["frac_at_run_clock"] = ach / (SM_COUNT * lanes * clocks["sm_mhz"] * 1e6 / 1e12)
    hbm = float(peaks.get("hbm_gbs", 6555.2))
    ex_ms = prof["expand_ms"]
    ex_ach = prof["expand_bytes"] / (ex_ms / 1e3) / 1e9 if ex_ms > 0 else 0.0
    roofline_expand = {"bound": "hbm", "kernel": "k_expand_pairs", "achieved": ex_ach, "peak": hbm, "unit": "GB/s",
                       "frac": ex_ach / hbm, "traffic": ncu_traffic("k_expand_pairs", args.config),
                       "avg_launch_ms": ex_ms / max(prof["expand_launches"], 1),
                       "bytes_per_launch": prof["expand_bytes"] / max(prof["expand_launches"], 1)}
    K = args.steps
    # main-stream FW time; the lookahead's side-stream pivot work overlaps phase 3 (fw_side_overlapped)
    fw_ms = prof["fw_init_ms"] + prof["fw_phase1_ms"] + prof["fw_phase2_ms"] + prof["fw_phase3_ms"] + prof["fw16_conv_ms"]
    if args.phase2 in ("sssp", "bcc_sssp"):   # the dominant kernel is the per-source SSSP
        # algorithmic work: Dijkstra's relaxation count, every arc of the solved graph once per source;
        # peak: each relaxation needs at least one shared-memory load of d(u) and an SM serves one
        # conflict-free 32-lane shared load per clock (the kernel is bound by its round
        # latency, far below this)
        sssp_ms = prof["sssp_ms"]
        n_ss = max(prof["sssp_launches"], 1)
        ach = prof["sssp_arcs"] / (sssp_ms / 1e3) / 1e9 if sssp_ms > 0 else 0.0
        peak_relax = SM_COUNT * 32 * sm_max * 1e6 / 1e9
        roofline = {"bound": "alu", "kernel": "k_sssp16 (Phase II: per-source near-far SSSP on the reduced pieces)",
                    "achieved": ach, "peak": peak_relax, "unit": "G relaxations/s", "frac": ach / peak_relax,
                    "traffic": ncu_traffic("k_sssp16", args.config), "avg_launch_ms": sssp_ms / n_ss,
                    "relaxations_per_launch": prof["sssp_arcs"] / n_ss,
                    "peak_basis": f"{SM_COUNT} SMs x 32 shared-memory lanes/clk x {sm_max:.0f} MHz: one conflict-free "
                                  "load of d(u) per relaxation (an upper bound; the kernel is round-latency bound, "
                                  "DESIGN.md 6b)"}
        if clocks.get("sm_mhz"):
            roofline["frac_at_run_clock"] = ach / (SM_COUNT * 32 * clocks["sm_mhz"] * 1e6 / 1e9)
    if args.phase2 == "part" and prof["part_mp_ms"] > 0:   # the region products (ALU, packed u16x2)
        pm_ms = prof["part_mp_ms"]
        n_pm = max(prof["part_mp_launches"], 1)
        ach = prof["part_minplus"] / (pm_ms / 1e3) / 1e12
        lanes = 2 * ALU_LANES_PER_SM
        peak_alu = SM_COUNT * lanes * sm_max * 1e6 / 1e12
        roofline = {"bound": "alu", "kernel": "k_region_prod (+ k_region_mp for boundaries > 32; Phase II by regions: "
                                              "the two min-plus products through the region boundaries, packed u16x2)",
                    "achieved": ach, "peak": peak_alu, "unit": "Tminplus/s", "frac": ach / peak_alu,
                    "traffic": ncu_traffic("k_region_prod", args.config), "avg_launch_ms": pm_ms / n_pm,
                    "minplus_per_launch": prof["part_minplus"] / n_pm,
                    "peak_basis": f"{SM_COUNT} SMs x {lanes} min-plus/clk/SM (64 VIADDMNMX.U16x2, two lanes each) "
                                  f"x {sm_max:.0f} MHz (sm_max_mhz of MEASURED_PEAKS.json; issue rate from "
                                  "microbench/minplus_peak.cu)"}
        if clocks.get("sm_mhz"):
            roofline["frac_at_run_clock"] = ach / (SM_COUNT * lanes * clocks["sm_mhz"] * 1e6 / 1e12)
    phases = {"decompose": prof["decompose_ms"] / K, "part": prof["part_ms"] / K, "part_mp": prof["part_mp_ms"] / K, "fw": fw_ms / K, "sssp": prof["sssp_ms"] / K, "fw_phase1": prof["fw_phase1_ms"] / K,
              "fw_phase2": prof["fw_phase2_ms"] / K, "fw_phase3": p3_ms / K, "comm": prof["comm_ms"] / K,
              "expand": ex_ms / K, "same_chain": prof["same_chain_ms"] / K,
              "bcc_pieces": prof["bcc_pieces_ms"] / K, "compose": prof["compose_ms"] / K,
              "fw16_conv": prof["fw16_conv_ms"] / K, "rereduce": prof["rereduce_ms"] / K,
              "bcc_prepare": prof["bcc_prepare_ms"] / K, "expand_d16": prof["expand_d16_ms"] / K,
              "fw_side_overlapped": prof["fw_side_ms"] / K}
    fw_minplus = prof["fw_phase2_minplus"] + prof["fw_phase3_minplus"]
    # "roofline" = the kernel with the largest share of the step (the expansion once Phase II runs by
    # regions); the other one is reported beside it
    phase2_ms = (prof["part_mp_ms"] if args.phase2 == "part" else prof["sssp_ms"] if args.phase2 in ("sssp", "bcc_sssp")
                 else p3_ms)
    roofline["step_share"] = phase2_ms / K / (profiled_ms or 1.0)
    roofline_expand["step_share"] = ex_ms / K / (profiled_ms or 1.0)
    if ex_ms >= phase2_ms:
        rooflines = {"roofline": roofline_expand, "roofline_phase2": roofline}
    else:
        rooflines = {"roofline": roofline, "roofline_expand": roofline_expand}
    del out
    torch.cuda.empty_cache()

    # Phase II alternatives (plain FW on all of G^r; SURVEY 8.f NEXT 2 per-source SSSP; NEXT 3 pieces)
    # (bit-identical D; reported beside the timed Phase II, not part of the timed steps)
    alt = fw_roof = None
    if world == 1 and not args.no_alt:
        alt = {"note": "Phase II only (D of G^r), one timed call after a warm-up call; --phase2 X times the full step"}
        for name, fl in (("fw", 0), ("sssp", ea.FLAG_SSSP), ("bcc", ea.FLAG_BCC), ("bcc_sssp", ea.FLAG_BCC | ea.FLAG_SSSP),
                         ("part", ea.FLAG_PART)):
            if name == args.phase2:
                continue
            p2 = ea.ear_decompose(g.n, src, dst, w, flags=fl)
            D2 = ea.alloc_D(p2)
            ea.apsp_reduced(p2, D2)            # warm-up (builds the reduced CSR / block structure once)
            torch.cuda.synchronize()
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            ea.apsp_reduced(p2, D2)
            a1.record(stream)
            torch.cuda.synchronize()
            alt[f"{name}_phase2_ms"] = a0.elapsed_time(a1)
            if name == "fw":   # the blocked FW of row a5: its phase-3 tile kernel against its ALU peak
                ea.profile_reset()
                ea.profile_enable(True)
                ea.apsp_reduced(p2, D2)
                torch.cuda.synchronize()
                pf = ea.profile_read()
                ea.profile_enable(False)
                packed = pf["fw_phase3_16_minplus"] > 0
                mp_ = pf["fw_phase3_16_minplus"] if packed else pf["fw_phase3_minplus"]
                ms_ = pf["fw_phase3_16_ms"] if packed else pf["fw_phase3_ms"]
                lanes_ = (2 if packed else 1) * ALU_LANES_PER_SM
                pk = SM_COUNT * lanes_ * sm_max * 1e6 / 1e12
                ach_ = mp_ / (ms_ / 1e3) / 1e12 if ms_ > 0 else 0.0
                fw_roof = {"bound": "alu", "kernel": "k_fw_tiles<Frag16>" if packed else "k_fw_tiles<Frag32>",
                           "route": "--phase2 fw (blocked FW on all of G^r, one apsp_reduced call)",
                           "achieved": ach_, "peak": pk, "unit": "Tminplus/s", "frac": ach_ / pk if pk else None,
                           "minplus": mp_, "phase3_ms": ms_,
                           "traffic": ncu_traffic("k_fw_tiles<Frag16>" if packed else "k_fw_tiles<Frag32>", args.config)}
            del D2
            p2.destroy()
            torch.cuda.empty_cache()

    # e2e through the host-buffer C-ABI entry point: H2D edges + D2H output rows inside the region
    e2e = None
    if not args.no_e2e:
        hs = torch.as_tensor(g.src).pin_memory()
        hd = torch.as_tensor(g.dst).pin_memory()
        hw = torch.as_tensor(g.w).pin_memory()
        e2e_steps = max(1, min(args.steps, args.e2e_steps))
        out_bytes = 4 * rows * g.n
        pipelined = args.e2e_mode == "pipelined"
        # two pinned output buffers when the host has room (job i+1 never lands in job i's rows)
        nbuf = args.e2e_bufs or (2 if pipelined and psutil.virtual_memory().available > 2.5 * out_bytes else 1)
        houts = [torch.empty((rows, g.n), dtype=torch.int32, pin_memory=True) for _ in range(nbuf)]
        if pipelined:   # warm-up in the timed mode: two jobs in flight grow the library's memory pool to its
            # steady-state size (fresh pool pages appear to queue behind the row copies on the copy engines)
            wj = [ea.apsp_full_host_async(g.n, hs, hd, hw, out=houts[i % nbuf], row_begin=r0, row_end=r1,
                                          flags=flags, comm=comm, stream=stream) for i in range(2)]
            for j in wj:
                j.wait()
        else:
            ea.apsp_full_host(g.n, hs, hd, hw, out=houts[0], row_begin=r0, row_end=r1, flags=flags, comm=comm,
                              stream=stream)
        barrier()
        t = time.perf_counter()
        if pipelined:   # one job in flight ahead: job i+1's Phases I-II overlap job i's expansion + row copies
            prev = None
            for i in range(e2e_steps):
                job = ea.apsp_full_host_async(g.n, hs, hd, hw, out=houts[i % nbuf], row_begin=r0, row_end=r1,
                                              flags=flags, comm=comm, stream=stream)
                if prev is not None:
                    prev.wait()
                prev = job
            prev.wait()
        else:
            for _ in range(e2e_steps):
                ea.apsp_full_host(g.n, hs, hd, hw, out=houts[0], row_begin=r0, row_end=r1, flags=flags, comm=comm,
                                  stream=stream)
        torch.cuda.synchronize()
        e2e_s = max_over_ranks(time.perf_counter() - t, world, dev)
        barrier()
        e2e = {"value": float(g.n) * g.n * e2e_steps / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 3 * 4 * g.m,
               "d2h_bytes_per_step": out_bytes, "steps": e2e_steps, "mode": args.e2e_mode, "host_out_buffers": nbuf,
               "api": ("apsp_full_host_async + ear_job_wait, one job in flight ahead" if pipelined else "apsp_full_host")
               + " (pinned host edge list in, read in place; pinned host rows out)"}
        del houts

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, nrows, dt, thr = oracle_sample(g, args.cpu_seconds)
        cpu = {"value": v, "unit": UNIT, "cores": thr, "kind": "oracle",
               "sample": f"Dijkstra from the first {nrows} sources of the uncontracted {args.config} graph "
                         f"({dt:.1f} s on {thr} threads); entries = sources x N"}
        cpu.update(host_info())
        cpu["cfg1_one_core"] = cfg1_one_core()

    seeds = None
    if world == 1 and not args.no_seeds:   # seeds 0/1/2, median of 5 single-step times each
        seeds = {"note": "median of 5 single-step device times after 1 warm-up step; seed 0 from the timed region",
                 "0": {"median_ms": statistics.median(step_ms), "entries_per_s": g.n * g.n / (statistics.median(step_ms) / 1e3)}}
        for sd in (1, 2):
            gs = gg.config(args.config, sd)
            ss, sd_, sw = (torch.as_tensor(x).to(dev) for x in (gs.src, gs.dst, gs.w))
            o2 = torch.empty((gs.n, gs.n), dtype=torch.int32, device=dev)
            run = lambda: ea.apsp_full(gs.n, ss, sd_, sw, out=o2, flags=flags, stream=stream)  # noqa: E731
            run()
            torch.cuda.synchronize()
            ts = []
            for _ in range(5):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                run()
                b.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            med = statistics.median(ts)
            seeds[str(sd)] = {"median_ms": med, "entries_per_s": gs.n * gs.n / (med / 1e3), "n_reduced":
                              ea.ear_decompose(gs.n, ss, sd_, sw).info().n_reduced}
            del o2
            torch.cuda.empty_cache()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
                "ms_per_step": ms_max / K, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
                "dtype": ("int32 (SSSP: u16 shared-memory rows, exact below 0xFFFF; int32 fallback)"
                          if args.phase2 in ("sssp", "bcc_sssp") else
                          "int32 (regions: packed u16x2 min-plus, exact while no u16 sum can reach 0x10000; other routes "
                          "otherwise)" if args.phase2 == "part" else
                          "int32" if prof["fw16_used"] == 0 else "int32 (FW: packed u16x2, exact below 0x7FFF)"),
                "data": "synthetic (seeded generator, spatially coherent labels)",
                "fw16": {"used": int(prof["fw16_used"]) // K, "fallbacks": int(prof["fw16_fallbacks"]) // K},
                "config": {"workload": WORKLOADS.get(args.config, args.config), "name": args.config,
                           "n": g.n, "m": g.m, "n_reduced": info.n_reduced, "n_reduced_padded": info.n_reduced_padded,
                           "n_chains": info.n_chains, "max_chain_len": info.max_chain_len,
                           "degree2_frac": stats["deg2_frac"], "seed": args.seed, "rows_per_rank": rows,
                           "parallelism": f"row-block x{world}" if world > 1 else "single GPU",
                           "phase2": args.phase2, "bcc": bcc, "part": part,
                           "l2": "inputs larger than L2 (D %.1f GB, output %.1f GB per step)" % (
                               4.0 * info.n_reduced_padded ** 2 / 1e9, 4.0 * g.n * g.n / 1e9)},
                **rooflines, "roofline_fw": fw_roof,
                "fw_minplus_gops": fw_minplus / (fw_ms / 1e3) / 1e9 if fw_ms > 0 else None,
                "phases_ms": phases, "phase2_alternatives": alt, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "gpu_launches": launches, "step_ms": step_ms, "seeds": seeds,
                "profiled_pass": {"ms_per_step": profiled_ms, "note": "roofline objects and phases_ms come from this "
                                  "separate pass of the same K steps with CUDA events around every library launch; "
                                  "the headline value is timed with them off"},
                "gpu_launches_note": "own kernels in the timed region (CUB sort/scan launches of Phase I excluded)",
                "mteps_context": g.m * g.n / (ms_max / K / 1e3) / 1e6}
        print(json.dumps(line), flush=True)
    if comm is not None:
        comm.destroy()


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="cfg4")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--phase2", choices=["part", "bcc_sssp", "bcc", "fw", "sssp"], default="part",
                    help="Phase II: the biconnected pieces of G^r (paper sec. 2.2) each reduced again and solved by "
                         "per-source SSSP (the paper's own Phase II, P:101; default), the same pieces by blocked FW, "
                         "blocked FW on all of G^r, or per-source SSSP on all of G^r")
    ap.add_argument("--fw32", action="store_true", help="int32 FW throughout (EAR_FLAG_FW32)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=4)
    ap.add_argument("--e2e-bufs", type=int, choices=[0, 1, 2], default=0,
                    help="pinned host output buffers for the pipelined e2e (0: two when the host has room)")
    ap.add_argument("--e2e-mode", choices=["sync", "pipelined"], default="pipelined",
                    help="e2e calls: synchronous apsp_full_host, or async jobs pipelined one deep")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-alt", action="store_true", help="skip the one-off SSSP Phase II timing")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--no-seeds", action="store_true", help="skip the seed 1/2 medians (SURVEY 8.d)")
    args = ap.parse_args()

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        log(f"note: --gpus {args.gpus} but WORLD_SIZE={world}; using WORLD_SIZE")
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
