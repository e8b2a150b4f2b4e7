"""B200-native ear-reduced all-pairs shortest paths (Dutta, Chaitanya, Kothapalli, Bera; IPDPS-W 2017).

The hot path lives in ``libearapsp.so`` (sm_100a CUDA kernels behind the C ABI of
``include/ear_apsp.h``); :mod:`.ear_apsp` is its thin ctypes binding and :mod:`.graphgen` builds the
seeded synthetic workloads.  There is no CPU fallback.
"""
from .ear_apsp import (FLAG_BCC, FLAG_FW32, FLAG_NO_CONTRACT, FLAG_NONE, FLAG_PART, FLAG_SSSP, INF, TILE, Comm, EarError, Plan, alloc_D, apsp_full,  # noqa: F401
                       apsp_full_host, apsp_full_host_async, apsp_reduced, apsp_reduced_emulated, apsp_reduced_rank_timing, ear_decompose, expand_ears, gather_reduced, lib, Mcb, mcb, profile_enable,
                       profile_read, profile_reset, query_pairs, row_block, version)
