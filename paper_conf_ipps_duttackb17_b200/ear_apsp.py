"""Thin ctypes binding of libearapsp.so (include/ear_apsp.h) -- argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; torch is used only for device memory,
streams and (for multi-GPU) the process group that distributes the NCCL unique id.  There is no CPU
fallback: if the shared library is missing or cannot be loaded, every call raises.

Names follow the C ABI (and the paper's Algorithm 1):
    ear_decompose  -> Plan        Phase I, Reduce(G)
    apsp_reduced(plan, D)         Phase II, APSP on G^r         (blocked FW)
    expand_ears(plan, D, ...)     Phase III, UPDATE_DISTANCE
    apsp_full(...)                all of Algorithm 1
    apsp_full_host(...)           all of Algorithm 1 with host buffers (end-to-end)
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np
import torch

from . import _build

INF = 0x3FFFFFFF
TILE = 128
FLAG_NONE = 0
FLAG_NO_CONTRACT = 1
FLAG_SSSP = 2
FLAG_BCC = 4
FLAG_FW32 = 8
FLAG_PART = 16

_lib = None


class EarError(RuntimeError):
    pass


class _Info(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int32), ("n_reduced", ctypes.c_int32), ("n_reduced_padded", ctypes.c_int32),
                ("n_chains", ctypes.c_int32), ("max_chain_len", ctypes.c_int32), ("n_promoted", ctypes.c_int32),
                ("n_reduced_edges", ctypes.c_int64), ("m_simple", ctypes.c_int64), ("rank_rounds", ctypes.c_int32),
                ("max_weight", ctypes.c_int32)]


class _Profile(ctypes.Structure):
    _fields_ = [("launches", ctypes.c_int64), ("decompose_ms", ctypes.c_double), ("fw_init_ms", ctypes.c_double),
                ("fw_phase1_ms", ctypes.c_double), ("fw_phase2_ms", ctypes.c_double), ("fw_phase3_ms", ctypes.c_double),
                ("fw_phase1_launches", ctypes.c_int64), ("fw_phase2_launches", ctypes.c_int64),
                ("fw_phase3_launches", ctypes.c_int64), ("fw_phase2_minplus", ctypes.c_double),
                ("fw_phase3_minplus", ctypes.c_double), ("comm_ms", ctypes.c_double), ("expand_ms", ctypes.c_double),
                ("same_chain_ms", ctypes.c_double), ("expand_launches", ctypes.c_int64),
                ("expand_bytes", ctypes.c_double), ("sssp_ms", ctypes.c_double), ("sssp_launches", ctypes.c_int64),
                ("sssp_arcs", ctypes.c_double), ("bcc_pieces_ms", ctypes.c_double), ("compose_ms", ctypes.c_double),
                ("compose_bytes", ctypes.c_double), ("fw16_used", ctypes.c_int64), ("fw16_fallbacks", ctypes.c_int64),
                ("fw16_conv_ms", ctypes.c_double), ("fw_phase3_16_ms", ctypes.c_double),
                ("fw_phase3_16_minplus", ctypes.c_double), ("fw_side_ms", ctypes.c_double),
                ("rereduce_ms", ctypes.c_double), ("bcc_prepare_ms", ctypes.c_double),
                ("fw16_prechecked", ctypes.c_int64), ("expand_d16_ms", ctypes.c_double),
                ("part_ms", ctypes.c_double), ("part_mp_ms", ctypes.c_double), ("part_mp_launches", ctypes.c_int64),
                ("part_minplus", ctypes.c_double)]


class _BccInfo(ctypes.Structure):
    _fields_ = [("n_components", ctypes.c_int32), ("n_blocks", ctypes.c_int32), ("n_articulation", ctypes.c_int32),
                ("n_pieces", ctypes.c_int32), ("largest_piece", ctypes.c_int32), ("tree_levels", ctypes.c_int32),
                ("sum_cubes", ctypes.c_double), ("rereduced_pieces", ctypes.c_int32), ("largest_reduced", ctypes.c_int32),
                ("rereduce_levels", ctypes.c_int32)]


class _PartInfo(ctypes.Structure):
    _fields_ = [("n_regions", ctypes.c_int32), ("n_boundary", ctypes.c_int32), ("max_region", ctypes.c_int32),
                ("max_boundary", ctypes.c_int32), ("passes", ctypes.c_int32), ("multi_component", ctypes.c_int32),
                ("sum_region_boundary", ctypes.c_double)]


class _McbInfo(ctypes.Structure):
    _fields_ = [("dim", ctypes.c_int32), ("weight", ctypes.c_int64), ("n_reduced", ctypes.c_int32),
                ("m_reduced", ctypes.c_int64), ("components", ctypes.c_int32), ("n_candidates", ctypes.c_int64),
                ("tree_depth", ctypes.c_int32)]


# (name, restype, argtypes) for every symbol declared in include/ear_apsp.h
_P, _I32, _I64, _U32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
SIGNATURES = {
    "ear_decompose": (_I32, [_I32, _I64, _P, _P, _P, _U32, _P, ctypes.POINTER(_P)]),
    "ear_plan_info": (_I32, [_P, _I32, ctypes.POINTER(_Info)]),
    "ear_plan_export": (_I32, [_P, _P, _P, _P, _P, _P, _P, _P]),
    "ear_plan_export_reduced_edges": (_I32, [_P, _P, _P, _P, _P]),
    "ear_plan_destroy": (None, [_P]),
    "ear_bcc_info": (_I32, [_P, ctypes.POINTER(_BccInfo)]),
    "ear_part_info": (_I32, [_P, ctypes.POINTER(_PartInfo)]),
    "apsp_reduced": (_I32, [_P, _P, _I64, _P, _P]),
    "apsp_reduced_emulated": (_I32, [_P, _I32, _P, _I64, _P]),
    "apsp_reduced_rank_timing": (_I32, [_P, _I32, _I32, _P]),
    "ear_owned_tile_rows": (_I32, [_I32, _I32, _I32]),
    "ear_gather_reduced": (_I32, [_P, _P, _I64, _P, _I64, _P, _P]),
    "expand_ears": (_I32, [_P, _P, _I64, _I32, _I32, _P, _I64, _P]),
    "ear_query_pairs": (_I32, [_P, _P, _I64, _I64, _P, _P, _P, _P]),
    "apsp_full": (_I32, [_I32, _I64, _P, _P, _P, _U32, _I32, _I32, _P, _I64, _P, _P]),
    "apsp_full_host": (_I32, [_I32, _I64, _P, _P, _P, _U32, _I32, _I32, _P, _I64, _P, _P]),
    "apsp_full_host_async": (_I32, [_I32, _I64, _P, _P, _P, _U32, _I32, _I32, _P, _I64, _P, _P, ctypes.POINTER(_P)]),
    "ear_job_wait": (_I32, [_P]),
    "ear_mcb": (_I32, [_I32, _I64, _P, _P, _P, _P, ctypes.POINTER(_P)]),
    "ear_mcb_info": (_I32, [_P, ctypes.POINTER(_McbInfo)]),
    "ear_mcb_cycle_weights": (_I32, [_P, _P, _P]),
    "ear_mcb_cycle": (_I32, [_P, _I32, _P, _I32, ctypes.POINTER(_I32), _P]),
    "ear_mcb_destroy": (None, [_P]),
    "ear_row_block": (None, [_I32, _I32, _I32, ctypes.POINTER(_I32), ctypes.POINTER(_I32)]),
    "ear_comm_init": (_I32, [_I32, _I32, _P, _P, ctypes.POINTER(_P)]),
    "ear_comm_info": (_I32, [_P, ctypes.POINTER(_I32), ctypes.POINTER(_I32)]),
    "ear_comm_destroy": (None, [_P]),
    "ear_profile_enable": (None, [_I32]),
    "ear_profile_reset": (None, []),
    "ear_profile_read": (_I32, [ctypes.POINTER(_Profile)]),
    "ear_status_string": (ctypes.c_char_p, [_I32]),
    "ear_last_error": (ctypes.c_char_p, []),
    "ear_version": (ctypes.c_char_p, []),
}


def lib_path() -> str:
    # EAR_LIB: another in-tree build of the same library (A/B timing in tools/); default libearapsp.so
    return os.environ.get("EAR_LIB") or _build.LIB


def lib():
    """Load libearapsp.so (built in-tree by __graft_entry__.build()).  Raises if it is missing."""
    global _lib
    if _lib is None:
        path = lib_path()
        if not os.path.exists(path):
            raise EarError(f"{path} is missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(path)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _check(status: int, what: str):
    if status != 0:
        L = lib()
        raise EarError(f"{what}: {L.ear_status_string(status).decode()} ({L.ear_last_error().decode()})")


def _stream(stream=None) -> int:
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def _check_out(out: torch.Tensor, rows: int, n: int, cuda: bool):
    """`out` must hold rows x n int32 entries with unit column stride (the library writes every one)."""
    where = "CUDA" if cuda else "host"
    if out.is_cuda != cuda or out.dtype != torch.int32 or out.dim() != 2 or out.stride(1) != 1:
        raise EarError(f"out must be a 2-D int32 {where} tensor with unit column stride")
    if out.shape[0] < rows or out.shape[1] < n or out.stride(0) < n:
        raise EarError(f"out is {tuple(out.shape)} (row stride {out.stride(0)}); need at least {rows} x {n}")


def _dev_i32(t: torch.Tensor, name: str) -> torch.Tensor:
    if not (t.is_cuda and t.dtype == torch.int32 and t.is_contiguous()):
        raise EarError(f"{name} must be a contiguous int32 CUDA tensor")
    return t


@dataclass
class PlanInfo:
    n: int
    n_reduced: int
    n_reduced_padded: int
    n_chains: int
    max_chain_len: int
    n_promoted: int
    n_reduced_edges: int
    m_simple: int
    rank_rounds: int
    max_weight: int


# int32_t (*ear_allgather_fn)(const void *send, void *recv, int64_t bytes, void *ctx)
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p)


class Comm:
    """This rank's communicator (one process per GPU; several processes may share a GPU): the
    library's peer-memory exchange windows.  The library trades CUDA IPC handles through a host
    all-gather callback, implemented here with torch.distributed (any backend; gloo works for ranks
    that share a GPU)."""

    def __init__(self, handle, nranks: int, rank: int, keep=None):
        self.handle, self.nranks, self.rank, self._keep = handle, nranks, rank, keep

    @classmethod
    def from_torch_distributed(cls, group=None) -> "Comm":
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)

        def allgather(send, recv, nbytes, _ctx):
            try:
                out = [None] * world
                dist.all_gather_object(out, ctypes.string_at(send, nbytes), group=group)
                buf = b"".join(out)
                if len(buf) != nbytes * world:
                    return 1
                ctypes.memmove(recv, buf, len(buf))
                return 0
            except Exception:  # noqa: BLE001  (reported to the library as a failed collective)
                return 1

        fn = ALLGATHER_FN(allgather)
        h = _P()
        _check(lib().ear_comm_init(world, rank, ctypes.cast(fn, _P), None, ctypes.byref(h)), "ear_comm_init")
        return cls(h, world, rank, keep=fn)

    @classmethod
    def single(cls) -> "Comm":
        """A one-rank communicator (the sharded code path on one process, no peers)."""
        h = _P()
        _check(lib().ear_comm_init(1, 0, None, None, ctypes.byref(h)), "ear_comm_init")
        return cls(h, 1, 0)

    def destroy(self):
        if self.handle:
            lib().ear_comm_destroy(self.handle)
            self.handle = None


def _comm_handle(comm):
    return None if comm is None else comm.handle


class Plan:
    """Reduce(G) result (library-owned device descriptors)."""

    def __init__(self, handle, n):
        self.handle, self.n = handle, n

    def info(self, nranks: int = 1) -> PlanInfo:
        i = _Info()
        _check(lib().ear_plan_info(self.handle, nranks, ctypes.byref(i)), "ear_plan_info")
        return PlanInfo(*[getattr(i, f) for f, _ in _Info._fields_])

    def bcc_info(self) -> dict:
        """Block structure of G^r used by FLAG_BCC (ear_bcc_info; builds it on first use, synchronises)."""
        i = _BccInfo()
        _check(lib().ear_bcc_info(self.handle, ctypes.byref(i)), "ear_bcc_info")
        return {f: getattr(i, f) for f, _ in _BccInfo._fields_}

    def part_info(self) -> dict:
        """Region partition of G^r used by FLAG_PART (ear_part_info; builds it on first use, synchronises)."""
        i = _PartInfo()
        _check(lib().ear_part_info(self.handle, ctypes.byref(i)), "ear_part_info")
        return {f: getattr(i, f) for f, _ in _PartInfo._fields_}

    def export(self, stream=None) -> dict:
        """Per-vertex descriptors as CUDA int32 tensors (tests)."""
        names = ["tid", "ear", "left", "right", "off_left", "off_right"]
        out = {k: torch.empty(self.n, dtype=torch.int32, device="cuda") for k in names}
        _check(lib().ear_plan_export(self.handle, *[out[k].data_ptr() for k in names], _stream(stream)),
               "ear_plan_export")
        return out

    def reduced_edges(self, stream=None):
        e = self.info().n_reduced_edges
        u, v, w = (torch.empty(max(e, 1), dtype=torch.int32, device="cuda") for _ in range(3))
        _check(lib().ear_plan_export_reduced_edges(self.handle, u.data_ptr(), v.data_ptr(), w.data_ptr(),
                                                   _stream(stream)), "ear_plan_export_reduced_edges")
        return u[:e], v[:e], w[:e]

    def destroy(self):
        if self.handle:
            lib().ear_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):  # pragma: no cover
        try:
            self.destroy()
        except Exception:
            pass


def ear_decompose(n: int, src: torch.Tensor, dst: torch.Tensor, w: torch.Tensor, flags: int = 0,
                  stream=None) -> Plan:
    src, dst, w = _dev_i32(src, "src"), _dev_i32(dst, "dst"), _dev_i32(w, "w")
    h = _P()
    _check(lib().ear_decompose(n, src.numel(), src.data_ptr(), dst.data_ptr(), w.data_ptr(), flags,
                               _stream(stream), ctypes.byref(h)), "ear_decompose")
    return Plan(h, n)


def alloc_D(plan: Plan, comm: Comm | None = None) -> torch.Tensor:
    """Device buffer for apsp_reduced: full Np x Np (single GPU) or this rank's owned tile rows."""
    if comm is None:
        Np = plan.info(1).n_reduced_padded
        return torch.empty((Np, Np), dtype=torch.int32, device="cuda")
    Np = plan.info(comm.nranks).n_reduced_padded
    nown = lib().ear_owned_tile_rows(Np, comm.nranks, comm.rank)
    return torch.empty((max(nown, 1) * TILE, Np), dtype=torch.int32, device="cuda")


def apsp_reduced(plan: Plan, D: torch.Tensor, comm: Comm | None = None, stream=None) -> torch.Tensor:
    D = _dev_i32(D, "D")
    _check(lib().apsp_reduced(plan.handle, D.data_ptr(), D.stride(0), _comm_handle(comm), _stream(stream)),
           "apsp_reduced")
    return D


def apsp_reduced_emulated(plan: Plan, nranks: int, D: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """The multi-GPU (row-block sharded) FW schedule for `nranks` ranks, emulated on this GPU."""
    if D is None:
        Np = plan.info(nranks).n_reduced_padded
        D = torch.empty((Np, Np), dtype=torch.int32, device="cuda")
    _dev_i32(D, "D")
    _check(lib().apsp_reduced_emulated(plan.handle, nranks, D.data_ptr(), D.stride(0), _stream(stream)),
           "apsp_reduced_emulated")
    return D


def apsp_reduced_rank_timing(plan: Plan, nranks: int, rank: int, stream=None) -> None:
    """Diagnostic: the device work of one rank of an nranks-rank packed sharded FW (no exchange, no result)."""
    _check(lib().apsp_reduced_rank_timing(plan.handle, nranks, rank, _stream(stream)), "apsp_reduced_rank_timing")


def gather_reduced(plan: Plan, D_block: torch.Tensor, comm: Comm, D_full: torch.Tensor | None = None,
                   stream=None) -> torch.Tensor:
    Np = plan.info(comm.nranks).n_reduced_padded
    if D_full is None:
        D_full = torch.empty((Np, Np), dtype=torch.int32, device="cuda")
    _check(lib().ear_gather_reduced(plan.handle, D_block.data_ptr(), D_block.stride(0), D_full.data_ptr(),
                                    D_full.stride(0), _comm_handle(comm), _stream(stream)), "ear_gather_reduced")
    return D_full


def expand_ears(plan: Plan, D_full: torch.Tensor, row_begin: int, row_end: int, out: torch.Tensor | None = None,
                stream=None) -> torch.Tensor:
    if out is None:
        out = torch.empty((row_end - row_begin, plan.n), dtype=torch.int32, device="cuda")
    _dev_i32(D_full, "D_full")
    _check_out(out, row_end - row_begin, plan.n, cuda=True)
    _check(lib().expand_ears(plan.handle, D_full.data_ptr(), D_full.stride(0), row_begin, row_end, out.data_ptr(),
                             out.stride(0), _stream(stream)), "expand_ears")
    return out


def query_pairs(plan: Plan, D_full: torch.Tensor, s: torch.Tensor, t: torch.Tensor,
                out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Compact/query mode: S[s[i], t[i]] from D and the plan's descriptors (no N x N matrix)."""
    s, t = _dev_i32(s, "s"), _dev_i32(t, "t")
    if t.numel() != s.numel():
        raise EarError(f"s and t differ in length ({s.numel()} vs {t.numel()})")
    if out is None:
        out = torch.empty(s.numel(), dtype=torch.int32, device="cuda")
    _dev_i32(out, "out")
    if out.numel() < s.numel():
        raise EarError(f"out holds {out.numel()} entries for {s.numel()} pairs")
    _check(lib().ear_query_pairs(plan.handle, _dev_i32(D_full, "D_full").data_ptr(), D_full.stride(0), s.numel(),
                                 s.data_ptr(), t.data_ptr(), out.data_ptr(), _stream(stream)), "ear_query_pairs")
    return out


def row_block(rows: int, nranks: int, rank: int):
    b, e = _I32(), _I32()
    lib().ear_row_block(rows, nranks, rank, ctypes.byref(b), ctypes.byref(e))
    return b.value, e.value


def apsp_full(n: int, src: torch.Tensor, dst: torch.Tensor, w: torch.Tensor, out: torch.Tensor | None = None,
              row_begin: int = 0, row_end: int | None = None, flags: int = 0, comm: Comm | None = None,
              stream=None) -> torch.Tensor:
    """Algorithm 1 APSP(G) on device buffers: rows [row_begin, row_end) of S (caller order)."""
    row_end = n if row_end is None else row_end
    src, dst, w = _dev_i32(src, "src"), _dev_i32(dst, "dst"), _dev_i32(w, "w")
    if out is None:
        out = torch.empty((row_end - row_begin, n), dtype=torch.int32, device="cuda")
    _check_out(out, row_end - row_begin, n, cuda=True)
    _check(lib().apsp_full(n, src.numel(), src.data_ptr(), dst.data_ptr(), w.data_ptr(), flags, row_begin, row_end,
                           out.data_ptr(), out.stride(0), _comm_handle(comm), _stream(stream)), "apsp_full")
    return out


def apsp_full_host(n: int, src: np.ndarray | torch.Tensor, dst, w, out: torch.Tensor | None = None,
                   row_begin: int = 0, row_end: int | None = None, flags: int = 0, comm: Comm | None = None,
                   stream=None) -> torch.Tensor:
    """Algorithm 1 APSP(G) from HOST edge arrays into a HOST (preferably pinned) int32 tensor."""
    row_end = n if row_end is None else row_end
    tens = [torch.as_tensor(np.ascontiguousarray(x, dtype=np.int32)) if not isinstance(x, torch.Tensor) else x
            for x in (src, dst, w)]
    for t in tens:
        if t.is_cuda or t.dtype != torch.int32 or not t.is_contiguous():
            raise EarError("apsp_full_host takes contiguous int32 host arrays")
    if out is None:
        out = torch.empty((row_end - row_begin, n), dtype=torch.int32, pin_memory=True)
    _check_out(out, row_end - row_begin, n, cuda=False)
    _check(lib().apsp_full_host(n, tens[0].numel(), tens[0].data_ptr(), tens[1].data_ptr(), tens[2].data_ptr(),
                                flags, row_begin, row_end, out.data_ptr(), out.stride(0), _comm_handle(comm),
                                _stream(stream)), "apsp_full_host")
    return out


class HostJob:
    """An apsp_full_host_async call in flight: wait() returns the filled host tensor."""

    def __init__(self, handle, out, keep):
        self.handle, self.out, self._keep = handle, out, keep

    def wait(self) -> torch.Tensor:
        if self.handle is not None:
            h, self.handle = self.handle, None
            _check(lib().ear_job_wait(h), "ear_job_wait")
        return self.out

    def __del__(self):  # pragma: no cover
        # a job dropped without wait() still owns device scratch and writes into `out`: finish it
        # before `out` (possibly torch's cached pinned memory) can be handed to anyone else
        try:
            self.wait()
        except Exception:
            pass


def apsp_full_host_async(n: int, src, dst, w, out: torch.Tensor | None = None, row_begin: int = 0,
                         row_end: int | None = None, flags: int = 0, comm: Comm | None = None,
                         stream=None) -> HostJob:
    """apsp_full_host that returns once Phases I-II are enqueued (the expansion and the row copies
    complete in the background; the next call's Phases I-II overlap them).  Call .wait() before reading
    `out`; the host arrays must stay alive until then."""
    row_end = n if row_end is None else row_end
    tens = [torch.as_tensor(np.ascontiguousarray(x, dtype=np.int32)) if not isinstance(x, torch.Tensor) else x
            for x in (src, dst, w)]
    for t in tens:
        if t.is_cuda or t.dtype != torch.int32 or not t.is_contiguous():
            raise EarError("apsp_full_host_async takes contiguous int32 host arrays")
    if out is None:
        out = torch.empty((row_end - row_begin, n), dtype=torch.int32, pin_memory=True)
    _check_out(out, row_end - row_begin, n, cuda=False)
    h = ctypes.c_void_p()
    _check(lib().apsp_full_host_async(n, tens[0].numel(), tens[0].data_ptr(), tens[1].data_ptr(), tens[2].data_ptr(),
                                      flags, row_begin, row_end, out.data_ptr(), out.stride(0), _comm_handle(comm),
                                      _stream(stream), ctypes.byref(h)), "apsp_full_host_async")
    return HostJob(h, out, tens)


class Mcb:
    """Minimum cycle basis of G (paper sec. 3) computed on G^r (library-owned result)."""

    def __init__(self, handle, n):
        self.handle, self.n = handle, n

    def info(self) -> dict:
        i = _McbInfo()
        _check(lib().ear_mcb_info(self.handle, ctypes.byref(i)), "ear_mcb_info")
        return {f: getattr(i, f) for f, _ in _McbInfo._fields_}

    def weights(self, stream=None) -> torch.Tensor:
        """The basis cycles' weights in phase order (int64, on the device)."""
        f = self.info()["dim"]
        out = torch.empty(max(f, 1), dtype=torch.int64, device="cuda")
        _check(lib().ear_mcb_cycle_weights(self.handle, out.data_ptr(), _stream(stream)), "ear_mcb_cycle_weights")
        return out[:f]

    def cycle(self, i: int, stream=None) -> torch.Tensor:
        """Post-processing (sec. 3.3.3): basis cycle i as a closed walk of G, caller vertex ids."""
        n = _I32()
        _check(lib().ear_mcb_cycle(self.handle, i, None, 0, ctypes.byref(n), _stream(stream)), "ear_mcb_cycle")
        out = torch.empty(max(n.value, 1), dtype=torch.int32, device="cuda")
        _check(lib().ear_mcb_cycle(self.handle, i, out.data_ptr(), n.value, ctypes.byref(n), _stream(stream)),
               "ear_mcb_cycle")
        return out[:n.value]

    def destroy(self):
        if self.handle:
            lib().ear_mcb_destroy(self.handle)
            self.handle = None

    def __del__(self):  # pragma: no cover
        try:
            self.destroy()
        except Exception:
            pass


def mcb(n: int, src: torch.Tensor, dst: torch.Tensor, w: torch.Tensor, stream=None) -> Mcb:
    """Minimum cycle basis of the graph (device edge arrays), by the paper's sec. 3 method on G^r."""
    src, dst, w = _dev_i32(src, "src"), _dev_i32(dst, "dst"), _dev_i32(w, "w")
    h = _P()
    _check(lib().ear_mcb(n, src.numel(), src.data_ptr(), dst.data_ptr(), w.data_ptr(), _stream(stream),
                         ctypes.byref(h)), "ear_mcb")
    return Mcb(h, n)


def profile_enable(on: bool = True):
    """CUDA-event timing of every library kernel launch (per kernel class), see ear_profile_t."""
    lib().ear_profile_enable(1 if on else 0)


def profile_reset():
    lib().ear_profile_reset()


def profile_read() -> dict:
    p = _Profile()
    _check(lib().ear_profile_read(ctypes.byref(p)), "ear_profile_read")
    return {f: getattr(p, f) for f, _ in _Profile._fields_}


def version() -> str:
    return lib().ear_version().decode()
