"""B200-native ECL-SCC hot path -- thin Python binding of libeclscc.so (include/ecl_scc.h).

Argument marshalling only: every step of the path runs in the CUDA kernels behind the C
ABI.  There is no CPU fallback -- if the extension is missing this module raises.
PyTorch supplies device memory and streams (tensors are int32, CUDA, contiguous).

    import paper_conf_sc_alabandisbb23_b200 as E
    labels = E.ecl_scc(row_ptr, col_idx)             # row_ptr/col_idx: torch.int32 cuda
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libeclscc.so")

OK, EINVAL, ERANGE, ENOMEM, ECUDA, ENCCL, EUNSUPPORTED = range(7)
NO_TRIM, NO_VALIDATE, SYNC_PASSES, TIME_STAGES = 0x1, 0x4, 0x8, 0x10
IDENTITY_IDS, NO_DIRTY, NO_REORDER = 0x20, 0x40, 0x200
FORCE_REORDER, NO_PACK, NO_ASYNC = 0x400, 0x800, 0x1000
TRIM2, FOUR_SIG, HALO_ALLREDUCE, COMPRESS, RAISE, CLUSTER = 0x4000, 0x8000, 0x10000, 0x2, 0x20000, 0x40000
NO_KW = 0x80000
TRACE_MAX = 64

_lib = None


class EclSccError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        super().__init__(f"{where}: status {status} ({status_string(status)}): {msg}")
        self.status = status


class Stats(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_int32), ("trace_len", ctypes.c_int32),
                ("passes", ctypes.c_int64),
                ("edges_in", ctypes.c_int64 * TRACE_MAX), ("vertices_in", ctypes.c_int64 * TRACE_MAX),
                ("edges_kept", ctypes.c_int64 * TRACE_MAX), ("passes_iter", ctypes.c_int64 * TRACE_MAX),
                ("prop_bytes", ctypes.c_int64), ("kernel_launches", ctypes.c_int64),
                ("ms_ingest", ctypes.c_double), ("ms_compact", ctypes.c_double), ("ms_prop", ctypes.c_double),
                ("ms_prop_iter", ctypes.c_double * TRACE_MAX), ("ms_compact_iter", ctypes.c_double * TRACE_MAX),
                ("ms_comm", ctypes.c_double), ("comm_bytes", ctypes.c_int64), ("exchanges", ctypes.c_int64)]

    def as_dict(self) -> dict:
        k = self.trace_len
        return dict(iterations=self.iterations, passes=self.passes, prop_bytes=self.prop_bytes,
                    kernel_launches=self.kernel_launches, ms_ingest=self.ms_ingest,
                    ms_compact=self.ms_compact, ms_prop=self.ms_prop,
                    edges_in=list(self.edges_in[:k]), vertices_in=list(self.vertices_in[:k]),
                    edges_kept=list(self.edges_kept[:max(k - 1, 0)]),
                    passes_iter=list(self.passes_iter[:k]),
                    ms_prop_iter=[round(x, 4) for x in self.ms_prop_iter[:k]],
                    ms_compact_iter=[round(x, 4) for x in self.ms_compact_iter[:k + 1]],
                    ms_comm=self.ms_comm, comm_bytes=self.comm_bytes, exchanges=self.exchanges)


def lib() -> ctypes.CDLL:
    """Load libeclscc.so (built by __graft_entry__.build() / build.py).  Raises if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} is missing: run `python -m paper_conf_sc_alabandisbb23_b200.build` "
                          "(the CUDA extension is required; there is no CPU fallback)")
    L = ctypes.CDLL(_LIB_PATH)
    vp, i32, i64, u32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
    sig = {
        "ecl_scc": [i32, i64, vp, vp, vp],
        "ecl_scc_async": [i32, i64, vp, vp, vp, vp, vp, vp],
        "ecl_scc_debug_run": [i32, i64, vp, vp, u32, i32, vp, vp, vp, vp],
        "ecl_scc_plan_create": [i32, i64, u32, vp],
        "ecl_scc_plan_destroy": [vp],
        "ecl_scc_batched": [i32, vp, vp, vp, vp, vp, vp, vp, vp],
        "ecl_scc_batched_host": [i32, vp, vp, vp, vp, vp, vp, vp, vp],
        "ecl_scc_get_unique_id": [vp],
        "ecl_scc_comm_create": [i32, i32, vp, vp],
        "ecl_scc_comm_destroy": [vp],
        "ecl_scc_partitioned": [vp, i32, i32, i32, i64, vp, vp, vp, vp, vp, vp],
        "ecl_scc_part_plan_create": [i32, i32, i32, i64, u32, vp],
        "ecl_scc_part_plan_destroy": [vp],
        "ecl_scc_partitioned_emulated": [i32, i32, i64, vp, vp, vp, u32, vp, vp, vp],
        "ecl_scc_emulated_plan_create": [i32, i32, i64, vp, u32, vp],
        "ecl_scc_emulated_plan_destroy": [vp],
        "ecl_scc_comm_info": [vp, vp],
        "ecl_scc_multimem_probe": [vp],
        "ecl_scc_partition_rows": [i32, i32, vp, vp],
        "ecl_scc_status_string": [ctypes.c_int],
        "ecl_scc_last_error": [],
        "ecl_scc_version": [],
        "ecl_scc_plan_counters": [vp, vp],
        "ecl_scc_levels": [i32, i64, vp, vp, vp, vp, vp, vp, vp],
        "ecl_scc_host": [i32, i64, vp, vp, vp, vp, vp, vp],
    }
    for name, args in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    L.ecl_scc_status_string.restype = ctypes.c_char_p
    L.ecl_scc_last_error.restype = ctypes.c_char_p
    _lib = L
    return L


# names exported by include/ecl_scc.h (the CPU test checks the .so exports all of them)
ABI_SYMBOLS = ("ecl_scc", "ecl_scc_async", "ecl_scc_debug_run", "ecl_scc_plan_create",
               "ecl_scc_plan_destroy", "ecl_scc_batched", "ecl_scc_batched_host", "ecl_scc_get_unique_id",
               "ecl_scc_comm_create", "ecl_scc_comm_destroy", "ecl_scc_partitioned",
               "ecl_scc_partitioned_emulated", "ecl_scc_partition_rows", "ecl_scc_status_string",
               "ecl_scc_last_error", "ecl_scc_version", "ecl_scc_plan_counters", "ecl_scc_levels",
               "ecl_scc_host", "ecl_scc_part_plan_create", "ecl_scc_part_plan_destroy", "ecl_scc_comm_info",
               "ecl_scc_emulated_plan_create", "ecl_scc_emulated_plan_destroy", "ecl_scc_multimem_probe")


def status_string(s: int) -> str:
    return lib().ecl_scc_status_string(s).decode()


def _check(status: int, where: str):
    if status != OK:
        raise EclSccError(status, where, lib().ecl_scc_last_error().decode())


def _dev_i32(t: torch.Tensor, name: str) -> int:
    if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != torch.int32 or not t.is_contiguous():
        raise TypeError(f"{name} must be a contiguous torch.int32 CUDA tensor")
    return t.data_ptr()


def _stream(stream) -> int:
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


class Plan:
    """Reusable workspace (ecl_scc_plan_t) for graphs up to n_max vertices / nnz_max edges."""

    def __init__(self, n_max: int, nnz_max: int, flags: int = 0):
        h = ctypes.c_void_p()
        _check(lib().ecl_scc_plan_create(n_max, nnz_max, flags, ctypes.byref(h)), "ecl_scc_plan_create")
        self.handle, self.n_max, self.nnz_max, self.flags = h, n_max, nnz_max, flags

    def counters(self) -> list[int]:
        """Kernel event counters of the last run (non-zero only in -DECL_PROF builds)."""
        out = (ctypes.c_uint64 * 8)()
        _check(lib().ecl_scc_plan_counters(self.handle, out), "ecl_scc_plan_counters")
        return list(out)

    def close(self):
        if self.handle:
            lib().ecl_scc_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def ecl_scc(row_ptr: torch.Tensor, col_idx: torch.Tensor, labels_out: torch.Tensor | None = None,
            stream=None, plan: Plan | None = None, stats: bool = False):
    """SCC labels (largest vertex ID of each SCC) of the CSR graph on the GPU.

    Returns labels (and a stats dict if stats=True).  Calls ecl_scc_async on `stream`
    (default: torch's current stream)."""
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    if labels_out is None:
        labels_out = torch.empty(max(n, 0), dtype=torch.int32, device=row_ptr.device)
    st = Stats() if stats else None
    _check(lib().ecl_scc_async(n, nnz, _dev_i32(row_ptr, "row_ptr"), _dev_i32(col_idx, "col_idx") if nnz else None,
                               _dev_i32(labels_out, "labels_out"), _stream(stream),
                               plan.handle if plan else None, ctypes.byref(st) if st else None), "ecl_scc")
    return (labels_out, st.as_dict()) if stats else labels_out


def ecl_scc_host(row_ptr: torch.Tensor, col_idx: torch.Tensor, labels_out: torch.Tensor | None = None,
                 stream=None, plan: Plan | None = None, stats: bool = False):
    """ecl_scc on HOST (CPU, preferably pinned) tensors: the library copies the CSR in, runs,
    and copies the labels back (ecl_scc_host).  Returns labels (host) and optional stats."""
    for t, nm in ((row_ptr, "row_ptr"), (col_idx, "col_idx")):
        if t.device.type != "cpu" or t.dtype != torch.int32 or not t.is_contiguous():
            raise ValueError(f"{nm} must be a contiguous int32 CPU tensor")
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    if labels_out is None:
        labels_out = torch.empty(max(n, 0), dtype=torch.int32).pin_memory()
    st = Stats() if stats else None
    _check(lib().ecl_scc_host(n, nnz, row_ptr.data_ptr(), col_idx.data_ptr() if nnz else None,
                              labels_out.data_ptr(), _stream(stream), plan.handle if plan else None,
                              ctypes.byref(st) if st else None), "ecl_scc_host")
    return (labels_out, st.as_dict()) if stats else labels_out


def ecl_scc_levels(row_ptr: torch.Tensor, col_idx: torch.Tensor, labels: torch.Tensor,
                   levels_out: torch.Tensor | None = None, stream=None, plan: Plan | None = None):
    """Sweep levels of the SCC condensation (Table 2 "DAG depth"): returns (levels per
    vertex = longest condensation path ending in its SCC, depth = max level + 1).  `labels`
    are ecl_scc()'s output for the same graph."""
    n = row_ptr.numel() - 1
    nnz = col_idx.numel()
    if levels_out is None:
        levels_out = torch.empty(max(n, 0), dtype=torch.int32, device=row_ptr.device)
    depth = ctypes.c_int32(0)
    _check(lib().ecl_scc_levels(n, nnz, _dev_i32(row_ptr, "row_ptr"), _dev_i32(col_idx, "col_idx") if nnz else None,
                                _dev_i32(labels, "labels"), _dev_i32(levels_out, "levels_out"),
                                ctypes.byref(depth), _stream(stream), plan.handle if plan else None),
           "ecl_scc_levels")
    return levels_out, int(depth.value)


def ecl_scc_debug_run(row_ptr: torch.Tensor, col_idx: torch.Tensor, stop_iter: int, flags: int = 0, stream=None):
    """Signatures (v_in, v_out) after Phase 2 of outer iteration `stop_iter`, plus stats."""
    n = row_ptr.numel() - 1
    sin = torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    sout = torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    st = Stats()
    _check(lib().ecl_scc_debug_run(n, col_idx.numel(), _dev_i32(row_ptr, "row_ptr"),
                                   _dev_i32(col_idx, "col_idx") if col_idx.numel() else None, flags, stop_iter,
                                   _dev_i32(sin, "sig_in"), _dev_i32(sout, "sig_out"), _stream(stream),
                                   ctypes.byref(st)), "ecl_scc_debug_run")
    return sin, sout, st.as_dict()


def ecl_scc_batched(graphs, labels_out=None, stream=None, plan: Plan | None = None, stats: bool = False):
    """graphs: list of (row_ptr, col_idx) CUDA int32 tensors.  Returns per-graph local labels."""
    G = len(graphs)
    ns = (ctypes.c_int32 * max(G, 1))(*[g[0].numel() - 1 for g in graphs])
    ms = (ctypes.c_int64 * max(G, 1))(*[g[1].numel() for g in graphs])
    if labels_out is None:
        labels_out = [torch.empty(g[0].numel() - 1, dtype=torch.int32, device=g[0].device) for g in graphs]
    rps = (ctypes.c_void_p * max(G, 1))(*[_dev_i32(g[0], "row_ptr") for g in graphs])
    cis = (ctypes.c_void_p * max(G, 1))(*[_dev_i32(g[1], "col_idx") if g[1].numel() else None for g in graphs])
    los = (ctypes.c_void_p * max(G, 1))(*[_dev_i32(l, "labels_out") if l.numel() else None for l in labels_out])
    st = Stats() if stats else None
    _check(lib().ecl_scc_batched(G, ns, ms, rps, cis, los, _stream(stream), plan.handle if plan else None,
                                 ctypes.byref(st) if st else None), "ecl_scc_batched")
    return (labels_out, st.as_dict()) if stats else labels_out


def ecl_scc_batched_host(graphs, labels_out=None, stream=None, plan: Plan | None = None, stats: bool = False):
    """ecl_scc_batched on HOST (CPU, preferably pinned) tensors: graphs = list of (row_ptr,
    col_idx) int32 CPU tensors; the library copies the batch in, runs the union and copies
    every graph's local labels back (ecl_scc_batched_host)."""
    G = len(graphs)
    for rp, ci in graphs:
        for t, nm in ((rp, "row_ptr"), (ci, "col_idx")):
            if t.device.type != "cpu" or t.dtype != torch.int32 or not t.is_contiguous():
                raise ValueError(f"{nm} must be a contiguous int32 CPU tensor")
    ns = (ctypes.c_int32 * max(G, 1))(*[g[0].numel() - 1 for g in graphs])
    ms = (ctypes.c_int64 * max(G, 1))(*[g[1].numel() for g in graphs])
    if labels_out is None:
        labels_out = [torch.empty(g[0].numel() - 1, dtype=torch.int32).pin_memory() for g in graphs]
    rps = (ctypes.c_void_p * max(G, 1))(*[g[0].data_ptr() for g in graphs])
    cis = (ctypes.c_void_p * max(G, 1))(*[g[1].data_ptr() if g[1].numel() else None for g in graphs])
    los = (ctypes.c_void_p * max(G, 1))(*[l.data_ptr() if l.numel() else None for l in labels_out])
    st = Stats() if stats else None
    _check(lib().ecl_scc_batched_host(G, ns, ms, rps, cis, los, _stream(stream), plan.handle if plan else None,
                                      ctypes.byref(st) if st else None), "ecl_scc_batched_host")
    return (labels_out, st.as_dict()) if stats else labels_out


def ecl_scc_partition_rows(P: int, row_ptr_host) -> list[int]:
    """Balanced contiguous row ranges (host helper of the partitioned mode)."""
    import numpy as np
    rp = np.ascontiguousarray(row_ptr_host, dtype=np.int32)
    out = np.zeros(P + 1, dtype=np.int32)
    _check(lib().ecl_scc_partition_rows(P, rp.shape[0] - 1, rp.ctypes.data, out.ctypes.data), "ecl_scc_partition_rows")
    return out.tolist()


class EmulatedPlan:
    """Workspaces of P emulated ranks (ecl_scc_emulated_plan_t) for one graph size and flags."""

    def __init__(self, P: int, row_ptr: torch.Tensor, nnz: int, flags: int = 0):
        h = ctypes.c_void_p()
        _check(lib().ecl_scc_emulated_plan_create(P, row_ptr.numel() - 1, nnz, _dev_i32(row_ptr, "row_ptr"), flags,
                                                  ctypes.byref(h)), "ecl_scc_emulated_plan_create")
        self.handle = h

    def close(self):
        if self.handle:
            lib().ecl_scc_emulated_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def ecl_scc_partitioned_emulated(P: int, row_ptr, col_idx, labels_out=None, stream=None, stats: bool = False,
                                 flags: int = 0, plan: EmulatedPlan | None = None):
    n = row_ptr.numel() - 1
    if labels_out is None:
        labels_out = torch.empty(n, dtype=torch.int32, device=row_ptr.device)
    st = Stats() if stats else None
    _check(lib().ecl_scc_partitioned_emulated(P, n, col_idx.numel(), _dev_i32(row_ptr, "row_ptr"),
                                              _dev_i32(col_idx, "col_idx") if col_idx.numel() else None,
                                              _dev_i32(labels_out, "labels_out"), flags, _stream(stream),
                                              plan.handle if plan else None,
                                              ctypes.byref(st) if st else None), "ecl_scc_partitioned_emulated")
    return (labels_out, st.as_dict()) if stats else labels_out


def multimem_probe() -> int:
    """Run ecl_scc_multimem_probe: the NVLS multimem push path on this device alone (raises
    EclSccError with status EUNSUPPORTED when the device has no multicast support)."""
    n = ctypes.c_int32(0)
    _check(lib().ecl_scc_multimem_probe(ctypes.byref(n)), "ecl_scc_multimem_probe")
    return int(n.value)


def get_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(lib().ecl_scc_get_unique_id(buf), "ecl_scc_get_unique_id")
    return bytes(buf)


class Comm:
    """NCCL communicator for the edge-partitioned mode (one rank per GPU)."""

    def __init__(self, nranks: int, rank: int, uid: bytes):
        h = ctypes.c_void_p()
        buf = (ctypes.c_uint8 * 128)(*uid)
        _check(lib().ecl_scc_comm_create(nranks, rank, buf, ctypes.byref(h)), "ecl_scc_comm_create")
        self.handle, self.nranks, self.rank = h, nranks, rank

    def info(self) -> dict:
        """ranks, rank, and whether the fused halo exchange uses the NCCL device API / NVLS."""
        out = (ctypes.c_int32 * 4)()
        _check(lib().ecl_scc_comm_info(self.handle, out), "ecl_scc_comm_info")
        return dict(nranks=out[0], rank=out[1], device_api=bool(out[2]), multimem=bool(out[3]))

    def close(self):
        if self.handle:
            lib().ecl_scc_comm_destroy(self.handle)
            self.handle = None


class PartPlan:
    """Per-rank workspace of the partitioned mode (ecl_scc_part_plan_t): rows [row_begin,
    row_end) of an n-vertex graph, at most local_nnz_max local edges."""

    def __init__(self, comm, n: int, row_begin: int, row_end: int, local_nnz_max: int, flags: int = 0):
        h = ctypes.c_void_p()
        _check(lib().ecl_scc_part_plan_create(n, row_begin, row_end, local_nnz_max, flags, ctypes.byref(h)),
               "ecl_scc_part_plan_create")
        self.handle = h

    def close(self):
        if self.handle:
            lib().ecl_scc_part_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def ecl_scc_partitioned(comm: Comm, n: int, row_begin: int, row_end: int, local_row_ptr, local_col_idx,
                        labels_out=None, stream=None, plan: PartPlan | None = None, stats: bool = False):
    if labels_out is None:
        labels_out = torch.empty(n, dtype=torch.int32, device=local_row_ptr.device)
    st = Stats() if stats else None
    nnz = local_col_idx.numel()
    _check(lib().ecl_scc_partitioned(comm.handle, n, row_begin, row_end, nnz, _dev_i32(local_row_ptr, "local_row_ptr"),
                                     _dev_i32(local_col_idx, "local_col_idx") if nnz else None,
                                     _dev_i32(labels_out, "labels_out"), _stream(stream),
                                     plan.handle if plan else None, ctypes.byref(st) if st else None),
           "ecl_scc_partitioned")
    return (labels_out, st.as_dict()) if stats else labels_out
