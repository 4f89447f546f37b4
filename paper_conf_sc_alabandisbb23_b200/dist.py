"""Host-side plumbing of the multi-GPU modes (torch.distributed for process groups only).

* edge-partitioned single graph: ``split_rows`` (balanced source-row ranges, the C ABI's
  ecl_scc_partition_rows), ``local_csr`` (a rank's rows with rebased offsets and global
  column IDs), ``share_unique_id`` (the NCCL id travels over the torch process group,
  because torch does not expose its own ncclComm_t).
* batched graphs (one per discrete ordinate): ``split_batch`` gives rank r the
  graphs [G*r/P, G*(r+1)/P) -- no collective on the data path.
* timing: ``max_over_ranks`` (every multi-GPU number is the max over ranks).
"""
from __future__ import annotations

import numpy as np


def split_rows(P: int, row_ptr) -> list[int]:
    from . import ecl_scc_partition_rows
    return ecl_scc_partition_rows(P, np.asarray(row_ptr))


def local_csr(row_ptr, col_idx, rb: int, re: int) -> tuple[np.ndarray, np.ndarray]:
    rp = np.asarray(row_ptr)
    lo, hi = int(rp[rb]), int(rp[re])
    return (rp[rb:re + 1] - lo).astype(np.int32), np.ascontiguousarray(np.asarray(col_idx)[lo:hi], dtype=np.int32)


def split_batch(G: int, P: int, r: int) -> range:
    return range(G * r // P, G * (r + 1) // P)


def share_unique_id(dist, rank: int, make_id) -> bytes:
    """Rank 0 creates the 128-byte NCCL id, everyone receives it over the process group."""
    box = [make_id() if rank == 0 else None]
    dist.broadcast_object_list(box, src=0)
    return box[0]


def max_over_ranks(dist, value: float, device=None) -> float:
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
