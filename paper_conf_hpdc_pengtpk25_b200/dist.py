"""Row-sharded multi-GPU execution: one process per GPU.

Each C row depends only on its A row and B, so A is split into contiguous
row ranges (balanced by a per-row weight), every rank builds the CELL of its
own range (a row_ptr view: no copy), B is replicated (broadcast once), the
local SpMM writes the rank's C rows, and the rows are all-gathered over NCCL
(NVLink / NVSwitch).  Host-side logic here is backend-agnostic so it is
covered by world-size-2 gloo tests on CPU.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def row_weights(row_ptr: np.ndarray, J: int, mode: str = "nnz") -> np.ndarray:
    """Per-row balancing weight: nnz (ALU-bound inputs) or bytes 8*l + 4*J
    (HBM-bound inputs: index+value stream plus one C row)."""
    l = np.diff(np.asarray(row_ptr, dtype=np.int64))
    if mode == "nnz":
        return l
    if mode == "bytes":
        return 8 * l + 4 * int(J)
    raise ValueError(mode)


def shard_bounds(row_ptr: np.ndarray, world: int, J: int = 0, mode: str = "nnz") -> np.ndarray:
    """world+1 row boundaries: boundary r is the first row i whose cumulative
    weight reaches r/world of the total (contiguous, monotone, covers all rows)."""
    I = len(row_ptr) - 1
    w = row_weights(row_ptr, J, mode)
    cum = np.concatenate([[0], np.cumsum(w)])
    total = cum[-1]
    b = np.zeros(world + 1, np.int64)
    for r in range(1, world):
        b[r] = np.searchsorted(cum, r * total / world, side="left") if total > 0 else (r * I) // world
        b[r] = min(max(b[r], b[r - 1]), I)
    b[world] = I
    return b


def gather_rows(C_local: torch.Tensor, bounds, group=None) -> torch.Tensor:
    """All-gather the ranks' row blocks of C into the full [I, J] matrix.
    Shards are padded to the largest shard so a single all_gather_into_tensor
    (NCCL) moves them; the padding is dropped on unpacking."""
    world = dist.get_world_size(group)
    sizes = np.diff(np.asarray(bounds, np.int64))
    rmax = int(sizes.max()) if len(sizes) else 0
    J = C_local.shape[1]
    pad = torch.zeros((rmax, J), dtype=C_local.dtype, device=C_local.device)
    pad[:C_local.shape[0]] = C_local
    if dist.get_backend(group) == "nccl":
        buf = torch.empty((world * rmax, J), dtype=C_local.dtype, device=C_local.device)
        dist.all_gather_into_tensor(buf, pad, group=group)
        parts = [buf[r * rmax: r * rmax + int(sizes[r])] for r in range(world)]
    else:
        bufs = [torch.empty_like(pad) for _ in range(world)]
        dist.all_gather(bufs, pad, group=group)
        parts = [bufs[r][:int(sizes[r])] for r in range(world)]
    return torch.cat(parts, dim=0)


def broadcast_B(B: torch.Tensor, src: int = 0, group=None) -> torch.Tensor:
    dist.broadcast(B, src=src, group=group)
    return B


def spmm_rowsharded(A_full, B: torch.Tensor, J: int, group=None, mode: str = "nnz", gather: bool = True,
                    **configure_kw):
    """C = A . B with A's rows sharded over the group.  A_full is this rank's
    handle on the whole CSR (lf.Csr on the local GPU); returns the full C (or
    the local block when gather=False) and the bounds."""
    from . import CellMatrix, Csr, configure
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    rp_host = A_full.row_ptr.cpu().numpy()
    bounds = shard_bounds(rp_host, world, J, mode)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    shard = Csr(A_full.row_ptr[lo:hi + 1], A_full.col_ind, A_full.val, A_full.n_cols,
                int(rp_host[hi] - rp_host[lo]))
    params, stats = configure(shard, J, **configure_kw)
    M = CellMatrix.build(shard, params, stats)
    C_local = M.spmm(B)
    if not gather:
        return C_local, bounds
    return gather_rows(C_local, bounds, group), bounds
