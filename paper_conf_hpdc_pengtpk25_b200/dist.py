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


def exchange_rows(C: torch.Tensor, bounds, group=None) -> torch.Tensor:
    """In place: C is the full [I, J] result on every rank, whose rows
    [bounds[rank], bounds[rank+1]) this rank computed.  Every rank sends its
    block to every peer and receives theirs straight into their rows (one
    batched set of point-to-point transfers, exact sizes: no padding and no
    staging copy; NCCL over NVLink/NVSwitch on GPUs)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    if world == 1:
        return C
    b = [int(x) for x in bounds]
    mine = C[b[rank]:b[rank + 1]]
    ops = []
    for r in range(world):
        if r == rank:
            continue
        peer = dist.get_global_rank(group, r) if group is not None else r
        if b[rank + 1] > b[rank]:
            ops.append(dist.P2POp(dist.isend, mine, peer, group))
        if b[r + 1] > b[r]:
            ops.append(dist.P2POp(dist.irecv, C[b[r]:b[r + 1]], peer, group))
    if ops:
        for req in dist.batch_isend_irecv(ops):
            req.wait()
    return C


def gather_rows(C_local: torch.Tensor, bounds, group=None) -> torch.Tensor:
    """All-gather the ranks' row blocks of C into a new full [I, J] matrix
    (exchange_rows after placing the local block)."""
    rank = dist.get_rank(group)
    b = [int(x) for x in bounds]
    C = torch.empty((b[-1], C_local.shape[1]), dtype=C_local.dtype, device=C_local.device)
    C[b[rank]:b[rank + 1]] = C_local
    return exchange_rows(C, bounds, group)


def col_bounds(J: int, world: int, align: int = 4) -> np.ndarray:
    """world+1 column boundaries of B / C for the large-J mode:
    near-equal slabs, every inner boundary a multiple of `align` (so each
    slab keeps the 16-byte vector path of lf_spmm when J % 4 == 0)."""
    units = -(-int(J) // align)
    b = np.array([min(int(J), ((r * units) // world) * align) for r in range(world + 1)], np.int64)
    b[world] = int(J)
    return b


def gather_cols(C_slab: torch.Tensor, cbounds, group=None) -> torch.Tensor:
    """All-gather column slabs [I, J_r] into the full [I, J] C: one
    all_gather of the slabs (padded only when the slabs differ in width) and
    ONE permuting copy [world, I, w] -> [I, world * w] into C."""
    world = dist.get_world_size(group)
    cb = [int(x) for x in cbounds]
    widths = [cb[r + 1] - cb[r] for r in range(world)]
    wmax = max(widths)
    I = C_slab.shape[0]
    equal = all(w == wmax for w in widths)
    src = C_slab.contiguous() if equal else torch.nn.functional.pad(C_slab, (0, wmax - C_slab.shape[1]))
    buf = torch.empty((world, I, wmax), dtype=C_slab.dtype, device=C_slab.device)
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(buf, src, group=group)
    else:
        dist.all_gather(list(buf.unbind(0)), src, group=group)
    if equal:
        return buf.permute(1, 0, 2).reshape(I, cb[-1])
    C = torch.empty((I, cb[-1]), dtype=C_slab.dtype, device=C_slab.device)
    for r in range(world):
        C[:, cb[r]:cb[r + 1]] = buf[r, :, :widths[r]]
    return C


def broadcast_B(B: torch.Tensor, src: int = 0, group=None) -> torch.Tensor:
    dist.broadcast(B, src=src, group=group)
    return B


def symmetric_C(n_rows: int, J: int, device, group=None):
    """A full [n_rows, J] C on every rank in symmetric memory (peer-mapped
    over NVLink) and the device addresses of every rank's copy, rank order:
    the destinations of the fused row exchange.  None where the process group
    or device cannot provide symmetric memory."""
    try:
        import torch.distributed._symmetric_memory as symm
        C = symm.empty((n_rows, J), dtype=torch.float32, device=device)
        h = symm.rendezvous(C, group if group is not None else dist.group.WORLD)
        return C, h, [int(p) for p in h.buffer_ptrs]
    except Exception:  # pragma: no cover - depends on the box
        return None


def spmm_rowsharded_fused(A_full, B: torch.Tensor, J: int, group=None, mode: str = "nnz", **configure_kw):
    """C = A . B with A's rows sharded and the C rows exchanged INSIDE the SpMM
    (SURVEY 8(f) NEXT-3): every rank's kernels write their C rows straight into
    every rank's symmetric-memory C (lf_spmm_ex destinations = all peers'
    buffers over NVLink), so no all-gather follows the compute; a barrier over
    the symmetric-memory signal pads orders the reads.  Returns (C, bounds);
    falls back to spmm_rowsharded when symmetric memory is unavailable."""
    from . import CellMatrix, Csr, configure
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    sym = symmetric_C(A_full.n_rows, B.shape[1], B.device, group)
    if sym is None:
        return spmm_rowsharded(A_full, B, J, group, mode, True, **configure_kw)
    C, h, ptrs = sym
    rp_host = A_full.row_ptr.cpu().numpy()
    bounds = shard_bounds(rp_host, world, J, mode)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    shard = Csr(A_full.row_ptr[lo:hi + 1], A_full.col_ind, A_full.val, A_full.n_cols,
                int(rp_host[hi] - rp_host[lo]))
    params, stats = configure(shard, J, force_format=1, **configure_kw)
    M = CellMatrix.build(shard, params, stats)
    M.spmm(B, dst=ptrs, row_base=lo)
    if world > 1:
        h.barrier(channel=0)
    return C, bounds


def spmm_rowsharded(A_full, B: torch.Tensor, J: int, group=None, mode: str = "nnz", gather: bool = True,
                    **configure_kw):
    """C = A . B with A's rows sharded over the group.  A_full is this rank's
    handle on the whole CSR (lf.Csr on the local GPU); returns the full C (or
    the local block when gather=False) and the bounds.  The local SpMM writes
    straight into its rows of the full C, which exchange_rows completes."""
    from . import CellMatrix, Csr, configure
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    rp_host = A_full.row_ptr.cpu().numpy()
    bounds = shard_bounds(rp_host, world, J, mode)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    shard = Csr(A_full.row_ptr[lo:hi + 1], A_full.col_ind, A_full.val, A_full.n_cols,
                int(rp_host[hi] - rp_host[lo]))
    params, stats = configure(shard, J, **configure_kw)
    M = CellMatrix.build(shard, params, stats)
    if not gather:
        return M.spmm(B), bounds
    C = torch.empty((A_full.n_rows, B.shape[1]), dtype=torch.float32, device=B.device)
    M.spmm(B, out=C[lo:hi])
    return exchange_rows(C, bounds, group), bounds


def spmm_colsplit(A_full, B: torch.Tensor, group=None, gather: bool = True, **configure_kw):
    """Large-J mode: every rank holds all of A (one CELL
    handle) and multiplies its column slab of B, C[:, j0:j1] = A . B[:, j0:j1]
    (lf_spmm on strided views: ldb = ldc = J, no slab copies of B).  Returns
    the full C (or this rank's [I, j1-j0] slab when gather=False) and the
    column bounds."""
    from . import CellMatrix, configure
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    J = B.shape[1]
    cb = col_bounds(J, world)
    j0, j1 = int(cb[rank]), int(cb[rank + 1])
    params, stats = configure(A_full, max(j1 - j0, 1), **configure_kw)
    M = CellMatrix.build(A_full, params, stats)
    C_slab = M.spmm(B[:, j0:j1])
    if not gather:
        return C_slab, cb
    return gather_cols(C_slab, cb, group), cb
