"""Host-resident problems through the hot path with the PCIe transfers overlapped.

``HostPipeline`` takes a CSR matrix and a dense B that live in (pinned) host
memory, runs configure -> CSR->CELL build -> CELL SpMM on the GPU (the same
C-ABI calls as ``CellMatrix``) and returns C in host memory.  Consecutive
submissions are double-buffered over three CUDA streams:

    h2d stream      copy problem k+1's CSR and B into device slot (k+1) % 2
    compute stream  configure / build / SpMM of problem k in slot k % 2
    d2h stream      copy problem k-1's C back to its host buffer

so the host->device copy of the next problem, the device->host copy of the
previous result (PCIe is full duplex) and the GPU work of the current one
overlap.  Events order every reuse of a slot.  Streams and memory come from
PyTorch; every compute step runs in liblf.so.
"""
from __future__ import annotations

import torch

from . import CellMatrix, Csr, configure


class HostPipeline:
    def __init__(self, n_rows: int, n_cols: int, max_nnz: int, J: int, device=None, **configure_kw):
        self.dev = torch.device(device if device is not None else "cuda")
        self.n_rows, self.n_cols, self.J = int(n_rows), int(n_cols), int(J)
        self.kw = configure_kw
        mk = lambda n, dt: torch.empty(n, dtype=dt, device=self.dev)  # noqa: E731
        self.slots = [dict(rp=mk(self.n_rows + 1, torch.int64), ci=mk(max(max_nnz, 1), torch.int32),
                           va=mk(max(max_nnz, 1), torch.float32), B=mk((self.n_cols, self.J), torch.float32),
                           C=mk((self.n_rows, self.J), torch.float32)) for _ in range(2)]
        self.s_h2d = torch.cuda.Stream(self.dev)
        self.s_cmp = torch.cuda.Stream(self.dev)
        self.s_d2h = torch.cuda.Stream(self.dev)
        ev = lambda: [torch.cuda.Event(), torch.cuda.Event()]  # noqa: E731
        self.h2d_done, self.cmp_done, self.d2h_done = ev(), ev(), ev()
        self.k = 0
        self.last_params = None

    def submit(self, h_rp: torch.Tensor, h_ci: torch.Tensor, h_va: torch.Tensor, h_B: torch.Tensor,
               h_C: torch.Tensor) -> torch.cuda.Event:
        """Enqueue one problem: host CSR (row_ptr starting at 0) and B in, C out
        into h_C (pinned, [n_rows, J]).  Returns the event that completes when
        h_C holds the result.  The host blocks only inside configure (its two
        small statistics copies), never on the transfers."""
        s = self.k % 2
        slot = self.slots[s]
        nnz = int(h_ci.numel())
        if self.k >= 2:  # slot s was last used by problem k-2
            self.s_h2d.wait_event(self.cmp_done[s])
        with torch.cuda.stream(self.s_h2d):
            slot["rp"].copy_(h_rp, non_blocking=True)
            slot["ci"][:nnz].copy_(h_ci, non_blocking=True)
            slot["va"][:nnz].copy_(h_va, non_blocking=True)
            slot["B"].copy_(h_B, non_blocking=True)
            self.h2d_done[s].record(self.s_h2d)
        self.s_cmp.wait_event(self.h2d_done[s])
        if self.k >= 2:  # C of slot s drained to the host
            self.s_cmp.wait_event(self.d2h_done[s])
        with torch.cuda.stream(self.s_cmp):
            A = Csr(slot["rp"], slot["ci"][:nnz], slot["va"][:nnz], self.n_cols, nnz)
            params, stats = configure(A, self.J, stream=self.s_cmp, **self.kw)
            M = CellMatrix.build(A, params, stats, stream=self.s_cmp)
            M.spmm(slot["B"], out=slot["C"], stream=self.s_cmp)
            M.close()
            self.cmp_done[s].record(self.s_cmp)
        self.last_params = params
        self.s_d2h.wait_event(self.cmp_done[s])
        with torch.cuda.stream(self.s_d2h):
            h_C.copy_(slot["C"], non_blocking=True)
            self.d2h_done[s].record(self.s_d2h)
        self.k += 1
        return self.d2h_done[s]

    def synchronize(self):
        for st in (self.s_h2d, self.s_cmp, self.s_d2h):
            st.synchronize()
