"""Paper-design comparator: EL-Rec's Eff-TT table as the paper builds it, on the same B200.

This is NOT the product path (that is libttemb.so); it is the in-run "paper's own design"
baseline of SURVEY.md 8(f1).  It follows the paper's GPU design with stock library
calls, the way P:346 describes its implementation ("cuBLAS batched GEMM"):

  forward  (Alg. 1; Fig. 5(b)):
    per table: Buf_idx = idx / m3 -> the unique prefixes of the batch are the
    Reuse buffer (the flag claim of Alg. 1 is done with torch.unique: one owner per
    prefix), stage 1 = batched GEMM C1[i1] (n1 x R) . C2[i2] (R x n2 R) per unique prefix
    (P:178), stage 2 = batched GEMM P[prefix(idx)] (n1 n2 x R) . C3[i3] (R x n3) per
    unique index (sample-level reuse, Eq. 5, is subsumed by the dedup), then sum pooling
    (Eq. 4) with index_add.
  backward (Fig. 6):
    in-advance gradient aggregation per unique index with index_add, then the
    TT core gradients of every unique index by batched GEMMs (Eq. 6 read as
    left^T . dL/de . right^T, R6) -- per unique index, without the per-prefix
    dP aggregation of our kernels --, reduction into the dense core-gradient buffer with
    index_add (Fig. 6(a) step 2), and the SGD update of the touched slices.

fp32 throughout (TF32 disabled), so it is checked against the oracle at the same
tolerances as the CUDA path (tests/test_paper_comparator.py).
Everything is torch / cuBLAS: it exists to put a number for "the paper's design on
this GPU" next to ours, and is imported only by bench.py (--impl paper) and tests.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

import torch


class PaperDesignTT:
    """Table-batched TT-EmbeddingBag (sum pooling), the paper's design in torch/cuBLAS."""

    def __init__(self, table_rows: Sequence[int], row_factors: Sequence[Tuple[int, int, int]],
                 col_factors: Tuple[int, int, int], rank: int, device):
        self.table_rows = [int(x) for x in table_rows]
        self.row_factors = [tuple(int(y) for y in f) for f in row_factors]
        self.n1, self.n2, self.n3 = (int(x) for x in col_factors)
        self.N = self.n1 * self.n2 * self.n3
        self.R = int(rank)
        self.T = len(self.table_rows)
        self.device = torch.device(device)
        self.cores: List[List[torch.Tensor]] = []
        self.grads: List[List[torch.Tensor]] = []
        self._saved = None

    def load_cores(self, cores) -> None:
        """cores: per table (C1[m1][n1][R], C2[m2][R][n2][R], C3[m3][R][n3]) (R4)."""
        self.cores = [[torch.as_tensor(c, dtype=torch.float32, device=self.device).contiguous()
                       for c in tab] for tab in cores]
        self.grads = [[torch.zeros_like(c) for c in tab] for tab in self.cores]

    def forward(self, indices: torch.Tensor, offsets: torch.Tensor, batch: int) -> torch.Tensor:
        n1, n2, n3, R, N, T = self.n1, self.n2, self.n3, self.R, self.N, self.T
        out = torch.zeros(batch, T, N, dtype=torch.float32, device=self.device)
        saved = []
        offsets = offsets.cpu()            # bag boundaries on the host (slicing); no-op if already there
        for t in range(T):
            m1, m2, m3 = self.row_factors[t]
            lo, hi = int(offsets[t * batch]), int(offsets[(t + 1) * batch])
            if hi == lo:
                saved.append(None)
                continue
            idx = indices[lo:hi]
            lens = (offsets[t * batch + 1:(t + 1) * batch + 1] - offsets[t * batch:(t + 1) * batch]).to(self.device)
            bag = torch.repeat_interleave(torch.arange(batch, device=self.device), lens)
            urow, inv = torch.unique(idx, return_inverse=True)            # unique indices
            pfx = torch.div(urow, m3, rounding_mode="floor")              # Buf_idx = idx / length_3
            upfx, pinv = torch.unique(pfx, return_inverse=True)           # Reuse buffer owners
            i1 = torch.div(upfx, m2, rounding_mode="floor")
            i2 = upfx - i1 * m2
            i3 = urow - pfx * m3
            C1, C2, C3 = self.cores[t]
            A = C1[i1]                                                    # [P, n1, R]
            Bm = C2[i2].reshape(-1, R, n2 * R)                            # [P, R, n2 R]
            Pbuf = torch.bmm(A, Bm).reshape(-1, n1 * n2, R)               # stage 1
            Pr = Pbuf[pinv]                                               # [U, n1 n2, R]
            E = torch.bmm(Pr, C3[i3]).reshape(-1, N)                      # stage 2 (Fig. 5(b) step 3)
            out[:, t, :].index_add_(0, bag, E[inv])                       # Eq. 4 (step 4)
            saved.append((bag, inv, i1, i2, i3, pinv, Pr, A, Bm))
        self._saved = saved
        self.batch = batch
        return out

    def backward(self, grad_out: torch.Tensor) -> None:
        n1, n2, n3, R, N = self.n1, self.n2, self.n3, self.R, self.N
        for t, sv in enumerate(self._saved):
            g1, g2, g3 = self.grads[t]
            g1.zero_(); g2.zero_(); g3.zero_()
            if sv is None:
                continue
            bag, inv, i1, i2, i3, pinv, Pr, A, Bm = sv
            U = Pr.shape[0]
            G = torch.zeros(U, N, dtype=torch.float32, device=self.device)
            G.index_add_(0, inv, grad_out[bag, t, :])                     # in-advance aggregation
            G = G.reshape(U, n1 * n2, n3)
            C3 = self.cores[t][2]
            # dC3[i3] += P^T G ;  dP = G C3[i3]^T   (Eq. 6, R6)
            g3.index_add_(0, i3, torch.bmm(Pr.transpose(1, 2), G))
            dP = torch.bmm(G, C3[i3].transpose(1, 2)).reshape(U, n1, n2 * R)
            # dC2[i2] += C1[i1]^T dP ;  dC1[i1] += dP C2[i2]^T   per unique index (no prefix aggregation)
            Ar, Br = A[pinv], Bm[pinv]
            g2.index_add_(0, i2[pinv], torch.bmm(Ar.transpose(1, 2), dP).reshape(U, R, n2, R))
            g1.index_add_(0, i1[pinv], torch.bmm(dP, Br.transpose(1, 2)))

    def update_sgd(self, lr: float) -> None:
        """C -= lr dC on every core (untouched slices have zero gradient)."""
        for tab, gt in zip(self.cores, self.grads):
            for c, g in zip(tab, gt):
                c.add_(g, alpha=-lr)
