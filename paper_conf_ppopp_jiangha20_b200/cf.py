"""Collaborative-filtering gradient descent over one reordered plan.

The paper's motivating iterative workload (Tables 3/4): matrix factorisation
R ≈ U·Vᵀ on the observed pattern Ω of a ratings matrix R (M users × N items), loss
    L = ½ Σ_{(i,j)∈Ω} (⟨U_i, V_j⟩ − r_ij)² + ½ λ (‖U‖² + ‖V‖²),
whose gradient is one SDDMM and two SpMMs per iteration:
    P   = SDDMM(Ω; U, V)          (values set to 1: P_ij = ⟨U_i, V_j⟩ on Ω, Alg 2)
    E   = P − R                   (on Ω, caller nnz order)
    ∇U  = E·V + λU                (SpMM over R's plan with values E, Alg 1)
    ∇V  = Eᵀ·U + λV               (SpMM over Rᵀ's plan with values Eᵀ)
The two plans (R and Rᵀ) are built once (LSH + Alg 3 + ASpT) and reused every iteration
through sr_set_values, which is how the preprocessing is amortised.  The sparse products
run in libsr's kernels; the O(nnz) residual and the O((M+N)·K) updates are PyTorch
elementwise ops (plumbing, not part of the §8(a) hot path).
"""
from __future__ import annotations

import numpy as np

from . import SparseMatrix, default_params


def transpose_csr(nrows: int, ncols: int, rowptr, colidx):
    """CSR of Aᵀ plus perm with (Aᵀ nnz t) = (A nnz perm[t]), columns sorted per row."""
    rowptr = np.asarray(rowptr, np.int64)
    colidx = np.asarray(colidx, np.int32)
    rows = np.repeat(np.arange(nrows, dtype=np.int32), np.diff(rowptr))
    perm = np.lexsort((rows, colidx)).astype(np.int64)  # by column, then row
    t_rowptr = np.zeros(ncols + 1, np.int64)
    np.cumsum(np.bincount(colidx, minlength=ncols), out=t_rowptr[1:])
    return t_rowptr, rows[perm].astype(np.int32), perm


class CFModel:
    """U (M×K), V (N×K) on one GPU with the plans of R and Rᵀ."""

    def __init__(self, R, K: int, device: int = 0, params=None, seed: int = 0, reorder: bool = True):
        import torch
        self.torch = torch
        self.dev = torch.device("cuda", device)
        self.K = K
        self.M, self.N, self.nnz = R.nrows, R.ncols, R.nnz
        self.r = torch.from_numpy(np.ascontiguousarray(R.vals, np.float32)).to(self.dev)
        t_rowptr, t_col, perm = transpose_csr(R.nrows, R.ncols, R.rowptr, R.colidx)
        self.tperm = torch.from_numpy(perm).to(self.dev)
        self.A = SparseMatrix(R.nrows, R.ncols, R.rowptr, R.colidx, R.vals, device)
        self.At = SparseMatrix(R.ncols, R.nrows, t_rowptr, t_col, np.asarray(R.vals, np.float32)[perm], device)
        self.plan_stats = None
        if reorder:
            p = params if params is not None else default_params()
            self.plan_stats = (self.A.reorder(p), self.At.reorder(p))
        g = torch.Generator(device="cpu").manual_seed(seed)
        self.U = (0.1 * torch.randn(self.M, K, generator=g)).to(self.dev)
        self.V = (0.1 * torch.randn(self.N, K, generator=g)).to(self.dev)
        self.ones = torch.ones(self.nnz, dtype=torch.float32, device=self.dev)
        self.P = torch.empty(self.nnz, dtype=torch.float32, device=self.dev)
        self.gU = torch.empty_like(self.U)
        self.gV = torch.empty_like(self.V)

    def gradients(self, lam: float = 0.0):
        """(E, ∇U, ∇V) at the current U, V (async on the current stream)."""
        self.A.set_values(self.ones)
        self.A.sddmm(self.U, self.V, self.P)            # P_ij = <U_i, V_j> on Ω
        E = self.P - self.r
        self.A.set_values(E)
        self.A.spmm(self.V, self.gU)                     # E·V
        self.At.set_values(E.index_select(0, self.tperm).contiguous())
        self.At.spmm(self.U, self.gV)                    # Eᵀ·U
        if lam:
            self.gU.add_(self.U, alpha=lam)
            self.gV.add_(self.V, alpha=lam)
        return E, self.gU, self.gV

    def step(self, lr: float, lam: float = 0.0) -> float:
        """One full-batch gradient step; returns the data loss ½ Σ E² before the step."""
        E, gU, gV = self.gradients(lam)
        loss = 0.5 * float(E.double().square().sum())
        self.U.sub_(gU, alpha=lr)
        self.V.sub_(gV, alpha=lr)
        return loss

    def close(self):
        self.A.close()
        self.At.close()
