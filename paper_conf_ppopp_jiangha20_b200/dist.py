"""Row-panel sharding across GPUs (north_star).

One process per GPU (torchrun).  Every rank builds the same plan (the reorder is
deterministic per seed) and keeps its nnz-balanced contiguous panel range
(`sr_reorder(world, rank)`); B/X/Y are replicated.  The step needs no collective.  When the
caller wants the full C (or the full SDDMM values) on every rank, `gather_spmm` /
`gather_sddmm` all-gather the packed shard outputs (NCCL over NVLink via
torch.distributed, padded to the largest shard) and scatter them back to original
positions with libsr's scatter kernels.
"""
from __future__ import annotations

import torch
import torch.distributed as tdist

import paper_conf_ppopp_jiangha20_b200 as sr


def allgather_padded(t: torch.Tensor, group=None) -> list:
    """All-gather tensors whose first dimension differs across ranks: pad to the maximum,
    all_gather_into_tensor, return the list of unpadded pieces in rank order."""
    world = tdist.get_world_size(group)
    n = torch.tensor([t.shape[0]], dtype=torch.int64, device=t.device)
    sizes = [torch.zeros_like(n) for _ in range(world)]
    tdist.all_gather(sizes, n, group=group)
    sizes = [int(s.item()) for s in sizes]
    mx = max(sizes)
    pad = torch.zeros((mx,) + tuple(t.shape[1:]), dtype=t.dtype, device=t.device)
    pad[: t.shape[0]] = t
    buf = torch.empty((world * mx,) + tuple(t.shape[1:]), dtype=t.dtype, device=t.device)
    tdist.all_gather_into_tensor(buf, pad, group=group)
    return [buf[r * mx: r * mx + sizes[r]] for r in range(world)]


def gather_spmm(M: "sr.SparseMatrix", C_local: torch.Tensor, group=None) -> torch.Tensor:
    """Full C (original row order) on every rank from the packed shard outputs."""
    rows = torch.from_numpy(M.shard_rows()).to(C_local.device)
    pieces = allgather_padded(C_local, group)
    ids = allgather_padded(rows, group)
    C = torch.empty((M.nrows, C_local.shape[1]), dtype=C_local.dtype, device=C_local.device)
    for piece, rid in zip(pieces, ids):
        sr.scatter_rows(piece, rid.to(torch.int32).contiguous(), C)
    return C


def gather_sddmm(M: "sr.SparseMatrix", out_local: torch.Tensor, group=None) -> torch.Tensor:
    """Full SDDMM values (caller's nnz order) on every rank from the packed shard outputs."""
    ids = torch.from_numpy(M.shard_nnz_ids()).to(out_local.device)
    pieces = allgather_padded(out_local, group)
    idp = allgather_padded(ids, group)
    out = torch.empty(M.nnz, dtype=out_local.dtype, device=out_local.device)
    for piece, i in zip(pieces, idp):
        sr.scatter_values(piece.contiguous(), i.contiguous(), out)
    return out
