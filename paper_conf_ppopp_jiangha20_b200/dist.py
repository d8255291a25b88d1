"""Row-panel sharding across GPUs (north_star).

One process per GPU (torchrun).  The plan is built once: rank 0 reorders the whole matrix
(`sr_reorder`), broadcasts the plan image (`broadcast_bytes`), and every rank installs its
nnz-balanced contiguous panel range with `sr_plan_load(world, rank)` (`load_shard`; the
reorder is deterministic per seed, so `sr_reorder(world, rank)` on every rank gives the same
shards at the cost of repeating it).  B/X/Y are replicated.  The step needs no collective.  When the
caller wants the full C (or the full SDDMM values) on every rank, `gather_spmm` /
`gather_sddmm` all-gather the packed shard outputs (NCCL over NVLink via
torch.distributed, padded to the largest shard) and scatter them back to original
positions with libsr's scatter kernels.
"""
from __future__ import annotations

import torch
import torch.distributed as tdist

import paper_conf_ppopp_jiangha20_b200 as sr


def broadcast_bytes(data: bytes | None, src: int = 0, group=None, device=None) -> bytes:
    """Broadcast a byte string from rank `src` (the plan image): its length, then the bytes as a
    uint8 tensor (on `device`: a CUDA device for NCCL, None = CPU for gloo)."""
    rank = tdist.get_rank(group)
    n = torch.tensor([len(data) if rank == src else 0], dtype=torch.int64, device=device)
    tdist.broadcast(n, src, group=group)
    if rank == src:
        buf = torch.frombuffer(bytearray(data), dtype=torch.uint8).to(device) if n.item() else \
            torch.empty(0, dtype=torch.uint8, device=device)
    else:
        buf = torch.empty(int(n.item()), dtype=torch.uint8, device=device)
    tdist.broadcast(buf, src, group=group)
    return bytes(buf.cpu().numpy().tobytes())


def load_shard(A, image: bytes, world: int, rank: int, device: int) -> "sr.SparseMatrix":
    """A handle of matrix A on `device` holding shard `rank` of `world` of a saved plan."""
    M = sr.SparseMatrix.from_csr(A, device=device)
    M.load_plan(image, world=world, rank=rank)
    return M


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
