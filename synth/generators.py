"""Seeded synthetic CSR workloads and dense operands.

This module is the ONLY code shared by the CUDA path (bench / GPU tests) and the
CPU oracle: it draws the inputs and holds none of the method's arithmetic (no
hashing, no similarity, no clustering, no tiling, no multiplication).  Every
generator is a pure function of its seeds (numpy PCG64), so the oracle and the
library always see bit-identical inputs.

Workload shapes follow BASELINE.json `configs` (PAPER.md has no datasets we can
use: its 1084 SuiteSparse/NetworkRepository matrices, are OUT of scope):

  C1 tiny     1024x1024, row degree U{5..15}, columns uniform w/o replacement
  C2 rmat     Graph500 R-MAT scale 20, edge factor 16, (a,b,c,d)=(.57,.19,.19,.05),
              deduplicated, rows randomly permuted (columns untouched)
  C3 banded   2^21 rows, 32-row blocks sharing 16 base columns in a +-256 window
              around the block diagonal, + 4 private columns per row in +-1024
  C4 gnn      232,965 nodes, 50 communities, lognormal out-degree (mean ~492),
              80% intra-community edges, node ids shuffled, directed
  C5 cf       480,189 users x 17,770 items, lognormal user degree (mean ~209),
              Zipf(0.9) item popularity without replacement, item ids shuffled,
              integer ratings 1..5

Seeds: struct=1, values=2, dense=3 (the LSH seed 4 is a reorder
parameter, not an input).
"""
from __future__ import annotations

import dataclasses

import numpy as np

SEED_STRUCT = 1
SEED_VAL = 2
SEED_DENSE = 3
SEED_LSH = 4


@dataclasses.dataclass
class CSR:
    nrows: int
    ncols: int
    rowptr: np.ndarray  # int64[nrows+1]
    colidx: np.ndarray  # int32[nnz]
    vals: np.ndarray    # float32[nnz]
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])


def _sorted_unique(key: np.ndarray) -> np.ndarray:
    """np.unique without its (slow, hash-based in numpy 2.3) path: sort + adjacent mask."""
    key = np.sort(key, kind="stable")
    if key.size == 0:
        return key
    keep = np.empty(key.size, dtype=bool)
    keep[0] = True
    np.not_equal(key[1:], key[:-1], out=keep[1:])
    return key[keep]


def _from_coo(nrows: int, ncols: int, row: np.ndarray, col: np.ndarray) -> tuple:
    """Deduplicate (row, col) pairs and build a row-major, column-sorted CSR pattern."""
    key = _sorted_unique(row.astype(np.int64) * np.int64(ncols) + col.astype(np.int64))
    r = (key // ncols).astype(np.int64)
    c = (key % ncols).astype(np.int32)
    counts = np.bincount(r, minlength=nrows).astype(np.int64)
    rowptr = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return rowptr, c


def _uniform_vals(nnz: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return (rng.random(nnz, dtype=np.float32) * np.float32(2.0) - np.float32(1.0)).astype(np.float32)


def dense(rows: int, cols: int, seed: int = SEED_DENSE, stream: int = 0) -> np.ndarray:
    """Dense operand ~ U(-1, 1) fp32, row-major [rows, cols].  `stream` selects an
    independent sub-stream (B / X / Y of the same run)."""
    rng = np.random.default_rng([seed, stream])
    out = rng.random((rows, cols), dtype=np.float32)
    out *= np.float32(2.0)
    out -= np.float32(1.0)
    return out


# ----------------------------------------------------------------------------
# C1 tiny
# ----------------------------------------------------------------------------
def tiny(n: int = 1024, dmin: int = 5, dmax: int = 15, seed_struct: int = SEED_STRUCT,
         seed_val: int = SEED_VAL) -> CSR:
    rng = np.random.default_rng(seed_struct)
    deg = rng.integers(dmin, dmax + 1, size=n)
    rows, cols = [], []
    for i in range(n):
        c = rng.choice(n, size=int(deg[i]), replace=False)
        rows.append(np.full(c.size, i, dtype=np.int64))
        cols.append(c.astype(np.int64))
    rowptr, colidx = _from_coo(n, n, np.concatenate(rows), np.concatenate(cols))
    return CSR(n, n, rowptr, colidx, _uniform_vals(colidx.size, seed_val), "tiny")


def random_csr(nrows: int, ncols: int, density: float, seed: int, empty_frac: float = 0.0,
               seed_val: int | None = None) -> CSR:
    """Small Bernoulli(density) matrix with an optional fraction of forced-empty rows
    (property / edge-case tests)."""
    rng = np.random.default_rng(seed)
    mask = rng.random((nrows, ncols)) < density
    if empty_frac > 0:
        mask[rng.random(nrows) < empty_frac, :] = False
    r, c = np.nonzero(mask)
    rowptr, colidx = _from_coo(nrows, ncols, r, c)
    return CSR(nrows, ncols, rowptr, colidx,
               _uniform_vals(colidx.size, seed + 7919 if seed_val is None else seed_val), "random")


# ----------------------------------------------------------------------------
# C2 R-MAT
# ----------------------------------------------------------------------------
def rmat(scale: int = 20, edge_factor: int = 16, abcd=(0.57, 0.19, 0.19, 0.05),
         seed_struct: int = SEED_STRUCT, seed_val: int = SEED_VAL, permute_rows: bool = True) -> CSR:
    n = 1 << scale
    m = edge_factor * n
    a, b, c, _ = abcd
    rng = np.random.default_rng(seed_struct)
    row = np.zeros(m, dtype=np.int64)
    col = np.zeros(m, dtype=np.int64)
    for level in range(scale):
        u = rng.random(m)
        rbit = u >= (a + b)                                  # quadrant c or d
        cbit = ((u >= a) & (u < a + b)) | (u >= a + b + c)   # quadrant b or d
        row |= rbit.astype(np.int64) << level
        col |= cbit.astype(np.int64) << level
        del u, rbit, cbit
    if permute_rows:
        perm = rng.permutation(n).astype(np.int64)
        row = perm[row]
    rowptr, colidx = _from_coo(n, n, row, col)
    return CSR(n, n, rowptr, colidx, _uniform_vals(colidx.size, seed_val), f"rmat{scale}")


# ----------------------------------------------------------------------------
# C3 banded / clustered
# ----------------------------------------------------------------------------
def banded(nrows: int = 1 << 21, block: int = 32, base_cols: int = 16, base_win: int = 256,
           priv_cols: int = 4, priv_win: int = 1024, seed_struct: int = SEED_STRUCT,
           seed_val: int = SEED_VAL) -> CSR:
    n = nrows
    nblocks = (n + block - 1) // block
    rng = np.random.default_rng(seed_struct)
    center = np.arange(nblocks, dtype=np.int64) * block + block // 2
    base = center[:, None] + rng.integers(-base_win, base_win + 1, size=(nblocks, base_cols))
    base = np.clip(base, 0, n - 1)
    rows_b = np.repeat(np.arange(n, dtype=np.int64), base_cols)
    cols_b = base[np.arange(n) // block].reshape(-1)
    rid = np.arange(n, dtype=np.int64)
    priv = rid[:, None] + rng.integers(-priv_win, priv_win + 1, size=(n, priv_cols))
    priv = np.clip(priv, 0, n - 1)
    rows_p = np.repeat(rid, priv_cols)
    rowptr, colidx = _from_coo(n, n, np.concatenate([rows_b, rows_p]),
                               np.concatenate([cols_b, priv.reshape(-1)]))
    return CSR(n, n, rowptr, colidx, _uniform_vals(colidx.size, seed_val), "banded")


# ----------------------------------------------------------------------------
# C4 GNN-shaped graph
# ----------------------------------------------------------------------------
def gnn(nodes: int = 232_965, communities: int = 50, mean_deg: float = 492.0, sigma: float = 1.0,
        p_intra: float = 0.8, seed_struct: int = SEED_STRUCT, seed_val: int = SEED_VAL) -> CSR:
    n = nodes
    rng = np.random.default_rng(seed_struct)
    mu = np.log(mean_deg) - 0.5 * sigma * sigma
    deg = np.clip(np.rint(rng.lognormal(mu, sigma, size=n)), 1, n - 1).astype(np.int64)
    bounds = (np.arange(communities + 1, dtype=np.int64) * n) // communities
    src = np.repeat(np.arange(n, dtype=np.int64), deg)
    comm = np.searchsorted(bounds, src, side="right") - 1
    lo = bounds[comm]
    size = bounds[comm + 1] - lo
    intra = rng.random(src.size) < p_intra
    u = rng.random(src.size)
    dst = np.where(intra, lo + (u * size).astype(np.int64), (u * n).astype(np.int64))
    dst = np.minimum(dst, n - 1)
    del comm, lo, size, intra, u
    perm = rng.permutation(n).astype(np.int64)
    rowptr, colidx = _from_coo(n, n, perm[src], perm[dst])
    return CSR(n, n, rowptr, colidx, _uniform_vals(colidx.size, seed_val), "gnn")


# ----------------------------------------------------------------------------
# C5 collaborative filtering ratings
# ----------------------------------------------------------------------------
def cf(users: int = 480_189, items: int = 17_770, mean_deg: float = 209.0, sigma: float = 1.0,
       zipf_s: float = 0.9, oversample: float = 1.6, seed_struct: int = SEED_STRUCT,
       seed_val: int = SEED_VAL) -> CSR:
    rng = np.random.default_rng(seed_struct)
    mu = np.log(mean_deg) - 0.5 * sigma * sigma
    deg = np.clip(np.rint(rng.lognormal(mu, sigma, size=users)), 1, items).astype(np.int64)
    pop = 1.0 / np.power(np.arange(1, items + 1, dtype=np.float64), zipf_s)
    cdf = np.cumsum(pop)
    cdf /= cdf[-1]
    # sample with replacement (oversampled), dedupe, then keep a random `deg` of them
    draws = np.minimum(np.ceil(deg * oversample).astype(np.int64) + 2, items)
    src = np.repeat(np.arange(users, dtype=np.int64), draws)
    it = np.searchsorted(cdf, rng.random(src.size), side="right").astype(np.int64)
    it = np.minimum(it, items - 1)
    key = _sorted_unique(src * items + it)
    del src, it
    u = key // items
    prio = rng.integers(0, 1 << 32, size=key.size, dtype=np.int64)
    order = np.argsort((u << 32) | prio)  # random order within each user
    del prio
    key = key[order]
    u = u[order]
    start = np.searchsorted(u, np.arange(users, dtype=np.int64), side="left")
    rank = np.arange(key.size, dtype=np.int64) - start[u]
    keep = rank < deg[u]
    key = key[keep]
    item_perm = rng.permutation(items).astype(np.int64)
    rowptr, colidx = _from_coo(users, items, key // items, item_perm[key % items])
    vals = np.random.default_rng(seed_val).integers(1, 6, size=colidx.size).astype(np.float32)
    return CSR(users, items, rowptr, colidx, vals, "cf")


# ----------------------------------------------------------------------------
# worked example of PAPER.md Fig 1a (reconstructed)
# ----------------------------------------------------------------------------
def fig1a() -> CSR:
    """S0={0,4} S1={1,2,3} S2={4,5} S3={1} S4={0,3,4} S5={2,5}; constraints P:47, P:71,
    P:111.  Values are 1..13 so
    every nnz is distinguishable."""
    rowptr = np.array([0, 2, 5, 7, 8, 11, 13], dtype=np.int64)
    colidx = np.array([0, 4, 1, 2, 3, 4, 5, 1, 0, 3, 4, 2, 5], dtype=np.int32)
    vals = np.arange(1, 14, dtype=np.float32)
    return CSR(6, 6, rowptr, colidx, vals, "fig1a")


def fig7a() -> CSR:
    """A well clustered matrix: two groups of three identical rows whose
    consecutive-row Jaccard similarities are 1,1,0,1,1 -> average 0.8."""
    rows = [[0, 1, 2], [0, 1, 2], [0, 1, 2], [3, 4, 5], [3, 4, 5], [3, 4, 5]]
    rowptr = np.array([0, 3, 6, 9, 12, 15, 18], dtype=np.int64)
    colidx = np.array(sum(rows, []), dtype=np.int32)
    return CSR(6, 6, rowptr, colidx, np.ones(18, dtype=np.float32), "fig7a")


def diagonal(n: int = 64) -> CSR:
    """Fig 7b: an extremely scattered (diagonal) matrix."""
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32),
               np.ones(n, dtype=np.float32), "diagonal")


def shuffle_within_rows(A: CSR, seed: int = 11) -> CSR:
    """Same matrix with each row's entries in a random order (ingest must sort them)."""
    rng = np.random.default_rng(seed)
    key = np.repeat(np.arange(A.nrows, dtype=np.int64), np.diff(A.rowptr))
    order = np.lexsort((rng.random(A.nnz), key))
    return CSR(A.nrows, A.ncols, A.rowptr.copy(), A.colidx[order].copy(), A.vals[order].copy(),
               A.name + "_unsorted")


CONFIGS = {
    "tiny": dict(make=tiny, K=(32,)),
    "rmat": dict(make=rmat, K=(32, 128)),
    "banded": dict(make=banded, K=(128,)),
    "gnn": dict(make=gnn, K=(128,)),
    "cf": dict(make=cf, K=(128,)),
}


def make(name: str, **kw) -> CSR:
    return CONFIGS[name]["make"](**kw)
