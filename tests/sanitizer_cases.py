"""Small invocations of every kernel path of libsr, run under compute-sanitizer (memcheck,
racecheck, synccheck) by tests/test_sanitizers.py.  Exits non-zero on a parity failure.
Covers: phase-S task kernels (SpMM K = 32·p and 128·p, SDDMM), the one-row-per-warp kernels
(K = 36), phase D (TMA producer / mbarrier ring, SpMM and SDDMM), read-modify-write rows,
split long rows (ordered combine), a hub panel split over several units (ordered combine),
sr_set_values and the scatter helpers."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ppopp_jiangha20_b200 as sr  # noqa: E402
from oracle import oracle as O  # noqa: E402
from synth import generators as g  # noqa: E402


def matrix_with_long_rows_and_hub():
    rng = np.random.default_rng(0)
    rows, cols = [], []
    n, m = 96, 3000
    for i in range(n):
        d = 700 if i % 29 == 0 else (0 if i % 11 == 0 else int(rng.integers(1, 20)))
        rows.append(np.full(d, i))
        cols.append(rng.choice(m, size=d, replace=False))
    for i in range(0, 16):  # rows 0..15 share 600 columns: a panel with ~10 tiles -> split units
        rows.append(np.full(600, i))
        cols.append(np.arange(2000, 2600))
    rowptr, colidx = g._from_coo(n, m, np.concatenate(rows), np.concatenate(cols))
    return g.CSR(n, m, rowptr, colidx, g._uniform_vals(colidx.size, 3))


def run(A, params, Ks):
    M = sr.SparseMatrix.from_csr(A)
    if params is not None:
        M.reorder(params)
    for K in Ks:
        B, X, Y = g.dense(A.ncols, K), g.dense(A.nrows, K, stream=1), g.dense(A.ncols, K, stream=2)
        C = M.spmm(torch.from_numpy(B).cuda())
        out = M.sddmm(torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda())
        torch.cuda.synchronize()
        ref, bound = O.spmm_rows(A, B, np.arange(A.nrows))
        assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-4 * bound + 1e-30), ("spmm", K)
        oref, ob = O.sddmm(A, X, Y)
        assert np.all(np.abs(out.cpu().numpy() - oref) <= 1e-4 * ob + 1e-30), ("sddmm", K)
    return M


def main():
    tiny = g.random_csr(300, 200, 0.05, 7, empty_frac=0.1)
    run(tiny, None, (32, 36, 128))
    force = dict(siglen=32, bsize=2, seed=4, max_bucket=0, threshold_size=256, panel_rows=16, dense_min=2,
                 mode=sr.FORCE, tile_cols=16)
    run(tiny, sr.default_params(**force), (32, 128))
    run(tiny, sr.default_params(**dict(force, panel_rows=8)), (32, 36, 128, 132))  # register-tile phase D
    H = matrix_with_long_rows_and_hub()
    M = run(H, sr.default_params(**force), (32, 128, 256))
    run(H, sr.default_params(**dict(force, panel_rows=8, mode=sr.OFF)), (32, 128, 256))  # split register tiles
    st = M.stats()
    assert st["dense1"] > 0 and st["ntiles"] > 8, st
    # new values on the same plan
    vals2 = g._uniform_vals(H.nnz, 9)
    M.set_values(torch.from_numpy(vals2).cuda())
    H2 = g.CSR(H.nrows, H.ncols, H.rowptr, H.colidx, vals2)
    K = 128
    B = g.dense(H.ncols, K)
    C = M.spmm(torch.from_numpy(B).cuda())
    torch.cuda.synchronize()
    ref, bound = O.spmm_rows(H2, B, np.arange(H.nrows))
    assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-4 * bound + 1e-30), "set_values"
    # a shard and the scatter helpers
    Ms = sr.SparseMatrix.from_csr(tiny)
    Ms.reorder(sr.default_params(**force, world=2, rank=1))
    Bt = torch.from_numpy(g.dense(tiny.ncols, 32)).cuda()
    full = torch.zeros((tiny.nrows, 32), device="cuda")
    sr.scatter_rows(Ms.spmm(Bt), torch.from_numpy(Ms.shard_rows()).cuda(), full)
    torch.cuda.synchronize()
    print("sanitizer cases ok")


if __name__ == "__main__":
    main()
