"""GPU parity: libsr (C ABI, sm_100a kernels) against the CPU oracle on the same seeded
inputs.  Plan metadata must be bit-exact; fp32 outputs must satisfy the north_star bound
|err| <= 1e-4·Σ_k|a_ik||b_kj| (SpMM) and |err| <= 1e-4·|a_ij|·Σ_k|x_ik||y_jk| (SDDMM)."""
import numpy as np
import pytest

from synth import generators as g

pytestmark = pytest.mark.gpu

TOL = 1e-4


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("a CUDA device is required for -m gpu tests")
    import paper_conf_ppopp_jiangha20_b200 as sr
    sr.lib()
    return sr, torch


def _spmm_check(oracle, A, B, C_gpu, rows=None):
    if rows is None:
        ref, bound = oracle.spmm_rows(A, B, np.arange(A.nrows))
        got = C_gpu
    else:
        ref, bound = oracle.spmm_rows(A, B, rows)
        got = C_gpu[rows]
    err = np.abs(got.astype(np.float64) - ref)
    bad = err > TOL * bound + 1e-30
    assert not bad.any(), f"{bad.sum()} entries out of tolerance; worst {err.max()}"


def _sddmm_check(oracle, A, X, Y, out_gpu):
    ref, bound = oracle.sddmm(A, X, Y)
    err = np.abs(out_gpu.astype(np.float64) - ref)
    bad = err > TOL * bound + 1e-30
    assert not bad.any(), f"{bad.sum()} entries out of tolerance; worst {err.max()}"


def _run(env, A, K, params=None, seed=3):
    sr, torch = env
    M = sr.SparseMatrix.from_csr(A)
    if params is not None:
        M.reorder(params)
    B = g.dense(A.ncols, K, seed=seed)
    X = g.dense(A.nrows, K, seed=seed, stream=1)
    Y = g.dense(A.ncols, K, seed=seed, stream=2)
    Bd, Xd, Yd = (torch.from_numpy(t).cuda() for t in (B, X, Y))
    C = M.spmm(Bd)
    out = M.sddmm(Xd, Yd)
    torch.cuda.synchronize()
    return M, B, X, Y, C.cpu().numpy(), out.cpu().numpy()


# ------------------------------------------------------------------ identity plan
@pytest.mark.parametrize("K", [32, 128])
def test_tiny_identity_plan(env, oracle, K):
    A = g.tiny()
    M, B, X, Y, C, out = _run(env, A, K)
    _spmm_check(oracle, A, B, C)
    _sddmm_check(oracle, A, X, Y, out)
    assert M.last_launch_count() >= 1


# ------------------------------------------------------------------ plan bit-exactness
def _plan_kw(panel_rows=8, mode=1, max_bucket=0, tile_cols=16):
    return dict(siglen=128, bsize=2, seed=4, max_bucket=max_bucket, threshold_size=256,
                panel_rows=panel_rows, dense_min=2, mode=mode)


def _assert_plan_equal(M, ref):
    np.testing.assert_array_equal(M.perm(1), ref["perm1"])
    np.testing.assert_array_equal(M.perm(2), ref["perm2"])
    t = M.tiles()
    for k in ("dense_ptr", "dense_cols", "drow_ptr", "d_slot", "d_pos", "rrow_ptr", "r_col", "r_pos"):
        np.testing.assert_array_equal(t[k], ref[k], err_msg=k)
    st = M.stats()
    for k in ("dense0", "dense1", "avgsim_num", "avgsim_den", "round1", "round2", "E1", "E2", "npanels",
              "ndense_cols"):
        assert st[k] == ref["stats"][k], k


@pytest.mark.parametrize("mode", [0, 1, 2])
@pytest.mark.parametrize("panel_rows,max_bucket", [(8, 0), (64, 0), (16, 4)])
def test_tiny_plan_bit_exact(env, oracle, mode, panel_rows, max_bucket):
    sr, _ = env
    A = g.tiny()
    kw = _plan_kw(panel_rows, mode, max_bucket)
    ref = oracle.plan(A, **kw)
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**kw, tile_cols=16))
    _assert_plan_equal(M, ref)


def test_worked_example_plan(env, oracle):
    """Fig 1a in FORCE mode, panel 3, dense >= 2."""
    sr, _ = env
    A = g.fig1a()
    kw = _plan_kw(3, 1, 0)
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**kw, tile_cols=2))
    _assert_plan_equal(M, oracle.plan(A, **kw))
    # DenseRatio0 = 2/13
    assert M.stats()["dense0"] == 2


@pytest.mark.parametrize("case", ["fig1a", "tiny_auto2", "tiny_auto4"])
def test_auto_decision_threshold_plan(env, oracle, case):
    """R28: AUTO's DenseRatio0 under auto_dense_min while the plan tiles with dense_min;
    the library's decision, stats and plan equal the oracle's."""
    sr, _ = env
    if case == "fig1a":
        A, kw = g.fig1a(), dict(_plan_kw(3, 0, 0), dense_min=3, auto_dense_min=2)
    else:
        A = g.tiny()
        kw = dict(_plan_kw(16, 0, 0), dense_min=8, auto_dense_min=2 if case == "tiny_auto2" else 4)
    ref = oracle.plan(A, **kw)
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**kw, tile_cols=16))
    _assert_plan_equal(M, ref)
    assert M.get_params().auto_dense_min == kw["auto_dense_min"]
    if case == "fig1a":
        assert (M.stats()["dense0"], M.stats()["round1"]) == (2, 0)


# ------------------------------------------------------------------ numerics over the plan
@pytest.mark.parametrize("panel", [8, 16])
@pytest.mark.parametrize("K", [1, 3, 4, 8, 32, 36, 64, 128, 132, 256])
def test_k_sweep_forced_plan(env, oracle, K, panel):
    """panel 16: phase D on the TMA shared-memory engine; panel 8: the register-tile engine."""
    sr, _ = env
    A = g.random_csr(700, 500, 0.03, 5, empty_frac=0.1)
    M, B, X, Y, C, out = _run(env, A, K, sr.default_params(**_plan_kw(panel, 1, 8), tile_cols=8))
    assert M.stats()["dense1"] > 0
    _spmm_check(oracle, A, B, C)
    _sddmm_check(oracle, A, X, Y, out)


@pytest.mark.parametrize("tile_cols", [1, 5, 64, 1024])
def test_tile_widths(env, oracle, tile_cols):
    sr, _ = env
    A = g.random_csr(300, 60, 0.2, 9, empty_frac=0.05)  # dense-ish -> many dense columns
    M, B, X, Y, C, out = _run(env, A, 32, sr.default_params(**_plan_kw(32, 1, 0), tile_cols=tile_cols))
    assert M.stats()["ndense_cols"] > 60
    _spmm_check(oracle, A, B, C)
    _sddmm_check(oracle, A, X, Y, out)


def test_long_rows_split_and_rmw(env, oracle):
    """Rows far longer than one work item (split + ordered combine), some of them also
    with dense-tile nnz (read-modify-write of C), and empty rows (zero fill)."""
    sr, _ = env
    rng = np.random.default_rng(0)
    rows, cols = [], []
    n, m = 200, 20000
    for i in range(n):
        d = 5000 if i % 37 == 0 else (0 if i % 11 == 0 else int(rng.integers(1, 40)))
        c = rng.choice(m, size=d, replace=False)
        rows.append(np.full(d, i))
        cols.append(c)
    # a shared hub block so panels get dense columns
    hub = np.arange(32)
    for i in range(0, n, 3):
        rows.append(np.full(32, i))
        cols.append(hub)
    rowptr, colidx = g._from_coo(n, m, np.concatenate(rows), np.concatenate(cols))
    A = g.CSR(n, m, rowptr, colidx, g._uniform_vals(colidx.size, 3))
    for params in (None, sr.default_params(**_plan_kw(16, 1, 8)), sr.default_params(**_plan_kw(16, 2, 0)),
                   sr.default_params(**_plan_kw(8, 1, 8))):
        for K in (32, 128, 256):  # 256: two 128-column passes of the SpMM task kernel
            M, B, X, Y, C, out = _run(env, A, K, params)
            _spmm_check(oracle, A, B, C)
            _sddmm_check(oracle, A, X, Y, out)
            # the result is deterministic (ordered combine of split rows)
            _, _, _, _, C2, _ = _run(env, A, K, params)
            np.testing.assert_array_equal(C, C2)


@pytest.mark.parametrize("K", [32, 128, 256])
def test_register_tiles_split_hub_panels(env, oracle, K):
    """Panels of 8 rows on the register-tile engine where one panel holds thousands of dense
    entries: it is cut into chunks (one warp each) whose partial sums the last chunk adds in
    chunk order; the result is deterministic and matches the oracle."""
    sr, torch = env
    rng = np.random.default_rng(3)
    n, m = 64, 6000
    rows, cols = [], []
    for i in range(n):
        d = int(rng.integers(1, 30))
        rows.append(np.full(d, i))
        cols.append(rng.choice(m, size=d, replace=False))
    for i in range(8, 16):  # panel 1: 8 rows sharing 2500 columns -> ~22 k entries, ~22 chunks
        rows.append(np.full(2500, i))
        cols.append(np.arange(3000, 5500))
    rowptr, colidx = g._from_coo(n, m, np.concatenate(rows), np.concatenate(cols))
    A = g.CSR(n, m, rowptr, colidx, g._uniform_vals(colidx.size, 5))
    params = sr.default_params(**_plan_kw(8, 2, 0))  # OFF: identity order, tiles only
    M, B, X, Y, C, out = _run(env, A, K, params)
    assert M.stats()["dense1"] >= 8 * 2500
    _spmm_check(oracle, A, B, C)
    _sddmm_check(oracle, A, X, Y, out)
    _, _, _, _, C2, _ = _run(env, A, K, params)
    np.testing.assert_array_equal(C, C2)


@pytest.mark.parametrize("K", [128, 256])
def test_tma_engine_split_hub_panel(env, oracle, K):
    """A 16-row panel with 5000 shared columns: 79 staged tiles of 64 columns, more than one
    phase-D unit holds (32 tiles), so the panel runs as three units whose partial sums the
    last one adds in unit order (release / acquire through one thread per CTA)."""
    sr, _ = env
    rng = np.random.default_rng(5)
    n, m = 64, 9000
    rows, cols = [], []
    hub = rng.choice(m, size=5000, replace=False)
    for i in range(n):
        if i < 16:
            rows.append(np.full(hub.size, i))
            cols.append(hub)
        d = int(rng.integers(0, 30))
        extra = np.setdiff1d(rng.choice(m, size=d, replace=False), hub if i < 16 else [])
        rows.append(np.full(extra.size, i))
        cols.append(extra)
    rowptr, colidx = g._from_coo(n, m, np.concatenate(rows), np.concatenate(cols))
    A = g.CSR(n, m, rowptr, colidx, g._uniform_vals(colidx.size, 4))
    M, B, X, Y, C, out = _run(env, A, K, sr.default_params(**dict(_plan_kw(16, 2, 0)), tile_cols=64))
    assert M.stats()["dense1"] >= 16 * 5000
    _spmm_check(oracle, A, B, C)
    _sddmm_check(oracle, A, X, Y, out)
    _, _, _, _, C2, _ = _run(env, A, K, sr.default_params(**dict(_plan_kw(16, 2, 0)), tile_cols=64))
    np.testing.assert_array_equal(C, C2)  # deterministic ordered combine


def test_unsorted_input_keeps_caller_nnz_order(env, oracle):
    sr, _ = env
    A = g.random_csr(120, 90, 0.1, 12, empty_frac=0.1)
    U = g.shuffle_within_rows(A, seed=3)
    for params in (None, sr.default_params(**_plan_kw(8, 1, 0))):
        M, B, X, Y, C, out = _run(env, U, 32, params)
        _sddmm_check(oracle, U, X, Y, out)  # oracle works in the given (unsorted) order
        _spmm_check(oracle, U, B, C)
        if params is not None:
            ref = oracle.plan(A, **_plan_kw(8, 1, 0))  # plan of the canonical matrix
            np.testing.assert_array_equal(M.perm(1), ref["perm1"])
            t = M.tiles()
            # d_pos / r_pos refer to the caller's (unsorted) positions
            np.testing.assert_array_equal(np.sort(np.concatenate([t["d_pos"], t["r_pos"]])), np.arange(U.nnz))
            np.testing.assert_array_equal(U.colidx[t["r_pos"]], t["r_col"])


@pytest.mark.parametrize("K", [32, 128])
def test_repeated_launches_fresh_results(env, oracle, K):
    """Consecutive SpMM / SDDMM calls on one handle, each with new operands into a poisoned
    output: every call must compute every task (the K = 128 SDDMM kernel hands tasks out through a
    ticket counter that its last warp resets for the next launch, exec.cu: first_ticket)."""
    sr, torch = env
    A = g.rmat(scale=17)  # 2.1 M nnz: ~10^4 tasks, several per warp of the resident grid
    M = sr.SparseMatrix.from_csr(A)
    for it in range(3):
        B = g.dense(A.ncols, K, seed=20 + it)
        X, Y = g.dense(A.nrows, K, seed=20 + it, stream=1), g.dense(A.ncols, K, seed=20 + it, stream=2)
        C = torch.full((A.nrows, K), float("nan"), device="cuda")
        out = torch.full((A.nnz,), float("nan"), device="cuda")
        M.spmm(torch.from_numpy(B).cuda(), C)
        M.sddmm(torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda(), out)
        torch.cuda.synchronize()
        _spmm_check(oracle, A, B, C.cpu().numpy())
        _sddmm_check(oracle, A, X, Y, out.cpu().numpy())


def test_strided_and_misaligned_operands(env, oracle):
    sr, torch = env
    A = g.random_csr(150, 100, 0.08, 4, empty_frac=0.1)
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**_plan_kw(16, 1, 0)))
    K = 32
    B = g.dense(100, K)
    # ldb = 40 (vector path), and a 1-float offset base (scalar path)
    Bbig = torch.zeros((100, 41), device="cuda")
    Bbig[:, :K] = torch.from_numpy(B).cuda()
    C1 = torch.full((150, 40), 7.0, device="cuda")
    M.spmm(Bbig[:, :K], C1[:, :K])
    Bmis = torch.zeros(100 * K + 1, device="cuda")
    Bmis[1:] = torch.from_numpy(B.reshape(-1)).cuda()
    C2 = M.spmm(Bmis[1:].view(100, K))
    torch.cuda.synchronize()
    _spmm_check(oracle, A, B, C1[:, :K].cpu().numpy())
    _spmm_check(oracle, A, B, C2.cpu().numpy())
    assert torch.all(C1[:, K:] == 7.0)  # padding columns untouched


def test_binding_rejects_bad_operands(env):
    """The C ABI sees only pointers and leading dimensions: the binding must refuse operands the
    kernels would read or write out of bounds or scramble."""
    sr, torch = env
    A = g.random_csr(50, 40, 0.1, 3)
    M = sr.SparseMatrix.from_csr(A)
    K = 8
    B = torch.ones((40, K), device="cuda")
    X, Y = torch.ones((50, K), device="cuda"), torch.ones((40, K), device="cuda")
    bad = [lambda: M.spmm(torch.ones((39, K), device="cuda")),                      # too few B rows
           lambda: M.spmm(B.double()),                                             # dtype
           lambda: M.spmm(B.cpu()),                                                # host tensor
           lambda: M.spmm(B, torch.empty((49, K), device="cuda")),                 # C too small
           lambda: M.spmm(B, torch.empty((50, 2 * K), device="cuda")[:, ::2]),     # C column stride 2
           lambda: M.spmm(B.t().contiguous().t()),                                 # B column stride != 1
           lambda: M.sddmm(torch.ones((49, K), device="cuda"), Y),                 # X rows
           lambda: M.sddmm(X, torch.ones((40, K + 1), device="cuda")),             # K mismatch
           lambda: M.sddmm(X, Y, torch.empty(2 * A.nnz, device="cuda")[::2]),      # out not contiguous
           lambda: M.set_values(torch.ones(A.nnz - 1, device="cuda"))]             # value count
    for f in bad:
        with pytest.raises(ValueError):
            f()
    torch.cuda.synchronize()


def test_empty_and_degenerate(env, oracle):
    sr, torch = env
    # all rows empty
    A = g.CSR(10, 10, np.zeros(11, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    M = sr.SparseMatrix.from_csr(A)
    C = M.spmm(torch.ones((10, 8), device="cuda"))
    torch.cuda.synchronize()
    assert torch.all(C == 0)
    M.reorder(sr.default_params(**_plan_kw(4, 1, 0)))
    C = M.spmm(torch.ones((10, 8), device="cuda"))
    torch.cuda.synchronize()
    assert torch.all(C == 0)
    # single row / single column
    for A in (g.random_csr(1, 64, 0.5, 1), g.random_csr(64, 1, 0.5, 2), g.diagonal(100)):
        M, B, X, Y, C, out = _run(env, A, 8, sr.default_params(**_plan_kw(8, 1, 0)))
        _spmm_check(oracle, A, B, C)
        _sddmm_check(oracle, A, X, Y, out)


def test_reorder_twice_is_a_state_error(env):
    sr, _ = env
    M = sr.SparseMatrix.from_csr(g.tiny())
    M.reorder(sr.default_params())
    with pytest.raises(sr.SRError) as e:
        M.reorder(sr.default_params())
    assert e.value.code == sr.SR_ESTATE


def test_bad_params(env):
    sr, _ = env
    M = sr.SparseMatrix.from_csr(g.tiny())
    for kw in (dict(siglen=10, bsize=3), dict(panel_rows=0), dict(tile_cols=0), dict(threshold_size=1),
               dict(mode=7), dict(world=2, rank=2)):
        with pytest.raises(sr.SRError) as e:
            M.reorder(sr.default_params(**kw))
        assert e.value.code == sr.SR_EINVAL, kw
    with pytest.raises(sr.SRError) as e:
        M.reorder(sr.default_params(siglen=12, bsize=4))
    assert e.value.code == sr.SR_EUNSUPPORTED


# ------------------------------------------------------------------ sharded plans on one GPU
@pytest.mark.parametrize("panel", [8, 16])
@pytest.mark.parametrize("world", [2, 3])
def test_shard_simulation(env, oracle, world, panel):
    """Run every shard's plan on the same GPU and reassemble (SURVEY §4 tier 4a)."""
    sr, torch = env
    A = g.random_csr(500, 300, 0.03, 21, empty_frac=0.1)
    K = 32
    B = torch.from_numpy(g.dense(300, K)).cuda()
    X = torch.from_numpy(g.dense(500, K, stream=1)).cuda()
    Y = torch.from_numpy(g.dense(300, K, stream=2)).cuda()
    C = np.full((500, K), np.nan, np.float32)
    out = np.full(A.nnz, np.nan, np.float32)
    ref_cuts = None
    for r in range(world):
        M = sr.SparseMatrix.from_csr(A)
        M.reorder(sr.default_params(**_plan_kw(panel, 1, 0), world=world, rank=r))
        st = M.stats()
        Cr = M.spmm(B)
        outr = M.sddmm(X, Y)
        torch.cuda.synchronize()
        rows = M.shard_rows()
        assert Cr.shape[0] == rows.size == st["shard_nrows"]
        C[rows] = Cr.cpu().numpy()
        out[M.shard_nnz_ids()] = outr.cpu().numpy()
        if ref_cuts is None:
            ref = oracle.plan(A, **_plan_kw(panel, 1, 0))
            P = panel
            w = [int(ref["drow_ptr"][min(500, (p + 1) * P)] - ref["drow_ptr"][p * P]
                     + ref["rrow_ptr"][min(500, (p + 1) * P)] - ref["rrow_ptr"][p * P]) for p in range(ref["npanels"])]
            ref_cuts = oracle.partition(np.array(w), world)
        assert (st["shard_panel_begin"], st["shard_panel_end"]) == (ref_cuts[r], ref_cuts[r + 1])
    assert not np.isnan(C).any() and not np.isnan(out).any()
    _spmm_check(oracle, A, B.cpu().numpy(), C)
    _sddmm_check(oracle, A, X.cpu().numpy(), Y.cpu().numpy(), out)


# ------------------------------------------------------------------ full-size configs
# bench.py's plan parameters (the launch configuration it times): AUTO, dense_min 64 for the
# kernels, auto_dense_min 8 for the round-1 decision (R28), max_bucket 32 (R14)
BENCH_KW = dict(siglen=128, bsize=2, seed=4, max_bucket=32, threshold_size=256, panel_rows=64, dense_min=64,
                auto_dense_min=8, mode=0)


def _sampled_rows(A, n=2000):
    rng = np.random.default_rng(0)
    deg = np.diff(A.rowptr)
    return np.unique(np.concatenate([rng.integers(0, A.nrows, n), np.argsort(deg)[-20:]]))


@pytest.mark.slow
@pytest.mark.parametrize("config", ["rmat", "banded", "gnn", "cf"])
def test_full_size_plan_bench_params(env, oracle, config):
    """C2-C5 at full size with bench.py's plan parameters: perm1, perm2, tiles and the AUTO
    decisions bit-exact against the oracle (AUTO runs both rounds on C2 and C4, none on C3,
    round 2 on C5); SpMM (K=128) on 2000 sampled rows + the 20 longest, SDDMM on all their nnz.
    C5's round 2 at max_bucket 32 has E2 = 275 M candidates, beyond what the oracle's plain
    priority queue clusters in minutes: C5 runs here with max_bucket 8, and its bench-parameter
    plan is checked by test_full_size_cf_bench_params.  C4 runs bench.py's per-config plan
    parameters (32-row panels, dense_min 4: half its nnz on the phase-D TMA engine)."""
    sr, torch = env
    A = g.make(config)
    import bench
    kw = dict(BENCH_KW, **bench.PLAN_DEFAULTS.get(config, {}))  # C4: 32-row panels, dense_min 4
    if config == "cf":
        kw["max_bucket"] = 8
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**kw))
    ref = oracle.plan(A, **kw)
    _assert_plan_equal(M, ref)
    del ref
    rows = _sampled_rows(A)
    deg = np.diff(A.rowptr)
    B = g.dense(A.ncols, 128)
    C = M.spmm(torch.from_numpy(B).cuda())
    torch.cuda.synchronize()
    _spmm_check(oracle, A, B, C.cpu().numpy(), rows=rows)
    del C
    X, Y = g.dense(A.nrows, 128, stream=1), g.dense(A.ncols, 128, stream=2)
    out = M.sddmm(torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda()).cpu().numpy()
    sel = np.concatenate([np.arange(A.rowptr[r], A.rowptr[r + 1]) for r in rows])
    sub = g.CSR(rows.size, A.ncols, np.concatenate([[0], np.cumsum(deg[rows])]).astype(np.int64),
                A.colidx[sel], A.vals[sel])
    ref_o, bound = oracle.sddmm(sub, X[rows], Y)
    err = np.abs(out[sel] - ref_o)
    assert not (err > TOL * bound + 1e-30).any()


@pytest.mark.slow
def test_full_size_cf_bench_params(env, oracle):
    """C5 with exactly bench.py's plan parameters (max_bucket 32, E2 = 275 M): the AUTO
    decisions (DenseRatio0 under R28, AvgSim of the remainder) and the tiling of perm1 are
    bit-exact against the oracle's O10/O11 (round 1 is skipped, so perm1 is the identity), and
    perm2 lists every non-empty remainder position exactly once."""
    sr, torch = env
    A = g.make("cf")
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**BENCH_KW))
    st = M.stats()
    t0 = oracle.tile(A, np.arange(A.nrows), BENCH_KW["panel_rows"], BENCH_KW["auto_dense_min"])
    assert st["dense0"] == t0["n_dense"] and st["round1"] == 0 and t0["n_dense"] * 10 > A.nnz
    np.testing.assert_array_equal(M.perm(1), np.arange(A.nrows))
    t = oracle.tile(A, np.arange(A.nrows), BENCH_KW["panel_rows"], BENCH_KW["dense_min"])
    mt = M.tiles()
    for k in ("dense_ptr", "dense_cols", "drow_ptr", "d_slot", "d_pos", "rrow_ptr", "r_col", "r_pos"):
        np.testing.assert_array_equal(mt[k], t[k], err_msg=k)
    num, den = oracle.avgsim(t["rrow_ptr"], t["r_col"])
    assert (st["avgsim_num"], st["avgsim_den"]) == (num, den)
    assert st["round2"] == (0 if num * 10 > den else 1)
    nonempty = np.flatnonzero(np.diff(t["rrow_ptr"]) > 0)
    np.testing.assert_array_equal(np.sort(M.perm(2)), nonempty)


@pytest.mark.slow
@pytest.mark.parametrize("K", [32, 128])
def test_full_size_rmat_whole_output(env, oracle, K):
    """C2 (bench.py's workload) with bench.py's plan: every entry of C = A·B (1,048,576 × K) and
    every one of the 16,086,011 SDDMM values against the fp64 oracle, element by element."""
    sr, torch = env
    A = g.make("rmat")
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**BENCH_KW))
    B = g.dense(A.ncols, K)
    C = M.spmm(torch.from_numpy(B).cuda()).cpu().numpy()
    step = 1 << 17
    for r0 in range(0, A.nrows, step):
        rows = np.arange(r0, min(A.nrows, r0 + step))
        ref, bound = oracle.spmm_rows(A, B, rows)
        err = np.abs(C[rows].astype(np.float64) - ref)
        bad = err > TOL * bound + 1e-30
        assert not bad.any(), f"rows {r0}+: {bad.sum()} entries out of tolerance, worst {err.max()}"
    del C
    X, Y = g.dense(A.nrows, K, stream=1), g.dense(A.ncols, K, stream=2)
    out = M.sddmm(torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda()).cpu().numpy()
    _sddmm_check(oracle, A, X, Y, out)


def test_scatter_helpers_reassemble_shards(env, oracle):
    """The device scatter kernels (used by dist.gather_*) put packed shard outputs back."""
    sr, torch = env
    A = g.random_csr(400, 250, 0.03, 23, empty_frac=0.1)
    K = 16
    B = torch.from_numpy(g.dense(250, K)).cuda()
    X = torch.from_numpy(g.dense(400, K, stream=1)).cuda()
    Y = torch.from_numpy(g.dense(250, K, stream=2)).cuda()
    C = torch.full((400, K), float("nan"), device="cuda")
    out = torch.full((A.nnz,), float("nan"), device="cuda")
    for r in range(2):
        M = sr.SparseMatrix.from_csr(A)
        M.reorder(sr.default_params(**_plan_kw(16, 1, 0), world=2, rank=r))
        sr.scatter_rows(M.spmm(B), torch.from_numpy(M.shard_rows()).cuda(), C)
        sr.scatter_values(M.sddmm(X, Y), torch.from_numpy(M.shard_nnz_ids()).cuda(), out)
    torch.cuda.synchronize()
    _spmm_check(oracle, A, B.cpu().numpy(), C.cpu().numpy())
    _sddmm_check(oracle, A, X.cpu().numpy(), Y.cpu().numpy(), out.cpu().numpy())


def test_dist_gather_single_rank_nccl(env, oracle):
    """dist.gather_spmm / gather_sddmm through a real NCCL process group (world size 1)."""
    sr, torch = env
    import socket
    import torch.distributed as tdist
    from paper_conf_ppopp_jiangha20_b200 import dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    tdist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1)
    try:
        A = g.random_csr(300, 200, 0.04, 5, empty_frac=0.1)
        M = sr.SparseMatrix.from_csr(A)
        M.reorder(sr.default_params(**_plan_kw(16, 1, 0)))
        B = torch.from_numpy(g.dense(200, 32)).cuda()
        X = torch.from_numpy(g.dense(300, 32, stream=1)).cuda()
        Y = torch.from_numpy(g.dense(200, 32, stream=2)).cuda()
        C = dist.gather_spmm(M, M.spmm(B))
        out = dist.gather_sddmm(M, M.sddmm(X, Y))
        torch.cuda.synchronize()
        _spmm_check(oracle, A, B.cpu().numpy(), C.cpu().numpy())
        _sddmm_check(oracle, A, X.cpu().numpy(), Y.cpu().numpy(), out.cpu().numpy())
    finally:
        tdist.destroy_process_group()


# ------------------------------------------------------------------ alternative engines
@pytest.mark.parametrize("var,val", [("SR_PHASE_S", "0"), ("SR_GATHER4", "0"),
                                     ("SR_TASK_NNZ", "1"), ("SR_TASK_NNZ", "1024")])
def test_engines_subprocess(env, var, val):
    """Process-wide kernel choices (SR_PHASE_S=0: the one-row-per-warp phase-S kernels instead of
    the row-group task kernels; SR_GATHER4=0: per-row cp.async.bulk staging instead of TMA
    tile::gather4 in phase D; SR_TASK_NNZ: task size, 1 = one row per task) are fixed once per
    process; rerun the numeric parity cases that exercise them (K sweep incl. multi-pass K,
    tile widths, split rows + RMW rows) under the non-default choices."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    e = dict(os.environ, **{var: val})
    r = subprocess.run([sys.executable, "-m", "pytest", os.path.join(root, "tests", "test_gpu_parity.py"), "-m", "gpu",
                        "-q", "-x", "-p", "no:cacheprovider", "-k", "k_sweep or tile_widths or long_rows"],
                       cwd=root, env=e, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]


# ------------------------------------------------------------------ offline plans + trial (§8(f) N1)
def test_plan_save_load_roundtrip(env, oracle):
    """A saved plan (offline reordering) loads onto a fresh handle of the same
    matrix without LSH / clustering and gives the identical plan and identical outputs."""
    sr, torch = env
    A = g.random_csr(600, 400, 0.03, 31, empty_frac=0.1)
    kw = _plan_kw(16, 1, 8)
    M1 = sr.SparseMatrix.from_csr(A)
    M1.reorder(sr.default_params(**kw, tile_cols=8))
    img = M1.save_plan()
    assert img[:8] == b"SRPLAN01"
    M2 = sr.SparseMatrix.from_csr(A)
    st = M2.load_plan(img)
    assert st["t_lsh1_s"] == 0.0 and st["t_cluster1_s"] == 0.0
    ref = oracle.plan(A, **kw)
    _assert_plan_equal(M2, ref)
    assert M2.save_plan() == img  # canonical image
    for K in (32, 128):
        B = torch.from_numpy(g.dense(400, K)).cuda()
        X = torch.from_numpy(g.dense(600, K, stream=1)).cuda()
        Y = torch.from_numpy(g.dense(400, K, stream=2)).cuda()
        C1, C2 = M1.spmm(B), M2.spmm(B)
        o1, o2 = M1.sddmm(X, Y), M2.sddmm(X, Y)
        torch.cuda.synchronize()
        assert torch.equal(C1, C2) and torch.equal(o1, o2)
        _spmm_check(oracle, A, B.cpu().numpy(), C2.cpu().numpy())


def test_plan_load_shards_and_errors(env, oracle):
    sr, torch = env
    A = g.random_csr(500, 300, 0.03, 21, empty_frac=0.1)
    M = sr.SparseMatrix.from_csr(A)
    M.reorder(sr.default_params(**_plan_kw(16, 1, 0)))
    img = M.save_plan()
    # a shard of the loaded plan equals the shard of a directly reordered handle
    for r in range(2):
        Md = sr.SparseMatrix.from_csr(A)
        Md.reorder(sr.default_params(**_plan_kw(16, 1, 0), world=2, rank=r))
        Ml = sr.SparseMatrix.from_csr(A)
        Ml.load_plan(img, world=2, rank=r)
        np.testing.assert_array_equal(Ml.shard_rows(), Md.shard_rows())
        np.testing.assert_array_equal(Ml.shard_nnz_ids(), Md.shard_nnz_ids())
        B = torch.from_numpy(g.dense(300, 32)).cuda()
        Cd, Cl = Md.spmm(B), Ml.spmm(B)
        torch.cuda.synchronize()
        assert torch.equal(Cd, Cl)
    # corrupted image, other matrix, second plan, bad shard
    bad = bytearray(img)
    bad[100] ^= 1
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix.from_csr(A).load_plan(bytes(bad))
    assert e.value.code == sr.SR_EINVAL
    other = g.random_csr(500, 300, 0.03, 22, empty_frac=0.1)
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix.from_csr(other).load_plan(img)
    assert e.value.code == sr.SR_EINVAL
    with pytest.raises(sr.SRError) as e:
        M.load_plan(img)
    assert e.value.code == sr.SR_ESTATE
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix.from_csr(A).load_plan(img, world=2, rank=2)
    assert e.value.code == sr.SR_EINVAL
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix.from_csr(A).save_plan()  # no plan yet
    assert e.value.code == sr.SR_ESTATE


def test_trial_selects_and_results_agree(env, oracle):
    """sr_trial times the candidates and returns the fastest; every candidate
    computes the same product (checked against the oracle)."""
    sr, torch = env
    A = g.random_csr(2000, 1500, 0.01, 41, empty_frac=0.1)
    orig = sr.SparseMatrix.from_csr(A)
    reo = sr.SparseMatrix.from_csr(A)
    reo.reorder(sr.default_params(**_plan_kw(16, 1, 8)))
    B = torch.from_numpy(g.dense(1500, 64)).cuda()
    best, ms = sr.trial([orig, reo], "spmm", B, reps=3)
    assert best in (0, 1) and len(ms) == 2 and all(t > 0 for t in ms)
    assert ms[best] == min(ms)
    X = torch.from_numpy(g.dense(2000, 64, stream=1)).cuda()
    Y = torch.from_numpy(g.dense(1500, 64, stream=2)).cuda()
    best2, ms2 = sr.trial([reo, orig], "sddmm", X, Y, reps=3)
    assert ms2[best2] == min(ms2)
    for M in (orig, reo):
        C = M.spmm(B)
        torch.cuda.synchronize()
        _spmm_check(oracle, A, B.cpu().numpy(), C.cpu().numpy())
    other = sr.SparseMatrix.from_csr(g.random_csr(1999, 1500, 0.01, 42))
    with pytest.raises(sr.SRError):
        sr.trial([orig, other], "spmm", B)


def test_set_values_reuses_the_plan(env, oracle):
    """sr_set_values (iterative use of one plan with new values): SpMM and
    SDDMM over the same plan with replaced values match the oracle on the new matrix; the
    sharded form takes values in the packed shard order."""
    sr, torch = env
    A = g.random_csr(700, 500, 0.03, 5, empty_frac=0.1)
    A2 = g.CSR(A.nrows, A.ncols, A.rowptr, A.colidx, g._uniform_vals(A.nnz, 77))
    for params in (None, sr.default_params(**_plan_kw(16, 1, 8), tile_cols=8), sr.default_params(**_plan_kw(8, 1, 8))):
        M = sr.SparseMatrix.from_csr(A)
        if params is not None:
            M.reorder(params)
        M.set_values(torch.from_numpy(A2.vals).cuda())
        for K in (32, 128):
            B = g.dense(A.ncols, K)
            X, Y = g.dense(A.nrows, K, stream=1), g.dense(A.ncols, K, stream=2)
            C = M.spmm(torch.from_numpy(B).cuda())
            out = M.sddmm(torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda())
            torch.cuda.synchronize()
            _spmm_check(oracle, A2, B, C.cpu().numpy())
            _sddmm_check(oracle, A2, X, Y, out.cpu().numpy())
    # sharded: packed order
    K = 32
    B = g.dense(A.ncols, K)
    C = np.full((A.nrows, K), np.nan, np.float32)
    for r in range(2):
        M = sr.SparseMatrix.from_csr(A)
        M.reorder(sr.default_params(**_plan_kw(16, 1, 0), world=2, rank=r))
        ids = M.shard_nnz_ids()
        M.set_values(torch.from_numpy(np.ascontiguousarray(A2.vals[ids])).cuda())
        Cr = M.spmm(torch.from_numpy(B).cuda())
        torch.cuda.synchronize()
        C[M.shard_rows()] = Cr.cpu().numpy()
    _spmm_check(oracle, A2, B, C)


def test_cf_gradient_loop(env):
    """N2: the CF gradient (one SDDMM + two SpMMs over the reordered plans of R and Rᵀ)
    against dense fp64 numpy on a small ratings matrix; the loss decreases."""
    sr, torch = env
    from paper_conf_ppopp_jiangha20_b200.cf import CFModel
    A = g.random_csr(300, 200, 0.05, 9, empty_frac=0.05)
    R = g.CSR(A.nrows, A.ncols, A.rowptr, A.colidx,
              np.random.default_rng(1).integers(1, 6, A.nnz).astype(np.float32))
    K = 16
    m = CFModel(R, K, params=sr.default_params(**_plan_kw(16, 1, 8)))
    U, V = m.U.double().cpu().numpy(), m.V.double().cpu().numpy()
    E, gU, gV = m.gradients(lam=0.0)
    torch.cuda.synchronize()
    rows = np.repeat(np.arange(R.nrows), np.diff(R.rowptr))
    Pd = np.einsum("ik,ik->i", U[rows], V[R.colidx])
    Ed = Pd - R.vals
    D = np.zeros((R.nrows, R.ncols))
    D[rows, R.colidx] = Ed
    np.testing.assert_allclose(E.cpu().numpy(), Ed, rtol=1e-5, atol=1e-4)
    bU = np.abs(D) @ np.abs(V) + 1e-30
    bV = np.abs(D).T @ np.abs(U) + 1e-30
    assert (np.abs(gU.cpu().numpy() - D @ V) <= 1e-4 * bU + 1e-6).all()
    assert (np.abs(gV.cpu().numpy() - D.T @ U) <= 1e-4 * bV + 1e-6).all()
    losses = [m.step(lr=0.01) for _ in range(20)]
    assert losses[-1] < losses[0]
    m.close()
