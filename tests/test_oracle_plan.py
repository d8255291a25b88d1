"""Pins of oracle O8-O14: Alg 3 clustering (Fig 6), ASpT tiling (P:111,
P:131), the access-count model, AvgSim, the
AUTO decision rules and the nnz-balanced partition.  Expected values
come from the paper's worked example (tests/golden) or are derived by hand below.
CPU only."""
import numpy as np
import pytest

from synth import generators as g
from conftest import golden


def _csr(sets, ncols):
    rowptr = np.zeros(len(sets) + 1, np.int64)
    np.cumsum([len(s) for s in sets], out=rowptr[1:])
    colidx = np.array([c for s in sets for c in sorted(s)], np.int32)
    return g.CSR(len(sets), ncols, rowptr, colidx, np.ones(colidx.size, np.float32))


# ------------------------------------------------------------------ Alg 3
def test_fig6_trace(oracle):
    gd = golden("fig1a.json")["fig6"]
    A = g.fig1a()
    perm = oracle.cluster(A.rowptr, A.colidx, oracle.pack_pairs(gd["candidates"]), gd["threshold_size"])
    assert perm.tolist() == gd["reordered_rows"]


def test_fig6_with_precomputed_similarities(oracle):
    """Same trace when the candidates' (inter, uni) come in from outside."""
    A = g.fig1a()
    pairs = oracle.pack_pairs([(0, 4), (2, 4)])
    perm = oracle.cluster(A.rowptr, A.colidx, pairs, 256, inter=np.array([2, 1]), uni=np.array([3, 4]))
    assert perm.tolist() == [0, 2, 4, 1, 3, 5]


def test_round2_either_pair_gives_fig4c(oracle):
    """for the remaining sparse part, LSH generating either (1,4) or (2,5)
    groups 1,4 / 2,5 together (Fig 4c).  Positional ids (R19): after round 1 the
    remainder positions are q=1 (row 2, {5}), q=2 (row 4, {3}), q=3 (row 1, {3}),
    q=5 (row 5, {5}); rows 1,4 = positions 3,2 and rows 2,5 = positions 1,5."""
    A = g.fig1a()
    t = oracle.tile(A, [0, 2, 4, 1, 3, 5], 3, 2)
    R_ptr, R_col = t["rrow_ptr"], t["r_col"]
    nonempty = lambda perm: [q for q in perm if R_ptr[q + 1] > R_ptr[q]]
    both = nonempty(oracle.cluster(R_ptr, R_col, oracle.pack_pairs([(2, 3), (1, 5)]), 256))
    only14 = nonempty(oracle.cluster(R_ptr, R_col, oracle.pack_pairs([(2, 3)]), 256))
    only25 = nonempty(oracle.cluster(R_ptr, R_col, oracle.pack_pairs([(1, 5)]), 256))
    for order in (both, only14, only25):
        # the grouping of Fig 4c: consecutive pairs share their column
        assert oracle.access_count(t, order, 2) == 4 + 2


def test_threshold_deletes_cluster(oracle):
    """Hand trace, threshold_size = 2: pop (0,1) J=1 -> merge, size 2 >= 2 -> deleted;
    pop (1,2): 1 is not a root, root(1) = 0 is deleted -> skip.  Output rule B:
    cluster {0,1}, then singletons 2, 3."""
    A = _csr([{1, 2}, {1, 2}, {1, 2, 3}, {9}], 10)
    pairs = oracle.pack_pairs([(0, 1), (1, 2)])
    assert oracle.cluster(A.rowptr, A.colidx, pairs, 2).tolist() == [0, 1, 2, 3]
    # with a large threshold, 2 joins (re-inserted pair (0,2) J = 2/3)
    assert oracle.cluster(A.rowptr, A.colidx, pairs, 256).tolist() == [0, 1, 2, 3]
    # order check: cluster members ascending, clusters before singletons
    B = _csr([{7}, {1, 2}, {5}, {1, 2}], 10)
    assert oracle.cluster(B.rowptr, B.colidx, oracle.pack_pairs([(1, 3)]), 256).tolist() == [1, 3, 0, 2]


def test_larger_cluster_wins_and_tie_goes_to_smaller_index(oracle):
    """R6 / P:149: merge smaller into larger; equal size -> smaller index is the root.
    Rows 3,4 merge first (J=1, root 3); then pair (2,3) (J=1/2... ) merges {2} into
    the larger cluster rooted at 3 -> output [2,3,4] as one cluster, 0 and 1 after."""
    A = _csr([{20}, {21}, {1, 9}, {1}, {1}], 30)
    perm = oracle.cluster(A.rowptr, A.colidx, oracle.pack_pairs([(3, 4), (2, 3)]), 256)
    assert perm.tolist() == [2, 3, 4, 0, 1]


def test_equal_size_root_is_smaller_index_output_order(oracle):
    """R6 (Fig 6 first merge (0,4) -> root 0) seen through rule B's root order:
    pairs (0,3) and (1,2), both J = 1, equal sizes.  Smaller-index roots 0 and 1 ->
    clusters emitted as [0,3] then [1,2]; larger-index roots (3 and 2) would emit [1,2]
    first (hand-derived)."""
    A = _csr([{1}, {2}, {2}, {1}], 4)
    perm = oracle.cluster(A.rowptr, A.colidx, oracle.pack_pairs([(0, 3), (1, 2)]), 256)
    assert perm.tolist() == [0, 3, 1, 2]


def test_size_update_drives_threshold_deletion(oracle):
    """R4 + R7: after merging (0,1) the cluster has size 2 >= threshold 2 and is
    deleted, so the later pair (1,3) (root 0 deleted) is skipped and row 3 stays a singleton:
    [0,1,2,3].  Without the size update the cluster would absorb row 3 through the
    re-inserted pair (0,3) (J = 2/3) and give [0,1,3,2] (hand-derived)."""
    A = _csr([{1, 2}, {1, 2}, {7}, {1, 2, 3}], 8)
    perm = oracle.cluster(A.rowptr, A.colidx, oracle.pack_pairs([(0, 1), (1, 3)]), 2)
    assert perm.tolist() == [0, 1, 2, 3]
    assert oracle.cluster(A.rowptr, A.colidx, oracle.pack_pairs([(0, 1), (1, 3)]), 256).tolist() == [0, 1, 3, 2]


def _check_invariants(perm, M, threshold):
    assert sorted(perm.tolist()) == list(range(M))


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_cluster_invariants_random(oracle, seed):
    A = g.random_csr(300, 80, 0.05, seed, empty_frac=0.2)
    thr = 8
    E = oracle.candidates(A.rowptr, A.colidx, 32, 2, 4, 0)
    perm = oracle.cluster(A.rowptr, A.colidx, E, thr)
    _check_invariants(perm, 300, thr)
    # empty rows are singletons (R16); rule B puts all singletons, ascending, after
    # the clusters, so the tail from the first empty row on is ascending
    deg = np.diff(A.rowptr)
    empties = [r for r in range(300) if deg[r] == 0]
    first = min(perm.tolist().index(r) for r in empties)
    tail = perm[first:].tolist()
    assert tail == sorted(tail) and set(empties) <= set(tail)


def test_no_candidates_is_identity(oracle):
    A = g.random_csr(50, 50, 0.1, 4)
    perm = oracle.cluster(A.rowptr, A.colidx, np.zeros(0, np.uint64), 256)
    assert perm.tolist() == list(range(50))


# ------------------------------------------------------------------ tiler + access model
def test_aspt_identity_fig3(oracle):
    gd = golden("fig1a.json")["aspt"]
    A = g.fig1a()
    t = oracle.tile(A, np.arange(6), gd["panel_rows"], gd["dense_min"])
    assert t["n_dense"] == gd["identity_dense_nnz"]
    assert [t["dense_cols"][t["dense_ptr"][p]:t["dense_ptr"][p + 1]].tolist() for p in range(2)] \
        == gd["identity_dense_cols"]
    order = [q for q in range(6) if t["rrow_ptr"][q + 1] > t["rrow_ptr"][q]]
    assert oracle.access_count(t, order, gd["warps_per_cta"]) == gd["identity_accesses"]
    # row-wise implementation: no dense tiles at all
    t0 = oracle.tile(A, np.arange(6), gd["panel_rows"], 10 ** 6)
    assert t0["n_dense"] == 0
    assert oracle.access_count(t0, list(range(6)), gd["warps_per_cta"]) == gd["rowwise_accesses"]


def test_aspt_after_reordering_fig4(oracle):
    gd = golden("fig1a.json")["aspt"]
    A = g.fig1a()
    t = oracle.tile(A, golden("fig1a.json")["fig6"]["reordered_rows"], 3, 2)
    assert t["n_dense"] == gd["reordered_dense_nnz"]
    assert t["dense_ptr"][-1] == gd["reordered_dense_col_count"]
    # panel 0 = rows 0,2,4: column 4 (3 nnz) first, then column 0 (2 nnz) (R18)
    assert t["dense_cols"][:2].tolist() == [4, 0]
    # every nnz is in exactly one of dense tiles / remainder
    assert sorted(np.concatenate([t["d_pos"], t["r_pos"]]).tolist()) == list(range(13))
    # full FORCE pipeline: round-2 LSH finds exactly the two identical-column pairs
    R_ptr, R_col = t["rrow_ptr"], t["r_col"]
    E = oracle.candidates(R_ptr, R_col, 128, 2, 4, 0)
    assert [(int(e) >> 32, int(e) & 0xFFFFFFFF) for e in E] == [(1, 5), (2, 3)]
    perm2, _ = oracle.reorder_rows(R_ptr, R_col, 128, 2, 4, 0, 256)
    order = [q for q in perm2 if R_ptr[q + 1] > R_ptr[q]]
    assert oracle.access_count(t, order, 2) == gd["reordered_accesses_with_round2"]
    assert oracle.access_count(t, [1, 2, 3, 5], 2) == 8  # without round 2 (hand-derived)


def test_dense_ratio_and_avgsim_of_example(oracle):
    """DenseRatio of the original matrix 2/13; AvgSim of the remainder after
    round 1 = 1/3 (hand-derived from Fig 4b)."""
    A = g.fig1a()
    p = oracle.plan(A, panel_rows=3, dense_min=2, mode=oracle.MODE_OFF)
    assert (p["stats"]["dense0"], p["stats"]["nnz"]) == (2, 13)
    t = oracle.tile(A, [0, 2, 4, 1, 3, 5], 3, 2)
    num, den = oracle.avgsim(t["rrow_ptr"], t["r_col"])
    assert num * 3 == den


def test_fig7a_avgsim_and_tiles(oracle):
    gd = golden("fig7a.json")
    A = _csr([set(r) for r in gd["rows"]], 6)
    num, den = oracle.avgsim(A.rowptr, A.colidx)
    assert num * gd["avgsim"][1] == den * gd["avgsim"][0]
    assert oracle.tile(A, np.arange(6), gd["panel_rows"], 2)["n_dense"] == gd["dense_nnz"]


def test_avgsim_fixed_point_rounding(oracle):
    """R27: each term floor(2^32·inter/uni), exact sum.  J = 1/3 -> floor(2^32/3)."""
    A = _csr([{0, 1, 2}, {2}, set(), {2, 5}], 6)
    num, den = oracle.avgsim(A.rowptr, A.colidx)
    assert den == 2 << 32
    assert num == (2 ** 32) // 3 + (2 ** 32) // 2


def test_tiler_invariants_random(oracle):
    A = g.random_csr(500, 120, 0.05, 41, empty_frac=0.1)
    perm = np.random.default_rng(1).permutation(500).astype(np.int32)
    P, dmin = 16, 2
    t = oracle.tile(A, perm, P, dmin)
    assert sorted(np.concatenate([t["d_pos"], t["r_pos"]]).tolist()) == list(range(A.nnz))
    rowof = np.repeat(np.arange(500), np.diff(A.rowptr))
    for p in range(t["npanels"]):
        D = t["dense_cols"][t["dense_ptr"][p]:t["dense_ptr"][p + 1]]
        rows = perm[p * P:(p + 1) * P]
        cnt = {}
        for r in rows:
            for c in A.colidx[A.rowptr[r]:A.rowptr[r + 1]]:
                cnt[c] = cnt.get(c, 0) + 1
        expect = sorted([c for c, n in cnt.items() if n >= dmin], key=lambda c: (-cnt[c], c))
        assert D.tolist() == expect
        for q in range(p * P, min((p + 1) * P, 500)):
            ds = t["d_slot"][t["drow_ptr"][q]:t["drow_ptr"][q + 1]]
            dp = t["d_pos"][t["drow_ptr"][q]:t["drow_ptr"][q + 1]]
            assert np.all(np.diff(ds) > 0)
            assert np.all(rowof[dp] == perm[q]) and np.all(D[ds] == A.colidx[dp])
            rp = t["r_pos"][t["rrow_ptr"][q]:t["rrow_ptr"][q + 1]]
            assert np.all(rowof[rp] == perm[q]) and np.all(np.diff(rp) > 0)
            assert not set(A.colidx[rp].tolist()) & set(D.tolist())


# ------------------------------------------------------------------ driver
def test_auto_skips_round1_on_clustered_matrix(oracle):
    """skip round 1 if DenseRatio > 10%; skip round 2 if AvgSim > 0.1."""
    gd = golden("fig7a.json")
    A = _csr([set(r) for r in gd["rows"]], 6)
    p = oracle.plan(A, panel_rows=3, dense_min=2, mode=oracle.MODE_AUTO)
    assert p["stats"]["round1"] == 0 and p["perm1"].tolist() == list(range(6))
    assert p["stats"]["E1"] == 0


def test_auto_runs_round1_on_scattered_matrix(oracle):
    A = g.random_csr(512, 512, 0.008, 8)
    p = oracle.plan(A, panel_rows=8, dense_min=2, mode=oracle.MODE_AUTO, seed=4)
    assert p["stats"]["dense0"] * 10 <= p["stats"]["nnz"]
    assert p["stats"]["round1"] == 1
    assert sorted(p["perm1"].tolist()) == list(range(512))


def test_auto_on_fig1a_skips_round1_runs_round2(oracle):
    """Fig 1a under AUTO with the example's ASpT parameters (panel 3, dense >= 2):
    DenseRatio0 = 2/13 > 1/10 -> round 1 skipped, perm1 = identity.  The
    remainder of the identity tiling is {0}, {1,2,3}, {5} | {1}, {0,3,4}, {2,5} (column 4 of
    panel 0 is the only dense column): no two consecutive rows share a column, so
    AvgSim = 0 <= 1/10 and round 2 runs (hand-derived)."""
    A = g.fig1a()
    p = oracle.plan(A, panel_rows=3, dense_min=2, mode=oracle.MODE_AUTO)
    st = p["stats"]
    assert (st["dense0"], st["nnz"]) == (2, 13)
    assert st["round1"] == 0 and p["perm1"].tolist() == list(range(6))
    assert st["avgsim_num"] == 0 and st["round2"] == 1
    assert sorted(p["perm2"].tolist()) == list(range(6))


def test_auto_skips_round2_when_remainder_is_clustered(oracle):
    """skip round 2 iff AvgSim > 0.1.  Rows {0,1},{0,1},{5,6},{5,6}, no dense
    columns (dense_min 100): DenseRatio0 = 0 -> round 1 runs; LSH pairs the identical
    rows (every band collides), Alg 3 keeps perm1 = [0,1,2,3]; AvgSim = (1+0+1)/3 = 2/3
    > 1/10 -> round 2 skipped, perm2 = [0,1,2,3], E2 = 0 (hand-derived)."""
    A = _csr([{0, 1}, {0, 1}, {5, 6}, {5, 6}], 8)
    p = oracle.plan(A, panel_rows=2, dense_min=100, mode=oracle.MODE_AUTO)
    st = p["stats"]
    assert st["round1"] == 1 and p["perm1"].tolist() == [0, 1, 2, 3]
    assert st["avgsim_num"] * 3 == st["avgsim_den"] * 2
    assert st["round2"] == 0 and st["E2"] == 0 and p["perm2"].tolist() == [0, 1, 2, 3]


@pytest.mark.parametrize("pairs,expect_round2", [(1, 1), (2, 0)])
def test_auto_round2_threshold_is_strict(oracle, pairs, expect_round2):
    """"greater than 0.1" (R20 strict >).  11 non-empty rows with one identical
    pair (rows 0, 5): round 1 clusters them (rule B: [0, 5, 1, 2, 3, 4, 6, ...]) and the
    remainder's AvgSim is exactly 1/10 -> round 2 runs.  12 rows with two identical
    pairs (0, 5) and (6, 11): AvgSim = 2/11 > 1/10 -> round 2 skipped."""
    n = 11 if pairs == 1 else 12
    sets = [{20 + i} for i in range(n)]
    sets[0] = sets[5] = {0, 1}
    if pairs == 2:
        sets[6] = sets[11] = {2, 3}
    A = _csr(sets, 40)
    p = oracle.plan(A, panel_rows=4, dense_min=100, mode=oracle.MODE_AUTO)
    st = p["stats"]
    clustered = [0, 5] if pairs == 1 else [0, 5, 6, 11]
    expect1 = clustered + [r for r in range(n) if r not in clustered]
    assert st["round1"] == 1 and p["perm1"].tolist() == expect1
    assert st["avgsim_num"] * (n - 1) == st["avgsim_den"] * pairs
    assert st["round2"] == expect_round2


def test_auto_decision_threshold_separate_from_execution_threshold(oracle):
    """R28: DenseRatio0 of the AUTO decision is taken with the decision's dense
    criterion auto_dense_min, the tiling the kernels run with uses dense_min.  Fig 1a with
    execution threshold 3 (no column of a 3-row panel has 3 nnz): decided at 2, DenseRatio0
    = 2/13 > 1/10 -> round 1 skipped, and the identity plan has no dense nnz; decided at the
    execution threshold (auto_dense_min 0), DenseRatio0 = 0 -> round 1 runs (hand-derived)."""
    A = g.fig1a()
    p = oracle.plan(A, panel_rows=3, dense_min=3, auto_dense_min=2, mode=oracle.MODE_AUTO)
    st = p["stats"]
    assert (st["dense0"], st["round1"], st["dense1"]) == (2, 0, 0)
    assert p["perm1"].tolist() == list(range(6)) and p["dense_ptr"].tolist() == [0, 0, 0]
    q = oracle.plan(A, panel_rows=3, dense_min=3, auto_dense_min=0, mode=oracle.MODE_AUTO)
    assert (q["stats"]["dense0"], q["stats"]["round1"]) == (0, 1)


def test_plan_modes_consistent(oracle):
    A = g.random_csr(200, 150, 0.04, 9, empty_frac=0.15)
    off = oracle.plan(A, panel_rows=8, mode=oracle.MODE_OFF)
    assert off["perm1"].tolist() == list(range(200))
    nonempty = [q for q in range(200) if off["rrow_ptr"][q + 1] > off["rrow_ptr"][q]]
    assert off["perm2"].tolist() == nonempty
    force = oracle.plan(A, panel_rows=8, mode=oracle.MODE_FORCE)
    assert force["stats"]["round1"] == 1 and force["stats"]["round2"] == 1
    assert sorted(force["perm2"].tolist()) == sorted(
        q for q in range(200) if force["rrow_ptr"][q + 1] > force["rrow_ptr"][q])


# ------------------------------------------------------------------ partition
def _bruteforce_cuts(w, G):
    total = sum(w)
    prefix = np.concatenate([[0], np.cumsum(w)])
    cuts = [0]
    for gg in range(1, G):
        cuts.append(min([p for p in range(len(w) + 1) if prefix[p] * G >= gg * total] + [len(w)]))
    return cuts + [len(w)]


@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
def test_partition(oracle, G):
    rng = np.random.default_rng(G)
    for trial in range(20):
        w = rng.integers(0, 50, size=int(rng.integers(1, 40)))
        if trial == 0:
            w[-3:] = 0  # trailing empty panels must still be covered
        cuts = oracle.partition(w, G)
        assert cuts.tolist() == _bruteforce_cuts(w.tolist(), G)
        assert cuts[0] == 0 and cuts[-1] == w.size and np.all(np.diff(cuts) >= 0)
        total = w.sum()
        for gg in range(G):
            nnz_g = w[cuts[gg]:cuts[gg + 1]].sum()
            assert abs(nnz_g * G - total) <= max(w.max(), 0) * G + G  # within one panel
