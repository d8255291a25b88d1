"""CPU-only checks of the C ABI: libsr.so loads and exports every symbol include/sr.h
declares; argument validation; the host half of the pipeline (Alg 3 clustering, panel
partition) is bit-exact against the oracle.  No GPU compute calls."""
import ctypes as C
import os
import re

import numpy as np
import pytest

from synth import generators as g

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def sr():
    import paper_conf_ppopp_jiangha20_b200 as sr
    if not os.path.exists(sr.LIB_PATH):
        from paper_conf_ppopp_jiangha20_b200 import _build
        _build.build()
    sr.lib()
    return sr


def test_exports_every_declared_symbol(sr):
    hdr = open(os.path.join(ROOT, "include", "sr.h")).read()
    declared = set(re.findall(r"^\s*(?:int|void|const char\*)\s+(sr_\w+)\s*\(", hdr, re.M))
    assert len(declared) >= 15
    lib = C.CDLL(sr.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name
    assert declared == set(sr.EXPORTED)


def test_no_unresolved_library_symbols(sr):
    """Every symbol of the library's own namespace is defined inside libsr.so (a declaration
    without a definition would only fail when the library is loaded on the GPU box)."""
    import subprocess
    out = subprocess.check_output(["nm", "-D", "--undefined-only", sr.LIB_PATH], text=True)
    missing = [l for l in out.splitlines() if "_ZN2sr" in l or " sr_" in l]
    assert not missing, missing


def _c_layout(struct, fields):
    """sizeof / offsetof of a struct of include/sr.h, compiled with gcc (the header is the
    authority the ctypes binding must match)."""
    import subprocess
    import tempfile
    body = "".join(f'  printf("%zu\\n", offsetof({struct}, {f}));\n' for f in fields)
    src = ("#include <stddef.h>\n#include <stdio.h>\n#include \"sr.h\"\n"
           f"int main(void) {{\n  printf(\"%zu\\n\", sizeof({struct}));\n{body}  return 0;\n}}\n")
    with tempfile.TemporaryDirectory() as d:
        c, exe = os.path.join(d, "l.c"), os.path.join(d, "l")
        with open(c, "w") as f:
            f.write(src)
        subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), c, "-o", exe])
        vals = [int(x) for x in subprocess.check_output([exe]).split()]
    return vals[0], dict(zip(fields, vals[1:]))


@pytest.mark.parametrize("struct,cls", [("sr_reorder_params", "ReorderParams"), ("sr_plan_stats", "PlanStats"),
                                        ("sr_traffic_model", "TrafficModel")])
def test_struct_layouts_match_header(sr, struct, cls):
    T = getattr(sr, cls)
    fields = [f for f, _ in T._fields_]
    size, off = _c_layout(struct, fields)
    assert C.sizeof(T) == size
    for f in fields:
        assert getattr(T, f).offset == off[f], f


def test_default_params(sr):
    p = sr.default_params()
    assert (p.siglen, p.bsize, p.threshold_size, p.max_bucket, p.seed) == (128, 2, 256, 32, 4)
    assert (p.panel_rows, p.dense_min, p.tile_cols, p.mode) == (64, 2, 64, sr.AUTO)
    assert (p.skip_dense_num, p.skip_dense_den, p.skip_sim_num, p.skip_sim_den) == (1, 10, 1, 10)
    assert (p.world, p.rank, p.auto_dense_min, p.reserved0) == (1, 0, 0, 0)


def test_create_validates_before_touching_a_device(sr):
    A = g.fig1a()
    bad = A.colidx.copy()
    bad[0] = 99
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix(6, 6, A.rowptr, bad, A.vals)
    assert e.value.code == sr.SR_EINVAL
    dup = A.colidx.copy()
    dup[1] = 0
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix(6, 6, A.rowptr, dup, A.vals)
    assert e.value.code == sr.SR_EINVAL
    rp = A.rowptr.copy()
    rp[2] = 1  # decreasing
    with pytest.raises(sr.SRError) as e:
        sr.SparseMatrix(6, 6, rp, A.colidx, A.vals)
    assert e.value.code == sr.SR_EINVAL


def _sorted_pairs(E):
    return np.sort(E)


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_host_cluster_bit_exact_vs_oracle(sr, oracle, seed):
    A = g.random_csr(400, 120, 0.04, seed, empty_frac=0.15)
    E = oracle.candidates(A.rowptr, A.colidx, 32, 2, 4, 0)
    for thr in (2, 5, 256):
        ref = oracle.cluster(A.rowptr, A.colidx, E, thr)
        got = sr.host_cluster(A.rowptr, A.colidx, E, thr)
        np.testing.assert_array_equal(got, ref)
        inter, uni = oracle.jaccard_pairs(A.rowptr, A.colidx, E)
        got2 = sr.host_cluster(A.rowptr, A.colidx, E, thr, inter=inter, uni=uni)
        np.testing.assert_array_equal(got2, ref)


@pytest.mark.parametrize("seed", [5, 6, 7])
def test_host_cluster_reinserts_and_zero_similarity_pairs(sr, oracle, seed):
    """The library's Alg 3 keeps re-inserted pairs with J = 0 apart from the heap and proves
    J = 0 from row digests: compare with the oracle's plain priority queue on matrices where
    most re-inserts have J = 0 (power-law-ish columns, many clusters), and with caller-given
    candidates that include J = 0 pairs (allowed by sr_host_cluster, never made by the LSH)."""
    rng = np.random.default_rng(seed)
    A = g.random_csr(3000, 4000, 0.002, seed, empty_frac=0.1)
    E = oracle.candidates(A.rowptr, A.colidx, 32, 2, 4, 8)
    extra = rng.integers(0, 3000, size=(400, 2))
    E2 = oracle.pack_pairs([(int(i), int(j)) for i, j in extra if i != j] +
                           [(int(e) >> 32, int(e) & 0xFFFFFFFF) for e in E])
    for pairs in (E, E2):
        for thr in (3, 16, 256):
            ref = oracle.cluster(A.rowptr, A.colidx, pairs, thr)
            np.testing.assert_array_equal(sr.host_cluster(A.rowptr, A.colidx, pairs, thr), ref)


def test_host_cluster_fig6(sr):
    A = g.fig1a()
    from oracle import oracle as O
    assert sr.host_cluster(A.rowptr, A.colidx, O.pack_pairs([(0, 4), (2, 4)]), 256).tolist() == [0, 2, 4, 1, 3, 5]


def test_host_cluster_rejects_unsorted_pairs(sr):
    A = g.fig1a()
    with pytest.raises(sr.SRError):
        sr.host_cluster(A.rowptr, A.colidx, np.array([(2 << 32) | 4, 4], np.uint64), 256)


@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_host_partition_matches_oracle(sr, oracle, G):
    rng = np.random.default_rng(G)
    for _ in range(25):
        w = rng.integers(0, 1000, size=int(rng.integers(1, 300)))
        w[rng.random(w.size) < 0.2] = 0
        np.testing.assert_array_equal(sr.host_partition(w, G), oracle.partition(w, G))


def test_transpose_csr_matches_dense():
    """cf.transpose_csr (host helper of the CF loop): Aᵀ and the nnz permutation."""
    import numpy as np
    from paper_conf_ppopp_jiangha20_b200.cf import transpose_csr
    from synth import generators as g
    A = g.random_csr(40, 30, 0.2, 3, empty_frac=0.1)
    trp, tcol, perm = transpose_csr(A.nrows, A.ncols, A.rowptr, A.colidx)
    D = np.zeros((A.nrows, A.ncols))
    rows = np.repeat(np.arange(A.nrows), np.diff(A.rowptr))
    D[rows, A.colidx] = A.vals
    T = np.zeros((A.ncols, A.nrows))
    trows = np.repeat(np.arange(A.ncols), np.diff(trp))
    T[trows, tcol] = A.vals[perm]
    np.testing.assert_array_equal(T, D.T)
    for r in range(A.ncols):  # columns sorted within each row of Aᵀ
        assert np.all(np.diff(tcol[trp[r]:trp[r + 1]]) > 0)
