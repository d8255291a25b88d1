"""Pins of oracle O3-O7 (minhash LSH, P:151-153 and ref [28] ch.3; exact Jaccard,
P:143-147) against published test vectors, algebraic inverses, the minhash
probability law, and brute-force Python enumeration.  CPU only."""
import math

import numpy as np
import pytest

from synth import generators as g
from conftest import golden

MASK32 = 0xFFFFFFFF


def test_splitmix64_published_vector(oracle):
    # SplitMix64 reference outputs for seed 1234567 (Steele/Lea/Vigna test vector)
    assert oracle.splitmix64_stream(1234567, 5) == [
        6457827717110365317, 3203168211198807973, 9817491932198370423,
        4593380528125082431, 16408922859458223821]


def test_fmix32_published_vectors(oracle):
    # MurmurHash3_x86_32("", seed) = fmix32(seed ^ 0): published values
    assert oracle.fmix32(0) == 0
    assert oracle.fmix32(1) == 0x514E28B7
    assert oracle.fmix32(0xFFFFFFFF) == 0x81F16F39


def _inv_fmix32(h):
    """Algebraic inverse of the Murmur3 finalizer (not the same formula)."""
    def unxorshift(x, s):
        y = x
        for _ in range(32 // s + 1):
            y = x ^ (y >> s)
        return y & MASK32
    h = unxorshift(h, 16)
    h = (h * pow(0xC2B2AE35, -1, 1 << 32)) & MASK32
    h = unxorshift(h, 13)
    h = (h * pow(0x85EBCA6B, -1, 1 << 32)) & MASK32
    return unxorshift(h, 16)


def test_hash_is_bijective(oracle):
    """h_s(c) = fmix32(a·c + b): a odd => affine map invertible; fmix32 invertible.
    Check the explicit inverse on random points, so equal minima imply a shared column."""
    a, b = oracle.hash_params(4, 8)
    assert np.all(a % 2 == 1)
    rng = np.random.default_rng(0)
    for s in range(8):
        ainv = pow(int(a[s]), -1, 1 << 32)
        for c in rng.integers(0, 1 << 32, size=200, dtype=np.uint64):
            h = oracle.hash_(int(a[s]), int(b[s]), int(c))
            back = (_inv_fmix32(h) - int(b[s])) * ainv & MASK32
            assert back == int(c)


def test_hash_params_deterministic_and_seeded(oracle):
    a1, b1 = oracle.hash_params(4, 128)
    a2, b2 = oracle.hash_params(4, 128)
    a3, _ = oracle.hash_params(5, 128)
    assert np.array_equal(a1, a2) and np.array_equal(b1, b2)
    assert not np.array_equal(a1, a3)
    assert len(set(a1.tolist())) == 128


def _pair_csr(sets, ncols):
    rowptr = np.zeros(len(sets) + 1, np.int64)
    np.cumsum([len(s) for s in sets], out=rowptr[1:])
    colidx = np.array([c for s in sets for c in sorted(s)], np.int32)
    return g.CSR(len(sets), ncols, rowptr, colidx, np.ones(colidx.size, np.float32))


def test_signature_is_min_over_row(oracle):
    A = g.random_csr(20, 50, 0.2, 8, empty_frac=0.2)
    sig = oracle.signatures(A.rowptr, A.colidx, 16, 4)
    a, b = oracle.hash_params(4, 16)
    for i in range(20):
        cols = A.colidx[A.rowptr[i]:A.rowptr[i + 1]]
        for s in range(16):
            if cols.size == 0:
                assert sig[i, s] == 0xFFFFFFFF  # untouched (R16)
            else:
                assert sig[i, s] == min(oracle.hash_(int(a[s]), int(b[s]), int(c)) for c in cols)


@pytest.mark.parametrize("J_target", [0.1, 0.3, 0.6])
def test_minhash_match_fraction_estimates_jaccard(oracle, J_target):
    """Mining of Massive Datasets ch.3: P[sig_i[s] == sig_j[s]] = J(S_i, S_j).  Over
    300 pairs x 128 hash functions the mean match fraction is within 4 sigma."""
    rng = np.random.default_rng(int(J_target * 100))
    sets, Js = [], []
    n = 40
    for _ in range(300):
        shared = int(round(2 * n * J_target / (1 + J_target)))
        pool = rng.choice(100000, size=2 * n, replace=False)
        s1 = set(pool[:n].tolist())
        s2 = set(pool[:shared].tolist()) | set(pool[n:2 * n - shared].tolist())
        sets += [s1, s2]
        Js.append(len(s1 & s2) / len(s1 | s2))
    A = _pair_csr(sets, 100000)
    sig = oracle.signatures(A.rowptr, A.colidx, 128, 4)
    match = (sig[0::2] == sig[1::2]).mean(axis=1)
    J = np.array(Js)
    err = match.mean() - J.mean()
    sigma = math.sqrt(np.mean(J * (1 - J)) / (128 * 300))
    assert abs(err) < 4 * sigma + 1e-3, (match.mean(), J.mean())


def test_candidate_probability_law(oracle):
    """P[candidate] = 1 - (1 - J^bsize)^(siglen/bsize) (ref [28] ch.3 S-curve), checked
    at J = 0.1 (0.474) and J = 0.2 (0.927) with siglen 128, bsize 2 over many pairs."""
    for J_target in (0.1, 0.2):
        rng = np.random.default_rng(7)
        sets = []
        n = 45
        shared = int(round(2 * n * J_target / (1 + J_target)))
        Jexact = shared / (2 * n - shared)
        npairs = 400
        for _ in range(npairs):
            pool = rng.choice(10 ** 7, size=2 * n, replace=False)
            sets += [set(pool[:n].tolist()), set(pool[:shared].tolist()) | set(pool[n:2 * n - shared].tolist())]
        A = _pair_csr(sets, 10 ** 7)
        E = oracle.candidates(A.rowptr, A.colidx, 128, 2, 4, 0)
        emitted = set(E.tolist())
        hits = sum(1 for p in range(npairs) if ((2 * p) << 32 | (2 * p + 1)) in emitted)
        expect = 1 - (1 - Jexact ** 2) ** 64
        frac = hits / npairs
        sigma = math.sqrt(expect * (1 - expect) / npairs)
        assert abs(frac - expect) < 4 * sigma + 0.02, (J_target, frac, expect)


def _bruteforce_candidates(sig, live, bsize, max_bucket):
    siglen = sig.shape[1]
    pairs = set()
    for band in range(siglen // bsize):
        buckets = {}
        for r in live:
            buckets.setdefault(tuple(sig[r, band * bsize:(band + 1) * bsize].tolist()), []).append(r)
        for members in buckets.values():
            members = sorted(members)
            chunk = max_bucket if max_bucket > 0 else len(members)
            for c0 in range(0, len(members), chunk):
                ch = members[c0:c0 + chunk]
                for x in range(len(ch)):
                    for y in range(x + 1, len(ch)):
                        pairs.add((ch[x] << 32) | ch[y])
    return np.array(sorted(pairs), np.uint64)


@pytest.mark.parametrize("bsize,max_bucket", [(2, 0), (2, 3), (4, 0), (1, 2)])
def test_candidates_match_bruteforce_banding(oracle, bsize, max_bucket):
    # clustered rows so buckets are large
    rng = np.random.default_rng(3)
    base = [rng.choice(60, size=6, replace=False) for _ in range(5)]
    sets = []
    for i in range(80):
        s = set(base[i % 5].tolist())
        if rng.random() < 0.5:
            s.add(int(rng.integers(60, 100)))
        if i % 17 == 0:
            s = set()
        sets.append(s)
    A = _pair_csr(sets, 100)
    siglen = 16
    sig = oracle.signatures(A.rowptr, A.colidx, siglen, 4)
    live = [i for i in range(80) if sets[i]]
    ref = _bruteforce_candidates(sig, live, bsize, max_bucket)
    got = oracle.candidates(A.rowptr, A.colidx, siglen, bsize, 4, max_bucket)
    np.testing.assert_array_equal(got, ref)
    assert np.all((got >> np.uint64(32)) < (got & np.uint64(MASK32)))


def test_candidates_share_a_column(oracle):
    """Bijective hash: equal band key => the rows share a column => J > 0."""
    A = g.random_csr(200, 300, 0.02, 17, empty_frac=0.1)
    E = oracle.candidates(A.rowptr, A.colidx, 32, 2, 4, 0)
    assert E.size > 0
    inter, uni = oracle.jaccard_pairs(A.rowptr, A.colidx, E)
    assert np.all(inter > 0)


def test_bad_band_parameters(oracle):
    A = g.fig1a()
    with pytest.raises(ValueError):
        oracle.candidates(A.rowptr, A.colidx, 10, 3, 4, 0)  # R24


def test_diagonal_has_no_candidates(oracle):
    """Fig 7b: no similar rows -> LSH generates no candidate pairs -> no reordering."""
    D = g.diagonal(64)
    assert oracle.candidates(D.rowptr, D.colidx, 128, 2, 4, 0).size == 0
    perm, E = oracle.reorder_rows(D.rowptr, D.colidx)
    assert E == 0 and np.array_equal(perm, np.arange(64))


def test_jaccard_paper_values(oracle):
    gd = golden("fig1a.json")
    A = g.fig1a()
    for rec in gd["jaccard"]:
        assert oracle.jaccard(A.rowptr, A.colidx, rec["i"], rec["j"]) == (rec["inter"], rec["uni"])


def test_jaccard_matches_python_sets(oracle):
    A = g.random_csr(60, 40, 0.15, 23, empty_frac=0.1)
    rows = [set(A.colidx[A.rowptr[i]:A.rowptr[i + 1]].tolist()) for i in range(60)]
    pairs = oracle.pack_pairs([(i, j) for i in range(60) for j in range(i + 1, 60) if rows[i] or rows[j]])
    inter, uni = oracle.jaccard_pairs(A.rowptr, A.colidx, pairs)
    for e, key in enumerate(pairs.tolist()):
        i, j = key >> 32, key & MASK32
        assert inter[e] == len(rows[i] & rows[j]) and uni[e] == len(rows[i] | rows[j])


def _splitmix64_py(seed: int, n: int):
    """SplitMix64 (Steele, Lea & Flood 2014) written out in Python, independent of the oracle."""
    M64 = (1 << 64) - 1
    s, out = seed & M64, []
    for _ in range(n):
        s = (s + 0x9E3779B97F4A7C15) & M64
        z = s
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
        out.append(z ^ (z >> 31))
    return out


def test_python_splitmix64_matches_published_vector():
    assert _splitmix64_py(1234567, 5) == [
        6457827717110365317, 3203168211198807973, 9817491932198370423,
        4593380528125082431, 16408922859458223821]


@pytest.mark.parametrize("seed,siglen", [(4, 128), (0, 7), (2 ** 63 + 5, 33)])
def test_hash_params_draw_order(oracle, seed, siglen):
    """R13 (O3): for s = 0..siglen-1 in order, a_s = (next() & 0xFFFFFFFF) | 1 and then
    b_s = next() & 0xFFFFFFFF from one SplitMix64 stream seeded with `seed`; i.e. draw 2s
    is a_s's and draw 2s+1 is b_s's.  A swapped (a, b) draw order or a per-array stream
    fails here."""
    st = _splitmix64_py(seed, 2 * siglen)
    a, b = oracle.hash_params(seed, siglen)
    assert a.tolist() == [(st[2 * s] & MASK32) | 1 for s in range(siglen)]
    assert b.tolist() == [st[2 * s + 1] & MASK32 for s in range(siglen)]
