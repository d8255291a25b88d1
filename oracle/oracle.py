"""ctypes wrapper of the CPU oracle (oracle/oracle.cpp).  TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference)
may import this module.  The product package never does.  Argument marshalling
only: every computation happens in oracle.cpp, each function citing PAPER.md.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")

MODE_AUTO, MODE_FORCE, MODE_OFF = 0, 1, 2


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared",
                               _SRC, "-o", _LIB + ".tmp"])
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        i64, i32, u64, u32 = C.c_int64, C.c_int32, C.c_uint64, C.c_uint32
        sig = {
            "or_canonicalize": (C.c_int, [i64, i64, i64, P, P, P, P, P, P]),
            "or_spmm": (None, [i64, i64, P, P, P, P, i64, P]),
            "or_spmm_rows": (None, [i64, P, i64, P, P, P, P, i64, P, P]),
            "or_sddmm": (None, [i64, i64, P, P, P, P, i64, P, i64, P, P]),
            "or_hash_params": (None, [u64, i32, P, P]),
            "or_hash": (u32, [u32, u32, u32]),
            "or_splitmix64": (u64, [P]),
            "or_fmix32": (u32, [u32]),
            "or_signatures": (None, [i64, P, P, i32, u64, P]),
            "or_candidates": (i64, [i64, P, P, i32, i32, u64, i32, P]),
            "or_free": (None, [P]),
            "or_jaccard": (None, [P, P, i64, i64, P, P]),
            "or_jaccard_pairs": (None, [P, P, i64, P, P, P]),
            "or_cluster": (i64, [i64, P, P, i64, P, P, P, i32, P]),
            "or_reorder_rows": (i64, [i64, P, P, i32, i32, u64, i32, i32, P]),
            "or_tile": (i64, [i64, i64, P, P, P, i32, i32, P, P, P, P, P, P, P, P]),
            "or_avgsim": (u64, [i64, P, P, P]),
            "or_plan": (C.c_int, [i64, i64, P, P, i32, i32, u64, i32, i32, i32, i32, i32, i32, i32,
                                  i32, i32, i32, P, P, P, P, P, P, P, P, P, P, P, P]),
            "or_partition": (None, [i64, P, i32, P]),
            "or_access_count": (i64, [i64, P, P, P, i64, P, i32]),
            "or_num_threads": (C.c_int, []),
            "or_set_num_threads": (None, [C.c_int]),
        }
        for name, (res, args) in sig.items():
            f = getattr(_lib, name)
            f.restype = res
            f.argtypes = args
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def num_threads() -> int:
    return lib().or_num_threads()


def set_num_threads(n: int) -> None:
    """OpenMP threads of the oracle's parallel loops (timing legs only; results unchanged)."""
    lib().or_set_num_threads(int(n))


# ---------------------------------------------------------------- O0 .. O2
def canonicalize(A):
    col = np.empty(A.nnz, np.int32)
    val = np.empty(A.nnz, np.float32)
    pos = np.empty(A.nnz, np.int64)
    rp, ci, v = _c(A.rowptr, np.int64), _c(A.colidx, np.int32), _c(A.vals, np.float32)
    rc = lib().or_canonicalize(A.nrows, A.ncols, A.nnz, _p(rp), _p(ci), _p(v), _p(col), _p(val), _p(pos))
    if rc != 0:
        raise ValueError("oracle: malformed CSR or duplicate (row, col)")
    return col, val, pos


def spmm(A, B: np.ndarray) -> np.ndarray:
    B = _c(B, np.float32)
    K = B.shape[1]
    out = np.empty((A.nrows, K), np.float64)
    rp, ci, v = _c(A.rowptr, np.int64), _c(A.colidx, np.int32), _c(A.vals, np.float32)
    lib().or_spmm(A.nrows, K, _p(rp), _p(ci), _p(v), _p(B), K, _p(out))
    return out


def spmm_rows(A, B: np.ndarray, rows: np.ndarray):
    B = _c(B, np.float32)
    K = B.shape[1]
    rows = _c(rows, np.int64)
    out = np.empty((rows.size, K), np.float64)
    absb = np.empty((rows.size, K), np.float64)
    rp, ci, v = _c(A.rowptr, np.int64), _c(A.colidx, np.int32), _c(A.vals, np.float32)
    lib().or_spmm_rows(rows.size, _p(rows), K, _p(rp), _p(ci), _p(v), _p(B), K, _p(out), _p(absb))
    return out, absb


def sddmm(A, X: np.ndarray, Y: np.ndarray):
    X, Y = _c(X, np.float32), _c(Y, np.float32)
    K = X.shape[1]
    out = np.empty(A.nnz, np.float64)
    absb = np.empty(A.nnz, np.float64)
    rp, ci, v = _c(A.rowptr, np.int64), _c(A.colidx, np.int32), _c(A.vals, np.float32)
    lib().or_sddmm(A.nrows, K, _p(rp), _p(ci), _p(v), _p(X), K, _p(Y), K, _p(out), _p(absb))
    return out, absb


# ---------------------------------------------------------------- O3 .. O9
def hash_params(seed: int, siglen: int):
    a = np.empty(siglen, np.uint32)
    b = np.empty(siglen, np.uint32)
    lib().or_hash_params(seed, siglen, _p(a), _p(b))
    return a, b


def hash_(a: int, b: int, c: int) -> int:
    return lib().or_hash(a, b, c)


def splitmix64_stream(seed: int, n: int):
    st = np.array([seed], np.uint64)
    return [lib().or_splitmix64(_p(st)) for _ in range(n)]


def fmix32(h: int) -> int:
    return lib().or_fmix32(h)


def signatures(rowptr, colidx, siglen: int, seed: int) -> np.ndarray:
    rowptr, colidx = _c(rowptr, np.int64), _c(colidx, np.int32)
    M = rowptr.size - 1
    sig = np.full((M, siglen), 0xFFFFFFFF, np.uint32)
    lib().or_signatures(M, _p(rowptr), _p(colidx), siglen, seed, _p(sig))
    return sig


def candidates(rowptr, colidx, siglen: int, bsize: int, seed: int, max_bucket: int) -> np.ndarray:
    rowptr, colidx = _c(rowptr, np.int64), _c(colidx, np.int32)
    M = rowptr.size - 1
    ptr = C.c_void_p()
    n = lib().or_candidates(M, _p(rowptr), _p(colidx), siglen, bsize, seed, max_bucket, C.byref(ptr))
    if n < 0:
        raise ValueError("oracle: siglen % bsize != 0")
    out = np.ctypeslib.as_array(C.cast(ptr, C.POINTER(C.c_uint64)), shape=(max(n, 1),))[:n].copy()
    lib().or_free(ptr)
    return out


def jaccard(rowptr, colidx, i: int, j: int):
    rowptr, colidx = _c(rowptr, np.int64), _c(colidx, np.int32)
    n, u = C.c_uint64(), C.c_uint64()
    lib().or_jaccard(_p(rowptr), _p(colidx), i, j, C.byref(n), C.byref(u))
    return n.value, u.value


def jaccard_pairs(rowptr, colidx, pairs: np.ndarray):
    rowptr, colidx, pairs = _c(rowptr, np.int64), _c(colidx, np.int32), _c(pairs, np.uint64)
    inter = np.empty(pairs.size, np.uint32)
    uni = np.empty(pairs.size, np.uint32)
    lib().or_jaccard_pairs(_p(rowptr), _p(colidx), pairs.size, _p(pairs), _p(inter), _p(uni))
    return inter, uni


def pack_pairs(pairs) -> np.ndarray:
    """[(i, j), ...] -> sorted unique packed (min<<32 | max)."""
    out = sorted({(min(i, j) << 32) | max(i, j) for i, j in pairs})
    return np.array(out, dtype=np.uint64)


def cluster(rowptr, colidx, pairs: np.ndarray, threshold_size: int, inter=None, uni=None):
    rowptr, colidx, pairs = _c(rowptr, np.int64), _c(colidx, np.int32), _c(pairs, np.uint64)
    M = rowptr.size - 1
    perm = np.empty(M, np.int32)
    if inter is not None:
        inter, uni = _c(inter, np.uint32), _c(uni, np.uint32)
        lib().or_cluster(M, _p(rowptr), _p(colidx), pairs.size, _p(pairs), _p(inter), _p(uni),
                         threshold_size, _p(perm))
    else:
        lib().or_cluster(M, _p(rowptr), _p(colidx), pairs.size, _p(pairs), None, None,
                         threshold_size, _p(perm))
    return perm


def reorder_rows(rowptr, colidx, siglen=128, bsize=2, seed=4, max_bucket=0, threshold_size=256):
    rowptr, colidx = _c(rowptr, np.int64), _c(colidx, np.int32)
    M = rowptr.size - 1
    perm = np.empty(M, np.int32)
    E = lib().or_reorder_rows(M, _p(rowptr), _p(colidx), siglen, bsize, seed, max_bucket,
                              threshold_size, _p(perm))
    if E < 0:
        raise ValueError("oracle: bad LSH parameters")
    return perm, E


# ---------------------------------------------------------------- O10 .. O14
def tile(A, perm, panel_rows: int, dense_min: int) -> dict:
    M, N, nnz = A.nrows, A.ncols, A.nnz
    rp, ci = _c(A.rowptr, np.int64), _c(A.colidx, np.int32)
    perm = _c(perm, np.int32)
    npan = (M + panel_rows - 1) // panel_rows
    t = dict(dense_ptr=np.zeros(npan + 1, np.int64), dense_cols=np.zeros(max(nnz, 1), np.int32),
             drow_ptr=np.zeros(M + 1, np.int64), d_slot=np.zeros(max(nnz, 1), np.int32),
             d_pos=np.zeros(max(nnz, 1), np.int64), rrow_ptr=np.zeros(M + 1, np.int64),
             r_col=np.zeros(max(nnz, 1), np.int32), r_pos=np.zeros(max(nnz, 1), np.int64))
    nd = lib().or_tile(M, N, _p(rp), _p(ci), _p(perm), panel_rows, dense_min,
                       *[_p(t[k]) for k in ("dense_ptr", "dense_cols", "drow_ptr", "d_slot", "d_pos",
                                            "rrow_ptr", "r_col", "r_pos")])
    return _trim(t, nd, npan)


def _trim(t: dict, nd: int, npan: int) -> dict:
    ndc = int(t["dense_ptr"][npan])
    nr = int(t["rrow_ptr"][-1])
    t["dense_cols"] = t["dense_cols"][:ndc]
    t["d_slot"] = t["d_slot"][:nd]
    t["d_pos"] = t["d_pos"][:nd]
    t["r_col"] = t["r_col"][:nr]
    t["r_pos"] = t["r_pos"][:nr]
    t["n_dense"] = nd
    t["npanels"] = npan
    return t


def avgsim(rowptr, colidx):
    rowptr, colidx = _c(rowptr, np.int64), _c(colidx, np.int32)
    den = C.c_uint64()
    num = lib().or_avgsim(rowptr.size - 1, _p(rowptr), _p(colidx), C.byref(den))
    return num, den.value


STAT_KEYS = ("dense0", "dense1", "nnz", "avgsim_num", "avgsim_den", "round1", "round2", "E1", "E2",
             "npanels", "ndense_cols")


def plan(A, siglen=128, bsize=2, seed=4, max_bucket=0, threshold_size=256, panel_rows=64,
         dense_min=2, mode=MODE_AUTO, skip_dense=(1, 10), skip_sim=(1, 10), auto_dense_min=0) -> dict:
    M, N, nnz = A.nrows, A.ncols, A.nnz
    rp, ci = _c(A.rowptr, np.int64), _c(A.colidx, np.int32)
    npan = (M + panel_rows - 1) // panel_rows
    perm1 = np.zeros(M, np.int32)
    perm2 = np.zeros(max(M, 1), np.int32)
    n2 = C.c_int64()
    stats = np.zeros(16, np.int64)
    t = dict(dense_ptr=np.zeros(npan + 1, np.int64), dense_cols=np.zeros(max(nnz, 1), np.int32),
             drow_ptr=np.zeros(M + 1, np.int64), d_slot=np.zeros(max(nnz, 1), np.int32),
             d_pos=np.zeros(max(nnz, 1), np.int64), rrow_ptr=np.zeros(M + 1, np.int64),
             r_col=np.zeros(max(nnz, 1), np.int32), r_pos=np.zeros(max(nnz, 1), np.int64))
    rc = lib().or_plan(M, N, _p(rp), _p(ci), siglen, bsize, seed, max_bucket, threshold_size,
                       panel_rows, dense_min, auto_dense_min, mode, skip_dense[0], skip_dense[1], skip_sim[0],
                       skip_sim[1], _p(perm1), _p(perm2), C.byref(n2),
                       *[_p(t[k]) for k in ("dense_ptr", "dense_cols", "drow_ptr", "d_slot", "d_pos",
                                            "rrow_ptr", "r_col", "r_pos")], _p(stats))
    if rc != 0:
        raise ValueError("oracle: bad plan parameters")
    t = _trim(t, int(stats[1]), npan)
    t["perm1"] = perm1
    t["perm2"] = perm2[:n2.value].copy()
    t["stats"] = {k: int(stats[i]) for i, k in enumerate(STAT_KEYS)}
    return t


def partition(weights, G: int) -> np.ndarray:
    w = _c(weights, np.int64)
    cuts = np.zeros(G + 1, np.int64)
    lib().or_partition(w.size, _p(w), G, _p(cuts))
    return cuts


def access_count(t: dict, order, W: int) -> int:
    order = _c(order, np.int32)
    return lib().or_access_count(t["npanels"], _p(_c(t["dense_ptr"], np.int64)),
                                 _p(_c(t["rrow_ptr"], np.int64)), _p(_c(t["r_col"], np.int32)),
                                 order.size, _p(order), W)
