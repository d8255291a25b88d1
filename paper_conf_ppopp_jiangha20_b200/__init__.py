"""Python binding of libsr — the B200 (sm_100a) row-reordered, adaptively tiled SpMM / SDDMM
library of Jiang, Hong & Agrawal (PPoPP'20).  See include/sr.h for the C ABI.

Argument marshalling only: every step of the path runs in libsr.so (CUDA kernels for
sm_100a + host C++).  PyTorch supplies device memory and streams.  There is no CPU
fallback: if the shared library is missing or no CUDA device is present, calls fail loudly.
"""
from __future__ import annotations

import ctypes as C
import dataclasses
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsr.so")

SR_OK, SR_EINVAL, SR_ENOMEM, SR_ECUDA, SR_ESTATE, SR_EUNSUPPORTED = 0, -1, -2, -3, -4, -5
AUTO, FORCE, OFF = 0, 1, 2
SR_OP_SPMM, SR_OP_SDDMM = 0, 1


class SRError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libsr error {code}: {msg}")
        self.code = code


class ReorderParams(C.Structure):
    _fields_ = [("siglen", C.c_int32), ("bsize", C.c_int32), ("threshold_size", C.c_int32),
                ("max_bucket", C.c_int32), ("seed", C.c_uint64), ("panel_rows", C.c_int32),
                ("dense_min", C.c_int32), ("tile_cols", C.c_int32), ("mode", C.c_int32),
                ("skip_dense_num", C.c_int32), ("skip_dense_den", C.c_int32),
                ("skip_sim_num", C.c_int32), ("skip_sim_den", C.c_int32),
                ("world", C.c_int32), ("rank", C.c_int32), ("auto_dense_min", C.c_int32),
                ("reserved0", C.c_int32)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class PlanStats(C.Structure):
    _fields_ = [("nnz", C.c_int64), ("dense0", C.c_int64), ("dense1", C.c_int64),
                ("avgsim_num", C.c_uint64), ("avgsim_den", C.c_uint64),
                ("round1", C.c_int32), ("round2", C.c_int32), ("E1", C.c_int64), ("E2", C.c_int64),
                ("npanels", C.c_int64), ("ndense_cols", C.c_int64), ("ntiles", C.c_int64),
                ("n_perm2", C.c_int64), ("shard_panel_begin", C.c_int64), ("shard_panel_end", C.c_int64),
                ("shard_nrows", C.c_int64), ("shard_nnz", C.c_int64),
                ("t_lsh1_s", C.c_double), ("t_cluster1_s", C.c_double), ("t_tile_s", C.c_double),
                ("t_lsh2_s", C.c_double), ("t_cluster2_s", C.c_double), ("t_total_s", C.c_double),
                ("t_plan_s", C.c_double)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class TrafficModel(C.Structure):
    _fields_ = [(k, C.c_int64) for k in (
        "dense_nnz", "sparse_nnz", "dense_panels", "sparse_items", "dense_rows", "sparse_rows", "zero_rows",
        "rmw_rows", "dense_col_loads", "dense_distinct_cols", "sparse_group_loads", "sparse_distinct_cols")]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


KERNEL_KINDS = {1: "spmm_dense_tiles", 2: "spmm_sparse_rows", 3: "sddmm_dense_tiles", 4: "sddmm_sparse_rows",
                5: "spmm_register_tiles", 6: "sddmm_register_tiles"}

EXPORTED = ("sr_csr_create", "sr_default_params", "sr_reorder", "sr_spmm", "sr_sddmm", "sr_destroy",
            "sr_get_perm", "sr_get_plan_stats", "sr_export_tiles", "sr_shard_rows", "sr_shard_nnz_ids",
            "sr_last_launch_count", "sr_last_error", "sr_host_cluster", "sr_host_partition", "sr_version",
            "sr_get_traffic_model", "sr_set_profiling", "sr_last_kernel_times", "sr_scatter_rows",
            "sr_scatter_values", "sr_plan_save", "sr_plan_load", "sr_trial", "sr_set_values", "sr_get_params")

_lib = None


def lib():
    """Load libsr.so (built by __graft_entry__.build()).  Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(LIB_PATH)
    P, i64, i32, u64 = C.c_void_p, C.c_int64, C.c_int32, C.c_uint64
    sig = {
        "sr_csr_create": (C.c_int, [i64, i64, i64, P, P, P, C.c_int, C.POINTER(P)]),
        "sr_default_params": (None, [C.POINTER(ReorderParams)]),
        "sr_reorder": (C.c_int, [P, C.POINTER(ReorderParams), P]),
        "sr_spmm": (C.c_int, [P, P, i64, i64, P, i64, P]),
        "sr_sddmm": (C.c_int, [P, P, i64, P, i64, i64, P, P]),
        "sr_destroy": (C.c_int, [P]),
        "sr_get_perm": (C.c_int, [P, C.c_int, P, i64, C.POINTER(i64)]),
        "sr_get_plan_stats": (C.c_int, [P, C.POINTER(PlanStats)]),
        "sr_get_params": (C.c_int, [P, C.POINTER(ReorderParams)]),
        "sr_export_tiles": (C.c_int, [P] + [P] * 8),
        "sr_shard_rows": (C.c_int, [P, P, i64, C.POINTER(i64)]),
        "sr_shard_nnz_ids": (C.c_int, [P, P, i64, C.POINTER(i64)]),
        "sr_last_launch_count": (C.c_int, [P, C.POINTER(i32)]),
        "sr_last_error": (C.c_char_p, []),
        "sr_host_cluster": (C.c_int, [i64, P, P, i64, P, P, P, i32, P]),
        "sr_host_partition": (C.c_int, [i64, P, i32, P]),
        "sr_version": (C.c_char_p, []),
        "sr_get_traffic_model": (C.c_int, [P, C.POINTER(TrafficModel)]),
        "sr_set_profiling": (C.c_int, [P, C.c_int]),
        "sr_last_kernel_times": (C.c_int, [P, P, P, i32, C.POINTER(i32)]),
        "sr_scatter_rows": (C.c_int, [P, i64, P, i64, i64, P, i64, P]),
        "sr_scatter_values": (C.c_int, [P, P, i64, P, P]),
        "sr_plan_save": (C.c_int, [P, P, i64, C.POINTER(i64)]),
        "sr_set_values": (C.c_int, [P, P, P]),
        "sr_plan_load": (C.c_int, [P, P, i64, i32, i32, P]),
        "sr_trial": (C.c_int, [P, i32, i32, P, i64, P, i64, i64, P, i64, i32, P, C.POINTER(i32), P]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _check(rc: int):
    if rc != SR_OK:
        raise SRError(rc, lib().sr_last_error().decode())


def _np(a, dtype):
    a = np.ascontiguousarray(a, dtype=dtype)
    return a, a.ctypes.data_as(C.c_void_p)


def default_params(**overrides) -> ReorderParams:
    p = ReorderParams()
    lib().sr_default_params(C.byref(p))
    for k, v in overrides.items():
        if k in ("skip_dense", "skip_sim"):
            setattr(p, k + "_num", v[0])
            setattr(p, k + "_den", v[1])
        else:
            setattr(p, k, v)
    return p


def _ptr(t) -> C.c_void_p:
    return C.c_void_p(int(t.data_ptr()))


def _stream(stream, device: int | None = None):
    """cudaStream_t of `stream`; None = torch's current stream of `device` (the matrix's GPU)."""
    if stream is None:
        import torch
        stream = torch.cuda.current_stream(device)
    return C.c_void_p(int(stream.cuda_stream))


def _check_dense(name: str, T, rows: int, device: int, K: int | None = None, contiguous: bool = False):
    """The C ABI receives only pointers and leading dimensions, so the binding checks what the
    kernels will read or write: fp32, CUDA, this matrix's device, 2-D with unit column stride
    (or contiguous 1-D), and the row count the operation indexes."""
    import torch
    if T.dtype != torch.float32 or not T.is_cuda:
        raise ValueError(f"{name} must be an fp32 CUDA tensor")
    if T.device.index != device:
        raise ValueError(f"{name} is on cuda:{T.device.index}, the matrix on cuda:{device}")
    if contiguous:
        if T.dim() != 1 or not T.is_contiguous() or T.numel() != rows:
            raise ValueError(f"{name} must be a contiguous 1-D tensor of {rows} values")
        return
    if T.dim() != 2 or T.stride(1) != 1 or T.stride(0) < T.shape[1]:
        raise ValueError(f"{name} must be 2-D with unit column stride and row stride >= its width")
    if T.shape[0] != rows:
        raise ValueError(f"{name} has {T.shape[0]} rows, expected {rows}")
    if K is not None and T.shape[1] != K:
        raise ValueError(f"{name} has {T.shape[1]} columns, expected K = {K}")


class SparseMatrix:
    """A CSR matrix resident on one GPU plus its execution plan (sr_csr handle)."""

    def __init__(self, nrows: int, ncols: int, rowptr, colidx, vals, device: int = 0):
        rp, prp = _np(rowptr, np.int64)
        ci, pci = _np(colidx, np.int32)
        vv, pvv = _np(vals, np.float32)
        h = C.c_void_p()
        _check(lib().sr_csr_create(nrows, ncols, int(rp[-1]) if rp.size else 0, prp, pci, pvv, device,
                                   C.byref(h)))
        self._h = h
        self.nrows, self.ncols, self.nnz, self.device = nrows, ncols, int(rp[-1]), device
        self.params: ReorderParams | None = None

    @classmethod
    def from_csr(cls, A, device: int = 0) -> "SparseMatrix":
        return cls(A.nrows, A.ncols, A.rowptr, A.colidx, A.vals, device)

    # -- lifecycle
    def close(self):
        if getattr(self, "_h", None):
            lib().sr_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- plan
    def reorder(self, params: ReorderParams | None = None, stream=None, **overrides) -> dict:
        p = params if params is not None else default_params(**overrides)
        s = C.c_void_p(int(stream.cuda_stream)) if stream is not None else C.c_void_p()
        _check(lib().sr_reorder(self._h, C.byref(p), s))
        self.params = p
        return self.stats()

    def save_plan(self) -> bytes:
        """Canonical byte image of the plan (sr_plan_save: offline reordering)."""
        n = C.c_int64()
        _check(lib().sr_plan_save(self._h, None, 0, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _check(lib().sr_plan_save(self._h, C.cast(buf, C.c_void_p), n.value, C.byref(n)))
        return buf.raw[:n.value]

    def load_plan(self, image: bytes, world: int = 1, rank: int = 0, stream=None) -> dict:
        """Install a saved plan of this matrix (sr_plan_load; no LSH / clustering)."""
        s = C.c_void_p(int(stream.cuda_stream)) if stream is not None else C.c_void_p()
        buf = C.create_string_buffer(bytes(image), len(image))
        _check(lib().sr_plan_load(self._h, C.cast(buf, C.c_void_p), len(image), world, rank, s))
        self.params = self.get_params()
        return self.stats()

    def get_params(self) -> ReorderParams:
        """The parameters of this handle's plan (sr_get_params)."""
        p = ReorderParams()
        _check(lib().sr_get_params(self._h, C.byref(p)))
        return p

    def stats(self) -> dict:
        st = PlanStats()
        _check(lib().sr_get_plan_stats(self._h, C.byref(st)))
        return st.as_dict()

    def perm(self, which: int) -> np.ndarray:
        n = C.c_int64()
        _check(lib().sr_get_perm(self._h, which, None, 0, C.byref(n)))
        out = np.empty(n.value, np.int32)
        _check(lib().sr_get_perm(self._h, which, out.ctypes.data_as(C.c_void_p), out.size, C.byref(n)))
        return out

    def tiles(self) -> dict:
        st = self.stats()
        M, nd = self.nrows, st["dense1"]
        t = dict(dense_ptr=np.empty(st["npanels"] + 1, np.int64), dense_cols=np.empty(st["ndense_cols"], np.int32),
                 drow_ptr=np.empty(M + 1, np.int64), d_slot=np.empty(nd, np.int32), d_pos=np.empty(nd, np.int64),
                 rrow_ptr=np.empty(M + 1, np.int64), r_col=np.empty(self.nnz - nd, np.int32),
                 r_pos=np.empty(self.nnz - nd, np.int64))
        _check(lib().sr_export_tiles(self._h, *[t[k].ctypes.data_as(C.c_void_p) for k in
                                                ("dense_ptr", "dense_cols", "drow_ptr", "d_slot", "d_pos",
                                                 "rrow_ptr", "r_col", "r_pos")]))
        return t

    def shard_rows(self) -> np.ndarray:
        n = C.c_int64()
        _check(lib().sr_shard_rows(self._h, None, 0, C.byref(n)))
        out = np.empty(n.value, np.int32)
        _check(lib().sr_shard_rows(self._h, out.ctypes.data_as(C.c_void_p), out.size, C.byref(n)))
        return out

    def shard_nnz_ids(self) -> np.ndarray:
        n = C.c_int64()
        _check(lib().sr_shard_nnz_ids(self._h, None, 0, C.byref(n)))
        out = np.empty(n.value, np.int64)
        _check(lib().sr_shard_nnz_ids(self._h, out.ctypes.data_as(C.c_void_p), out.size, C.byref(n)))
        return out

    def traffic_model(self) -> dict:
        t = TrafficModel()
        _check(lib().sr_get_traffic_model(self._h, C.byref(t)))
        return t.as_dict()

    def set_profiling(self, on: bool = True):
        _check(lib().sr_set_profiling(self._h, 1 if on else 0))

    def last_kernel_times(self) -> list:
        """[(kernel name, device ms), ...] of the last spmm / sddmm call (waits for it)."""
        kinds = (C.c_int32 * 4)()
        ms = (C.c_float * 4)()
        n = C.c_int32()
        _check(lib().sr_last_kernel_times(self._h, C.cast(kinds, C.c_void_p), C.cast(ms, C.c_void_p), 4,
                                          C.byref(n)))
        return [(KERNEL_KINDS[kinds[i]], float(ms[i])) for i in range(n.value)]

    def last_launch_count(self) -> int:
        n = C.c_int32()
        _check(lib().sr_last_launch_count(self._h, C.byref(n)))
        return n.value

    @property
    def out_rows(self) -> int:
        if self.params is not None and self.params.world > 1:
            return int(self.stats()["shard_nrows"])
        return self.nrows

    @property
    def out_nnz(self) -> int:
        if self.params is not None and self.params.world > 1:
            return int(self.stats()["shard_nnz"])
        return self.nnz

    # -- compute (torch tensors on this matrix's device; asynchronous on `stream`)
    def spmm(self, B, C_out=None, stream=None):
        """C := A·B (Alg 1).  B: [ncols, K] fp32 CUDA tensor on this matrix's device (row stride
        >= K); C_out: [out_rows, K] (row stride >= K) or None."""
        import torch
        _check_dense("B", B, self.ncols, self.device)
        K = B.shape[1]
        if C_out is None:
            C_out = torch.empty((self.out_rows, K), dtype=torch.float32, device=B.device)
        _check_dense("C_out", C_out, self.out_rows, self.device, K)
        _check(lib().sr_spmm(self._h, _ptr(B), K, B.stride(0), _ptr(C_out), C_out.stride(0),
                             _stream(stream, self.device)))
        return C_out

    def set_values(self, vals, stream=None):
        """Replace the nonzero values the kernels use (sr_set_values): fp32 CUDA tensor of
        out_nnz values in the order sddmm() writes."""
        _check_dense("vals", vals, self.out_nnz, self.device, contiguous=True)
        _check(lib().sr_set_values(self._h, _ptr(vals), _stream(stream, self.device)))

    def sddmm(self, X, Y, out=None, stream=None):
        """out[p] := vals[p]·<X[row(p)], Y[col(p)]> (Alg 2) in the caller's nnz order.
        X: [nrows, K], Y: [ncols, K] fp32 CUDA tensors; out: contiguous [out_nnz] or None."""
        import torch
        _check_dense("X", X, self.nrows, self.device)
        K = X.shape[1]
        _check_dense("Y", Y, self.ncols, self.device, K)
        if out is None:
            out = torch.empty(self.out_nnz, dtype=torch.float32, device=X.device)
        _check_dense("out", out, self.out_nnz, self.device, contiguous=True)
        _check(lib().sr_sddmm(self._h, _ptr(X), X.stride(0), _ptr(Y), Y.stride(0), K, _ptr(out),
                              _stream(stream, self.device)))
        return out


def trial(cands, op: str, U, V=None, out=None, reps: int = 5, stream=None):
    """Trial-and-error plan selection (sr_trial): time `op` ("spmm": U = B, out = C;
    "sddmm": U = X, V = Y) on every candidate SparseMatrix (plans of one matrix, e.g. a
    reordered one and one in the original order) and return (index of the fastest, [median ms])."""
    import torch
    n = len(cands)
    hs = (C.c_void_p * n)(*[c._h for c in cands])
    K = U.shape[1]
    if op == "spmm":
        code, pv, ldv = SR_OP_SPMM, None, 0
        if out is None:
            out = torch.empty((cands[0].out_rows, K), dtype=torch.float32, device=U.device)
        ldo = out.stride(0)
    elif op == "sddmm":
        code, pv, ldv = SR_OP_SDDMM, _ptr(V), V.stride(0)
        if out is None:
            out = torch.empty(cands[0].out_nnz, dtype=torch.float32, device=U.device)
        ldo = 1
    else:
        raise ValueError("op must be 'spmm' or 'sddmm'")
    best = C.c_int32()
    ms = (C.c_float * n)()
    dev = cands[0].device
    _check_dense("U", U, cands[0].ncols if op == "spmm" else cands[0].nrows, dev)
    if op == "sddmm":
        _check_dense("V", V, cands[0].ncols, dev, K)
    _check(lib().sr_trial(C.cast(hs, C.c_void_p), n, code, _ptr(U), U.stride(0), pv, ldv, K, _ptr(out), ldo, reps,
                          _stream(stream, dev), C.byref(best), C.cast(ms, C.c_void_p)))
    return best.value, [float(x) for x in ms]


# ---------------------------------------------------------------- host-only entry points
def host_cluster(rowptr, colidx, pairs, threshold_size: int, inter=None, uni=None) -> np.ndarray:
    rp, prp = _np(rowptr, np.int64)
    ci, pci = _np(colidx, np.int32)
    pr, ppr = _np(pairs, np.uint64)
    M = rp.size - 1
    perm = np.empty(M, np.int32)
    if inter is not None:
        it, pit = _np(inter, np.uint32)
        un, pun = _np(uni, np.uint32)
    else:
        pit = pun = None
    _check(lib().sr_host_cluster(M, prp, pci, pr.size, ppr, pit, pun, threshold_size,
                                 perm.ctypes.data_as(C.c_void_p)))
    return perm


def host_partition(weights, G: int) -> np.ndarray:
    w, pw = _np(weights, np.int64)
    cuts = np.empty(G + 1, np.int64)
    _check(lib().sr_host_partition(w.size, pw, G, cuts.ctypes.data_as(C.c_void_p)))
    return cuts


def scatter_rows(src, rows, dst, stream=None):
    """dst[rows[r]] = src[r] on the device (rows: int32 CUDA tensor; -1 entries skipped)."""
    _check(lib().sr_scatter_rows(_ptr(src), src.stride(0), _ptr(rows), rows.numel(), src.shape[1], _ptr(dst),
                                 dst.stride(0), _stream(stream, dst.device.index)))
    return dst


def scatter_values(src, ids, dst, stream=None):
    """dst[ids[i]] = src[i] on the device (ids: int64 CUDA tensor; -1 entries skipped)."""
    _check(lib().sr_scatter_values(_ptr(src), _ptr(ids), ids.numel(), _ptr(dst), _stream(stream, dst.device.index)))
    return dst


def version() -> str:
    return lib().sr_version().decode()
