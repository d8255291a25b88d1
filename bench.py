#!/usr/bin/env python3
"""bench.py — SpMM / SDDMM throughput of the row-reordered, adaptively tiled path on B200.

Metric (BASELINE.json): SpMM/SDDMM GFLOP/s (2·nnz·K per op) and HBM GB/s as a fraction of
roofline.  Workload at N=1: C2, the R-MAT scale-20 matrix (configs[1]), K=128 (headline) and
K=32 (`extra_K`).

One step = one pass of the execution hot path over the planned matrix: C := A·B (SpMM)
and out := A ⊙ (X·Yᵀ) on A's pattern (SDDMM), both through the C ABI (libsr.so).  The
reorder preprocessing (LSH on the GPU + Alg 3 on the host + ASpT tiling) runs once
before the timed region and is reported separately (`preprocess`), as the paper does
(P:277).  Inputs are resident in HBM; a 512 MB write flushes L2 between steps
(outside the device-timed intervals).

Multi-GPU (`--gpus N`): one process per GPU.  Without torchrun's environment the script
re-launches itself under `torch.distributed.run` with N ranks; it fails if fewer than N GPUs
are visible.  Rank 0 reorders the whole matrix once and broadcasts the plan image; every
rank loads its nnz-balanced panel shard (sr_plan_load(world, rank)) and computes its rows
(strong scaling, no collective inside the step; `--gather` times the optional all-gather).
`--simulate-world N` runs the N shard plans one after another on one GPU and reports
the per-shard step times (load balance; labelled as a simulation, never as n_gpus).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config rmat] [--K 128] [--ops spmm,sddmm] [--simulate-world N]
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import socket
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import generators as gen  # noqa: E402

METRIC = "SpMM+SDDMM GFLOP/s (2*nnz*K per op)"  # both arms print this string (BASELINE.json metric)
FP32_PEAK_GFLOPS = 148 * 128 * 2 * 1.965  # dense FP32 FMA peak (74.4 TFLOP/s), DESIGN.md §5
PAPER_CONTEXT = ("P100 (paper, P:334, P:350): ASpT-RR up to 2.91x SpMM vs best of ASpT-NR/cuSPARSE and "
                 "up to 3.19x SDDMM vs ASpT-NR; geomean 1.19x / 1.49x (K=1024)")


# ASpT panel height and dense-column threshold per workload (R17).  On C2, C3 and C5
# the staged tiles lose to the L2 gather path at every threshold, so dense_min 64 keeps only
# columns the whole 64-row panel shares (equal to no tiles); on the GNN matrix C4, 32-row panels
# with columns shared by >= 4 rows beat the untiled plan by 7-8 % (profiles/r02/NOTES.md, r02aa).
PLAN_DEFAULTS = {"gnn": dict(panel_rows=32, dense_min=4)}
PLAN_DEFAULT = dict(panel_rows=64, dense_min=64)


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="rmat", choices=list(gen.CONFIGS))
    ap.add_argument("--K", type=int, default=128)
    ap.add_argument("--extra-K", default=None,
                    help="comma list of further K timed on the same plan (default: 32 for rmat at K=128; 'none')")
    ap.add_argument("--ops", default="spmm,sddmm")
    ap.add_argument("--mode", default="auto", choices=["auto", "force", "off"])
    # plan parameters per workload (None = the config's default, PLAN_DEFAULTS below)
    ap.add_argument("--panel-rows", type=int, default=None)
    ap.add_argument("--tile-cols", type=int, default=64)
    ap.add_argument("--max-bucket", type=int, default=32)
    # ASpT dense-column threshold (R17).  The paper's example is 2 (a P100 with 64 KB of
    # shared memory per SM); on B200 (126 MB L2, row-group task kernels gathering from L2 at ~15 TB/s)
    # staging pays only for columns shared by (nearly) the whole 64-row panel: sweeps in
    # profiles/r01/NOTES.md (session 3: 64 best with tiles present, equal to no tiles).
    ap.add_argument("--dense-min", type=int, default=None)
    # dense criterion of the AUTO round-1 decision (R28): a column shared by 1/8 of the panel
    ap.add_argument("--auto-dense-min", type=int, default=8)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target CPU work of cpu_baseline")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-oracle-reorder", action="store_true", help="skip the oracle reorder timing leg")
    ap.add_argument("--gather", action="store_true", help="also time the optional NCCL all-gather of C")
    ap.add_argument("--simulate-world", type=int, default=0,
                    help="also time the N shard plans one after another on this GPU (load balance)")
    ap.add_argument("--min-warm-s", type=float, default=1.0, help="keep warming up until this long (clocks)")
    ap.add_argument("--plan-cache", default=None,
                    help="experiments only: load the plan image from this file if present, else save it there "
                         "(preprocess then reports the load, not the reorder)")
    args = ap.parse_args(argv)
    for k, v in PLAN_DEFAULTS.get(args.config, PLAN_DEFAULT).items():
        if getattr(args, k) is None:
            setattr(args, k, v)
    return args


def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def host_cpu() -> dict:
    """Host CPU description for every oracle timing: model, logical CPUs,
    physical cores (unique (package, core id) pairs)."""
    model, pairs, logical = None, set(), 0
    phys = core = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                k, _, v = line.partition(":")
                k, v = k.strip(), v.strip()
                if k == "processor":
                    logical += 1
                elif k == "model name" and model is None:
                    model = v
                elif k == "physical id":
                    phys = v
                elif k == "core id":
                    core = v
                elif not k and phys is not None:
                    pairs.add((phys, core))
                    phys = core = None
        if phys is not None:
            pairs.add((phys, core))
    except OSError:
        pass
    return {"model": model, "logical_cpus": logical or os.cpu_count(),
            "physical_cores": len(pairs) or None, "nproc": os.cpu_count()}


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.proc = None
        self.path = f"/tmp/bench_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-lms", "100", "-i", str(self.gpu)], stdout=open(self.path, "w"),
                                         stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        self.proc.wait()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                smax.append(float(parts[2]))
            except ValueError:
                continue
            for n, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        os.unlink(self.path)
        load = [s for s in sm if s > 0.5 * max(sm)] if sm else []
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- oracle legs
def row_prefix(A, R):
    return gen.CSR(R, A.ncols, A.rowptr[:R + 1].copy(), A.colidx[:A.rowptr[R]], A.vals[:A.rowptr[R]])


def oracle_sample(A, K, target_s, ops):
    """Time the CPU oracle (oracle/, fp64, OpenMP over the host cores) on a bounded row
    sample of the workload: rows [0, R) with R grown until ~target_s of work."""
    from oracle import oracle as O
    O.build()
    B = gen.dense(A.ncols, K, stream=0)
    Y = gen.dense(A.ncols, K, stream=2) if "sddmm" in ops else None
    R = max(1, A.nrows // 256)
    while True:
        sub = row_prefix(A, R)
        X = gen.dense(R, K, stream=1) if "sddmm" in ops else None
        t0 = time.perf_counter()
        if "spmm" in ops:
            O.spmm(sub, B)
        if "sddmm" in ops:
            O.sddmm(sub, X, Y)
        dt = time.perf_counter() - t0
        if dt * 4 >= target_s or R >= A.nrows:
            break
        R = min(A.nrows, int(R * max(2.0, min(8.0, target_s / 2 / max(dt, 1e-3)))))
    nnz = int(sub.rowptr[-1])
    flops = 2.0 * nnz * K * len(ops)
    return dict(sub=sub, B=B, X=X, Y=Y, rows=R, nnz=nnz, flops=flops, seconds=dt, O=O)


def cpu_baseline(A, K, args, ops, name):
    s = oracle_sample(A, K, args.cpu_seconds, ops)
    # measured leg: ~target seconds of repeated passes over the sample
    reps = max(1, int(round(args.cpu_seconds / max(s["seconds"], 1e-3))))
    O = s["O"]
    t0 = time.perf_counter()
    for _ in range(reps):
        if "spmm" in ops:
            O.spmm(s["sub"], s["B"])
        if "sddmm" in ops:
            O.sddmm(s["sub"], s["X"], s["Y"])
    dt = time.perf_counter() - t0
    cores = O.num_threads()
    # single-thread leg (O1/O2 timed single-thread and on all cores), on a
    # 1/cores share of the sample's rows so it stays within the same time budget
    R1 = max(1, s["rows"] // max(cores, 1))
    sub1 = row_prefix(A, R1)
    X1 = s["X"][:R1] if s["X"] is not None else None
    O.set_num_threads(1)
    try:
        t1 = time.perf_counter()
        if "spmm" in ops:
            O.spmm(sub1, s["B"])
        if "sddmm" in ops:
            O.sddmm(sub1, X1, s["Y"])
        dt1 = time.perf_counter() - t1
    finally:
        O.set_num_threads(cores)
    st_value = 2.0 * int(sub1.rowptr[-1]) * K * len(ops) / max(dt1, 1e-9) / 1e9
    return {"value": s["flops"] * reps / dt / 1e9, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
            "host": host_cpu(),
            "sample": f"{name} rows [0,{s['rows']}) = {s['nnz']} nnz of {A.nnz}, K={K}, {'+'.join(ops)} in fp64, "
                      f"{reps} pass(es), {dt:.1f} s",
            "single_thread": {"value": st_value, "unit": "GFLOP/s", "cores": 1,
                              "sample": f"rows [0,{R1}) = {int(sub1.rowptr[-1])} nnz, {dt1:.1f} s"}}


def oracle_reorder(A, params: dict, target_s: float = 20.0) -> dict:
    """The reorder oracle (O3-O13: LSH, Alg 3, tiling, decisions; oracle.plan) timed on the
    host on a bounded row prefix of the workload, grown until ~target_s (set
    beside the GPU reorder time).  O4 runs on all OpenMP threads, Alg 3 on one."""
    from oracle import oracle as O
    O.build()
    kw = {k: params[k] for k in ("siglen", "bsize", "seed", "max_bucket", "threshold_size", "panel_rows",
                                 "dense_min", "auto_dense_min")}
    kw["mode"] = {"auto": O.MODE_AUTO, "force": O.MODE_FORCE, "off": O.MODE_OFF}[params["mode"]]
    R = max(params["panel_rows"], A.nrows // 64)
    while True:
        sub = row_prefix(A, R)
        t0 = time.perf_counter()
        p = O.plan(sub, **kw)
        dt = time.perf_counter() - t0
        if dt * 3 >= target_s or R >= A.nrows:
            break
        R = min(A.nrows, int(R * max(1.5, min(4.0, target_s / 2 / max(dt, 1e-3)))))
    return {"seconds": dt, "rows": R, "nnz": int(sub.rowptr[-1]), "rows_per_s": R / dt,
            "nnz_per_s": int(sub.rowptr[-1]) / dt, "round1": p["stats"]["round1"], "round2": p["stats"]["round2"],
            "E1": p["stats"]["E1"], "E2": p["stats"]["E2"], "threads": O.num_threads(), "host": host_cpu(),
            "sample": f"rows [0,{R}) of {A.nrows} ({int(sub.rowptr[-1])} of {A.nnz} nnz), same parameters"}


def run_reference(args, A, ops):
    s = oracle_sample(A, args.K, max(2.0, args.cpu_seconds / 4), ops)
    O = s["O"]

    def step():
        if "spmm" in ops:
            O.spmm(s["sub"], s["B"])
        if "sddmm" in ops:
            O.sddmm(s["sub"], s["X"], s["Y"])
    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = time.perf_counter() - t0
    value = s["flops"] * args.steps / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "GFLOP/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(args, A, ops, 1),
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": O.num_threads(), "kind": "oracle",
                         "host": host_cpu(),
                         "sample": f"rows [0,{s['rows']}) = {s['nnz']} nnz of {A.nnz} per step"},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def workload_config(args, A, ops, world) -> dict:
    return {"workload": f"{args.config} (configs[{list(gen.CONFIGS).index(args.config)}])",
            "nrows": A.nrows, "ncols": A.ncols, "nnz": A.nnz, "K": args.K, "ops": ops,
            "parallelism": f"row-panel shards x{world}" if world > 1 else "single GPU",
            "l2": "512 MB write between steps (outside timed intervals); "
                  + ("B/X/Y larger than the 126 MB L2" if 4.0 * args.K * A.ncols > 126e6
                     else "gathered operand fits the L2 (cold at each step start)")}


# ----------------------------------------------------------------------------- our arm
def algorithmic_bytes(kind: str, tm: dict, K: int) -> float:
    """Compulsory bytes of one launch: every sparse entry's
    (col, val) once (SDDMM also its 4-byte output index and 4-byte output write), every work
    item descriptor once, every distinct gathered dense row once, every output row written once."""
    row = 4.0 * K
    if kind == "spmm_sparse_rows":
        return (8.0 * tm["sparse_nnz"] + 16.0 * tm["sparse_items"] + row * tm["sparse_distinct_cols"]
                + row * (tm["sparse_rows"] + tm["zero_rows"]) + row * tm["rmw_rows"])
    if kind == "spmm_register_tiles":  # the dense part on the register-tile engine
        kind = "spmm_dense_tiles"
    if kind == "sddmm_register_tiles":
        kind = "sddmm_dense_tiles"
    if kind == "spmm_dense_tiles":
        return 8.0 * tm["dense_nnz"] + row * tm["dense_distinct_cols"] + row * tm["dense_rows"]
    if kind == "sddmm_sparse_rows":
        return (16.0 * tm["sparse_nnz"] + 16.0 * tm["sparse_items"] + row * tm["sparse_distinct_cols"]
                + row * tm["sparse_rows"])
    if kind == "sddmm_dense_tiles":
        return 16.0 * tm["dense_nnz"] + row * tm["dense_distinct_cols"] + row * tm["dense_rows"]
    raise KeyError(kind)


def model_bytes(kind: str, tm: dict, K: int) -> float:
    """SURVEY §8(d) bytes model: B-row traffic from the access-count model (O14)."""
    row = 4.0 * K
    if kind.endswith("sparse_rows"):
        return algorithmic_bytes(kind, tm, K) + row * (tm["sparse_group_loads"] - tm["sparse_distinct_cols"])
    return algorithmic_bytes(kind, tm, K) + row * (tm["dense_col_loads"] - tm["dense_distinct_cols"])


def gathered_bytes(kind: str, tm: dict, K: int) -> float:
    """Bytes the kernel moves from L2/HBM into the SMs for its gathered dense rows: one K·4-byte
    row per remainder nnz (phase S), one per staged dense column of a tile (phase D)."""
    row = 4.0 * K
    return row * (tm["sparse_nnz"] if kind.endswith("sparse_rows") else tm["dense_col_loads"])


def gather_ceiling(K: int):
    """Measured ceiling of random row gathers that HIT the L2 (profiles/gather_bw.cu, committed
    results in profiles/r01/gather_bw.jsonl: the largest rate over the L2-resident table sizes
    <= 64 MB, 8 CTAs/SM, nearest row width 128 or 512 bytes)."""
    path = os.path.join(ROOT, "profiles", "r01", "gather_bw.jsonl")
    if not os.path.exists(path):
        return None, None
    rb = 512 if K * 4 >= 320 else 128
    best = None
    with open(path) as f:
        for line in f:
            d = json.loads(line)
            if d.get("row_bytes") == rb and d.get("ctas_per_sm") == 8 and d.get("table_MB", 1e9) <= 64:
                best = max(best or 0.0, d["gather_GBs"])
    if best is None:
        return None, None
    return best, f"profiles/r01/gather_bw.jsonl: L2-resident random {rb}-byte row gathers (max over <= 64 MB tables)"


def kernel_source_sig() -> str:
    """Hash of the kernel sources: an ncu traffic record is used only if it was captured from
    the same kernels (profiles/ncu_traffic.py stores the same signature)."""
    h = hashlib.sha256()
    for f in ("exec.cu", "internal.h"):
        with open(os.path.join(ROOT, "paper_conf_ppopp_jiangha20_b200", "csrc", f), "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()[:16]


def ncu_records(config: str, K: int) -> dict:
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(path):
        return {}
    with open(path) as f:
        tr = json.load(f)
    sig = kernel_source_sig()
    out = {}
    for key, rec in tr.items():
        pre = f"{config}_K{K}_"
        if key.startswith(pre) and rec.get("kernel_sig") == sig:
            out[key[len(pre):]] = rec
    return out


class Stepper:
    """Times SpMM + SDDMM steps of one handle at one K with CUDA events on the launching
    stream (per op) and the library's per-launch events (per kernel)."""

    def __init__(self, torch, M, A, K, ops, dev, flush, stream):
        self.torch, self.M, self.K, self.ops, self.flush, self.stream = torch, M, K, ops, flush, stream
        self.B = torch.from_numpy(gen.dense(A.ncols, K, stream=0)).to(dev) if "spmm" in ops else None
        self.X = torch.from_numpy(gen.dense(A.nrows, K, stream=1)).to(dev) if "sddmm" in ops else None
        self.Y = torch.from_numpy(gen.dense(A.ncols, K, stream=2)).to(dev) if "sddmm" in ops else None
        self.C = torch.empty((M.out_rows, K), dtype=torch.float32, device=dev) if "spmm" in ops else None
        self.out = torch.empty(M.out_nnz, dtype=torch.float32, device=dev) if "sddmm" in ops else None
        self.ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in ops]
        self.kern_ms: dict = {}
        self.step_ms: list = []
        self.launches = 0
        M.set_profiling(True)

    def step(self, record: bool) -> float:
        self.flush.fill_(1.0)
        total = 0.0
        for i, op in enumerate(self.ops):
            self.ev[i][0].record(self.stream)
            if op == "spmm":
                self.M.spmm(self.B, self.C, stream=self.stream)
            else:
                self.M.sddmm(self.X, self.Y, self.out, stream=self.stream)
            self.ev[i][1].record(self.stream)
            n = self.M.last_launch_count()
            times = self.M.last_kernel_times()  # waits for the library's own events of this op
            self.ev[i][1].synchronize()
            total += self.ev[i][0].elapsed_time(self.ev[i][1])
            if record:
                self.launches += n
                for name, ms in times:
                    self.kern_ms.setdefault(name, []).append(ms)
        if record:
            self.step_ms.append(total)
        return total

    def kernels(self, tm: dict, records: dict) -> dict:
        kern = {}
        tot = sum(self.step_ms)
        for k, v in self.kern_ms.items():
            d = {"launches": len(v), "avg_ms": sum(v) / len(v), "median_ms": statistics.median(v), "total_ms": sum(v)}
            d["algorithmic_bytes"] = algorithmic_bytes(k, tm, self.K)
            d["model_bytes"] = model_bytes(k, tm, self.K)
            d["achieved_gbs"] = d["algorithmic_bytes"] / (d["avg_ms"] / 1e3) / 1e9
            d["model_gbs"] = d["model_bytes"] / (d["avg_ms"] / 1e3) / 1e9
            d["share_of_step"] = d["total_ms"] / tot if tot > 0 else None
            rec = records.get(k)
            if rec is not None:
                d["dram_bytes_ncu"] = rec["bytes"]
                d["dram_gbs"] = rec["bytes"] / (d["avg_ms"] / 1e3) / 1e9
                for hk in ("l2_hit_pct", "l1_hit_pct"):
                    if hk in rec:
                        d[hk + "_ncu"] = rec[hk]
            kern[k] = d
        return kern


def roofline_of(kern: dict, tm: dict, K: int, records: dict, peak: float, peak_src: str):
    if not kern:
        return None, None
    dom = max(kern, key=lambda k: kern[k]["total_ms"])
    d = kern[dom]
    rec = records.get(dom)
    traffic = rec["bytes"] if rec is not None else None
    roof = {"kernel": dom, "bound": "hbm", "achieved": d["achieved_gbs"], "peak": peak, "unit": "GB/s",
            "frac": d["achieved_gbs"] / peak, "traffic": traffic, "peak_source": peak_src,
            "algorithmic_bytes_per_launch": d["algorithmic_bytes"], "avg_ms": d["avg_ms"],
            "traffic_source": (rec or {}).get("source")}
    if traffic:
        # north_star's "achieved HBM GB/s": ncu DRAM bytes per launch / this run's launch time
        roof["dram_gbs"] = traffic / (d["avg_ms"] / 1e3) / 1e9
        roof["dram_frac"] = roof["dram_gbs"] / peak
    gather = None
    ceil_gbs, ceil_src = gather_ceiling(K)
    if ceil_gbs:
        gb = gathered_bytes(dom, tm, K)
        ach = gb / (d["avg_ms"] / 1e3) / 1e9
        gather = {"kernel": dom, "bound": "l2_gather", "achieved": ach, "peak": ceil_gbs, "unit": "GB/s",
                  "frac": ach / ceil_gbs, "gathered_bytes_per_launch": gb, "peak_source": ceil_src}
    return roof, gather


def per_op(kern: dict, nnz: int, K: int, world: int) -> dict:
    res = {}
    for name in ("spmm", "sddmm"):
        ks = [k for k in kern if k.startswith(name)]
        if ks:
            ms = sum(kern[k]["avg_ms"] for k in ks)
            gf = 2.0 * nnz * K / (ms / 1e3) / 1e9 if world == 1 else None
            # FP32 fraction: against 148 SMs x 128 FP32 lanes x 2 x 1.965 GHz
            res[name] = {"ms": ms, "gflops": gf, "fp32_frac": gf / FP32_PEAK_GFLOPS if gf else None}
    return res


def build_plan(sr, A, params, world, rank, local_rank):
    """Rank 0 reorders the whole matrix once; the plan image goes to every rank, which loads
    its shard.  Returns (handle, reorder seconds on rank 0, stats of the full plan, image,
    shard load seconds)."""
    import torch
    full, st_full, image = None, None, None
    t0 = time.perf_counter()
    if rank == 0:
        full = sr.SparseMatrix.from_csr(A, device=local_rank)  # ingest (a1) is not preprocessing
        t0 = time.perf_counter()
        full.reorder(params)
        st_full = full.stats()
        if world > 1:
            image = full.save_plan()
    t_reorder = time.perf_counter() - t0
    if world == 1:
        return full, t_reorder, st_full, None, 0.0
    from paper_conf_ppopp_jiangha20_b200 import dist
    image = dist.broadcast_bytes(image, 0, device=torch.device("cuda", local_rank))
    if full is not None:
        full.close()
    t1 = time.perf_counter()
    M = dist.load_shard(A, image, world, rank, local_rank)
    return M, t_reorder, st_full, image, time.perf_counter() - t1


def run_ours(args, A, ops, rank, world, local_rank):
    import torch
    import paper_conf_ppopp_jiangha20_b200 as sr
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    K = args.K
    mode = {"auto": sr.AUTO, "force": sr.FORCE, "off": sr.OFF}[args.mode]
    pdict = dict(mode=args.mode, panel_rows=args.panel_rows, tile_cols=args.tile_cols, max_bucket=args.max_bucket,
                 dense_min=args.dense_min, auto_dense_min=args.auto_dense_min, siglen=128, bsize=2,
                 threshold_size=256, seed=4)
    params = sr.default_params(mode=mode, panel_rows=args.panel_rows, tile_cols=args.tile_cols,
                               max_bucket=args.max_bucket, dense_min=args.dense_min,
                               auto_dense_min=args.auto_dense_min)
    if args.plan_cache and world == 1 and os.path.exists(args.plan_cache):
        M = sr.SparseMatrix.from_csr(A, device=local_rank)
        t0 = time.perf_counter()
        with open(args.plan_cache, "rb") as f:
            M.load_plan(f.read())
        t_pre, st_full, image, t_load = time.perf_counter() - t0, M.stats(), None, 0.0
    else:
        M, t_pre, st_full, image, t_load = build_plan(sr, A, params, world, rank, local_rank)
        if args.plan_cache and world == 1:
            with open(args.plan_cache, "wb") as f:
                f.write(M.save_plan())
    tm = M.traffic_model()
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream(dev)
    S = Stepper(torch, M, A, K, ops, dev, flush, stream)

    dist = world > 1
    if dist:
        import torch.distributed as tdist
    clocks = ClockSampler(local_rank)
    clocks.start()
    t_w = time.perf_counter()
    for _ in range(max(3, args.warmup)):
        S.step(False)
    while time.perf_counter() - t_w < args.min_warm_s:  # let the sampler see the GPU under load
        S.step(False)
    if dist:
        tdist.barrier()
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    dev_ms = 0.0
    for _ in range(args.steps):
        dev_ms += S.step(True)
    torch.cuda.synchronize()
    if dist:
        tdist.barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    t = torch.tensor([dev_ms, statistics.median(S.step_ms)], dtype=torch.float64, device=dev)
    if dist:
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    max_ms, med_ms = float(t[0].item()), float(t[1].item())
    flops_per_step = 2.0 * A.nnz * K * len(ops)  # whole matrix, all ranks together
    value = flops_per_step * args.steps / (max_ms / 1e3) / 1e9

    peak, peak_src = measured_peaks()
    records = ncu_records(args.config, K) if world == 1 else {}
    kern = S.kernels(tm, records)
    roofline, gather_roof = roofline_of(kern, tm, K, records, peak, peak_src)
    launches = S.launches

    # further K on the same plan (BASELINE metric: K = 32 and 128)
    extra = {}
    ks = args.extra_K if args.extra_K is not None else ("32" if args.config == "rmat" and K == 128 else "")
    ks = "" if ks == "none" else ks
    for k2 in [int(x) for x in ks.split(",") if x.strip()]:
        S2 = Stepper(torch, M, A, k2, ops, dev, flush, stream)
        for _ in range(max(3, args.warmup)):
            S2.step(False)
        if dist:
            tdist.barrier()
        ms2 = sum(S2.step(True) for _ in range(args.steps))
        t2 = torch.tensor([ms2], dtype=torch.float64, device=dev)
        if dist:
            tdist.all_reduce(t2, op=tdist.ReduceOp.MAX)
        rec2 = ncu_records(args.config, k2) if world == 1 else {}
        kern2 = S2.kernels(tm, rec2)
        roof2, _ = roofline_of(kern2, tm, k2, rec2, peak, peak_src)
        extra[str(k2)] = {"value": 2.0 * A.nnz * k2 * len(ops) * args.steps / (float(t2.item()) / 1e3) / 1e9,
                          "unit": "GFLOP/s", "ms_per_step": float(t2.item()) / args.steps,
                          "ms_per_step_median": statistics.median(S2.step_ms), "kernels": kern2,
                          "roofline": roof2, "per_op_gflops": per_op(kern2, A.nnz, k2, world),
                          "gpu_launches": S2.launches}
        del S2

    # end to end through the public API with host buffers (pinned), per step
    e2e = None
    if args.e2e_steps > 0:
        B, X, Y, C, out = S.B, S.X, S.Y, S.C, S.out
        hB = torch.from_numpy(gen.dense(A.ncols, K, stream=0)).pin_memory() if "spmm" in ops else None
        hX = torch.from_numpy(gen.dense(A.nrows, K, stream=1)).pin_memory() if "sddmm" in ops else None
        hY = torch.from_numpy(gen.dense(A.ncols, K, stream=2)).pin_memory() if "sddmm" in ops else None
        hC = torch.empty(C.shape, dtype=torch.float32).pin_memory() if "spmm" in ops else None
        hO = torch.empty(out.shape, dtype=torch.float32).pin_memory() if "sddmm" in ops else None
        h2d = (hB.numel() * 4 if "spmm" in ops else 0) + ((hX.numel() + hY.numel()) * 4 if "sddmm" in ops else 0)
        d2h = (hC.numel() * 4 if "spmm" in ops else 0) + (hO.numel() * 4 if "sddmm" in ops else 0)
        M.set_profiling(False)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        side = torch.cuda.Stream(device=dev)  # SDDMM's copies and kernels overlap SpMM's
        side_done = torch.cuda.Event()
        tot = 0.0
        for i in range(args.e2e_steps + 1):
            flush.fill_(1.0)
            e0.record(stream)
            side.wait_event(e0)
            if "spmm" in ops:
                with torch.cuda.stream(stream):
                    B.copy_(hB, non_blocking=True)
                    M.spmm(B, C, stream=stream)
                    hC.copy_(C, non_blocking=True)
            if "sddmm" in ops:
                with torch.cuda.stream(side):
                    X.copy_(hX, non_blocking=True)
                    Y.copy_(hY, non_blocking=True)
                    M.sddmm(X, Y, out, stream=side)
                    hO.copy_(out, non_blocking=True)
            side_done.record(side)
            stream.wait_event(side_done)
            e1.record(stream)
            e1.synchronize()
            if i > 0:
                tot += e0.elapsed_time(e1)
        te = torch.tensor([tot], dtype=torch.float64, device=dev)
        if dist:
            tdist.all_reduce(te, op=tdist.ReduceOp.MAX)
        e2e = {"value": flops_per_step * args.e2e_steps / (float(te.item()) / 1e3) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "note": "pinned host operands copied in and outputs copied out every step, through SparseMatrix; "
                       "SpMM and SDDMM (copies + kernels) on two streams"}
        M.set_profiling(True)

    # offline plan (sr_plan_save / sr_plan_load): what a deployment that saved the
    # plan pays instead of the reorder preprocessing
    if world == 1:
        t0 = time.perf_counter()
        image = M.save_plan()
        t_save = time.perf_counter() - t0
        M2 = sr.SparseMatrix.from_csr(A, device=local_rank)
        t0 = time.perf_counter()
        M2.load_plan(image)
        t_load1 = time.perf_counter() - t0
        M2.close()
        offline = {"image_bytes": len(image), "save_s": t_save, "load_s": t_load1,
                   "preprocess_to_load_ratio": t_pre / max(t_load1, 1e-9)}
    else:
        offline = {"image_bytes": len(image), "load_s": t_load}

    # shard simulation on this one GPU: every shard's plan timed in turn (load balance of the
    # nnz-balanced panel partition); a proxy, reported apart from the measured line
    sim = None
    if args.simulate_world > 1 and world == 1:
        Wn = args.simulate_world
        ms, nnzs = [], []
        for r in range(Wn):
            Ms = sr.SparseMatrix.from_csr(A, device=local_rank)
            Ms.load_plan(image, world=Wn, rank=r)
            Ss = Stepper(torch, Ms, A, K, ops, dev, flush, stream)
            for _ in range(max(3, args.warmup)):
                Ss.step(False)
            ms.append(sum(Ss.step(True) for _ in range(args.steps)) / args.steps)
            nnzs.append(Ms.stats()["shard_nnz"])
            del Ss
            Ms.close()
        sim = {"world": Wn, "per_shard_ms": ms, "per_shard_nnz": nnzs, "max_ms": max(ms),
               "balance_mean_over_max": (sum(ms) / Wn) / max(ms),
               "value_if_shards_ran_in_parallel": flops_per_step / (max(ms) / 1e3) / 1e9,
               "speedup_vs_1": (max_ms / args.steps) / max(ms),
               "note": "each shard's plan timed alone on this one GPU (simulation, not a multi-GPU measurement)"}

    gather = None
    if args.gather and dist and "spmm" in ops:
        from paper_conf_ppopp_jiangha20_b200 import dist as sdist
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        tdist.barrier()
        g0.record()
        sdist.gather_spmm(M, S.C)
        g1.record()
        torch.cuda.synchronize()
        gt = torch.tensor([g0.elapsed_time(g1)], dtype=torch.float64, device=dev)
        tdist.all_reduce(gt, op=tdist.ReduceOp.MAX)
        gather = {"ms": float(gt.item()), "op": "dist.gather_spmm (padded all-gather + scatter)"}

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu = cpu_baseline(A, K, args, ops, args.config)
        oreo = None
        if not args.no_oracle_reorder and world == 1:
            oreo = oracle_reorder(A, pdict)
        stp = st_full
        cfg = workload_config(args, A, ops, world)
        cfg["plan"] = pdict
        line = {
            "metric": METRIC,
            "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": max_ms / args.steps, "ms_per_step_median": med_ms,
            "value_at_median_step": flops_per_step / (med_ms / 1e3) / 1e9,
            "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": cfg,
            "roofline": roofline,
            "gather_roofline": gather_roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
            "kernels": kern,
            "per_op_gflops": per_op(kern, A.nnz, K, world),
            "extra_K": extra,
            "preprocess": {"seconds": t_pre, "lsh1_s": stp["t_lsh1_s"], "cluster1_s": stp["t_cluster1_s"],
                           "tile_s": stp["t_tile_s"], "lsh2_s": stp["t_lsh2_s"], "cluster2_s": stp["t_cluster2_s"],
                           "plan_build_s": stp["t_plan_s"], "reorder_call_s": stp["t_total_s"],
                           "round1": stp["round1"], "round2": stp["round2"], "E1": stp["E1"], "E2": stp["E2"],
                           "dense_ratio0": stp["dense0"] / max(1, stp["nnz"]),
                           "dense_ratio": stp["dense1"] / max(1, stp["nnz"]),
                           "avgsim": (stp["avgsim_num"] / stp["avgsim_den"]) if stp["avgsim_den"] else 0.0,
                           "ratio_to_step": t_pre / (max_ms / args.steps / 1e3),
                           "shard_load_s": t_load if world > 1 else None,
                           "oracle": oreo},
            "offline_plan": offline,
            "shard_simulation": sim,
            "traffic_model": tm,
            "wall_s": wall,
            "gather": gather,
            "paper_context": PAPER_CONTEXT,
        }
        print(json.dumps(line), flush=True)


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def spawn_ranks(n: int, argv) -> int:
    """Re-launch this script under torch.distributed.run with n ranks (one per GPU)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + list(argv)
    return subprocess.call(cmd)


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    args = parse(argv)
    ops = [o.strip() for o in args.ops.split(",") if o.strip()]
    env_world = os.environ.get("WORLD_SIZE")
    if args.impl == "ours" and args.gpus > 1 and env_world is None:
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            raise SystemExit(f"bench.py --gpus {args.gpus}: only {have} CUDA device(s) visible")
        sys.exit(spawn_ranks(args.gpus, argv))
    world = int(env_world or "1")
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if env_world is not None and args.gpus not in (1, world):
        raise SystemExit(f"bench.py --gpus {args.gpus} under a launcher with WORLD_SIZE={world}")
    if args.impl == "reference":
        if rank != 0:
            return  # the oracle arm runs on rank 0 only
        run_reference(args, gen.make(args.config), ops)
        return
    A = gen.make(args.config)
    if world > 1:
        import torch
        import torch.distributed as tdist
        if torch.cuda.device_count() <= local_rank:
            raise SystemExit(f"rank {rank}: no CUDA device {local_rank} ({torch.cuda.device_count()} visible)")
        torch.cuda.set_device(local_rank)
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    run_ours(args, A, ops, rank, world, local_rank)
    if world > 1:
        import torch.distributed as tdist
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
