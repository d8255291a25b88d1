#!/usr/bin/env python3
"""bench.py — SpMM / SDDMM throughput of the row-reordered, adaptively tiled path on B200.

Metric (BASELINE.json): SpMM/SDDMM GFLOP/s (2·nnz·K per op) and HBM GB/s as a fraction of
roofline.  Workload at N=1: C2, the R-MAT scale-20 matrix (configs[1]), K=128.

One step = one pass of the execution hot path over the planned matrix: C := A·B (SpMM)
and out := A ⊙ (X·Yᵀ) on A's pattern (SDDMM), both through the C ABI (libsr.so).  The
reorder preprocessing (LSH on the GPU + Alg 3 on the host + ASpT tiling) runs once
before the timed region and is reported separately (`preprocess`), as the paper does
(P:277).  Inputs are resident in HBM; a 512 MB write flushes L2 between steps
(outside the device-timed intervals).  Multi-GPU: torchrun, one rank per GPU, rank r
computes its nnz-balanced panel shard (strong scaling, no collective in the step).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config rmat] [--K 128] [--ops spmm,sddmm]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import generators as gen  # noqa: E402

FP32_PEAK_GFLOPS = 148 * 128 * 2 * 1.965  # dense FP32 FMA peak (74.4 TFLOP/s), DESIGN.md §5
PAPER_CONTEXT = ("P100 (paper, P:334, P:350): ASpT-RR up to 2.91x SpMM vs best of ASpT-NR/cuSPARSE and "
                 "up to 3.19x SDDMM vs ASpT-NR; geomean 1.19x / 1.49x (K=1024)")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="rmat", choices=list(gen.CONFIGS))
    ap.add_argument("--K", type=int, default=128)
    ap.add_argument("--ops", default="spmm,sddmm")
    ap.add_argument("--mode", default="auto", choices=["auto", "force", "off"])
    ap.add_argument("--panel-rows", type=int, default=64)
    ap.add_argument("--tile-cols", type=int, default=64)
    ap.add_argument("--max-bucket", type=int, default=32)
    # ASpT dense-column threshold (R17).  The paper's example is 2 (a P100 with 64 KB of
    # shared memory per SM); on B200 (126 MB L2, row-group task kernels gathering from L2 at ~15 TB/s)
    # staging pays only for columns shared by (nearly) the whole 64-row panel: sweeps in
    # profiles/r01/NOTES.md (session 3: 64 best with tiles present, equal to no tiles).
    ap.add_argument("--dense-min", type=int, default=64)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target CPU work of cpu_baseline")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--gather", action="store_true", help="also time the optional NCCL all-gather of C")
    ap.add_argument("--min-warm-s", type=float, default=1.0, help="keep warming up until this long (clocks)")
    return ap.parse_args()


def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


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
def oracle_sample(A, K, target_s, ops):
    """Time the CPU oracle (oracle/, fp64, OpenMP over the host cores) on a bounded row
    sample of the workload: rows [0, R) with R grown until ~target_s of work."""
    from oracle import oracle as O
    O.build()
    B = gen.dense(A.ncols, K, stream=0)
    Y = gen.dense(A.ncols, K, stream=2) if "sddmm" in ops else None
    R = max(1, A.nrows // 256)
    while True:
        sub = gen.CSR(R, A.ncols, A.rowptr[:R + 1].copy(), A.colidx[:A.rowptr[R]], A.vals[:A.rowptr[R]])
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
    sub1 = gen.CSR(R1, A.ncols, A.rowptr[:R1 + 1].copy(), A.colidx[:A.rowptr[R1]], A.vals[:A.rowptr[R1]])
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
            "sample": f"{name} rows [0,{s['rows']}) = {s['nnz']} nnz of {A.nnz}, K={K}, {'+'.join(ops)} in fp64, "
                      f"{reps} pass(es), {dt:.1f} s",
            "single_thread": {"value": st_value, "unit": "GFLOP/s", "cores": 1,
                              "sample": f"rows [0,{R1}) = {int(sub1.rowptr[-1])} nnz, {dt1:.1f} s"}}


def run_reference(args, A, ops, rank, world):
    if rank != 0:
        return
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
        "impl": "reference", "metric": "SpMM+SDDMM GFLOP/s (2*nnz*K per op)", "value": value, "unit": "GFLOP/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": args.config, "K": args.K, "ops": ops, "nnz": A.nnz, "nrows": A.nrows,
                   "ncols": A.ncols},
        "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": O.num_threads(), "kind": "oracle",
                         "sample": f"rows [0,{s['rows']}) = {s['nnz']} nnz of {A.nnz} per step"},
        "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def algorithmic_bytes(kind: str, tm: dict, K: int) -> float:
    """Compulsory bytes of one launch: every sparse entry's (col, val) once,
    every distinct gathered dense row once, every output written once."""
    row = 4.0 * K
    if kind == "spmm_sparse_rows":
        return (8.0 * tm["sparse_nnz"] + 16.0 * tm["sparse_items"] + row * tm["sparse_distinct_cols"]
                + row * (tm["sparse_rows"] + tm["zero_rows"]) + row * tm["rmw_rows"])
    if kind == "spmm_dense_tiles":
        return 8.0 * tm["dense_nnz"] + row * tm["dense_distinct_cols"] + row * tm["dense_rows"]
    if kind == "sddmm_sparse_rows":
        return (12.0 * tm["sparse_nnz"] + 16.0 * tm["sparse_items"] + row * tm["sparse_distinct_cols"]
                + row * tm["sparse_rows"])
    if kind == "sddmm_dense_tiles":
        return 12.0 * tm["dense_nnz"] + row * tm["dense_distinct_cols"] + row * tm["dense_rows"]
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
    <= 64 MB, 8 CTAs/SM, nearest row width 128 or 512 bytes).  Every gathered row of phase S
    crosses the L2 -> SM path once, so gathered bytes / this rate bounds the kernel's time from
    below whatever its L2 hit rate (misses only add HBM time)."""
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


def run_ours(args, A, ops, rank, world, local_rank):
    import torch
    import paper_conf_ppopp_jiangha20_b200 as sr
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    K = args.K
    mode = {"auto": sr.AUTO, "force": sr.FORCE, "off": sr.OFF}[args.mode]
    params = sr.default_params(mode=mode, panel_rows=args.panel_rows, tile_cols=args.tile_cols,
                               max_bucket=args.max_bucket, dense_min=args.dense_min, world=world, rank=rank)
    M = sr.SparseMatrix.from_csr(A, device=local_rank)
    t0 = time.perf_counter()
    st = M.reorder(params)
    t_pre = time.perf_counter() - t0
    tm = M.traffic_model()
    B = torch.from_numpy(gen.dense(A.ncols, K, stream=0)).to(dev)
    X = torch.from_numpy(gen.dense(A.nrows, K, stream=1)).to(dev)
    Y = torch.from_numpy(gen.dense(A.ncols, K, stream=2)).to(dev)
    C = torch.empty((M.out_rows, K), dtype=torch.float32, device=dev)
    out = torch.empty(M.out_nnz, dtype=torch.float32, device=dev)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    stream = torch.cuda.current_stream()
    M.set_profiling(True)
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in ops]
    kern_ms: dict = {}
    launches = 0

    def step(record: bool):
        nonlocal launches
        flush.fill_(1.0)
        total = 0.0
        for i, op in enumerate(ops):
            ev[i][0].record(stream)
            if op == "spmm":
                M.spmm(B, C, stream=stream)
            else:
                M.sddmm(X, Y, out, stream=stream)
            ev[i][1].record(stream)
            n = M.last_launch_count()
            times = M.last_kernel_times()  # waits for the library's own events of this op
            ev[i][1].synchronize()
            total += ev[i][0].elapsed_time(ev[i][1])
            if record:
                launches += n
                for name, ms in times:
                    kern_ms.setdefault(name, []).append(ms)
        return total

    dist = world > 1
    if dist:
        import torch.distributed as tdist
    clocks = ClockSampler(local_rank)
    clocks.start()
    t_w = time.perf_counter()
    for i in range(max(3, args.warmup)):
        step(False)
    while time.perf_counter() - t_w < args.min_warm_s:  # let the sampler see the GPU under load
        step(False)
    if dist:
        tdist.barrier()
    torch.cuda.synchronize()
    wall0 = time.perf_counter()
    dev_ms = 0.0
    for i in range(args.steps):
        dev_ms += step(True)
    torch.cuda.synchronize()
    if dist:
        tdist.barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    t = torch.tensor([dev_ms], dtype=torch.float64, device=dev)
    if dist:
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    max_ms = float(t.item())
    flops_per_step = 2.0 * A.nnz * K * len(ops)  # whole matrix, all ranks together
    value = flops_per_step * args.steps / (max_ms / 1e3) / 1e9

    # per-kernel roofline of the dominant kernel
    peak, peak_src = measured_peaks()
    kern = {k: {"launches": len(v), "avg_ms": sum(v) / len(v), "total_ms": sum(v)} for k, v in kern_ms.items()}
    for k, d in kern.items():
        d["algorithmic_bytes"] = algorithmic_bytes(k, tm, K)
        d["model_bytes"] = model_bytes(k, tm, K)
        d["achieved_gbs"] = d["algorithmic_bytes"] / (d["avg_ms"] / 1e3) / 1e9
        d["model_gbs"] = d["model_bytes"] / (d["avg_ms"] / 1e3) / 1e9
        d["share_of_step"] = d["total_ms"] / dev_ms if dev_ms > 0 else None
    dom = max(kern, key=lambda k: kern[k]["total_ms"]) if kern else None
    traffic = None
    prof_path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if dom and os.path.exists(prof_path):
        with open(prof_path) as f:
            tr = json.load(f)
        rec = tr.get(f"{args.config}_K{K}_{dom}")
        if rec is not None and world == 1:
            traffic = rec["bytes"]  # ncu --set full, per launch (profiles/ncu_traffic.py)
    roofline = None
    if dom:
        d = kern[dom]
        roofline = {"kernel": dom, "bound": "hbm", "achieved": d["achieved_gbs"], "peak": peak, "unit": "GB/s",
                    "frac": d["achieved_gbs"] / peak, "traffic": traffic, "peak_source": peak_src,
                    "algorithmic_bytes_per_launch": d["algorithmic_bytes"], "avg_ms": d["avg_ms"]}
        if traffic:
            # north_star's "achieved HBM GB/s": ncu DRAM bytes per launch / this run's launch time
            roofline["dram_gbs"] = traffic / (d["avg_ms"] / 1e3) / 1e9
            roofline["dram_frac"] = roofline["dram_gbs"] / peak
        # the same for every kernel with an ncu record
        if os.path.exists(prof_path) and world == 1:
            with open(prof_path) as f:
                tr_all = json.load(f)
            for k, dk in kern.items():
                rec = tr_all.get(f"{args.config}_K{K}_{k}")
                if rec is not None:
                    dk["dram_bytes_ncu"] = rec["bytes"]
                    dk["dram_gbs"] = rec["bytes"] / (dk["avg_ms"] / 1e3) / 1e9
                    for hk in ("l2_hit_pct", "l1_hit_pct"):
                        if hk in rec:
                            dk[hk + "_ncu"] = rec[hk]

    # the same kernel against the L2 -> SM gather ceiling (the path every gathered row takes;
    # DESIGN.md §5): a conservative efficiency for a gather-bound kernel whose HBM bytes are
    # far below the bytes it moves into the SMs
    gather_roof = None
    if dom:
        d = kern[dom]
        gb = gathered_bytes(dom, tm, K)
        ceil_gbs, ceil_src = gather_ceiling(K)
        if ceil_gbs:
            ach = gb / (d["avg_ms"] / 1e3) / 1e9
            gather_roof = {"kernel": dom, "bound": "l2_gather", "achieved": ach, "peak": ceil_gbs, "unit": "GB/s",
                           "frac": ach / ceil_gbs, "gathered_bytes_per_launch": gb, "peak_source": ceil_src}

    # end to end through the public API with host buffers (pinned), per step
    e2e = None
    if args.e2e_steps > 0:
        hB = torch.from_numpy(gen.dense(A.ncols, K, stream=0)).pin_memory()
        hX = torch.from_numpy(gen.dense(A.nrows, K, stream=1)).pin_memory()
        hY = hB if "sddmm" not in ops else torch.from_numpy(gen.dense(A.ncols, K, stream=2)).pin_memory()
        hC = torch.empty(C.shape, dtype=torch.float32).pin_memory()
        hO = torch.empty(out.shape, dtype=torch.float32).pin_memory()
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

    # offline plan (sr_plan_save / sr_plan_load): what a deployment that saved the
    # plan pays instead of the reorder preprocessing
    offline = None
    if world == 1:
        t0 = time.perf_counter()
        img = M.save_plan()
        t_save = time.perf_counter() - t0
        M2 = sr.SparseMatrix.from_csr(A, device=local_rank)
        t0 = time.perf_counter()
        M2.load_plan(img)
        t_load = time.perf_counter() - t0
        M2.close()
        offline = {"image_bytes": len(img), "save_s": t_save, "load_s": t_load,
                   "preprocess_to_load_ratio": t_pre / max(t_load, 1e-9)}

    gather = None
    if args.gather and dist and "spmm" in ops:
        rows_max = torch.tensor([C.shape[0]], device=dev)
        tdist.all_reduce(rows_max, op=tdist.ReduceOp.MAX)
        pad = torch.zeros((int(rows_max.item()), K), device=dev)
        pad[:C.shape[0]] = C
        bufs = torch.empty((world, int(rows_max.item()), K), device=dev)
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record()
        tdist.all_gather_into_tensor(bufs, pad)
        g1.record()
        torch.cuda.synchronize()
        gather = {"ms": g0.elapsed_time(g1), "bytes_per_rank": pad.numel() * 4}

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu = cpu_baseline(A, K, args, ops, args.config)
        stp = M.stats()
        line = {
            "metric": "SpMM+SDDMM GFLOP/s (2*nnz*K per op) and HBM GB/s (fraction of roofline)",
            "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": max_ms / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{args.config} (configs[{list(gen.CONFIGS).index(args.config)}])",
                       "nrows": A.nrows, "ncols": A.ncols, "nnz": A.nnz, "K": K, "ops": ops,
                       "parallelism": f"row-panel shards x{world}" if world > 1 else "single GPU",
                       "l2": "512 MB write between steps (outside timed intervals); "
                             + ("B/X/Y larger than the 126 MB L2" if 4.0 * K * A.ncols > 126e6
                                else "gathered operand fits the L2 (cold at each step start)"),
                       "plan": {"mode": args.mode, "panel_rows": args.panel_rows, "tile_cols": args.tile_cols,
                                "max_bucket": args.max_bucket, "dense_min": args.dense_min, "siglen": 128, "bsize": 2, "threshold_size": 256,
                                "seed": 4}},
            "roofline": roofline,
            "gather_roofline": gather_roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk,
            "kernels": kern,
            "per_op_gflops": None,
            "preprocess": {"seconds": t_pre, "lsh1_s": stp["t_lsh1_s"], "cluster1_s": stp["t_cluster1_s"],
                           "tile_s": stp["t_tile_s"], "lsh2_s": stp["t_lsh2_s"], "cluster2_s": stp["t_cluster2_s"],
                           "round1": stp["round1"], "round2": stp["round2"], "E1": stp["E1"], "E2": stp["E2"],
                           "dense_ratio0": stp["dense0"] / max(1, stp["nnz"]),
                           "dense_ratio": stp["dense1"] / max(1, stp["nnz"]),
                           "avgsim": (stp["avgsim_num"] / stp["avgsim_den"]) if stp["avgsim_den"] else 0.0,
                           "ratio_to_step": t_pre / (max_ms / args.steps / 1e3)},
            "offline_plan": offline,
            "traffic_model": tm,
            "wall_s": wall,
            "gather": gather,
            "paper_context": PAPER_CONTEXT,
        }
        per_op = {}
        for name in ("spmm", "sddmm"):
            ks = [k for k in kern if k.startswith(name)]
            if ks:
                ms = sum(kern[k]["avg_ms"] for k in ks)
                gf = 2.0 * A.nnz * K / (ms / 1e3) / 1e9 if world == 1 else None
                # FP32 fraction: against 148 SMs x 128 FP32 lanes x 2 x 1.965 GHz
                per_op[name] = {"ms": ms, "gflops": gf, "fp32_frac": gf / FP32_PEAK_GFLOPS if gf else None}
        line["per_op_gflops"] = per_op
        print(json.dumps(line), flush=True)


def main():
    args = parse()
    ops = [o.strip() for o in args.ops.split(",") if o.strip()]
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference" and rank != 0:
        return  # the oracle arm runs on rank 0 only
    A = gen.make(args.config)
    if args.impl == "reference":
        run_reference(args, A, ops, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as tdist
        torch.cuda.set_device(local_rank)
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    run_ours(args, A, ops, rank, world, local_rank)
    if world > 1:
        import torch.distributed as tdist
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
