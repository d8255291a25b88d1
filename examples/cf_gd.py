#!/usr/bin/env python3
"""CF gradient descent over reordered plans (Tables 3/4).

Builds the plans of R and Rᵀ once, then runs full-batch gradient steps (one SDDMM + two
SpMMs + set_values per step, paper_conf_ppopp_jiangha20_b200/cf.py) and prints one JSON
line: preprocessing seconds, device ms per iteration (CUDA events, median), the ratio of
preprocessing to one iteration (the paper's Tables 3/4 quantity), the iterations after which
reordering has paid for itself against the original-order plans, and the loss trajectory.

  python examples/cf_gd.py [--config cf] [--K 128] [--iters 20] [--lr 1e-6]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from synth import generators as gen  # noqa: E402


def run(R, K, iters, lr, reorder, params):
    import torch
    from paper_conf_ppopp_jiangha20_b200.cf import CFModel
    t0 = time.perf_counter()
    m = CFModel(R, K, params=params, reorder=reorder)
    torch.cuda.synchronize()
    t_pre = time.perf_counter() - t0
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(iters)]
    losses = []
    for i in range(iters):
        ev[i][0].record()
        losses.append(m.step(lr))  # syncs on the loss
        ev[i][1].record()
    torch.cuda.synchronize()
    ms = [a.elapsed_time(b) for a, b in ev[2:]] or [ev[-1][0].elapsed_time(ev[-1][1])]
    m.close()
    return t_pre, statistics.median(ms), losses


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cf", choices=list(gen.CONFIGS))
    ap.add_argument("--K", type=int, default=128)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--lr", type=float, default=1e-6)
    ap.add_argument("--dense-min", type=int, default=64)
    args = ap.parse_args()
    import paper_conf_ppopp_jiangha20_b200 as sr
    R = gen.make(args.config)
    params = sr.default_params(dense_min=args.dense_min)
    pre_r, it_r, loss_r = run(R, args.K, args.iters, args.lr, True, params)
    pre_o, it_o, loss_o = run(R, args.K, args.iters, args.lr, False, params)
    gain = it_o - it_r
    line = {"workload": f"cf-gd on {args.config}", "nnz": R.nnz, "K": args.K, "iters": args.iters,
            "reordered": {"preprocess_s": pre_r, "iter_ms": it_r, "loss_first": loss_r[0], "loss_last": loss_r[-1]},
            "original": {"preprocess_s": pre_o, "iter_ms": it_o, "loss_first": loss_o[0], "loss_last": loss_o[-1]},
            "preprocess_to_iter_ratio": (pre_r - pre_o) / (it_r / 1e3),
            "breakeven_iters": ((pre_r - pre_o) / (gain / 1e3)) if gain > 0 else None,
            "note": "iteration = set_values(1) + SDDMM + residual + set_values(E) + SpMM(R) + "
                    "set_values(E^T) + SpMM(R^T) + update, device time; preprocess = both plans"}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
