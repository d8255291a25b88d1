"""Measure the B200's L2-resident copy bandwidth (the ceiling of a gather kernel whose rows hit
L2) and the HBM copy bandwidth, with CUDA events.  Writes one JSON line.

  python profiles/l2_bw.py
"""
import json

import torch


def bw(nbytes, reps=200):
    n = nbytes // 4
    x = torch.rand(n, device="cuda")
    y = torch.empty_like(x)
    for _ in range(10):
        y.copy_(x)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s.record()
    for _ in range(reps):
        y.copy_(x)
    e.record()
    torch.cuda.synchronize()
    return 2 * nbytes * reps / (s.elapsed_time(e) / 1e3) / 1e9


if __name__ == "__main__":
    res = {f"copy_{mb}MB_GBs": bw(mb << 20) for mb in (8, 16, 32, 48)}
    res["copy_4096MB_GBs"] = bw(4096 << 20, reps=10)
    res["note"] = "read+write bytes / time of torch copy_; <=48 MB working sets are L2-resident (126 MB L2)"
    print(json.dumps(res))
