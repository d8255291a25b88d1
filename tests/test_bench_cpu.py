"""CPU-only checks of bench.py's contract plumbing: both arms print the same metric string,
`--gpus N` refuses to run with fewer than N GPUs (instead of silently running one rank),
the roofline bytes model counts SDDMM's output write, host CPU description, and the plan
image broadcast of the multi-GPU path over gloo (world size 2)."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_reference_arm_prints_the_metric_of_our_arm():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "tiny",
                        "--K", "32", "--steps", "2", "--warmup", "1", "--cpu-seconds", "0.2"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["metric"] == bench.METRIC
    assert line["unit"] == "GFLOP/s" and line["higher_is_better"] is True
    assert line["cpu_baseline"]["host"]["logical_cpus"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0


def test_gpus_flag_fails_loudly_without_enough_gpus():
    if torch.cuda.device_count() >= 2:
        return
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT, env=env)
    assert r.returncode != 0
    assert "--gpus 2" in r.stderr and "device" in r.stderr


def test_plan_parameters_per_config():
    """The GNN matrix runs its measured tiled plan (32-row panels, dense_min 4: phase D beats the
    untiled plan there, profiles/r02/NOTES.md r02aa); the others keep dense_min 64; explicit flags win."""
    a = bench.parse(["--config", "gnn"])
    assert (a.panel_rows, a.dense_min) == (32, 4)
    a = bench.parse([])
    assert (a.config, a.panel_rows, a.dense_min) == ("rmat", 64, 64)
    a = bench.parse(["--config", "gnn", "--panel-rows", "16", "--dense-min", "3"])
    assert (a.panel_rows, a.dense_min) == (16, 3)


def test_sddmm_bytes_count_output_write():
    tm = dict(sparse_nnz=10, sparse_items=2, sparse_distinct_cols=3, sparse_rows=2, zero_rows=1, rmw_rows=0,
              dense_nnz=4, dense_distinct_cols=1, dense_rows=1, sparse_group_loads=5, dense_col_loads=1)
    K = 8
    # per nnz: col + val (8) + output index (4) + output write (4); per item 16; rows K*4
    assert bench.algorithmic_bytes("sddmm_sparse_rows", tm, K) == 16 * 10 + 16 * 2 + 32 * 3 + 32 * 2
    assert bench.algorithmic_bytes("sddmm_dense_tiles", tm, K) == 16 * 4 + 32 * 1 + 32 * 1
    assert bench.algorithmic_bytes("spmm_sparse_rows", tm, K) == 8 * 10 + 16 * 2 + 32 * 3 + 32 * 3


def test_host_cpu_description():
    h = bench.host_cpu()
    assert h["logical_cpus"] >= 1 and h["nproc"] >= 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _bcast_worker(rank, world, port, out_dir):
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ppopp_jiangha20_b200 import dist
    payload = bytes(np.random.default_rng(5).integers(0, 256, 100_003, dtype=np.uint8)) if rank == 0 else None
    got = dist.broadcast_bytes(payload, 0)
    empty = dist.broadcast_bytes(b"" if rank == 0 else None, 0)
    with open(os.path.join(out_dir, f"r{rank}.bin"), "wb") as f:
        f.write(got)
    assert empty == b""
    tdist.destroy_process_group()


def test_plan_image_broadcast_gloo(tmp_path):
    mp.spawn(_bcast_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    ref = bytes(np.random.default_rng(5).integers(0, 256, 100_003, dtype=np.uint8))
    for r in range(2):
        assert (tmp_path / f"r{r}.bin").read_bytes() == ref
