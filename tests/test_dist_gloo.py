"""Multi-process host logic of the row-panel sharding, world size 2 over the
gloo backend on CPU: nnz-balanced partition (libsr host entry point), per-rank shard of the
plan, padded all-gather (paper_conf_ppopp_jiangha20_b200.dist.allgather_padded) and
reassembly into original row / nnz order.  Per-shard numerics come from the oracle (test
infrastructure), so this runs without a GPU."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as tdist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, result_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ppopp_jiangha20_b200 as sr
    from paper_conf_ppopp_jiangha20_b200.dist import allgather_padded
    from oracle import oracle as O
    from synth import generators as g

    A = g.random_csr(300, 200, 0.04, 17, empty_frac=0.1)
    P = 16
    plan = O.plan(A, panel_rows=P, mode=O.MODE_FORCE, max_bucket=0)
    M = A.nrows
    w = [int(plan["drow_ptr"][min(M, (p + 1) * P)] - plan["drow_ptr"][p * P]
             + plan["rrow_ptr"][min(M, (p + 1) * P)] - plan["rrow_ptr"][p * P]) for p in range(plan["npanels"])]
    cuts = sr.host_partition(np.array(w), world)
    q0, q1 = int(cuts[rank]) * P, min(M, int(cuts[rank + 1]) * P)
    rows = plan["perm1"][q0:q1]
    # packed SpMM rows of this shard
    B = g.dense(A.ncols, 8)
    C_local, _ = O.spmm_rows(A, B, rows.astype(np.int64))
    # packed SDDMM nnz of this shard: by position, dense (slot order) then remainder
    ids = np.concatenate([np.concatenate([plan["d_pos"][plan["drow_ptr"][q]:plan["drow_ptr"][q + 1]],
                                          plan["r_pos"][plan["rrow_ptr"][q]:plan["rrow_ptr"][q + 1]]])
                          for q in range(q0, q1)] or [np.zeros(0, np.int64)]).astype(np.int64)
    X, Y = g.dense(A.nrows, 8, stream=1), g.dense(A.ncols, 8, stream=2)
    full_out, _ = O.sddmm(A, X, Y)
    out_local = full_out[ids]
    # gather
    Cp = allgather_padded(torch.from_numpy(C_local))
    Rp = allgather_padded(torch.from_numpy(rows.astype(np.int64)))
    Op = allgather_padded(torch.from_numpy(out_local))
    Ip = allgather_padded(torch.from_numpy(ids))
    C = np.full((M, 8), np.nan)
    for c, r in zip(Cp, Rp):
        C[r.numpy()] = c.numpy()
    out = np.full(A.nnz, np.nan)
    for o, i in zip(Op, Ip):
        out[i.numpy()] = o.numpy()
    ref, _ = O.spmm_rows(A, B, np.arange(M))
    ok = bool(np.array_equal(C, ref) and np.array_equal(out, full_out))
    sizes = [int(x.shape[0]) for x in Rp]
    np.save(os.path.join(result_dir, f"r{rank}.npy"), np.array([ok, sum(sizes) == M, len(set(
        np.concatenate([r.numpy() for r in Rp]).tolist())) == M], dtype=bool))
    tdist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_sharded_gather_gloo(tmp_path, world):
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path)), nprocs=world, join=True)
    for r in range(world):
        res = np.load(tmp_path / f"r{r}.npy")
        assert res.all(), (r, res)
