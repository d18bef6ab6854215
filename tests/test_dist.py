"""Multi-rank host logic on CPU with gloo, world size 2: flop-balanced partition, per-rank
row blocks, rebase + allgatherv of C blocks, max-over-ranks timing.  The per-rank compute is
the oracle (CPU only here); the GPU data path is covered by the gpu tests."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, name, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import oracle
    import workloads as W
    from paper_conf_ipps_ramamoorthybsk15_b200 import dist as D

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        if name == "random":
            A = W.random_csr(300, 200, 0.03, 5)
            B = W.random_csr(200, 250, 0.03, 6)
        else:
            A, B = W.make(name)
        f = oracle.row_flops(A, B)
        s = oracle.split_points(f, world)
        rb, re = D.rank_rows(s, rank)
        rp, col, val, _ = oracle.spgemm(A, B, rb, re, with_abs=False)
        frp, fcol, fval = D.allgatherv_c(rp, col, val, s)
        t = D.max_over_ranks(float(rank + 1))
        # every rank's block carries about F/P products (+ one row)
        blk = int(f[rb:re].sum())
        ok_balance = blk * world <= f.sum() + world * int(f.max(initial=0))
        if rank == 0:
            ref = oracle.spgemm(A, B, with_abs=False)
            out_q.put((np.array_equal(frp, ref[0]), np.array_equal(fcol, ref[1]),
                       np.array_equal(fval, ref[2]), t, ok_balance))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["random", "cl10k"])
def test_gloo_partition_allgatherv(name):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, name, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    rp_ok, col_ok, val_ok, t, bal = q.get(timeout=10)
    assert rp_ok and col_ok and val_ok
    assert t == 2.0          # max over ranks of (rank + 1)
    assert bal


def test_rank_rows_cover():
    from paper_conf_ipps_ramamoorthybsk15_b200 import dist as D
    s = np.array([0, 3, 3, 10])
    assert [D.rank_rows(s, r) for r in range(3)] == [(0, 3), (3, 3), (3, 10)]
