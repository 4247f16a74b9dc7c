"""Multi-process (world_size 2, gloo, CPU) checks of the multi-GPU layer's host logic:
the contiguous sample-id split and the single SUM all_reduce of
{sum, sumsq, n_valid, n} reproduce the single-range aggregate.  Per-rank partials
come from the oracle here (test infrastructure); on GPUs they come from the kernels
(tests/test_gpu_parity.py covers split-range invariance on the device)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_journals_pacmmod_yelsg24_b200.distributed import allreduce_sum4, combine_host, rank_range
from paper_journals_pacmmod_yelsg24_b200 import finalize


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, n_total, seed, q):
    import oracle
    from workloads import gen
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g, qs = gen.config_c0()
    first, cnt = rank_range(n_total, rank, world, first=1000)
    y, _ = oracle.sample_range(g, qs[2], 1, seed, first, cnt, records=False)
    agg = oracle.aggregate(y)
    t = torch.tensor([agg["sum"], agg["sumsq"], agg["n_valid"], agg["n"]], dtype=torch.float64)
    allreduce_sum4(t)
    q.put((rank, t.numpy().tolist()))
    dist.destroy_process_group()


def test_rank_range_partition():
    for n in (0, 1, 7, 100, 10**10 + 3):
        for P in (1, 2, 3, 8):
            parts = [rank_range(n, r, P, first=5) for r in range(P)]
            assert parts[0][0] == 5
            for (f0, c0), (f1, _) in zip(parts, parts[1:]):
                assert f0 + c0 == f1
            assert sum(c for _, c in parts) == n
            assert max(c for _, c in parts) - min(c for _, c in parts) <= 1


def test_gloo_two_ranks_combine():
    import oracle
    from workloads import gen
    world, n_total, seed = 2, 40_001, 17
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_total, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0] == res[1]
    combined = finalize(res[0])
    g, qs = gen.config_c0()
    y, _ = oracle.sample_range(g, qs[2], 1, seed, 1000, n_total, records=False)
    ref = oracle.aggregate(y)
    assert combined["n"] == n_total and combined["n_valid"] == ref["n_valid"]
    assert combined["sum"] == pytest.approx(ref["sum"], rel=1e-12)
    assert combined["sumsq"] == pytest.approx(ref["sumsq"], rel=1e-12)
    host = combine_host([[ref["sum"], ref["sumsq"], ref["n_valid"], ref["n"]]])
    assert host["estimate"] == pytest.approx(ref["estimate"], rel=1e-15)


def _bcast_worker(rank, world, port, q):
    from paper_journals_pacmmod_yelsg24_b200.distributed import broadcast_graph
    from workloads import gen
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    if rank == 0:
        g, _ = gen.config_c0()
        out = broadcast_graph(g.row_ptr, g.label_sorted_col(), g.labels, g.n_labels, device="cpu")
    else:
        out = broadcast_graph(device="cpu")
    rp, cl, lb, nl = out
    q.put((rank, rp.numpy().tolist()[:50], int(cl.sum()), int(lb.sum()), nl, int(cl.numel())))
    dist.destroy_process_group()


def test_gloo_broadcast_graph():
    from workloads import gen
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_bcast_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict((r[0], r[1:]) for r in (q.get(timeout=300) for _ in range(2)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res[0] == res[1]
    g, _ = gen.config_c0()
    assert res[0][0] == g.row_ptr.tolist()[:50] and res[0][4] == g.col.shape[0] and res[0][3] == 4


def test_label_sorted_col():
    from workloads import gen
    g = gen.random_small_graph(20, 0.4, 3, seed=1)
    c = g.label_sorted_col()
    for v in range(g.n):
        row = c[g.row_ptr[v]:g.row_ptr[v + 1]]
        keys = list(zip(g.labels[row].tolist(), row.tolist()))
        assert keys == sorted(keys) and sorted(row.tolist()) == g.neighbors(v).tolist()
