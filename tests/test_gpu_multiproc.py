"""The multi-GPU layer (north_star (4)) executed on the single-GPU lease.

* Two processes share cuda:0, each runs the sampling + reduction kernels on its
  rank_range slice of the sample ids (estimate_async), and the kernels' 4-vectors are
  combined with one gloo all_reduce (NCCL refuses two ranks on one device).  The result
  must equal a one-process run of the whole range: n and n_valid exactly, sum and sumsq
  within 1e-12 (BASELINE.json north_star).
* estimate_distributed under a 1-rank NCCL process group (init_from_env with
  single_rank_group, as bench.py runs at N = 1): the NCCL all_reduce call site runs on the
  launch stream and returns the single-range result.
"""
import os
import socket

import pytest

pytestmark = pytest.mark.gpu

REL = 1e-12


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _slice_worker(rank, world, port, n_total, seed, qi, out_q):
    import torch
    import torch.distributed as dist

    import paper_journals_pacmmod_yelsg24_b200 as G
    from paper_journals_pacmmod_yelsg24_b200.distributed import allreduce_sum4, rank_range
    from workloads import gen

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g, qs = gen.config_c0()
    res = []
    with G.Context(0) as ctx:
        stream = torch.cuda.Stream(0)
        ctx.set_stream(stream)
        ctx.load_graph_obj(g)
        ctx.load_query_obj(qs[qi])
        first, cnt = rank_range(n_total, rank, world)
        for m in (G.WJ, G.ALLEY):
            out = torch.zeros(4, dtype=torch.float64, device="cuda:0")
            ctx.estimate_async(m, first, cnt, seed, out)
            stream.synchronize()
            t = out.cpu()
            allreduce_sum4(t)  # the combine of the kernels' partials
            res.append(t.tolist())
    out_q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


def _nccl_worker(n_total, seed, out_q):
    import torch
    import torch.distributed as dist

    import paper_journals_pacmmod_yelsg24_b200 as G
    from paper_journals_pacmmod_yelsg24_b200.distributed import estimate_distributed, init_from_env
    from workloads import gen

    for k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_PORT"):
        os.environ.pop(k, None)
    init_from_env("nccl", single_rank_group=True)
    backend = dist.get_backend() if dist.is_initialized() else None
    g, qs = gen.config_c0()
    res = []
    with G.Context(0) as ctx:
        torch.cuda.set_stream(torch.cuda.Stream(0))
        ctx.load_graph_obj(g)
        ctx.load_query_obj(qs[3])
        for m in (G.WJ, G.ALLEY):
            d = estimate_distributed(ctx, m, n_total, seed)
            s = ctx.estimate(m, n_total, seed)
            res.append((d, s))
    out_q.put((backend, res))
    if dist.is_initialized():
        dist.destroy_process_group()


def _spawn(target, args, n):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=target, args=(*(a(r) if callable(a) else a for a in args), q)) for r in range(n)]
    for p in procs:
        p.start()
    out = [q.get(timeout=600) for _ in range(n)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    return out


def test_two_processes_share_the_gpu_and_combine_kernel_partials():
    import paper_journals_pacmmod_yelsg24_b200 as G
    from workloads import gen

    world, n_total, seed, qi = 2, 3_000_001, 23, 2
    port = _free_port()
    out = _spawn(_slice_worker, (lambda r: r, world, port, n_total, seed, qi), world)
    combined = {rank: res for rank, res in out}
    assert combined[0] == combined[1]  # every rank holds the same combined vector
    g, qs = gen.config_c0()
    with G.Context(0) as ctx:
        ctx.load_graph_obj(g)
        ctx.load_query_obj(qs[qi])
        for i, m in enumerate((G.WJ, G.ALLEY)):
            full = ctx.estimate(m, n_total, seed)
            s, sq, nv, n = combined[0][i]
            assert n == n_total == full["n"] and nv == full["n_valid"]
            assert s == pytest.approx(full["sum"], rel=REL, abs=0.0)
            assert sq == pytest.approx(full["sumsq"], rel=REL, abs=0.0)


def test_estimate_distributed_under_a_one_rank_nccl_group():
    (backend, res), = _spawn(_nccl_worker, (2_000_000, 31), 1)
    assert backend == "nccl"
    for d, s in res:
        assert d["n"] == s["n"] and d["n_valid"] == s["n_valid"]
        assert d["sum"] == pytest.approx(s["sum"], rel=REL, abs=0.0)
        assert d["sumsq"] == pytest.approx(s["sumsq"], rel=REL, abs=0.0)


def _bench_line(args, nproc, torchrun=False):
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    common = ["bench.py", "--quick", "--steps", "2", "--warmup", "1", "--no-qerror", "--no-cpu-baseline",
              "--no-cyclic"] + args
    if nproc == 1 and not torchrun:
        cmd = [sys.executable] + common
    else:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
               "--master-addr", "127.0.0.1", "--master-port", str(_free_port())] + common + ["--gpus", str(nproc)]
    out = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    # stdout is the one JSON line and nothing else (native banners such as NCCL's version line
    # under NCCL_DEBUG=VERSION go to stderr)
    lines = [ln for ln in out.stdout.splitlines() if ln.strip()]
    assert len(lines) == 1 and lines[0].startswith("{"), out.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_two_ranks_on_one_gpu_matches_one_rank():
    """bench.py's N > 1 path (graph broadcast over the process group, device-side graph load,
    rank_range split, the all_reduce inside the timed step and inside e2e, max-over-ranks
    timing) run as 2 ranks sharing cuda:0 over gloo: the combined estimates equal a one-rank
    run over the same 4e6 sample ids."""
    two = _bench_line(["--samples", "2e6", "--dist-backend", "gloo", "--same-device"], 2)
    one = _bench_line(["--samples", "4e6"], 1)
    assert two["n_gpus"] == 2 and one["n_gpus"] == 1 and two["value"] > 0 and two["e2e"]["value"] > 0
    for m in ("wj", "alley"):
        a, b = two["per_method"][m], one["per_method"][m]
        assert a["valid_fraction"] == b["valid_fraction"]
        assert a["estimate"] == pytest.approx(b["estimate"], rel=REL, abs=0.0)


def test_bench_under_torchrun_with_one_rank():
    """The driver's N = 1 launch form (torch.distributed.run, one rank): bench.py joins the
    launcher's store with a 1-rank NCCL group, runs the all_reduce in the step, and prints
    one line equal to the plain run's estimates; the reference arm prints its line too."""
    tr = _bench_line(["--samples", "2e6"], 1, torchrun=True)
    plain = _bench_line(["--samples", "2e6"], 1)
    assert tr["n_gpus"] == 1 and "NCCL" in tr["config"]["combine"]
    for m in ("wj", "alley"):
        assert tr["per_method"][m]["estimate"] == pytest.approx(plain["per_method"][m]["estimate"], rel=REL, abs=0.0)
    ref = _bench_line(["--impl", "reference", "--cpu-samples", "2000"], 1, torchrun=True)
    assert ref["impl"] == "reference" and ref["value"] > 0
