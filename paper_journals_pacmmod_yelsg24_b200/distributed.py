"""Multi-GPU layer (BASELINE.json north_star (4)).

G is replicated on every rank (each rank loads the same canonical CSR), the global
sample-id range is split contiguously, each rank runs the sampling +
reduction kernels on its slice, and ONE all_reduce(SUM) of the 4 fp64 values
{sum, sumsq, n_valid, n} combines them.  Counter-based Philox makes the union of the
slices bit-identical, sample by sample, to a single-GPU run of the whole range.
"""
from __future__ import annotations

from typing import Dict, Optional, Tuple

from .gsword import Context, finalize


def rank_range(n_total: int, rank: int, world: int, first: int = 0) -> Tuple[int, int]:
    """Rank r of P takes [first + floor(r n / P), first + floor((r+1) n / P)).
    Returns (first_sample_id, count)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    a = (n_total * rank) // world
    b = (n_total * (rank + 1)) // world
    return first + a, b - a


def allreduce_sum4(t4, group=None):
    """The one collective of the path: SUM over ranks of the 4-vector (in place)."""
    import torch.distributed as dist
    dist.all_reduce(t4, op=dist.ReduceOp.SUM, group=group)
    return t4


def estimate_distributed(ctx: Context, method: int, n_total: int, seed: int, first: int = 0, group=None,
                         out4=None) -> Dict[str, float]:
    """Every rank calls this with the same arguments; every rank gets the combined
    result.  The kernels and the NCCL all_reduce run on torch's current stream, so no
    host synchronisation sits between them."""
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group) if dist.is_initialized() else 0
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    f, cnt = rank_range(n_total, rank, world, first)
    dev = torch.device("cuda", ctx.device)
    stream = torch.cuda.current_stream(dev)
    ctx.set_stream(stream)
    if out4 is None:
        out4 = torch.zeros(4, dtype=torch.float64, device=dev)
    else:
        out4.zero_()
    if cnt > 0:
        ctx.estimate_async(method, f, cnt, seed, out4)
    if dist.is_initialized():  # the combine runs whenever a group exists (a no-op sum at world 1)
        allreduce_sum4(out4, group)
    return finalize(out4.cpu().numpy())


def broadcast_graph(row_ptr=None, col=None, labels=None, n_labels: int = 1, device=None, src: int = 0, group=None):
    """Replicate the graph from rank `src` to every rank over the process group (NCCL over
    NVLink for CUDA tensors; gloo for CPU tensors).  Rank src passes numpy/torch arrays
    (col sorted by (label, id) per row); the others pass None.  Returns (row_ptr, col,
    labels, n_labels) as tensors on `device`, ready for Context.load_graph_device."""
    import numpy as np
    import torch
    import torch.distributed as dist

    rank = dist.get_rank(group)
    hdr = torch.zeros(3, dtype=torch.int64, device=device)
    if rank == src:
        hdr[0] = int(len(row_ptr) - 1)
        hdr[1] = int(len(col))
        hdr[2] = int(n_labels)
    dist.broadcast(hdr, src, group=group)
    n, nnz, nl = (int(x) for x in hdr.tolist())
    if rank == src:
        rp = torch.as_tensor(np.ascontiguousarray(row_ptr, np.int64)).to(device)
        cl = torch.as_tensor(np.ascontiguousarray(col, np.int32)).to(device)
        lb = torch.as_tensor(np.ascontiguousarray(labels if labels is not None else np.zeros(n, np.int32),
                                                  np.int32)).to(device)
    else:
        rp = torch.empty(n + 1, dtype=torch.int64, device=device)
        cl = torch.empty(nnz, dtype=torch.int32, device=device)
        lb = torch.empty(n, dtype=torch.int32, device=device)
    for t in (rp, cl, lb):
        dist.broadcast(t, src, group=group)
    return rp, cl, lb, nl


def combine_host(values4_per_rank) -> Dict[str, float]:
    """Host-side equivalent of the all_reduce + finalize (for checkpoint/resume of
    partial ranges): element-wise sum of {sum, sumsq, n_valid, n} then finalize."""
    import numpy as np
    acc = np.zeros(4, np.float64)
    for v in values4_per_rank:
        acc += np.asarray(v, np.float64).reshape(4)
    return finalize(acc)


def init_from_env(backend: Optional[str] = None, single_rank_group: bool = False):
    """torchrun plumbing: init the process group from RANK/WORLD_SIZE/MASTER_* and bind
    LOCAL_RANK's GPU.  With single_rank_group, a 1-rank group is created at world size 1
    too (MASTER_ADDR 127.0.0.1 and a free port unless set), so the combine step of the path
    runs at every N; if that group cannot be created the caller proceeds without one.
    Returns (rank, world, local_rank)."""
    import os
    import socket

    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if backend is None:
        backend = "nccl" if torch.cuda.is_available() else "gloo"
    if backend == "nccl" or torch.cuda.is_available():
        torch.cuda.set_device(local)
    if dist.is_initialized():
        return rank, world, local
    if world > 1:
        if backend == "nccl":
            dist.init_process_group(backend, device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    elif single_rank_group:
        if "MASTER_PORT" not in os.environ:
            with socket.socket() as s:
                s.bind(("127.0.0.1", 0))
                os.environ["MASTER_PORT"] = str(s.getsockname()[1])
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        try:
            kw = {"device_id": torch.device("cuda", local)} if backend == "nccl" else {}
            dist.init_process_group(backend, rank=0, world_size=1, **kw)
        except Exception:  # no group: the 4-vector needs no combining at world size 1
            pass
    return rank, world, local
