#!/usr/bin/env python
"""Benchmark of the gSWORD hot path on B200 (BASELINE.json metric, configs[1]).

Workload (config.workload): the eu2005-shaped synthetic power-law graph of
BASELINE.json configs[1] (|V| = 862,664, |E| = 16,138,468, unlabelled; recipe in
DESIGN.md §7) and its dense random-walk-extracted 8-vertex query.  One STEP = one
pass of the whole hot path: WanderJoin over 1e8 samples, then
Alley over 1e8 samples (sample ids 0..1e8-1 per rank slice), each = queue reset +
persistent sampling kernel + grid reduction + the NCCL all_reduce of the 4-vector
(a 1-rank group at N = 1), inputs resident in HBM.

value  = samples of all ranks and both methods / max-over-ranks device time (CUDA
         events on the launching stream), L2 flushed (256 MB write) before every step.
e2e    = the same metric through the public API from host buffers: per step the host
         query arrays are loaded (H2D), each method is estimated and combined over the
         ranks (estimate_distributed: kernels + all_reduce + D2H of the result);
         e2e.first_call is the first such call, whose query load runs the autotune pilots.
per_method.cyclic: the same two methods on C1's cyclic query (4 non-tree edges), timed
         separately (not part of `value`).
roofline: algorithmic sectors of reading A26 (the oracle-pinned model)
         counted by the kernel's counting build over the launch, x 32 B / sampling-kernel
         time, against the measured HBM copy peak; dram_frac from ncu DRAM bytes;
         gather_frac against the random-gather rate (K5) measured live.
--impl reference: the CPU oracle (oracle/, plain C) on the host cores, a bounded sample
         of the same workload (the same sample count as cpu_baseline).

Usage: python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
       (N > 1: launched by torch.distributed.run, one rank per GPU, NCCL).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "samples/sec per B200 and 8-GPU box; q-error vs exact count; % gather roofline"
UNIT = "samples/s"
WORKLOAD = ("C1: eu2005-shaped Chung-Lu power-law graph, |V|=862664, |E|=16138468, unlabelled; "
            "dense 8-vertex random-walk query (seed 21); WanderJoin + Alley, 1e8 samples each per step")
# the paper's own numbers for this graph shape (context, not a like-for-like target)
PAPER_CONTEXT = {
    "wanderjoin_samples_per_s": 1.03e7, "alley_samples_per_s": 2.79e6,
    "gpu": "NVIDIA RTX 2080 Ti (Turing, sm_75)",
    "workload": "eu2005 (862,664 vertices, 16,138,468 edges, 40 random labels), 16-vertex queries, "
                "1e6 samples per query on the candidate graph",
    "cite": "PAPER.md P:L1085-L1086 (Tab. 2: 97 ms and 359 ms per query), P:L1055, P:L1061",
}
CPU_SAMPLES = 300_000  # oracle samples per method per step (cpu_baseline and --impl reference)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--samples", type=float, default=1e8, help="samples per method per rank per step")
    ap.add_argument("--query", choices=["dense", "sparse", "cyclic"], default="dense")
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-samples", type=int, default=CPU_SAMPLES,
                    help="oracle samples per method per step (cpu_baseline and --impl reference)")
    ap.add_argument("--traffic-file", default=os.path.join(ROOT, "profiles", "traffic_latest.json"))
    ap.add_argument("--quick", action="store_true", help="small config for smoke-testing the script")
    ap.add_argument("--no-qerror", action="store_true", help="skip the (untimed) C0 q-error leg")
    ap.add_argument("--no-cyclic", action="store_true", help="skip the cyclic-query leg")
    # test aids for the N > 1 path on a one-GPU box (not bench numbers): every rank on cuda:0,
    # gloo instead of NCCL (NCCL refuses two ranks on one device)
    ap.add_argument("--dist-backend", choices=["nccl", "gloo"], default="nccl", help=argparse.SUPPRESS)
    ap.add_argument("--same-device", action="store_true", help=argparse.SUPPRESS)
    return ap.parse_args()


# ---------------------------------------------------------------- clocks sampler
class ClockSampler:
    """SM clock + throttle reasons during the timed region (B200_PROFILING.md clocks rule).

    `device` is the CUDA ordinal; NVML numbers GPUs in PCI order and CUDA only the visible
    ones, so the NVML handle is resolved from the device's UUID (or PCI bus id) and
    nvidia-smi is given the same UUID."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int, uuid: str = None, pci_bus_id: str = None):
        self.index = device
        self.uuid = uuid
        self.pci_bus_id = pci_bus_id
        self.rows = []
        self._stop = threading.Event()
        self._t = None
        self.source = None

    @staticmethod
    def for_torch_device(device: int) -> "ClockSampler":
        uuid = bus = None
        try:
            import torch
            props = torch.cuda.get_device_properties(device)
            u = str(getattr(props, "uuid", "") or "")
            if u:
                uuid = u if u.startswith("GPU-") else "GPU-" + u
            bus = "%04x:%02x:%02x.0" % (getattr(props, "pci_domain_id", 0), props.pci_bus_id, props.pci_device_id)
        except Exception:
            pass
        return ClockSampler(device, uuid, bus)

    def _nvml_handle(self, pynvml):
        if self.uuid:
            try:
                return pynvml.nvmlDeviceGetHandleByUUID(self.uuid)
            except Exception:
                pass
        if self.pci_bus_id:
            try:
                return pynvml.nvmlDeviceGetHandleByPciBusId(self.pci_bus_id)
            except Exception:
                pass
        if os.environ.get("CUDA_VISIBLE_DEVICES"):
            raise RuntimeError("cannot map the CUDA device to NVML without its UUID")
        return pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def _run_nvml(self) -> bool:
        """NVML (nvidia_ml_py) reads take ~1 ms, so the region gets a sample every ~20 ms."""
        try:
            import pynvml
            pynvml.nvmlInit()
        except Exception:
            return False
        try:
            h = self._nvml_handle(pynvml)
            get_reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        except Exception:
            pynvml.nvmlShutdown()
            return False
        # NVML reason bits: sw_power_cap 0x4, hw_slowdown 0x8, sw_thermal 0x20, hw_thermal 0x40
        bits = (0x8, 0x40, 0x20, 0x4)
        got = 0
        while not self._stop.is_set():
            try:
                sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                r = int(get_reasons(h))
                self.rows.append([str(self.index), str(sm), str(mx), "", hex(r)] +
                                 ["Active" if r & b else "Not Active" for b in bits])
                got += 1
            except Exception:
                pass
            self._stop.wait(0.02)
        pynvml.nvmlShutdown()
        if got == 0:
            return False  # every read failed: let nvidia-smi try
        self.source = "nvml"
        return True

    def _run(self):
        if self._run_nvml():
            return
        self.source = "nvidia-smi"
        target = self.uuid or str(self.index)
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", target, f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.2)

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0,
                    "source": self.source}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nme in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(nme)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows), "source": self.source,
                "device_uuid": self.uuid}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def build_workload(args):
    from workloads import gen
    if args.quick:
        g = gen.chung_lu(50_000, 500_000, gamma=2.1, max_over_mean=500.0, seed=2005, name="quick")
        qs = [gen.extract_query(g, 8, seed=20, dense=False), gen.extract_query(g, 8, seed=21, dense=True),
              gen.extract_query(g, 8, seed=22, dense=True, min_non_tree=3)._renamed("cyclic")]
    else:
        g, qs = gen.config_c1()
    idx = {"sparse": 0, "dense": 1, "cyclic": 2}[args.query]
    return g, qs[idx], qs[2]


# ---------------------------------------------------------------- oracle timing (CPU)
def oracle_step(g, q, per_method: int, threads: int, seed: int) -> float:
    """One oracle step: WanderJoin then Alley over sample ids [0, per_method), `threads`
    host threads with dynamic chunking; candidate sets built once per call.
    Returns the wall time in seconds."""
    import oracle
    t0 = time.perf_counter()
    for m in (0, 1):
        oracle.sample_range(g, q, m, seed, 0, per_method, records=False, threads=threads)
    return time.perf_counter() - t0


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    g, q, _ = build_workload(args)
    cores = host_cores()
    per_method = args.cpu_samples
    times = []
    for i in range(args.warmup + args.steps):
        dt = oracle_step(g, q, per_method, cores, args.seed)
        if i >= args.warmup:
            times.append(dt)
    value = 2 * per_method * len(times) / sum(times)
    sample = (f"{per_method} WanderJoin + {per_method} Alley sample ids [0,{per_method}) per step, same "
              f"graph/query/seed as the GPU arm, {cores} threads ({cpu_model()})")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64 weights / i32 ids",
        "data": "synthetic", "config": {"workload": WORKLOAD, "samples_per_step": 2 * per_method,
                                        "query": q.name},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    emit(line)
    return 0


# ---------------------------------------------------------------- q-error
def star_count(g, s: int) -> int:
    """Embeddings of the star K_{1,s} in an unlabelled graph: sum_v deg(v)^(falling s)
    (the closed form pinned against brute force in tests/test_oracle_pins.py)."""
    import numpy as np
    deg = np.diff(g.row_ptr).astype(np.int64)
    tot = 0
    for dv in deg[deg >= s].tolist():
        f = 1
        for i in range(s):
            f *= dv - i
        tot += f
    return tot


def qerror_leg(G, ctx, args, g1=None, samples: int = 100_000_000):
    """q-error against the exact count where one exists: the C1 graph (the bench's, still
    loaded) with stars K_{1,3} and K_{1,4} (closed form), then BASELINE configs[0] (C0) with
    exact counts from tests/golden/c0_exact_counts.txt (written by the oracle's enumerator).
    Untimed; runs after the timed region on the same context."""
    from workloads import gen
    c1 = None
    if g1 is not None:
        c1 = {}
        for s in (3, 4):
            q = gen.star_query(s)
            truth = star_count(g1, s)
            ctx.load_query_obj(q)
            for m, key in ((G.WJ, "wj"), (G.ALLEY, "alley")):
                r = ctx.estimate(m, samples, args.seed)
                c1[f"star{s}_{key}"] = {"exact": truth, "estimate": r["estimate"],
                                        "qerror": G.qerror(truth, r["estimate"]),
                                        "rel_std_err": (r["variance"] ** 0.5) / r["estimate"] if r["estimate"] else None}
    path = os.path.join(ROOT, "tests", "golden", "c0_exact_counts.txt")
    exact = {}
    for line in open(path):
        if line.strip() and not line.startswith("#"):
            i, qname, c = line.split()
            exact[qname] = int(c)
    g, qs = gen.config_c0()
    ctx.load_graph_obj(g)
    out = {}
    for m, key in ((G.WJ, "wj"), (G.ALLEY, "alley")):
        errs = []
        for q in qs:
            ctx.load_query_obj(q)
            r = ctx.estimate(m, samples, args.seed)
            errs.append(G.qerror(exact[q.name], r["estimate"]))
        out[key] = {"median": statistics.median(errs), "max": max(errs)}
    return {"config": "C0 (BASELINE configs[0]): 11 four-vertex queries", "samples_per_query": samples,
            "exact_from": "tests/golden/c0_exact_counts.txt (oracle enumerator)", **out,
            "c1_stars": c1, "c1_exact_from": "closed form sum_v deg(v)^(falling s) (SURVEY P5)"}


# ---------------------------------------------------------------- our arm
def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_journals_pacmmod_yelsg24_b200 as G
    from paper_journals_pacmmod_yelsg24_b200.distributed import (allreduce_sum4, estimate_distributed,
                                                                  init_from_env, rank_range)

    # one process per GPU; a process group (NCCL) exists at every N, so the combine step
    # runs inside every timed step, a 1-rank all_reduce at N = 1
    if args.same_device:
        os.environ["LOCAL_RANK"] = "0"
    rank, world, local = init_from_env(args.dist_backend, single_rank_group=True)
    combine = dist.is_initialized()
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    n_per_rank = int(args.samples)
    n_total = n_per_rank * world  # weak scaling: fixed samples per GPU

    ctx = G.Context(local)
    stream = torch.cuda.Stream(dev)  # our kernels, the flush, the all_reduce and the events share it
    torch.cuda.set_stream(stream)
    ctx.set_stream(stream)
    if world == 1:
        g, q, qc = build_workload(args)
        t0 = time.perf_counter()
        ctx.load_graph_obj(g)
        graph_load_s = time.perf_counter() - t0
    else:
        # rank 0 builds G; the CSR is replicated over NCCL (NVLink) and loaded from device
        # memory on every rank; the queries travel as small objects
        from paper_journals_pacmmod_yelsg24_b200.distributed import broadcast_graph
        g, q, qc = build_workload(args) if rank == 0 else (None, None, None)
        t0 = time.perf_counter()
        if rank == 0:
            rp, cl, lb, nl = broadcast_graph(g.row_ptr, g.label_sorted_col(), g.labels, g.n_labels, device=dev)
        else:
            rp, cl, lb, nl = broadcast_graph(device=dev)
        obj = [q, qc]
        dist.broadcast_object_list(obj, src=0)
        q, qc = obj
        ctx.load_graph_device(rp, cl, lb if nl > 1 else None, nl)
        graph_load_s = time.perf_counter() - t0
    first, cnt = rank_range(n_total, rank, world)
    methods = (G.WJ, G.ALLEY)
    name = {G.WJ: "wj", G.ALLEY: "alley"}

    # ---- e2e through the public API, host buffers (the first call runs the autotune) ----
    def host_query(qq):
        qrp, qcol = qq.csr()
        return [np.ascontiguousarray(a) for a in (qrp, qcol, qq.labels, qq.order)]

    e2e_out4 = torch.zeros(4, dtype=torch.float64, device=dev)

    def e2e_call(h_q):
        h2d = ctx.load_query(*h_q)
        for m in methods:
            if combine:  # kernels + all_reduce on the stream + D2H of the combined 4-vector
                estimate_distributed(ctx, m, n_total, args.seed, out4=e2e_out4)
            else:
                ctx.estimate(m, cnt, args.seed, first=first)  # synchronous, host result (D2H)
        return h2d

    h_q = host_query(q)
    if combine:
        dist.barrier()
    torch.cuda.synchronize(dev)
    t0 = time.perf_counter()
    e2e_call(h_q)
    first_call_s = time.perf_counter() - t0

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    out4 = {m: torch.zeros(4, dtype=torch.float64, device=dev) for m in methods}

    def step():
        flush.fill_(1.0)  # evict L2 (126 MB) before the step
        ev = []
        for m in methods:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            ctx.estimate_async(m, first, cnt, args.seed, out4[m])
            if combine:
                allreduce_sum4(out4[m])
            e1.record(stream)
            ev.append((m, e0, e1))
        return ev

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize(dev)
    if combine:
        dist.barrier()
    torch.cuda.synchronize(dev)
    per_method_ms = {m: [] for m in methods}
    step_ms = []
    with ClockSampler.for_torch_device(local) as clocks:
        for _ in range(args.steps):
            ev = step()
            torch.cuda.synchronize(dev)
            tot = 0.0
            for m, e0, e1 in ev:
                dt = e0.elapsed_time(e1)
                per_method_ms[m].append(dt)
                tot += dt
            step_ms.append(tot)
    torch.cuda.synchronize(dev)
    results = {m: G.finalize(out4[m].cpu().numpy()) for m in methods}  # combined over the ranks

    local_time = sum(step_ms) / 1e3
    tt = torch.tensor([local_time], dtype=torch.float64, device=dev)
    if combine:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    max_time = float(tt.item())
    total_samples = n_total * len(methods) * args.steps
    value = total_samples / max_time

    # ---- e2e, cached calls ----
    e2e_times = []
    h2d = 0
    if combine:
        dist.barrier()
    for i in range(args.warmup + args.steps):
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        h2d = e2e_call(h_q)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            e2e_times.append(dt)
    et = torch.tensor([sum(e2e_times), first_call_s], dtype=torch.float64, device=dev)
    if combine:
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
    e2e_value = total_samples / float(et[0].item())
    e2e_first = n_total * len(methods) / float(et[1].item())

    # ---- untimed measurement legs (after the timed regions) ----
    def kernel_ms_of(m, qq_first, qq_cnt, reps=2):
        ks = []
        for _ in range(reps):
            ctx.estimate_async(m, qq_first, qq_cnt, args.seed, out4[m])
            ks.append(1e3 * ctx.last_kernel_seconds())
        return statistics.mean(ks)

    def sample_stats(m, n_first):
        """SURVEY §8(d) report over the first 1e6 sample ids (trace records): depth reached,
        valid fraction, algorithmic sectors (mean, p99)."""
        rec = ctx.trace_samples(m, first, n_first, args.seed)
        dr = rec["depth_reached"].astype(np.float64)
        sec = rec["sectors"].astype(np.float64)
        return {"samples": int(rec.shape[0]), "mean_depth_reached": float(dr.mean()),
                "p99_depth_reached": float(np.percentile(dr, 99)), "valid_fraction": float(rec["valid"].mean()),
                "sectors_mean": float(sec.mean()), "sectors_p99": float(np.percentile(sec, 99)),
                "sectors_max": float(sec.max())}

    kernel_ms = {m: kernel_ms_of(m, first, cnt) for m in methods}
    counts = {m: ctx.count_sectors(m, first, cnt, args.seed) for m in methods}  # (model, touched) sums
    stats = {m: sample_stats(m, min(cnt, 1_000_000)) for m in methods}
    qinfo = ctx.query_info()

    per_method = {}
    for m in methods:
        r = results[m]
        per_method[name[m]] = {
            "samples_per_s": n_total * args.steps / (sum(per_method_ms[m]) / 1e3),
            "kernel_ms": kernel_ms[m], "estimate": r["estimate"],
            "std_err": r["variance"] ** 0.5 if r["variance"] > 0 else 0.0,
            "valid_fraction": r["n_valid"] / r["n"],
            "alg_sectors_per_sample": counts[m][0] / cnt, "touched_sectors_per_sample": counts[m][1] / cnt,
            "kernel_alg_gbs": counts[m][0] * 32.0 / (kernel_ms[m] * 1e-3) / 1e9,
            "refill_min": qinfo["refill_min"][m], "ctas_per_sm": qinfo["occupancy"][m],
            "first_1e6": stats[m]}

    # ---- the cyclic query (>= 3 non-tree edges): Alley's intersections at work ----
    cyclic = None
    if not args.no_cyclic:
        ctx.load_query_obj(qc)  # autotune pilots for this query (untimed)
        n_cyc_count = min(cnt, 10_000_000)
        cyc = {}
        for m in methods:
            for _ in range(max(1, args.warmup)):
                ctx.estimate_async(m, first, cnt, args.seed, out4[m])
            ms = []
            for _ in range(args.steps):
                flush.fill_(1.0)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                ctx.estimate_async(m, first, cnt, args.seed, out4[m])
                e1.record(stream)
                torch.cuda.synchronize(dev)
                ms.append(e0.elapsed_time(e1))
            r = G.finalize(out4[m].cpu().numpy())
            kms = kernel_ms_of(m, first, cnt)
            mod, tch = ctx.count_sectors(m, first, n_cyc_count, args.seed)
            cyc[name[m]] = {
                "samples_per_s": cnt / (statistics.mean(ms) / 1e3), "kernel_ms": kms, "estimate": r["estimate"],
                "std_err": r["variance"] ** 0.5 if r["variance"] > 0 else 0.0,
                "valid_fraction": r["n_valid"] / r["n"],
                "alg_sectors_per_sample": mod / n_cyc_count, "touched_sectors_per_sample": tch / n_cyc_count,
                "sectors_counted_over": n_cyc_count,
                "kernel_alg_gbs": mod / n_cyc_count * cnt * 32.0 / (kms * 1e-3) / 1e9,
                "first_1e6": sample_stats(m, min(cnt, 1_000_000))}
        cyclic = {"query": qc.name, "query_edges": len(qc.edges()), "non_tree_edges": len(qc.edges()) - (qc.nq - 1),
                  "samples_per_method": n_total, "note": "rank-local device time, L2 flushed per launch; "
                  "not part of value", **cyc}
        ctx.load_query_obj(q)

    if rank != 0:
        ctx.close()
        if combine:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    # ---- roofline of the dominant kernel (reading A26 model, oracle-pinned) ----
    dom = max(methods, key=lambda m: kernel_ms[m])
    dom_s = kernel_ms[dom] * 1e-3
    alg_bytes = counts[dom][0] * 32.0
    achieved = alg_bytes / dom_s / 1e9
    peak, peak_kind = measured_peaks()
    traffic = None
    ncu_counters = None
    try:
        with open(args.traffic_file) as f:
            tf = json.load(f)
        if tf.get("workload") == WORKLOAD and name[dom] in tf.get("dram_bytes_per_sample", {}):
            # ncu --set full capture (cold cache, serialised) scaled to this launch's samples
            traffic = float(tf["dram_bytes_per_sample"][name[dom]]) * cnt
            ncu_counters = dict(tf.get("counters", {}), source=tf.get("source"))
    except Exception:
        traffic = None
    # K5 random-gather rates of this device, measured now
    gather = {"l2_resident_64MB": ctx.gather_roofline(64 << 20, 4),
              "col_size": ctx.gather_roofline(max(4096, int(g.col.shape[0]) * 4 if g is not None else 1 << 27), 4),
              "hbm_2GB": ctx.gather_roofline(2 << 30, 4)}
    sec_rate = counts[dom][0] / dom_s
    roofline = {
        "bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
        "traffic": traffic, "kernel": f"sample_kernel<{name[dom]}>", "peak_kind": peak_kind,
        "alg_sectors_per_launch": counts[dom][0], "samples_per_launch": cnt, "kernel_ms": kernel_ms[dom],
        "dram_gbs": traffic / dom_s / 1e9 if traffic else None,
        "dram_frac": traffic / dom_s / 1e9 / peak if traffic else None,
        "gather_sectors_per_s": gather, "alg_sectors_per_s": sec_rate,
        "gather_frac": sec_rate / gather["l2_resident_64MB"], "gather_frac_hbm": sec_rate / gather["hbm_2GB"],
        # against uniform random gathers over a buffer the size of `col` (the graph's adjacency)
        "gather_frac_col": sec_rate / gather["col_size"],
        "ncu_counters": ncu_counters,
        "model": "reading A26 (DESIGN.md §3): offsets + drawn/selected vertices + Alley driver scans at "
                 "|B(d)|>=2 + one sector per membership question; counted by the kernel's counting build "
                 "over this launch, equal to the oracle's count (tests/test_gpu_sectors.py)",
    }

    cpu_base = None
    if world == 1 and not args.no_cpu_baseline:
        cores = host_cores()
        per = args.cpu_samples
        dt = oracle_step(g, q, per, cores, args.seed)
        per1 = max(1000, per // 20)
        dt1 = oracle_step(g, q, per1, 1, args.seed)
        cpu_base = {"value": 2 * per / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
                    "sample": f"{per} WanderJoin + {per} Alley samples (ids [0,{per})), same graph/query/seed, "
                              f"{dt:.1f} s on {cores} threads ({cpu_model()}); the same sample as --impl reference",
                    # SURVEY §8(d) oracle timing (i): the same oracle on one thread
                    "single_thread": {"value": 2 * per1 / dt1, "cores": 1,
                                      "sample": f"{per1} + {per1} samples, {dt1:.1f} s"}}

    info = ctx.launch_info()
    qerr = qerror_leg(G, ctx, args, g1=g) if not (args.quick or args.no_qerror) else None
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * max_time / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64 weights / i32 ids", "data": "synthetic",
        "config": {"workload": WORKLOAD if not args.quick else "quick (not a bench number)",
                   "samples_per_method_per_gpu": n_per_rank, "methods": ["wanderjoin", "alley"],
                   "query": q.name, "query_edges": len(q.edges()), "seed": args.seed,
                   "l2": "flushed before every step (256 MB write)", "parallelism": f"sample-range split x{world}",
                   "combine": "NCCL all_reduce of 4 fp64 per method inside the step" if combine else "none",
                   "grid": info["grid"], "threads": info["threads"]},
        "per_method": {**per_method, "cyclic": cyclic},
        "roofline": roofline,
        "paper_context": PAPER_CONTEXT,
        "cpu_baseline": cpu_base,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": 32 * len(methods), "graph_load_s": graph_load_s,
                "first_call": {"value": e2e_first, "unit": UNIT, "seconds": float(et[1].item()),
                               "note": "the first load_query of the query (refill-threshold and occupancy "
                                       "autotune pilots) + one estimate per method"},
                "note": "per step: gsword_load_query from host arrays (cached autotune) + per method the "
                        "estimate, the all_reduce over the ranks and the D2H of the result; graph loaded "
                        "once (P:L1057 excludes it)"},
        "qerror": qerr,
        # our kernels in the timed region: sampling kernel + grid reduction per method and step
        # (the all_reduce is NCCL's kernel, the L2 flush torch's fill)
        "gpu_launches": 2 * len(methods) * args.steps,
        "clocks": clocks.summary(),
    }
    emit(line)
    ctx.close()
    if combine:
        dist.barrier()
        dist.destroy_process_group()
    return 0


_JSON_FD = None  # the process's original stdout, kept for the one JSON line


def reserve_stdout():
    """stdout carries exactly one JSON line (the driver's contract).  Native libraries write
    banners to file descriptor 1 directly — NCCL prints "NCCL version ..." at communicator
    init when NCCL_DEBUG=VERSION, which the GPU boxes set — so fd 1 is pointed at stderr for
    the whole run and the JSON line is written to a duplicate of the original stdout."""
    global _JSON_FD
    try:
        sys.stdout.flush()
        fd = os.dup(1)
        os.dup2(2, 1)
        _JSON_FD = fd
    except OSError:
        _JSON_FD = None


def emit(line) -> None:
    text = json.dumps(line) + "\n"
    if _JSON_FD is None:
        sys.stdout.write(text)
        sys.stdout.flush()
    else:
        os.write(_JSON_FD, text.encode())


def main():
    args = parse()
    reserve_stdout()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
