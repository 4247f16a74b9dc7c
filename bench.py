#!/usr/bin/env python
"""Benchmark of the gSWORD hot path on B200 (BASELINE.json metric, configs[1]).

Workload (config.workload): the eu2005-shaped synthetic power-law graph of
BASELINE.json configs[1] (|V| = 862,664, |E| = 16,138,468, unlabelled; recipe in
DESIGN.md §7) and its dense random-walk-extracted 8-vertex query.  One STEP = one
pass of the whole hot path: WanderJoin over 1e8 samples, then Alley over 1e8
samples (sample ids 0..1e8-1 per rank slice), each = queue reset + persistent
sampling kernel + grid reduction, inputs resident in HBM.

value  = samples of all ranks and both methods / max-over-ranks device time (CUDA
         events on the launching stream), L2 flushed (256 MB write) before every step.
e2e    = the same metric through the public API from host buffers: per step the host
         query arrays are loaded (H2D) and gsword_estimate returns its host result (D2H).
--impl reference: the CPU oracle (oracle/, plain C) on the host cores, bounded sample.

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


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--samples", type=float, default=1e8, help="samples per method per rank per step")
    ap.add_argument("--query", choices=["dense", "sparse"], default="dense")
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="budget of the oracle timing")
    ap.add_argument("--traffic-file", default=os.path.join(ROOT, "profiles", "traffic_latest.json"))
    ap.add_argument("--quick", action="store_true", help="small config for smoke-testing the script")
    ap.add_argument("--no-qerror", action="store_true", help="skip the (untimed) C0 q-error leg")
    return ap.parse_args()


# ---------------------------------------------------------------- clocks sampler
class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region (B200_PROFILING.md)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None
        self.source = None

    def _run_nvml(self) -> bool:
        """NVML (nvidia_ml_py) reads take ~1 ms, so the region gets a sample every ~20 ms."""
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            get_reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        except Exception:
            return False
        # NVML reason bits: sw_power_cap 0x4, hw_slowdown 0x8, sw_thermal 0x20, hw_thermal 0x40
        bits = (0x8, 0x40, 0x20, 0x4)
        while not self._stop.is_set():
            try:
                sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                r = int(get_reasons(h))
                self.rows.append([str(self.index), str(sm), str(mx), "", hex(r)] +
                                 ["Active" if r & b else "Not Active" for b in bits])
            except Exception:
                pass
            self._stop.wait(0.02)
        self.source = "nvml"
        return True

    def _run(self):
        if self._run_nvml():
            return
        self.source = "nvidia-smi"
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
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
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nme in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(nme)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows), "source": self.source}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


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
        qs = [gen.extract_query(g, 8, seed=20, dense=False), gen.extract_query(g, 8, seed=21, dense=True)]
    else:
        g, qs = gen.config_c1()
    q = qs[1] if args.query == "dense" else qs[0]
    return g, q


# ---------------------------------------------------------------- oracle timing (CPU)
def oracle_rate(g, q, seconds: float, threads: int, seed: int):
    """Times the oracle as it stands on `threads` host threads over a bounded sample
    (both methods, equal counts) sized to about `seconds`.  Returns (samples/s, n, dt)."""
    import oracle
    probe = 4000
    t0 = time.perf_counter()
    for m in (0, 1):
        oracle.sample_range(g, q, m, seed, 0, probe, records=False, threads=threads)
    dt = time.perf_counter() - t0
    per_method = max(probe, int(seconds / max(dt, 1e-6) * probe / 2) // 1000 * 1000)
    t0 = time.perf_counter()
    for m in (0, 1):
        oracle.sample_range(g, q, m, seed, 0, per_method, records=False, threads=threads)
    dt = time.perf_counter() - t0
    return 2 * per_method / dt, per_method, dt


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    g, q = build_workload(args)
    cores = host_cores()
    times = []
    per_method = None
    for i in range(args.warmup + args.steps):
        budget = args.cpu_seconds if per_method is None else None
        if per_method is None:
            rate, per_method, dt = oracle_rate(g, q, budget / max(1, args.steps), cores, args.seed)
        else:
            import oracle
            t0 = time.perf_counter()
            for m in (0, 1):
                oracle.sample_range(g, q, m, args.seed, 0, per_method, records=False, threads=cores)
            dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    value = 2 * per_method * len(times) / sum(times)
    sample = f"{per_method} WanderJoin + {per_method} Alley sample ids [0,{per_method}) per step, same graph/query"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": {"workload": WORKLOAD, "samples_per_step": 2 * per_method},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                         "cpu": cpu_model()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------- q-error
def qerror_leg(G, ctx, args, samples: int = 100_000_000):
    """q-error against the exact count where one exists: BASELINE configs[0] (C0), exact
    counts from tests/golden/c0_exact_counts.txt (written by the oracle's enumerator).
    Untimed; runs after the timed region on the same context."""
    from workloads import gen
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
            "exact_from": "tests/golden/c0_exact_counts.txt (oracle enumerator)", **out}


# ---------------------------------------------------------------- our arm
def run_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_journals_pacmmod_yelsg24_b200 as G
    from paper_journals_pacmmod_yelsg24_b200.distributed import allreduce_sum4, init_from_env, rank_range

    rank, world, local = init_from_env("nccl")
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    n_per_rank = int(args.samples)
    n_total = n_per_rank * world  # weak scaling: fixed samples per GPU

    ctx = G.Context(local)
    stream = torch.cuda.Stream(dev)  # our kernels, the flush and the events share this stream
    torch.cuda.set_stream(stream)
    ctx.set_stream(stream)
    if world == 1:
        g, q = build_workload(args)
        t0 = time.perf_counter()
        ctx.load_graph_obj(g)
        graph_load_s = time.perf_counter() - t0
    else:
        # rank 0 builds G; the CSR is replicated over NCCL (NVLink) and loaded from device
        # memory on every rank; the query travels as a small object
        from paper_journals_pacmmod_yelsg24_b200.distributed import broadcast_graph
        g, q = build_workload(args) if rank == 0 else (None, None)
        t0 = time.perf_counter()
        if rank == 0:
            rp, cl, lb, nl = broadcast_graph(g.row_ptr, g.label_sorted_col(), g.labels, g.n_labels, device=dev)
        else:
            rp, cl, lb, nl = broadcast_graph(device=dev)
        obj = [q]
        dist.broadcast_object_list(obj, src=0)
        q = obj[0]
        ctx.load_graph_device(rp, cl, lb if nl > 1 else None, nl)
        graph_load_s = time.perf_counter() - t0
    ctx.load_query_obj(q)
    first, cnt = rank_range(n_total, rank, world)
    methods = (G.WJ, G.ALLEY)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    out4 = {m: torch.zeros(4, dtype=torch.float64, device=dev) for m in methods}

    def step(timed: bool):
        flush.fill_(1.0)  # evict L2 (126 MB) before the step
        ev = []
        for m in methods:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            ctx.estimate_async(m, first, cnt, args.seed, out4[m])
            e1.record(stream)
            ev.append((m, e0, e1))
        return ev

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize(dev)

    # algorithmic sectors per launch (counting build, untimed), SURVEY §8(d)
    sectors = {m: ctx.count_sectors(m, first, cnt, args.seed) for m in methods}
    # sample statistics over the first 1e6 sample ids: depth reached, valid
    # fraction (per-sample trace records, untimed)
    depth_stats = {}
    for m in methods:
        rec = ctx.trace_samples(m, first, min(cnt, 1_000_000), args.seed)
        dr = rec["depth_reached"].astype(np.float64)
        depth_stats[m] = {"samples": int(rec.shape[0]), "mean_depth_reached": float(dr.mean()),
                          "p99_depth_reached": float(np.percentile(dr, 99)),
                          "valid_fraction": float(rec["valid"].mean())}

    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    per_method_ms = {m: [] for m in methods}
    kernel_ms = {m: [] for m in methods}
    step_ms = []
    with ClockSampler(local) as clocks:
        for _ in range(args.steps):
            ev = step(True)
            torch.cuda.synchronize(dev)
            tot = 0.0
            for m, e0, e1 in ev:
                dt = e0.elapsed_time(e1)
                per_method_ms[m].append(dt)
                tot += dt
            # sampling-kernel-only time of the last method is exposed by the library;
            # re-derive per method from a dedicated launch below
            step_ms.append(tot)
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    # dominant-kernel duration: events around the sampling kernel alone (library-internal)
    for m in methods:
        for _ in range(2):
            ctx.estimate_async(m, first, cnt, args.seed, out4[m])
            kernel_ms[m].append(1e3 * ctx.last_kernel_seconds())
    results = {}
    for m in methods:
        t = out4[m].clone()
        if world > 1:
            allreduce_sum4(t)
        results[m] = G.finalize(t.cpu().numpy())

    local_time = sum(step_ms) / 1e3
    tt = torch.tensor([local_time], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    max_time = float(tt.item())
    total_samples = n_total * len(methods) * args.steps
    value = total_samples / max_time

    # ---- e2e through the public API, host buffers ----
    qrp, qcol = q.csr()
    h_q = [np.ascontiguousarray(a) for a in (qrp, qcol, q.labels, q.order)]
    e2e_times = []
    h2d = 0
    ctx_e2e = ctx
    if world > 1:
        dist.barrier()
    for i in range(args.warmup + args.steps):
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        h2d = ctx_e2e.load_query(*h_q)
        for m in methods:
            ctx_e2e.estimate(m, cnt, args.seed, first=first)  # synchronous, host result (D2H)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            e2e_times.append(dt)
    et = torch.tensor([sum(e2e_times)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
    e2e_value = total_samples / float(et.item())

    if rank != 0:
        ctx.close()
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return 0

    # ---- roofline of the dominant kernel ----
    dom = max(methods, key=lambda m: sum(kernel_ms[m]))
    dom_ms = statistics.mean(kernel_ms[dom])
    alg_bytes = sectors[dom] * 32.0
    achieved = alg_bytes / (dom_ms * 1e-3) / 1e9
    peak, peak_kind = measured_peaks()
    traffic = None
    try:
        with open(args.traffic_file) as f:
            tf = json.load(f)
        key = "wj" if dom == G.WJ else "alley"
        if tf.get("workload") == WORKLOAD and key in tf.get("dram_bytes_per_sample", {}):
            # ncu capture (cold cache, serialised) scaled to this launch's samples
            traffic = float(tf["dram_bytes_per_sample"][key]) * cnt
    except Exception:
        traffic = None

    cpu_base = None
    if world == 1 and not args.no_cpu_baseline:
        cores = host_cores()
        rate, per_method, dt = oracle_rate(g, q, args.cpu_seconds, cores, args.seed)
        rate1, per1, dt1 = oracle_rate(g, q, min(5.0, args.cpu_seconds / 3), 1, args.seed)
        cpu_base = {"value": rate, "unit": UNIT, "cores": cores, "kind": "oracle",
                    "sample": f"{per_method} WanderJoin + {per_method} Alley samples (ids [0,{per_method})), "
                              f"same graph/query/seed, {dt:.1f} s on {cores} threads ({cpu_model()})",
                    # SURVEY §8(d) oracle timing (i): the same oracle on one thread
                    "single_thread": {"value": rate1, "cores": 1,
                                      "sample": f"{per1} + {per1} samples, {dt1:.1f} s"}}

    info = ctx.launch_info()
    name = {G.WJ: "wj", G.ALLEY: "alley"}
    # random-gather roofline of this device (K5): context for the "hbm" fraction above
    gather = {"l2_64MB_sectors_per_s": ctx.gather_roofline(64 << 20, 4),
              "hbm_2GB_sectors_per_s": ctx.gather_roofline(2 << 30, 4)}
    gather["dominant_kernel_sectors_per_s"] = sectors[dom] / (dom_ms * 1e-3)
    gather["note"] = ("one 4-byte load per random 32-byte sector, full occupancy (gsword_gather_roofline); "
                      "the kernel mixes L2 hits and DRAM misses")
    qerr = qerror_leg(G, ctx, args) if not (args.quick or args.no_qerror) else None
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * max_time / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64 weights / i32 ids", "data": "synthetic",
        "config": {"workload": WORKLOAD if not args.quick else "quick (not a bench number)",
                   "samples_per_method_per_gpu": n_per_rank, "methods": ["wanderjoin", "alley"],
                   "query": q.name, "query_edges": len(q.edges()), "seed": args.seed,
                   "l2": "flushed before every step (256 MB write)", "parallelism": f"sample-range split x{world}",
                   "grid": info["grid"], "threads": info["threads"]},
        "per_method": {name[m]: {"samples_per_s": n_total * args.steps / (sum(per_method_ms[m]) / 1e3),
                                 "kernel_ms": statistics.mean(kernel_ms[m]),
                                 "estimate": results[m]["estimate"], "std_err": results[m]["variance"] ** 0.5
                                 if results[m]["variance"] > 0 else 0.0,
                                 "valid_fraction": results[m]["n_valid"] / results[m]["n"],
                                 "alg_sectors_per_sample": sectors[m] / cnt,
                                 "first_1e6": depth_stats[m]} for m in methods},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic, "kernel": f"sample_kernel<{name[dom]}>",
                     "peak_kind": peak_kind,
                     "note": "algorithmic 32-B sectors (DESIGN.md §6 model) x 32 B / sampling-kernel time"},
        "gather_roofline": gather,
        "cpu_baseline": cpu_base,
        "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": 32 * len(methods), "graph_load_s": graph_load_s,
                "note": "per step: gsword_load_query from host arrays + gsword_estimate per method "
                        "(synchronous, host result); graph loaded once (P:L1057 excludes it); the "
                        "refill-threshold autotune runs at the first load of the query and is cached "
                        "per (query, options) afterwards"},
        "qerror": qerr,
        "gpu_launches": 2 * len(methods) * args.steps,
        "clocks": clocks.summary(),
    }
    print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
