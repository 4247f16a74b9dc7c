"""Throughput and accuracy over the BASELINE.json configs beyond the bench line.

For each config's queries and both methods: samples/s of the sampling kernel (CUDA
events inside the library), valid fraction, estimate and its standard error, the q-error
 against the exact count where one exists (C0: oracle enumeration, test
infrastructure), and SURVEY §8(d)'s report: the A26 algorithmic sectors per sample over the
whole run (counting build) with the resulting fraction of the HBM copy peak, and over the
first 1e6 sample ids the mean / p99 sectors and depth reached.  One JSON line per (config,
query, method).
usage: python scripts/bench_configs.py --configs C0,C2,C3 --samples 1e8
"""
import argparse
import json
import math

import numpy as np
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="C0,C2,C3")
ap.add_argument("--samples", type=float, default=1e8)
ap.add_argument("--seed", type=int, default=42)
ap.add_argument("--exact", type=int, default=1, help="compute exact counts for C0 with the oracle enumerator")
ap.add_argument("--filter", type=int, default=0, help="candidate filter: 0 label, 1 LDF, 2 NLF")
args = ap.parse_args()
try:
    PEAK = float(json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                             "MEASURED_PEAKS.json")))["hbm_gbs"])
except Exception:
    PEAK = 6650.0  # B200_PROFILING.md fallback

with G.Context(0) as ctx:
    for name in args.configs.split(","):
        t0 = time.time()
        g, qs = gen.CONFIGS[name]()
        tgen = time.time() - t0
        ctx.load_graph_obj(g)
        ctx.set_option(G.OPT_FILTER, args.filter)
        for q in qs:
            exact = None
            if args.exact and name == "C0":
                import oracle  # test infrastructure: exact count for the q-error only
                exact = oracle.count_embeddings(g, q)
            ctx.load_query_obj(q)
            qi = ctx.query_info()
            for m in (G.WJ, G.ALLEY):
                ctx.estimate(m, 1_000_000, 1)
                r = ctx.estimate(m, int(args.samples), args.seed)
                ks = ctx.last_kernel_seconds()
                model, touched = ctx.count_sectors(m, 0, int(args.samples), args.seed)
                rec = ctx.trace_samples(m, 0, min(int(args.samples), 1_000_000), args.seed)
                sec = rec["sectors"].astype(np.float64)
                dr = rec["depth_reached"].astype(np.float64)
                line = {"config": name, "graph": {"n": g.n, "m": g.n_edges, "labels": g.n_labels},
                        "query": q.name, "nq": q.nq, "edges": len(q.edges()),
                        "method": "wj" if m == G.WJ else "alley", "samples": int(args.samples),
                        "kernel_s": ks, "samples_per_s": args.samples / ks,
                        "valid_fraction": r["n_valid"] / r["n"], "estimate": r["estimate"],
                        "std_err": math.sqrt(r["variance"]) if r["variance"] > 0 else 0.0,
                        "exact": exact, "qerror": G.qerror(exact, r["estimate"]) if exact is not None else None,
                        "graph_gen_s": tgen, "filter": args.filter, "cg_entries": qi["cg_entries"],
                        "cg_build_s": qi["build_seconds"], "candidates": qi["candidates"],
                        "alg_sectors_per_sample": model / args.samples,
                        "touched_sectors_per_sample": touched / args.samples,
                        "frac_of_hbm_copy_peak": model * 32.0 / ks / 1e9 / PEAK,
                        "first_1e6": {"sectors_mean": float(sec.mean()), "sectors_p99": float(np.percentile(sec, 99)),
                                      "depth_mean": float(dr.mean()), "depth_p99": float(np.percentile(dr, 99)),
                                      "valid_fraction": float(rec["valid"].mean())}}
                print(json.dumps(line), flush=True)
