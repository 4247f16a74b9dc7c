"""Throughput and accuracy over the BASELINE.json configs beyond the bench line.

For each config's queries and both methods: samples/s of the sampling kernel (CUDA
events inside the library), valid fraction, estimate and its standard error, and the
q-error against the exact count where one exists (C0: oracle enumeration,
test infrastructure).  Prints one JSON line per (config, query, method).
usage: python scripts/bench_configs.py --configs C0,C2,C3 --samples 1e8
"""
import argparse
import json
import math
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
                line = {"config": name, "graph": {"n": g.n, "m": g.n_edges, "labels": g.n_labels},
                        "query": q.name, "nq": q.nq, "edges": len(q.edges()),
                        "method": "wj" if m == G.WJ else "alley", "samples": int(args.samples),
                        "kernel_s": ks, "samples_per_s": args.samples / ks,
                        "valid_fraction": r["n_valid"] / r["n"], "estimate": r["estimate"],
                        "std_err": math.sqrt(r["variance"]) if r["variance"] > 0 else 0.0,
                        "exact": exact, "qerror": G.qerror(exact, r["estimate"]) if exact is not None else None,
                        "graph_gen_s": tgen, "filter": args.filter, "cg_entries": qi["cg_entries"],
                        "cg_build_s": qi["build_seconds"], "candidates": qi["candidates"]}
                print(json.dumps(line), flush=True)
