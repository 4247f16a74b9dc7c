"""Option sweep on one workload (one process, graph loaded once): prints samples/s per
(method, option setting).  usage: python scripts/sweep.py --config C1 --query 1 --samples 1e8"""
import argparse
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C1")
ap.add_argument("--query", type=int, default=1)
ap.add_argument("--samples", type=float, default=1e8)
ap.add_argument("--grid", default='{"coop": [32]}', help="JSON dict option -> list of values")
ap.add_argument("--methods", default="0,1")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--filter", type=int, default=0)
args = ap.parse_args()
OPT = {"coop": G.OPT_COOP_THRESHOLD, "threads": G.OPT_THREADS, "chunk": G.OPT_CHUNK, "bps": G.OPT_BLOCKS_PER_SM,
       "l2": G.OPT_L2_PERSIST, "bloom": G.OPT_BLOOM, "eset": G.OPT_EDGE_SET,
       "sched": G.OPT_SCHEDULE, "rmin": G.OPT_REFILL_MIN, "stream": G.OPT_STREAMING}
DEF = {"coop": 64, "threads": 256, "chunk": 256, "bps": 0, "l2": 2, "bloom": 1, "eset": 1, "sched": 0, "rmin": 16,
       "stream": 0}
grid = json.loads(args.grid)
g, qs = gen.CONFIGS[args.config]()
queries = qs if args.query < 0 else [qs[args.query]]
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_FILTER, args.filter)
    for q in queries:
        ctx.load_query_obj(q)
        qi = ctx.query_info()
        for m in [int(x) for x in args.methods.split(",")]:
            ctx.estimate(m, 1_000_000, 1)
            keys = list(grid)
            for vals in itertools.product(*[grid[k] for k in keys]):
                for k, v in DEF.items():
                    ctx.set_option(OPT[k], v)
                for k, v in zip(keys, vals):
                    ctx.set_option(OPT[k], v)
                best = None
                for _ in range(args.reps):
                    r = ctx.estimate(m, int(args.samples), 42)
                    t = ctx.last_kernel_seconds()
                    best = t if best is None else min(best, t)
                print(json.dumps({"config": args.config, "query": q.name, "method": m, "filter": args.filter,
                                  "cg_entries": qi["cg_entries"], "cg_build_s": qi["build_seconds"],
                                  "candidates": qi["candidates"],
                                  "opts": dict(zip(keys, vals)), "kernel_s": best,
                                  "rate": args.samples / best, "valid": r["n_valid"], "est": r["estimate"],
                                  "var": r["variance"], "var_x_s": r["variance"] * best}),
                      flush=True)
