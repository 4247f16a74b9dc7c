"""Trawling (NEXT-2) vs plain sampling on the underestimation regime (BASELINE configs[2],
WordNet shape): estimate, standard error, kernel time and the work-normalised variance
var(estimate) * seconds (lower is better) for each method and filter.
usage: python scripts/trawl_eval.py --config C2 --samples 1e8 --trawl-samples 1e6"""
import argparse
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--samples", type=float, default=1e8)
ap.add_argument("--trawl-samples", type=float, default=1e6)
ap.add_argument("--budget", type=int, default=1_000_000)
ap.add_argument("--filters", default="0,2")
args = ap.parse_args()
g, qs = gen.CONFIGS[args.config]()
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    for filt in [int(x) for x in args.filters.split(",")]:
        ctx.set_option(G.OPT_FILTER, filt)
        for q in qs:
            ctx.load_query_obj(q)
            for m in (G.WJ, G.ALLEY):
                for mode in ("plain", "trawl", "trawl_lane"):
                    if mode == "plain":
                        r = ctx.estimate(m, int(args.samples), 42)
                        r["n_timeout"] = 0
                    else:
                        # trawl: warp-cooperative enumeration (default); trawl_lane: one lane
                        # per sample, depth first (round 1's kernel)
                        ctx.set_option(G.OPT_TRAWL_WARP, 1 if mode == "trawl" else 0)
                        r = ctx.trawl(m, int(args.trawl_samples), 42, node_budget=args.budget)
                        ctx.set_option(G.OPT_TRAWL_WARP, 1)
                    se = math.sqrt(r["variance"]) if r["variance"] > 0 else 0.0
                    print(json.dumps({"config": args.config, "query": q.name, "filter": filt,
                                      "method": "wj" if m == G.WJ else "alley", "mode": mode, "n": r["n"],
                                      "n_timeout": r["n_timeout"], "nonzero": r["n_valid"],
                                      "estimate": r["estimate"], "std_err": se, "seconds": r["seconds"],
                                      "var_x_seconds": r["variance"] * r["seconds"]}), flush=True)
