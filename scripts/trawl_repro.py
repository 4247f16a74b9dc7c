"""Trawling on C2 at one (query, method, n, budget) — a short driver for sanitizer runs.
usage: python scripts/trawl_repro.py [n] [budget] [warp] [query]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

n = int(float(sys.argv[1])) if len(sys.argv) > 1 else 100_000
budget = int(float(sys.argv[2])) if len(sys.argv) > 2 else 1_000_000
warp = int(sys.argv[3]) if len(sys.argv) > 3 else 1
qi = int(sys.argv[4]) if len(sys.argv) > 4 else 0
g, qs = gen.config_c2()
with G.Context(0) as ctx:
    ctx.set_option(G.OPT_TRAWL_WARP, warp)
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[qi])
    for m in (G.WJ, G.ALLEY):
        r = ctx.trawl(m, n, 42, node_budget=budget)
        print(m, n, budget, warp, r["n"], r["n_timeout"], r["n_valid"], r["estimate"], r["seconds"], flush=True)
