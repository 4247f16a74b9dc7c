"""Warp-cycle split of the sampling loop (count build), per method and query.
usage: python scripts/phases.py --config C1 --samples 2e7"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

NAMES = ["refill", "draw+getmin", "wj/alley-kind", "pool", "select", "coop", "epilogue", "exit"]
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C1")
ap.add_argument("--samples", type=float, default=2e7)
ap.add_argument("--coop", type=int, default=32)
args = ap.parse_args()
g, qs = gen.CONFIGS[args.config]()
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_COOP_THRESHOLD, args.coop)
    for q in qs:
        ctx.load_query_obj(q)
        for m in (G.WJ, G.ALLEY):
            sec = ctx.count_sectors(m, 0, int(args.samples), 42)[0]
            ph = ctx.phase_cycles()
            tot = sum(ph)
            print(f"{q.name:14s} m={m} sectors/sample={sec / args.samples:7.2f} " +
                  " ".join(f"{n}={v / tot:5.1%}" for n, v in zip(NAMES, ph)), flush=True)
