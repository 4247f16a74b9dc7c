"""Short, fixed launch sequence for ncu captures (one GPU, never multi-rank):
2 warm-up estimates (WanderJoin, Alley; 1e6 samples), then WanderJoin and Alley at
--samples each on the bench workload, bracketed by cudaProfilerStart/Stop so that
`ncu --profile-from-start off -k regex:sample_kernel` captures exactly those two launches
(whatever the autotune at query load launched before)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--samples", type=float, default=1e7)
ap.add_argument("--config", default="C1")
ap.add_argument("--query", type=int, default=1)
ap.add_argument("--l2", type=int, default=-1, help="GSWORD_OPT_L2_PERSIST; -1 = the product default (the bench's)")
ap.add_argument("--coop", type=int, default=-1)
ap.add_argument("--threads", type=int, default=0)
ap.add_argument("--chunk", type=int, default=0)
ap.add_argument("--bps", type=int, default=0)
ap.add_argument("--methods", default="0,1")
args = ap.parse_args()

g, qs = gen.CONFIGS[args.config]()
q = qs[args.query]
with G.Context(0) as ctx:
    if args.l2 >= 0:
        ctx.set_option(G.OPT_L2_PERSIST, args.l2)
    if args.coop >= 0:
        ctx.set_option(G.OPT_COOP_THRESHOLD, args.coop)
    if args.threads:
        ctx.set_option(G.OPT_THREADS, args.threads)
    if args.chunk:
        ctx.set_option(G.OPT_CHUNK, args.chunk)
    if args.bps:
        ctx.set_option(G.OPT_BLOCKS_PER_SM, args.bps)
    ctx.load_graph_obj(g)
    ctx.load_query_obj(q)
    methods = [int(x) for x in args.methods.split(",")]
    for m in methods:
        ctx.estimate(m, 1_000_000, 42)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    res = {m: ctx.estimate(m, int(args.samples), 42) for m in methods}
    torch.cuda.profiler.stop()
    for m, r in res.items():
        print(f"method={m} samples={int(args.samples)} seconds={r['seconds']:.4f} "
              f"rate={args.samples / r['seconds']:.3e}/s est={r['estimate']:.4e} valid={r['n_valid']}")
