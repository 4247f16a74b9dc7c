"""Small estimate / trace runs for compute-sanitizer (memcheck, racecheck, synccheck,
initcheck): both methods, every refine path (coop thresholds 0 and 64), every occupancy
variant, refill thresholds 16 and 32 (the depth-synchronous Alley kernel), trace and counting
builds, and a query loaded with the NLF candidate graph (Fig. 4 layout build + sampling)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

g = gen.chung_lu(2000, 30_000, gamma=2.2, max_over_mean=40.0, seed=3, labels=gen.uniform_labels(2000, 2, 4),
                 n_labels=2)
q = gen.extract_query(g, 6, seed=5, dense=True, require_dense=True)
qt = gen.extract_query(g, 6, seed=6, dense=False)  # tree order: the TREE estimate kernels
with G.Context(0) as ctx:
    ctx.set_option(G.OPT_AUTOTUNE, 0)  # no pilots under the sanitizer; variants forced below
    ctx.load_graph_obj(g)
    for qq in (q, qt):
        ctx.load_query_obj(qq)
        for coop in (0, 64):
            ctx.set_option(G.OPT_COOP_THRESHOLD, coop)
            for m in (G.WJ, G.ALLEY):
                for occ in (0, 1, 2):  # every occupancy variant of the estimate kernel
                    ctx.set_option(G.OPT_OCCUPANCY, occ)
                    for rmin in (16, 32):  # 32: the depth-synchronous (LOCK) Alley kernel
                        ctx.set_option(G.OPT_REFILL_MIN, rmin)
                        r = ctx.estimate(m, 20_000, 1)
                    ctx.set_option(G.OPT_REFILL_MIN, 16)
                ctx.set_option(G.OPT_OCCUPANCY, -1)
                rec = ctx.trace_samples(m, 0, 2000, 1)
                s = ctx.count_sectors(m, 0, 2000, 1)
                print(qq.name, m, coop, r["n_valid"], int(rec["valid"].sum()), s)
    ctx.set_option(G.OPT_FILTER, 2)  # the candidate graph (three-CSR layout) build and its samplers
    ctx.load_query_obj(q)
    for m in (G.WJ, G.ALLEY):
        r = ctx.estimate(m, 20_000, 1)
        rec = ctx.trace_samples(m, 0, 2000, 1)
        print("nlf", q.name, m, r["n_valid"], int(rec["valid"].sum()), ctx.query_info()["cg_bytes"])
    # trawling: the warp-cooperative enumeration (shared-memory stack; estimates) and the
    # per-lane kernel (traces), label-only and under the candidate graph
    for filt in (0, 2):
        ctx.set_option(G.OPT_FILTER, filt)
        ctx.load_query_obj(q)
        for m in (G.WJ, G.ALLEY):
            for warp in (1, 0):
                ctx.set_option(G.OPT_TRAWL_WARP, warp)
                r = ctx.trawl(m, 3000, 1, node_budget=5000)
            ctx.set_option(G.OPT_TRAWL_WARP, 1)
            tr = ctx.trace_trawl(m, 0, 500, 1, 5000)
            print("trawl", filt, m, r["n_valid"], r["n_timeout"], int((tr["status"] == 1).sum()))
