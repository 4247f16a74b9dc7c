"""Edge-filter size x L2 window sweep on C1 (graph reloaded per filter size)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

g, qs = gen.config_c1()
with G.Context(0) as ctx:
    import ctypes
    for bits in (4, 8, 16, 32):
        ctx.set_option(G.OPT_BLOOM_BITS, bits)
        ctx.set_option(G.OPT_L2_PERSIST, 0)
        ctx.load_graph_obj(g)
        for l2 in (0, 2):
            ctx.set_option(G.OPT_L2_PERSIST, l2)
            for q in qs:
                ctx.load_query_obj(q)
                for m in (0, 1):
                    ctx.estimate(m, 1_000_000, 1)
                    best = min((ctx.estimate(m, 100_000_000, 42), ctx.last_kernel_seconds())[1] for _ in range(2))
                    print(json.dumps({"bits": bits, "l2": l2, "query": q.name, "method": m, "ms": best * 1e3}),
                          flush=True)
