"""Launch efficiency at small sample counts: device time of gsword_estimate (events
around the whole call: queue reset, sampling kernel, reduction) for n = 1e5 .. 1e8 on the
bench workload, per method.  Shows the fixed cost per launch (tail of the persistent
grid) that pilot runs and small estimate_until batches pay."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

g, qs = gen.config_c1()
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[1])
    for m in (G.WJ, G.ALLEY):
        ctx.estimate(m, 2_000_000, 1)
        for n in (100_000, 300_000, 1_000_000, 2_000_000, 4_000_000, 10_000_000, 30_000_000, 100_000_000):
            ts, ks = [], []
            for rep in range(3):
                r = ctx.estimate(m, n, 42 + rep)
                ts.append(r["seconds"])
                ks.append(ctx.last_kernel_seconds())
            print(json.dumps({"method": m, "n": n, "call_ms": 1e3 * min(ts), "kernel_ms": 1e3 * min(ks),
                              "samples_per_s": n / min(ts)}), flush=True)
