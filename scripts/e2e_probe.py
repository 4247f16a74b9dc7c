import sys, time, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_journals_pacmmod_yelsg24_b200 as G
from workloads import gen
g, qs = gen.config_c1(); q = qs[1]
qrp, qcol = q.csr()
h_q = [np.ascontiguousarray(a) for a in (qrp, qcol, q.labels, q.order)]
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    for at in (1, 0):
        ctx.set_option(G.OPT_AUTOTUNE, at)
        for i in range(4):
            torch.cuda.synchronize(); t0 = time.perf_counter()
            ctx.load_query(*h_q)
            t1 = time.perf_counter()
            r0 = ctx.estimate(0, 100_000_000, 42); t2 = time.perf_counter()
            r1 = ctx.estimate(1, 100_000_000, 42); t3 = time.perf_counter()
            print(f"autotune={at} load_query {1e3*(t1-t0):.2f} ms  wj {1e3*(t2-t1):.2f} (dev {1e3*r0['seconds']:.2f})  alley {1e3*(t3-t2):.2f} (dev {1e3*r1['seconds']:.2f}) info {ctx.query_info()['refill_min']}")
