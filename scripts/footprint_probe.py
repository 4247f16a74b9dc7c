"""Working-set probe: the same query pattern (C1's dense 8-vertex query) on Chung-Lu
graphs with C1's degree distribution shape (gamma 2.1, same max/mean weight ratio and
mean degree) at scales 1, 1/2, 1/4, 1/8 of |V| and |E|.  Per-sample work is similar at
every scale; what changes is the footprint of col / edge filter / edge set against the
126 MB L2.  Prints one JSON line per (scale, method): kernel ms, samples/s, algorithmic
sectors per sample.  Used to decide whether shrinking the graph's bytes
can pay."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402

N = int(float(sys.argv[1])) if len(sys.argv) > 1 else 100_000_000
scales = [float(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [1.0, 0.5, 0.25, 0.125]
# optional gsword_set_option pairs applied before the loads, e.g. "5=0" (filter off)
opts = [tuple(int(v) for v in o.split("=")) for o in sys.argv[3].split(",")] if len(sys.argv) > 3 else []
_, qs = gen.config_c1()
q = qs[1]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with G.Context(0) as ctx:
    for k, v in opts:
        ctx.set_option(k, v)
    for s in scales:
        n, m = int(862_664 * s), int(16_138_468 * s)
        g = gen.chung_lu(n, m, gamma=2.1, max_over_mean=68_963 / 37.4, seed=2005, name=f"cl_{s}")
        ctx.load_graph_obj(g)
        ctx.load_query_obj(q)
        for meth in (G.WJ, G.ALLEY):
            ctx.estimate(meth, 2_000_000, 1)
            ts = []
            for rep in range(3):
                flush.fill_(rep)
                torch.cuda.synchronize()
                r = ctx.estimate(meth, N, 42)
                ts.append(ctx.last_kernel_seconds())
            sec = ctx.count_sectors(meth, 0, 1_000_000, 42)[0] / 1_000_000
            t = min(ts)
            print(json.dumps({"opts": opts, "scale": s, "n": n, "m": m, "col_mb": 8 * m / 2**20, "method": meth, "kernel_ms": 1e3 * t,
                              "samples_per_s": N / t, "sectors_per_sample": sec, "valid_fraction": r["n_valid"] / N,
                              "GBps_alg": sec * 32 * N / t / 1e9}), flush=True)
