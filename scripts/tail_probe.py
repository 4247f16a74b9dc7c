"""Sampling-kernel time against the range size (2.5e7 .. 2e8 ids) on C1's dense and cyclic
queries: the slope is the steady-state cost, 2 t(n) - t(2n) the per-launch tail.
usage: python scripts/tail_probe.py > profiles/r02_tail_probe.jsonl"""
import sys, json, torch
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_journals_pacmmod_yelsg24_b200 as G
from workloads import gen
g, qs = gen.config_c1()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with G.Context(0) as ctx:
    ctx.load_graph_obj(g)
    for qi in (1, 2):
        ctx.load_query_obj(qs[qi])
        for m in (0, 1):
            ctx.estimate(m, 4_000_000, 1)
            res = {}
            for n in (25_000_000, 50_000_000, 100_000_000, 200_000_000):
                ts = []
                for rep in range(3):
                    flush.fill_(rep); torch.cuda.synchronize()
                    ctx.estimate(m, n, 42)
                    ts.append(ctx.last_kernel_seconds())
                res[n] = 1e3 * min(ts)
            print(json.dumps({"query": qs[qi].name, "method": m, "kernel_ms": res}), flush=True)
