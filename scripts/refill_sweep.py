"""Refill threshold x occupancy variant sweep of the estimate kernels with the autotune off
(best of 3, L2 flushed): which candidates the query-load autotune should time.
usage: python scripts/refill_sweep.py [--work C1:1,C1:2] [--samples 1e8] > profiles/r02_refill_sweep.jsonl"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import paper_journals_pacmmod_yelsg24_b200 as G
    from workloads import gen
    ap = argparse.ArgumentParser()
    ap.add_argument("--work", default="C1:1,C1:2,C1:0")
    ap.add_argument("--samples", type=float, default=1e8)
    ap.add_argument("--refills", default="12,16,20,24,28,32")
    args = ap.parse_args()
    n = int(args.samples)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    cache = {}
    with G.Context(0) as ctx:
        ctx.set_option(G.OPT_AUTOTUNE, 0)
        for w in args.work.split(","):
            cfg, qi = w.split(":")
            if cfg not in cache:
                cache.clear()
                cache[cfg] = gen.CONFIGS[cfg]()
                ctx.load_graph_obj(cache[cfg][0])
            q = cache[cfg][1][int(qi)]
            ctx.load_query_obj(q)
            for m in (G.WJ, G.ALLEY):
                for rmin in (int(x) for x in args.refills.split(",")):
                    for occ in (0, 1, 2):
                        ctx.set_option(G.OPT_REFILL_MIN, rmin)
                        ctx.set_option(G.OPT_OCCUPANCY, occ)
                        ctx.estimate(m, min(n, 4_000_000), 1)
                        ts = []
                        for rep in range(3):
                            flush.fill_(rep)
                            torch.cuda.synchronize()
                            ctx.estimate(m, n, 42)
                            ts.append(ctx.last_kernel_seconds())
                        print(json.dumps({"config": cfg, "query": q.name, "method": m, "refill_min": rmin, "occ": occ,
                                          "kernel_ms": 1e3 * min(ts)}), flush=True)
            ctx.set_option(G.OPT_OCCUPANCY, -1)


if __name__ == "__main__":
    main()
