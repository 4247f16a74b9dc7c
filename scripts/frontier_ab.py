"""A/B of the two Alley sampler paths on the bench workloads: the persistent refill kernel
(GSWORD_OPT_PATH = 0, its autotuned refill threshold and occupancy) against the
level-synchronous frontier kernels (GSWORD_OPT_PATH = 1).  Best of 3 device times over the
sample range (L2 flushed before each), plus the autotuned default's choice.
usage: python scripts/frontier_ab.py [--work C1:1,C1:2,C1:0,C2:0,C3:2] [--samples 1e8]"""
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
    ap.add_argument("--work", default="C1:1,C1:2,C1:0,C2:0,C3:2")
    ap.add_argument("--samples", type=float, default=1e8)
    ap.add_argument("--coop", default="64")
    args = ap.parse_args()
    n = int(args.samples)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    cache = {}
    with G.Context(0) as ctx:
        for w in args.work.split(","):
            cfg, qi = w.split(":")
            if cfg not in cache:
                cache.clear()
                cache[cfg] = gen.CONFIGS[cfg]()
                ctx.load_graph_obj(cache[cfg][0])
            g, qs = cache[cfg]
            q = qs[int(qi)]
            row = {"config": cfg, "query": q.name, "samples": n}
            for coop in (int(c) for c in args.coop.split(",")):
                ctx.set_option(G.OPT_COOP_THRESHOLD, coop)
                for path in (0, 1, -1):
                    ctx.set_option(G.OPT_PATH, path)
                    ctx.load_query_obj(q)
                    ctx.estimate(G.ALLEY, min(n, 4_000_000), 1)
                    ts = []
                    for rep in range(3):
                        flush.fill_(rep)
                        torch.cuda.synchronize()
                        r = ctx.estimate(G.ALLEY, n, 42)
                        ts.append(ctx.last_kernel_seconds())
                    key = {0: "persistent", 1: "frontier", -1: "auto"}[path] + f"_coop{coop}"
                    row[key] = {"kernel_ms": 1e3 * min(ts), "samples_per_s": n / min(ts),
                                "n_valid": r["n_valid"], "sum": r["sum"], "path": ctx.query_info()["path"][1]}
            ctx.set_option(G.OPT_COOP_THRESHOLD, 64)
            ctx.set_option(G.OPT_PATH, -1)
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
