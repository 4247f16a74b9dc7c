"""BASELINE.json configs at their stated budgets on one B200: C3 (LiveJournal shape, 16 labels,
12-vertex queries) Alley 1e10 samples per query, and C4 (Kronecker, 1e8 edges) Alley at 1e10
for its 8- and 12-vertex dense queries.  Device time (CUDA events in the library), estimate,
relative standard error, valid fraction.  One JSON line per run.
usage: python scripts/full_budget.py > profiles/r02_full_budget.jsonl"""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import paper_journals_pacmmod_yelsg24_b200 as G
    from workloads import gen
    runs = [("C3", None, 10_000_000_000), ("C4", ("dense8_s5008", "dense12_s5012"), 10_000_000_000)]
    with G.Context(0) as ctx:
        for cfg, names, n in runs:
            g, qs = gen.CONFIGS[cfg]()
            ctx.load_graph_obj(g)
            for q in qs:
                if names and q.name not in names:
                    continue
                ctx.load_query_obj(q)
                r = ctx.estimate(G.ALLEY, n, 42)
                se = math.sqrt(r["variance"]) if r["variance"] > 0 else 0.0
                print(json.dumps({"config": cfg, "query": q.name, "method": "alley", "samples": n,
                                  "seconds": r["seconds"], "samples_per_s": n / r["seconds"],
                                  "estimate": r["estimate"], "rel_std_err": se / r["estimate"] if r["estimate"] else None,
                                  "valid_fraction": r["n_valid"] / r["n"]}), flush=True)


if __name__ == "__main__":
    main()
