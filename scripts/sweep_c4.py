"""BASELINE configs[4]: query-size sweep (4-16 vertices, paths / dense / stars) on the
~1e8-edge Kronecker graph: samples/s and q-error versus the sample budget.
Exact counts for the labelled stars come from the closed form star_count (pinned against
brute force in tests/test_sweep_c4.py); the other queries are scored against a reference
estimate (Alley, NLF candidate graph, --ref-samples), labelled as such.
usage: python scripts/sweep_c4.py [--scale 23 --edges 1e8] [--budgets 1e6,1e7,1e8,1e9]"""
import argparse
import json
import math
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def star_count(g, center_label: int, leaf_labels) -> float:
    """Embeddings of a labelled star K_{1,s}: sum over centres v with label a
    of prod_c n_c(v)^(falling m_c), n_c(v) = neighbours of v with label c, m_c = number of
    leaves with label c."""
    n = g.n
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(g.row_ptr))
    cnt = np.bincount(src * g.n_labels + g.labels[g.col].astype(np.int64), minlength=n * g.n_labels)
    cnt = cnt.reshape(n, g.n_labels).astype(np.float64)
    prod = np.ones(n, np.float64)
    for c in set(int(x) for x in leaf_labels):
        m = sum(1 for x in leaf_labels if int(x) == c)
        f = np.ones(n, np.float64)
        for i in range(m):
            f *= np.maximum(cnt[:, c] - i, 0.0)
        prod *= f
    return float(prod[g.labels == center_label].sum())


def main():
    import paper_journals_pacmmod_yelsg24_b200 as G
    from workloads import gen
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=23)
    ap.add_argument("--edges", type=float, default=1e8)
    ap.add_argument("--budgets", default="1e6,1e7,1e8,1e9")
    ap.add_argument("--ref-samples", type=float, default=1e10)
    ap.add_argument("--sizes", default="4,6,8,10,12,14,16")
    args = ap.parse_args()
    t0 = time.time()
    g, qs = gen.config_c4(args.scale, int(args.edges), tuple(int(x) for x in args.sizes.split(",")))
    tgen = time.time() - t0
    budgets = [int(float(b)) for b in args.budgets.split(",")]
    with G.Context(0) as ctx:
        t0 = time.time()
        ctx.load_graph_obj(g)
        tload = time.time() - t0
        print(json.dumps({"graph": g.name, "n": g.n, "m": g.n_edges, "max_degree": int(g.degree().max()),
                          "gen_s": tgen, "load_s": tload}), flush=True)
        for q in qs:
            is_star = q.name.startswith("star")
            if is_star:
                truth, kind = star_count(g, int(q.labels[0]), [int(x) for x in q.labels[1:]]), "exact"
            else:
                ctx.set_option(G.OPT_FILTER, 2)
                ctx.load_query_obj(q)
                r = ctx.estimate(G.ALLEY, int(args.ref_samples), 12345)
                truth, kind = r["estimate"], f"reference (Alley, NLF, {args.ref_samples:.0e} samples, " \
                                             f"rel. s.e. {math.sqrt(max(r['variance'], 0)) / max(r['estimate'], 1e-300):.2e})"
            for filt in (0, 2):
                ctx.set_option(G.OPT_FILTER, filt)
                ctx.load_query_obj(q)
                for m in (G.WJ, G.ALLEY):
                    for b in budgets:
                        r = ctx.estimate(m, b, 42)
                        ks = ctx.last_kernel_seconds()
                        print(json.dumps({"query": q.name, "nq": q.nq, "edges": len(q.edges()), "filter": filt,
                                          "method": "wj" if m == G.WJ else "alley", "budget": b,
                                          "samples_per_s": b / ks, "estimate": r["estimate"],
                                          "truth": truth, "truth_kind": kind,
                                          "qerror": G.qerror(truth, r["estimate"]),
                                          "valid_fraction": r["n_valid"] / r["n"]}), flush=True)


if __name__ == "__main__":
    main()
