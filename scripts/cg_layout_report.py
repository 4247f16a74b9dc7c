"""Candidate graph in the three-CSR format of Fig. 4 (NEXT-1; Tab. 3):
build time, device bytes (against the round-1 layout: one dense (|V|+1)-entry offset row
per directed query edge), and what the filter buys the samplers: samples/s, positions
sampled per second (the per-step rate, which separates the layout's cost from the longer
walks a filter produces), valid fraction and variance x time (lower is better) for the
label-only lists (filter 0) and NLF (filter 2).

usage: python scripts/cg_layout_report.py [--configs C1,C2,C3,C4] > profiles/r02_cg_layout.jsonl
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import paper_journals_pacmmod_yelsg24_b200 as G
    from workloads import gen
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C4")
    ap.add_argument("--samples", type=float, default=1e8)
    ap.add_argument("--c4-queries", default="dense16_s5016,dense12_s5012,sparse16_s4016,dense8_s5008")
    args = ap.parse_args()
    n = int(args.samples)
    for cfg in args.configs.split(","):
        t0 = time.time()
        g, qs = gen.CONFIGS[cfg]()
        gen_s = time.time() - t0
        if cfg == "C4":
            want = set(args.c4_queries.split(","))
            qs = [q for q in qs if q.name in want]
        with G.Context(0) as ctx:
            ctx.load_graph_obj(g)
            for q in qs:
                directed = 2 * len(q.edges())
                row = {"config": cfg, "graph": g.name, "n": g.n, "m": g.n_edges, "query": q.name, "nq": q.nq,
                       "query_edges": len(q.edges()), "gen_s": gen_s,
                       "r01_dense_offset_bytes": directed * (g.n + 1) * 4}
                for filt in (0, 2):
                    ctx.set_option(G.OPT_FILTER, filt)
                    ctx.load_query_obj(q)
                    info = ctx.query_info()
                    if filt:
                        row.update({"build_ms": 1e3 * info["build_seconds"], "cg_bytes": info["cg_bytes"],
                                    "cg_entries": info["cg_entries"], "cand_sum": int(sum(info["candidates"])),
                                    "cg_bytes_over_r01_offsets": info["cg_bytes"] / row["r01_dense_offset_bytes"]})
                    for m, mn in ((G.WJ, "wj"), (G.ALLEY, "alley")):
                        ctx.estimate(m, min(n, 10_000_000), 42)  # warm-up
                        r = ctx.estimate(m, n, 42)
                        rec = ctx.trace_samples(m, 0, 100_000, 42)
                        depth = float(rec["depth_reached"].astype(np.float64).mean()) + 1.0
                        var = r["variance"] if r["variance"] == r["variance"] else float("nan")
                        row[f"f{filt}_{mn}"] = {
                            "samples_per_s": n / r["seconds"], "seconds": r["seconds"],
                            "positions_per_s": n * depth / r["seconds"], "mean_positions": depth,
                            "valid_fraction": r["n_valid"] / r["n"], "estimate": r["estimate"],
                            "rel_std_err": (var ** 0.5 / r["estimate"]) if r["estimate"] > 0 and var > 0 else None,
                            "var_x_seconds": var * r["seconds"] if var == var else None}
                ctx.set_option(G.OPT_FILTER, 0)
                print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
