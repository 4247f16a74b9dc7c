"""Algorithmic sectors of the C1 queries from the CPU oracle only (reading A26): mean, p99 and max
per sample over the first --samples ids, and, for the |B(d)| >= 2 Alley steps, the probe model's
membership questions against a scan-min variant (each other list costs min(questions, ceil(len/8)),
i.e. a merge scan where it reads fewer sectors).  Test/measurement infrastructure: calls oracle/.
usage: python scripts/sector_model_report.py [--samples 20000] > profiles/r02_sector_model.jsonl"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import oracle  # noqa: E402
from workloads import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--samples", type=int, default=20000)
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    args = ap.parse_args()
    g, qs = gen.config_c1()
    deg = np.diff(g.row_ptr)  # unlabelled: S_j = N(M[j])
    for q in qs:
        order = [int(x) for x in q.order]
        back = {d: [j for j in range(d) if q.adj[order[j], order[d]]] for d in range(q.nq)}
        for m, mn in ((oracle.WJ, "wj"), (oracle.ALLEY, "alley")):
            _, rec = oracle.sample_range(g, q, m, 42, 0, args.samples, records=True, threads=args.threads)
            sec = rec["sectors"].astype(np.float64)
            row = {"query": q.name, "method": mn, "samples": args.samples, "sectors_mean": float(sec.mean()),
                   "sectors_p99": float(np.percentile(sec, 99)), "sectors_max": float(sec.max()),
                   "valid_fraction": float(rec["valid"].mean())}
            if m == oracle.ALLEY:
                probe = scanmin = 0
                for r in rec:
                    for d in range(1, int(r["depth_reached"]) + 1):
                        if len(back[d]) < 2:
                            continue
                        lens = [int(deg[r["path"][j]]) for j in back[d]]
                        p = int(np.argmin(lens))
                        a = lens[p]
                        for k, ln in enumerate(lens):
                            if k != p:  # upper bound of the questions against this list: a
                                probe += a
                                scanmin += min(a, -(-ln // 8))
                row["multi_step_questions_per_sample"] = probe / args.samples
                row["multi_step_scan_min_per_sample"] = scanmin / args.samples
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
