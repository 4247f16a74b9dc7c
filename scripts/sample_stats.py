"""Per-sample statistics of SURVEY §8(d) "Report": over the first 1e6 samples of each config
query and method, the valid fraction, the mean depth reached, and the mean and p99 of the
algorithmic sectors per sample.

Two sector models are reported:
* `survey_*`: the model of SURVEY §8(d) written out literally (binary-search membership /
  validation, Alley driver scan on every step), evaluated per sample in numpy from the GPU's
  trace records (path, csize, depth_reached) and the graph — this gives the distribution (p99);
* `kernel_mean`: the kernel's own counting build (`gsword_count_sectors`, the model adapted
  to the edge index) over the same sample ids — mean only.

usage: python scripts/sample_stats.py --configs C0,C1,C2,C3 --samples 1e6 > profiles/r01_sample_stats.jsonl
"""
import argparse
import json
import math
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402
from workloads import gen  # noqa: E402


def bs_sectors(length):
    """1 + ceil(log2(ceil(len / 8))) sectors for a binary search (the last 8 ids share a sector)."""
    length = np.asarray(length, np.int64)
    c = (length + 7) // 8
    out = 1 + np.where(c > 1, np.ceil(np.log2(np.maximum(c, 1))).astype(np.int64), 0)
    return np.where(length > 0, out, 0)


class GraphTables:
    def __init__(self, g):
        self.g = g
        self.n = g.n
        deg = np.diff(g.row_ptr)
        src = np.repeat(np.arange(g.n, dtype=np.int64), deg)
        self.keys = src * g.n + g.col.astype(np.int64)  # sorted (rows ascending, ids ascending)
        self.nl = g.n_labels
        if self.nl > 1:
            self.cnt = np.bincount(src * self.nl + g.labels[g.col], minlength=g.n * self.nl).astype(np.int32)
        else:
            self.cnt = deg.astype(np.int32)

    def nlen(self, v, l):
        v = np.asarray(v, np.int64)
        return self.cnt[v * self.nl + l] if self.nl > 1 else self.cnt[v]

    def adjacent(self, a, b):
        k = np.asarray(a, np.int64) * self.n + np.asarray(b, np.int64)
        i = np.searchsorted(self.keys, k)
        i = np.minimum(i, self.keys.size - 1)
        return self.keys[i] == k


def survey_sectors(T, q, rec, method):
    order = [int(x) for x in q.order]
    qlab = [int(q.labels[u]) for u in order]
    path = rec["path"].astype(np.int64)
    dr = rec["depth_reached"].astype(np.int64)
    csize = rec["csize"].astype(np.int64)
    N = rec.shape[0]
    sec = np.ones(N, np.int64)  # seed: one bucket element
    for d in range(1, q.nq):
        alive = dr >= d
        if not alive.any():
            break
        back = [j for j in range(d) if q.adj[order[j], order[d]]]
        lens = np.stack([T.nlen(np.where(alive, path[:, j], 0), qlab[d]) for j in back], axis=1)
        p = np.argmin(lens, axis=1)  # ties -> first (smallest j)
        lp = lens[np.arange(N), p]
        s = np.full(N, len(back), np.int64)  # seg pairs
        if method == G.WJ:
            drawn = csize[:, d] > 0
            s += drawn
            v = np.where(drawn, path[:, d], 0)
            ok = drawn.copy()
            for j in range(d):  # DupCheck (registers, free)
                ok &= v != path[:, j]
            for bi, j in enumerate(back):
                chk = ok & (p != bi)
                lm = np.minimum(lens[:, bi], T.nlen(v, qlab[j]))
                s += np.where(chk, bs_sectors(lm), 0)
                ok &= ~chk | T.adjacent(path[:, j], v)
        else:
            s += (4 * lp + 31) // 32  # driver scan
            for bi in range(len(back)):
                other = p != bi
                lj = lens[:, bi]
                s += np.where(other, np.minimum(lp * bs_sectors(lj), (4 * lj + 31) // 32), 0)
        sec += np.where(alive, s, 0)
    return sec


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C0,C1,C2,C3")
    ap.add_argument("--samples", type=float, default=1e6)
    ap.add_argument("--seed", type=int, default=42)
    args = ap.parse_args()
    n = int(args.samples)

    with G.Context(0) as ctx:
        for name in args.configs.split(","):
            g, qs = gen.CONFIGS[name]()
            ctx.load_graph_obj(g)
            T = GraphTables(g)
            for q in qs:
                ctx.load_query_obj(q)
                for m in (G.WJ, G.ALLEY):
                    rec = ctx.trace_samples(m, 0, n, args.seed)
                    sec = survey_sectors(T, q, rec, m)
                    kmean = ctx.count_sectors(m, 0, n, args.seed) / n
                    line = {"config": name, "query": q.name, "nq": q.nq, "method": "wj" if m == G.WJ else "alley",
                            "samples": n, "valid_fraction": float(rec["valid"].mean()),
                            "mean_depth_reached": float(rec["depth_reached"].mean()),
                            "survey_sectors_mean": float(sec.mean()), "survey_sectors_p99": float(np.percentile(sec, 99)),
                            "survey_bytes_mean": 32.0 * float(sec.mean()),
                            "kernel_sectors_mean": float(kmean)}
                    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
