"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the estimator (no candidate sets, no random
draws of the sampler, no weights).  It only builds inputs:

* canonical labelled data graphs in CSR form: undirected,
  simple, symmetric, vertex ids 0..n-1, each adjacency list in ascending id;
* query graphs (dense adjacency over <= 16 vertices) with labels;
* a connected matching order (Def. 2; every prefix connected,
  DESIGN.md reading A13);
* the named workloads of BASELINE.json configs[0..4] (recipes in DESIGN.md).

Every function is a pure function of its arguments and seed (numpy PCG64).
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional, Sequence, Tuple

import numpy as np

MAX_QV = 16


# --------------------------------------------------------------------------
# containers
# --------------------------------------------------------------------------
@dataclasses.dataclass
class Graph:
    """Canonical CSR: row_ptr int64[n+1], col int32[2|E|], labels int32[n]."""

    row_ptr: np.ndarray
    col: np.ndarray
    labels: np.ndarray
    n_labels: int
    name: str = ""

    @property
    def n(self) -> int:
        return int(self.row_ptr.shape[0] - 1)

    @property
    def n_edges(self) -> int:  # undirected edges
        return int(self.col.shape[0] // 2)

    def degree(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def neighbors(self, v: int) -> np.ndarray:
        return self.col[self.row_ptr[v]:self.row_ptr[v + 1]]

    def label_sorted_col(self) -> np.ndarray:
        """Adjacency with each row ordered by (label, id) (layout for device loading)."""
        src = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.row_ptr))
        key = (src * max(self.n_labels, 1) + self.labels[self.col].astype(np.int64)) * self.n + self.col
        return self.col[np.argsort(key, kind="stable")].astype(np.int32)


@dataclasses.dataclass
class Query:
    """Query graph q: symmetric 0/1 adjacency, labels, matching order phi."""

    adj: np.ndarray  # uint8 [nq, nq]
    labels: np.ndarray  # int32 [nq]
    order: np.ndarray  # int32 [nq], a permutation of 0..nq-1
    name: str = ""

    @property
    def nq(self) -> int:
        return int(self.labels.shape[0])

    def edges(self) -> List[Tuple[int, int]]:
        nq = self.nq
        return [(a, b) for a in range(nq) for b in range(a + 1, nq) if self.adj[a, b]]

    def csr(self) -> Tuple[np.ndarray, np.ndarray]:
        """Symmetric query CSR (q_row_ptr int32[nq+1], q_col int32)."""
        rp = [0]
        cols: List[int] = []
        for a in range(self.nq):
            nb = [b for b in range(self.nq) if self.adj[a, b]]
            cols.extend(nb)
            rp.append(len(cols))
        return np.asarray(rp, np.int32), np.asarray(cols, np.int32)

    def with_order(self, order: Sequence[int]) -> "Query":
        return Query(self.adj.copy(), self.labels.copy(), np.asarray(order, np.int32), self.name)

    def _renamed(self, name: str) -> "Query":
        return Query(self.adj, self.labels, self.order, name)


# --------------------------------------------------------------------------
# CSR construction
# --------------------------------------------------------------------------
def _sorted_unique(x: np.ndarray) -> np.ndarray:
    x = np.sort(x)
    if x.shape[0] == 0:
        return x
    keep = np.empty(x.shape[0], bool)
    keep[0] = True
    np.not_equal(x[1:], x[:-1], out=keep[1:])
    return x[keep]


def csr_from_pairs(n: int, u: np.ndarray, v: np.ndarray) -> Tuple[np.ndarray, np.ndarray]:
    """Canonical symmetric CSR from undirected pairs (drops self loops and duplicates)."""
    u = np.asarray(u, np.int64)
    v = np.asarray(v, np.int64)
    keep = u != v
    u, v = u[keep], v[keep]
    a = np.minimum(u, v)
    b = np.maximum(u, v)
    key = _sorted_unique(a * n + b)
    a = key // n
    b = key % n
    src = np.concatenate([a, b])
    dst = np.concatenate([b, a])
    skey = np.sort(src * n + dst)
    src = skey // n
    dst = skey % n
    counts = np.bincount(src, minlength=n)
    row_ptr = np.zeros(n + 1, np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return row_ptr, dst.astype(np.int32)


def make_graph(n: int, u, v, labels: Optional[np.ndarray], n_labels: int, name: str = "") -> Graph:
    row_ptr, col = csr_from_pairs(n, np.asarray(u), np.asarray(v))
    if labels is None:
        labels = np.zeros(n, np.int32)
        n_labels = 1
    return Graph(row_ptr, col, np.asarray(labels, np.int32), int(n_labels), name)


def _sample_unique_pairs(n: int, m: int, draw, rng: np.random.Generator) -> np.ndarray:
    """Draw endpoint pairs with `draw(rng, size)` until >= m distinct undirected pairs
    exist, then keep a seeded uniform subset of exactly m (sorted keys a*n+b, a<b)."""
    keys = np.zeros(0, np.int64)
    while keys.shape[0] < m:
        need = m - keys.shape[0]
        size = int(need * 1.3) + 1024
        a = draw(rng, size)
        b = draw(rng, size)
        ok = a != b
        a, b = a[ok], b[ok]
        k = np.minimum(a, b).astype(np.int64) * n + np.maximum(a, b)
        keys = _sorted_unique(np.concatenate([keys, k]))
    if keys.shape[0] > m:
        sel = np.sort(rng.choice(keys.shape[0], size=m, replace=False))
        keys = keys[sel]
    return keys


# --------------------------------------------------------------------------
# data-graph generators
# --------------------------------------------------------------------------
def uniform_labels(n: int, n_labels: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.integers(0, n_labels, size=n, dtype=np.int64).astype(np.int32)


def skewed_labels(n: int, probs: Sequence[float], seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    p = np.asarray(probs, np.float64)
    p = p / p.sum()
    return rng.choice(len(p), size=n, p=p).astype(np.int32)


def erdos_renyi(n: int, m: int, seed: int, n_labels: int = 1, label_seed: int = 0, name: str = "") -> Graph:
    """G(n, m): m distinct pairs uniform without replacement (config C0 recipe)."""
    rng = np.random.default_rng(seed)
    keys = _sample_unique_pairs(n, m, lambda r, s: r.integers(0, n, size=s, dtype=np.int64), rng)
    labels = uniform_labels(n, n_labels, label_seed) if n_labels > 1 else None
    return make_graph(n, keys // n, keys % n, labels, n_labels, name or f"er{n}_{m}")


def chung_lu(n: int, m: int, gamma: float, max_over_mean: float, seed: int,
             labels: Optional[np.ndarray] = None, n_labels: int = 1, name: str = "") -> Graph:
    """Chung-Lu power-law graph with exactly m undirected edges.

    Weights w_i = (i + i0)^(-1/(gamma-1)); i0 is chosen so that w_max / mean(w)
    equals `max_over_mean`.  Endpoints are drawn independently with P ∝ w,
    self loops and duplicates dropped, topped up to exactly m.
    """
    alpha = 1.0 / (gamma - 1.0)
    idx = np.arange(n, dtype=np.float64)

    def ratio(i0: float) -> float:
        w = (idx + i0) ** (-alpha)
        return float(w[0] / w.mean())

    lo, hi = 1e-3, float(n)
    for _ in range(60):  # ratio is decreasing in i0
        mid = np.sqrt(lo * hi)
        if ratio(mid) > max_over_mean:
            lo = mid
        else:
            hi = mid
    w = (idx + hi) ** (-alpha)

    p = w / w.sum()

    def draw(r: np.random.Generator, size: int) -> np.ndarray:
        # endpoint multiset ~ Multinomial(size, p), then a seeded shuffle
        counts = r.multinomial(size, p)
        x = np.repeat(np.arange(n, dtype=np.int64), counts)
        return r.permutation(x)

    rng = np.random.default_rng(seed)
    keys = _sample_unique_pairs(n, m, draw, rng)
    if labels is None:
        n_labels = 1
    return make_graph(n, keys // n, keys % n, labels, n_labels, name or f"cl{n}_{m}")


def kronecker(scale: int, n_edges_target: int, seed: int, abcd=(0.57, 0.19, 0.19, 0.05),
              labels_seed: Optional[int] = None, n_labels: int = 1, name: str = "") -> Graph:
    """Graph500-style Kronecker graph, random vertex permutation, exactly n_edges_target edges."""
    n = 1 << scale
    a, b, c, _ = abcd
    rng = np.random.default_rng(seed)
    perm = rng.permutation(n).astype(np.int64)

    def draw_pairs(r: np.random.Generator, size: int):
        u = np.zeros(size, np.int64)
        v = np.zeros(size, np.int64)
        for lvl in range(scale):
            x = r.random(size)
            ubit = x >= (a + b)
            vbit = ((x >= a) & (x < a + b)) | (x >= a + b + c)
            u |= ubit.astype(np.int64) << lvl
            v |= vbit.astype(np.int64) << lvl
        return perm[u], perm[v]

    keys = np.zeros(0, np.int64)
    while keys.shape[0] < n_edges_target:
        need = n_edges_target - keys.shape[0]
        total = int(need * 1.3) + 1024
        parts = []
        for c0 in range(0, total, 1 << 24):  # bounded memory per chunk
            pu, pv = draw_pairs(rng, min(1 << 24, total - c0))
            ok = pu != pv
            pu, pv = pu[ok], pv[ok]
            parts.append(_sorted_unique(np.minimum(pu, pv) * n + np.maximum(pu, pv)))
        keys = _sorted_unique(np.concatenate([keys] + parts))
    if keys.shape[0] > n_edges_target:
        keys = keys[np.sort(rng.choice(keys.shape[0], size=n_edges_target, replace=False))]
    labels = uniform_labels(n, n_labels, labels_seed) if n_labels > 1 else None
    return make_graph(n, keys // n, keys % n, labels, n_labels, name or f"kron{scale}")


def ring_graph(n: int) -> Graph:
    i = np.arange(n)
    return make_graph(n, i, (i + 1) % n, None, 1, f"ring{n}")


def grid_graph(a: int, b: int) -> Graph:
    u, v = [], []
    for r in range(a):
        for c in range(b):
            x = r * b + c
            if c + 1 < b:
                u.append(x); v.append(x + 1)
            if r + 1 < a:
                u.append(x); v.append(x + b)
    return make_graph(a * b, np.array(u), np.array(v), None, 1, f"grid{a}x{b}")


def complete_graph(n: int) -> Graph:
    u, v = np.triu_indices(n, 1)
    return make_graph(n, u, v, None, 1, f"K{n}")


def regular_circulant(n: int, k: int) -> Graph:
    """2k-regular circulant graph C_n(1..k) (used for regular-star closed forms)."""
    i = np.arange(n)
    us, vs = [], []
    for s in range(1, k + 1):
        us.append(i); vs.append((i + s) % n)
    return make_graph(n, np.concatenate(us), np.concatenate(vs), None, 1, f"circ{n}_{k}")


def random_small_graph(n: int, p: float, n_labels: int, seed: int) -> Graph:
    rng = np.random.default_rng(seed)
    u, v = np.triu_indices(n, 1)
    keep = rng.random(u.shape[0]) < p
    labels = rng.integers(0, n_labels, size=n).astype(np.int32)
    return make_graph(n, u[keep], v[keep], labels, n_labels, f"rnd{n}_{seed}")


# --------------------------------------------------------------------------
# queries and matching orders
# --------------------------------------------------------------------------
def query_from_edges(nq: int, edges: Sequence[Tuple[int, int]], labels: Optional[Sequence[int]] = None,
                     order: Optional[Sequence[int]] = None, name: str = "") -> Query:
    adj = np.zeros((nq, nq), np.uint8)
    for a, b in edges:
        if a == b:
            raise ValueError("self loop in query")
        adj[a, b] = adj[b, a] = 1
    lab = np.zeros(nq, np.int32) if labels is None else np.asarray(labels, np.int32)
    q = Query(adj, lab, np.arange(nq, dtype=np.int32), name)
    return q.with_order(order if order is not None else greedy_order(q))


def path_query(k: int, labels=None) -> Query:
    return query_from_edges(k, [(i, i + 1) for i in range(k - 1)], labels, list(range(k)), f"P{k}")


def cycle_query(k: int, labels=None) -> Query:
    return query_from_edges(k, [(i, (i + 1) % k) for i in range(k)], labels, list(range(k)), f"C{k}")


def star_query(s: int, labels=None) -> Query:
    """K_{1,s}: centre 0, leaves 1..s."""
    return query_from_edges(s + 1, [(0, i) for i in range(1, s + 1)], labels, list(range(s + 1)), f"S{s}")


def clique_query(k: int, labels=None) -> Query:
    return query_from_edges(k, [(a, b) for a in range(k) for b in range(a + 1, k)], labels,
                            list(range(k)), f"K{k}")


def named_small_queries() -> List[Query]:
    """Shapes used in C0: P4, K1,3, C4, paw, diamond, K4 (4 vertices)."""
    return [
        query_from_edges(4, [(0, 1), (1, 2), (2, 3)], name="P4"),
        query_from_edges(4, [(0, 1), (0, 2), (0, 3)], name="K13"),
        query_from_edges(4, [(0, 1), (1, 2), (2, 3), (3, 0)], name="C4"),
        query_from_edges(4, [(0, 1), (1, 2), (2, 0), (2, 3)], name="paw"),
        query_from_edges(4, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 0)], name="diamond"),
        query_from_edges(4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)], name="K4"),
    ]


def greedy_order(q: Query) -> List[int]:
    """QuickSI-like connected order (input preparation, not the method).

    Start at the max-degree vertex (ties: smallest id); then repeatedly take the
    unmatched vertex with the most edges into the matched prefix (ties: larger
    degree, then smaller id).  Every prefix is connected when q is connected.
    """
    nq = q.nq
    deg = q.adj.sum(axis=1)
    first = int(np.lexsort((np.arange(nq), -deg))[0])
    order = [first]
    used = {first}
    while len(order) < nq:
        best = None
        for u in range(nq):
            if u in used:
                continue
            back = int(sum(q.adj[u, w] for w in order))
            if back == 0:
                continue
            keyv = (back, int(deg[u]), -u)
            if best is None or keyv > best[0]:
                best = (keyv, u)
        if best is None:
            raise ValueError("query is not connected")
        order.append(best[1])
        used.add(best[1])
    return order


def random_connected_order(q: Query, seed: int) -> List[int]:
    rng = np.random.default_rng(seed)
    nq = q.nq
    order = [int(rng.integers(nq))]
    while len(order) < nq:
        frontier = sorted({u for u in range(nq) if u not in order and any(q.adj[u, w] for w in order)})
        if not frontier:
            raise ValueError("query is not connected")
        order.append(int(frontier[rng.integers(len(frontier))]))
    return order


def random_connected_query(nq: int, extra_edge_p: float, n_labels: int, seed: int) -> Query:
    """Random tree on nq vertices plus each remaining pair with prob extra_edge_p."""
    rng = np.random.default_rng(seed)
    edges = set()
    for i in range(1, nq):
        j = int(rng.integers(i))
        edges.add((j, i))
    for a in range(nq):
        for b in range(a + 1, nq):
            if (a, b) not in edges and rng.random() < extra_edge_p:
                edges.add((a, b))
    labels = rng.integers(0, n_labels, size=nq)
    q = query_from_edges(nq, sorted(edges), labels, list(range(nq)), f"rq{nq}_{seed}")
    return q.with_order(random_connected_order(q, seed + 7))


def extract_query(g: Graph, k: int, seed: int, dense: bool, max_tries: int = 1000,
                  require_dense: bool = False, min_non_tree: int = 0) -> Query:
    """Random-walk query extraction.

    dense=True : random walk until k distinct vertices, query = induced subgraph;
                 with require_dense, walks are retried until the query's maximum
                 degree is >= 3 (the paper's dense/sparse split).
                 min_non_tree retries until |E_q| - (k - 1) >= min_non_tree (cyclic
                 queries, where Alley's intersections do real work).
    dense=False: self-avoiding walk of k vertices, query = the walk path
                 (max degree 2 < 3, "sparse" per P:L1055).
    Labels are copied from the data vertices, so the count is >= 1.
    """
    rng = np.random.default_rng(seed)
    deg = g.degree()
    cand_start = np.nonzero(deg > 0)[0]
    for _ in range(max_tries):
        start = int(cand_start[rng.integers(cand_start.shape[0])])
        verts = [start]
        tree_edges = []
        cur = start
        steps = 0
        ok = True
        while len(verts) < k:
            steps += 1
            if steps > 50 * k:
                ok = False
                break
            nb = g.neighbors(cur)
            if dense:
                nxt = int(nb[rng.integers(nb.shape[0])])
                if nxt not in verts:
                    tree_edges.append((verts.index(cur), len(verts)))
                    verts.append(nxt)
                cur = nxt
            else:
                free = [int(x) for x in nb if int(x) not in verts]
                if not free:
                    ok = False
                    break
                nxt = free[rng.integers(len(free))]
                tree_edges.append((len(verts) - 1, len(verts)))
                verts.append(nxt)
                cur = nxt
        if not ok:
            continue
        if dense:
            edges = []
            vs = np.asarray(verts)
            for a in range(k):
                nb = set(g.neighbors(int(vs[a])).tolist())
                for b in range(a + 1, k):
                    if int(vs[b]) in nb:
                        edges.append((a, b))
            if require_dense:
                degs = np.zeros(k, np.int64)
                for a, b in edges:
                    degs[a] += 1
                    degs[b] += 1
                if degs.max() < 3:
                    continue
            if len(edges) - (k - 1) < min_non_tree:
                continue
        else:
            edges = tree_edges
        labels = g.labels[np.asarray(verts)]
        q = query_from_edges(k, edges, labels, None, f"{'dense' if dense else 'sparse'}{k}_s{seed}")
        return q
    raise RuntimeError("query extraction failed")


# --------------------------------------------------------------------------
# named workloads (BASELINE.json configs)
# --------------------------------------------------------------------------
def config_c0() -> Tuple[Graph, List[Query]]:
    """C0: ER G(1000, 5000) seed 1, 4 uniform labels seed 2, 4-vertex queries."""
    g = erdos_renyi(1000, 5000, seed=1, n_labels=4, label_seed=2, name="C0_er1k")
    qs = [extract_query(g, 4, seed=s, dense=True) for s in range(10, 15)]
    # the named shapes, labelled from an instance found by a dense extraction
    for i, shape in enumerate(named_small_queries()):
        lab = extract_query(g, 4, seed=100 + i, dense=True).labels
        qs.append(Query(shape.adj, lab.copy(), shape.order, shape.name))
    return g, qs


def config_c1() -> Tuple[Graph, List[Query]]:
    """C1: eu2005-shaped Chung-Lu (|V|=862,664, |E|=16,138,468), unlabelled, 8-vertex queries:
    sparse (a path), dense (the bench's headline query) and cyclic (>= 3 non-tree edges)."""
    g = chung_lu(862_664, 16_138_468, gamma=2.1, max_over_mean=68_963 / 37.4, seed=2005, name="C1_eu2005")
    qs = [extract_query(g, 8, seed=20, dense=False), extract_query(g, 8, seed=21, dense=True, require_dense=True),
          # cyclic: >= 3 non-tree edges, so several positions intersect two or more lists
          extract_query(g, 8, seed=22, dense=True, min_non_tree=3)._renamed("cyclic8_s22")]
    return g, qs


def config_c2() -> Tuple[Graph, List[Query]]:
    """C2: WordNet-shaped Chung-Lu (|V|=76,853, |E|=120,399), 5 skewed labels, 8-vertex dense."""
    n = 76_853
    lab = skewed_labels(n, (0.60, 0.20, 0.10, 0.06, 0.04), seed=5)
    g = chung_lu(n, 120_399, gamma=2.5, max_over_mean=300.0, seed=76_853, labels=lab, n_labels=5,
                 name="C2_wordnet")
    qs = [extract_query(g, 8, seed=s, dense=True, require_dense=True) for s in (30, 31, 32)]
    return g, qs


def config_c3() -> Tuple[Graph, List[Query]]:
    """C3: LiveJournal-shaped Chung-Lu (|V|=4,847,571, |E|=42,851,237), 16 uniform labels, 12-vertex."""
    n = 4_847_571
    lab = uniform_labels(n, 16, seed=16)
    g = chung_lu(n, 42_851_237, gamma=2.4, max_over_mean=20_000 / 17.7, seed=4847, labels=lab, n_labels=16,
                 name="C3_lj")
    qs = [extract_query(g, 12, seed=s, dense=d, require_dense=d) for s, d in ((40, False), (41, False), (42, True),
                                                                             (43, True))]
    return g, qs


def star_query_from(g: Graph, s: int, seed: int) -> Query:
    """K_{1,s} labelled from a data vertex of degree >= s and s of its neighbours."""
    rng = np.random.default_rng(seed)
    deg = g.degree()
    cand = np.nonzero(deg >= s)[0]
    v = int(cand[rng.integers(cand.shape[0])])
    nb = rng.choice(g.neighbors(v), size=s, replace=False)
    labels = [int(g.labels[v])] + [int(g.labels[w]) for w in nb]
    return star_query(s, labels).with_order(list(range(s + 1)))._renamed(f"star{s}_s{seed}")


def config_c4(scale: int = 23, n_edges: int = 100_000_000, sizes=(4, 6, 8, 10, 12, 14, 16)):
    """C4: Graph500 Kronecker (0.57, 0.19, 0.19, 0.05), 2^scale vertices, exactly n_edges
    undirected edges, random vertex permutation (seed 500), 16 uniform labels (seed 16);
    queries: for each size k a labelled path (sparse) and a dense random-walk query, plus
    labelled stars K_{1,3..5} (exact counts by closed form)."""
    g = kronecker(scale, n_edges, seed=500, n_labels=16, labels_seed=16, name=f"C4_kron{scale}")
    qs = []
    for k in sizes:
        qs.append(extract_query(g, k, seed=4000 + k, dense=False))
        qs.append(extract_query(g, k, seed=5000 + k, dense=True, require_dense=True))
    qs += [star_query_from(g, s, 6000 + s) for s in (3, 4, 5)]
    return g, qs


CONFIGS = {"C0": config_c0, "C1": config_c1, "C2": config_c2, "C3": config_c3, "C4": config_c4}
