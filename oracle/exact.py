"""Exact quantities that pin the oracle — TEST INFRASTRUCTURE ONLY (pure Python).

* brute_force_count: the estimand written out as its plain definition (reading A1):
  the number of injective maps f: V_q -> V_G with L(f(u)) = L_q(u) and every query
  edge mapped onto a data edge (non-induced).  itertools over all vertex tuples;
  only for tiny graphs (n <= ~10).
* tree_walk: expands EVERY branch of the sampler's own candidate-set construction
  (SURVEY §8(c) R2-R5, P:L538 WanderJoin, P:L540 Alley) with exact rational
  probabilities.  Unbiasedness of the HT estimator (Eq. 1) means
  sum over complete leaves of P(leaf) * W(leaf) equals brute_force_count exactly;
  sum P * W^2 gives E[Y^2] and hence the exact variance of one sample.  It also
  returns |C_d| for every reachable prefix, so oracle records can be checked node by
  node.
Neither function shares code with oracle.c or with the CUDA path.
"""
from __future__ import annotations

import itertools
from fractions import Fraction
from typing import Dict, Tuple


def _adjacency_sets(g):
    return [set(int(x) for x in g.col[g.row_ptr[v]:g.row_ptr[v + 1]]) for v in range(g.n)]


def brute_force_count(g, q) -> int:
    adj = _adjacency_sets(g)
    lab = [int(x) for x in g.labels]
    qlab = [int(x) for x in q.labels]
    edges = q.edges()
    count = 0
    for f in itertools.permutations(range(g.n), q.nq):
        if any(lab[f[u]] != qlab[u] for u in range(q.nq)):
            continue
        if all(f[b] in adj[f[a]] for a, b in edges):
            count += 1
    return count


def candidate_sets(g, q, filter: int = 0):
    """Global candidate sets C(u) (Def. 4) written out from their definitions:
    0 label; 1 + deg(v) >= deg_q(u) (LDF); 2 + |N_l(v)| >= |N_l^q(u)| for every label l
    (NLF) — DESIGN.md readings A2, A21."""
    adj = _adjacency_sets(g)
    lab = [int(x) for x in g.labels]
    out = []
    for u in range(q.nq):
        qn = [w for w in range(q.nq) if q.adj[u, w]]
        need = {}
        for w in qn:
            need[int(q.labels[w])] = need.get(int(q.labels[w]), 0) + 1
        cu = set()
        for v in range(g.n):
            if lab[v] != int(q.labels[u]):
                continue
            if filter >= 1 and len(adj[v]) < len(qn):
                continue
            if filter >= 2 and any(sum(1 for x in adj[v] if lab[x] == l) < c for l, c in need.items()):
                continue
            cu.add(v)
        out.append(cu)
    return out


def embeddings(g, q):
    """All embeddings as tuples f[u] (brute force, tiny graphs only)."""
    adj = _adjacency_sets(g)
    lab = [int(x) for x in g.labels]
    edges = q.edges()
    return [f for f in itertools.permutations(range(g.n), q.nq)
            if all(lab[f[u]] == int(q.labels[u]) for u in range(q.nq)) and all(f[b] in adj[f[a]] for a, b in edges)]


def tree_walk(g, q, method: int, filter: int = 0,
              variant: int = 0) -> Tuple[Fraction, Fraction, Dict[tuple, Tuple[int, ...]]]:
    """Returns (E[Y], E[Y^2], cand) where cand[prefix] = the candidate list C_d the
    sampler draws from after matching `prefix` (len(prefix) = d).
    variant bits (readings A3 / A5): 2 = WanderJoin walks from the first backward
    position's list; 4 = Alley keeps matched vertices in C_d and a drawn one ends the sample
    (Fig. 19 DupCheck after Sample)."""
    adj = _adjacency_sets(g)
    order = [int(x) for x in q.order]
    nq = q.nq
    csets = candidate_sets(g, q, filter)
    cand: Dict[tuple, Tuple[int, ...]] = {}

    def local(v: int, u: int):  # C(u', u, v) = N(v) ∩ C(u)
        return sorted(w for w in adj[v] if w in csets[u])

    def candidates(prefix: tuple):
        d = len(prefix)
        u = order[d]
        if d == 0:
            return sorted(csets[u]), None
        back = [j for j in range(d) if q.adj[order[j], u]]
        lists = [local(prefix[j], u) for j in back]
        p = min(range(len(back)), key=lambda b: (len(lists[b]), b))
        if method == 0:  # WanderJoin: the smallest local list (or the first one), unfiltered
            if variant & 2:
                p = 0
            return lists[p], (back, lists, p)
        inter = [x for x in lists[p] if all(x in set(lists[b]) for b in range(len(back)))
                 and (variant & 4 or x not in prefix)]
        return inter, None

    ey = Fraction(0)
    ey2 = Fraction(0)
    stack = [((), Fraction(1), 1)]
    while stack:
        prefix, prob, w = stack.pop()
        d = len(prefix)
        if d == nq:
            ey += prob * w
            ey2 += prob * w * w
            continue
        c, info = candidates(prefix)
        cand[prefix] = tuple(c)
        if not c:
            continue
        w2 = w * len(c)
        p2 = prob / len(c)
        for v in c:
            if method == 0 and d > 0:
                back, lists, p = info
                if v in prefix:
                    continue
                if any(v not in set(lists[b]) for b in range(len(back)) if b != p):
                    continue
            if method == 1 and variant & 4 and v in prefix:
                continue  # the post-sampling DupCheck kills the sample
            stack.append((prefix + (v,), p2, w2))
    return ey, ey2, cand


def is_embedding_prefix(g, q, path) -> bool:
    """True iff path[0..len-1] is an injective, label- and edge-preserving partial
    match of phi[0..len-1] (Def. 3 partial instance)."""
    adj = _adjacency_sets(g) if not hasattr(g, "_adjsets") else g._adjsets
    order = [int(x) for x in q.order]
    if len(set(path)) != len(path):
        return False
    for i, v in enumerate(path):
        if int(g.labels[v]) != int(q.labels[order[i]]):
            return False
        for j in range(i):
            if q.adj[order[j], order[i]] and path[j] not in adj[v]:
                return False
    return True


def trawl_d_probs(nq: int):
    """P(d = j) proportional to 2^-j for j in [3, nq]; d = nq when nq <= 3."""
    if nq <= 3:
        return {nq: Fraction(1)}
    w = {j: Fraction(1, 2 ** j) for j in range(3, nq + 1)}
    z = sum(w.values())
    return {j: x / z for j, x in w.items()}


def trawl_expectation(g, q, method: int, filter: int = 0) -> Fraction:
    """E[T] of the trawling estimator (Alg. 4) computed exactly: sum over d of P(d) times the
    sum over sampled prefixes s of length d of P(s) * W(s) * cnt(s), where cnt(s) counts the
    embeddings whose first d matched vertices are s (brute force)."""
    order = [int(x) for x in q.order]
    embs = embeddings(g, q)
    _, _, cand = tree_walk(g, q, method, filter)
    adj = _adjacency_sets(g)
    total = Fraction(0)
    for d, pd in trawl_d_probs(q.nq).items():
        # enumerate the sampler's prefixes of length d with their probability and weight
        stack = [((), Fraction(1), 1)]
        while stack:
            prefix, prob, w = stack.pop()
            if len(prefix) == d:
                cnt = sum(1 for f in embs if all(f[order[i]] == prefix[i] for i in range(d)))
                total += pd * prob * w * cnt
                continue
            c = cand.get(prefix, ())
            if not c:
                continue
            for v in c:
                if method == 0 and len(prefix) > 0:  # WanderJoin: Validate the drawn vertex
                    u = order[len(prefix)]
                    if v in prefix or any(q.adj[order[j], u] and v not in adj[prefix[j]] for j in range(len(prefix))):
                        continue
                stack.append((prefix + (v,), prob / len(c), w * len(c)))
    return total


def inheritance_expectation_check(g, q, method, seed_values, count, inherit_fn):
    """Helper for tests: mean of the inheritance estimator over several seeds."""
    return [inherit_fn(g, q, method, s, 0, count)["estimate"] for s in seed_values]


def alley_candidates(g, q, prefix, adj=None):
    """The Alley candidate set C_d after matching `prefix` (label-only filter), written out
    from its definition: the data vertices with label L_q(phi[d]) that
    are adjacent to the match of every backward query neighbour and not already matched,
    ascending.  Independent of the choice of driver list."""
    adj = adj if adj is not None else _adjacency_sets(g)
    order = [int(x) for x in q.order]
    d = len(prefix)
    u = order[d]
    want = int(q.labels[u])
    back = [j for j in range(d) if q.adj[order[j], u]]
    if d == 0:
        return [v for v in range(g.n) if int(g.labels[v]) == want]
    common = set(adj[prefix[back[0]]])
    for j in back[1:]:
        common &= adj[prefix[j]]
    return sorted(v for v in common if int(g.labels[v]) == want and v not in prefix)
