"""Pins of the oracle's comparison variants (readings A3 and A5):

* WJ_PARENT_FIRST: WanderJoin walks from the first backward position's local list (the
  "vertex that has been previously selected" of P:L538) instead of GetMinCandidate's
  smallest list (Alg. 1 l.8);
* ALLEY_DUPCHECK_POST: Alley's refined set keeps already-matched vertices and the drawn
  vertex is DupChecked after sampling (Fig. 19 AL Validate).

Both are unbiased; the pins are the exact tree walk (rational E[Y] = brute-force count),
every record against the tree node, and identities that hold on tree-shaped queries.
"""
import math

import numpy as np
import pytest

import oracle
from oracle import exact
from workloads import gen

PF = oracle.VARIANT_WJ_PARENT_FIRST
POST = oracle.VARIANT_ALLEY_DUPCHECK_POST
CASES = [(oracle.WJ, PF), (oracle.ALLEY, POST)]


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("method,variant", CASES)
def test_variant_tree_walk_equals_brute_force(seed, method, variant):
    g = gen.random_small_graph(7, 0.55, n_labels=1 + seed % 2, seed=700 + seed)
    q = gen.random_connected_query(2 + seed % 4, 0.6, g.n_labels, 800 + seed)
    ey, ey2, _ = exact.tree_walk(g, q, method, variant=variant)
    assert ey == exact.brute_force_count(g, q)
    assert ey2 >= ey * ey


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("method,variant", CASES)
@pytest.mark.parametrize("select", [oracle.SELECT_INDEX, oracle.SELECT_STREAM])
def test_variant_records_follow_the_tree(seed, method, variant, select):
    g = gen.random_small_graph(8, 0.55, n_labels=1 + seed % 2, seed=900 + seed)
    q = gen.random_connected_query(3 + seed % 3, 0.6, g.n_labels, 1000 + seed)
    _, _, cand = exact.tree_walk(g, q, method, variant=variant)
    _, rec = oracle.sample_range(g, q, method, seed, 0, 600, select=select, variant=variant)
    for r in rec:
        dr = int(r["depth_reached"])
        w = 1.0
        for d in range(dr + 1):
            c = cand[tuple(int(x) for x in r["path"][:d])]
            assert int(r["csize"][d]) == len(c)
            w *= len(c)
            assert (int(r["path"][d]) in c) if c else int(r["path"][d]) == -1
        assert r["weight"] == w
        full = tuple(int(x) for x in r["path"][:q.nq])
        assert bool(r["valid"]) == (dr == q.nq - 1 and -1 not in full and exact.is_embedding_prefix(g, q, full))


def test_variants_on_tree_queries_reduce_to_wanderjoin(c0):
    """With one backward neighbour per position there is no choice of parent and no
    intersection: WJ_PARENT_FIRST is WanderJoin, and Alley with the post-sampling DupCheck
    draws exactly WanderJoin's vertices (same C_d = N_l(M[parent]), same draw, same
    DupCheck): byte-identical records."""
    g, _ = c0
    for q in (gen.path_query(4, labels=[0, 1, 2, 3]), gen.star_query(3, labels=[1, 0, 0, 2]),
              gen.path_query(6, labels=[0, 0, 1, 1, 0, 0])):
        _, wj = oracle.sample_range(g, q, oracle.WJ, 3, 0, 20_000)
        _, pf = oracle.sample_range(g, q, oracle.WJ, 3, 0, 20_000, variant=PF)
        _, post = oracle.sample_range(g, q, oracle.ALLEY, 3, 0, 20_000, variant=POST)
        assert wj.tobytes() == pf.tobytes() == post.tobytes()
        _, al = oracle.sample_range(g, q, oracle.ALLEY, 3, 0, 20_000)
        assert al["valid"].mean() >= post["valid"].mean()


def test_alley_post_ring_closed_form():
    """Ring C_n, path P_k: every C_d = both ring neighbours (|C_d| = 2), the step back is drawn
    w.p. 1/2 and killed by the DupCheck: valid w.p. 2^-(k-2), W = n 2^(k-1)."""
    n, k = 13, 5
    y, rec = oracle.sample_range(gen.ring_graph(n), gen.path_query(k), oracle.ALLEY, 2, 0, 4000, variant=POST)
    for r in rec:
        dr = int(r["depth_reached"])
        assert list(r["csize"][:dr + 1]) == [n] + [2] * dr
    assert set(np.unique(y).tolist()) <= {0.0, float(n * 2 ** (k - 1))}
    frac = float(np.mean(rec["valid"]))
    assert abs(frac - 2.0 ** -(k - 2)) < 5 * math.sqrt(0.125 * 0.875 / 4000)


def test_parent_first_changes_dense_queries(c0):
    """On a query with several backward neighbours the variant walks other lists: the
    records differ while both estimates stay within 5 sigma of the exact count."""
    g, qs = c0
    q = next(x for x in qs if x.name.startswith("dense"))
    truth = oracle.count_embeddings(g, q)
    _, a = oracle.sample_range(g, q, oracle.WJ, 5, 0, 5000)
    _, b = oracle.sample_range(g, q, oracle.WJ, 5, 0, 5000, variant=PF)
    if any(len([j for j in range(d) if q.adj[q.order[j], q.order[d]]]) > 1 for d in range(1, q.nq)):
        assert a.tobytes() != b.tobytes()
    for v in (0, PF):
        agg = oracle.estimate(g, q, oracle.WJ, 6, 200_000, threads=4, variant=v)
        assert abs(agg["estimate"] - truth) <= 5 * math.sqrt(agg["variance"]) + 1e-9
