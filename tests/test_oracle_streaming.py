"""Pins of the oracle's warp-streaming selection (Alg. 3; reading A25).

Warp streaming changes WHICH vertex of the Alley candidate set C_d a sample draws (a
weighted reservoir over 32-candidate chunks instead of count-then-index), not the set
itself nor the weight |C_d|.  Theorem 2 says the pick is uniform over C_d.  The
pins: closed forms that hold for any pick, every record against C_d written out from its
definition (oracle/exact.py), chi-square uniformity of the pick in both phases of Alg. 3
(a reservoir that merges chunks with the wrong probability fails these), and unbiasedness
against exact counts, with and without sample inheritance.
"""
import math

import numpy as np
import pytest
from scipy import stats

import oracle
from oracle import exact
from workloads import gen

S = oracle.SELECT_STREAM


def _falling(n, k):
    out = 1
    for i in range(k):
        out *= n - i
    return out


def test_stream_zero_variance_closed_forms():
    # K_40 / 4-clique: driver lists of 39 (one collaborative chunk + 7 independent)
    y, rec = oracle.sample_range(gen.complete_graph(40), gen.clique_query(4), oracle.ALLEY, 3, 0, 400, select=S)
    assert np.all(rec["valid"] == 1) and np.all(y == _falling(40, 4))
    assert np.all(rec["csize"][:, :4] == np.array([40, 39, 38, 37]))
    assert all(len(set(r["path"][:4].tolist())) == 4 for r in rec)
    # ring / path: lists of 2 (independent phase only)
    y, _ = oracle.sample_range(gen.ring_graph(30), gen.path_query(9), oracle.ALLEY, 5, 17, 300, select=S)
    assert np.all(y == 60)
    # 40-regular circulant, star K_{1,3}: n * 40 * 39 * 38 for every sample
    g = gen.regular_circulant(80, 20)
    y, _ = oracle.sample_range(g, gen.star_query(3), oracle.ALLEY, 9, 0, 300, select=S)
    assert np.all(y == 80 * _falling(40, 3))


def _chi2_uniform_p(ranks, k):
    counts = np.bincount(ranks, minlength=k)
    return stats.chisquare(counts).pvalue


def test_stream_pick_uniform_complete_graph():
    """K_75 / triangle: C_1 = N(M0) (74 = 2 chunks + 10 independent), C_2 = 73.  The rank of
    the pick in C_d must be uniform (Theorem 2)."""
    n, count = 75, 40_000
    _, rec = oracle.sample_range(gen.complete_graph(n), gen.clique_query(3), oracle.ALLEY, 7, 0, count, select=S)
    p = rec["path"][:, :3].astype(np.int64)
    assert np.all(rec["csize"][:, :3] == np.array([75, 74, 73]))
    r1 = p[:, 1] - (p[:, 1] > p[:, 0])
    r2 = p[:, 2] - (p[:, 2] > p[:, 0]) - (p[:, 2] > p[:, 1])
    assert r1.min() >= 0 and r1.max() < 74 and r2.max() < 73
    assert _chi2_uniform_p(r1, 74) > 1e-4
    assert _chi2_uniform_p(r2, 73) > 1e-4
    # the first chunk, the second chunk and the independent tail are each hit in proportion
    assert abs(np.mean(r1 < 32) - 32 / 74) < 0.02 and abs(np.mean(r1 >= 64) - 10 / 74) < 0.02


def test_stream_pick_uniform_with_refine_survivors():
    """Dense random graph / triangle: at d = 2 only ~half of the driver survives refine, so
    chunks carry different total weights.  Every pick lies in C_2 (from the definition),
    csize = |C_2|, and the randomised rank (rank + U) / |C_2| is Uniform(0, 1)."""
    g = gen.erdos_renyi(150, 5600, seed=3)
    q = gen.clique_query(3)
    _, rec = oracle.sample_range(g, q, oracle.ALLEY, 11, 0, 20_000, select=S)
    adj = [set(g.col[g.row_ptr[v]:g.row_ptr[v + 1]].tolist()) for v in range(g.n)]
    rng = np.random.default_rng(0)
    u = []
    for r in rec:
        if r["depth_reached"] < 2 or r["csize"][2] == 0:
            continue
        prefix = (int(r["path"][0]), int(r["path"][1]))
        c2 = exact.alley_candidates(g, q, prefix, adj)
        assert int(r["csize"][2]) == len(c2)
        k = c2.index(int(r["path"][2]))
        u.append((k + rng.random()) / len(c2))
    assert len(u) > 15_000
    counts = np.histogram(u, bins=20, range=(0.0, 1.0))[0]
    assert stats.chisquare(counts).pvalue > 1e-4


@pytest.mark.parametrize("seed", range(4))
def test_stream_records_follow_definition(seed):
    g = gen.random_small_graph(44, 0.85, n_labels=1 + seed % 2, seed=500 + seed)
    q = gen.random_connected_query(3 + seed % 3, 0.5, g.n_labels, 600 + seed)
    _, rec = oracle.sample_range(g, q, oracle.ALLEY, seed, 0, 400, select=S)
    adj = [set(g.col[g.row_ptr[v]:g.row_ptr[v + 1]].tolist()) for v in range(g.n)]
    for r in rec:
        dr = int(r["depth_reached"])
        w = 1.0
        for d in range(dr + 1):
            c = exact.alley_candidates(g, q, tuple(int(x) for x in r["path"][:d]), adj)
            assert int(r["csize"][d]) == len(c)
            w *= len(c)
            assert (int(r["path"][d]) in c) if c else int(r["path"][d]) == -1
        assert r["weight"] == w
        assert bool(r["valid"]) == (dr == q.nq - 1 and int(r["csize"][dr]) > 0)


def test_stream_z_scores_tiny():
    g = gen.random_small_graph(9, 0.5, n_labels=2, seed=77)
    q = gen.extract_query(g, 4, seed=78, dense=True)
    ey, ey2, _ = exact.tree_walk(g, q, oracle.ALLEY)
    truth = exact.brute_force_count(g, q)
    assert ey == truth and truth > 0
    var1 = float(ey2 - ey * ey)
    zs = []
    for seed in range(30):
        y, _ = oracle.sample_range(g, q, oracle.ALLEY, seed, 0, 3000, records=False, select=S)
        zs.append((y.mean() - truth) / math.sqrt(var1 / 3000) if var1 > 0 else 0.0)
    zs = np.array(zs)
    assert np.all(np.abs(zs) < 5) and abs(zs.mean()) < 5 / math.sqrt(30)


def test_stream_unbiased_long_lists():
    """Lists of ~35 (both phases): mean of 30 estimates within 5 standard errors of the exact
    count (the C enumerator, pinned against brute force in test_oracle_pins)."""
    g = gen.random_small_graph(40, 0.85, n_labels=1, seed=91)
    q = gen.extract_query(g, 4, seed=92, dense=True)
    truth = oracle.count_embeddings(g, q)
    ests = np.array([oracle.estimate(g, q, oracle.ALLEY, s, 2000, select=S)["estimate"] for s in range(30)])
    assert abs(ests.mean() - truth) <= 5 * ests.std(ddof=1) / math.sqrt(len(ests)) + 1e-9


def test_stream_does_not_change_wanderjoin(c0):
    g, qs = c0
    for q in qs[:3]:
        _, a = oracle.sample_range(g, q, oracle.WJ, 4, 0, 2000)
        _, b = oracle.sample_range(g, q, oracle.WJ, 4, 0, 2000, select=S)
        assert a.tobytes() == b.tobytes()


def test_stream_c0_within_3_sigma(c0):
    g, qs = c0
    for q in qs[:4]:
        truth = oracle.count_embeddings(g, q)
        agg = oracle.estimate(g, q, oracle.ALLEY, seed=2, n_samples=100_000, threads=4, select=S)
        sigma = math.sqrt(agg["variance"]) if agg["variance"] > 0 else 0.0
        assert abs(agg["estimate"] - truth) <= 3 * sigma + 1e-9, (q.name, truth, agg)


def test_inheritance_with_streaming_unbiased():
    """The paper's O2 (inheritance + warp streaming, Fig. 12): unbiased (Theorems 1, 2)."""
    g = gen.random_small_graph(40, 0.8, n_labels=2, seed=57)
    q = gen.extract_query(g, 5, seed=58, dense=True)
    truth = oracle.count_embeddings(g, q)
    ests = np.array([oracle.inherit_range(g, q, oracle.ALLEY, s, 0, 1024, select=S)["estimate"]
                     for s in range(40)])
    assert truth > 0
    assert abs(ests.mean() - truth) <= 4 * ests.std(ddof=1) / math.sqrt(len(ests))
