"""Pins of the oracle's algorithmic-sector counter (reading A26).

The per-sample `sectors` field of the oracle's records is checked against hand counts
(tests/golden/sector_model_cases.txt) and against closed forms that follow from the model's
rules on structured inputs (complete graphs, complete tripartite graphs, rings, labelled
stars) — never against a re-implementation of the counter.  The GPU's counting and trace
builds are then compared with this oracle (tests/test_gpu_parity.py).
"""
import math

import numpy as np
import pytest

import oracle
from gsword_testutil import read_golden
from workloads import gen


def tripartite(m):
    n = 3 * m
    u, v = [], []
    for a in range(n):
        for b in range(a + 1, n):
            if a // m != b // m:
                u.append(a)
                v.append(b)
    return gen.make_graph(n, np.array(u), np.array(v), None, 1, name=f"K{m},{m},{m}")


def diamond():
    e = np.array([(0, 1), (0, 2), (1, 2), (1, 3), (2, 3)])
    return gen.make_graph(4, e[:, 0], e[:, 1], None, 1, name="diamond")


def build_graph(spec):
    kind, _, arg = spec.partition(":")
    if kind == "ring":
        return gen.ring_graph(int(arg))
    if kind == "complete":
        return gen.complete_graph(int(arg))
    if kind == "tripartite":
        return tripartite(int(arg))
    if kind == "diamond":
        return diamond()
    raise ValueError(spec)


def build_query(spec):
    kind, _, arg = spec.partition(":")
    return {"path": gen.path_query, "clique": gen.clique_query}[kind](int(arg))


@pytest.mark.parametrize("row", read_golden("sector_model_cases.txt"), ids=lambda r: r[0])
def test_hand_counted_cases(row):
    name, gspec, qspec, meth, filt, rule, val = row
    g, q = build_graph(gspec), build_query(qspec)
    m = {"WJ": oracle.WJ, "AL": oracle.ALLEY}[meth]
    _, rec = oracle.sample_range(g, q, m, seed=5, first=0, count=400, records=True, filter=int(filt))
    sec = rec["sectors"].astype(np.int64)
    if rule == "const":
        assert np.all(sec == int(val)), (name, np.unique(sec))
    else:
        assert rule == "new2"
        new = np.array([p[2] not in (p[0], p[1]) for p in rec["path"]])
        assert np.all(sec == int(val) + new), name
        assert new.any() and (~new).any(), "both branches exercised"


@pytest.mark.parametrize("n,k", [(9, 3), (9, 4), (12, 5), (80, 3), (100, 4)])
def test_alley_clique_closed_form(n, k):
    # K_n, k-clique, Alley: d = 1 costs 2; d >= 2 costs d offsets + ceil((n-1)/8) scan +
    # (n - d) unmatched driver elements x (d - 1) questions that all pass
    want = 2 + sum(d + -(-(n - 1) // 8) + (n - d) * (d - 1) for d in range(2, k))
    _, rec = oracle.sample_range(gen.complete_graph(n), gen.clique_query(k), oracle.ALLEY, 3, 0, 200)
    assert np.all(rec["sectors"] == want)


@pytest.mark.parametrize("n,k", [(6, 3), (9, 4), (30, 5)])
def test_wj_clique_closed_form(n, k):
    # K_n, k-clique, WanderJoin: each position d <= depth reached costs d offsets + the draw
    # + (d - 1) IsEdge questions (all pass) unless DupCheck rejects the draw
    _, rec = oracle.sample_range(gen.complete_graph(n), gen.clique_query(k), oracle.WJ, 4, 0, 2000)
    for r in rec:
        path = list(r["path"])
        want = sum(d + 1 + (d - 1) * (path[d] not in path[:d]) for d in range(1, r["depth_reached"] + 1))
        assert r["sectors"] == want


@pytest.mark.parametrize("m", [2, 5, 17, 40])
def test_tripartite_k4_alley_closed_form(m):
    # every Alley sample of K_4 in K_{m,m,m} dies at d = 3 after 3 + 2 ceil(2m/8) + 5m sectors
    _, rec = oracle.sample_range(tripartite(m), gen.clique_query(4), oracle.ALLEY, 9, 0, 300)
    assert np.all(rec["depth_reached"] == 3) and not rec["valid"].any()
    assert np.all(rec["sectors"] == 3 + 2 * -(-2 * m // 8) + 5 * m)


@pytest.mark.parametrize("n,k", [(10, 4), (12, 7), (40, 9)])
def test_ring_path_closed_form(n, k):
    # ring C_n, path P_k along the order, unlabelled.  Alley: position d costs 1 offset +
    # max(0, d - 2) exclusion questions (j <= d - 3; j = d - 2 is known in S_p) + 1 select;
    # with a candidate graph (LDF keeps every vertex) the known shortcut is gone: d - 1
    # questions.  WanderJoin: 1 offset + 1 draw per position reached.
    g, q = gen.ring_graph(n), gen.path_query(k)
    _, rec = oracle.sample_range(g, q, oracle.ALLEY, 1, 0, 300)
    assert np.all(rec["sectors"] == sum(2 + max(0, d - 2) for d in range(1, k)))
    _, rec = oracle.sample_range(g, q, oracle.ALLEY, 1, 0, 300, filter=oracle.FILTER_LDF)
    assert np.all(rec["sectors"] == sum(d + 1 for d in range(1, k)))
    _, rec = oracle.sample_range(g, q, oracle.WJ, 1, 0, 300)
    assert np.all(rec["sectors"] == 2 * rec["depth_reached"].astype(np.int64))


def test_labelled_star_seed_and_known_exclusions():
    # labelled graph (C(phi[0]) != V: the seed costs 1).  Star with the centre first and two
    # leaves of the same label b: the second b-leaf's exclusion "is M[1] in S_p?" is known
    # (leaf and centre share a query edge) with label-only lists, one question with LDF.
    g = gen.random_small_graph(60, 0.3, 3, seed=77)
    q = gen.star_query(3, labels=[0, 1, 1, 2])  # centre 0 (label 0), leaves 1, 2 (label 1), 3 (label 2)
    for m in (oracle.WJ, oracle.ALLEY):
        for filt in (0, 1):
            _, rec = oracle.sample_range(g, q, m, 11, 0, 3000, filter=filt)
            for r in rec:
                dr = int(r["depth_reached"])
                if r["csize"][0] == 0:
                    assert r["sectors"] == 0
                    continue
                want = 1  # seed
                for d in range(1, dr + 1):
                    want += 1 + (r["csize"][d] > 0)  # offsets + drawn/selected vertex
                    if d == 2 and m == oracle.ALLEY and filt == 1:
                        # the exclusion question about M[1], asked when S_p is not empty
                        c0 = r["path"][0]
                        want += int(any(g.labels[w] == 1 for w in g.neighbors(c0)))
                assert r["sectors"] == want, (m, filt, r)
            assert (rec["depth_reached"] == 3).any()


def test_streaming_is_not_modelled():
    g = gen.complete_graph(12)
    _, rec = oracle.sample_range(g, gen.clique_query(4), oracle.ALLEY, 2, 0, 100, select=oracle.SELECT_STREAM)
    assert np.all(rec["sectors"] == 0)
    _, rec = oracle.sample_range(g, gen.clique_query(4), oracle.WJ, 2, 0, 100, select=oracle.SELECT_STREAM)
    assert np.all(rec["sectors"] > 0)  # streaming leaves WanderJoin unchanged


def test_sector_count_does_not_change_samples():
    # the counter is bookkeeping only: records without it equal the paths/weights pinned
    # elsewhere, and the Y values do not depend on requesting records
    g, qs = gen.config_c0()
    y0, rec = oracle.sample_range(g, qs[2], oracle.ALLEY, 3, 0, 5000, records=True)
    y1, _ = oracle.sample_range(g, qs[2], oracle.ALLEY, 3, 0, 5000, records=False)
    assert np.array_equal(y0, y1)
    assert np.all(rec["pad"] == 0)
    assert math.isfinite(float(rec["sectors"].mean()))
