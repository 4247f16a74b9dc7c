"""GPU parity of the warp-streaming comparison mode (GSWORD_OPT_STREAMING, Alg. 3,
P:L914-L968; reading A25) against the oracle's streaming selection: per-sample
records bit-exact, aggregates within 1e-12, with every schedule and under a candidate
filter.  The graphs include driver lists well above 32 so both phases of Alg. 3 (the
warp-collaborative chunks and the per-lane tail) run."""
import numpy as np
import pytest

import oracle
from workloads import gen

pytestmark = pytest.mark.gpu

REL = 1e-12
S = oracle.SELECT_STREAM


@pytest.fixture(scope="module")
def G():
    import paper_journals_pacmmod_yelsg24_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    c = G.Context(0)
    c.set_option(G.OPT_STREAMING, 1)
    yield c
    c.close()


def _check(ctx, g, q, method, seed, first, count, filt=0, threads=8):
    ctx.load_query_obj(q)
    rec = ctx.trace_samples(method, first, count, seed)
    y, ref = oracle.sample_range(g, q, method, seed, first, count, records=True, threads=threads, filter=filt,
                                 select=S)
    if rec.tobytes() != ref.tobytes():
        diff = np.nonzero([rec[i].tobytes() != ref[i].tobytes() for i in range(count)])[0]
        i = int(diff[0])
        raise AssertionError(f"{g.name}/{q.name}/m{method}: {diff.size} records differ; first sid "
                             f"{int(ref['sample_id'][i])}: gpu={rec[i]} oracle={ref[i]}")
    agg = ctx.estimate(method, count, seed, first=first)
    ra = oracle.aggregate(y)
    assert agg["n"] == ra["n"] and agg["n_valid"] == ra["n_valid"]
    for k in ("sum", "sumsq"):
        assert agg[k] == pytest.approx(ra[k], rel=REL, abs=0.0), k
    return rec


def _long_list_cases():
    dense = gen.erdos_renyi(150, 5600, seed=3)
    cases = [(gen.complete_graph(75), [gen.clique_query(3), gen.clique_query(5)]),
             (dense, [gen.clique_query(3), gen.extract_query(dense, 5, seed=8, dense=True),
                      gen.extract_query(dense, 6, seed=9, dense=False)]),
             (gen.regular_circulant(80, 20), [gen.star_query(3), gen.path_query(5)])]
    for s in range(3):
        g = gen.random_small_graph(44, 0.85, n_labels=1 + s % 2, seed=500 + s)
        cases.append((g, [gen.random_connected_query(3 + s, 0.5, g.n_labels, 600 + s)]))
    return cases


def test_streaming_parity_long_lists(ctx, G):
    for g, qs in _long_list_cases():
        ctx.load_graph_obj(g)
        for i, q in enumerate(qs):
            _check(ctx, g, q, G.ALLEY, seed=3 + i, first=11, count=20_000)


def test_streaming_parity_c0_and_wj_unchanged(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        _check(ctx, g, q, G.ALLEY, seed=1 + i, first=0, count=50_000)
    # WanderJoin has no refine stage: the option leaves it byte-identical to the plain sampler
    q = qs[0]
    ctx.load_query_obj(q)
    rec = ctx.trace_samples(G.WJ, 0, 20_000, 5)
    _, ref = oracle.sample_range(g, q, G.WJ, 5, 0, 20_000)
    assert rec.tobytes() == ref.tobytes()


def test_streaming_parity_filtered(ctx, G, c0):
    g, qs = c0
    ctx.set_option(G.OPT_FILTER, G.FILTER_NLF)
    try:
        ctx.load_graph_obj(g)
        for i, q in enumerate(qs[:5]):
            _check(ctx, g, q, G.ALLEY, seed=7 + i, first=0, count=30_000, filt=2)
        dense = gen.erdos_renyi(150, 5600, seed=3, n_labels=2, label_seed=4)
        ctx.load_graph_obj(dense)
        q = gen.extract_query(dense, 5, seed=8, dense=True)
        _check(ctx, dense, q, G.ALLEY, seed=2, first=0, count=20_000, filt=2)
    finally:
        ctx.set_option(G.OPT_FILTER, 0)


def test_streaming_parity_c2_c1(ctx, G):
    g, qs = gen.config_c2()
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        _check(ctx, g, q, G.ALLEY, seed=10 + i, first=0, count=30_000)
    g, qs = gen.config_c1()
    ctx.load_graph_obj(g)
    for q in qs:
        _check(ctx, g, q, G.ALLEY, seed=42, first=0, count=4_000, threads=16)
        _check(ctx, g, q, G.ALLEY, seed=42, first=77_000_000, count=2_000, threads=16)


def test_streaming_sample_sync_and_inheritance(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_SCHEDULE, G.SCHED_SAMPLE_SYNC)
    try:
        for i, q in enumerate(qs[:3]):
            _check(ctx, g, q, G.ALLEY, seed=21 + i, first=5, count=30_000)
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_INHERIT)
        dense = gen.erdos_renyi(150, 5600, seed=3)
        for gg, q in [(g, qs[0]), (g, qs[3]), (dense, gen.extract_query(dense, 5, seed=8, dense=True))]:
            ctx.load_graph_obj(gg)
            ctx.load_query_obj(q)
            for first, count in ((0, 64_000), (7, 10_013)):
                r = ctx.estimate(G.ALLEY, count, 31, first=first)
                ref = oracle.inherit_range(gg, q, G.ALLEY, 31, first, count, select=S)
                assert r["n"] == count and r["n_valid"] == ref["n_valid"], q.name
                assert r["sum"] == pytest.approx(ref["sum"], rel=REL, abs=1e-300)
                assert r["sumsq"] == pytest.approx(ref["sumsq"], rel=REL, abs=1e-300)
    finally:
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)


def test_streaming_matches_plain_in_distribution(ctx, G, c0):
    """Same estimator, different draws: streaming and count-then-index Alley estimates of
    the same query agree within their combined 5 sigma, and |C_d| statistics coincide."""
    g, qs = c0
    ctx.load_graph_obj(g)
    q = qs[2]
    ctx.load_query_obj(q)
    a = ctx.estimate(G.ALLEY, 2_000_000, 9)
    ctx.set_option(G.OPT_STREAMING, 0)
    try:
        b = ctx.estimate(G.ALLEY, 2_000_000, 9)
    finally:
        ctx.set_option(G.OPT_STREAMING, 1)
    assert abs(a["estimate"] - b["estimate"]) <= 5 * np.sqrt(a["variance"] + b["variance"]) + 1e-9
