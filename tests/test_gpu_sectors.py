"""GPU algorithmic-sector counter (reading A26) against the oracle.

The trace build writes each sample's model count into its record (compared byte for byte
with the oracle everywhere in tests/test_gpu_parity.py); here the counting build's range
total (gsword_count_sectors, the number bench.py's roofline uses) must equal the sum of the
oracle's per-sample counts exactly, on the hand-counted cases, C0 and C1 prefixes (all
three C1 queries, the cyclic one included) and under a candidate filter.
"""
import numpy as np
import pytest

import oracle
from workloads import gen

from test_oracle_sectors import build_graph, build_query, tripartite
from gsword_testutil import read_golden

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def G():
    import paper_journals_pacmmod_yelsg24_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    c = G.Context(0)
    yield c
    c.close()


def _check(ctx, g, q, m, seed, first, count, filt=0, threads=8, loaded=False):
    if not loaded:
        ctx.load_graph_obj(g)
    ctx.set_option(7, filt)  # GSWORD_OPT_FILTER
    try:
        ctx.load_query_obj(q)
        model, touched = ctx.count_sectors(m, first, count, seed)
        rec = ctx.trace_samples(m, first, count, seed)
    finally:
        ctx.set_option(7, 0)
    _, ref = oracle.sample_range(g, q, m, seed, first, count, records=True, threads=threads, filter=filt)
    assert np.array_equal(rec["sectors"], ref["sectors"]), f"{g.name}/{q.name}/m{m}: per-sample sectors"
    want = float(ref["sectors"].astype(np.int64).sum())
    assert model == want, f"{g.name}/{q.name}/m{m}: counting build {model} != oracle {want}"
    assert touched > 0
    return want / count, touched / count


@pytest.mark.parametrize("row", read_golden("sector_model_cases.txt"), ids=lambda r: r[0])
def test_hand_counted_cases_on_gpu(ctx, row):
    name, gspec, qspec, meth, filt, rule, val = row
    m = {"WJ": 0, "AL": 1}[meth]
    _check(ctx, build_graph(gspec), build_query(qspec), m, seed=5, first=0, count=3000, filt=int(filt))


def test_structured_cases_on_gpu(ctx):
    for m_ in (2, 40):  # 2m = 80 > 64: the warp-cooperative refine
        _check(ctx, tripartite(m_), gen.clique_query(4), 1, seed=9, first=0, count=5000)
    for n, k in ((9, 4), (100, 4)):
        for m in (0, 1):
            _check(ctx, gen.complete_graph(n), gen.clique_query(k), m, seed=3, first=7, count=5000)


def test_c0_counting_build_equals_oracle(ctx, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        for m in (0, 1):
            _check(ctx, g, q, m, seed=1 + i, first=0, count=20_000, loaded=True)
        _check(ctx, g, q, 1, seed=1 + i, first=0, count=20_000, filt=2, loaded=True)


@pytest.fixture(scope="module")
def c1():
    return gen.config_c1()


def test_c1_counting_build_equals_oracle(ctx, c1):
    g, qs = c1
    ctx.load_graph_obj(g)
    for q in qs:
        for m in (0, 1):
            _check(ctx, g, q, m, seed=42, first=0, count=20_000, loaded=True)
    # deep in the bench's 1e8 range
    ctx.load_query_obj(qs[1])
    for m in (0, 1):
        _check(ctx, g, qs[1], m, seed=42, first=99_990_000, count=10_000, loaded=True)
