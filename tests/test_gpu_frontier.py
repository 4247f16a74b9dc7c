"""The level-synchronous frontier path of the Alley sampler (GSWORD_OPT_PATH = 1,
csrc/gsword_frontier.cu) against the CPU oracle: per-sample records byte for byte (path,
csize, validity, fp64 weight, A26 sectors) through its trace build, aggregates within
1e-12 (BASELINE.json north_star), across batches, under candidate filters, on the
warp-cooperative refine (drivers > 64) and on every config shape; and the autotuned default
is result-identical to both paths."""
import math

import numpy as np
import pytest

import oracle
from gsword_testutil import variance_tolerance
from workloads import gen

from test_oracle_sectors import tripartite

pytestmark = pytest.mark.gpu

REL = 1e-12
ALLEY = 1


@pytest.fixture(scope="module")
def G():
    import paper_journals_pacmmod_yelsg24_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    c = G.Context(0)
    c.set_option(G.OPT_PATH, 1)
    yield c
    c.close()


def _records_equal(gpu, ref, what):
    if gpu.tobytes() == ref.tobytes():
        return
    for f in ("sample_id", "valid", "depth_reached", "sectors", "path", "csize", "weight"):
        bad = np.nonzero(np.any((gpu[f] != ref[f]).reshape(gpu.shape[0], -1), axis=1))[0]
        if bad.size:
            i = int(bad[0])
            raise AssertionError(f"{what}: field {f} differs at {bad.size} samples; first sid "
                                 f"{int(ref['sample_id'][i])}: gpu={gpu[i]} oracle={ref[i]}")
    raise AssertionError(f"{what}: records differ in padding")


def _parity(ctx, g, q, seed, first, count, filt=0, threads=8, loaded=False):
    if not loaded:
        ctx.load_graph_obj(g)
    ctx.set_option(7, filt)
    try:
        ctx.load_query_obj(q)
        assert ctx.query_info()["path"][ALLEY] == (1 if q.nq >= 2 else 0)
        rec = ctx.trace_samples(ALLEY, first, count, seed)
        agg = ctx.estimate(ALLEY, count, seed, first=first)
    finally:
        ctx.set_option(7, 0)
    y, ref = oracle.sample_range(g, q, ALLEY, seed, first, count, records=True, threads=threads, filter=filt)
    _records_equal(rec, ref, f"{g.name}/{q.name}/f{filt}")
    r = oracle.aggregate(y)
    assert agg["n"] == r["n"] and agg["n_valid"] == r["n_valid"]
    for k in ("sum", "sumsq", "estimate"):
        assert agg[k] == pytest.approx(r[k], rel=REL, abs=0.0), k
    if r["n"] >= 2:
        assert abs(agg["variance"] - r["variance"]) <= variance_tolerance(r) + REL * abs(r["variance"])


def test_frontier_c0(ctx, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        _parity(ctx, g, q, seed=1 + i, first=0, count=100_000, loaded=True)


@pytest.mark.parametrize("seed", range(12))
def test_frontier_fuzz_small(ctx, seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(5, 40))
    nl = int(rng.integers(1, 4))
    g = gen.random_small_graph(n, float(rng.uniform(0.2, 0.7)), nl, seed=5000 + seed)
    nq = int(rng.integers(2, min(n, 9) + 1))
    try:
        q = gen.extract_query(g, nq, 6000 + seed, dense=bool(seed % 2))
        q = q.with_order(gen.random_connected_order(q, seed))
    except RuntimeError:
        q = gen.random_connected_query(nq, 0.4, nl, 7000 + seed)
    _parity(ctx, g, q, seed=seed, first=int(rng.integers(0, 2**40)), count=5000)


def test_frontier_batches_and_coop(ctx, G):
    """Batches smaller than the range (2^10 samples), drivers above the cooperative
    threshold (K_100, K_{40,40,40}), a query of two vertices (level 1 is also the last)."""
    ctx.set_option(G.OPT_FRONTIER_BATCH, 1024)
    try:
        _parity(ctx, gen.complete_graph(100), gen.clique_query(4), seed=3, first=11, count=20_000)
        _parity(ctx, tripartite(40), gen.clique_query(4), seed=4, first=0, count=20_000)
        _parity(ctx, gen.complete_graph(9), gen.clique_query(2), seed=5, first=7, count=5000)
        _parity(ctx, gen.ring_graph(50), gen.path_query(9), seed=6, first=0, count=5000)
    finally:
        ctx.set_option(G.OPT_FRONTIER_BATCH, 1 << 22)
    r = ctx.estimate(ALLEY, 50_000, seed=6)
    assert r["n_valid"] == 50_000 and r["estimate"] == 100.0  # ring C_50, P_9: W = 2n, zero variance


@pytest.mark.parametrize("filt", [1, 2])
def test_frontier_filtered(ctx, c0, filt):
    g, qs = c0
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs[:6]):
        _parity(ctx, g, q, seed=20 + i, first=0, count=50_000, filt=filt, loaded=True)


def test_frontier_c1_c2(ctx):
    g, qs = gen.config_c1()
    ctx.load_graph_obj(g)
    for q in qs:
        _parity(ctx, g, q, seed=42, first=0, count=20_000, loaded=True)
        _parity(ctx, g, q, seed=42, first=99_990_000, count=10_000, loaded=True)
    _parity(ctx, g, qs[1], seed=42, first=0, count=20_000, filt=2, loaded=True)
    g, qs = gen.config_c2()
    ctx.load_graph_obj(g)
    for q in qs:
        _parity(ctx, g, q, seed=10, first=0, count=50_000, loaded=True)


def test_frontier_equals_persistent_at_full_size(ctx, G):
    """C1 at the bench's 1e8 budget (25 batches of 2^22): the frontier and the persistent
    kernel give the same aggregate (n and n_valid exact, sums within 1e-12), and the
    autotuned default (whichever path it picks) equals both."""
    g, qs = gen.config_c1()
    ctx.load_graph_obj(g)
    for q in qs[1:]:
        ctx.load_query_obj(q)
        n = 100_000_000 if q.name.startswith("dense") else 20_000_000
        fr = ctx.estimate(ALLEY, n, 42)
        ctx.set_option(G.OPT_PATH, 0)
        pe = ctx.estimate(ALLEY, n, 42)
        ctx.set_option(G.OPT_PATH, -1)
        ctx.load_query_obj(q)
        au = ctx.estimate(ALLEY, n, 42)
        ctx.set_option(G.OPT_PATH, 1)
        for other in (pe, au):
            assert fr["n"] == other["n"] == n and fr["n_valid"] == other["n_valid"]
            assert fr["sum"] == pytest.approx(other["sum"], rel=REL, abs=0.0)
            assert fr["sumsq"] == pytest.approx(other["sumsq"], rel=REL, abs=0.0)
        assert math.isfinite(fr["estimate"])


def test_frontier_falls_back_when_not_applicable(ctx, G, c0):
    """Comparison modes (variants, streaming, sample synchronisation) and one-vertex
    queries keep the persistent kernel; results stay those of the oracle."""
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_VARIANT, G.VARIANT_ALLEY_DUPCHECK_POST)
    try:
        ctx.load_query_obj(qs[2])
        assert ctx.query_info()["path"][ALLEY] == 0
        rec = ctx.trace_samples(ALLEY, 0, 5000, 9)
        _, ref = oracle.sample_range(g, qs[2], ALLEY, 9, 0, 5000, records=True,
                                     variant=oracle.VARIANT_ALLEY_DUPCHECK_POST)
        _records_equal(rec, ref, "variant A5 falls back")
    finally:
        ctx.set_option(G.OPT_VARIANT, 0)
    one = gen.query_from_edges(1, [], [int(g.labels[0])], [0], "one")
    _parity(ctx, g, one, seed=2, first=0, count=3000, loaded=True)
