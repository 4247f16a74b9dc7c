"""GPU parity of the comparison variants of readings A3 / A5 (GSWORD_OPT_VARIANT):

* VARIANT_WJ_PARENT_FIRST — WanderJoin walks from the first backward position's list
   instead of GetMinCandidate's smallest list (Alg. 1 l.8);
* VARIANT_ALLEY_DUPCHECK_POST — Alley keeps matched vertices in C_d and kills a sample
  whose drawn vertex is already matched (Fig. 19 AL Validate).

The oracle implements both step by step (oracle.c `step_at`, flags OR_WJ_PARENT_FIRST /
OR_ALLEY_DUPCHECK_POST; pinned by tests/test_oracle_variants.py against the exact tree
walk).  Here the CUDA path must reproduce every per-sample record byte for byte and the
aggregates to 1e-12, on every Alley refine path (single list, pooled refine mask,
warp-cooperative chunks), under warp streaming, sample synchronisation, inheritance and
a candidate filter.  Query labels are drawn from few labels so that same-label positions
(the DupCheck candidates) are common."""
import numpy as np
import pytest

import oracle
from workloads import gen

pytestmark = pytest.mark.gpu

REL = 1e-12
PF = oracle.VARIANT_WJ_PARENT_FIRST
POST = oracle.VARIANT_ALLEY_DUPCHECK_POST


@pytest.fixture(scope="module")
def G():
    import paper_journals_pacmmod_yelsg24_b200 as G
    assert G.VARIANT_WJ_PARENT_FIRST == PF and G.VARIANT_ALLEY_DUPCHECK_POST == POST
    return G


@pytest.fixture(scope="module")
def ctx(G):
    c = G.Context(0)
    yield c
    c.close()


def _check(ctx, G, g, q, method, variant, seed, first, count, filt=0, select=0, threads=8):
    ctx.set_option(G.OPT_VARIANT, variant)
    try:
        ctx.load_query_obj(q)
        rec = ctx.trace_samples(method, first, count, seed)
        agg = ctx.estimate(method, count, seed, first=first)
    finally:
        ctx.set_option(G.OPT_VARIANT, 0)
    y, ref = oracle.sample_range(g, q, method, seed, first, count, records=True, threads=threads, filter=filt,
                                 select=select, variant=variant)
    if rec.tobytes() != ref.tobytes():
        diff = np.nonzero([rec[i].tobytes() != ref[i].tobytes() for i in range(count)])[0]
        i = int(diff[0])
        raise AssertionError(f"{g.name}/{q.name}/m{method}/v{variant}: {diff.size} records differ; first sid "
                             f"{int(ref['sample_id'][i])}: gpu={rec[i]} oracle={ref[i]}")
    ra = oracle.aggregate(y)
    assert agg["n"] == ra["n"] and agg["n_valid"] == ra["n_valid"]
    for k in ("sum", "sumsq"):
        assert agg[k] == pytest.approx(ra[k], rel=REL, abs=0.0), k
    return rec, ref


def _cases():
    """Small graphs with few labels (same-label positions are common), plus long driver
    lists (> 128) so Alley's warp-cooperative path runs."""
    out = []
    for s in range(6):
        rng = np.random.default_rng(70 + s)
        n = int(rng.integers(12, 45))
        nl = 1 + s % 2
        g = gen.random_small_graph(n, float(rng.uniform(0.3, 0.8)), nl, seed=7000 + s)
        nq = int(rng.integers(3, 7))
        try:
            q = gen.extract_query(g, nq, 7100 + s, dense=bool(s % 2))
            q = q.with_order(gen.random_connected_order(q, s))
        except RuntimeError:
            q = gen.random_connected_query(nq, 0.5, nl, 7200 + s)
        out.append((g, [q]))
    dense = gen.erdos_renyi(300, 30000, seed=4)
    out.append((dense, [gen.clique_query(4), gen.extract_query(dense, 6, seed=5, dense=True),
                        gen.extract_query(dense, 7, seed=6, dense=False)]))
    out.append((gen.regular_circulant(90, 30), [gen.star_query(3), gen.path_query(6)]))
    return out


@pytest.mark.parametrize("variant", [PF, POST, PF | POST])
def test_variant_parity_small_and_long(ctx, G, variant):
    for gi, (g, qs) in enumerate(_cases()):
        ctx.load_graph_obj(g)
        for qi, q in enumerate(qs):
            for m in (G.WJ, G.ALLEY):
                _check(ctx, G, g, q, m, variant, seed=gi * 10 + qi, first=3 + gi, count=6000)


def test_variant_parity_c0(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        _check(ctx, G, g, q, G.WJ, PF, seed=40 + i, first=0, count=50_000)
        _check(ctx, G, g, q, G.ALLEY, POST, seed=40 + i, first=0, count=50_000)


def test_variants_change_only_their_method(ctx, G, c0):
    """PARENT_FIRST leaves Alley byte-identical to the default and DUPCHECK_POST leaves
    WanderJoin so; under each variant some samples differ from the default (the variants
    are really applied)."""
    g, qs = c0
    ctx.load_graph_obj(g)
    changed = {G.WJ: 0, G.ALLEY: 0}
    for q in qs:
        ctx.load_query_obj(q)
        base = {m: ctx.trace_samples(m, 0, 20_000, 9) for m in (G.WJ, G.ALLEY)}
        for variant, other in ((PF, G.ALLEY), (POST, G.WJ)):
            ctx.set_option(G.OPT_VARIANT, variant)
            try:
                assert ctx.trace_samples(other, 0, 20_000, 9).tobytes() == base[other].tobytes()
                mine = G.WJ if other == G.ALLEY else G.ALLEY
                changed[mine] += int(ctx.trace_samples(mine, 0, 20_000, 9).tobytes() != base[mine].tobytes())
            finally:
                ctx.set_option(G.OPT_VARIANT, 0)
    assert changed[G.WJ] > 0 and changed[G.ALLEY] > 0


def test_variant_with_streaming_sync_and_filter(ctx, G, c0):
    g, qs = c0
    dense = gen.erdos_renyi(300, 30000, seed=4)
    dq = gen.extract_query(dense, 6, seed=5, dense=True)
    try:
        ctx.set_option(G.OPT_STREAMING, 1)
        ctx.load_graph_obj(dense)
        _check(ctx, G, dense, dq, G.ALLEY, POST, seed=2, first=0, count=8000, select=oracle.SELECT_STREAM)
        ctx.load_graph_obj(g)
        for i, q in enumerate(qs[:4]):
            _check(ctx, G, g, q, G.ALLEY, POST, seed=50 + i, first=0, count=20_000, select=oracle.SELECT_STREAM)
        ctx.set_option(G.OPT_STREAMING, 0)
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_SAMPLE_SYNC)
        for i, q in enumerate(qs[:4]):
            for m in (G.WJ, G.ALLEY):
                _check(ctx, G, g, q, m, PF | POST, seed=60 + i, first=1, count=20_000)
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)
        ctx.set_option(G.OPT_FILTER, 2)
        for i, q in enumerate(qs[:6]):
            for m in (G.WJ, G.ALLEY):
                _check(ctx, G, g, q, m, PF | POST, seed=70 + i, first=0, count=20_000, filt=2)
    finally:
        ctx.set_option(G.OPT_STREAMING, 0)
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)
        ctx.set_option(G.OPT_FILTER, 0)
        ctx.set_option(G.OPT_VARIANT, 0)


def test_variant_inheritance_matches_oracle(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_SCHEDULE, G.SCHED_INHERIT)
    try:
        for q in qs[:6]:
            for m, variant in ((G.WJ, PF), (G.ALLEY, POST)):
                ctx.set_option(G.OPT_VARIANT, variant)
                ctx.load_query_obj(q)
                r = ctx.estimate(m, 20_000, 31, first=5)
                ref = oracle.inherit_range(g, q, m, 31, 5, 20_000, variant=variant)
                assert r["n"] == 20_000 and r["n_valid"] == ref["n_valid"], (q.name, m)
                assert r["sum"] == pytest.approx(ref["sum"], rel=REL, abs=1e-300)
                assert r["sumsq"] == pytest.approx(ref["sumsq"], rel=REL, abs=1e-300)
    finally:
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)
        ctx.set_option(G.OPT_VARIANT, 0)


def test_variant_option_errors(ctx, G):
    with pytest.raises(G.GswordError):
        ctx.set_option(G.OPT_VARIANT, 1)
    with pytest.raises(G.GswordError):
        ctx.set_option(G.OPT_VARIANT, 8)
    ctx.set_option(G.OPT_VARIANT, 0)
