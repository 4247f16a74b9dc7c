"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Per sample: bit-exact records (path, csize, validity, fp64 weight) for every sample
id compared.  Aggregates: sum and sumsq within a relative 1e-12 (BASELINE.json
north_star), n and n_valid exact, variance within the cancellation-aware bound of
DESIGN.md §4.  Inputs are the seeded workloads of workloads/gen.py.
"""
import math

import numpy as np
import pytest

import oracle
from gsword_testutil import variance_tolerance
from workloads import gen

pytestmark = pytest.mark.gpu

REL = 1e-12


@pytest.fixture(scope="module")
def G():
    import paper_journals_pacmmod_yelsg24_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    c = G.Context(0)
    yield c
    c.close()


def _records_equal(gpu, ref, what=""):
    assert gpu.shape == ref.shape
    if gpu.tobytes() == ref.tobytes():
        return
    for f in ("sample_id", "valid", "depth_reached", "path", "csize", "weight"):
        bad = np.nonzero(np.any((gpu[f] != ref[f]).reshape(gpu.shape[0], -1), axis=1))[0]
        if bad.size:
            i = int(bad[0])
            raise AssertionError(f"{what}: field {f} differs at {bad.size} samples; first sid "
                                 f"{int(ref['sample_id'][i])}: gpu={gpu[i]} oracle={ref[i]}")
    raise AssertionError(f"{what}: records differ in padding")


def _agg_close(gpu, ref, G):
    assert gpu["n"] == ref["n"]
    assert gpu["n_valid"] == ref["n_valid"]
    for k in ("sum", "sumsq", "estimate"):
        assert gpu[k] == pytest.approx(ref[k], rel=REL, abs=0.0), k
    if gpu["n"] >= 2:
        assert abs(gpu["variance"] - ref["variance"]) <= variance_tolerance(ref) + REL * abs(ref["variance"])


def _parity(ctx, G, g, q, method, seed, first, count, threads=8, loaded=False):
    if not loaded:
        ctx.load_graph_obj(g)
    ctx.load_query_obj(q)
    rec = ctx.trace_samples(method, first, count, seed)
    y, ref = oracle.sample_range(g, q, method, seed, first, count, records=True, threads=threads)
    _records_equal(rec, ref, f"{g.name}/{q.name}/m{method}")
    agg = ctx.estimate(method, count, seed, first=first)
    _agg_close(agg, oracle.aggregate(y), G)
    return rec


# ------------------------------------------------------------------ C0 (BASELINE configs[0])
@pytest.mark.parametrize("method", [0, 1])
def test_c0_full_parity(ctx, G, c0, method):
    g, qs = c0
    ctx.load_graph_obj(g)
    for qi, q in enumerate(qs):
        _parity(ctx, G, g, q, method, seed=1 + qi, first=0, count=100_000, loaded=True)


def test_c0_estimate_near_exact(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    for q in qs[:6]:
        truth = oracle.count_embeddings(g, q)
        ctx.load_query_obj(q)
        for m in (G.WJ, G.ALLEY):
            r = ctx.estimate(m, 1_000_000, seed=7)
            assert abs(r["estimate"] - truth) <= 3 * math.sqrt(max(r["variance"], 0.0)) + 1e-9


# ------------------------------------------------------------------ fuzz: tiny random inputs
@pytest.mark.parametrize("seed", range(16))
def test_fuzz_small(ctx, G, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 40))
    nl = int(rng.integers(1, 5))
    g = gen.random_small_graph(n, float(rng.uniform(0.15, 0.7)), nl, seed=1000 + seed)
    nq = int(rng.integers(1, min(n, 9) + 1))
    if seed % 2 == 0:
        q = gen.random_connected_query(nq, float(rng.uniform(0, 0.6)), nl, 2000 + seed)
    else:
        try:
            q = gen.extract_query(g, nq, 3000 + seed, dense=bool(seed % 4 == 1))
            q = q.with_order(gen.random_connected_order(q, seed))
        except RuntimeError:
            q = gen.random_connected_query(nq, 0.3, nl, 2000 + seed)
    ctx.load_graph_obj(g)
    for m in (0, 1):
        _parity(ctx, G, g, q, m, seed=seed, first=int(rng.integers(0, 2**40)), count=3000, loaded=True)


# ------------------------------------------------------------------ closed forms on the GPU
def test_alley_zero_variance_on_gpu(ctx, G):
    for n, k in ((9, 4), (80, 3), (100, 5)):  # n-1 >= 64 exercises the warp-cooperative refine
        g = gen.complete_graph(n)
        ctx.load_graph_obj(g)
        ctx.load_query_obj(gen.clique_query(k))
        r = ctx.estimate(G.ALLEY, 20_000, seed=3)
        want = float(math.factorial(n) // math.factorial(n - k))
        assert r["n_valid"] == 20_000 and r["estimate"] == want and abs(r["variance"]) <= variance_tolerance(r)


@pytest.mark.parametrize("coop", [0, 1, 17, 32, 64, 100, 128])
def test_coop_threshold_invariance(ctx, G, coop):
    """The warp-cooperative and per-lane refine paths give identical samples."""
    g = gen.chung_lu(3000, 60_000, gamma=2.2, max_over_mean=40.0, seed=5, labels=gen.uniform_labels(3000, 2, 6),
                     n_labels=2)
    q = gen.extract_query(g, 6, seed=8, dense=True)
    ctx.set_option(G.OPT_COOP_THRESHOLD, coop)
    try:
        _parity(ctx, G, g, q, G.ALLEY, seed=4, first=0, count=20_000)
    finally:
        ctx.set_option(G.OPT_COOP_THRESHOLD, 64)


@pytest.mark.parametrize("bloom,eset", [(0, 0), (1, 0), (0, 1), (1, 1)])
def test_edge_index_invariance(ctx, G, bloom, eset):
    """Bloom pre-test / exact edge set / binary search answer the same adjacency
    questions: identical samples with every combination."""
    g = gen.chung_lu(5000, 150_000, gamma=2.1, max_over_mean=60.0, seed=11,
                     labels=gen.uniform_labels(5000, 2, 12) if bloom != eset else None, n_labels=2 if bloom != eset else 1)
    ctx.set_option(G.OPT_BLOOM, bloom)
    ctx.set_option(G.OPT_EDGE_SET, eset)
    try:
        for dense, qs in ((True, 12), (False, 13)):
            q = gen.extract_query(g, 7, seed=qs, dense=dense)
            for m in (0, 1):
                _parity(ctx, G, g, q, m, seed=6, first=0, count=20_000)
    finally:
        ctx.set_option(G.OPT_BLOOM, 1)
        ctx.set_option(G.OPT_EDGE_SET, 1)
        ctx.set_option(G.OPT_REFILL_MIN, 16)
        ctx.set_option(G.OPT_EDGE_SET, 1)


def test_edge_cases(ctx, G):
    g = gen.random_small_graph(30, 0.3, 3, seed=9)
    ctx.load_graph_obj(g)
    # single-vertex query: every sample valid with W = |C(u)|
    q1 = gen.query_from_edges(1, [], labels=[1], order=[0])
    ctx.load_query_obj(q1)
    r = ctx.estimate(G.WJ, 1000, seed=1)
    assert r["n_valid"] == 1000 and r["estimate"] == float(np.sum(g.labels == 1))
    # one sample
    q = gen.extract_query(g, 3, seed=2, dense=True)
    _parity(ctx, G, g, q, G.ALLEY, seed=5, first=123, count=1, loaded=True)
    # a query label that no data vertex has: every sample dead, estimate 0
    lab = np.asarray(g.labels).copy()
    lab[lab == 2] = 0
    g2 = gen.Graph(g.row_ptr, g.col, lab, 3)
    q2 = gen.query_from_edges(2, [(0, 1)], labels=[2, 0], order=[0, 1])
    for m in (0, 1):
        _parity(ctx, G, g2, q2, m, seed=1, first=0, count=500)
    # the largest query: 16-clique in K_20 (W = 20!/4! beyond 2^53: fp64 rounding order)
    _parity(ctx, G, gen.complete_graph(20), gen.clique_query(16), G.ALLEY, seed=2, first=0, count=2000)
    _parity(ctx, G, gen.complete_graph(20), gen.clique_query(16), G.WJ, seed=2, first=0, count=2000)


def test_degenerate_inputs(ctx, G):
    """Empty and boundary inputs (SURVEY §8(b) conventions): an edgeless graph, isolated
    vertices next to a component, n_samples = 0 and 1, a range ending at 2^64 - 1 and
    one that overflows."""
    # edgeless graph: every sample dies at depth 1; the single-vertex query is still exact
    g0 = gen.make_graph(40, [], [], gen.uniform_labels(40, 2, seed=3), 2, name="edgeless")
    q = gen.query_from_edges(2, [(0, 1)], labels=[0, 1], order=[0, 1])
    for m in (0, 1):
        rec = _parity(ctx, G, g0, q, m, seed=4, first=0, count=300)
        assert not rec["valid"].any()
        r = ctx.estimate(m, 300, seed=4)
        assert r["estimate"] == 0.0 and r["n_valid"] == 0 and r["n"] == 300
    # isolated vertices around a triangle (seed candidates that die at once)
    n = 64
    g1 = gen.make_graph(n, [0, 1, 2], [1, 2, 0], None, 1, name="triangle+isolated")
    for m in (0, 1):
        _parity(ctx, G, g1, gen.cycle_query(3), m, seed=8, first=17, count=4000)
    # n_samples = 0 is an error for the aggregates, a no-op for traces
    ctx.load_graph_obj(g1)
    ctx.load_query_obj(gen.cycle_query(3))
    for m in (0, 1):
        with pytest.raises(G.GswordError) as e:
            ctx.estimate(m, 0, seed=1)
        assert e.value.status == -1
        assert ctx.trace_samples(m, 0, 0, seed=1).shape == (0,)
    # one sample: variance undefined
    r = ctx.estimate(1, 1, seed=1)
    assert r["n"] == 1 and math.isnan(r["variance"])
    # the last ids of the u64 space (exclusive end 2^64 - 1), and ranges that would wrap
    top = 2**64 - 1001
    _parity(ctx, G, g1, gen.cycle_query(3), 0, seed=3, first=top, count=1000, loaded=True)
    for call in (lambda: ctx.estimate(0, 1001, seed=3, first=top),
                 lambda: ctx.trace_samples(1, top, 1001, seed=3),
                 lambda: ctx.trawl(0, 1001, seed=3, first=top),
                 lambda: ctx.trace_trawl(1, top, 1001, seed=3)):
        with pytest.raises(G.GswordError) as e:
            call()
        assert e.value.status == -1


def test_errors(G):
    c = G.Context(0)
    with pytest.raises(G.GswordError) as e:
        c.estimate(G.WJ, 10, 1)
    assert e.value.status == -2
    g = gen.ring_graph(10)
    c.load_graph_obj(g)
    with pytest.raises(G.GswordError) as e:
        c.estimate(G.WJ, 10, 1)
    assert e.value.status == -3
    q = gen.path_query(3)
    with pytest.raises(G.GswordError) as e:
        c.load_query(*q.csr(), q.labels, [0, 2, 1])
    assert e.value.status == -4
    bad_col = g.col.copy()
    bad_col[0], bad_col[1] = bad_col[1], bad_col[0]
    with pytest.raises(G.GswordError) as e:
        c.load_graph(g.row_ptr, bad_col)
    assert e.value.status == -5
    c.close()


# ------------------------------------------------------------------ C2 / C1 (paper-shaped)
def test_c2_parity(ctx, G):
    g, qs = gen.config_c2()
    ctx.load_graph_obj(g)
    for i, q in enumerate(qs):
        for m in (0, 1):
            _parity(ctx, G, g, q, m, seed=10 + i, first=0, count=50_000, loaded=True)
            # BASELINE configs[2] budget (1e8 samples): windows deep in the id range, and the
            # whole 1e8 aggregate equal to the sum of two split ranges
            for first in (50_000_000, 100_000_000 - 4000):
                rec = ctx.trace_samples(m, first, 4000, 10 + i)
                _, ref = oracle.sample_range(g, q, m, 10 + i, first, 4000, records=True, threads=8)
                _records_equal(rec, ref, f"C2/{q.name}/m{m}@{first}")
            full = ctx.estimate(m, 100_000_000, 10 + i)
            a = ctx.estimate(m, 61_000_000, 10 + i)
            b = ctx.estimate(m, 39_000_000, 10 + i, first=61_000_000)
            assert full["n_valid"] == a["n_valid"] + b["n_valid"]
            assert full["sum"] == pytest.approx(a["sum"] + b["sum"], rel=REL)


@pytest.fixture(scope="module")
def c1():
    return gen.config_c1()


def test_c1_parity_prefix(ctx, G, c1):
    g, qs = c1
    ctx.load_graph_obj(g)
    for q in qs:
        for m in (0, 1):
            _parity(ctx, G, g, q, m, seed=42, first=0, count=20_000, loaded=True)


def test_c1_full_size_sampled_and_split(ctx, G, c1):
    """BASELINE configs[1] at its full budget (1e8 samples, the bench launch config):
    sampled sample ids against the oracle, plus split-range invariance of the whole."""
    g, qs = c1
    ctx.load_graph_obj(g)
    n = 100_000_000
    for q in qs:
        ctx.load_query_obj(q)
        for m in (0, 1):
            for first in (0, 31_415_926, n - 1500):
                rec = ctx.trace_samples(m, first, 1500, 42)
                _, ref = oracle.sample_range(g, q, m, 42, first, 1500, records=True, threads=8)
                _records_equal(rec, ref, f"C1/{q.name}/m{m}@{first}")
            full = ctx.estimate(m, n, 42)
            a = ctx.estimate(m, 37_000_000, 42, first=0)
            b = ctx.estimate(m, n - 37_000_000, 42, first=37_000_000)
            assert full["n"] == n and a["n"] + b["n"] == n
            assert full["n_valid"] == a["n_valid"] + b["n_valid"]
            assert full["sum"] == pytest.approx(a["sum"] + b["sum"], rel=REL)
            assert full["sumsq"] == pytest.approx(a["sumsq"] + b["sumsq"], rel=REL)


def test_c3_parity_sampled(ctx, G):
    """BASELINE configs[3] (LiveJournal shape, 16 labels, 12-vertex queries, a 1e10
    budget): a prefix and two windows deep in the 1e10 id range, every query/method."""
    g, qs = gen.config_c3()
    ctx.load_graph_obj(g)
    for q in qs:
        for m in (0, 1):
            _parity(ctx, G, g, q, m, seed=7, first=0, count=10_000, loaded=True, threads=16)
            for first in (5_000_000_000, 10_000_000_000 - 2000):
                ctx.load_query_obj(q)
                rec = ctx.trace_samples(m, first, 2000, 7)
                _, ref = oracle.sample_range(g, q, m, 7, first, 2000, records=True, threads=16)
                _records_equal(rec, ref, f"C3/{q.name}/m{m}@{first}")


def test_c4_full_size_sampled(ctx, G):
    """BASELINE configs[4] at full size (Kronecker scale 23, 1e8 undirected edges, 16
    labels; budgets up to 1e11 in the sweep): 4-, 8- and 16-vertex queries and a star,
    both methods, label-only and NLF candidate filtering, a prefix checked record by
    record and in aggregate, and windows deep in the 1e11 id range."""
    g, qs = gen.config_c4()
    ctx.load_graph_obj(g)
    pick = [q for q in qs if q.name in ("dense4_s5004", "sparse8_s4008", "dense8_s5008", "dense16_s5016", "star4_s6004")]
    assert len(pick) == 5
    for filt in (0, 2):
        ctx.set_option(G.OPT_FILTER, filt)
        try:
            for q in pick if filt == 0 else pick[2:4]:
                for m in (0, 1):
                    ctx.load_query_obj(q)
                    for first, count in ((0, 10_000), (50_000_000_000, 2000), (100_000_000_000 - 2000, 2000)):
                        rec = ctx.trace_samples(m, first, count, 11)
                        y, ref = oracle.sample_range(g, q, m, 11, first, count, records=True, threads=1, filter=filt)
                        _records_equal(rec, ref, f"C4/{q.name}/f{filt}/m{m}@{first}")
                        if first == 0:
                            _agg_close(ctx.estimate(m, count, 11), oracle.aggregate(y), G)
        finally:
            ctx.set_option(G.OPT_FILTER, 0)


def test_scheduling_invariance(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    q = qs[3]
    ctx.load_query_obj(q)
    base = {m: ctx.estimate(m, 400_000, 9) for m in (0, 1)}
    try:
        for opt, val in ((G.OPT_CHUNK, 1), (G.OPT_CHUNK, 4096), (G.OPT_BLOCKS_PER_SM, 1),
                         (G.OPT_THREADS, 64), (G.OPT_L2_PERSIST, 1), (G.OPT_L2_PERSIST, 0), (G.OPT_BLOOM, 0),
                         (G.OPT_EDGE_SET, 0), (G.OPT_REFILL_MIN, 1), (G.OPT_REFILL_MIN, 32)):
            ctx.set_option(opt, val)
            for m in (0, 1):
                r = ctx.estimate(m, 400_000, 9)
                assert r["n_valid"] == base[m]["n_valid"]
                assert r["sum"] == pytest.approx(base[m]["sum"], rel=REL)
                assert r["sumsq"] == pytest.approx(base[m]["sumsq"], rel=REL)
    finally:
        ctx.set_option(G.OPT_CHUNK, 256)
        ctx.set_option(G.OPT_BLOCKS_PER_SM, 0)
        ctx.set_option(G.OPT_THREADS, 256)
        ctx.set_option(G.OPT_L2_PERSIST, 2)
        ctx.set_option(G.OPT_BLOOM, 1)
        ctx.set_option(G.OPT_EDGE_SET, 1)


def test_async_matches_sync_on_torch_stream(ctx, G, c0):
    import torch
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[0])
    s = torch.cuda.Stream()
    ctx.set_stream(s)
    try:
        out = torch.zeros(4, dtype=torch.float64, device="cuda")
        with torch.cuda.stream(s):
            ctx.estimate_async(G.ALLEY, 0, 50_000, 3, out)
        s.synchronize()
        r = G.finalize(out.cpu().numpy())
        ref = ctx.estimate(G.ALLEY, 50_000, 3)
        assert r["sum"] == ref["sum"] and r["n_valid"] == ref["n_valid"]
    finally:
        ctx.set_stream(None)


# ------------------------------------------------------------------ NEXT-1: candidate graph
def _parity_filtered(ctx, G, g, q, method, seed, first, count, filt, threads=8):
    ctx.load_query_obj(q)
    rec = ctx.trace_samples(method, first, count, seed)
    y, ref = oracle.sample_range(g, q, method, seed, first, count, records=True, threads=threads, filter=filt)
    _records_equal(rec, ref, f"{g.name}/{q.name}/m{method}/f{filt}")
    _agg_close(ctx.estimate(method, count, seed, first=first), oracle.aggregate(y), G)


@pytest.mark.parametrize("filt", [1, 2])
def test_filtered_parity_small_and_c0(ctx, G, c0, filt):
    ctx.set_option(G.OPT_FILTER, filt)
    try:
        for seed in range(8):
            rng = np.random.default_rng(seed)
            g = gen.random_small_graph(int(rng.integers(6, 30)), 0.4, int(rng.integers(1, 4)), seed=900 + seed)
            try:
                q = gen.extract_query(g, int(rng.integers(2, 6)), seed=seed, dense=bool(seed % 2))
            except RuntimeError:
                q = gen.random_connected_query(3, 0.5, g.n_labels, seed)
            ctx.load_graph_obj(g)
            for m in (0, 1):
                _parity_filtered(ctx, G, g, q, m, seed, 0, 3000, filt)
        g, qs = c0
        ctx.load_graph_obj(g)
        for i, q in enumerate(qs):
            for m in (0, 1):
                _parity_filtered(ctx, G, g, q, m, 3 + i, 0, 50_000, filt)
            info = ctx.query_info()
            cs = oracle.candidate_sets(g, q, filt)
            assert info["filter"] == filt and info["candidates"] == [int(x) for x in cs.sum(axis=1)]
    finally:
        ctx.set_option(G.OPT_FILTER, 0)


@pytest.mark.parametrize("threads", [64, 96, 256])
def test_filtered_large_query_any_cta_size(ctx, G, threads):
    """Candidate-graph runs of positions >= 8 under every CTA size: the per-query-edge index
    table staged in shared memory must be complete however many threads stage it (a
    12-vertex query with NLF at 64 / 96 / 256 threads per CTA, sampling and trawling)."""
    g = gen.chung_lu(3000, 60_000, gamma=2.2, max_over_mean=40.0, seed=21, labels=gen.uniform_labels(3000, 2, 22),
                     n_labels=2)
    q = gen.extract_query(g, 12, seed=23, dense=True)
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_THREADS, threads)
    try:
        for filt in (0, 2):
            ctx.set_option(G.OPT_FILTER, filt)
            for m in (0, 1):
                _parity_filtered(ctx, G, g, q, m, 5, 0, 20_000, filt)
                _trawl_parity(ctx, G, g, q, m, 6, 0, 3000, 20_000, filt=filt)
    finally:
        ctx.set_option(G.OPT_FILTER, 0)
        ctx.set_option(G.OPT_THREADS, 256)


def test_many_labels(ctx, G):
    """A label alphabet far larger than the configs' (1,000 labels, half the vertices on label
    0, the rest spread over 999): the label-segment table has |V| x 1,000 + 1 entries; records
    and aggregates against the oracle, label-only and NLF, both methods, and trawling."""
    n = 4000
    rng = np.random.default_rng(77)
    lab = np.where(rng.random(n) < 0.5, 0, rng.integers(1, 1000, size=n)).astype(np.int32)
    g = gen.chung_lu(n, 80_000, gamma=2.2, max_over_mean=40.0, seed=78, labels=lab, n_labels=1000)
    ctx.load_graph_obj(g)
    for qs, dense in ((79, True), (80, False)):
        q = gen.extract_query(g, 7, seed=qs, dense=dense)
        for filt in (0, 2):
            ctx.set_option(G.OPT_FILTER, filt)
            try:
                for m in (0, 1):
                    _parity_filtered(ctx, G, g, q, m, 9, 0, 20_000, filt)
                    _trawl_parity(ctx, G, g, q, m, 10, 0, 2000, 50_000, filt=filt)
            finally:
                ctx.set_option(G.OPT_FILTER, 0)


@pytest.mark.parametrize("filt", [1, 2])
def test_filtered_parity_c2_c1(ctx, G, c1, filt):
    ctx.set_option(G.OPT_FILTER, filt)
    try:
        for g, qs, count in (gen.config_c2() + (20_000,), c1 + (10_000,)):
            ctx.load_graph_obj(g)
            for q in qs:
                for m in (0, 1):
                    _parity_filtered(ctx, G, g, q, m, 5, 0, count, filt, threads=16)
                    for coop in (0, 128):
                        ctx.set_option(G.OPT_COOP_THRESHOLD, coop)
                        ctx.load_query_obj(q)
                        rec = ctx.trace_samples(m, 777, 2000, 5)
                        _, ref = oracle.sample_range(g, q, m, 5, 777, 2000, records=True, threads=16, filter=filt)
                        _records_equal(rec, ref, f"{q.name}/f{filt}/coop{coop}")
                    ctx.set_option(G.OPT_COOP_THRESHOLD, 64)
    finally:
        ctx.set_option(G.OPT_FILTER, 0)


# ------------------------------------------------------------------ NEXT-4: matching order
def _trial_candidates(q, qo):
    """The documented candidate set of GSWORD_ORDER_TRIAL (include/gsword.h)."""
    adj = q.adj
    cands = [list(qo)]
    for a in range(q.nq):
        for b in range(q.nq):
            if not adj[a, b]:
                continue
            o = [a, b]
            while len(o) < q.nq:
                nxt = next((c for c in qo if c not in o and any(adj[x, c] for x in o)), None)
                if nxt is None:
                    break
                o.append(nxt)
            if len(o) == q.nq and o not in cands:
                cands.append(o)
    return cands


@pytest.mark.parametrize("method", [0, 1])
def test_order_selection_trial_matches_oracle(ctx, G, c0, method):
    g, qs = c0
    ctx.load_graph_obj(g)
    for q in qs[:6]:
        qrp, qcol = q.csr()
        qo = G.quicksi_order(g.row_ptr, g.col, g.labels, g.n_labels, qrp, qcol, q.labels)
        order, score = ctx.select_order(G.ORDER_TRIAL, method, qrp, qcol, q.labels, pilot_samples=20_000, seed=9)
        scores = []
        for o in _trial_candidates(q, qo):
            agg = oracle.aggregate(oracle.sample_range(g, q.with_order(o), method, 9, 0, 20_000, records=False)[0])
            scores.append((agg["variance"] * agg["n"], o))
        best = min(scores, key=lambda t: t[0])  # min keeps the first of equal scores
        assert order == best[1]
        assert score == pytest.approx(best[0], rel=1e-9, abs=1e-9)
        # the chosen order is loaded: estimates now follow it
        r = ctx.estimate(method, 5000, 3)
        ref = oracle.aggregate(oracle.sample_range(g, q.with_order(order), method, 3, 0, 5000, records=False)[0])
        assert r["sum"] == pytest.approx(ref["sum"], rel=1e-12)
        o2, _ = ctx.select_order(G.ORDER_QUICKSI, method, qrp, qcol, q.labels)
        assert o2 == qo


# ------------------------------------------------------------------ NEXT-2: trawling
def _trawl_parity(ctx, G, g, q, method, seed, first, count, budget, filt=0, threads=8):
    ctx.load_query_obj(q)
    rec = ctx.trace_trawl(method, first, count, seed, budget)
    t, st, ref = oracle.trawl_range(g, q, method, seed, first, count, budget=budget, filter=filt, threads=threads)
    assert rec.tobytes() == ref.tobytes(), f"trawl records differ ({q.name}, m{method}, budget {budget})"
    agg = oracle.trawl_aggregate(t, st)
    # both enumeration kernels of gsword_trawl_range: warp-cooperative (default) and per-lane
    for warp in (1, 0):
        ctx.set_option(G.OPT_TRAWL_WARP, warp)
        try:
            r = ctx.trawl(method, count, seed, first=first, node_budget=budget)
        finally:
            ctx.set_option(G.OPT_TRAWL_WARP, 1)
        assert r["n_timeout"] == agg["n_timeout"] and r["n"] == agg["n"] and r["n_valid"] == agg["n_valid"], warp
        assert r["sum"] == pytest.approx(agg["sum"], rel=REL)
        assert r["sumsq"] == pytest.approx(agg["sumsq"], rel=REL)
    # the warp-cooperative kernel sample by sample: a one-id range gives T (bit-exact) or
    # the timeout of that sample
    for i in list(np.nonzero(st == 1)[0][:12]) + list(np.nonzero(st == 2)[0][:4]) + list(np.nonzero(st == 0)[0][:2]):
        r = ctx.trawl(method, 1, seed, first=first + int(i), node_budget=budget)
        assert r["n_timeout"] == int(st[i] == 2)
        assert r["sum"] == (float(t[i]) if st[i] == 1 else 0.0), (q.name, method, int(i), r["sum"], float(t[i]))


@pytest.mark.parametrize("method", [0, 1])
def test_trawl_parity(ctx, G, c0, method):
    for seed in range(6):
        g = gen.random_small_graph(12 + seed, 0.4, 1 + seed % 3, seed=2000 + seed)
        try:
            q = gen.extract_query(g, 4 + seed % 3, seed=2100 + seed, dense=bool(seed % 2))
        except RuntimeError:
            q = gen.random_connected_query(4, 0.5, g.n_labels, 2100 + seed)
        ctx.load_graph_obj(g)
        for budget in (2**62, 3, 0):
            _trawl_parity(ctx, G, g, q, method, seed, 17, 2000, budget)
    g, qs = c0
    ctx.load_graph_obj(g)
    for q in qs:
        _trawl_parity(ctx, G, g, q, method, 5, 0, 20_000, 2**62)
        truth = oracle.count_embeddings(g, q)
        r = ctx.trawl(method, 1_000_000, 8)
        assert abs(r["estimate"] - truth) <= 3 * math.sqrt(max(r["variance"], 0.0)) + 1e-9


def test_trawl_parity_c2_and_filter(ctx, G):
    g, qs = gen.config_c2()
    ctx.load_graph_obj(g)
    for filt in (0, 2):
        ctx.set_option(G.OPT_FILTER, filt)
        try:
            for q in qs:
                for m in (0, 1):
                    _trawl_parity(ctx, G, g, q, m, 3, 0, 5000, 100_000, filt=filt, threads=16)
        finally:
            ctx.set_option(G.OPT_FILTER, 0)


# ------------------------------------------------------------------ NEXT-3: schedules
def test_sample_sync_schedule_parity(ctx, G, c0):
    """Sample synchronisation changes only when lanes take new ids: identical samples."""
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_SCHEDULE, G.SCHED_SAMPLE_SYNC)
    try:
        for q in qs[:4]:
            for m in (0, 1):
                _parity(ctx, G, g, q, m, seed=21, first=5, count=30_000, loaded=True)
    finally:
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)


@pytest.mark.parametrize("filt", [0, 2])
def test_inheritance_matches_oracle(ctx, G, c0, filt):
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_FILTER, filt)
    ctx.set_option(G.OPT_SCHEDULE, G.SCHED_INHERIT)
    try:
        for first, count in ((0, 64_000), (7, 10_013)):  # a ragged last group
            for q in qs:
                ctx.load_query_obj(q)
                for m in (0, 1):
                    r = ctx.estimate(m, count, 31, first=first)
                    ref = oracle.inherit_range(g, q, m, 31, first, count, filter=filt)
                    assert r["n"] == count and r["n_valid"] == ref["n_valid"], (q.name, m)
                    assert r["sum"] == pytest.approx(ref["sum"], rel=REL, abs=1e-300)
                    assert r["sumsq"] == pytest.approx(ref["sumsq"], rel=REL, abs=1e-300)
                    if ref["sumsq"] > 0:
                        assert r["variance"] == pytest.approx(ref["variance"], rel=1e-9, abs=1e-12 * ref["sumsq"])
        with pytest.raises(G.GswordError):
            ctx.trace_samples(0, 0, 10, 1)
    finally:
        ctx.set_option(G.OPT_SCHEDULE, G.SCHED_REFILL)
        ctx.set_option(G.OPT_FILTER, 0)


# ------------------------------------------------------------------ device-resident graph load
def test_load_graph_device_equals_host(ctx, G, c0):
    import torch
    cases = [c0[0], gen.chung_lu(4000, 40_000, gamma=2.2, max_over_mean=50.0, seed=9), gen.config_c2()[0]]
    for g in cases:
        q = gen.extract_query(g, 5, seed=4, dense=True)
        ctx.load_graph_obj(g)
        ctx.load_query_obj(q)
        ref = {m: ctx.trace_samples(m, 0, 20_000, 2) for m in (0, 1)}
        qo_host = G.quicksi_order(g.row_ptr, g.col, g.labels, g.n_labels, *q.csr(), q.labels)
        rp = torch.as_tensor(g.row_ptr).cuda()
        cl = torch.as_tensor(g.label_sorted_col()).cuda()
        lb = torch.as_tensor(g.labels).cuda()
        ctx.load_graph_device(rp, cl, lb if g.n_labels > 1 else None, g.n_labels)
        ctx.load_query_obj(q)
        for m in (0, 1):
            assert ctx.trace_samples(m, 0, 20_000, 2).tobytes() == ref[m].tobytes()
        order, _ = ctx.select_order(G.ORDER_QUICKSI, 0, *q.csr(), q.labels)
        assert order == qo_host
    # non-canonical device input is rejected
    g = c0[0]
    bad = torch.as_tensor(g.col).cuda()  # id-sorted, not (label, id)-sorted
    with pytest.raises(G.GswordError) as e:
        ctx.load_graph_device(torch.as_tensor(g.row_ptr).cuda(), bad, torch.as_tensor(g.labels).cuda(), g.n_labels)
    assert e.value.status == -5


def test_autotune_does_not_change_results(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    q = qs[1]
    ctx.set_option(G.OPT_AUTOTUNE, 0)
    ctx.load_query_obj(q)
    ref = {m: ctx.trace_samples(m, 0, 30_000, 4) for m in (0, 1)}
    ctx.set_option(G.OPT_AUTOTUNE, 1)
    ctx.load_query_obj(q)
    info = ctx.query_info()
    assert all(r in (8, 16, 24, 28, 32) for r in info["refill_min"])
    assert info["occupancy"][0] in (5, 6, 7) and info["occupancy"][1] in (4, 5, 6)
    for m in (0, 1):
        assert ctx.trace_samples(m, 0, 30_000, 4).tobytes() == ref[m].tobytes()
    # reloading the same query reuses the tuned thresholds (no pilots); a graph reload
    # forgets them
    ctx.load_query_obj(q)
    assert ctx.query_info()["refill_min"] == info["refill_min"]
    assert ctx.query_info()["occupancy"] == info["occupancy"]
    # every occupancy variant of the estimate kernel (forced), and a limited grid, gives the
    # oracle's aggregate, for a tree order (TREE kernels) and a non-tree one
    for qq in (q, gen.path_query(4, labels=[int(x) for x in q.labels[:4]]) if q.nq >= 4 else q):
        ctx.load_query_obj(qq)
        for m in (0, 1):
            y, _ = oracle.sample_range(g, qq, m, 9, 0, 50_000, records=False, threads=8)
            ref_agg = oracle.aggregate(y)
            for occ, bps in ((0, 0), (1, 0), (2, 0), (-1, 3)):
                ctx.set_option(G.OPT_OCCUPANCY, occ)
                ctx.set_option(G.OPT_BLOCKS_PER_SM, bps)
                try:
                    agg = ctx.estimate(m, 50_000, 9)
                finally:
                    ctx.set_option(G.OPT_OCCUPANCY, -1)
                    ctx.set_option(G.OPT_BLOCKS_PER_SM, 0)
                _agg_close(agg, ref_agg, G)
    ctx.load_graph_obj(g)
    ctx.load_query_obj(q)
    assert all(r in (8, 16, 24, 28, 32) for r in ctx.query_info()["refill_min"])


def test_estimate_until(ctx, G, c0):
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[0])
    r = ctx.estimate_until(G.ALLEY, 5, rel_se=1e-3, min_samples=10_000, max_samples=10**9)
    assert math.sqrt(r["variance"]) <= 1e-3 * r["estimate"]
    full = ctx.estimate(G.ALLEY, r["n"], 5)  # same sample ids: same aggregate
    assert full["n_valid"] == r["n_valid"]
    assert full["sum"] == pytest.approx(r["sum"], rel=REL)
    with pytest.raises(G.GswordError):
        ctx.estimate_until(G.ALLEY, 5, rel_se=0.0)


def test_fault_injection_queue_corruption_is_caught(ctx, G, c0):
    """a corrupted sample-queue counter skips sample ids; the n / n_valid
    accounting of the synchronous calls catches it (GSWORD_EFAULT) and the option is
    one-shot, so the next call is clean."""
    import torch
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[1])
    n = 50_000
    clean = ctx.estimate(G.ALLEY, n, seed=3)
    for call in (lambda: ctx.estimate(G.ALLEY, n, seed=3),
                 lambda: ctx.trace_samples(G.WJ, 0, n, 3),
                 lambda: ctx.count_sectors(G.ALLEY, 0, n, 3)):
        ctx.set_option(G.OPT_FAULT_QUEUE, 4096)
        with pytest.raises(G.GswordError) as ei:
            call()
        assert ei.value.status == -9 and "accounted for 45904" in str(ei.value)
    again = ctx.estimate(G.ALLEY, n, seed=3)
    assert again["n"] == n and again["sum"] == clean["sum"] and again["n_valid"] == clean["n_valid"]
    # the asynchronous form leaves the check to the caller: n in the 4-vector is short
    out = torch.zeros(4, dtype=torch.float64, device="cuda:0")
    ctx.set_stream(torch.cuda.current_stream())
    ctx.set_option(G.OPT_FAULT_QUEUE, 10 * n)  # beyond the range: nothing runs
    ctx.estimate_async(G.ALLEY, 0, n, 3, out)
    assert out.cpu().tolist()[3] == 0.0
    ctx.set_stream(None)


@pytest.mark.parametrize("occ", [0, 1, 2])
def test_refill32_depth_synchronous_kernel(ctx, G, c0, occ):
    """Refill threshold 32 selects the depth-synchronous Alley estimate kernel (each lane runs
    its own exclusion tests, no task pool; LOCK in gsword_kernels.cu): aggregates equal the
    oracle's on C0, small random graphs, the three C1 queries and C2, for every occupancy
    variant and the spanning-tree specialisation (paths)."""
    ctx.set_option(G.OPT_AUTOTUNE, 0)
    ctx.set_option(G.OPT_REFILL_MIN, 32)
    ctx.set_option(G.OPT_OCCUPANCY, occ)
    try:
        cases = []
        g, qs = c0
        cases += [(g, q, 100_000) for q in qs]
        for s in range(4):
            gs = gen.random_small_graph(30, 0.4, 2, seed=900 + s)
            cases.append((gs, gen.random_connected_query(6, 0.5, 2, 910 + s), 30_000))
        g1, q1 = gen.config_c1()
        cases += [(g1, q, 100_000) for q in q1]
        g2, q2 = gen.config_c2()
        cases += [(g2, q, 100_000) for q in q2]
        loaded = None
        for gg, q, n in cases:
            if loaded is not gg:
                ctx.load_graph_obj(gg)
                loaded = gg
            ctx.load_query_obj(q)
            agg = ctx.estimate(G.ALLEY, n, seed=13, first=5)
            y, _ = oracle.sample_range(gg, q, G.ALLEY, 13, 5, n, records=False, threads=8)
            _agg_close(agg, oracle.aggregate(y), G)
    finally:
        ctx.set_option(G.OPT_AUTOTUNE, 1)
        ctx.set_option(G.OPT_REFILL_MIN, 16)
        ctx.set_option(G.OPT_OCCUPANCY, -1)


def test_wanderjoin_alley_cross_check(ctx, G, c0):
    """on the same (G, q) the two estimators agree within their combined 3
    sigma where both see at least 1e5 valid samples (C0 at 1e7, C1 dense at 1e8), and on
    cyclic queries Alley's relative standard error is below WanderJoin's.  On C1's
    cyclic query WanderJoin is in the heavy-tailed underestimation regime (~4e4 valid of 1e8,
    P:L381): its sample variance misses the rare huge weights, so a 3-sigma agreement is not
    expected there (seed 17: WJ 1.45e23 +- 0.58e23 against Alley 1.56e24 +- 0.15e24; seed 42
    in the bench: 1.88e24 +- 1.12e24 against 1.91e24 +- 0.40e24)."""
    cases = []
    g, qs = c0
    cases += [(g, q, 10_000_000) for q in qs]
    g1, q1 = gen.config_c1()
    cases += [(g1, q, 100_000_000) for q in q1[1:]]
    loaded = None
    agreed = 0
    for gg, q, n in cases:
        if loaded is not gg:
            ctx.load_graph_obj(gg)
            loaded = gg
        ctx.load_query_obj(q)
        wj = ctx.estimate(G.WJ, n, seed=17)
        al = ctx.estimate(G.ALLEY, n, seed=17)
        if min(wj["n_valid"], al["n_valid"]) >= 100_000:
            se = math.sqrt(max(wj["variance"], 0.0) + max(al["variance"], 0.0))
            assert abs(wj["estimate"] - al["estimate"]) <= 3 * se + 1e-9, (q.name, wj, al)
            agreed += 1
        if len(q.edges()) > q.nq - 1 and wj["n_valid"] > 0 and al["n_valid"] > 0:
            rel = lambda r: math.sqrt(max(r["variance"], 0.0)) / r["estimate"]
            assert rel(al) <= rel(wj), q.name
    assert agreed >= 8


def test_stream_switch_orders_reused_buffers(ctx, G, c0):
    """gsword_set_stream: work issued on a new stream starts after the context's
    work on the old one (every launch reuses the queue, partials and output buffers).  A long
    Alley estimate on stream A, a switch to stream B and a WanderJoin estimate there must give
    the sequential results."""
    import torch
    g, qs = c0
    ctx.load_graph_obj(g)
    ctx.load_query_obj(qs[6])
    ref_al = ctx.estimate(G.ALLEY, 30_000_000, seed=21)
    ref_wj = ctx.estimate(G.WJ, 3_000_000, seed=22)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    oa = torch.zeros(4, dtype=torch.float64, device="cuda:0")
    ob = torch.zeros(4, dtype=torch.float64, device="cuda:0")
    try:
        ctx.set_stream(sa)
        ctx.estimate_async(G.ALLEY, 0, 30_000_000, 21, oa)
        ctx.set_stream(sb)
        ctx.estimate_async(G.WJ, 0, 3_000_000, 22, ob)
        sa.synchronize()
        sb.synchronize()
    finally:
        ctx.set_stream(None)
    for out, ref in ((oa, ref_al), (ob, ref_wj)):
        r = G.finalize(out.cpu().numpy())
        assert r["n"] == ref["n"] and r["n_valid"] == ref["n_valid"]
        assert r["sum"] == pytest.approx(ref["sum"], rel=REL, abs=0.0)


def test_two_contexts_run_concurrently(G, c0):
    """Two contexts on one device (e.g. two serving workers) on their own streams, launched
    back to back without host synchronisation: both results equal the sequential ones."""
    import torch
    g, qs = c0
    with G.Context(0) as c1, G.Context(0) as c2:
        for c in (c1, c2):
            c.load_graph_obj(g)
        c1.load_query_obj(qs[0])
        c2.load_query_obj(qs[7])
        ref1 = c1.estimate(G.ALLEY, 20_000_000, seed=5)
        ref2 = c2.estimate(G.WJ, 20_000_000, seed=6)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        o1 = torch.zeros(4, dtype=torch.float64, device="cuda:0")
        o2 = torch.zeros(4, dtype=torch.float64, device="cuda:0")
        c1.set_stream(s1)
        c2.set_stream(s2)
        c1.estimate_async(G.ALLEY, 0, 20_000_000, 5, o1)
        c2.estimate_async(G.WJ, 0, 20_000_000, 6, o2)
        torch.cuda.synchronize()
        for out, ref in ((o1, ref1), (o2, ref2)):
            r = G.finalize(out.cpu().numpy())
            assert r["n"] == ref["n"] and r["n_valid"] == ref["n_valid"]
            assert r["sum"] == pytest.approx(ref["sum"], rel=REL, abs=0.0)
        c1.set_stream(None)
        c2.set_stream(None)


def test_estimate_instance_per_sample(ctx, G, c0, c1):
    """The timed estimate instance (the autotuned OCC / TREE / LOCK specialisation that
    bench.py launches, not the trace build) checked sample by sample: a one-id range makes its
    aggregate the sample's own weight, which must equal the oracle's bit for bit (a single
    value passes the compensated sums and the double-double reduction unchanged); 64-id windows
    (two warps' worth of lanes sharing the task pool and the refill queue) must match the
    oracle's window sums at 1e-12 with n_valid exact.  C0 and the C1 bench queries, the
    cyclic one included."""
    for (g, qs), qidx in ((c0, range(len(c0[1]))), (c1, range(len(c1[1])))):
        ctx.load_graph_obj(g)
        for qi in qidx:
            q = qs[qi]
            ctx.load_query_obj(q)
            for m in (0, 1):
                y, ref = oracle.sample_range(g, q, m, 42, 0, 6400, records=True, threads=8)
                y = np.asarray(y, dtype=np.float64)
                valid = np.nonzero(ref["valid"])[0]
                invalid = np.nonzero(ref["valid"] == 0)[0]
                ids = list(valid[:40]) + list(invalid[:8]) + [6399]
                for i in ids:
                    r = ctx.estimate(m, 1, 42, first=int(i))
                    assert r["n"] == 1 and r["n_valid"] == int(ref["valid"][i])
                    w = float(y[i])
                    assert r["sum"] == w, (g.name, q.name, m, int(i), r["sum"], w)
                for first in range(0, 6400, 640):
                    r = ctx.estimate(m, 64, 42, first=first)
                    w = y[first:first + 64]
                    assert r["n"] == 64 and r["n_valid"] == int((ref["valid"][first:first + 64] != 0).sum())
                    assert r["sum"] == pytest.approx(float(np.sum(w)), rel=REL, abs=0.0)
                    assert r["sumsq"] == pytest.approx(float(np.sum(w * w)), rel=REL, abs=0.0)



@pytest.mark.parametrize("occ", [0, 1, 2])
def test_estimate_instance_per_sample_each_occupancy(ctx, G, c1, occ):
    """Every occupancy variant of the estimate kernel, forced (the autotune picks variant 2 for C1
    dense Alley since the register trims), checked sample by sample on the C1
    dense and cyclic queries: one-id ranges bit-exact against the oracle's weight, 64-id windows
    at 1e-12 with n_valid exact."""
    g, qs = c1
    ctx.load_graph_obj(g)
    ctx.set_option(G.OPT_OCCUPANCY, occ)
    try:
        for q in qs[1:]:
            ctx.load_query_obj(q)
            for m in (0, 1):
                y, ref = oracle.sample_range(g, q, m, 43, 0, 3200, records=True, threads=8)
                y = np.asarray(y, dtype=np.float64)
                valid = np.nonzero(ref["valid"])[0]
                invalid = np.nonzero(ref["valid"] == 0)[0]
                for i in list(valid[:24]) + list(invalid[:6]):
                    r = ctx.estimate(m, 1, 43, first=int(i))
                    assert r["n"] == 1 and r["n_valid"] == int(ref["valid"][i])
                    assert r["sum"] == float(y[i]), (q.name, m, occ, int(i))
                for first in range(0, 3200, 640):
                    r = ctx.estimate(m, 64, 43, first=first)
                    w = y[first:first + 64]
                    assert r["n_valid"] == int((ref["valid"][first:first + 64] != 0).sum())
                    assert r["sum"] == pytest.approx(float(np.sum(w)), rel=REL, abs=0.0)
                    assert r["sumsq"] == pytest.approx(float(np.sum(w * w)), rel=REL, abs=0.0)
    finally:
        ctx.set_option(G.OPT_OCCUPANCY, -1)