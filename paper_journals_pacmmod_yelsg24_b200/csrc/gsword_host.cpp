// gsword_host.cpp — host side of the C ABI declared in include/gsword.h.
//
// Owns the context (device buffers, stream, events), validates and re-lays out the
// data graph (canonical CSR -> adjacency sorted by (label, id) + per-(vertex, label)
// segment offsets + label buckets), compiles the query + matching order into the
// per-depth plan that the kernels stage in shared memory (Def. 2
// GetMinCandidate inputs), and launches the sampling + reduction kernels.
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <limits>
#include <map>
#include <string>
#include <thread>
#include <vector>

#include "internal.h"

using gsword::DeviceGraph;
using gsword::LaunchCfg;
using gsword::Partial;
using gsword::Plan;

namespace {

thread_local std::string g_last_error;

int fail(int status, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return status;
}

int cuda_fail(cudaError_t e, const char* what) {
    return fail(GSWORD_ECUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define CUDA_TRY(expr)                                  \
    do {                                                \
        cudaError_t _e = (expr);                        \
        if (_e != cudaSuccess) return cuda_fail(_e, #expr); \
    } while (0)

unsigned host_threads() {
    unsigned t = std::thread::hardware_concurrency();
    return t == 0 ? 1 : std::min(t, 32u);
}

// Run f(lo, hi) over [0, n) split into contiguous ranges on host threads.
template <class F>
void parallel_for(int64_t n, F f) {
    const unsigned T = (n < (1 << 16)) ? 1u : host_threads();
    if (T == 1) {
        f((int64_t)0, n);
        return;
    }
    std::vector<std::thread> ts;
    for (unsigned t = 0; t < T; ++t) {
        const int64_t lo = n * t / T, hi = n * (t + 1) / T;
        ts.emplace_back([=] { f(lo, hi); });
    }
    for (auto& th : ts) th.join();
}

int check_graph_impl(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                     int32_t n_labels) {
    if (n < 0 || !row_ptr) return fail(GSWORD_EINVAL, "load_graph: n_vertices < 0 or row_ptr NULL");
    if (n_labels < 1) return fail(GSWORD_EINVAL, "load_graph: n_labels must be >= 1");
    if (!labels && n_labels != 1) return fail(GSWORD_EINVAL, "load_graph: labels NULL requires n_labels == 1");
    if (n >= (int64_t)1 << 31) return fail(GSWORD_ELIMIT, "load_graph: |V| >= 2^31");
    if (n * (int64_t)n_labels >= ((int64_t)1 << 31)) return fail(GSWORD_ELIMIT, "load_graph: |V| * n_labels >= 2^31");
    if (row_ptr[0] != 0) return fail(GSWORD_EGRAPH, "load_graph: row_ptr[0] != 0");
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] < row_ptr[v]) return fail(GSWORD_EGRAPH, "load_graph: row_ptr decreasing at %lld", (long long)v);
    const int64_t nnz = row_ptr[n];
    if (nnz >= ((int64_t)1 << 31) - 1) return fail(GSWORD_ELIMIT, "load_graph: 2|E| >= 2^31");
    if (nnz > 0 && !col) return fail(GSWORD_EINVAL, "load_graph: col NULL");
    if (labels) {
        for (int64_t v = 0; v < n; ++v)
            if (labels[v] < 0 || labels[v] >= n_labels)
                return fail(GSWORD_EINVAL, "load_graph: label of vertex %lld out of range", (long long)v);
    }
    std::atomic<int64_t> bad_row{-1};
    std::atomic<int> bad_kind{0};
    parallel_for(n, [&](int64_t lo, int64_t hi) {
        for (int64_t v = lo; v < hi && bad_row.load(std::memory_order_relaxed) < 0; ++v) {
            for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) {
                const int32_t w = col[i];
                int kind = 0;
                if (w < 0 || w >= n) kind = 1;
                else if (w == v) kind = 2;
                else if (i > row_ptr[v] && col[i - 1] >= w) kind = 3;
                else {
                    const int32_t* b = col + row_ptr[w];
                    const int32_t* e = col + row_ptr[w + 1];
                    if (!std::binary_search(b, e, (int32_t)v)) kind = 4;
                }
                if (kind) {
                    int64_t expect = -1;
                    if (bad_row.compare_exchange_strong(expect, v)) bad_kind = kind;
                    return;
                }
            }
        }
    });
    if (bad_row >= 0) {
        static const char* what[] = {"", "neighbour id out of range", "self loop", "row not strictly ascending",
                                     "asymmetric adjacency"};
        return fail(GSWORD_EGRAPH, "load_graph: %s at vertex %lld", what[bad_kind.load()], (long long)bad_row.load());
    }
    return GSWORD_OK;
}

int plan_query_impl(int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                    const int32_t* order, int32_t n_labels, Plan* plan, gsword_plan_info* info) {
    if (nq < 1) return fail(GSWORD_EINVAL, "load_query: n_qv < 1");
    if (nq > GSWORD_MAX_QV) return fail(GSWORD_ELIMIT, "load_query: n_qv > %d", GSWORD_MAX_QV);
    if (!q_row_ptr || !q_labels || !order) return fail(GSWORD_EINVAL, "load_query: NULL argument");
    if (q_row_ptr[0] != 0 || (q_row_ptr[nq] > 0 && !q_col)) return fail(GSWORD_EINVAL, "load_query: bad query CSR");
    bool adj[GSWORD_MAX_QV][GSWORD_MAX_QV] = {};
    for (int u = 0; u < nq; ++u) {
        if (q_row_ptr[u + 1] < q_row_ptr[u]) return fail(GSWORD_EINVAL, "load_query: bad query CSR");
        if (q_labels[u] < 0 || q_labels[u] >= n_labels)
            return fail(GSWORD_EINVAL, "load_query: label of query vertex %d out of range", u);
        for (int32_t i = q_row_ptr[u]; i < q_row_ptr[u + 1]; ++i) {
            const int32_t w = q_col[i];
            if (w < 0 || w >= nq || w == u) return fail(GSWORD_EINVAL, "load_query: bad query edge (%d,%d)", u, w);
            adj[u][w] = true;
        }
    }
    for (int u = 0; u < nq; ++u)
        for (int w = 0; w < nq; ++w)
            if (adj[u][w] != adj[w][u]) return fail(GSWORD_EINVAL, "load_query: query adjacency not symmetric");
    bool seen[GSWORD_MAX_QV] = {};
    for (int d = 0; d < nq; ++d) {
        if (order[d] < 0 || order[d] >= nq || seen[order[d]])
            return fail(GSWORD_EORDER, "load_query: order is not a permutation");
        seen[order[d]] = true;
    }
    Plan p;
    std::memset(&p, 0, sizeof(p));
    p.nq = nq;
    for (int d = 0; d < nq; ++d) {
        const int u = order[d];
        gsword::PlanStep& s = p.step[d];
        s.label = q_labels[u];
        for (int j = 0; j < d; ++j) {
            if (adj[order[j]][u]) s.back |= 1u << j;
            if (q_labels[order[j]] == q_labels[u]) s.dup |= 1u << j;
        }
        s.nback = __builtin_popcount(s.back);
        p.uq[d] = (uint8_t)u;
        for (int j = 0; j < nq; ++j)
            if (j != d && adj[order[j]][u]) p.qadj[d] |= 1u << j;
        if (d > 0 && s.back == 0)
            return fail(GSWORD_EORDER, "load_query: order prefix %d is not connected (reading A13)", d);
    }
    // directed query edges (a -> b), enumerated in (a, b) order: candidate-graph rows
    int eid[GSWORD_MAX_QV][GSWORD_MAX_QV];
    int ne = 0;
    for (int a = 0; a < nq; ++a)
        for (int b = 0; b < nq; ++b) eid[a][b] = adj[a][b] ? ne++ : -1;
    for (int d = 0; d < nq; ++d)
        for (int j = 0; j < d; ++j)
            if (adj[order[j]][order[d]]) p.eidx[d][j] = (uint8_t)eid[order[j]][order[d]];
    if (plan) *plan = p;
    if (info) {
        std::memset(info, 0, sizeof(*info));
        info->nq = nq;
        for (int d = 0; d < nq; ++d) {
            info->label[d] = p.step[d].label;
            info->back_mask[d] = p.step[d].back;
            info->dup_mask[d] = p.step[d].dup;
        }
    }
    return GSWORD_OK;
}

}  // namespace

struct gsword_ctx {
    int device = 0;
    int num_sms = 148;
    cudaStream_t own_stream = nullptr;
    cudaStream_t stream = nullptr;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;    // around a whole estimate
    cudaEvent_t evk0 = nullptr, evk1 = nullptr;  // around the last sampling-kernel launch
    cudaEvent_t ev_switch = nullptr;             // orders a stream switch after the old stream's work
    // graph
    bool graph_loaded = false;
    int32_t* d_col = nullptr;
    bool own_col = true;      // false: borrowed from the caller (gsword_load_graph_device)
    bool own_vlabel = true;
    uint32_t* d_seg = nullptr;
    void* d_hot = nullptr;     // one allocation: [Bloom filter words][seg] (the L2-window target)
    size_t hot_bytes = 0;
    int32_t* d_bucket = nullptr;
    unsigned long long* d_bloom = nullptr;
    uint64_t bloom_words = 0;
    unsigned long long* d_eset = nullptr;
    uint64_t eset_buckets = 0;
    int64_t n = 0, nnz = 0;
    int32_t n_labels = 1;
    std::vector<int64_t> label_off;
    // query
    bool query_loaded = false;
    Plan plan{};
    int32_t* d_vlabel = nullptr;      // vertex labels (filters need them on the device)
    std::vector<uint64_t> pair_freq;  // data adjacency entries per (label, label) (QuickSI order)
    // candidate graph of the loaded query (filters 1-2, NEXT-1)
    int opt_filter = 0;
    int q_filter = 0;                 // filter the loaded query was built with
    uint32_t* d_cbits = nullptr;
    uint32_t* d_crank = nullptr;   // rank directory of d_cbits (Fig. 4, 2nd CSR)
    uint2* d_cg_edge = nullptr;    // per directed query edge: {offset base, source u}
    uint64_t cg_bytes = 0;         // device bytes of the candidate graph
    uint32_t* d_cg_off = nullptr;
    int32_t* d_clist = nullptr;
    int32_t* d_cand0 = nullptr;
    uint32_t cwords = 0;
    uint64_t cg_entries = 0;
    double cg_seconds = 0.0;
    uint64_t cand_count[GSWORD_MAX_QV] = {};

    void free_query() {
        if (d_cbits) cudaFree(d_cbits);
        if (d_crank) cudaFree(d_crank);
        if (d_cg_edge) cudaFree(d_cg_edge);
        if (d_cg_off) cudaFree(d_cg_off);
        if (d_clist) cudaFree(d_clist);
        if (d_cand0) cudaFree(d_cand0);
        d_cbits = nullptr;
        d_crank = nullptr;
        d_cg_edge = nullptr;
        cg_bytes = 0;
        d_cg_off = nullptr;
        d_clist = nullptr;
        d_cand0 = nullptr;
        cg_entries = 0;
        q_filter = 0;
        query_loaded = false;
    }
    // scratch
    unsigned long long* d_queue = nullptr;
    Partial* d_partials = nullptr;
    int partial_cap = 0;
    double* d_out4 = nullptr;
    double* d_sectors = nullptr;
    unsigned long long* d_phase = nullptr;  // count build: warp cycles per loop phase
    double h_phase[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    // options
    int opt_blocks_per_sm = 0;
    int opt_threads = 256;
    int opt_chunk = 256;
    int opt_l2 = 2;  // L2 persistence window over the filter + seg (measured 3-5% on C1 Alley)
    int opt_coop = 64;
    int opt_bloom = 1;
    int opt_bloom_bits = 16;  // filter bits per undirected edge (applied at the next graph load)
    int opt_sched = 0;
    int opt_refill_min = 16;
    int opt_autotune = 1;         // pick the refill threshold per method with pilots at query load
    int opt_streaming = 0;        // Alley by warp streaming (Alg. 3, NEXT-3 comparison mode)
    int opt_variant = 0;          // GSWORD_VARIANT_* bits (readings A3/A5 comparison variants)
    int tuned_refill[2] = {0, 0}; // 0 = not tuned  // measured: 1.2-1.35x over refilling every round on C1, neutral on C2/C3
    // autotune results per (query, options) since the last graph load: reloading a query
    // (a serving loop re-issuing the same query) reuses them instead of re-running pilots
    int tuned_occ[2] = {0, 0};    // occupancy variant of the estimate kernel (kModeOccShift)
    int opt_occ = -1;             // GSWORD_OPT_OCCUPANCY: -1 autotuned, else forced
    uint64_t opt_fault_queue = 0;  // GSWORD_OPT_FAULT_QUEUE: one-shot corrupted queue start
    int opt_trawl_warp = 1;        // GSWORD_OPT_TRAWL_WARP: warp-cooperative trawling enumeration
    struct Tuned {
        int refill[2], occ[2];
    };
    std::map<std::string, Tuned> tune_cache;
    int opt_eset = 1;
    // last launch
    int last_grid = 0, last_threads = 0;

    void free_graph() {
        free_query();
        if (d_vlabel && own_vlabel) cudaFree(d_vlabel);
        d_vlabel = nullptr;
        if (d_col && own_col) cudaFree(d_col);
        own_col = own_vlabel = true;
        if (d_hot) cudaFree(d_hot);
        if (d_bucket) cudaFree(d_bucket);
        if (d_eset) cudaFree(d_eset);
        d_hot = nullptr;
        hot_bytes = 0;
        d_bloom = nullptr;
        bloom_words = 0;
        d_eset = nullptr;
        eset_buckets = 0;
        d_col = nullptr;
        d_seg = nullptr;
        d_bucket = nullptr;
        graph_loaded = false;
        tune_cache.clear();
        query_loaded = false;
    }
};

namespace {

// Failure detection: the kernels count every sample id they ran; the total
// must be the requested range size, else a queue counter or partial was corrupted.
int check_accounting(const double* h4, uint64_t n_samples, const char* what) {
    if ((uint64_t)h4[3] != n_samples || h4[2] > h4[3])
        return fail(GSWORD_EFAULT, "%s: the kernels accounted for %.0f samples (%.0f valid) of %llu requested", what,
                    h4[3], h4[2], (unsigned long long)n_samples);
    return GSWORD_OK;
}

int ensure_ready(gsword_ctx* ctx, int method) {
    if (!ctx) return fail(GSWORD_EINVAL, "NULL context");
    if (method != GSWORD_WJ && method != GSWORD_ALLEY) return fail(GSWORD_EINVAL, "unknown method %d", method);
    if (!ctx->graph_loaded) return fail(GSWORD_ENOGRAPH, "no graph loaded");
    if (!ctx->query_loaded) return fail(GSWORD_ENOQUERY, "no query loaded");
    cudaError_t e = cudaSetDevice(ctx->device);
    if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");
    return GSWORD_OK;
}

int apply_l2_window(gsword_ctx* ctx) {
    if (!ctx->graph_loaded) return GSWORD_OK;
    cudaStreamAttrValue attr;
    std::memset(&attr, 0, sizeof(attr));
    if (ctx->opt_l2) {
        int max_persist = 0, max_window = 0;
        CUDA_TRY(cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, ctx->device));
        CUDA_TRY(cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, ctx->device));
        // mode 1: the adjacency array; mode 2: the hot buffer (Bloom filter + seg)
        void* base = ctx->opt_l2 == 1 ? (void*)ctx->d_col : ctx->d_hot;
        const size_t bytes = ctx->opt_l2 == 1 ? (size_t)ctx->nnz * sizeof(int32_t) : ctx->hot_bytes;
        const size_t window = std::min(bytes, (size_t)max_window);
        const size_t persist = std::min((size_t)max_persist, window);
        CUDA_TRY(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, persist));
        attr.accessPolicyWindow.base_ptr = base;
        attr.accessPolicyWindow.num_bytes = window;
        attr.accessPolicyWindow.hitRatio = window ? (float)std::min(1.0, (double)persist / (double)window) : 0.f;
        attr.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    } else {
        attr.accessPolicyWindow.num_bytes = 0;
        attr.accessPolicyWindow.hitRatio = 0.f;
        attr.accessPolicyWindow.hitProp = cudaAccessPropertyNormal;
        attr.accessPolicyWindow.missProp = cudaAccessPropertyNormal;
    }
    CUDA_TRY(cudaStreamSetAttribute(ctx->stream, cudaStreamAttributeAccessPolicyWindow, &attr));
    return GSWORD_OK;
}

// occupancy variant of the estimate kernel in use for `method`
int occ_variant(const gsword_ctx* ctx, int method) {
    if (ctx->opt_occ >= 0) return ctx->opt_occ;
    return ctx->opt_autotune ? ctx->tuned_occ[method & 1] : 0;
}

// refill threshold in use for `method` (autotuned or GSWORD_OPT_REFILL_MIN)
int refill_min_of(const gsword_ctx* ctx, int method) {
    return (ctx->opt_autotune && ctx->tuned_refill[method & 1] > 0) ? ctx->tuned_refill[method & 1] : ctx->opt_refill_min;
}

// every position d >= 1 has exactly one backward neighbour (spanning-tree order)
bool plan_is_tree(const Plan& p) {
    for (int d = 1; d < p.nq; ++d)
        if (p.step[d].nback != 1) return false;
    return true;
}

int launch_config(gsword_ctx* ctx, int method, int mode, LaunchCfg* cfg) {
    size_t smem = 0;
    const int rows = gsword::sample_smem_rows(method, ctx->query_loaded ? std::max(1, ctx->plan.nq) : GSWORD_MAX_QV,
                                              ctx->opt_coop);
    const int occ = gsword::max_blocks_per_sm(method, mode, ctx->opt_threads, rows, &smem);
    if (occ <= 0) return fail(GSWORD_ECUDA, "kernel does not fit on the device (threads=%d)", ctx->opt_threads);
    const int bps = ctx->opt_blocks_per_sm > 0 ? std::min(ctx->opt_blocks_per_sm, occ) : occ;
    cfg->grid = ctx->num_sms * bps;
    cfg->threads = ctx->opt_threads;
    cfg->chunk = ctx->opt_sched ? ((ctx->opt_chunk + 31) / 32) * 32 : ctx->opt_chunk;  // groups of 32 ids
    cfg->coop_threshold = ctx->opt_coop;
    cfg->sched = ctx->opt_sched;
    cfg->ms_rows = rows;
    cfg->refill_min = (uint32_t)refill_min_of(ctx, method);
    if (cfg->grid > ctx->partial_cap) {
        if (ctx->d_partials) cudaFree(ctx->d_partials);
        ctx->d_partials = nullptr;
        CUDA_TRY(cudaMalloc(&ctx->d_partials, sizeof(Partial) * (size_t)cfg->grid));
        ctx->partial_cap = cfg->grid;
    }
    ctx->last_grid = cfg->grid;
    ctx->last_threads = cfg->threads;
    return GSWORD_OK;
}

DeviceGraph device_graph(const gsword_ctx* ctx) {
    DeviceGraph g;
    g.col = ctx->d_col;
    g.seg = ctx->d_seg;
    g.bucket = ctx->q_filter ? ctx->d_cand0 : ctx->d_bucket;
    g.clist = ctx->q_filter ? ctx->d_clist : ctx->d_col;
    g.cg_off = ctx->q_filter ? ctx->d_cg_off : nullptr;
    g.cbits = ctx->q_filter ? ctx->d_cbits : nullptr;
    g.crank = ctx->q_filter ? ctx->d_crank : nullptr;
    g.cg_edge = ctx->q_filter ? ctx->d_cg_edge : nullptr;
    g.cwords = ctx->cwords;
    g.bloom = ctx->opt_bloom ? ctx->d_bloom : nullptr;
    g.bloom_mask = ctx->bloom_words ? ctx->bloom_words - 1 : 0;
    g.eset = ctx->opt_eset ? ctx->d_eset : nullptr;
    g.eset_mask = ctx->eset_buckets ? ctx->eset_buckets - 1 : 0;
    g.n = ctx->n;
    g.nnz = ctx->nnz;
    g.n_labels = ctx->n_labels;
    return g;
}

int run(gsword_ctx* ctx, int method, int mode, uint64_t first, uint64_t count, uint64_t seed, double* d_out4,
        gsword_sample_record* d_records, double* d_sectors) {
    if (first + count < first) return fail(GSWORD_EINVAL, "sample-id range [first, first + n) overflows u64");
    if (ctx->q_filter) mode |= gsword::kModeCG;
    if (method == GSWORD_ALLEY && ctx->opt_streaming && (mode & 3) != gsword::kModeCount) mode |= gsword::kModeStream;
    if (ctx->opt_sched != 0) mode |= gsword::kModeSync;
    if ((mode & (3 | gsword::kModeSync | gsword::kModeStream)) == gsword::kModeEstimate) {
        mode |= occ_variant(ctx, method) << gsword::kModeOccShift;
        if (plan_is_tree(ctx->plan)) mode |= gsword::kModeTree;
        if (method == GSWORD_ALLEY && refill_min_of(ctx, method) == 32) mode |= gsword::kModeLock;
    }
    LaunchCfg cfg;
    int rc = launch_config(ctx, method, mode, &cfg);
    if (rc) return rc;
    cfg.queue_start = ctx->opt_fault_queue;
    ctx->opt_fault_queue = 0;
    CUDA_TRY(cudaEventRecord(ctx->evk0, ctx->stream));
    const bool counting = (mode & 3) == gsword::kModeCount;
    if (counting) CUDA_TRY(cudaMemsetAsync(ctx->d_phase, 0, 8 * sizeof(unsigned long long), ctx->stream));
    cudaError_t e = gsword::launch_sample(method, mode, device_graph(ctx),
                                          gsword::plan_variant(ctx->plan, method, ctx->opt_variant), cfg, first, count, seed,
                                          ctx->d_queue, ctx->d_partials, d_records,
                                          counting ? ctx->d_phase : nullptr, ctx->stream);
    if (e != cudaSuccess) return cuda_fail(e, "launch sample kernel");
    CUDA_TRY(cudaEventRecord(ctx->evk1, ctx->stream));
    e = gsword::launch_reduce(ctx->d_partials, cfg.grid, d_out4, d_sectors, ctx->stream);
    if (e != cudaSuccess) return cuda_fail(e, "launch reduce kernel");
    return GSWORD_OK;
}

// QuickSI-style matching order (NEXT-4, reading A22): infrequent edges first.
// vfreq[l] = |{v : L(v) = l}|; pfreq(l1, l2) = data adjacency entries with those labels.
int quicksi_order_impl(int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                       int32_t n_labels, const std::vector<int64_t>& label_off, const std::vector<uint64_t>& pfreq,
                       int32_t* order) {
    Plan tmp;
    std::vector<int32_t> ident((size_t)std::max(nq, 1));
    for (int i = 0; i < nq; ++i) ident[(size_t)i] = i;
    // validates the query CSR and labels (any order works for that; connectivity checked below)
    if (nq < 1) return fail(GSWORD_EINVAL, "order: n_qv < 1");
    if (nq > GSWORD_MAX_QV) return fail(GSWORD_ELIMIT, "order: n_qv > %d", GSWORD_MAX_QV);
    bool adj[GSWORD_MAX_QV][GSWORD_MAX_QV] = {};
    int deg[GSWORD_MAX_QV] = {};
    for (int u = 0; u < nq; ++u) {
        if (q_labels[u] < 0 || q_labels[u] >= n_labels) return fail(GSWORD_EINVAL, "order: label out of range");
        for (int32_t i = q_row_ptr[u]; i < q_row_ptr[u + 1]; ++i) {
            if (q_col[i] < 0 || q_col[i] >= nq || q_col[i] == u) return fail(GSWORD_EINVAL, "order: bad query edge");
            adj[u][q_col[i]] = adj[q_col[i]][u] = true;
        }
    }
    for (int u = 0; u < nq; ++u)
        for (int w = 0; w < nq; ++w) deg[u] += adj[u][w] ? 1 : 0;
    auto vf = [&](int u) { return (uint64_t)(label_off[(size_t)q_labels[u] + 1] - label_off[(size_t)q_labels[u]]); };
    auto ef = [&](int a, int b) -> uint64_t {
        if (pfreq.empty()) return vf(a) * vf(b);
        return pfreq[(size_t)q_labels[a] * (size_t)n_labels + (size_t)q_labels[b]];
    };
    if (nq == 1) {
        order[0] = 0;
        return GSWORD_OK;
    }
    // first edge: (freq, -(deg a + deg b), min id, max id)
    int ba = -1, bb = -1;
    for (int a = 0; a < nq; ++a)
        for (int b = a + 1; b < nq; ++b) {
            if (!adj[a][b]) continue;
            if (ba < 0) { ba = a; bb = b; continue; }
            const uint64_t f = ef(a, b), fb = ef(ba, bb);
            const int dg = deg[a] + deg[b], dgb = deg[ba] + deg[bb];
            if (f < fb || (f == fb && dg > dgb)) { ba = a; bb = b; }
        }
    if (ba < 0) return fail(GSWORD_EORDER, "order: query has no edge but %d vertices", nq);
    auto vkey_less = [&](int x, int y) {  // (vertex freq, -deg, id)
        if (vf(x) != vf(y)) return vf(x) < vf(y);
        if (deg[x] != deg[y]) return deg[x] > deg[y];
        return x < y;
    };
    bool used[GSWORD_MAX_QV] = {};
    order[0] = vkey_less(ba, bb) ? ba : bb;
    order[1] = order[0] == ba ? bb : ba;
    used[ba] = used[bb] = true;
    for (int d = 2; d < nq; ++d) {
        int best = -1;
        uint64_t bf = 0;
        for (int b = 0; b < nq; ++b) {
            if (used[b]) continue;
            for (int j = 0; j < d; ++j) {
                const int a = order[j];
                if (!adj[a][b]) continue;
                const uint64_t f = ef(a, b);
                if (best < 0 || f < bf || (f == bf && (deg[b] > deg[best] || (deg[b] == deg[best] && b < best)))) {
                    best = b;
                    bf = f;
                }
            }
        }
        if (best < 0) return fail(GSWORD_EORDER, "order: query is not connected");
        order[d] = best;
        used[best] = true;
    }
    (void)tmp;
    return GSWORD_OK;
}

void label_pair_freq(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int32_t nL,
                     std::vector<uint64_t>* out) {
    out->clear();
    if (nL > 1024) return;  // too many labels for a dense table: vertex frequencies only
    out->assign((size_t)nL * (size_t)nL, 0);
    for (int64_t v = 0; v < n; ++v) {
        const int32_t lv = labels ? labels[v] : 0;
        for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i)
            (*out)[(size_t)lv * (size_t)nL + (size_t)(labels ? labels[col[i]] : 0)] += 1;
    }
}

// Candidate graph of the query (NEXT-1; Def. 4-5) in the three-CSR format of
// Fig. 4 (DeviceGraph in internal.h): C(u) by the filter as a bitmap + rank
// directory per query vertex, then per directed query edge a -> b the |C(a)| + 1 offsets
// of the local lists C(a, b, v) = N(v) ∩ C(b) (v in C(a), ascending), chained across the
// edges into one list array, and the ascending list of C(phi[0]) for the seed.
int build_candidate_graph(gsword_ctx* ctx, int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col,
                          const int32_t* q_labels, const int32_t* order, Plan* p) {
    cudaStream_t st = ctx->stream;
    const int64_t n = ctx->n;
    cudaEvent_t e0, e1;
    CUDA_TRY(cudaEventCreate(&e0));
    CUDA_TRY(cudaEventCreate(&e1));
    CUDA_TRY(cudaEventRecord(e0, st));
    // per-vertex filter data
    gsword::QFilter qf[GSWORD_MAX_QV];
    std::memset(qf, 0, sizeof(qf));
    bool adj[GSWORD_MAX_QV][GSWORD_MAX_QV] = {};
    for (int u = 0; u < nq; ++u)
        for (int32_t i = q_row_ptr[u]; i < q_row_ptr[u + 1]; ++i) adj[u][q_col[i]] = true;
    for (int u = 0; u < nq; ++u) {
        qf[u].label = q_labels[u];
        for (int w = 0; w < nq; ++w) {
            if (!adj[u][w]) continue;
            qf[u].deg += 1;
            int k = 0;
            while (k < qf[u].npairs && qf[u].plabel[k] != q_labels[w]) ++k;
            if (k == qf[u].npairs) {
                qf[u].plabel[k] = q_labels[w];
                qf[u].pcount[k] = 0;
                qf[u].npairs += 1;
            }
            qf[u].pcount[k] += 1;
        }
    }
    // 1st CSR: the directed query edges in (a, b) order (the plan's eidx)
    int eid[GSWORD_MAX_QV][GSWORD_MAX_QV];
    int ne = 0;
    for (int a = 0; a < nq; ++a)
        for (int b = 0; b < nq; ++b) eid[a][b] = adj[a][b] ? ne++ : -1;
    ctx->cwords = (uint32_t)((n + 31) / 32) + 1;
    const size_t bits_words = (size_t)nq * ctx->cwords;
    gsword::QFilter* d_qf = nullptr;
    uint32_t* d_tmp = nullptr;
    unsigned long long* d_tot = nullptr;
    // scratch scans: a rank row (cwords) or an edge's offsets (<= n + 1 entries)
    const size_t tmpw = gsword::scan_tmp_words(std::max<int64_t>((int64_t)ctx->cwords, n + 1));
    cudaError_t e;
    if ((e = cudaMalloc(&ctx->d_cbits, sizeof(uint32_t) * bits_words)) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_crank, sizeof(uint32_t) * bits_words)) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_cg_edge, sizeof(uint2) * (size_t)std::max(ne, 1))) != cudaSuccess ||
        (e = cudaMalloc(&d_qf, sizeof(qf))) != cudaSuccess ||
        (e = cudaMalloc(&d_tmp, sizeof(uint32_t) * tmpw)) != cudaSuccess ||
        (e = cudaMalloc(&d_tot, sizeof(unsigned long long) * (size_t)(ne + nq + 1))) != cudaSuccess) {
        cudaFree(d_qf);
        cudaFree(d_tmp);
        cudaFree(d_tot);
        return fail(GSWORD_ENOMEM, "load_query: candidate graph allocation: %s", cudaGetErrorString(e));
    }
    auto cleanup = [&]() {
        cudaFree(d_qf);
        cudaFree(d_tmp);
        cudaFree(d_tot);
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
    };
#define CG_TRY(expr)                     \
    do {                                 \
        cudaError_t _e = (expr);         \
        if (_e != cudaSuccess) {         \
            cleanup();                   \
            return cuda_fail(_e, #expr); \
        }                                \
    } while (0)
    ctx->q_filter = ctx->opt_filter;
    gsword::DeviceGraph g = device_graph(ctx);
    g.cbits = ctx->d_cbits;
    g.crank = ctx->d_crank;
    g.cwords = ctx->cwords;
    CG_TRY(cudaMemcpyAsync(d_qf, qf, sizeof(qf), cudaMemcpyHostToDevice, st));
    CG_TRY(cudaMemsetAsync(ctx->d_cbits, 0, sizeof(uint32_t) * bits_words, st));
    CG_TRY(gsword::launch_filter(g, d_qf, nq, ctx->q_filter, ctx->d_cbits, ctx->d_vlabel, st));
    // 2nd CSR: rank directory per query vertex; d_tot[ne + u] = |C(u)|
    for (int u = 0; u < nq; ++u) {
        uint32_t* row = ctx->d_crank + (size_t)u * ctx->cwords;
        CG_TRY(gsword::launch_rank_words(ctx->d_cbits, ctx->cwords, u, ctx->d_crank, st));
        CG_TRY(gsword::launch_scan(row, (int64_t)ctx->cwords, nullptr, d_tmp, d_tot + ne + u, st));
    }
    unsigned long long csz[GSWORD_MAX_QV];
    CG_TRY(cudaMemcpyAsync(csz, d_tot + ne, sizeof(unsigned long long) * (size_t)nq, cudaMemcpyDeviceToHost, st));
    CG_TRY(cudaStreamSynchronize(st));
    // 3rd CSR offsets: edge a -> b gets |C(a)| + 1 entries at base[e]
    std::vector<uint2> edges((size_t)std::max(ne, 1));
    uint64_t off_total = 0;
    for (int a = 0; a < nq; ++a)
        for (int b = 0; b < nq; ++b)
            if (eid[a][b] >= 0) {
                edges[(size_t)eid[a][b]] = make_uint2((uint32_t)off_total, (uint32_t)a);
                off_total += csz[a] + 1;
            }
    if (off_total >= (1ull << 32)) {
        cleanup();
        return fail(GSWORD_ELIMIT, "load_query: candidate graph has %llu offsets (>= 2^32)",
                    (unsigned long long)off_total);
    }
    if ((e = cudaMalloc(&ctx->d_cg_off, sizeof(uint32_t) * (size_t)std::max<uint64_t>(off_total, 1))) != cudaSuccess) {
        cleanup();
        return fail(GSWORD_ENOMEM, "load_query: candidate graph offsets: %s", cudaGetErrorString(e));
    }
    CG_TRY(cudaMemcpyAsync(ctx->d_cg_edge, edges.data(), sizeof(uint2) * edges.size(), cudaMemcpyHostToDevice, st));
    CG_TRY(cudaMemsetAsync(ctx->d_cg_off, 0, sizeof(uint32_t) * (size_t)std::max<uint64_t>(off_total, 1), st));
    CG_TRY(cudaMemsetAsync(d_tot, 0, sizeof(unsigned long long), st));
    for (int a = 0; a < nq; ++a)
        for (int b = 0; b < nq; ++b) {
            const int ed = eid[a][b];
            if (ed < 0) continue;
            uint32_t* off = ctx->d_cg_off + edges[(size_t)ed].x;
            CG_TRY(gsword::launch_cg_count(g, a, b, q_labels[b], off, st));
            // offsets chained across the edges: absolute positions in the list array
            CG_TRY(gsword::launch_scan(off, (int64_t)csz[a] + 1, d_tot + ed, d_tmp, d_tot + ed + 1, st));
        }
    unsigned long long entries = 0;
    CG_TRY(cudaMemcpyAsync(&entries, d_tot + ne, sizeof(entries), cudaMemcpyDeviceToHost, st));
    CG_TRY(cudaStreamSynchronize(st));
    const uint64_t n0 = csz[order[0]];
    if (entries >= (1ull << 32)) {
        cleanup();
        return fail(GSWORD_ELIMIT, "load_query: candidate graph has %llu entries (>= 2^32)",
                    (unsigned long long)entries);
    }
    if ((e = cudaMalloc(&ctx->d_clist, sizeof(int32_t) * (size_t)std::max<uint64_t>(entries, 1))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_cand0, sizeof(int32_t) * (size_t)std::max<uint64_t>(n0, 1))) != cudaSuccess) {
        cleanup();
        return fail(GSWORD_ENOMEM, "load_query: candidate graph (%llu entries): %s", (unsigned long long)entries,
                    cudaGetErrorString(e));
    }
    CG_TRY(gsword::launch_cand_fill(g, order[0], ctx->d_cand0, st));
    for (int a = 0; a < nq; ++a)
        for (int b = 0; b < nq; ++b) {
            const int ed = eid[a][b];
            if (ed < 0) continue;
            CG_TRY(gsword::launch_cg_fill(g, a, b, q_labels[b], ctx->d_cg_off + edges[(size_t)ed].x, ctx->d_clist, st));
        }
    CG_TRY(cudaEventRecord(e1, st));
    CG_TRY(cudaStreamSynchronize(st));
    float ms = 0.f;
    CG_TRY(cudaEventElapsedTime(&ms, e0, e1));
#undef CG_TRY
    cleanup();
    for (int u = 0; u < nq; ++u) ctx->cand_count[u] = csz[u];
    ctx->cg_entries = entries;
    ctx->cg_seconds = ms * 1e-3;
    ctx->cg_bytes = sizeof(uint32_t) * (2 * bits_words + off_total + entries + n0) + sizeof(uint2) * (size_t)ne;
    p->seed_lo = 0;
    p->seed_len = (uint32_t)n0;
    p->seed_identity = 0;
    return GSWORD_OK;
}

}  // namespace

extern "C" {

int gsword_version(void) { return 200; }  // 2.00: A26 sectors in records, count_sectors(model, touched), EFAULT, cg_bytes

const char* gsword_last_error(void) { return g_last_error.c_str(); }

int gsword_create(int cuda_device, gsword_ctx** out) {
    if (!out) return fail(GSWORD_EINVAL, "create: out NULL");
    *out = nullptr;
    int count = 0;
    cudaError_t e = cudaGetDeviceCount(&count);
    if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
    if (cuda_device < 0 || cuda_device >= count) return fail(GSWORD_ECUDA, "create: no CUDA device %d", cuda_device);
    CUDA_TRY(cudaSetDevice(cuda_device));
    gsword_ctx* ctx = new (std::nothrow) gsword_ctx();
    if (!ctx) return fail(GSWORD_ENOMEM, "create: host allocation failed");
    ctx->device = cuda_device;
    cudaDeviceProp prop;
    e = cudaGetDeviceProperties(&prop, cuda_device);
    if (e == cudaSuccess) ctx->num_sms = prop.multiProcessorCount;
    if ((e = cudaStreamCreateWithFlags(&ctx->own_stream, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaEventCreate(&ctx->ev0)) != cudaSuccess || (e = cudaEventCreate(&ctx->ev1)) != cudaSuccess ||
        (e = cudaEventCreate(&ctx->evk0)) != cudaSuccess || (e = cudaEventCreate(&ctx->evk1)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&ctx->ev_switch, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_queue, sizeof(unsigned long long))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_out4, 4 * sizeof(double))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_sectors, 2 * sizeof(double))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_phase, 8 * sizeof(unsigned long long))) != cudaSuccess) {
        gsword_destroy(ctx);
        return cuda_fail(e, "create");
    }
    ctx->stream = ctx->own_stream;
    *out = ctx;
    return GSWORD_OK;
}

int gsword_destroy(gsword_ctx* ctx) {
    if (!ctx) return GSWORD_OK;
    cudaSetDevice(ctx->device);
    if (ctx->stream) cudaStreamSynchronize(ctx->stream);
    ctx->free_graph();
    if (ctx->d_queue) cudaFree(ctx->d_queue);
    if (ctx->d_partials) cudaFree(ctx->d_partials);
    if (ctx->d_out4) cudaFree(ctx->d_out4);
    if (ctx->d_sectors) cudaFree(ctx->d_sectors);
    if (ctx->d_phase) cudaFree(ctx->d_phase);
    if (ctx->ev0) cudaEventDestroy(ctx->ev0);
    if (ctx->ev1) cudaEventDestroy(ctx->ev1);
    if (ctx->evk0) cudaEventDestroy(ctx->evk0);
    if (ctx->evk1) cudaEventDestroy(ctx->evk1);
    if (ctx->ev_switch) cudaEventDestroy(ctx->ev_switch);
    if (ctx->own_stream) cudaStreamDestroy(ctx->own_stream);
    delete ctx;
    return GSWORD_OK;
}

int gsword_set_stream(gsword_ctx* ctx, void* cuda_stream) {
    if (!ctx) return fail(GSWORD_EINVAL, "set_stream: NULL context");
    cudaStream_t next = cuda_stream ? (cudaStream_t)cuda_stream : ctx->own_stream;
    if (next != ctx->stream) {
        // every launch reuses the context's queue, partials and output buffers: work issued on
        // the new stream must start after everything already issued on the old one
        CUDA_TRY(cudaSetDevice(ctx->device));
        CUDA_TRY(cudaEventRecord(ctx->ev_switch, ctx->stream));
        CUDA_TRY(cudaStreamWaitEvent(next, ctx->ev_switch, 0));
        ctx->stream = next;
    }
    return apply_l2_window(ctx);
}

int gsword_set_option(gsword_ctx* ctx, int option, int64_t value) {
    if (!ctx) return fail(GSWORD_EINVAL, "set_option: NULL context");
    switch (option) {
        case GSWORD_OPT_BLOCKS_PER_SM:
            if (value < 0 || value > 32) return fail(GSWORD_EINVAL, "blocks_per_sm out of range");
            ctx->opt_blocks_per_sm = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_THREADS:
            if (value < 64 || value > 256 || value % 32) return fail(GSWORD_EINVAL, "threads must be 64..256, /32");
            ctx->opt_threads = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_CHUNK:
            if (value < 1 || value > (1 << 20)) return fail(GSWORD_EINVAL, "chunk out of range");
            ctx->opt_chunk = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_L2_PERSIST:
            if (value < 0 || value > 2) return fail(GSWORD_EINVAL, "l2 window mode must be 0, 1 or 2");
            ctx->opt_l2 = (int)value;
            return apply_l2_window(ctx);
        case GSWORD_OPT_BLOOM:
            ctx->opt_bloom = value ? 1 : 0;
            return GSWORD_OK;
        case GSWORD_OPT_SCHEDULE:
            if (value < 0 || value > 2) return fail(GSWORD_EINVAL, "schedule must be 0, 1 or 2");
            ctx->opt_sched = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_REFILL_MIN:
            if (value < 1 || value > 32) return fail(GSWORD_EINVAL, "refill_min must be 1..32");
            ctx->opt_refill_min = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_AUTOTUNE:
            ctx->opt_autotune = value ? 1 : 0;
            if (!value) ctx->tuned_refill[0] = ctx->tuned_refill[1] = 0;
            return GSWORD_OK;
        case GSWORD_OPT_FILTER:
            if (value < 0 || value > 2) return fail(GSWORD_EINVAL, "filter must be 0 (label), 1 (LDF) or 2 (NLF)");
            ctx->opt_filter = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_BLOOM_BITS:
            if (value < 2 || value > 64) return fail(GSWORD_EINVAL, "bloom bits per edge must be 2..64");
            ctx->opt_bloom_bits = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_EDGE_SET:
            ctx->opt_eset = value ? 1 : 0;
            return GSWORD_OK;
        case GSWORD_OPT_STREAMING:
            ctx->opt_streaming = value ? 1 : 0;
            return GSWORD_OK;
        case GSWORD_OPT_OCCUPANCY:
            if (value < -1 || value > 2) return fail(GSWORD_EINVAL, "occupancy variant must be -1..2");
            ctx->opt_occ = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_VARIANT:
            if (value & ~(int64_t)(GSWORD_VARIANT_WJ_PARENT_FIRST | GSWORD_VARIANT_ALLEY_DUPCHECK_POST))
                return fail(GSWORD_EINVAL, "unknown variant bits 0x%llx", (unsigned long long)value);
            ctx->opt_variant = (int)value;
            return GSWORD_OK;
        case GSWORD_OPT_FAULT_QUEUE:
            if (value < 0) return fail(GSWORD_EINVAL, "fault queue start must be >= 0");
            ctx->opt_fault_queue = (uint64_t)value;
            return GSWORD_OK;
        case GSWORD_OPT_TRAWL_WARP:
            ctx->opt_trawl_warp = value ? 1 : 0;
            return GSWORD_OK;
        case GSWORD_OPT_COOP_THRESHOLD:
            if (value < 0 || value > 128) return fail(GSWORD_EINVAL, "coop threshold must be 0..128");
            ctx->opt_coop = (int)value;
            return GSWORD_OK;
        default:
            return fail(GSWORD_EINVAL, "unknown option %d", option);
    }
}

int gsword_check_graph(int64_t n_vertices, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                       int32_t n_labels) {
    return check_graph_impl(n_vertices, row_ptr, col, labels, n_labels);
}

int gsword_plan_query(int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int32_t n_labels, gsword_plan_info* out) {
    return plan_query_impl(n_qv, q_row_ptr, q_col, q_labels, order, n_labels, nullptr, out);
}

int gsword_quicksi_order(int64_t n_vertices, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                         int32_t n_labels, int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col,
                         const int32_t* q_labels, int32_t* order_out) {
    if (!row_ptr || !q_row_ptr || !q_labels || !order_out || n_vertices < 0 || n_labels < 1)
        return fail(GSWORD_EINVAL, "quicksi_order: bad argument");
    std::vector<int64_t> off((size_t)n_labels + 1, 0);
    for (int64_t v = 0; v < n_vertices; ++v) {
        const int32_t l = labels ? labels[v] : 0;
        if (l < 0 || l >= n_labels) return fail(GSWORD_EINVAL, "quicksi_order: label out of range");
        off[(size_t)l + 1] += 1;
    }
    for (int32_t l = 0; l < n_labels; ++l) off[(size_t)l + 1] += off[(size_t)l];
    std::vector<uint64_t> pf;
    label_pair_freq(n_vertices, row_ptr, col, labels, n_labels, &pf);
    return quicksi_order_impl(n_qv, q_row_ptr, q_col, q_labels, n_labels, off, pf, order_out);
}

int gsword_select_order(gsword_ctx* ctx, int strategy, gsword_method m, int32_t n_qv, const int32_t* q_row_ptr,
                        const int32_t* q_col, const int32_t* q_labels, uint64_t pilot_samples, uint64_t seed,
                        int32_t* order_out, double* score_out) {
    if (!ctx || !order_out) return fail(GSWORD_EINVAL, "select_order: NULL argument");
    if (!ctx->graph_loaded) return fail(GSWORD_ENOGRAPH, "select_order: no graph loaded");
    if (strategy != GSWORD_ORDER_QUICKSI && strategy != GSWORD_ORDER_TRIAL)
        return fail(GSWORD_EINVAL, "select_order: unknown strategy %d", strategy);
    int32_t qo[GSWORD_MAX_QV];
    int rc = quicksi_order_impl(n_qv, q_row_ptr, q_col, q_labels, ctx->n_labels, ctx->label_off, ctx->pair_freq, qo);
    if (rc) return rc;
    if (strategy == GSWORD_ORDER_QUICKSI) {
        std::memcpy(order_out, qo, sizeof(int32_t) * (size_t)n_qv);
        if (score_out) *score_out = 0.0;
        return gsword_load_query(ctx, n_qv, q_row_ptr, q_col, q_labels, order_out);
    }
    if (pilot_samples < 2) return fail(GSWORD_EINVAL, "select_order: pilot_samples must be >= 2");
    // candidate orders: QuickSI, then every directed query edge as the first two positions,
    // completed with the same infrequent-edge rule; each scored by a GPU pilot estimate
    // (G-CARE's trial): the variance of one sample, smallest wins (ties: first).
    bool adj[GSWORD_MAX_QV][GSWORD_MAX_QV] = {};
    for (int u = 0; u < n_qv; ++u)
        for (int32_t i = q_row_ptr[u]; i < q_row_ptr[u + 1]; ++i) adj[u][q_col[i]] = adj[q_col[i]][u] = true;
    std::vector<std::vector<int32_t>> cands;
    cands.emplace_back(qo, qo + n_qv);
    for (int a = 0; a < n_qv; ++a)
        for (int b = 0; b < n_qv; ++b) {
            if (!adj[a][b]) continue;
            std::vector<int32_t> o = {a, b};
            bool used[GSWORD_MAX_QV] = {};
            used[a] = used[b] = true;
            while ((int)o.size() < n_qv) {
                // the QuickSI order's relative preference: earliest position in qo among frontier vertices
                int best = -1;
                for (int t = 0; t < n_qv && best < 0; ++t) {
                    const int c = qo[t];
                    if (used[c]) continue;
                    for (int x : o)
                        if (adj[x][c]) { best = c; break; }
                }
                if (best < 0) break;
                o.push_back(best);
                used[best] = true;
            }
            if ((int)o.size() == n_qv) {
                bool dup = false;
                for (auto& c : cands) dup |= (c == o);
                if (!dup) cands.push_back(o);
            }
        }
    double best_score = 0.0;
    int best = -1;
    const int autotune = ctx->opt_autotune;
    ctx->opt_autotune = 0;  // pilots only matter for the order finally loaded
    for (size_t c = 0; c < cands.size(); ++c) {
        rc = gsword_load_query(ctx, n_qv, q_row_ptr, q_col, q_labels, cands[c].data());
        if (rc) {
            ctx->opt_autotune = autotune;
            return rc;
        }
        gsword_result r;
        rc = gsword_estimate_range(ctx, m, 0, pilot_samples, seed, &r);
        if (rc) {
            ctx->opt_autotune = autotune;
            return rc;
        }
        const double score = std::isnan(r.variance) ? 0.0 : r.variance * (double)r.n_samples;
        if (best < 0 || score < best_score) {
            best = (int)c;
            best_score = score;
        }
    }
    ctx->opt_autotune = autotune;
    std::memcpy(order_out, cands[(size_t)best].data(), sizeof(int32_t) * (size_t)n_qv);
    if (score_out) *score_out = best_score;
    return gsword_load_query(ctx, n_qv, q_row_ptr, q_col, q_labels, order_out);
}

int gsword_load_graph(gsword_ctx* ctx, int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t n_labels) {
    if (!ctx) return fail(GSWORD_EINVAL, "load_graph: NULL context");
    int rc = check_graph_impl(n, row_ptr, col, labels, n_labels);
    if (rc) return rc;
    CUDA_TRY(cudaSetDevice(ctx->device));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    ctx->free_graph();
    const int64_t nnz = row_ptr[n];
    const int32_t L = n_labels;
    // label buckets: vertices sorted by (label, id)
    std::vector<int64_t> off((size_t)L + 1, 0);
    for (int64_t v = 0; v < n; ++v) off[(size_t)(labels ? labels[v] : 0) + 1] += 1;
    for (int32_t l = 0; l < L; ++l) off[(size_t)l + 1] += off[(size_t)l];
    // adjacency sorted by (label, id) and segment offsets seg[v*L + l]
    std::vector<int32_t> col2;
    std::vector<uint32_t> seg((size_t)n * (size_t)L + 1);
    const int32_t* col_up = col;
    if (L == 1) {
        for (int64_t v = 0; v <= n; ++v) seg[(size_t)v] = (uint32_t)row_ptr[v];
    } else {
        col2.resize((size_t)nnz);
        parallel_for(n, [&](int64_t lo, int64_t hi) {
            std::vector<uint32_t> cnt((size_t)L + 1);
            for (int64_t v = lo; v < hi; ++v) {
                std::fill(cnt.begin(), cnt.end(), 0u);
                for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) cnt[(size_t)labels[col[i]] + 1] += 1;
                for (int32_t l = 0; l < L; ++l) cnt[(size_t)l + 1] += cnt[(size_t)l];
                for (int32_t l = 0; l < L; ++l) seg[(size_t)v * L + l] = (uint32_t)(row_ptr[v] + cnt[(size_t)l]);
                for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) {  // stable: ascending id per label
                    const int32_t w = col[i];
                    col2[(size_t)(row_ptr[v] + cnt[(size_t)labels[w]]++)] = w;
                }
            }
        });
        seg[(size_t)n * L] = (uint32_t)nnz;
        col_up = col2.data();
    }
    std::vector<int32_t> bucket;
    if (L > 1) {
        bucket.resize((size_t)n);
        std::vector<int64_t> pos(off.begin(), off.end() - 1);
        for (int64_t v = 0; v < n; ++v) bucket[(size_t)pos[(size_t)labels[v]]++] = (int32_t)v;
    }
    // blocked Bloom filter over the edge set: ~16 bits per undirected edge, power-of-two words
    uint64_t words = 1;
    {
        const uint64_t want = std::max<uint64_t>(1, (uint64_t)(nnz / 2) * (uint64_t)ctx->opt_bloom_bits / 64);
        while (words < want) words <<= 1;
    }
    cudaError_t e;
    const size_t hot_bytes = words * sizeof(unsigned long long) + sizeof(uint32_t) * seg.size();
    if ((e = cudaMalloc(&ctx->d_col, sizeof(int32_t) * (size_t)std::max<int64_t>(nnz, 1))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_hot, hot_bytes)) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_bucket, sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1))) != cudaSuccess) {
        ctx->free_graph();
        return fail(e == cudaErrorMemoryAllocation ? GSWORD_ENOMEM : GSWORD_ECUDA, "load_graph: cudaMalloc: %s",
                    cudaGetErrorString(e));
    }
    ctx->hot_bytes = hot_bytes;
    ctx->d_bloom = reinterpret_cast<unsigned long long*>(ctx->d_hot);
    ctx->d_seg = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ctx->d_hot) + words * sizeof(unsigned long long));
    if ((e = cudaMalloc(&ctx->d_vlabel, sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1))) != cudaSuccess) {
        ctx->free_graph();
        return fail(GSWORD_ENOMEM, "load_graph: cudaMalloc(labels): %s", cudaGetErrorString(e));
    }
    // every upload is ordered on the context stream (the builds and samplers run there too);
    // the host staging vectors live until the synchronisation below
    if (nnz > 0)
        CUDA_TRY(cudaMemcpyAsync(ctx->d_col, col_up, sizeof(int32_t) * (size_t)nnz, cudaMemcpyHostToDevice, ctx->stream));
    if (labels && n > 0)
        CUDA_TRY(cudaMemcpyAsync(ctx->d_vlabel, labels, sizeof(int32_t) * (size_t)n, cudaMemcpyHostToDevice, ctx->stream));
    else if (n > 0)
        CUDA_TRY(cudaMemsetAsync(ctx->d_vlabel, 0, sizeof(int32_t) * (size_t)n, ctx->stream));
    CUDA_TRY(cudaMemcpyAsync(ctx->d_seg, seg.data(), sizeof(uint32_t) * seg.size(), cudaMemcpyHostToDevice, ctx->stream));
    if (L > 1) {
        if (n > 0)
            CUDA_TRY(cudaMemcpyAsync(ctx->d_bucket, bucket.data(), sizeof(int32_t) * (size_t)n, cudaMemcpyHostToDevice,
                                     ctx->stream));
    } else if (n > 0) {
        CUDA_TRY(gsword::launch_build_bucket_identity(ctx->d_bucket, n, ctx->stream));
    }
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    // Bloom filter (allocated above) and exact edge set, both built on the device
    {
        // exact edge set: 4-key buckets, load factor <= 1/2
        const uint64_t want_b = std::max<uint64_t>(1, ((uint64_t)(nnz / 2) + 1) / 2);
        uint64_t buckets = 1;
        while (buckets < want_b) buckets <<= 1;
        int64_t* d_rp = nullptr;
        if ((e = cudaMalloc(&ctx->d_eset, buckets * 4 * sizeof(unsigned long long))) != cudaSuccess ||
            (e = cudaMalloc(&d_rp, sizeof(int64_t) * (size_t)(n + 1))) != cudaSuccess) {
            if (d_rp) cudaFree(d_rp);
            ctx->free_graph();
            return fail(GSWORD_ENOMEM, "load_graph: cudaMalloc(edge index): %s", cudaGetErrorString(e));
        }
        ctx->bloom_words = words;
        ctx->eset_buckets = buckets;
        CUDA_TRY(cudaMemsetAsync(ctx->d_bloom, 0, words * sizeof(unsigned long long), ctx->stream));
        CUDA_TRY(cudaMemsetAsync(ctx->d_eset, 0xFF, buckets * 4 * sizeof(unsigned long long), ctx->stream));
        CUDA_TRY(cudaMemcpyAsync(d_rp, row_ptr, sizeof(int64_t) * (size_t)(n + 1), cudaMemcpyHostToDevice, ctx->stream));
        CUDA_TRY(gsword::launch_build_bloom(d_rp, ctx->d_col, n, ctx->d_bloom, words - 1, ctx->stream));
        CUDA_TRY(gsword::launch_build_eset(d_rp, ctx->d_col, n, ctx->d_eset, buckets - 1, ctx->stream));
        CUDA_TRY(cudaStreamSynchronize(ctx->stream));
        cudaFree(d_rp);
    }
    ctx->n = n;
    ctx->nnz = nnz;
    ctx->n_labels = L;
    ctx->label_off = off;
    label_pair_freq(n, row_ptr, col, labels, L, &ctx->pair_freq);
    ctx->graph_loaded = true;
    ctx->query_loaded = false;
    return apply_l2_window(ctx);
}

int gsword_load_graph_device(gsword_ctx* ctx, int64_t n, const int64_t* d_row_ptr, const int32_t* d_col,
                             const int32_t* d_labels, int32_t n_labels) {
    if (!ctx) return fail(GSWORD_EINVAL, "load_graph_device: NULL context");
    if (n < 0 || !d_row_ptr || (n > 0 && !d_col)) return fail(GSWORD_EINVAL, "load_graph_device: bad argument");
    if (n_labels < 1 || (!d_labels && n_labels != 1))
        return fail(GSWORD_EINVAL, "load_graph_device: labels NULL requires n_labels == 1");
    if (n >= (int64_t)1 << 31 || n * (int64_t)n_labels >= ((int64_t)1 << 31))
        return fail(GSWORD_ELIMIT, "load_graph_device: |V| or |V| * n_labels >= 2^31");
    CUDA_TRY(cudaSetDevice(ctx->device));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    ctx->free_graph();
    cudaStream_t st = ctx->stream;
    int64_t h_rp[2] = {0, 0};
    CUDA_TRY(cudaMemcpyAsync(&h_rp[0], d_row_ptr, sizeof(int64_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaMemcpyAsync(&h_rp[1], d_row_ptr + n, sizeof(int64_t), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    const int64_t nnz = h_rp[1];
    if (h_rp[0] != 0) return fail(GSWORD_EGRAPH, "load_graph_device: row_ptr[0] != 0");
    if (nnz < 0 || nnz >= ((int64_t)1 << 31) - 1) return fail(GSWORD_ELIMIT, "load_graph_device: 2|E| >= 2^31");
    const int32_t L = n_labels;
    int* d_bad = nullptr;
    unsigned long long* d_hist = nullptr;
    CUDA_TRY(cudaMalloc(&d_bad, sizeof(int)));
    CUDA_TRY(cudaMalloc(&d_hist, sizeof(unsigned long long) * ((size_t)L + 2)));
    auto cleanup = [&]() {
        cudaFree(d_bad);
        cudaFree(d_hist);
    };
    int bad = 0;
    std::vector<unsigned long long> hist((size_t)L, 0);
    cudaError_t e = cudaMemsetAsync(d_bad, 0, sizeof(int), st);
    if (e == cudaSuccess) e = gsword::launch_dev_validate(d_row_ptr, d_col, d_labels, n, L, d_bad, st);
    if (e == cudaSuccess) e = cudaMemsetAsync(d_hist, 0, sizeof(unsigned long long) * (size_t)L, st);
    if (e == cudaSuccess) e = gsword::launch_label_hist(d_labels, n, d_hist, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(&bad, d_bad, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaMemcpyAsync(hist.data(), d_hist, sizeof(unsigned long long) * (size_t)L,
                                              cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
        cleanup();
        return cuda_fail(e, "load_graph_device: validation");
    }
    if (bad) {
        cleanup();
        return fail(bad & 1 ? GSWORD_EINVAL : GSWORD_EGRAPH,
                    "load_graph_device: CSR not canonical (flags %d: 1 label range, 2 row_ptr, 4 id range/self "
                    "loop, 8 row not ascending by (label, id), 16 asymmetric)", bad);
    }
    std::vector<int64_t> off((size_t)L + 1, 0);
    for (int32_t l = 0; l < L; ++l) off[(size_t)l + 1] = off[(size_t)l] + (int64_t)hist[(size_t)l];
    // hot buffer (Bloom words + seg), buckets, edge set; col and labels are borrowed
    uint64_t words = 1;
    {
        const uint64_t want = std::max<uint64_t>(1, (uint64_t)(nnz / 2) * (uint64_t)ctx->opt_bloom_bits / 64);
        while (words < want) words <<= 1;
    }
    const size_t seg_n = (size_t)n * (size_t)L + 1;
    const size_t hot_bytes = words * sizeof(unsigned long long) + sizeof(uint32_t) * seg_n;
    uint64_t buckets = 1;
    {
        const uint64_t want_b = std::max<uint64_t>(1, ((uint64_t)(nnz / 2) + 1) / 2);
        while (buckets < want_b) buckets <<= 1;
    }
    ctx->own_col = false;
    ctx->d_col = const_cast<int32_t*>(d_col);
    if ((e = cudaMalloc(&ctx->d_hot, hot_bytes)) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_bucket, sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1))) != cudaSuccess ||
        (e = cudaMalloc(&ctx->d_eset, buckets * 4 * sizeof(unsigned long long))) != cudaSuccess) {
        cleanup();
        ctx->free_graph();
        return fail(GSWORD_ENOMEM, "load_graph_device: cudaMalloc: %s", cudaGetErrorString(e));
    }
    if (d_labels) {
        ctx->own_vlabel = false;
        ctx->d_vlabel = const_cast<int32_t*>(d_labels);
    } else {
        if ((e = cudaMalloc(&ctx->d_vlabel, sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1))) != cudaSuccess) {
            cleanup();
            ctx->free_graph();
            return fail(GSWORD_ENOMEM, "load_graph_device: cudaMalloc(labels)");
        }
        CUDA_TRY(cudaMemsetAsync(ctx->d_vlabel, 0, sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1), st));
    }
    ctx->hot_bytes = hot_bytes;
    ctx->d_bloom = reinterpret_cast<unsigned long long*>(ctx->d_hot);
    ctx->d_seg = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ctx->d_hot) + words * sizeof(unsigned long long));
    ctx->bloom_words = words;
    ctx->eset_buckets = buckets;
    CUDA_TRY(gsword::launch_dev_seg(d_row_ptr, d_col, d_labels, n, L, ctx->d_seg, st));
    if (L == 1) {
        if (n > 0) CUDA_TRY(gsword::launch_build_bucket_identity(ctx->d_bucket, n, st));
    } else {
        uint32_t* d_cnt = nullptr;
        uint32_t* d_tmp = nullptr;
        unsigned long long* d_b = nullptr;
        const size_t tmpw = gsword::scan_tmp_words(n + 1);
        if ((e = cudaMalloc(&d_cnt, sizeof(uint32_t) * (size_t)(n + 1))) != cudaSuccess ||
            (e = cudaMalloc(&d_tmp, sizeof(uint32_t) * tmpw)) != cudaSuccess ||
            (e = cudaMalloc(&d_b, sizeof(unsigned long long) * 2 * (size_t)L)) != cudaSuccess) {
            cudaFree(d_cnt);
            cudaFree(d_tmp);
            cleanup();
            ctx->free_graph();
            return fail(GSWORD_ENOMEM, "load_graph_device: bucket scratch");
        }
        std::vector<unsigned long long> bases((size_t)L);
        for (int32_t l = 0; l < L; ++l) bases[(size_t)l] = (unsigned long long)off[(size_t)l];
        CUDA_TRY(cudaMemcpyAsync(d_b, bases.data(), sizeof(unsigned long long) * (size_t)L, cudaMemcpyHostToDevice, st));
        for (int32_t l = 0; l < L; ++l)
            CUDA_TRY(gsword::launch_label_bucket(d_labels, n, l, d_cnt, d_b + l, d_tmp, d_b + L + l, ctx->d_bucket, st));
        CUDA_TRY(cudaStreamSynchronize(st));
        cudaFree(d_cnt);
        cudaFree(d_tmp);
        cudaFree(d_b);
    }
    // label-pair frequencies (QuickSI order) for up to 64 labels
    ctx->pair_freq.clear();
    if (L <= 64) {
        unsigned long long* d_pf = nullptr;
        CUDA_TRY(cudaMalloc(&d_pf, sizeof(unsigned long long) * (size_t)L * (size_t)L));
        CUDA_TRY(cudaMemsetAsync(d_pf, 0, sizeof(unsigned long long) * (size_t)L * (size_t)L, st));
        CUDA_TRY(gsword::launch_pair_hist(d_row_ptr, d_col, d_labels, n, L, d_pf, st));
        std::vector<unsigned long long> pf((size_t)L * (size_t)L);
        CUDA_TRY(cudaMemcpyAsync(pf.data(), d_pf, sizeof(unsigned long long) * pf.size(), cudaMemcpyDeviceToHost, st));
        CUDA_TRY(cudaStreamSynchronize(st));
        cudaFree(d_pf);
        ctx->pair_freq.assign(pf.begin(), pf.end());
    }
    CUDA_TRY(cudaMemsetAsync(ctx->d_bloom, 0, words * sizeof(unsigned long long), st));
    CUDA_TRY(cudaMemsetAsync(ctx->d_eset, 0xFF, buckets * 4 * sizeof(unsigned long long), st));
    CUDA_TRY(gsword::launch_build_bloom(d_row_ptr, d_col, n, ctx->d_bloom, words - 1, st));
    CUDA_TRY(gsword::launch_build_eset(d_row_ptr, d_col, n, ctx->d_eset, buckets - 1, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    cleanup();
    ctx->n = n;
    ctx->nnz = nnz;
    ctx->n_labels = L;
    ctx->label_off = off;
    ctx->graph_loaded = true;
    ctx->query_loaded = false;
    return apply_l2_window(ctx);
}

int gsword_load_query(gsword_ctx* ctx, int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col,
                      const int32_t* q_labels, const int32_t* order) {
    if (!ctx) return fail(GSWORD_EINVAL, "load_query: NULL context");
    if (!ctx->graph_loaded) return fail(GSWORD_ENOGRAPH, "load_query: no graph loaded");
    Plan p;
    int rc = plan_query_impl(n_qv, q_row_ptr, q_col, q_labels, order, ctx->n_labels, &p, nullptr);
    if (rc) return rc;
    CUDA_TRY(cudaSetDevice(ctx->device));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    ctx->free_query();
    const int32_t l0 = p.step[0].label;
    p.seed_lo = (uint32_t)ctx->label_off[(size_t)l0];
    p.seed_len = (uint32_t)(ctx->label_off[(size_t)l0 + 1] - ctx->label_off[(size_t)l0]);
    p.seed_identity = (ctx->n_labels == 1) ? 1 : 0;
    for (int u = 0; u < n_qv; ++u)
        ctx->cand_count[u] = (uint64_t)(ctx->label_off[(size_t)q_labels[u] + 1] - ctx->label_off[(size_t)q_labels[u]]);
    if (ctx->opt_filter > 0) {
        rc = build_candidate_graph(ctx, n_qv, q_row_ptr, q_col, q_labels, order, &p);
        if (rc) {
            ctx->free_query();
            return rc;
        }
    }
    ctx->plan = p;
    ctx->query_loaded = true;
    ctx->tuned_refill[0] = ctx->tuned_refill[1] = 0;
    ctx->tuned_occ[0] = ctx->tuned_occ[1] = 0;
    std::string tkey;
    if (ctx->opt_autotune && ctx->opt_sched == 0) {
        // the query exactly as given plus every option that changes the kernels' schedule
        const int opts[] = {n_qv, ctx->opt_blocks_per_sm, ctx->opt_threads, ctx->opt_chunk, ctx->opt_l2,
                            ctx->opt_coop, ctx->opt_bloom, ctx->opt_eset, ctx->opt_filter, ctx->opt_streaming,
                            ctx->opt_variant, ctx->opt_occ};
        tkey.append(reinterpret_cast<const char*>(opts), sizeof(opts));
        tkey.append(reinterpret_cast<const char*>(q_row_ptr), sizeof(int32_t) * (size_t)(n_qv + 1));
        tkey.append(reinterpret_cast<const char*>(q_col), sizeof(int32_t) * (size_t)q_row_ptr[n_qv]);
        tkey.append(reinterpret_cast<const char*>(q_labels), sizeof(int32_t) * (size_t)n_qv);
        tkey.append(reinterpret_cast<const char*>(order), sizeof(int32_t) * (size_t)n_qv);
        const auto it = ctx->tune_cache.find(tkey);
        if (it != ctx->tune_cache.end()) {
            for (int m = 0; m < 2; ++m) {
                ctx->tuned_refill[m] = it->second.refill[m];
                ctx->tuned_occ[m] = it->second.occ[m];
            }
        }
    }
    if (ctx->opt_autotune && ctx->opt_sched == 0 && ctx->tuned_refill[0] == 0) {
        // schedule autotune (no effect on any result).  Phase 1: refill thresholds
        // 16/8/24/32/28 (samples of long-lived walks favour depth-synchronous warps, short-lived
        // ones frequent refills).  Phase 2 (below): the estimate kernel compiled
        // for one CTA/SM less (more registers, fewer spills) and one more, against the default.
        // Every phase-1 candidate is timed over the same id range of `big` samples, preceded
        // by a warm-up over a range of its own (short or repeated pilots favour whichever
        // candidate profits from the tail or from a warm L2); each phase queues its runs back
        // to back on the context stream, timed by events, with one host synchronisation.
        static const int cand[5] = {16, 8, 24, 32, 28};  // 28: C1 dense Alley (profiles/r02_refill_sweep.jsonl)
        const uint64_t big = 8000000, warm = 1000000, range0 = 1ull << 40;
        int rc2 = GSWORD_OK;
        cudaError_t e = cudaSuccess;
        std::vector<cudaEvent_t> evs;
        auto event = [&](cudaEvent_t* out) {
            if (e == cudaSuccess) e = cudaEventCreate(out);
            if (e == cudaSuccess) evs.push_back(*out);
        };
        // times[m][c] for candidate c of method m; sets tuned_* before each run
        auto time_phase = [&](int ncand, auto&& apply, float (*times)[5]) {
            cudaEvent_t ev[2][5][2];
            for (int m = 0; m < 2 && rc2 == GSWORD_OK && e == cudaSuccess; ++m)
                for (int c = 0; c < ncand && rc2 == GSWORD_OK && e == cudaSuccess; ++c) {
                    apply(m, c);
                    rc2 = run(ctx, m, gsword::kModeEstimate, range0 + big + warm * (uint64_t)(4 * m + c), warm,
                              0x5EEDull, ctx->d_out4, nullptr, nullptr);
                    event(&ev[m][c][0]);
                    event(&ev[m][c][1]);
                    if (rc2 == GSWORD_OK && e == cudaSuccess) e = cudaEventRecord(ev[m][c][0], ctx->stream);
                    if (rc2 == GSWORD_OK && e == cudaSuccess)
                        rc2 = run(ctx, m, gsword::kModeEstimate, range0, big, 0x5EEDull, ctx->d_out4, nullptr, nullptr);
                    if (rc2 == GSWORD_OK && e == cudaSuccess) e = cudaEventRecord(ev[m][c][1], ctx->stream);
                }
            if (rc2 == GSWORD_OK && e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
            for (int m = 0; m < 2 && rc2 == GSWORD_OK && e == cudaSuccess; ++m)
                for (int c = 0; c < ncand && e == cudaSuccess; ++c)
                    e = cudaEventElapsedTime(&times[m][c], ev[m][c][0], ev[m][c][1]);
        };
        float t1[2][5] = {};
        time_phase(5, [&](int m, int c) { ctx->tuned_refill[m] = cand[c]; }, t1);
        float best[2] = {0.f, 0.f};
        for (int m = 0; m < 2; ++m) {
            int bc = 0;
            for (int c = 1; c < 5; ++c)
                if (t1[m][c] < t1[m][bc]) bc = c;
            ctx->tuned_refill[m] = cand[bc];
            best[m] = t1[m][bc];
        }
        // Phase 2, at the chosen threshold: occupancy variants 0, 1, 2 compared by their
        // steady-state cost t(2N) - t(N), so the per-launch tail (a third of an 8e6-sample
        // pilot on C1 dense Alley) cancels; N is sized from phase 1 to ~4 ms per method, and the
        // two runs cover disjoint id ranges (neither finds the other's samples in L2).
        for (int m = 0; m < 2; ++m) ctx->tuned_occ[m] = 0;
        if (ctx->opt_occ < 0) {
            uint64_t n2[2];
            for (int m = 0; m < 2; ++m) {
                const double rate = best[m] > 0.f ? (double)big / (double)best[m] : 1e6;  // samples per ms
                // at least 4e6 samples: slow, heavy-tailed queries (C1 cyclic Alley, 8 ms of
                // per-launch tail) need the longer runs for a stable difference
                n2[m] = (uint64_t)std::min(1e8, std::max(4e6, 4.0 * rate));
            }
            cudaEvent_t ev[2][3][3];
            for (int m = 0; m < 2 && rc2 == GSWORD_OK && e == cudaSuccess; ++m)
                for (int c = 0; c < 3 && rc2 == GSWORD_OK && e == cudaSuccess; ++c) {
                    ctx->tuned_occ[m] = c;
                    rc2 = run(ctx, m, gsword::kModeEstimate, range0 + (3 * n2[m] + warm) * (uint64_t)(8 + 3 * m + c), warm,
                              0x5EEDull, ctx->d_out4, nullptr, nullptr);
                    for (int k = 0; k < 3; ++k) event(&ev[m][c][k]);
                    for (int k = 0; k < 2 && rc2 == GSWORD_OK && e == cudaSuccess; ++k) {
                        e = cudaEventRecord(ev[m][c][k], ctx->stream);
                        if (e == cudaSuccess)
                            rc2 = run(ctx, m, gsword::kModeEstimate, range0 + k * n2[m], n2[m] << k, 0x5EEDull,
                                      ctx->d_out4, nullptr, nullptr);
                    }
                    if (rc2 == GSWORD_OK && e == cudaSuccess) e = cudaEventRecord(ev[m][c][2], ctx->stream);
                }
            if (rc2 == GSWORD_OK && e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
            for (int m = 0; m < 2 && rc2 == GSWORD_OK && e == cudaSuccess; ++m) {
                float steady[3];
                for (int c = 0; c < 3 && e == cudaSuccess; ++c) {
                    float a = 0.f, b = 0.f;
                    e = cudaEventElapsedTime(&a, ev[m][c][0], ev[m][c][1]);
                    if (e == cudaSuccess) e = cudaEventElapsedTime(&b, ev[m][c][1], ev[m][c][2]);
                    steady[c] = b - a;
                }
                ctx->tuned_occ[m] = 0;
                for (int c = 1; c < 3 && e == cudaSuccess; ++c)
                    if (steady[c] < 0.99f * steady[ctx->tuned_occ[m]]) ctx->tuned_occ[m] = c;  // 1 % margin
            }
        }
        for (cudaEvent_t x : evs) cudaEventDestroy(x);
        if (rc2 != GSWORD_OK || e != cudaSuccess) {
            ctx->tuned_refill[0] = ctx->tuned_refill[1] = 0;
            ctx->tuned_occ[0] = ctx->tuned_occ[1] = 0;
            return rc2 != GSWORD_OK ? rc2 : cuda_fail(e, "autotune");
        }
        if (ctx->tune_cache.size() >= 4096) ctx->tune_cache.clear();
        ctx->tune_cache[tkey] = {{ctx->tuned_refill[0], ctx->tuned_refill[1]}, {ctx->tuned_occ[0], ctx->tuned_occ[1]}};
    }
    return GSWORD_OK;
}

int gsword_query_info(gsword_ctx* ctx, gsword_query_stats* out) {
    if (!ctx || !out) return fail(GSWORD_EINVAL, "query_info: NULL argument");
    if (!ctx->query_loaded) return fail(GSWORD_ENOQUERY, "query_info: no query loaded");
    std::memset(out, 0, sizeof(*out));
    out->nq = ctx->plan.nq;
    out->filter = ctx->q_filter;
    for (int u = 0; u < ctx->plan.nq; ++u) out->candidates[u] = ctx->cand_count[u];
    out->cg_entries = ctx->cg_entries;
    out->cg_bytes = ctx->cg_bytes;
    out->build_seconds = ctx->cg_seconds;
    out->refill_min[0] = ctx->tuned_refill[0] ? ctx->tuned_refill[0] : ctx->opt_refill_min;
    out->refill_min[1] = ctx->tuned_refill[1] ? ctx->tuned_refill[1] : ctx->opt_refill_min;
    for (int m = 0; m < 2; ++m) {
        int mode = gsword::kModeEstimate | (ctx->q_filter ? gsword::kModeCG : 0);
        if (ctx->opt_sched == 0 && !(m == GSWORD_ALLEY && ctx->opt_streaming)) {
            mode |= occ_variant(ctx, m) << gsword::kModeOccShift;
            if (plan_is_tree(ctx->plan)) mode |= gsword::kModeTree;
            if (m == GSWORD_ALLEY && refill_min_of(ctx, m) == 32) mode |= gsword::kModeLock;
        }
        if (m == GSWORD_ALLEY && ctx->opt_streaming) mode |= gsword::kModeStream;
        if (ctx->opt_sched != 0) mode |= gsword::kModeSync;
        const int occ = gsword::max_blocks_per_sm(
            m, mode, ctx->opt_threads, gsword::sample_smem_rows(m, std::max(1, ctx->plan.nq), ctx->opt_coop), nullptr);
        out->occupancy[m] = ctx->opt_blocks_per_sm > 0 ? std::min(ctx->opt_blocks_per_sm, occ) : occ;
    }
    return GSWORD_OK;
}

int gsword_estimate_async(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                          double* d_out4) {
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    if (!d_out4) return fail(GSWORD_EINVAL, "estimate_async: d_out4 NULL");
    if (n_samples == 0) return fail(GSWORD_EINVAL, "estimate: n_samples must be >= 1");
    if (first + n_samples < first) return fail(GSWORD_EINVAL, "estimate: sample-id range overflows u64");
    return run(ctx, (int)m, gsword::kModeEstimate, first, n_samples, seed, d_out4, nullptr, nullptr);
}

int gsword_finalize(const double* h, gsword_result* out) {
    if (!h || !out) return fail(GSWORD_EINVAL, "finalize: NULL argument");
    const double sum = h[0], sq = h[1], valid = h[2], n = h[3];
    out->sum = sum;
    out->sumsq = sq;
    out->n_valid = (uint64_t)valid;
    out->n_samples = (uint64_t)n;
    out->estimate = n > 0 ? sum / n : std::numeric_limits<double>::quiet_NaN();
    out->variance = n >= 2 ? (sq - sum * sum / n) / (n * (n - 1.0)) : std::numeric_limits<double>::quiet_NaN();
    out->seconds = 0.0;
    return GSWORD_OK;
}

int gsword_estimate_range(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                          gsword_result* out) {
    if (!out) return fail(GSWORD_EINVAL, "estimate: out NULL");
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    CUDA_TRY(cudaEventRecord(ctx->ev0, ctx->stream));
    rc = gsword_estimate_async(ctx, m, first, n_samples, seed, ctx->d_out4);
    if (rc) return rc;
    CUDA_TRY(cudaEventRecord(ctx->ev1, ctx->stream));
    double h[4];
    CUDA_TRY(cudaMemcpyAsync(h, ctx->d_out4, sizeof(h), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    rc = check_accounting(h, n_samples, "estimate");
    if (rc) return rc;
    float ms = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1));
    gsword_finalize(h, out);
    if (ctx->opt_sched == 2) {
        // inheritance: sumsq holds the squared group totals; the groups of 32 consecutive ids
        // are the independent units (reading A24)
        const double n = h[3], m = std::ceil(n / 32.0);
        out->variance = m >= 2 ? m * (h[1] - h[0] * h[0] / m) / ((m - 1.0) * n * n)
                               : std::numeric_limits<double>::quiet_NaN();
    }
    out->seconds = ms * 1e-3;
    return GSWORD_OK;
}

int gsword_estimate(gsword_ctx* ctx, gsword_method m, uint64_t n_samples, uint64_t seed, gsword_result* out) {
    return gsword_estimate_range(ctx, m, 0, n_samples, seed, out);
}

int gsword_estimate_until(gsword_ctx* ctx, gsword_method m, uint64_t seed, double rel_se_target, uint64_t min_samples,
                          uint64_t max_samples, gsword_result* out) {
    if (!out || !(rel_se_target > 0.0) || min_samples < 2 || max_samples < min_samples)
        return fail(GSWORD_EINVAL, "estimate_until: bad argument");
    if (ctx && ctx->opt_sched == 2) return fail(GSWORD_EINVAL, "estimate_until: not with sample inheritance");
    // sample ids 0, 1, 2, ... in doubling batches (resume = a new range, sums add exactly as
    // for a multi-GPU split); stop once sqrt(variance) / estimate <= target or at max_samples
    double acc[4] = {0, 0, 0, 0};
    uint64_t done = 0, batch = min_samples;
    double seconds = 0.0;
    while (done < max_samples) {
        const uint64_t cnt = std::min(batch, max_samples - done);
        gsword_result r;
        int rc = gsword_estimate_range(ctx, m, done, cnt, seed, &r);
        if (rc) return rc;
        acc[0] += r.sum;
        acc[1] += r.sumsq;
        acc[2] += (double)r.n_valid;
        acc[3] += (double)r.n_samples;
        seconds += r.seconds;
        done += cnt;
        gsword_finalize(acc, out);
        if (out->estimate > 0.0 && out->variance >= 0.0 && std::sqrt(out->variance) <= rel_se_target * out->estimate)
            break;
        batch = std::min<uint64_t>(batch * 2, (uint64_t)1 << 40);
    }
    out->seconds = seconds;
    return GSWORD_OK;
}

int gsword_trace_samples(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                         gsword_sample_record* host_out) {
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    if (!host_out) return fail(GSWORD_EINVAL, "trace: host_out NULL");
    if (ctx->opt_sched == 2) return fail(GSWORD_EINVAL, "trace: no per-sample records under sample inheritance");
    if (n_samples == 0) return GSWORD_OK;
    gsword_sample_record* d_rec = nullptr;
    const size_t bytes = sizeof(gsword_sample_record) * (size_t)n_samples;
    cudaError_t e = cudaMalloc(&d_rec, bytes);
    if (e != cudaSuccess) return fail(GSWORD_ENOMEM, "trace: cudaMalloc(%zu): %s", bytes, cudaGetErrorString(e));
    CUDA_TRY(cudaMemsetAsync(d_rec, 0, bytes, ctx->stream));
    rc = run(ctx, (int)m, gsword::kModeTrace, first, n_samples, seed, ctx->d_out4, d_rec, nullptr);
    if (rc == GSWORD_OK) {
        double h4[4];
        e = cudaMemcpyAsync(host_out, d_rec, bytes, cudaMemcpyDeviceToHost, ctx->stream);
        if (e == cudaSuccess) e = cudaMemcpyAsync(h4, ctx->d_out4, sizeof(h4), cudaMemcpyDeviceToHost, ctx->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
        if (e != cudaSuccess) rc = cuda_fail(e, "trace: copy back");
        else rc = check_accounting(h4, n_samples, "trace");
    }
    cudaFree(d_rec);
    return rc;
}

namespace {
int run_trawl(gsword_ctx* ctx, int m, uint64_t first, uint64_t n, uint64_t seed, uint64_t budget,
              gsword_trawl_record* d_rec, double* h4, double* h_timeout) {
    if (first + n < first) return fail(GSWORD_EINVAL, "trawl: sample-id range [first, first + n) overflows u64");
    const int grid = ctx->num_sms * 8;
    if (grid > ctx->partial_cap) {
        if (ctx->d_partials) cudaFree(ctx->d_partials);
        ctx->d_partials = nullptr;
        CUDA_TRY(cudaMalloc(&ctx->d_partials, sizeof(Partial) * (size_t)grid));
        ctx->partial_cap = grid;
    }
    CUDA_TRY(cudaEventRecord(ctx->evk0, ctx->stream));
    CUDA_TRY(gsword::launch_trawl(m, d_rec != nullptr, ctx->opt_trawl_warp != 0, ctx->q_filter != 0, device_graph(ctx), ctx->plan, grid, first,
                                  n, seed, budget, ctx->d_queue, ctx->d_partials, d_rec, ctx->stream));
    CUDA_TRY(cudaEventRecord(ctx->evk1, ctx->stream));
    CUDA_TRY(gsword::launch_reduce(ctx->d_partials, grid, ctx->d_out4, ctx->d_sectors, ctx->stream));
    CUDA_TRY(cudaMemcpyAsync(h4, ctx->d_out4, 4 * sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaMemcpyAsync(h_timeout, ctx->d_sectors, sizeof(double), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    return GSWORD_OK;
}
}  // namespace

int gsword_trawl_range(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                       uint64_t budget, gsword_result* out, uint64_t* n_timeout) {
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    if (!out) return fail(GSWORD_EINVAL, "trawl: out NULL");
    if (n_samples == 0) return fail(GSWORD_EINVAL, "trawl: n_samples must be >= 1");
    double h[4], to = 0.0;
    rc = run_trawl(ctx, (int)m, first, n_samples, seed, budget, nullptr, h, &to);
    if (rc) return rc;
    gsword_finalize(h, out);
    float ms = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&ms, ctx->evk0, ctx->evk1));
    out->seconds = ms * 1e-3;
    if (n_timeout) *n_timeout = (uint64_t)to;
    return GSWORD_OK;
}

int gsword_trace_trawl(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                       uint64_t budget, gsword_trawl_record* host_out) {
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    if (!host_out) return fail(GSWORD_EINVAL, "trace_trawl: host_out NULL");
    if (n_samples == 0) return GSWORD_OK;
    gsword_trawl_record* d_rec = nullptr;
    const size_t bytes = sizeof(gsword_trawl_record) * (size_t)n_samples;
    cudaError_t e = cudaMalloc(&d_rec, bytes);
    if (e != cudaSuccess) return fail(GSWORD_ENOMEM, "trace_trawl: cudaMalloc(%zu): %s", bytes, cudaGetErrorString(e));
    CUDA_TRY(cudaMemsetAsync(d_rec, 0, bytes, ctx->stream));
    double h[4], to = 0.0;
    rc = run_trawl(ctx, (int)m, first, n_samples, seed, budget, d_rec, h, &to);
    if (rc == GSWORD_OK) {
        e = cudaMemcpyAsync(host_out, d_rec, bytes, cudaMemcpyDeviceToHost, ctx->stream);
        if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
        if (e != cudaSuccess) rc = cuda_fail(e, "trace_trawl: copy back");
    }
    cudaFree(d_rec);
    return rc;
}

int gsword_count_sectors(gsword_ctx* ctx, gsword_method m, uint64_t first, uint64_t n_samples, uint64_t seed,
                         double* sectors_out, double* touched_out) {
    int rc = ensure_ready(ctx, (int)m);
    if (rc) return rc;
    if (!sectors_out) return fail(GSWORD_EINVAL, "count_sectors: NULL output");
    if (n_samples == 0) return fail(GSWORD_EINVAL, "count_sectors: n_samples must be >= 1");
    rc = run(ctx, (int)m, gsword::kModeCount, first, n_samples, seed, ctx->d_out4, nullptr, ctx->d_sectors);
    if (rc) return rc;
    double h[2];  // [0] touched by this implementation, [1] algorithmic (reading A26)
    CUDA_TRY(cudaMemcpyAsync(h, ctx->d_sectors, sizeof(h), cudaMemcpyDeviceToHost, ctx->stream));
    unsigned long long ph[8];
    CUDA_TRY(cudaMemcpyAsync(ph, ctx->d_phase, sizeof(ph), cudaMemcpyDeviceToHost, ctx->stream));
    double h4[4];
    CUDA_TRY(cudaMemcpyAsync(h4, ctx->d_out4, sizeof(h4), cudaMemcpyDeviceToHost, ctx->stream));
    CUDA_TRY(cudaStreamSynchronize(ctx->stream));
    rc = check_accounting(h4, n_samples, "count_sectors");
    if (rc) return rc;
    for (int i = 0; i < 8; ++i) ctx->h_phase[i] = (double)ph[i];
    *sectors_out = h[1];
    if (touched_out) *touched_out = h[0];
    return GSWORD_OK;
}

int gsword_phase_cycles(gsword_ctx* ctx, double* out8) {
    if (!ctx || !out8) return fail(GSWORD_EINVAL, "phase_cycles: NULL argument");
    for (int i = 0; i < 8; ++i) out8[i] = ctx->h_phase[i];
    return GSWORD_OK;
}

int gsword_last_kernel_seconds(gsword_ctx* ctx, double* seconds) {
    if (!ctx || !seconds) return fail(GSWORD_EINVAL, "last_kernel_seconds: NULL argument");
    CUDA_TRY(cudaSetDevice(ctx->device));
    CUDA_TRY(cudaEventSynchronize(ctx->evk1));
    float ms = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&ms, ctx->evk0, ctx->evk1));
    *seconds = (double)ms * 1e-3;
    return GSWORD_OK;
}

int gsword_gather_roofline(gsword_ctx* ctx, uint64_t buffer_bytes, int inflight, double* sectors_per_s) {
    if (!ctx || !sectors_per_s || buffer_bytes < 4096 || inflight < 1 || inflight > 8)
        return fail(GSWORD_EINVAL, "gather_roofline: bad argument");
    CUDA_TRY(cudaSetDevice(ctx->device));
    uint32_t* buf = nullptr;
    unsigned long long* sink = nullptr;
    cudaError_t e = cudaMalloc(&buf, buffer_bytes);
    if (e != cudaSuccess) return fail(GSWORD_ENOMEM, "gather_roofline: cudaMalloc(%llu)", (unsigned long long)buffer_bytes);
    e = cudaMalloc(&sink, sizeof(unsigned long long));
    if (e != cudaSuccess) {
        cudaFree(buf);
        return fail(GSWORD_ENOMEM, "gather_roofline: cudaMalloc(sink)");
    }
    const int threads = 256, blocks = ctx->num_sms * 8, steps = 256;
    const uint64_t words = buffer_bytes / 4;
    int rc = GSWORD_OK;
    float ms = 0.f;
    if ((e = cudaMemsetAsync(buf, 0x5A, buffer_bytes, ctx->stream)) != cudaSuccess ||
        (e = gsword::launch_gather(buf, words, 8, inflight, blocks, threads, sink, ctx->stream)) != cudaSuccess ||
        (e = cudaEventRecord(ctx->ev0, ctx->stream)) != cudaSuccess ||
        (e = gsword::launch_gather(buf, words, steps, inflight, blocks, threads, sink, ctx->stream)) != cudaSuccess ||
        (e = cudaEventRecord(ctx->ev1, ctx->stream)) != cudaSuccess || (e = cudaStreamSynchronize(ctx->stream)) != cudaSuccess ||
        (e = cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1)) != cudaSuccess)
        rc = cuda_fail(e, "gather_roofline");
    cudaFree(buf);
    cudaFree(sink);
    if (rc) return rc;
    *sectors_per_s = (double)blocks * threads * (double)steps * inflight / (ms * 1e-3);
    return GSWORD_OK;
}

int gsword_launch_info(gsword_ctx* ctx, int* grid, int* threads, int* launches) {
    if (!ctx) return fail(GSWORD_EINVAL, "launch_info: NULL context");
    if (grid) *grid = ctx->last_grid;
    if (threads) *threads = ctx->last_threads;
    if (launches) *launches = 2;  // sampling kernel + grid reduction
    return GSWORD_OK;
}

}  // extern "C"
