// internal.h — structures shared by the host library (gsword_host.cpp) and the
// sm_100a kernels (gsword_kernels.cu).  Not part of the public ABI.
#pragma once

#include <cstdint>

#include <cuda_runtime.h>

#include "../../include/gsword.h"

namespace gsword {

constexpr int kMaxQV = GSWORD_MAX_QV;

// One matching-order position, staged into shared memory (16 B => one LDS.128).
//   label : L_q(phi[d])
//   back  : bitmask of backward positions B(d) (j < d, query edge to phi[d])
//   dup   : bitmask of j < d with the same label (injectivity candidates, SURVEY R5')
struct alignas(16) PlanStep {
    int32_t label;
    uint32_t back;
    uint32_t dup;
    int32_t nback;
};

struct Plan {
    int32_t nq;
    int32_t seed_identity;  // 1: seed set C(phi[0]) is 0..n-1 (unlabelled) -> no bucket gather
    uint32_t seed_lo;       // C(phi[0]) = bucket[seed_lo, seed_lo + seed_len)
    uint32_t seed_len;
    PlanStep step[kMaxQV];
    uint32_t qadj[kMaxQV];  // bit j: (phi[j], phi[d]) is a query edge, any j != d
    uint8_t uq[kMaxQV];     // phi[d] (query vertex at depth d: row of cbits)
    uint8_t eidx[kMaxQV][kMaxQV];  // directed query edge (phi[j] -> phi[d]) index, j in B(d)
    // comparison variants (GSWORD_OPT_VARIANT, readings A3/A5), applied per launch:
    int32_t wj_parent_first;  // A3: WanderJoin draws from the first backward position's list
    uint32_t pdup[kMaxQV];    // A5: Alley DupCheck after the draw (step[d].dup is then 0)
    int32_t multi_back;       // some position d >= 1 has |B(d)| >= 2 (set per launch)
};

// Candidate filter of one query vertex (NEXT-1): label, degree, and the per-label
// neighbour counts NLF requires.
struct QFilter {
    int32_t label;
    int32_t deg;
    int32_t npairs;
    int32_t plabel[kMaxQV];
    int32_t pcount[kMaxQV];
};

// Device-resident data graph, relaid out for the sampler:
//   col[ seg[v*nL + l] .. seg[v*nL + l + 1] )  = N_l(v), ascending id
//   seg has n*nL + 1 entries; for nL == 1 it is exactly row_ptr (as u32)
//   bucket[ label_off[l] .. label_off[l+1] ) = {v : L(v) = l}, ascending id
//   bloom: blocked Bloom filter over the undirected edge set (one 64-bit word per
//   test, 3 bits, ~16 bits per edge): "no" is exact, "maybe" falls back to the
//   binary search.  NULL = disabled.
//   clist/cg_off/cbits/crank/cg_edge: the lists the sampler draws from.  Filter 0
//   (label only): clist = col, runs located through seg.  Filters 1-2 (LDF/NLF,
//   NEXT-1): the candidate graph in the three-CSR format of Fig. 4 (Def. 5, P:L526,
//   P:L770-L776):
//     1st CSR  the query edges: e = (u -> u') indexes cg_edge[e] = {base, u};
//     2nd CSR  C(u) in ascending id, held as the membership bitmap cbits row u with a
//              rank directory crank row u (exclusive popcount prefix per 32-bit word):
//              the position of v in C(u) is crank[u][v/32] + popc(cbits[u][v/32] below
//              v) -- two independent loads instead of the paper's search;
//     3rd CSR  per edge e, |C(u)| + 1 offsets at cg_off[base ...]: the local candidate
//              list C(u, u', v) = N(v) ∩ C(u') of the i-th v of C(u) is
//              clist[cg_off[base + i] .. cg_off[base + i + 1]), ascending.
//   Memory O(nq |V| / 8 + sum_e |C(u_e)| + entries), not O(|E_q| |V|); a lookup is only
//   made for v in C(u) (every matched vertex lies in its query vertex's candidate set).
struct DeviceGraph {
    const int32_t* col;
    const uint32_t* seg;
    const int32_t* bucket;     // seed list: label buckets, or C(phi[0]) under a filter
    const int32_t* clist;
    const uint32_t* cg_off;
    const uint32_t* cbits;
    const uint32_t* crank;     // rank directory of cbits (same shape)
    const uint2* cg_edge;      // per directed query edge: {offset base in cg_off, source u}
    uint32_t cwords;           // words per cbits row
    const unsigned long long* bloom;
    uint64_t bloom_mask;  // words - 1 (words is a power of two)
    // exact edge set: open addressing, 32-byte buckets of 4 keys (min<<32 | max),
    // linear probing over buckets, load <= 1/2.  NULL = use binary search instead.
    const unsigned long long* eset;
    uint64_t eset_mask;   // buckets - 1
    int64_t n;
    int64_t nnz;
    int32_t n_labels;
};

__host__ __device__ inline uint64_t edge_key(uint32_t a, uint32_t b) {
    return a < b ? (((uint64_t)a << 32) | b) : (((uint64_t)b << 32) | a);
}

// Hash of an undirected edge {a, b}: one 64-bit Fibonacci multiply, high half folded
// into the low half (the low bits index the filter word and the edge-set bucket, bits
// 40..57 pick the filter bits).  Used by the device-side builds and tests alike; any
// hash gives the same answers (both structures are exact on "no" / on membership), this
// one costs 5 instructions instead of splitmix64's ~14 with the same measured bucket
// overflow and filter false-positive rate on C1.
__host__ __device__ inline uint64_t edge_hash(uint32_t a, uint32_t b) {
    const uint64_t z = edge_key(a, b) * 0x9E3779B97F4A7C15ull;
    return z ^ (z >> 32);
}


// The four filter bits of h in one 64-bit word: a split block, two bits in each 32-bit half
// picked by four 5-bit fields of h's bits 40..62 (10 instructions; four positions anywhere in
// the word took ~22).  0.49 % false positives on random C1 vertex pairs at 16 bits per edge
// (0.48 % with four free positions).
__host__ __device__ inline uint64_t bloom_bits(uint64_t h) {
    const uint32_t hh = (uint32_t)(h >> 32);
    const uint32_t lo = (1u << ((hh >> 8) & 31u)) | (1u << ((hh >> 13) & 31u));
    const uint32_t hi = (1u << ((hh >> 18) & 31u)) | (1u << ((hh >> 23) & 31u));
    return ((uint64_t)hi << 32) | lo;
}

// Launch parameters of one estimate.
struct LaunchCfg {
    int grid;
    int threads;
    int chunk;
    int coop_threshold;
    int sched;  // 0 refill, 1 sample synchronisation, 2 + inheritance (NEXT-3)
    uint32_t refill_min;  // sched 0: refill when at least this many lanes are free (1..32)
    int ms_rows;          // rows of the dynamic shared array (sample_smem_rows)
    uint64_t queue_start = 0;  // initial sample-queue value (0; fault injection only)
};

// Applies the GSWORD_OPT_VARIANT bits to a copy of the loaded plan (readings A3, A5).
inline Plan plan_variant(const Plan& base, int method, int variant) {
    Plan p = base;
    p.wj_parent_first = (method == GSWORD_WJ && (variant & GSWORD_VARIANT_WJ_PARENT_FIRST)) ? 1 : 0;
    for (int d = 0; d < kMaxQV; ++d) p.pdup[d] = 0u;
    if (method == GSWORD_ALLEY && (variant & GSWORD_VARIANT_ALLEY_DUPCHECK_POST))
        for (int d = 0; d < kMaxQV; ++d) {
            p.pdup[d] = p.step[d].dup;
            p.step[d].dup = 0u;
        }
    return p;
}

// Per-CTA partial aggregate (written by the sampling kernel, reduced in CTA order).
struct Partial {
    double sum_hi, sum_lo;      // double-double sum of Y
    double sq_hi, sq_lo;        // double-double sum of Y*Y
    unsigned long long valid;   // complete instances
    unsigned long long n;       // samples
    double sectors;             // counting build: sectors the implementation touches (trawl: timeouts)
    double model;               // counting build: algorithmic sectors of reading A26
};

// Kernel entry points (gsword_kernels.cu).  All enqueue on `stream`.
cudaError_t launch_sample(int method, int mode, const DeviceGraph& g, const Plan& plan, const LaunchCfg& cfg,
                          uint64_t first, uint64_t count, uint64_t seed, unsigned long long* d_queue,
                          Partial* d_partials, gsword_sample_record* d_records, unsigned long long* d_phase,
                          cudaStream_t stream);
cudaError_t launch_reduce(const Partial* d_partials, int n_partials, double* d_out4, double* d_sectors,
                          cudaStream_t stream);
cudaError_t launch_build_bucket_identity(int32_t* bucket, int64_t n, cudaStream_t stream);
cudaError_t launch_gather(const uint32_t* buf, uint64_t words, int steps, int inflight, int blocks, int threads,
                          unsigned long long* sink, cudaStream_t stream);
// device-side graph load (gsword_load_graph_device)
cudaError_t launch_dev_validate(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n,
                                int32_t n_labels, int* d_bad, cudaStream_t stream);
cudaError_t launch_dev_seg(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n, int32_t L,
                           uint32_t* seg, cudaStream_t stream);
cudaError_t launch_label_hist(const int32_t* labels, int64_t n, unsigned long long* hist, cudaStream_t stream);
cudaError_t launch_pair_hist(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n, int32_t L,
                             unsigned long long* hist, cudaStream_t stream);
cudaError_t launch_label_bucket(const int32_t* labels, int64_t n, int32_t l, uint32_t* counts,
                                const unsigned long long* d_base, uint32_t* d_tmp, unsigned long long* d_total,
                                int32_t* bucket, cudaStream_t stream);
cudaError_t launch_trawl(int method, bool trace, bool warp, bool cg, const DeviceGraph& g, const Plan& plan, int grid,
                         uint64_t first, uint64_t count, uint64_t seed, uint64_t budget, unsigned long long* d_queue,
                         Partial* d_partials, gsword_trawl_record* d_records, cudaStream_t stream);
// candidate graph build (NEXT-1)
cudaError_t launch_filter(const DeviceGraph& g, const QFilter* d_qf, int nq, int filter, uint32_t* cbits,
                          const int32_t* d_vlabel, cudaStream_t stream);
// rank directory row u: crank[u][w] = popc(cbits[u][w]) (scanned afterwards)
cudaError_t launch_rank_words(const uint32_t* cbits, uint32_t cwords, int u, uint32_t* crank, cudaStream_t stream);
// counts[rank_u(v)] = |N_label2(v) ∩ C(u2)| for every v in C(u)  (g.cbits / g.crank set)
cudaError_t launch_cg_count(const DeviceGraph& g, int u, int u2, int32_t label2, uint32_t* counts,
                            cudaStream_t stream);
cudaError_t launch_cg_fill(const DeviceGraph& g, int u, int u2, int32_t label2, const uint32_t* off, int32_t* out,
                           cudaStream_t stream);
// out[rank_u(v)] = v for every v in C(u): the ascending list C(u)
cudaError_t launch_cand_fill(const DeviceGraph& g, int u, int32_t* out, cudaStream_t stream);
// exclusive scan of n u32 in place, offset by *d_base (64-bit, may be NULL = 0); the
// 64-bit grand total goes to *d_total.  d_tmp holds scan_tmp_words(n) words.
size_t scan_tmp_words(int64_t n);
cudaError_t launch_scan(uint32_t* data, int64_t n, const unsigned long long* d_base, uint32_t* d_tmp,
                        unsigned long long* d_total, cudaStream_t stream);
constexpr unsigned long long kEmptyKey = ~0ull;
cudaError_t launch_build_eset(const int64_t* d_row_ptr, const int32_t* col, int64_t n, unsigned long long* keys,
                              uint64_t mask, cudaStream_t stream);
cudaError_t launch_build_bloom(const int64_t* d_row_ptr, const int32_t* col, int64_t n, unsigned long long* bloom,
                               uint64_t mask, cudaStream_t stream);
// Rows of blockDim.x words of the sampling kernel's dynamic shared memory: n_q rows of
// matched vertices, plus for Alley the task-pool result row and ceil(coop/32) refine-mask
// rows.
// Row stride (words) of the sampling kernel's dynamic shared matrix: the largest CTA, a
// compile-time constant so the row indexing holds no register; smaller CTAs leave rows' tails unused.
constexpr int kSampleLanes = 256;
inline int sample_smem_rows(int method, int nq, int coop_threshold) {
    return nq + (method == GSWORD_ALLEY ? 1 + (coop_threshold + 31) / 32 : 0);
}
// ms_rows = sample_smem_rows(...)
int max_blocks_per_sm(int method, int mode, int threads, int ms_rows, size_t* smem_bytes);
// minimum resident CTAs per SM the sampling kernel is compiled for (launch bounds)
int occ_blocks(int method, int occ_variant);

enum Mode {
    kModeEstimate = 0,
    kModeTrace = 1,
    kModeCount = 2,
    kModeCG = 4,     // flag: candidate graph
    kModeStream = 8,  // flag: Alley by warp streaming (Alg. 3, NEXT-3)
    kModeSync = 16,   // flag: a scheduling mode other than refill (GSWORD_OPT_SCHEDULE != 0)
    kModeOccShift = 5,  // bits 5-6: occupancy variant of the estimate kernel (0 default, 1 one
                        // CTA/SM less, 2 one more; refill schedule only), see occ_blocks()
    kModeTree = 128,    // flag: every position has one backward neighbour (estimate kernels)
    kModeLock = 256     // flag: Alley estimate with refill threshold 32 (depth-synchronous warps)
};

}  // namespace gsword
