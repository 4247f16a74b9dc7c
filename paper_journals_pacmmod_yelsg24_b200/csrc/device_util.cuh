// device_util.cuh — device helpers of the sampling kernels (gsword_kernels.cu: the
// persistent refill kernels, warp streaming, trawling): Philox, edge index, list runs,
// compensated sums.  Not part of the public ABI; every function is inline.
#pragma once

#include <cstdint>

#include "internal.h"

namespace gsword {
namespace dev {

constexpr unsigned kFull = 0xffffffffu;

// ---------------------------------------------------------------- Philox4x32-10 (A6)
// counter = (sid, d, c3): c3 = 0 for the plain draws; warp streaming (reading A25) uses
// c3 = 1 + element index (reservoir keys) and 0x80000000 | chunk (chunk merges)
__device__ __forceinline__ uint64_t philox_rc(uint64_t seed, uint64_t sid, uint32_t d, uint32_t c3) {
    uint32_t c0 = (uint32_t)sid, c1 = (uint32_t)(sid >> 32), c2 = d;
    uint32_t k0 = (uint32_t)seed, k1 = (uint32_t)(seed >> 32);
#pragma unroll
    for (int i = 0; i < 10; ++i) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
        const uint32_t n0 = hi1 ^ c1 ^ k0;
        const uint32_t n2 = hi0 ^ c3 ^ k1;
        c0 = n0;
        c1 = lo1;
        c2 = n2;
        c3 = lo0;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    return ((uint64_t)c1 << 32) | (uint64_t)c0;
}

__device__ __forceinline__ uint64_t philox_r(uint64_t seed, uint64_t sid, uint32_t d) {
    return philox_rc(seed, sid, d, 0u);
}

__device__ __forceinline__ int32_t ldg_i32(const int32_t* p) { return __ldg(p); }
__device__ __forceinline__ uint32_t ldg_u32(const uint32_t* p) { return __ldg(p); }

// Branchless search over the ascending run col[lo, lo+n): the trip count depends on
// n only (no data-dependent branches).  Returns the index of the last element <= x
// (lo if none) and whether it equals x.
__device__ __forceinline__ uint32_t search_last_le(const int32_t* __restrict__ col, uint32_t lo, uint32_t n,
                                                   int32_t x, bool* found) {
    if (n == 0) {
        *found = false;
        return lo;
    }
    while (n > 1) {
        const uint32_t half = n >> 1;
        lo = (ldg_i32(col + lo + half) <= x) ? lo + half : lo;
        n -= half;
    }
    *found = ldg_i32(col + lo) == x;
    return lo;
}

__device__ __forceinline__ bool in_run(const int32_t* __restrict__ col, uint32_t lo, uint32_t hi, int32_t x) {
    bool f;
    search_last_le(col, lo, hi - lo, x, &f);
    return f;
}

// position of the k-th (0-based) set bit of m (k < popc(m))
__device__ __forceinline__ uint32_t fns32(uint32_t m, uint32_t k) {
    uint32_t pos = 0, c;
    c = __popc(m & 0xFFFFu); if (k >= c) { k -= c; m >>= 16; pos += 16; }
    c = __popc(m & 0xFFu);   if (k >= c) { k -= c; m >>= 8;  pos += 8; }
    c = __popc(m & 0xFu);    if (k >= c) { k -= c; m >>= 4;  pos += 4; }
    c = __popc(m & 0x3u);    if (k >= c) { k -= c; m >>= 2;  pos += 2; }
    c = m & 1u;              if (k >= c) { pos += 1; }
    return pos;
}

// the same for masks of query positions (<= 16 bits, k usually 0-2): clear k low bits
__device__ __forceinline__ int fns_small(uint32_t m, uint32_t k) {
    while (k--) m &= m - 1;
    return __ffs(m) - 1;
}

// algorithmic sectors of a binary search over a sorted run of `len` 4-byte ids
__device__ __forceinline__ uint32_t bs_sectors(uint32_t len) {
    if (len == 0) return 0;
    const uint32_t c = (len + 7) / 8;
    return 1 + (c > 1 ? 32 - __clz(c - 1) : 0);
}

__device__ __forceinline__ uint32_t scan_sectors(uint32_t len) { return (4 * len + 31) / 32; }

// Neumaier-compensated accumulation
__device__ __forceinline__ void nsum(double& s, double& c, double x) {
    const double t = __dadd_rn(s, x);
    if (fabs(s) >= fabs(x)) c = __dadd_rn(c, __dadd_rn(__dsub_rn(s, t), x));
    else c = __dadd_rn(c, __dadd_rn(__dsub_rn(x, t), s));
    s = t;
}

// double-double addition (a_hi, a_lo) += (b_hi, b_lo)
__device__ __forceinline__ void dd_add(double& ah, double& al, double bh, double bl) {
    const double s = __dadd_rn(ah, bh);
    const double v = __dsub_rn(s, ah);
    double e = __dadd_rn(__dsub_rn(ah, __dsub_rn(s, v)), __dsub_rn(bh, v));
    e = __dadd_rn(e, __dadd_rn(al, bl));
    ah = __dadd_rn(s, e);
    al = __dsub_rn(e, __dsub_rn(ah, s));
}

__device__ __forceinline__ double shfl_xor_d(double x, int m) { return __shfl_xor_sync(kFull, x, m); }

// segment of N_l(v): [seg[v*nL + l], seg[v*nL + l + 1])
__device__ __forceinline__ void segment(const DeviceGraph& g, uint32_t v, int32_t l, uint32_t* a, uint32_t* b) {
    const size_t i = (size_t)v * (size_t)g.n_labels + (size_t)l;
    *a = ldg_u32(g.seg + i);
    *b = ldg_u32(g.seg + i + 1);
}

// Run of the local candidate list C(phi[j], phi[d], v) in clist (Def. 4): the
// label-filtered adjacency run (filter 0) or the candidate-graph row of directed
// query edge e (filters 1-2).
template <bool CG>
__device__ __forceinline__ void local_run(const DeviceGraph& g, int e, uint32_t v, int32_t l, uint32_t* a,
                                          uint32_t* b) {
    if (CG) {
        // Fig. 4: query edge e (1st CSR) -> position of v in C(u) (2nd CSR, rank directory)
        // -> offsets of C(u, u', v) (3rd CSR); v lies in C(u) (it was matched to u)
        const uint2 ed = __ldg(g.cg_edge + e);
        const size_t w = (size_t)ed.y * g.cwords + (v >> 5);
        const uint32_t bits = ldg_u32(g.cbits + w), pre = ldg_u32(g.crank + w);
        const uint32_t* off = g.cg_off + (size_t)ed.x + pre + __popc(bits & ((1u << (v & 31u)) - 1u));
        *a = ldg_u32(off);
        *b = ldg_u32(off + 1);
    } else {
        segment(g, v, l, a, b);
    }
}

// v in C(u)?  (membership bitmap of the candidate graph; only used under a filter)
__device__ __forceinline__ bool in_cand(const DeviceGraph& g, int u, uint32_t v) {
    return (ldg_u32(g.cbits + (size_t)u * g.cwords + (v >> 5)) >> (v & 31u)) & 1u;
}

// Is {a, b} an edge of G?  Exact.  (1) blocked Bloom filter (L2-resident): "no" is
// final; (2) exact edge set (one 32-byte bucket per probe); without the edge set, a
// binary search of b in N_lb(a) (lb = L(b)).  `sec` accumulates the sectors touched.
template <bool COUNT>
__device__ __forceinline__ bool is_edge(const DeviceGraph& g, uint32_t a, uint32_t b, int32_t lb, double& sec) {
    const uint64_t h = edge_hash(a, b);
    if (g.bloom) {
        if (COUNT) sec += 1.0;
        const uint64_t m = bloom_bits(h);
        if ((__ldg(g.bloom + (h & g.bloom_mask)) & m) != m) return false;
    }
    if (g.eset) {
        const unsigned long long key = edge_key(a, b);
        uint64_t bk = h & g.eset_mask;
        while (true) {
            if (COUNT) sec += 1.0;
            const ulonglong2* p = reinterpret_cast<const ulonglong2*>(g.eset + 4 * bk);
            const ulonglong2 x0 = __ldg(p), x1 = __ldg(p + 1);
            if (x0.x == key || x0.y == key || x1.x == key || x1.y == key) return true;
            if (x0.x == kEmptyKey || x0.y == kEmptyKey || x1.x == kEmptyKey || x1.y == kEmptyKey) return false;
            bk = (bk + 1) & g.eset_mask;
        }
    }
    uint32_t lo, hi;
    segment(g, a, lb, &lo, &hi);
    if (COUNT) sec += 1.0 + (double)bs_sectors(hi - lo);
    return in_run(g.col, lo, hi, (int32_t)b);
}

// The two halves of is_edge: the filter test alone ("maybe", never a false "no"; true when
// there is no filter), and the exact test alone (edge-set buckets, or a binary search).
template <bool COUNT>
__device__ __forceinline__ bool bloom_maybe(const DeviceGraph& g, uint32_t a, uint32_t b, double& sec) {
    if (!g.bloom) return true;
    if (COUNT) sec += 1.0;
    const uint64_t h = edge_hash(a, b);
    const uint64_t m = bloom_bits(h);
    return (__ldg(g.bloom + (h & g.bloom_mask)) & m) == m;
}

template <bool COUNT>
__device__ __forceinline__ bool is_edge_exact(const DeviceGraph& g, uint32_t a, uint32_t b, int32_t lb, double& sec) {
    if (g.eset) {
        const unsigned long long key = edge_key(a, b);
        uint64_t bk = edge_hash(a, b) & g.eset_mask;
        while (true) {
            if (COUNT) sec += 1.0;
            const ulonglong2* p = reinterpret_cast<const ulonglong2*>(g.eset + 4 * bk);
            const ulonglong2 x0 = __ldg(p), x1 = __ldg(p + 1);
            if (x0.x == key || x0.y == key || x1.x == key || x1.y == key) return true;
            if (x0.x == kEmptyKey || x0.y == kEmptyKey || x1.x == kEmptyKey || x1.y == kEmptyKey) return false;
            bk = (bk + 1) & g.eset_mask;
        }
    }
    uint32_t lo, hi;
    segment(g, a, lb, &lo, &hi);
    if (COUNT) sec += 1.0 + (double)bs_sectors(hi - lo);
    return in_run(g.col, lo, hi, (int32_t)b);
}

// Is x in every N_l(M[j]) for j in `mask`?  M column `col_of` in shared memory.
template <bool COUNT>
__device__ __forceinline__ bool member_all(const DeviceGraph& g, const uint32_t* Ms, int stride, int col_of,
                                           uint32_t mask, int32_t l, int32_t x, double& sec) {
    while (mask) {
        const int j = __ffs(mask) - 1;
        mask &= mask - 1;
        if (!is_edge<COUNT>(g, Ms[j * stride + col_of], (uint32_t)x, l, sec)) return false;
    }
    return true;
}

// One-word signature of a lane's matched vertices: bit sig_bit(v) is set for every M[j].
// A clear bit proves x is not matched, so the exact scan of M is skipped (~80 % of the
// DupChecks of an 8-vertex query).
__device__ __forceinline__ uint32_t sig_bit(int32_t v) { return 1u << (((uint32_t)v * 0x9E3779B1u) >> 27); }

__device__ __forceinline__ bool not_matched(const uint32_t* Ms, int stride, int col_of, uint32_t dup, int32_t x) {
    while (dup) {
        const int j = __ffs(dup) - 1;
        dup &= dup - 1;
        if ((int32_t)Ms[j * stride + col_of] == x) return false;
    }
    return true;
}

__device__ __forceinline__ bool not_matched_sig(const uint32_t* Ms, int stride, int col_of, uint32_t dup, uint32_t sig,
                                                int32_t x) {
    return !(sig & sig_bit(x)) || not_matched(Ms, stride, col_of, dup, x);
}

// Algorithmic sectors (reading A26) of an Alley refine with |B(d)| >= 2 over the driver run
// clist[lo, lo + len): the driver scan, then for each driver element that is not a matched
// vertex one membership question per other list in ascending position up to the first "no".
// Trace / counting builds only (the estimate kernel never calls it).
__device__ inline uint32_t model_refine_sectors(const DeviceGraph& g, const uint32_t* Ms, int T, int tid, uint32_t lo,
                                         uint32_t len, uint32_t others, uint32_t dup, int32_t label) {
    uint32_t s = (len + 7u) / 8u;
    double unused = 0.0;
    for (uint32_t i = 0; i < len; ++i) {
        const int32_t x = ldg_i32(g.clist + lo + i);
        if (!not_matched(Ms + tid, T, 0, dup, x)) continue;
        uint32_t m = others;
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            s += 1u;
            if (!is_edge<false>(g, Ms[j * T + tid], (uint32_t)x, label, unused)) break;
        }
    }
    return s;
}

}  // namespace dev
}  // namespace gsword
