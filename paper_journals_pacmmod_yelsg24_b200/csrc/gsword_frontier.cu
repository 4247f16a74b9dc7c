// gsword_frontier.cu — level-synchronous ("frontier") Alley sampler for sm_100a.
//
// The persistent kernel (gsword_kernels.cu) keeps one sample per lane and refills lanes as
// samples die; lanes of a warp sit at different depths, so the depth-dependent work (which
// refine path, how many exclusion tests) diverges and is load-balanced through a warp task
// pool.  Here a batch of sample ids is advanced one matching-order position (depth) per
// kernel launch over a compacted frontier of the samples still alive:
//
//   * every thread of a launch runs the SAME position d, so the plan step, the refine kind
//     and the set of exclusion tests are warp-uniform: no divergence between kinds, no task
//     pool, and a thread issues all of its edge tests back to back (memory-level
//     parallelism inside the thread);
//   * dead samples leave the frontier (warp-aggregated compaction), so no lane idles on
//     them (the validate imbalance of P:L379 solved by compaction instead of refill);
//   * the frontier is structure-of-arrays (sample slot, W, M[0..d], and for traces csize
//     and the A26 sector count), read and written coalesced;
//   * drivers longer than the cooperative threshold are refined by the whole warp in
//     32-element coalesced chunks (ballot / popc / find-nth), as in the persistent kernel.
//
// Every random choice, every candidate set and every weight is the one of SURVEY R2-R9
// (Alley; Fig. 19 AL), so records and aggregates equal the persistent kernel's and
// the CPU oracle's (tests/test_gpu_frontier.py).  Readings: A5 (matched vertices removed inside
// refine), A6 (Philox, mulhi64), A7 (W = prod |C_d|), A26 (sector model, trace builds).
#include <cstdint>

#include "device_util.cuh"
#include "internal.h"

namespace gsword {
namespace {

using namespace dev;

struct FrontierArgs {
    FrontierBufs in, out;
    const uint32_t* n_in;   // alive samples entering this level (device counter)
    uint32_t* n_out;        // survivors leaving it
    uint32_t n_first;       // level 1: samples of the batch (the frontier is implicit)
    uint32_t cap;           // capacity of every frontier array
    uint64_t batch_first;   // sample id of slot 0
    uint64_t range_first;   // first sample id of the range (record index base)
    uint64_t seed;
    int d;                  // position advanced by this launch (>= 1)
    uint32_t coop_threshold;
};

__device__ __forceinline__ void accumulate(double& s, double& c, double& q, double& cq, double y) {
    nsum(s, c, y);
    nsum(q, cq, __dmul_rn(y, y));
}

// One launch = one position d of every alive sample of the frontier.
//   FIRST: d = 1, fused with the seed (position 0) of samples [0, n_first) of the batch
//   MULTI: |B(d)| >= 2 (intersection refine), else a single backward list (exclusion refine)
template <bool CG, bool TRACE, bool FIRST, bool MULTI>
__global__ void __launch_bounds__(256) frontier_kernel(const DeviceGraph g, const Plan plan_in,
                                                       const FrontierArgs A, Partial* __restrict__ partials,
                                                       gsword_sample_record* __restrict__ records) {
    __shared__ PlanStep plan_s[kMaxQV];
    __shared__ uint32_t qadj_s[kMaxQV];
    __shared__ uint8_t eidx_s[kMaxQV][kMaxQV];
    __shared__ uint8_t uq_s[kMaxQV];
    __shared__ Partial warp_part[8];
    const int tid = threadIdx.x, lane = tid & 31;
    if (tid < kMaxQV) {
        plan_s[tid] = plan_in.step[tid];
        qadj_s[tid] = plan_in.qadj[tid];
        uq_s[tid] = plan_in.uq[tid];
    }
    if (tid < kMaxQV * kMaxQV) eidx_s[tid / kMaxQV][tid % kMaxQV] = plan_in.eidx[tid / kMaxQV][tid % kMaxQV];
    __syncthreads();

    const int nq = plan_in.nq;
    const int d = A.d;
    const bool last = d + 1 == nq;
    const PlanStep ps = plan_s[d];
    const uint32_t cap = A.cap;
    const unsigned lt_mask = (1u << lane) - 1u;
    const uint32_t n = FIRST ? A.n_first : *A.n_in;

    double s_sum = 0.0, c_sum = 0.0, s_sq = 0.0, c_sq = 0.0;
    unsigned long long n_valid = 0, n_done = 0;

    const uint32_t warps_total = (gridDim.x * blockDim.x) >> 5;
    const uint32_t warp_id = (blockIdx.x * blockDim.x + tid) >> 5;
    for (uint32_t base = warp_id * 32u; base < n; base += warps_total * 32u) {
        const uint32_t i = base + (uint32_t)lane;
        bool alive = i < n;
        uint32_t slot = 0, msec = 0;
        double W = 0.0;
        int32_t m0 = 0;  // FIRST: the seed vertex M[0]
        uint32_t cs0 = 0;
        if (alive) {
            if (FIRST) {
                slot = i;
                n_done += 1;  // every sample id of the batch counts in n (reading A8)
                const uint32_t c0 = plan_in.seed_len;
                W = (double)c0;
                cs0 = c0;
                if (c0 == 0u) {
                    alive = false;
                    if (TRACE) {
                        gsword_sample_record* rec = records + (A.batch_first - A.range_first + slot);
                        rec->sample_id = A.batch_first + slot;
                        rec->valid = 0;
                        rec->depth_reached = 0;
                        rec->sectors = 0;
                        rec->weight = 0.0;
#pragma unroll
                        for (int j = 0; j < kMaxQV; ++j) {
                            rec->path[j] = -1;
                            rec->csize[j] = 0;
                        }
                    }
                } else {
                    const uint64_t k = __umul64hi(philox_r(A.seed, A.batch_first + slot, 0u), (uint64_t)c0);
                    m0 = plan_in.seed_identity ? (int32_t)(plan_in.seed_lo + k)
                                               : ldg_i32(g.bucket + plan_in.seed_lo + k);
                    if (TRACE && (int64_t)c0 != g.n) msec = 1u;  // A26: the seed is read from its list
                }
            } else {
                slot = A.in.slot[i];
                W = A.in.W[i];
                if (TRACE) msec = A.in.msec[i];
            }
        }
        // M[j] of this sample (j < d); position 0 comes from the seed at level 1
        auto Mj = [&](int j) -> int32_t { return FIRST ? m0 : A.in.M[(size_t)j * cap + i]; };
        const uint64_t sid = A.batch_first + slot;
        uint64_t r = 0;
        if (alive) r = philox_r(A.seed, sid, (uint32_t)d);

        uint32_t cnt = 0;
        int32_t v = -1;
        bool coop = false;
        uint32_t lo_p = 0, len_p = 0;
        int p = 0;
        if (!MULTI) {
            // ---- one backward list: C_d = S_p minus the matched same-label vertices in S_p
            p = __ffs(ps.back) - 1;
            int32_t vp = 0;
            uint32_t in_sp = 0;
            if (alive) {
                vp = Mj(p);
                uint32_t a, b;
                local_run<CG>(g, eidx_s[d][p], (uint32_t)vp, ps.label, &a, &b);
                const uint32_t cdup = ps.dup & ~(1u << p);
                const uint32_t qa = qadj_s[p];
                uint32_t known = 0, unk = 0;
                if (CG) {
                    // under a filter S_p lies in C(phi[d]): matched vertices outside it are not in S_p
                    uint32_t m = cdup;
                    while (m) {
                        const int j = __ffs(m) - 1;
                        m &= m - 1;
                        if (in_cand(g, uq_s[d], (uint32_t)Mj(j))) (qa >> j & 1u ? known : unk) |= 1u << j;
                    }
                } else {
                    known = cdup & qa;  // a partial instance: M[j] ~ M[p] when phi[j] ~ phi[p]
                    unk = cdup & ~qa;
                }
                // edge tests {M[p], M[j]}, four in flight: the filter words first, then the
                // edge-set buckets of the "maybe"s
                uint32_t m = unk;
                while (m) {
                    int jj[4];
                    uint64_t hh[4];
                    unsigned long long ww[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        jj[u] = m ? __ffs(m) - 1 : -1;
                        if (m) m &= m - 1;
                        hh[u] = jj[u] >= 0 ? edge_hash((uint32_t)vp, (uint32_t)Mj(jj[u])) : 0ull;
                        ww[u] = (jj[u] >= 0 && g.bloom) ? __ldg(g.bloom + (hh[u] & g.bloom_mask)) : ~0ull;
                    }
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        if (jj[u] < 0) continue;
                        const uint64_t mb = bloom_bits(hh[u]);
                        double unused = 0.0;
                        if ((!g.bloom || (ww[u] & mb) == mb) &&
                            is_edge_after_filter(g, (uint32_t)vp, (uint32_t)Mj(jj[u]), hh[u], ps.label, unused))
                            in_sp |= 1u << jj[u];
                    }
                }
                in_sp |= known;
                lo_p = a;
                len_p = b - a;
                cnt = len_p - (uint32_t)__popc(in_sp);
                if (TRACE) msec += 1u + (len_p ? (uint32_t)__popc(CG ? cdup : (cdup & ~qa)) : 0u) + (cnt ? 1u : 0u);
                if (cnt > 0) {
                    // the k-th survivor: smallest idx with idx = k + #{x in X : x <= S_p[idx]}
                    const uint32_t k = (uint32_t)__umul64hi(r, (uint64_t)cnt);
                    const int nx = __popc(in_sp);
                    if (nx <= 2) {
                        const int32_t* wb = g.clist + lo_p + k;
                        const int32_t w0 = ldg_i32(wb);
                        const int32_t w1 = nx >= 1 ? ldg_i32(wb + 1) : 0;
                        const int32_t w2 = nx >= 2 ? ldg_i32(wb + 2) : 0;
                        const int32_t x0 = nx >= 1 ? Mj(__ffs(in_sp) - 1) : INT32_MAX;
                        const int32_t x1 = nx >= 2 ? Mj(31 - __clz(in_sp)) : INT32_MAX;
                        uint32_t t = 0;
#pragma unroll
                        for (int it = 0; it < 2; ++it) {
                            const int32_t wi = t == 0 ? w0 : (t == 1 ? w1 : w2);
                            t = (uint32_t)(x0 <= wi) + (uint32_t)(x1 <= wi);
                        }
                        v = t == 0 ? w0 : (t == 1 ? w1 : w2);
                    } else {
                        for (uint32_t idx = k;;) {
                            v = ldg_i32(g.clist + lo_p + idx);
                            uint32_t c = 0, xm = in_sp;
                            while (xm) {
                                const int j = __ffs(xm) - 1;
                                xm &= xm - 1;
                                c += (Mj(j) <= v) ? 1u : 0u;
                            }
                            if (idx == k + c) break;
                            idx = k + c;
                        }
                    }
                }
            }
        } else {
            // ---- |B(d)| >= 2: GetMinCandidate, then the intersection minus matched vertices
            if (alive) {
                uint32_t bm = ps.back;
                len_p = 0xFFFFFFFFu;
                while (bm) {
                    const int j = __ffs(bm) - 1;
                    bm &= bm - 1;
                    uint32_t a, b;
                    local_run<CG>(g, eidx_s[d][j], (uint32_t)Mj(j), ps.label, &a, &b);
                    if (b - a < len_p) {
                        len_p = b - a;
                        lo_p = a;
                        p = j;
                    }
                }
                if (TRACE) msec += (uint32_t)ps.nback;
                coop = len_p > (A.coop_threshold < 64u ? A.coop_threshold : 64u);
                if (TRACE && len_p > 0) {
                    // A26 questions (trace builds only): scan + membership up to the first "no"
                    uint32_t s = (len_p + 7u) / 8u;
                    double unused = 0.0;
                    for (uint32_t e = 0; e < len_p; ++e) {
                        const int32_t x = ldg_i32(g.clist + lo_p + e);
                        bool matched = false;
                        for (uint32_t mm = ps.dup; mm; mm &= mm - 1) matched |= Mj(__ffs(mm) - 1) == x;
                        if (matched) continue;
                        for (uint32_t o = ps.back & ~(1u << p); o; o &= o - 1) {
                            s += 1u;
                            if (!is_edge<false>(g, (uint32_t)Mj(__ffs(o) - 1), (uint32_t)x, ps.label, unused)) break;
                        }
                    }
                    msec += s;
                }
                if (len_p > 0 && !coop) {
                    // short driver: this thread refines it, four elements in flight
                    const uint32_t others = ps.back & ~(1u << p);
                    uint64_t keep = 0;
                    for (uint32_t e0 = 0; e0 < len_p; e0 += 4) {
                        int32_t xs[4];
                        bool kp[4];
#pragma unroll
                        for (int u = 0; u < 4; ++u) {
                            kp[u] = e0 + u < len_p;
                            xs[u] = kp[u] ? ldg_i32(g.clist + lo_p + e0 + u) : 0;
                        }
                        for (uint32_t o = others; o; o &= o - 1) {
                            const uint32_t mj = (uint32_t)Mj(__ffs(o) - 1);
                            uint64_t hh[4];
                            unsigned long long ww[4];
#pragma unroll
                            for (int u = 0; u < 4; ++u) {
                                hh[u] = edge_hash(mj, (uint32_t)xs[u]);
                                ww[u] = (kp[u] && g.bloom) ? __ldg(g.bloom + (hh[u] & g.bloom_mask)) : ~0ull;
                            }
#pragma unroll
                            for (int u = 0; u < 4; ++u) {
                                if (!kp[u]) continue;
                                const uint64_t mb = bloom_bits(hh[u]);
                                double unused = 0.0;
                                kp[u] = (!g.bloom || (ww[u] & mb) == mb) &&
                                        is_edge_after_filter(g, mj, (uint32_t)xs[u], hh[u], ps.label, unused);
                            }
                        }
#pragma unroll
                        for (int u = 0; u < 4; ++u) {
                            if (!kp[u]) continue;
                            bool matched = false;
                            for (uint32_t mm = ps.dup; mm; mm &= mm - 1) matched |= Mj(__ffs(mm) - 1) == xs[u];
                            if (!matched) keep |= 1ull << (e0 + u);
                        }
                    }
                    cnt = (uint32_t)__popcll(keep);
                    if (cnt > 0) {
                        uint32_t k = (uint32_t)__umul64hi(r, (uint64_t)cnt);
                        const uint32_t lo32 = (uint32_t)keep, c32 = (uint32_t)__popc(lo32);
                        const uint32_t pos = k < c32 ? fns32(lo32, k) : 32u + fns32((uint32_t)(keep >> 32), k - c32);
                        v = ldg_i32(g.clist + lo_p + pos);
                    }
                }
            }
            // ---- long drivers: the whole warp refines one lane's list at a time
            unsigned cm = __ballot_sync(kFull, alive && coop);
            while (cm) {
                const int L = __ffs(cm) - 1;
                cm &= cm - 1;
                const uint32_t Llo = __shfl_sync(kFull, lo_p, L);
                const uint32_t Llen = __shfl_sync(kFull, len_p, L);
                const int Lp = __shfl_sync(kFull, p, L);
                const uint32_t Li = base + (uint32_t)L;  // frontier index of lane L's sample
                const uint32_t others = ps.back & ~(1u << Lp);
                const uint32_t Lr_lo = __shfl_sync(kFull, (uint32_t)r, L);
                const uint32_t Lr_hi = __shfl_sync(kFull, (uint32_t)(r >> 32), L);
                const int32_t Lm0 = __shfl_sync(kFull, m0, L);
                auto LMj = [&](int j) -> int32_t { return FIRST ? Lm0 : A.in.M[(size_t)j * cap + Li]; };
                auto keep_of = [&](int32_t x) -> bool {
                    double unused = 0.0;
                    for (uint32_t o = others; o; o &= o - 1)
                        if (!is_edge<false>(g, (uint32_t)LMj(__ffs(o) - 1), (uint32_t)x, ps.label, unused)) return false;
                    for (uint32_t mm = ps.dup; mm; mm &= mm - 1)
                        if (LMj(__ffs(mm) - 1) == x) return false;
                    return true;
                };
                uint32_t total = 0, my_bal = 0, gcnt = 0;
                const uint32_t G = (((Llen + 31u) >> 5) + 31u) >> 5;  // chunks per lane group
                const uint32_t g_lo = (uint32_t)lane * G;
                int32_t xn = ((uint32_t)lane < Llen) ? ldg_i32(g.clist + Llo + lane) : 0;
                for (uint32_t b0 = 0; b0 < Llen; b0 += 32) {
                    const uint32_t e = b0 + lane;
                    const int32_t x = xn;
                    if (e + 32u < Llen) xn = ldg_i32(g.clist + Llo + e + 32u);
                    const bool kp = e < Llen && keep_of(x);
                    const unsigned bal = __ballot_sync(kFull, kp);
                    if ((b0 >> 5) == (uint32_t)lane) my_bal = bal;
                    if ((b0 >> 5) - g_lo < G) gcnt += __popc(bal);
                    total += __popc(bal);
                }
                int32_t chosen = -1;
                if (total > 0) {
                    const uint64_t Lr = ((uint64_t)Lr_hi << 32) | Lr_lo;
                    const uint32_t k = (uint32_t)__umul64hi(Lr, (uint64_t)total);
                    if (Llen <= 32u * 32u) {
                        const uint32_t pc = __popc(my_bal);
                        uint32_t incl = pc;
#pragma unroll
                        for (int o = 1; o < 32; o <<= 1) {
                            const uint32_t y = __shfl_up_sync(kFull, incl, o);
                            if (lane >= o) incl += y;
                        }
                        const uint32_t excl = incl - pc;
                        const unsigned hm = __ballot_sync(kFull, k >= excl && k < incl);
                        const int c = __ffs(hm) - 1;
                        int32_t val = 0;
                        if (lane == c) val = ldg_i32(g.clist + Llo + (uint32_t)c * 32u + fns32(my_bal, k - excl));
                        chosen = __shfl_sync(kFull, val, c);
                    } else {
                        uint32_t incl = gcnt;
#pragma unroll
                        for (int o = 1; o < 32; o <<= 1) {
                            const uint32_t y = __shfl_up_sync(kFull, incl, o);
                            if (lane >= o) incl += y;
                        }
                        const unsigned hm = __ballot_sync(kFull, k >= incl - gcnt && k < incl);
                        const int gs = __ffs(hm) - 1;
                        uint32_t run = __shfl_sync(kFull, incl - gcnt, gs);
                        for (uint32_t b0 = (uint32_t)gs * G * 32u; b0 < Llen; b0 += 32) {
                            const uint32_t e = b0 + lane;
                            int32_t x = 0;
                            bool kp = false;
                            if (e < Llen) {
                                x = ldg_i32(g.clist + Llo + e);
                                kp = keep_of(x);
                            }
                            const unsigned bal = __ballot_sync(kFull, kp);
                            const uint32_t c = __popc(bal);
                            if (run + c > k) {
                                chosen = __shfl_sync(kFull, x, (int)fns32(bal, k - run));
                                break;
                            }
                            run += c;
                        }
                    }
                }
                if (lane == L) {
                    cnt = total;
                    v = chosen;
                }
            }
        }

        // ---- epilogue: HT weight, terminate or move to the next frontier
        bool survive = false;
        if (alive) {
            W = __dmul_rn(W, (double)cnt);
            const bool complete = cnt > 0 && last;
            survive = cnt > 0 && !last;
            if (complete) {
                n_valid += 1;
                accumulate(s_sum, c_sum, s_sq, c_sq, W);
            }
            if (TRACE && !survive) {
                gsword_sample_record* rec = records + (A.batch_first - A.range_first + slot);
                rec->sample_id = sid;
                rec->valid = complete ? 1 : 0;
                rec->depth_reached = (uint8_t)d;
                rec->sectors = msec;
                rec->weight = W;
#pragma unroll
                for (int j = 0; j < kMaxQV; ++j) {
                    int32_t pj = -1;
                    uint32_t cj = 0;
                    if (j < d) {
                        pj = Mj(j);
                        cj = (FIRST) ? cs0 : A.in.cs[(size_t)j * cap + i];
                    } else if (j == d) {
                        pj = cnt > 0 ? v : -1;
                        cj = cnt;
                    }
                    rec->path[j] = pj;
                    rec->csize[j] = cj;
                }
            }
        }
        const unsigned sm = __ballot_sync(kFull, survive);
        if (sm) {
            uint32_t pos0 = 0;
            if (lane == __ffs(sm) - 1) pos0 = atomicAdd(A.n_out, (uint32_t)__popc(sm));
            pos0 = __shfl_sync(kFull, pos0, __ffs(sm) - 1);
            if (survive) {
                const uint32_t o = pos0 + (uint32_t)__popc(sm & lt_mask);
                A.out.slot[o] = slot;
                A.out.W[o] = W;
                for (int j = 0; j < d; ++j) A.out.M[(size_t)j * cap + o] = Mj(j);
                A.out.M[(size_t)d * cap + o] = v;
                if (TRACE) {
                    for (int j = 0; j < d; ++j) A.out.cs[(size_t)j * cap + o] = FIRST ? cs0 : A.in.cs[(size_t)j * cap + i];
                    A.out.cs[(size_t)d * cap + o] = cnt;
                    A.out.msec[o] = msec;
                }
            }
        }
    }

    // ---- per-CTA partial, added to this CTA's running partial (fixed CTA order at the end)
    double sh = __dadd_rn(s_sum, c_sum), sl = __dsub_rn(c_sum, __dsub_rn(sh, s_sum));
    double qh = __dadd_rn(s_sq, c_sq), ql = __dsub_rn(c_sq, __dsub_rn(qh, s_sq));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double bh = shfl_xor_d(sh, o), bl = shfl_xor_d(sl, o);
        const double ch = shfl_xor_d(qh, o), cl = shfl_xor_d(ql, o);
        dd_add(sh, sl, bh, bl);
        dd_add(qh, ql, ch, cl);
        n_valid += __shfl_xor_sync(kFull, n_valid, o);
        n_done += __shfl_xor_sync(kFull, n_done, o);
    }
    if (lane == 0) warp_part[tid >> 5] = Partial{sh, sl, qh, ql, n_valid, n_done, 0.0, 0.0};
    __syncthreads();
    if (tid == 0 && (FIRST || last)) {
        Partial acc = partials[blockIdx.x];
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
            const Partial& o = warp_part[w];
            dd_add(acc.sum_hi, acc.sum_lo, o.sum_hi, o.sum_lo);
            dd_add(acc.sq_hi, acc.sq_lo, o.sq_hi, o.sq_lo);
            acc.valid += o.valid;
            acc.n += o.n;
        }
        partials[blockIdx.x] = acc;
    }
}

template <bool CG, bool TRACE>
const void* frontier_ptr(bool first, bool multi) {
    if (first) return reinterpret_cast<const void*>(&frontier_kernel<CG, TRACE, true, false>);
    return multi ? reinterpret_cast<const void*>(&frontier_kernel<CG, TRACE, false, true>)
                 : reinterpret_cast<const void*>(&frontier_kernel<CG, TRACE, false, false>);
}

const void* frontier_select(bool cg, bool trace, bool first, bool multi) {
    if (cg) return trace ? frontier_ptr<true, true>(first, multi) : frontier_ptr<true, false>(first, multi);
    return trace ? frontier_ptr<false, true>(first, multi) : frontier_ptr<false, false>(first, multi);
}

}  // namespace

int frontier_grid(bool cg, bool trace, int num_sms) {
    int best = 1 << 30;
    for (int f = 0; f < 2; ++f)
        for (int m = 0; m < 2; ++m) {
            int blocks = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, frontier_select(cg, trace, f, m), 256, 0) !=
                    cudaSuccess ||
                blocks <= 0)
                return 0;
            best = blocks < best ? blocks : best;
        }
    return best * num_sms;
}

cudaError_t launch_frontier(const DeviceGraph& g, const Plan& plan, bool cg, bool trace, const FrontierBufs& a,
                            const FrontierBufs& b, uint32_t cap, uint32_t batch, uint32_t* d_counts, uint64_t first,
                            uint64_t count, uint64_t seed, uint32_t coop_threshold, int grid, Partial* d_partials,
                            gsword_sample_record* d_records, cudaStream_t stream) {
    if (batch == 0 || batch > cap) batch = cap;
    cudaError_t e = cudaMemsetAsync(d_partials, 0, sizeof(Partial) * (size_t)grid, stream);
    if (e != cudaSuccess) return e;
    const int nq = plan.nq;
    for (uint64_t b0 = 0; b0 < count; b0 += batch) {
        const uint32_t nb = (uint32_t)((count - b0) < batch ? (count - b0) : batch);
        if ((e = cudaMemsetAsync(d_counts, 0, sizeof(uint32_t) * kMaxQV, stream)) != cudaSuccess) return e;
        for (int d = 1; d < nq; ++d) {
            FrontierArgs A;
            A.in = (d & 1) ? b : a;   // level d reads the frontier level d-1 wrote
            A.out = (d & 1) ? a : b;
            A.n_in = d_counts + (d - 1);
            A.n_out = d_counts + d;
            A.n_first = nb;
            A.cap = cap;
            A.batch_first = first + b0;
            A.range_first = first;
            A.seed = seed;
            A.d = d;
            A.coop_threshold = coop_threshold;
            void* args[] = {(void*)&g, (void*)&plan, (void*)&A, (void*)&d_partials, (void*)&d_records};
            e = cudaLaunchKernel(frontier_select(cg, trace, d == 1, plan.step[d].nback >= 2), dim3(grid), dim3(256),
                                 args, 0, stream);
            if (e != cudaSuccess) return e;
        }
    }
    return cudaSuccess;
}

}  // namespace gsword
