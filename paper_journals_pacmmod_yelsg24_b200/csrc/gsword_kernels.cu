// gsword_kernels.cu — sm_100a kernels of the gSWORD hot path.
//
// One persistent kernel per method (WanderJoin P:L538 / Alley P:L540) runs the
// Refine-Sample-Validate loop of Alg. 1 for many samples per lane:
//
//   * lanes are refilled from a global u64 sample queue as soon as their sample ends
//     (ballot -> one atomicAdd per warp chunk -> popc rank), so a warp never idles on
//     dead samples (the "validate imbalance" of P:L379, solved without inheritance);
//   * every random choice is k = mulhi64(Philox4x32-10(seed; sid, d), |C_d|), so each
//     sample's path is a pure function of (seed, sample id) (reading A6);
//   * Alley intersections with a long driver list are done by the whole warp over
//     coalesced 32-element chunks with ballot/popc/find-nth (the deterministic
//     replacement of warp streaming), short ones per lane in a 64-bit
//     register bitmask (the "refine array" of Fig. 19);
//   * the HT value Y = prod |C_d| (Eq. 1) is accumulated per lane in
//     compensated fp64, reduced warp -> CTA -> grid in a fixed order.
//
// The graph is read through the read-only path; candidate order is ascending vertex
// id everywhere, so results are bit-identical to the CPU oracle.
#include <cstdint>
#include <type_traits>

#include "device_util.cuh"
#include "internal.h"

namespace gsword {
namespace {

using namespace dev;

#ifndef GSWORD_SELECT_WINDOW
#define GSWORD_SELECT_WINDOW 1  // Alley single-list select: window load + register fixed point
#endif
#ifndef GSWORD_SMEM_ACC
#define GSWORD_SMEM_ACC 1  // Alley: per-lane compensated sums in shared memory
#endif
#ifndef GSWORD_SMEM_QUEUE
#define GSWORD_SMEM_QUEUE 1  // queue chunk and sample/valid counters in shared memory
#endif
#ifndef GSWORD_SMEM_LANE
#define GSWORD_SMEM_LANE 1  // sample id and running weight in shared memory
#endif
// Alley drivers longer than the coop threshold (<= 64) are refined by the whole warp.

// Warp-cooperative Alley refine + sample of one lane's long driver run clist[Llo, Llo+Llen)
// (Fig. 19 AL; reading A5): 32 coalesced elements per round, each lane tests its
// element against the other lists (`others`, the matched vertices of column colL) and the
// matched same-label vertices, `ballot` -> the chunk's survivor mask, held in lane c for chunk c
// (lists <= 1024) -> warp prefix sum of popcounts -> find-nth of the k-th survivor; longer lists
// keep per-lane group counts (G chunks per group) and re-test only the group holding the k-th.
// Deterministic replacement of the paper's reservoir warp streaming.  Every lane calls it;
// total (|C_d|) and chosen (the drawn vertex, -1 if none) are returned to every lane.
template <bool COUNT>
__device__ __forceinline__ void coop_refine(const DeviceGraph& g, const uint32_t* Ms, int T, int lane, int colL,
                                            uint32_t Llo, uint32_t Llen, uint32_t others, const PlanStep& Lps,
                                            uint32_t Lsig, uint64_t r_lane, int L, double& sectors,
                                            uint32_t& total_out, int32_t& chosen_out) {
    uint32_t total = 0, my_bal = 0;
    // lists longer than 32 chunks: lane g also counts the survivors of chunk group
    // g (G consecutive chunks), so the draw re-tests one group, not the whole prefix
    const uint32_t G = (((Llen + 31u) >> 5) + 31u) >> 5;  // chunks per group
    const uint32_t g_lo = (uint32_t)lane * G;
    uint32_t gcnt = 0;
    // the next chunk's driver elements are loaded while this chunk is tested
    int32_t xn = ((uint32_t)lane < Llen) ? ldg_i32(g.clist + Llo + lane) : 0;
    for (uint32_t base = 0; base < Llen; base += 32) {
        const uint32_t i = base + lane;
        bool keep = i < Llen;
        const int32_t x = xn;
        if (i + 32u < Llen) xn = ldg_i32(g.clist + Llo + i + 32u);
        if (keep) {
            keep = member_all<COUNT>(g, Ms, T, colL, others, Lps.label, x, sectors) &&
                   not_matched_sig(Ms, T, colL, Lps.dup, Lsig, x);
        }
        const unsigned bal = __ballot_sync(kFull, keep);
        if ((base >> 5) == (uint32_t)lane) my_bal = bal;
        if ((base >> 5) - g_lo < G) gcnt += __popc(bal);
        total += __popc(bal);
    }
    int32_t chosen = -1;
    if (total > 0) {
        // lane L's random word, fetched only now (not live across the count loop)
        const uint32_t Lr_lo = __shfl_sync(kFull, (uint32_t)r_lane, L);
        const uint32_t Lr_hi = __shfl_sync(kFull, (uint32_t)(r_lane >> 32), L);
        const uint64_t Lr = ((uint64_t)Lr_hi << 32) | Lr_lo;
        const uint32_t k = (uint32_t)__umul64hi(Lr, (uint64_t)total);
        if (Llen <= 32u * 32u) {
            // lane c holds the ballot of chunk c: warp scan of popcounts
            const uint32_t pc = __popc(my_bal);
            uint32_t incl = pc;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            const uint32_t excl = incl - pc;
            const bool here = (k >= excl) && (k < incl);
            const unsigned hm = __ballot_sync(kFull, here);
            const int c = __ffs(hm) - 1;
            int32_t val = 0;
            if (lane == c) val = ldg_i32(g.clist + Llo + (uint32_t)c * 32u + fns32(my_bal, k - excl));
            chosen = __shfl_sync(kFull, val, c);
        } else {
            // the group holding the k-th survivor (warp scan of the group counts),
            // then its chunks re-tested in order
            uint32_t incl = gcnt;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(kFull, incl, o);
                if (lane >= o) incl += y;
            }
            const unsigned hm = __ballot_sync(kFull, (k >= incl - gcnt) && (k < incl));
            const int gs = __ffs(hm) - 1;
            uint32_t run = __shfl_sync(kFull, incl - gcnt, gs);
            const uint32_t b0 = (uint32_t)gs * G * 32u;
            for (uint32_t base = b0; base < Llen; base += 32) {
                const uint32_t i = base + lane;
                bool keep = i < Llen;
                int32_t x = 0;
                if (keep) {
                    x = ldg_i32(g.clist + Llo + i);
                    keep = member_all<COUNT>(g, Ms, T, colL, others, Lps.label, x, sectors) &&
                           not_matched_sig(Ms, T, colL, Lps.dup, Lsig, x);
                }
                const unsigned bal = __ballot_sync(kFull, keep);
                const uint32_t c = __popc(bal);
                if (run + c > k) {
                    chosen = __shfl_sync(kFull, x, (int)fns32(bal, k - run));
                    break;
                }
                run += c;
            }
        }
    }
    total_out = total;
    chosen_out = chosen;
}

// A10: the CTA's partial in a fixed order.  Each lane's Neumaier pair becomes a double-double,
// a warp butterfly adds the lanes, lane 0 of every warp stores the warp's partial in
// warp_part[warp], and thread 0 adds the warps in warp order into partials[blockIdx.x].
// Every thread of the CTA calls it (it synchronises the CTA).
__device__ __forceinline__ void write_cta_partial(Partial* warp_part, Partial* __restrict__ partials, double s_sum,
                                                  double c_sum, double s_sq, double c_sq, unsigned long long valid,
                                                  unsigned long long n, double sectors, double model) {
    const int tid = threadIdx.x, lane = tid & 31;
    double sh = __dadd_rn(s_sum, c_sum), sl = __dsub_rn(c_sum, __dsub_rn(sh, s_sum));
    double qh = __dadd_rn(s_sq, c_sq), ql = __dsub_rn(c_sq, __dsub_rn(qh, s_sq));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double bh = shfl_xor_d(sh, o), bl = shfl_xor_d(sl, o);
        const double ch = shfl_xor_d(qh, o), cl = shfl_xor_d(ql, o);
        dd_add(sh, sl, bh, bl);
        dd_add(qh, ql, ch, cl);
        valid += __shfl_xor_sync(kFull, valid, o);
        n += __shfl_xor_sync(kFull, n, o);
        sectors += shfl_xor_d(sectors, o);
        model += shfl_xor_d(model, o);
    }
    if (lane == 0) warp_part[tid >> 5] = Partial{sh, sl, qh, ql, valid, n, sectors, model};
    __syncthreads();
    if (tid == 0) {
        Partial acc = warp_part[0];
        for (int w = 1; w < (int)(blockDim.x >> 5); ++w) {
            const Partial& o = warp_part[w];
            dd_add(acc.sum_hi, acc.sum_lo, o.sum_hi, o.sum_lo);
            dd_add(acc.sq_hi, acc.sq_lo, o.sq_hi, o.sq_lo);
            acc.valid += o.valid;
            acc.n += o.n;
            acc.sectors += o.sectors;
            acc.model += o.model;
        }
        partials[blockIdx.x] = acc;
    }
}

// Alley single-list select (|B(d)| = 1): the k-th (0-based) element of the ascending run
// clist[lo, ...) that is not one of the matched vertices in the position mask X (all of which
// lie in the run): the smallest idx with idx = k + #{x in X : x <= run[idx]}.  With at most two
// excluded vertices idx lies in [k, k + |X|]: that window is loaded at once and the fixed point
// found in registers (one memory round trip instead of up to |X| + 1 dependent ones).
// Ms_lane = this lane's column of the matched vertices (row stride T).
__device__ __forceinline__ int32_t select_excluding(const DeviceGraph& g, const uint32_t* Ms_lane, int T, uint32_t lo,
                                                    uint32_t k, uint32_t X) {
    const int nx = __popc(X);
#if GSWORD_SELECT_WINDOW
    if (nx <= 2) {
        const int32_t* wb = g.clist + lo + k;
        const int32_t w0 = ldg_i32(wb);
        const int32_t w1 = nx >= 1 ? ldg_i32(wb + 1) : 0;
        const int32_t w2 = nx >= 2 ? ldg_i32(wb + 2) : 0;
        const int32_t x0 = nx >= 1 ? (int32_t)Ms_lane[(__ffs(X) - 1) * T] : INT32_MAX;
        const int32_t x1 = nx >= 2 ? (int32_t)Ms_lane[(31 - __clz(X)) * T] : INT32_MAX;
        uint32_t i = 0;
#pragma unroll
        for (int it = 0; it < 2; ++it) {
            const int32_t wi = i == 0 ? w0 : (i == 1 ? w1 : w2);
            i = (uint32_t)(x0 <= wi) + (uint32_t)(x1 <= wi);
        }
        return i == 0 ? w0 : (i == 1 ? w1 : w2);
    }
#endif
    int32_t v = 0;
    for (uint32_t idx = k;;) {
        v = ldg_i32(g.clist + lo + idx);
        uint32_t c = 0, xm = X;
        while (xm) {
            const int j = __ffs(xm) - 1;
            xm &= xm - 1;
            c += ((int32_t)Ms_lane[j * T] <= v) ? 1u : 0u;
        }
        if (idx == k + c) break;
        idx = k + c;
    }
    return v;
}

// Alley short-driver refine (|B(d)| >= 2, |S_p| <= the cooperative threshold, <= 128): the
// refine mask over clist[lo, lo + len) is "not removed by a pooled membership test" (pool rows
// 1..4 of this lane, bit set = removed) and "not a matched same-label vertex" (injectivity, dup
// mask, signature sig); returns |C_d| and writes the k-th survivor (k = mulhi64(r, |C_d|)) to *v.
__device__ __forceinline__ uint32_t refine_mask_select(const DeviceGraph& g, const uint32_t* Ms_lane,
                                                       const uint32_t* pool_lane, int T, uint32_t lo, uint32_t len,
                                                       uint32_t dup, uint32_t sig, uint64_t r, int32_t* v) {
    uint32_t keep[4];
    uint32_t cnt = 0;
#pragma unroll
    for (int w = 0; w < 4; ++w) {
        const uint32_t n_w = (len > 32u * w) ? min(len - 32u * w, 32u) : 0u;
        uint32_t m = (n_w == 32u) ? 0xFFFFFFFFu : ((1u << n_w) - 1u);
        if (n_w) m &= ~pool_lane[(1 + w) * T];
        uint32_t mm = dup ? m : 0u;
        while (mm) {
            const int i = __ffs(mm) - 1;
            mm &= mm - 1;
            if (!not_matched_sig(Ms_lane, T, 0, dup, sig, ldg_i32(g.clist + lo + 32u * w + i))) m &= ~(1u << i);
        }
        keep[w] = m;
        cnt += __popc(m);
    }
    if (cnt > 0) {
        uint32_t k = (uint32_t)__umul64hi(r, (uint64_t)cnt);
        uint32_t pos = 0;
#pragma unroll
        for (int w = 0; w < 4; ++w) {
            const uint32_t c = __popc(keep[w]);
            if (k < c && pos == 0u) pos = 32u * w + fns32(keep[w], k) + 1u;  // +1: found marker
            if (pos == 0u) k -= c;
        }
        *v = ldg_i32(g.clist + lo + pos - 1u);
    }
    return cnt;
}

#ifndef GSWORD_WJ_MIN_BLOCKS
#define GSWORD_WJ_MIN_BLOCKS 6  // 42 registers: 48 warps per SM (measured best)
#endif
#ifndef GSWORD_AL_MIN_BLOCKS
#define GSWORD_AL_MIN_BLOCKS 5  // 51 registers: 40 warps per SM (measured best)
#endif

// Launch bounds per occupancy variant: 0 = the measured default, 1 = one CTA/SM less
// (more registers, fewer spills: better where samples die early, e.g. C3 Alley), 2 = one
// more.  The autotune in gsword_load_query picks per method and query.
__host__ __device__ constexpr int kOccBlocks(int method, int occ) {
    return (method == GSWORD_WJ ? GSWORD_WJ_MIN_BLOCKS : GSWORD_AL_MIN_BLOCKS) + (occ == 1 ? -1 : occ == 2 ? 1 : 0);
}

// SYNC: false = the default refill scheduler only (sched 0, the scheduling-mode logic
// compiled out); true = any GSWORD_OPT_SCHEDULE (NEXT-3 comparison modes)
// TREE: every position d >= 1 has exactly one backward neighbour (a spanning-tree query
// order, e.g. paths and stars): WanderJoin has no IsEdge validation and Alley only the
// single-list refine, so the multi-list code is compiled out (estimate kernels only).
// LOCK: refill threshold 32 (a warp takes new samples only when all 32 lanes are free), so
// every live lane of a warp is at the same depth: Alley's exclusion tests are the same set for
// every lane and each lane runs its own, two in flight, without the task pool (estimate only).
template <int METHOD, int MODE, bool CG, bool SYNC, int OCC = 0, bool TREE = false, bool LOCK = false>
__global__ void __launch_bounds__(256, kOccBlocks(METHOD, OCC))
    sample_kernel(const DeviceGraph g, const Plan plan_in, const uint64_t first,
                                                     const uint64_t count, const uint64_t seed, const int chunk,
                                                     const uint32_t coop_threshold, const int sched_arg,
                                                     const uint32_t refill_min,
                                                     unsigned long long* __restrict__ queue,
                                                     Partial* __restrict__ partials,
                                                     gsword_sample_record* __restrict__ records,
                                                     unsigned long long* __restrict__ phase_out) {
    __shared__ PlanStep plan_s[kMaxQV];
    __shared__ uint32_t qadj_s[kMaxQV];
    __shared__ uint8_t eidx_s[kMaxQV][kMaxQV];
    __shared__ uint8_t uq_s[kMaxQV];
    __shared__ uint32_t pdup_s[kMaxQV];  // variant A5: post-draw DupCheck positions
    __shared__ Partial warp_part[8];
    // dynamic shared memory, rows of kSampleLanes words (sized on the host by the query and
    // the coop threshold, so the rest of the SM's L1/shared array stays L1):
    //   Ms[j * T + tid]          = M[j] of this lane, j < n_q
    //   pool_s[w * T + tid]      (Alley) w = 0: task-pool results "matched vertex j lies in
    //                            S_p" (pool 1); w = 1..ceil(coop/32): refine-mask removals
    extern __shared__ uint32_t Ms[];

    const int tid = threadIdx.x;
    // row stride of Ms: a compile-time constant (no register) where multi-list steps raise the
    // register pressure; tree orders keep blockDim.x (measured 2 % faster there)
    const int T = TREE ? (int)blockDim.x : kSampleLanes;
    const int lane = tid & 31;
    const int wbase = tid - lane;
    const unsigned lt_mask = (1u << lane) - 1u;
    if (tid < kMaxQV) {
        plan_s[tid] = plan_in.step[tid];
        qadj_s[tid] = plan_in.qadj[tid];
        uq_s[tid] = plan_in.uq[tid];
        pdup_s[tid] = plan_in.pdup[tid];
    }
    for (int i = tid; i < kMaxQV * kMaxQV; i += blockDim.x) eidx_s[i / kMaxQV][i % kMaxQV] = plan_in.eidx[i / kMaxQV][i % kMaxQV];
    __syncthreads();

    const int nq = plan_in.nq;
    uint32_t* const pool_s = Ms + (size_t)nq * (size_t)T;
    const uint32_t mask_words = (coop_threshold + 31u) >> 5;  // refine-mask rows (<= 4)
    const int sched = SYNC ? sched_arg : 0;
    // some position has |B(d)| >= 2 (Alley refine kinds 2/3 can occur): a launch constant
    const bool multi_back = !TREE && plan_in.multi_back != 0;

    // lane state
    bool has = false;
    // signature of M[0..d-1] (sig_bit); Alley keeps it in shared memory with the sample id
    __shared__ uint32_t msig_s[(GSWORD_SMEM_LANE && METHOD == GSWORD_ALLEY) ? 256 : 1];
    uint32_t msig_r = 0u;
    uint32_t& msig = (GSWORD_SMEM_LANE && METHOD == GSWORD_ALLEY) ? msig_s[tid] : msig_r;
    msig = 0u;
    // GSWORD_SMEM_LANE (Alley): the sample id and the running weight W live in shared memory (read
    // once per step), 4 registers fewer in the sampling loop
    constexpr bool kSmemLane = GSWORD_SMEM_LANE && METHOD == GSWORD_ALLEY;
    __shared__ uint64_t sid_s[kSmemLane ? 256 : 1];
    __shared__ double W_s[kSmemLane ? 256 : 1];
    uint64_t sid_r = 0;
    double W_r = 0.0;
    uint64_t& sid = kSmemLane ? sid_s[tid] : sid_r;
    double& W = kSmemLane ? W_s[tid] : W_r;
    sid = 0;
    int d = 0;
    W = 0.0;
    // lane accumulators
    double s_sum = 0.0, c_sum = 0.0, s_sq = 0.0, c_sq = 0.0;
    unsigned long long n_valid = 0, n_done = 0;
    // Alley (GSWORD_SMEM_ACC): the compensated sums live in shared memory (touched only when
    // a sample completes), freeing 8 registers for the refine paths
    constexpr bool kSmemAcc = GSWORD_SMEM_ACC && METHOD == GSWORD_ALLEY;
    constexpr bool kSmemQueue = GSWORD_SMEM_QUEUE != 0;
    __shared__ double acc_s[kSmemAcc ? 4 : 1][256];
    if (kSmemAcc)
#pragma unroll
        for (int i = 0; i < 4; ++i) acc_s[i][tid] = 0.0;
    auto accumulate = [&](double y) {
        if (kSmemAcc) {
            double a = acc_s[0][tid], b = acc_s[1][tid], c = acc_s[2][tid], e = acc_s[3][tid];
            nsum(a, b, y);
            nsum(c, e, __dmul_rn(y, y));
            acc_s[0][tid] = a;
            acc_s[1][tid] = b;
            acc_s[2][tid] = c;
            acc_s[3][tid] = e;
        } else {
            nsum(s_sum, c_sum, y);
            nsum(s_sq, c_sq, __dmul_rn(y, y));
        }
    };
    double sectors = 0.0;  // counting build: sectors the implementation touches
    // trace / counting builds: algorithmic sectors of reading A26 (this lane's sample, and
    // the lane's total over its finished samples)
    uint32_t msec = 0u;
    double msum = 0.0;

    // warp chunk of the queue (warp-uniform)
    uint64_t q_next = 0, q_end = 0;
    bool exhausted = false;
    // GSWORD_SMEM_QUEUE: the warp's queue chunk, its sample count and the lanes' valid counts
    // live in shared memory (touched at refill / completion only): 8 registers fewer in the
    // sampling loop
    __shared__ unsigned long long wq_s[kSmemQueue ? 8 : 1][3];  // q_next, q_end, n of the warp
    __shared__ uint32_t nv_s[kSmemQueue ? 256 : 1];
    if (kSmemQueue) {
        if (lane == 0) wq_s[tid >> 5][0] = wq_s[tid >> 5][1] = wq_s[tid >> 5][2] = 0ull;
        nv_s[tid] = 0u;
        __syncwarp();
    }
    // scheduling (NEXT-3 comparison modes): 0 refill free lanes every round; 1 sample
    // synchronisation (a warp refills only when all 32 lanes are free); 2 sample
    // synchronisation + sample inheritance (Alg. 2, reading A24)
    bool member = false;   // the lane holds a sample id of the warp's current group
    double g_acc = 0.0;    // sched 2: this lane's complete-instance weights in the group
    bool group_open = false;

    // count build only: warp-level cycle split of the loop (lane 0 of every warp)
    unsigned long long ph[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    long long ph_t = clock64();
    int ph_cur = 0;
    auto mark = [&](int next) {
        if (MODE == kModeCount) {
            __syncwarp();
            const long long now = clock64();
            ph[ph_cur] += (unsigned long long)(now - ph_t);
            ph_t = now;
            ph_cur = next;
        }
    };

    while (true) {
        mark(0);
        // ---------------- A1: refill free lanes from the sample queue ----------------
        unsigned need = __ballot_sync(kFull, !has);
        if (sched == 2 && need == kFull && group_open) {
            // group finished: its total is one independent unit of the estimate
            double gsum = g_acc;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) gsum = __dadd_rn(gsum, shfl_xor_d(gsum, o));
            if (lane == 0) accumulate(gsum);
            g_acc = 0.0;
            group_open = false;
        }
        if (sched != 0 && need != kFull) need = 0u;  // sample synchronisation: wait for the group
        // refill only when at least `refill_min` lanes are free (1 = every round, 32 = sample sync)
        if (sched == 0 && (uint32_t)__popc(need) < refill_min) need = 0u;
        if (need == kFull) member = false;
        while (need && !exhausted) {
            if (kSmemQueue) {
                q_next = wq_s[tid >> 5][0];
                q_end = wq_s[tid >> 5][1];
            }
            if (q_next == q_end) {
                unsigned long long base = 0;
                if (lane == 0) base = atomicAdd(queue, (unsigned long long)chunk);
                base = __shfl_sync(kFull, base, 0);
                if (base >= count) {
                    exhausted = true;
                    break;
                }
                q_next = base;
                q_end = ((uint64_t)base + (uint64_t)chunk < count) ? (uint64_t)base + (uint64_t)chunk : count;
            }
            const uint32_t avail = (q_end - q_next) < 32 ? (uint32_t)(q_end - q_next) : 32u;
            const uint32_t rank = __popc(need & lt_mask);
            if (!has && rank < avail) {
                has = true;
                member = true;
                if (!kSmemQueue) n_done += 1;  // every sample id counts in n (reading A8)
                sid = first + q_next + rank;
                d = 0;
                W = 1.0;
                msig = 0u;
                msec = 0u;
                if (MODE == kModeTrace) {
                    gsword_sample_record* rec = records + (sid - first);
                    rec->sample_id = sid;
#pragma unroll
                    for (int i = 0; i < kMaxQV; ++i) {
                        rec->path[i] = -1;
                        rec->csize[i] = 0;
                    }
                }
            }
            const uint32_t took = min((uint32_t)__popc(need), avail);
            q_next += took;
            if (kSmemQueue) {
                __syncwarp();
                if (lane == 0) {
                    wq_s[tid >> 5][0] = q_next;
                    wq_s[tid >> 5][1] = q_end;
                    wq_s[tid >> 5][2] += took;  // every sample id counts in n (reading A8)
                }
                __syncwarp();
            }
            need = __ballot_sync(kFull, !has);
            group_open = true;
            if (sched != 0) break;  // one group of <= 32 consecutive ids at a time
        }
        if (!__any_sync(kFull, has)) break;
        __syncwarp();

        mark(1);
        // ---------------- per-lane prologue: draw + GetMinCandidate -----------------
        PlanStep ps = {0, 0u, 0u, 0};
        uint64_t r = 0;
        uint32_t lo_p = 0, len_p = 0;
        int p = -1;
        uint32_t seg_a = 0, seg_b = 0;
        bool deferred = false;
        if (has) {
            ps = plan_s[d];
            r = philox_r(seed, sid, (uint32_t)d);
            if (d == 0) {
                lo_p = plan_in.seed_lo;
                len_p = plan_in.seed_len;
                if (MODE == kModeCount) sectors += plan_in.seed_identity ? 0.0 : 1.0;
                // A26: the drawn seed is read from the stored list unless C(phi[0]) is all of V
                if (MODE != kModeEstimate && len_p != 0u && (int64_t)len_p != g.n) msec += 1u;
            } else if (METHOD == GSWORD_ALLEY && (TREE || ps.nback == 1)) {
                // one backward neighbour: p is fixed by the plan; the segment load is left
                // in flight and consumed after the exclusion tests (which need only M)
                p = __ffs(ps.back) - 1;
                local_run<CG>(g, eidx_s[d][p], Ms[p * T + tid], ps.label, &seg_a, &seg_b);
                deferred = true;
                if (MODE == kModeCount) sectors += 1.0;
                if (MODE != kModeEstimate) msec += 1u;  // A26: offsets of S_p
            } else if (TREE) {
                p = __ffs(ps.back) - 1;
                uint32_t a, b;
                local_run<CG>(g, eidx_s[d][p], Ms[p * T + tid], ps.label, &a, &b);
                lo_p = a;
                len_p = b - a;
            } else {
                // GetMinCandidate (Alg. 1 l.8): the smallest N_l(M[j]) over j in B(d)
                // (variant A3: WanderJoin takes the first backward position's list)
                uint32_t bm = ps.back;
                if (METHOD == GSWORD_WJ && plan_in.wj_parent_first) bm &= 0u - bm;
                len_p = 0xFFFFFFFFu;
                while (bm) {
                    const int j = __ffs(bm) - 1;
                    bm &= bm - 1;
                    uint32_t a, b;
                    local_run<CG>(g, eidx_s[d][j], Ms[j * T + tid], ps.label, &a, &b);
                    if (b - a < len_p) {
                        len_p = b - a;
                        lo_p = a;
                        p = j;
                    }
                }
                if (MODE == kModeCount) sectors += (METHOD == GSWORD_WJ && plan_in.wj_parent_first) ? 1.0 : (double)ps.nback;
                // A26: the offsets of every list GetMinCandidate compares
                if (MODE != kModeEstimate)
                    msec += (METHOD == GSWORD_WJ && plan_in.wj_parent_first) ? 1u : (uint32_t)ps.nback;
            }
        }

        mark(2);
        uint32_t cnt = 0;     // |C_d|
        int32_t v = -1;       // drawn vertex
        bool reject = false;  // WJ Validate failure
        if (METHOD == GSWORD_WJ) {
            if (has) {
                cnt = len_p;
                if (cnt > 0) {
                    const uint64_t k = __umul64hi(r, (uint64_t)cnt);
                    if (d == 0) {
                        v = plan_in.seed_identity ? (int32_t)(lo_p + k) : ldg_i32(g.bucket + lo_p + k);
                    } else {
                        v = ldg_i32(g.clist + lo_p + k);
                        if (MODE == kModeCount) sectors += 1.0;
                        if (MODE != kModeEstimate) msec += 1u;  // A26: the drawn vertex
                        // Validate: DupCheck, then IsEdge for the other matched neighbours
                        // (one edge-index question each, ascending position, first "no" ends it)
                        reject = !not_matched_sig(Ms + tid, T, 0, ps.dup, msig, v);
                        uint32_t bm = TREE ? 0u : ps.back & ~(1u << p);
                        while (bm && !reject) {
                            const int j = __ffs(bm) - 1;
                            bm &= bm - 1;
                            if (MODE != kModeEstimate) msec += 1u;  // A26: one IsEdge question
                            reject = !is_edge<MODE == kModeCount>(g, Ms[j * T + tid], (uint32_t)v, ps.label, sectors);
                        }
                    }
                }
            }
        } else {
            // ---------------- Alley Refine + Sample (Fig. 19 AL) ----------------
            // kind 1: |B(d)| = 1 -> C_d = S_p minus matched same-label vertices in S_p
            // kind 2: |B(d)| >= 2, |S_p| <= threshold -> refine bitmask over S_p, membership
            //         tests pooled across the warp
            // kind 3: |B(d)| >= 2, |S_p| > threshold -> warp-cooperative chunks (below)
            //
            // Warp task pool: the edge tests of all 32 lanes are dealt out round-robin (an
            // exclusive scan of per-lane counts, owner found by shuffle bisection), so every
            // lane is busy whichever lanes generated the work (the refine imbalance).
            // test(o, k) runs task k of owner lane o; every lane calls it (it shuffles).
            // test(o, k, valid, a, b, tgt, lb, soe) names the edge {a, b} of task k of owner
            // lane o (label lb = L(b)), the result bit tgt = (word << 5) | bit in pool_s, and
            // whether the bit is set on an edge (soe) or on a non-edge.  Every lane calls it
            // (it shuffles).
            auto pool = [&](uint32_t ntask, auto&& test) {
                if (!__any_sync(kFull, ntask != 0u)) return;
                uint32_t incl = ntask;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(kFull, incl, o);
                    if (lane >= o) incl += y;
                }
                const uint32_t total = __shfl_sync(kFull, incl, 31);
                const uint32_t excl = incl - ntask;
                for (uint32_t base = 0; base < total; base += 32) {
                    const uint32_t t = base + (uint32_t)lane;
                    const uint32_t tt = t < total ? t : total - 1;
                    int o = 0;  // owner lane: number of lanes whose inclusive count <= tt
#pragma unroll
                    for (int s2 = 16; s2 >= 1; s2 >>= 1) {
                        const uint32_t y = __shfl_sync(kFull, incl, o + s2 - 1);
                        if (y <= tt) o += s2;
                    }
                    uint32_t ea = 0, eb = 0, tg = 0;
                    int32_t lb = 0;
                    bool soe = false;
                    const bool valid = t < total;
                    test(o, tt - __shfl_sync(kFull, excl, o), valid, ea, eb, tg, lb, soe);
                    if (valid && is_edge<MODE == kModeCount>(g, ea, eb, lb, sectors) == soe)
                        atomicOr(pool_s + (tg >> 5), 1u << (tg & 31u));
                }
                __syncwarp();
            };
            // task of a kind-1 owner: exclusion test {M[p], M[j]} for the k-th j of `omask`,
            // result bit j of pool_s[0] on an edge
            auto excl_task = [&](int ocol, uint32_t omask, int op, uint32_t k, uint32_t& ea, uint32_t& eb,
                                 uint32_t& tg, bool& soe) {
                const int j = fns_small(omask, k);
                ea = Ms[op * T + ocol];
                eb = Ms[j * T + ocol];
                tg = ((uint32_t)ocol << 5) | (uint32_t)j;  // pool_s row 0, lane ocol, bit j
                soe = true;
            };
            // task of a kind-2 owner: is S_p[i] (label l_d) in N_l(M[j]), i.e. is {M[j], S_p[i]}
            // an edge?  task k = (list nth of `omask`, element i); result bit i of
            // pool_s[1 + i/32] on a non-edge
            auto memb_task = [&](int ocol, uint32_t omask, uint32_t olo, uint32_t olen, uint32_t k, uint32_t& ea,
                                 uint32_t& eb, uint32_t& tg, bool& soe) {
                uint32_t nth = 0u, i = k;
                if (omask & (omask - 1u)) {  // one other list is the common case
                    nth = k / olen;
                    i = k - nth * olen;
                }
                const int j = fns_small(omask, nth);
                ea = Ms[j * T + ocol];
                eb = (uint32_t)ldg_i32(g.clist + olo + i);
                tg = ((uint32_t)((1u + (i >> 5)) * (uint32_t)T + (uint32_t)ocol) << 5) | (i & 31u);
                soe = false;
            };
            int kind = 0;
            uint32_t unk = 0, known = 0, others = 0;
            uint32_t q_model = 0;  // A26: exclusion questions of a kind-1 step (trace / count)
#pragma unroll
            for (int w = 0; w < 5; ++w)
                if (METHOD == GSWORD_ALLEY && (uint32_t)w <= mask_words) pool_s[w * T + tid] = 0u;
            if (has && deferred) {
                // M[j] (same label) with (phi[j], phi[p]) a query edge lies in S_p by the
                // Alley invariant (every drawn prefix is a partial instance); M[p] never does
                // (no self loops); the rest need an edge test {M[p], M[j]}.
                const uint32_t qa = qadj_s[p];
                kind = 1;
                uint32_t cdup = ps.dup & ~(1u << p);
                // A26: one question per same-label matched M[j], j != p, except (label-only
                // lists) those known to lie in S_p
                if (MODE != kModeEstimate) q_model = (uint32_t)__popc(CG ? cdup : (cdup & ~qa));
                if (CG) {
                    // under a filter S_p lies inside C(phi[d]): matched vertices outside it
                    // cannot be in S_p
                    uint32_t m = cdup;
                    const int ud = uq_s[d];
                    while (m) {
                        const int j = __ffs(m) - 1;
                        m &= m - 1;
                        if (!in_cand(g, ud, Ms[j * T + tid])) cdup &= ~(1u << j);
                    }
                }
                known = cdup & qa;
                unk = cdup & ~qa;
                if (LOCK) {
                    // depth-synchronous warp: this lane's own exclusion tests, two in flight
                    // (the filter words of both, then the buckets of the "maybe"s), while the
                    // segment load of S_p is still in flight
                    const uint32_t a = Ms[p * T + tid];
                    uint32_t m = unk;
                    double unused = 0.0;
                    while (m) {
                        const int j0 = __ffs(m) - 1;
                        m &= m - 1;
                        const int j1 = m ? __ffs(m) - 1 : -1;
                        if (m) m &= m - 1;
                        const uint32_t x0 = Ms[j0 * T + tid], x1 = j1 >= 0 ? Ms[j1 * T + tid] : 0u;
                        const bool f0 = bloom_maybe<false>(g, a, x0, unused);
                        const bool f1 = j1 >= 0 && bloom_maybe<false>(g, a, x1, unused);
                        if (f0 && is_edge_exact<false>(g, a, x0, ps.label, unused)) known |= 1u << j0;
                        if (f1 && is_edge_exact<false>(g, a, x1, ps.label, unused)) known |= 1u << j1;
                    }
                    unk = 0u;
                }
            }
            __syncwarp();
            // kind 2 is known before the pool for lanes that waited on GetMinCandidate, so the
            // exclusion tests (kind 1) and the membership tests (kind 2) share one pool: one
            // pass of rounds instead of two
            if (!TREE && has && !deferred && d > 0 && len_p > 0 && len_p <= coop_threshold) {
                kind = 2;
                others = ps.back & ~(1u << p);
                if (MODE == kModeCount) sectors += (double)scan_sectors(len_p);
            }
            if (multi_back) {
                const uint32_t ntask = kind == 1 ? (uint32_t)__popc(unk) : kind == 2 ? len_p * (uint32_t)__popc(others) : 0u;
                // owner state in three words: kind | task mask (positions < 16), p or lo_p, len_p
                const uint32_t kmask = ((uint32_t)kind << 16) | (kind == 1 ? unk : others);
                const uint32_t pl = kind == 1 ? (uint32_t)p : lo_p;
                pool(ntask, [&](int o, uint32_t k, bool valid, uint32_t& ea, uint32_t& eb, uint32_t& tg, int32_t& lb,
                                bool& soe) {
                    const uint32_t okm = __shfl_sync(kFull, kmask, o);
                    const uint32_t opl = __shfl_sync(kFull, pl, o);
                    const uint32_t olen = __shfl_sync(kFull, len_p, o);
                    lb = __shfl_sync(kFull, ps.label, o);
                    if (valid) {
                        if ((okm >> 16) == 1u)
                            excl_task(wbase + o, okm & 0xFFFFu, (int)opl, k, ea, eb, tg, soe);
                        else
                            memb_task(wbase + o, okm & 0xFFFFu, opl, olen, k, ea, eb, tg, soe);
                    }
                });
            } else {
                // no position has two backward neighbours: exclusion tests only
                pool((kind == 1) ? (uint32_t)__popc(unk) : 0u,
                     [&](int o, uint32_t k, bool valid, uint32_t& ea, uint32_t& eb, uint32_t& tg, int32_t& lb, bool& soe) {
                    const uint32_t omask = __shfl_sync(kFull, unk, o);
                    const int op = __shfl_sync(kFull, p, o);
                    lb = __shfl_sync(kFull, ps.label, o);
                    if (valid) excl_task(wbase + o, omask, op, k, ea, eb, tg, soe);
                });
            }
            if (deferred) {
                lo_p = seg_a;
                len_p = seg_b - seg_a;
            }
            if (has) {
                if (d == 0) {
                    cnt = len_p;
                    if (cnt > 0) {
                        const uint64_t k = __umul64hi(r, (uint64_t)cnt);
                        v = plan_in.seed_identity ? (int32_t)(lo_p + k) : ldg_i32(g.bucket + lo_p + k);
                    }
                } else if (len_p == 0) {
                    kind = 0;
                } else if (!TREE && !deferred) {
                    if (len_p > coop_threshold) kind = 3;
                }
            }
            mark(3);
            mark(4);
            if (MODE != kModeEstimate && has && d > 0) {
                if (kind == 1) msec += q_model + ((len_p > (uint32_t)__popc(known | pool_s[tid])) ? 1u : 0u);
                if (!TREE && (kind == 2 || kind == 3))
                    msec += model_refine_sectors(g, Ms, T, tid, lo_p, len_p, ps.back & ~(1u << p), ps.dup, ps.label);
            }
            if (kind == 1) {
                const uint32_t in_sp = LOCK ? known : (known | pool_s[tid]);  // matched vertices inside S_p
                cnt = len_p - __popc(in_sp);
                if (cnt > 0) {
                    v = select_excluding(g, Ms + tid, T, lo_p, (uint32_t)__umul64hi(r, (uint64_t)cnt), in_sp);
                    if (MODE == kModeCount) sectors += 1.0;
                }
            } else if (!TREE && kind == 2) {
                cnt = refine_mask_select(g, Ms + tid, pool_s + tid, T, lo_p, len_p, ps.dup & ~(1u << p), msig, r, &v);
            }
            const bool coop = !TREE && (kind == 3);
            mark(5);

            // ---------------- warp-cooperative refine for long drivers ----------------
            unsigned cm = TREE ? 0u : __ballot_sync(kFull, coop);
            while (!TREE && cm) {
                const int L = __ffs(cm) - 1;
                cm &= cm - 1;
                const uint32_t Llo = __shfl_sync(kFull, lo_p, L);
                const uint32_t Llen = __shfl_sync(kFull, len_p, L);
                const int Lp = __shfl_sync(kFull, p, L);
                const int Ld = __shfl_sync(kFull, d, L);
                const PlanStep Lps = plan_s[Ld];
                const uint32_t others = Lps.back & ~(1u << Lp);
                const int colL = wbase + L;
                const uint32_t Lsig = __shfl_sync(kFull, msig, L);
                uint32_t total;
                int32_t chosen;
                coop_refine<MODE == kModeCount>(g, Ms, T, lane, colL, Llo, Llen, others, Lps, Lsig, r, L, sectors,
                                                total, chosen);
                if (lane == L) {
                    cnt = total;
                    v = chosen;
                    if (MODE == kModeCount) sectors += (double)scan_sectors(Llen);  // driver chunks
                }
            }
        }

        mark(6);
        // ---------------- common epilogue: HT weight, record, terminate ----------------
        if (has) {
            W = (d == 0) ? (double)cnt : __dmul_rn(W, (double)cnt);
            if (MODE == kModeTrace) {
                gsword_sample_record* rec = records + (sid - first);
                rec->csize[d] = cnt;
                rec->path[d] = (cnt > 0) ? v : -1;
            }
            bool dead = (cnt == 0) || reject;
            // variant A5 (Fig. 19 AL Validate): DupCheck of the drawn vertex
            if (METHOD == GSWORD_ALLEY && !dead && pdup_s[d] != 0u &&
                !not_matched_sig(Ms + tid, T, 0, pdup_s[d], msig, v))
                dead = true;
            bool complete = false;
            if (!dead) {
                Ms[d * T + tid] = (uint32_t)v;
                msig |= sig_bit(v);
                if (d + 1 == nq) complete = true;
            }
            if (dead || complete) {
                if (complete) {
                    if (kSmemQueue)
                        nv_s[tid] += 1u;
                    else
                        n_valid += 1;
                    if (sched == 2) {
                        g_acc = __dadd_rn(g_acc, W);
                    } else {
                        accumulate(W);
                    }
                }
                if (MODE == kModeTrace) {
                    gsword_sample_record* rec = records + (sid - first);
                    rec->valid = complete ? 1 : 0;
                    rec->depth_reached = (uint8_t)d;
                    rec->sectors = msec;
                    rec->weight = W;
                }
                if (MODE == kModeCount) msum += (double)msec;
                has = false;
            } else {
                d += 1;
            }
        }
        if (sched == 2) {
            // Alg. 2: members without a valid partial sample inherit the lowest valid one; the
            // parent and its k copies carry W / (k + 1) (push-down)
            const unsigned alive_m = __ballot_sync(kFull, has);
            const unsigned idle_m = __ballot_sync(kFull, member && !has);
            if (alive_m != 0u && idle_m != 0u) {
                const int par = __ffs(alive_m) - 1;
                const double Wn = __ddiv_rn(__shfl_sync(kFull, W, par), (double)(__popc(idle_m) + 1));
                const int dp = __shfl_sync(kFull, d, par);
                const uint32_t psig = __shfl_sync(kFull, msig, par);
                __syncwarp();
                if (lane == par) W = Wn;
                if ((idle_m >> lane) & 1u) {
                    for (int j = 0; j < dp; ++j) Ms[j * T + tid] = Ms[j * T + wbase + par];
                    msig = psig;
                    d = dp;
                    W = Wn;
                    has = true;
                }
                __syncwarp();
            }
        }
    }
    if (sched == 2 && group_open) {
        double gsum = g_acc;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) gsum = __dadd_rn(gsum, shfl_xor_d(gsum, o));
        if (lane == 0) accumulate(gsum);
    }
    if (kSmemAcc) {
        s_sum = acc_s[0][tid];
        c_sum = acc_s[1][tid];
        s_sq = acc_s[2][tid];
        c_sq = acc_s[3][tid];
    }

    mark(7);
    if (MODE == kModeCount && phase_out && lane == 0) {
#pragma unroll
        for (int i = 0; i < 8; ++i) atomicAdd(phase_out + i, ph[i]);
    }

    if (kSmemQueue) {
        __syncwarp();
        n_valid = nv_s[tid];
        n_done = (lane == 0) ? wq_s[tid >> 5][2] : 0ull;
    }
    // ---------------- A10: warp -> CTA partial, fixed order ----------------
    write_cta_partial(warp_part, partials, s_sum, c_sum, s_sq, c_sq, n_valid, n_done, sectors, msum);
}

// ---------------------------------------------------------------- warp streaming (NEXT-3)
// Alg. 3 (reading A25) as a comparison mode for Alley: each position's
// Refine + Sample is streamed over the driver list.  Collaborative phase (l.5-17): while
// some lane has >= 32 unprocessed candidates, the lowest such lane leads, every lane
// refines one candidate of the leader's sample, the survivor with the largest reservoir
// key (r(sid, d, 1 + i)) is the chunk's pick (warp max, ties -> lowest lane), and the
// leader replaces its pick with probability total / curTotal (mulhi64 of the chunk draw
// r(sid, d, 0x80000000 | c)).  Independent phase (l.18-22): each lane streams its last
// < 32 candidates alone.  |C_d| = curTotal, so W, records and the estimator are those of
// Alley; only the drawn vertex differs from count-then-index.  Scheduling (refill /
// sample synchronisation / inheritance) and the epilogue mirror sample_kernel.
template <bool CG>
__device__ __forceinline__ bool stream_keep(const DeviceGraph& g, const uint32_t* Ms, int T, int col_of,
                                            const PlanStep& ps, int p, int32_t x) {
    double sec = 0.0;
    return not_matched(Ms, T, col_of, ps.dup, x) &&
           member_all<false>(g, Ms, T, col_of, ps.back & ~(1u << p), ps.label, x, sec);
}

template <int MODE, bool CG>
__global__ void __launch_bounds__(256) stream_kernel(const DeviceGraph g, const Plan plan_in, const uint64_t first,
                                                     const uint64_t count, const uint64_t seed, const int chunk,
                                                     const uint32_t /*coop_threshold*/, const int sched,
                                                     const uint32_t refill_min,
                                                     unsigned long long* __restrict__ queue,
                                                     Partial* __restrict__ partials,
                                                     gsword_sample_record* __restrict__ records,
                                                     unsigned long long* __restrict__ /*phase_out*/) {
    __shared__ PlanStep plan_s[kMaxQV];
    __shared__ uint8_t eidx_s[kMaxQV][kMaxQV];
    __shared__ uint32_t pdup_s[kMaxQV];
    __shared__ Partial warp_part[32];
    extern __shared__ uint32_t Ms[];  // Ms[j * blockDim.x + tid] = M[j] of this lane

    const int tid = threadIdx.x;
    const int T = blockDim.x;
    const int lane = tid & 31;
    const int wbase = tid - lane;
    const unsigned lt_mask = (1u << lane) - 1u;
    if (tid < kMaxQV) {
        plan_s[tid] = plan_in.step[tid];
        pdup_s[tid] = plan_in.pdup[tid];
    }
    for (int i = tid; i < kMaxQV * kMaxQV; i += blockDim.x) eidx_s[i / kMaxQV][i % kMaxQV] = plan_in.eidx[i / kMaxQV][i % kMaxQV];
    __syncthreads();
    const int nq = plan_in.nq;

    bool has = false;
    uint64_t sid = 0;
    int d = 0;
    double W = 0.0;
    double s_sum = 0.0, c_sum = 0.0, s_sq = 0.0, c_sq = 0.0;
    unsigned long long n_valid = 0, n_done = 0;
    uint64_t q_next = 0, q_end = 0;
    bool exhausted = false;
    bool member = false;
    double g_acc = 0.0;
    bool group_open = false;

    while (true) {
        // ---------------- A1: refill (as sample_kernel) ----------------
        unsigned need = __ballot_sync(kFull, !has);
        if (sched == 2 && need == kFull && group_open) {
            double gsum = g_acc;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) gsum = __dadd_rn(gsum, shfl_xor_d(gsum, o));
            if (lane == 0) {
                nsum(s_sum, c_sum, gsum);
                nsum(s_sq, c_sq, __dmul_rn(gsum, gsum));
            }
            g_acc = 0.0;
            group_open = false;
        }
        if (sched != 0 && need != kFull) need = 0u;
        if (sched == 0 && (uint32_t)__popc(need) < refill_min) need = 0u;
        if (need == kFull) member = false;
        while (need && !exhausted) {
            if (q_next == q_end) {
                unsigned long long base = 0;
                if (lane == 0) base = atomicAdd(queue, (unsigned long long)chunk);
                base = __shfl_sync(kFull, base, 0);
                if (base >= count) {
                    exhausted = true;
                    break;
                }
                q_next = base;
                q_end = ((uint64_t)base + (uint64_t)chunk < count) ? (uint64_t)base + (uint64_t)chunk : count;
            }
            const uint32_t avail = (q_end - q_next) < 32 ? (uint32_t)(q_end - q_next) : 32u;
            const uint32_t rank = __popc(need & lt_mask);
            if (!has && rank < avail) {
                has = true;
                member = true;
                n_done += 1;
                sid = first + q_next + rank;
                d = 0;
                W = 1.0;
                if (MODE == kModeTrace) {
                    gsword_sample_record* rec = records + (sid - first);
                    rec->sample_id = sid;
#pragma unroll
                    for (int i = 0; i < kMaxQV; ++i) {
                        rec->path[i] = -1;
                        rec->csize[i] = 0;
                    }
                }
            }
            q_next += min((uint32_t)__popc(need), avail);
            need = __ballot_sync(kFull, !has);
            group_open = true;
            if (sched != 0) break;
        }
        if (!__any_sync(kFull, has)) break;
        __syncwarp();

        // ---------------- seed, or GetMinCandidate (the driver list) ----------------
        PlanStep ps = {0, 0u, 0u, 0};
        uint32_t lo_p = 0, len_p = 0, cnt = 0, it = 0, chunk_no = 0;
        int p = 0;
        int32_t v = -1;
        if (has) {
            ps = plan_s[d];
            if (d == 0) {
                cnt = plan_in.seed_len;
                if (cnt > 0) {
                    const uint64_t k = __umul64hi(philox_r(seed, sid, 0u), (uint64_t)cnt);
                    v = plan_in.seed_identity ? (int32_t)(plan_in.seed_lo + k) : ldg_i32(g.bucket + plan_in.seed_lo + k);
                }
            } else {
                uint32_t bm = ps.back;
                len_p = 0xFFFFFFFFu;
                while (bm) {
                    const int j = __ffs(bm) - 1;
                    bm &= bm - 1;
                    uint32_t a, b;
                    local_run<CG>(g, eidx_s[d][j], Ms[j * T + tid], ps.label, &a, &b);
                    if (b - a < len_p) {
                        len_p = b - a;
                        lo_p = a;
                        p = j;
                    }
                }
            }
        }

        // ---------------- collaborative phase (Alg. 3 l.5-17) ----------------
        while (true) {
            const unsigned wm = __ballot_sync(kFull, has && d > 0 && len_p - it >= 32u);
            if (!wm) break;
            const int L = __ffs(wm) - 1;
            const uint32_t Llo = __shfl_sync(kFull, lo_p, L);
            const uint32_t Lit = __shfl_sync(kFull, it, L);
            const int Ld = __shfl_sync(kFull, d, L);
            const int Lp = __shfl_sync(kFull, p, L);
            const uint64_t Lsid = __shfl_sync(kFull, (unsigned long long)sid, L);
            const PlanStep Lps = plan_s[Ld];
            const uint32_t i = Lit + (uint32_t)lane;
            const int32_t x = ldg_i32(g.clist + Llo + i);
            const bool keep = stream_keep<CG>(g, Ms, T, wbase + L, Lps, Lp, x);
            uint64_t bkey = keep ? philox_rc(seed, Lsid, (uint32_t)Ld, 1u + i) : 0ull;  // A-Res key (l.11)
            int best = keep ? lane : -1;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {  // reduce_max (l.12), ties -> lowest lane
                const int ob = __shfl_xor_sync(kFull, best, o);
                const uint64_t okey = __shfl_xor_sync(kFull, (unsigned long long)bkey, o);
                if (ob >= 0 && (best < 0 || okey > bkey || (okey == bkey && ob < best))) {
                    best = ob;
                    bkey = okey;
                }
            }
            const uint32_t total = (uint32_t)__popc(__ballot_sync(kFull, keep));  // reduce_sum (l.13)
            const int32_t xb = __shfl_sync(kFull, x, best < 0 ? 0 : best);
            if (lane == L) {  // l.14-17
                cnt += total;
                if (total > 0 &&
                    __umul64hi(philox_rc(seed, sid, (uint32_t)d, 0x80000000u | chunk_no), (uint64_t)cnt) < total)
                    v = xb;
                it += 32u;
                chunk_no += 1u;
            }
        }

        // ---------------- independent phase (Alg. 3 l.18-22) ----------------
        if (has && d > 0) {
            for (; it < len_p; ++it) {
                const int32_t x = ldg_i32(g.clist + lo_p + it);
                if (stream_keep<CG>(g, Ms, T, tid, ps, p, x)) {
                    cnt += 1u;
                    if (__umul64hi(philox_rc(seed, sid, (uint32_t)d, 1u + it), (uint64_t)cnt) == 0ull) v = x;
                }
            }
        }

        // ---------------- epilogue (as sample_kernel) ----------------
        if (has) {
            W = (d == 0) ? (double)cnt : __dmul_rn(W, (double)cnt);
            if (MODE == kModeTrace) {
                gsword_sample_record* rec = records + (sid - first);
                rec->csize[d] = cnt;
                rec->path[d] = (cnt > 0) ? v : -1;
            }
            const bool dead = cnt == 0 || (pdup_s[d] != 0u && !not_matched(Ms + tid, T, 0, pdup_s[d], v));  // A5
            bool complete = false;
            if (!dead) {
                Ms[d * T + tid] = (uint32_t)v;
                if (d + 1 == nq) complete = true;
            }
            if (dead || complete) {
                if (complete) {
                    n_valid += 1;
                    if (sched == 2) {
                        g_acc = __dadd_rn(g_acc, W);
                    } else {
                        nsum(s_sum, c_sum, W);
                        nsum(s_sq, c_sq, __dmul_rn(W, W));
                    }
                }
                if (MODE == kModeTrace) {
                    gsword_sample_record* rec = records + (sid - first);
                    rec->valid = complete ? 1 : 0;
                    rec->depth_reached = (uint8_t)d;
                    rec->weight = W;
                }
                has = false;
            } else {
                d += 1;
            }
        }
        __syncwarp();
        if (sched == 2) {
            const unsigned alive_m = __ballot_sync(kFull, has);
            const unsigned idle_m = __ballot_sync(kFull, member && !has);
            if (alive_m != 0u && idle_m != 0u) {
                const int par = __ffs(alive_m) - 1;
                const double Wn = __ddiv_rn(__shfl_sync(kFull, W, par), (double)(__popc(idle_m) + 1));
                const int dp = __shfl_sync(kFull, d, par);
                __syncwarp();
                if (lane == par) W = Wn;
                if ((idle_m >> lane) & 1u) {
                    for (int j = 0; j < dp; ++j) Ms[j * T + tid] = Ms[j * T + wbase + par];
                    d = dp;
                    W = Wn;
                    has = true;
                }
                __syncwarp();
            }
        }
    }
    if (sched == 2 && group_open) {
        double gsum = g_acc;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) gsum = __dadd_rn(gsum, shfl_xor_d(gsum, o));
        if (lane == 0) {
            nsum(s_sum, c_sum, gsum);
            nsum(s_sq, c_sq, __dmul_rn(gsum, gsum));
        }
    }

    // ---------------- A10: warp -> CTA partial, fixed order ----------------
    write_cta_partial(warp_part, partials, s_sum, c_sum, s_sq, c_sq, n_valid, n_done, 0.0, 0.0);
}

// ---------------------------------------------------------------- trawling (NEXT-2)
// Alg. 4 (reading A23): per sample, d ~ P(d = j) proportional to 2^-j,
// j in [3, |V_q|], drawn exactly in integers from r(sid, 31); the first d
// positions are sampled with the method's rules (the same Philox draws as the plain
// sampler), then every completion is counted by a per-lane depth-first enumeration
// (ascending candidates, node budget); T = W_d * count.  One lane per sample; samples
// are taken one at a time from the queue.
__device__ __forceinline__ int choose_d(uint64_t seed, uint64_t sid, int nq) {
    if (nq <= 3) return nq;
    const uint64_t total = (1ull << (nq - 2)) - 1ull;
    const uint64_t k = __umul64hi(philox_r(seed, sid, 31u), total);
    uint64_t acc = 0;
    for (int j = 3; j <= nq; ++j) {
        acc += 1ull << (nq - j);
        if (k < acc) return j;
    }
    return nq;
}

template <bool CG>
__device__ __forceinline__ void getmin_local(const DeviceGraph& g, const PlanStep& ps, const uint8_t (*eidx)[kMaxQV],
                                             int d, const int32_t* M, uint32_t* lo, uint32_t* len, int* p) {
    uint32_t bm = ps.back;
    *len = 0xFFFFFFFFu;
    while (bm) {
        const int j = __ffs(bm) - 1;
        bm &= bm - 1;
        uint32_t a, b;
        local_run<CG>(g, eidx[d][j], (uint32_t)M[j], ps.label, &a, &b);
        if (b - a < *len) {
            *len = b - a;
            *lo = a;
            *p = j;
        }
    }
}

// x (drawn from S_p) extends M[0..d-1] at position d: in every other backward list and
// not matched (the Alley refine predicate; the enumeration uses it at every level)
__device__ __forceinline__ bool extends(const DeviceGraph& g, const PlanStep& ps, int p, const int32_t* M, int d,
                                        int32_t x) {
    for (int j = 0; j < d; ++j)
        if (M[j] == x) return false;
    uint32_t bm = ps.back & ~(1u << p);
    double sec = 0.0;
    while (bm) {
        const int j = __ffs(bm) - 1;
        bm &= bm - 1;
        if (!is_edge<false>(g, (uint32_t)M[j], (uint32_t)x, ps.label, sec)) return false;
    }
    return true;
}

// The sampled prefix of a trawling sample: positions 0 .. dd-1 with the method's rules and the
// same draws as the plain sampler; M[0..dd-1] and W = prod |C_d| out, false when it dies.
template <int METHOD, bool TRACE, bool CG>
__device__ __forceinline__ bool trawl_prefix(const DeviceGraph& g, const Plan& plan_in, const PlanStep* plan_s,
                                             const uint8_t (*eidx_s)[kMaxQV], uint64_t seed, uint64_t sid, int dd,
                                             int32_t* M, double* Wout, gsword_trawl_record* rec) {
    double W = 0.0;
    for (int d = 0; d < dd; ++d) {
        const PlanStep ps = plan_s[d];
        const uint64_t r = philox_r(seed, sid, (uint32_t)d);
        uint32_t lo = 0, len = 0, cnt = 0;
        int p = 0;
        int32_t v = -1;
        if (d == 0) {
            lo = plan_in.seed_lo;
            cnt = len = plan_in.seed_len;
            if (cnt > 0) {
                const uint64_t k = __umul64hi(r, (uint64_t)cnt);
                v = plan_in.seed_identity ? (int32_t)(lo + k) : __ldg(g.bucket + lo + k);
            }
        } else {
            getmin_local<CG>(g, ps, eidx_s, d, M, &lo, &len, &p);
            if (METHOD == GSWORD_WJ) {
                cnt = len;
                if (cnt > 0) {
                    v = __ldg(g.clist + lo + __umul64hi(r, (uint64_t)cnt));
                }
            } else {
                for (uint32_t i = 0; i < len; ++i) cnt += extends(g, ps, p, M, d, __ldg(g.clist + lo + i)) ? 1u : 0u;
                if (cnt > 0) {
                    uint32_t k = (uint32_t)__umul64hi(r, (uint64_t)cnt);
                    for (uint32_t i = 0; i < len; ++i) {
                        const int32_t x = __ldg(g.clist + lo + i);
                        if (!extends(g, ps, p, M, d, x)) continue;
                        if (k == 0) {
                            v = x;
                            break;
                        }
                        --k;
                    }
                }
            }
        }
        W = (d == 0) ? (double)cnt : __dmul_rn(W, (double)cnt);
        if (TRACE) {
            rec->csize[d] = cnt;
            rec->path[d] = cnt > 0 ? v : -1;
        }
        *Wout = W;
        if (cnt == 0) return false;
        if (METHOD == GSWORD_WJ && d > 0 && !extends(g, ps, p, M, d, v)) return false;  // Validate
        M[d] = v;
    }
    *Wout = W;
    return true;
}

// T = W * count into the lane's compensated sums (status 1 = complete, 2 = timeout)
__device__ __forceinline__ void trawl_accumulate(uint8_t status, double W, unsigned long long cnt_all, double& s_sum,
                                                 double& c_sum, double& s_sq, double& c_sq, double& n_timeout,
                                                 unsigned long long& n_nonzero, unsigned long long& n_done) {
    if (status == 2) {
        n_timeout += 1.0;
    } else {
        n_done += 1;
        if (status == 1 && cnt_all > 0) {
            const double T = __dmul_rn(W, (double)cnt_all);
            n_nonzero += 1;
            nsum(s_sum, c_sum, T);
            nsum(s_sq, c_sq, __dmul_rn(T, T));
        }
    }
}

template <int METHOD, bool TRACE, bool CG>
__global__ void __launch_bounds__(128) trawl_kernel(const DeviceGraph g, const Plan plan_in, const uint64_t first,
                                                    const uint64_t count, const uint64_t seed, const uint64_t budget,
                                                    unsigned long long* __restrict__ queue,
                                                    Partial* __restrict__ partials,
                                                    gsword_trawl_record* __restrict__ records) {
    __shared__ PlanStep plan_s[kMaxQV];
    __shared__ uint8_t eidx_s[kMaxQV][kMaxQV];
    __shared__ Partial warp_part[32];
    const int tid = threadIdx.x;
    if (tid < kMaxQV) plan_s[tid] = plan_in.step[tid];
    for (int i = tid; i < kMaxQV * kMaxQV; i += blockDim.x) eidx_s[i / kMaxQV][i % kMaxQV] = plan_in.eidx[i / kMaxQV][i % kMaxQV];
    __syncthreads();
    const int nq = plan_in.nq;
    double s_sum = 0.0, c_sum = 0.0, s_sq = 0.0, c_sq = 0.0, n_timeout = 0.0;
    unsigned long long n_nonzero = 0, n_done = 0;
    int32_t M[kMaxQV];
    uint32_t lvl_lo[kMaxQV], lvl_len[kMaxQV], lvl_i[kMaxQV];
    int lvl_p[kMaxQV];
    while (true) {
        const unsigned long long idx = atomicAdd(queue, 1ull);
        if (idx >= count) break;
        const uint64_t sid = first + idx;
        const int dd = choose_d(seed, sid, nq);
        gsword_trawl_record* rec = TRACE ? records + idx : nullptr;
        if (TRACE) {
            rec->sample_id = sid;
            rec->d = (uint8_t)dd;
            for (int i = 0; i < kMaxQV; ++i) {
                rec->path[i] = -1;
                rec->csize[i] = 0;
            }
        }
        double W = 0.0;
        const bool alive = trawl_prefix<METHOD, TRACE, CG>(g, plan_in, plan_s, eidx_s, seed, sid, dd, M, &W, rec);
        // ---- enumeration of positions dd .. nq-1 (depth first, ascending candidates)
        unsigned long long cnt_all = 0, nodes = 0;
        bool timeout = false;
        if (alive) {
            if (dd == nq) {
                cnt_all = 1;
            } else {
                int t = dd;
                getmin_local<CG>(g, plan_s[t], eidx_s, t, M, &lvl_lo[t], &lvl_len[t], &lvl_p[t]);
                lvl_i[t] = 0;
                while (t >= dd) {
                    if (lvl_i[t] >= lvl_len[t]) {  // level exhausted: back to the parent's next candidate
                        --t;
                        if (t >= dd) ++lvl_i[t];
                        continue;
                    }
                    const int32_t x = __ldg(g.clist + lvl_lo[t] + lvl_i[t]);
                    if (!extends(g, plan_s[t], lvl_p[t], M, t, x)) {
                        ++lvl_i[t];
                        continue;
                    }
                    if (nodes == budget) {
                        timeout = true;
                        break;
                    }
                    ++nodes;
                    M[t] = x;
                    if (t + 1 == nq) {
                        ++cnt_all;
                        ++lvl_i[t];
                    } else {
                        ++t;
                        getmin_local<CG>(g, plan_s[t], eidx_s, t, M, &lvl_lo[t], &lvl_len[t], &lvl_p[t]);
                        lvl_i[t] = 0;
                    }
                }
            }
        }
        const uint8_t status = !alive ? 0 : (timeout ? 2 : 1);
        if (TRACE) {
            rec->status = status;
            rec->weight = W;
            rec->count = cnt_all;
            rec->nodes = nodes;
        }
        trawl_accumulate(status, W, cnt_all, s_sum, c_sum, s_sq, c_sq, n_timeout, n_nonzero, n_done);
    }
    // block partial (fixed order); timeouts ride in the `sectors` slot
    write_cta_partial(warp_part, partials, s_sum, c_sum, s_sq, c_sq, n_nonzero, n_done, n_timeout, 0.0);
}

// Warp-cooperative trawling (estimates; gsword_trawl_range with GSWORD_OPT_TRAWL_WARP = 1).
// A warp takes 32 sample ids, every lane samples its own prefix, then the warp enumerates the
// completions of its lanes' samples one sample at a time: the candidate run of a level is
// tested 32 elements per round (one lane each, ballot), survivors at the last position are
// counted by popcount without descending, and the depth-first descent takes the survivors
// of a round in ascending order.  The node total of a sample's enumeration tree does not
// depend on the visiting order, so "more than `budget` nodes" (the timeout, reading A23) is
// decided exactly as the per-lane depth-first kernel decides it; a sample that does not
// time out gets the same count.  (Traces keep the per-lane kernel: a timed-out record's
// partial count depends on the visiting order.)
template <int METHOD, bool CG>
__global__ void __launch_bounds__(128) trawl_warp_kernel(const DeviceGraph g, const Plan plan_in, const uint64_t first,
                                                         const uint64_t count, const uint64_t seed,
                                                         const uint64_t budget, unsigned long long* __restrict__ queue,
                                                         Partial* __restrict__ partials) {
    constexpr int kW = 4;  // warps per CTA
    __shared__ PlanStep plan_s[kMaxQV];
    __shared__ uint8_t eidx_s[kMaxQV][kMaxQV];
    __shared__ Partial warp_part[32];
    __shared__ int32_t Mw[kW][kMaxQV];  // the enumerated sample's matched vertices
    __shared__ uint32_t st_lo[kW][kMaxQV], st_len[kW][kMaxQV], st_pos[kW][kMaxQV], st_mask[kW][kMaxQV],
        st_base[kW][kMaxQV];
    __shared__ int st_p[kW][kMaxQV];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    if (tid < kMaxQV) plan_s[tid] = plan_in.step[tid];
    for (int i = tid; i < kMaxQV * kMaxQV; i += blockDim.x) eidx_s[i / kMaxQV][i % kMaxQV] = plan_in.eidx[i / kMaxQV][i % kMaxQV];
    __syncthreads();
    const int nq = plan_in.nq;
    double s_sum = 0.0, c_sum = 0.0, s_sq = 0.0, c_sq = 0.0, n_timeout = 0.0;
    unsigned long long n_nonzero = 0, n_done = 0;
    int32_t M[kMaxQV];
    int32_t* const Ms = Mw[w];
    while (true) {
        unsigned long long base_id = 0;
        if (lane == 0) base_id = atomicAdd(queue, 32ull);
        base_id = __shfl_sync(kFull, base_id, 0);
        if (base_id >= count) break;
        const unsigned long long idx = base_id + (unsigned long long)lane;
        const bool has = idx < count;
        const uint64_t sid = first + idx;
        int dd = nq;
        double W = 0.0;
        bool alive = false;
        if (has) {
            dd = choose_d(seed, sid, nq);
            alive = trawl_prefix<METHOD, false, CG>(g, plan_in, plan_s, eidx_s, seed, sid, dd, M, &W, nullptr);
        }
        unsigned long long cnt_all = (alive && dd == nq) ? 1ull : 0ull;
        bool timeout = false;
        uint32_t todo = __ballot_sync(kFull, alive && dd < nq);
        while (todo) {
            const int L = __ffs(todo) - 1;
            todo &= todo - 1;
            const int d0 = __shfl_sync(kFull, dd, L);
            if (lane == L)
                for (int j = 0; j < d0; ++j) Ms[j] = M[j];
            __syncwarp();
            unsigned long long nodes = 0, cnt = 0;
            bool to = false;
            int t = d0, p = 0;
            uint32_t lo = 0, len = 0, pos = 0, mask = 0, base = 0;
            getmin_local<CG>(g, plan_s[t], eidx_s, t, Ms, &lo, &len, &p);
            while (true) {
                if (mask == 0u) {
                    if (pos >= len) {  // level exhausted: back to the parent's pending survivors
                        if (t == d0) break;
                        --t;
                        lo = st_lo[w][t];
                        len = st_len[w][t];
                        pos = st_pos[w][t];
                        mask = st_mask[w][t];
                        base = st_base[w][t];
                        p = st_p[w][t];
                        __syncwarp();  // every lane has read the level before lane 0 rewrites it
                        continue;
                    }
                    const uint32_t i = pos + (uint32_t)lane;
                    const bool ok = i < len && extends(g, plan_s[t], p, Ms, t, __ldg(g.clist + lo + i));
                    mask = __ballot_sync(kFull, ok);
                    base = pos;
                    pos += 32u;
                    nodes += (unsigned long long)__popc(mask);
                    if (nodes > budget) {
                        to = true;
                        break;
                    }
                    if (t + 1 == nq) {
                        cnt += (unsigned long long)__popc(mask);
                        mask = 0u;
                    }
                    continue;
                }
                const int b = __ffs(mask) - 1;
                mask &= mask - 1u;
                const int32_t x = __ldg(g.clist + lo + base + (uint32_t)b);
                if (lane == 0) {
                    st_lo[w][t] = lo;
                    st_len[w][t] = len;
                    st_pos[w][t] = pos;
                    st_mask[w][t] = mask;
                    st_base[w][t] = base;
                    st_p[w][t] = p;
                    Ms[t] = x;
                }
                __syncwarp();
                ++t;
                getmin_local<CG>(g, plan_s[t], eidx_s, t, Ms, &lo, &len, &p);
                pos = 0u;
                mask = 0u;
                base = 0u;
            }
            if (lane == L) {
                cnt_all = cnt;
                timeout = to;
            }
            __syncwarp();
        }
        if (has) {
            const uint8_t status = !alive ? 0 : (timeout ? 2 : 1);
            trawl_accumulate(status, W, cnt_all, s_sum, c_sum, s_sq, c_sq, n_timeout, n_nonzero, n_done);
        }
    }
    write_cta_partial(warp_part, partials, s_sum, c_sum, s_sq, c_sq, n_nonzero, n_done, n_timeout, 0.0);
}

// Grid reduction in CTA order (one warp; lane-strided then a fixed butterfly).
__global__ void reduce_kernel(const Partial* __restrict__ partials, int n, double* __restrict__ out4,
                              double* __restrict__ sectors_out) {
    const int lane = threadIdx.x;
    double sh = 0, sl = 0, qh = 0, ql = 0, sec = 0, mod = 0;
    unsigned long long valid = 0, cnt = 0;
    for (int i = lane; i < n; i += 32) {
        const Partial p = partials[i];
        dd_add(sh, sl, p.sum_hi, p.sum_lo);
        dd_add(qh, ql, p.sq_hi, p.sq_lo);
        valid += p.valid;
        cnt += p.n;
        sec += p.sectors;
        mod += p.model;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double bh = shfl_xor_d(sh, o), bl = shfl_xor_d(sl, o);
        const double ch = shfl_xor_d(qh, o), cl = shfl_xor_d(ql, o);
        dd_add(sh, sl, bh, bl);
        dd_add(qh, ql, ch, cl);
        valid += __shfl_xor_sync(kFull, valid, o);
        cnt += __shfl_xor_sync(kFull, cnt, o);
        sec += shfl_xor_d(sec, o);
        mod += shfl_xor_d(mod, o);
    }
    if (lane == 0) {
        out4[0] = __dadd_rn(sh, sl);
        out4[1] = __dadd_rn(qh, ql);
        out4[2] = (double)valid;
        out4[3] = (double)cnt;
        if (sectors_out) {
            sectors_out[0] = sec;  // touched sectors (trawl: timeouts)
            sectors_out[1] = mod;  // algorithmic sectors (A26)
        }
    }
}

__global__ void set_u64_kernel(unsigned long long* p, unsigned long long v) { *p = v; }

__global__ void iota_kernel(int32_t* out, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int32_t)i;
}

// One thread per vertex v: insert every edge {v, w}, w > v, into the edge set.
__global__ void eset_kernel(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col, int64_t n,
                            unsigned long long* __restrict__ keys, uint64_t mask) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) {
            const int32_t w = col[i];
            if (w <= v) continue;
            const unsigned long long key = edge_key((uint32_t)v, (uint32_t)w);
            uint64_t bk = edge_hash((uint32_t)v, (uint32_t)w) & mask;
            bool done = false;
            while (!done) {
                for (int s = 0; s < 4 && !done; ++s) {
                    const unsigned long long prev = atomicCAS(keys + 4 * bk + s, kEmptyKey, key);
                    done = (prev == kEmptyKey) || (prev == key);
                }
                bk = (bk + 1) & mask;
            }
        }
    }
}

// One thread per vertex v: set the filter bits of every edge {v, w} with w > v.
__global__ void bloom_kernel(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col, int64_t n,
                             unsigned long long* __restrict__ bloom, uint64_t mask) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) {
            const int32_t w = col[i];
            if (w <= v) continue;
            const uint64_t h = edge_hash((uint32_t)v, (uint32_t)w);
            atomicOr(bloom + (h & mask), (unsigned long long)bloom_bits(h));
        }
    }
}

// ---------------------------------------------------------------- candidate graph build
// (NEXT-1; Def. 4-5, Fig. 4).  Load-time only.
__device__ __forceinline__ uint32_t nbr_count(const DeviceGraph& g, uint32_t v, int32_t l) {
    uint32_t a, b;
    segment(g, v, l, &a, &b);
    return b - a;
}

// cbits[u][v] for every query vertex u (warp-aligned vertex groups -> one word per ballot)
__global__ void filter_kernel(const DeviceGraph g, const QFilter* __restrict__ qf, int nq, int filter,
                              uint32_t* __restrict__ cbits, const int32_t* __restrict__ vlabel) {
    const int lane = threadIdx.x & 31;
    const int64_t nwarps = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int64_t warp = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    for (int64_t base = warp * 32; base < g.n; base += nwarps * 32) {
        const int64_t v = base + lane;
        const bool in = v < g.n;
        const int32_t lv = in ? vlabel[v] : -1;
        uint32_t deg = 0;
        if (in) {
            uint32_t a, b, a2, b2;
            segment(g, (uint32_t)v, 0, &a, &b);
            segment(g, (uint32_t)v, g.n_labels - 1, &a2, &b2);
            deg = b2 - a;
        }
        for (int u = 0; u < nq; ++u) {
            bool ok = in && lv == qf[u].label;
            if (ok && filter >= 1) ok = deg >= (uint32_t)qf[u].deg;
            if (ok && filter >= 2)
                for (int i = 0; i < qf[u].npairs && ok; ++i)
                    ok = nbr_count(g, (uint32_t)v, qf[u].plabel[i]) >= (uint32_t)qf[u].pcount[i];
            const unsigned word = __ballot_sync(0xffffffffu, ok);
            if (lane == 0) cbits[(size_t)u * g.cwords + (size_t)(base >> 5)] = word;
        }
    }
}

__device__ __forceinline__ bool bit_of(const uint32_t* cbits, uint32_t cwords, int u, uint32_t v) {
    return (cbits[(size_t)u * cwords + (v >> 5)] >> (v & 31u)) & 1u;
}

// position of v in the ascending list C(u) (v in C(u)): the rank directory of the bitmap
__device__ __forceinline__ uint32_t cand_rank(const DeviceGraph& g, int u, uint32_t v) {
    const size_t w = (size_t)u * g.cwords + (v >> 5);
    return g.crank[w] + __popc(g.cbits[w] & ((1u << (v & 31u)) - 1u));
}

// crank[u][w] = popc(cbits[u][w]); the exclusive scan of the row follows
__global__ void rank_words_kernel(const uint32_t* __restrict__ cbits, uint32_t cwords, int u,
                                  uint32_t* __restrict__ crank) {
    for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < cwords; w += (int64_t)gridDim.x * blockDim.x)
        crank[(size_t)u * cwords + w] = __popc(cbits[(size_t)u * cwords + w]);
}

// counts[rank_u(v)] = |N_{label2}(v) ∩ C(u2)| for v in C(u) (Fig. 4, 3rd CSR sizes)
__global__ void cg_count_kernel(const DeviceGraph g, int u, int u2, int32_t label2, uint32_t* __restrict__ counts) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < g.n; v += (int64_t)gridDim.x * blockDim.x) {
        if (!bit_of(g.cbits, g.cwords, u, (uint32_t)v)) continue;
        uint32_t c = 0, a, b;
        segment(g, (uint32_t)v, label2, &a, &b);
        for (uint32_t i = a; i < b; ++i) c += bit_of(g.cbits, g.cwords, u2, (uint32_t)g.col[i]) ? 1u : 0u;
        counts[cand_rank(g, u, (uint32_t)v)] = c;
    }
}

__global__ void cg_fill_kernel(const DeviceGraph g, int u, int u2, int32_t label2, const uint32_t* __restrict__ off,
                               int32_t* __restrict__ out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < g.n; v += (int64_t)gridDim.x * blockDim.x) {
        if (!bit_of(g.cbits, g.cwords, u, (uint32_t)v)) continue;
        uint32_t pos = off[cand_rank(g, u, (uint32_t)v)];
        uint32_t a, b;
        segment(g, (uint32_t)v, label2, &a, &b);
        for (uint32_t i = a; i < b; ++i) {
            const int32_t w = g.col[i];
            if (bit_of(g.cbits, g.cwords, u2, (uint32_t)w)) out[pos++] = w;
        }
    }
}

__global__ void cand_fill_kernel(const DeviceGraph g, int u, int32_t* __restrict__ out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < g.n; v += (int64_t)gridDim.x * blockDim.x)
        if (bit_of(g.cbits, g.cwords, u, (uint32_t)v)) out[cand_rank(g, u, (uint32_t)v)] = (int32_t)v;
}

// ---- exclusive scan (three phases): 2048 elements per block
constexpr int kScanThreads = 1024;
constexpr int kScanPer = 2048;

__device__ __forceinline__ uint32_t block_exclusive(uint32_t x, uint32_t* warp_tot, uint32_t* total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) warp_tot[w] = incl;
    __syncthreads();
    if (w == 0) {
        uint32_t t = warp_tot[lane];
        uint32_t ti = t;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, ti, o);
            if (lane >= o) ti += y;
        }
        warp_tot[lane] = ti - t;
        if (lane == 31) *total = ti;
    }
    __syncthreads();
    const uint32_t r = warp_tot[w] + incl - x;
    __syncthreads();
    return r;
}

__global__ void scan_local_kernel(uint32_t* __restrict__ data, int64_t n, uint32_t* __restrict__ block_sums) {
    __shared__ uint32_t wt[32];
    __shared__ uint32_t tot;
    const int64_t i0 = (int64_t)blockIdx.x * kScanPer + 2 * threadIdx.x;
    const uint32_t a = i0 < n ? data[i0] : 0u;
    const uint32_t b = i0 + 1 < n ? data[i0 + 1] : 0u;
    const uint32_t ex = block_exclusive(a + b, wt, &tot);
    if (i0 < n) data[i0] = ex;
    if (i0 + 1 < n) data[i0 + 1] = ex + a;
    if (threadIdx.x == 0) block_sums[blockIdx.x] = tot;
}

// one block: exclusive scan of the block sums (in 64-bit, offset by *base_in);
// total_out[0] = base + sum (64-bit, for the overflow check on the host)
__global__ void scan_sums_kernel(uint32_t* __restrict__ block_sums, int64_t nb, const unsigned long long* base_in,
                                 unsigned long long* total_out) {
    __shared__ unsigned long long carry;
    __shared__ uint32_t wt[32];
    __shared__ uint32_t tot;
    if (threadIdx.x == 0) carry = base_in ? *base_in : 0ull;
    __syncthreads();
    for (int64_t b0 = 0; b0 < nb; b0 += kScanThreads) {
        const int64_t i = b0 + threadIdx.x;
        const uint32_t x = i < nb ? block_sums[i] : 0u;
        const uint32_t ex = block_exclusive(x, wt, &tot);
        const unsigned long long c = carry;
        if (i < nb) block_sums[i] = (uint32_t)(c + ex);  // absolute offset (checked < 2^32 on host)
        __syncthreads();
        if (threadIdx.x == 0) carry = c + tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) *total_out = carry;
}

__global__ void scan_add_kernel(uint32_t* __restrict__ data, int64_t n, const uint32_t* __restrict__ block_sums) {
    const int64_t i0 = (int64_t)blockIdx.x * kScanPer + 2 * threadIdx.x;
    const uint32_t add = block_sums[blockIdx.x];
    if (i0 < n) data[i0] += add;
    if (i0 + 1 < n) data[i0 + 1] += add;
}

template <int METHOD, bool CG, bool TREE, bool LOCK>
const void* estimate_ptr(int occ) {
    if (occ == 1) return reinterpret_cast<const void*>(&sample_kernel<METHOD, kModeEstimate, CG, false, 1, TREE, LOCK>);
    if (occ == 2) return reinterpret_cast<const void*>(&sample_kernel<METHOD, kModeEstimate, CG, false, 2, TREE, LOCK>);
    return reinterpret_cast<const void*>(&sample_kernel<METHOD, kModeEstimate, CG, false, 0, TREE, LOCK>);
}

template <int METHOD, int MODE, bool CG>
const void* kernel_ptr(bool sync, int occ = 0, bool tree = false, bool lock = false) {
    if (MODE == kModeEstimate && !sync) {
        if (METHOD == GSWORD_ALLEY && lock)
            return tree ? estimate_ptr<METHOD, CG, true, true>(occ) : estimate_ptr<METHOD, CG, false, true>(occ);
        return tree ? estimate_ptr<METHOD, CG, true, false>(occ) : estimate_ptr<METHOD, CG, false, false>(occ);
    }
    return sync ? reinterpret_cast<const void*>(&sample_kernel<METHOD, MODE, CG, true>)
                : reinterpret_cast<const void*>(&sample_kernel<METHOD, MODE, CG, false>);
}

template <bool CG>
const void* select_kernel_cg(int method, int mode) {
    if (mode & kModeStream) {  // warp streaming (Alley only; the host never asks for WJ or count)
        return (mode & 3) == kModeTrace ? reinterpret_cast<const void*>(&stream_kernel<kModeTrace, CG>)
                                        : reinterpret_cast<const void*>(&stream_kernel<kModeEstimate, CG>);
    }
    const bool sync = (mode & kModeSync) != 0;
    const int occ = (mode >> kModeOccShift) & 3;
    const bool tree = (mode & kModeTree) != 0;
    const bool lock = (mode & kModeLock) != 0;
    mode &= 3;
    if (method == GSWORD_WJ) {
        if (mode == kModeTrace) return kernel_ptr<GSWORD_WJ, kModeTrace, CG>(sync);
        if (mode == kModeCount) return kernel_ptr<GSWORD_WJ, kModeCount, CG>(sync);
        return kernel_ptr<GSWORD_WJ, kModeEstimate, CG>(sync, occ, tree);
    }
    if (mode == kModeTrace) return kernel_ptr<GSWORD_ALLEY, kModeTrace, CG>(sync);
    if (mode == kModeCount) return kernel_ptr<GSWORD_ALLEY, kModeCount, CG>(sync);
    return kernel_ptr<GSWORD_ALLEY, kModeEstimate, CG>(sync, occ, tree, lock);
}

// mode: kMode* | kModeCG when the query was loaded with a candidate filter
const void* select_kernel(int method, int mode) {
    return (mode & kModeCG) ? select_kernel_cg<true>(method, mode & ~kModeCG)
                            : select_kernel_cg<false>(method, mode & ~kModeCG);
}

}  // namespace

// Grid of the grid-stride load-time kernels: `per_sm` CTAs on every SM of the current
// device (multiProcessorCount, queried once per device).
int sm_grid(int per_sm) {
    static int cached[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148 * per_sm;
    if (cached[dev] == 0) {
        int sms = 0;
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) sms = 148;
        cached[dev] = sms;
    }
    return cached[dev] * per_sm;
}

int occ_blocks(int method, int occ_variant) { return kOccBlocks(method, occ_variant); }

int max_blocks_per_sm(int method, int mode, int threads, int ms_rows, size_t* smem_bytes) {
    (void)threads;  // every sampling kernel's rows are kSampleLanes words (rows: sample_smem_rows)
    const size_t smem = (size_t)ms_rows * (size_t)kSampleLanes * sizeof(uint32_t);
    if (smem_bytes) *smem_bytes = smem;
    int blocks = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, select_kernel(method, mode), threads, smem) !=
        cudaSuccess)
        return 0;
    return blocks;
}

cudaError_t launch_sample(int method, int mode, const DeviceGraph& g, const Plan& plan, const LaunchCfg& cfg,
                          uint64_t first, uint64_t count, uint64_t seed, unsigned long long* d_queue,
                          Partial* d_partials, gsword_sample_record* d_records, unsigned long long* d_phase,
                          cudaStream_t stream) {
    cudaError_t e = cudaMemsetAsync(d_queue, 0, sizeof(unsigned long long), stream);
    if (e != cudaSuccess) return e;
    if (cfg.queue_start) {  // fault injection: a corrupted queue counter
        set_u64_kernel<<<1, 1, 0, stream>>>(d_queue, cfg.queue_start);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    // rows of the dynamic array (sample_smem_rows): sizing it by the query and the coop
    // threshold leaves the rest of the 256 KB L1/shared array to the L1 cache (spill slots,
    // hot CSR entries; measured: Alley is L1-capacity sensitive)
    const size_t smem = (size_t)cfg.ms_rows * (size_t)kSampleLanes * sizeof(uint32_t);
    const uint32_t thr = (uint32_t)cfg.coop_threshold;
    Plan pl = plan;
    pl.multi_back = 0;
    for (int d = 1; d < pl.nq; ++d) pl.multi_back |= pl.step[d].nback >= 2 ? 1 : 0;
    void* args[] = {(void*)&g,      (void*)&pl,  (void*)&first,   (void*)&count,     (void*)&seed,
                    (void*)&cfg.chunk, (void*)&thr, (void*)&cfg.sched, (void*)&cfg.refill_min, (void*)&d_queue,
                    (void*)&d_partials,
                    (void*)&d_records,
                    (void*)&d_phase};
    return cudaLaunchKernel(select_kernel(method, mode), dim3(cfg.grid), dim3(cfg.threads), args, smem, stream);
}

cudaError_t launch_reduce(const Partial* d_partials, int n_partials, double* d_out4, double* d_sectors,
                          cudaStream_t stream) {
    reduce_kernel<<<1, 32, 0, stream>>>(d_partials, n_partials, d_out4, d_sectors);
    return cudaGetLastError();
}

cudaError_t launch_build_bloom(const int64_t* d_row_ptr, const int32_t* col, int64_t n, unsigned long long* bloom,
                               uint64_t mask, cudaStream_t stream) {
    bloom_kernel<<<sm_grid(8), 256, 0, stream>>>(d_row_ptr, col, n, bloom, mask);
    return cudaGetLastError();
}

cudaError_t launch_build_eset(const int64_t* d_row_ptr, const int32_t* col, int64_t n, unsigned long long* keys,
                              uint64_t mask, cudaStream_t stream) {
    eset_kernel<<<sm_grid(8), 256, 0, stream>>>(d_row_ptr, col, n, keys, mask);
    return cudaGetLastError();
}

cudaError_t launch_filter(const DeviceGraph& g, const QFilter* d_qf, int nq, int filter, uint32_t* cbits,
                          const int32_t* d_vlabel, cudaStream_t stream) {
    filter_kernel<<<sm_grid(4), 256, 0, stream>>>(g, d_qf, nq, filter, cbits, d_vlabel);
    return cudaGetLastError();
}

cudaError_t launch_rank_words(const uint32_t* cbits, uint32_t cwords, int u, uint32_t* crank, cudaStream_t stream) {
    rank_words_kernel<<<sm_grid(2), 256, 0, stream>>>(cbits, cwords, u, crank);
    return cudaGetLastError();
}

cudaError_t launch_cg_count(const DeviceGraph& g, int u, int u2, int32_t label2, uint32_t* counts,
                            cudaStream_t stream) {
    cg_count_kernel<<<sm_grid(8), 256, 0, stream>>>(g, u, u2, label2, counts);
    return cudaGetLastError();
}

cudaError_t launch_cg_fill(const DeviceGraph& g, int u, int u2, int32_t label2, const uint32_t* off, int32_t* out,
                           cudaStream_t stream) {
    cg_fill_kernel<<<sm_grid(8), 256, 0, stream>>>(g, u, u2, label2, off, out);
    return cudaGetLastError();
}

cudaError_t launch_cand_fill(const DeviceGraph& g, int u, int32_t* out, cudaStream_t stream) {
    cand_fill_kernel<<<sm_grid(4), 256, 0, stream>>>(g, u, out);
    return cudaGetLastError();
}

size_t scan_tmp_words(int64_t n) { return (size_t)((n + kScanPer - 1) / kScanPer) + 1; }

cudaError_t launch_scan(uint32_t* data, int64_t n, const unsigned long long* d_base, uint32_t* d_tmp,
                        unsigned long long* d_total, cudaStream_t stream) {
    const int64_t nb = (n + kScanPer - 1) / kScanPer;
    scan_local_kernel<<<(unsigned)nb, kScanThreads, 0, stream>>>(data, n, d_tmp);
    scan_sums_kernel<<<1, kScanThreads, 0, stream>>>(d_tmp, nb, d_base, d_total);
    scan_add_kernel<<<(unsigned)nb, kScanThreads, 0, stream>>>(data, n, d_tmp);
    return cudaGetLastError();
}

cudaError_t launch_trawl(int method, bool trace, bool warp, bool cg, const DeviceGraph& g, const Plan& plan, int grid,
                         uint64_t first, uint64_t count, uint64_t seed, uint64_t budget, unsigned long long* d_queue,
                         Partial* d_partials, gsword_trawl_record* d_records, cudaStream_t stream) {
    cudaError_t e = cudaMemsetAsync(d_queue, 0, sizeof(unsigned long long), stream);
    if (e != cudaSuccess) return e;
#define GSWORD_TRAWL(M, TR, CGF) \
    trawl_kernel<M, TR, CGF><<<grid, 128, 0, stream>>>(g, plan, first, count, seed, budget, d_queue, d_partials, d_records)
#define GSWORD_TRAWL_WARP(M, CGF) \
    trawl_warp_kernel<M, CGF><<<grid, 128, 0, stream>>>(g, plan, first, count, seed, budget, d_queue, d_partials)
    if (warp && !trace) {
        if (method == GSWORD_WJ) { if (cg) GSWORD_TRAWL_WARP(GSWORD_WJ, true); else GSWORD_TRAWL_WARP(GSWORD_WJ, false); }
        else { if (cg) GSWORD_TRAWL_WARP(GSWORD_ALLEY, true); else GSWORD_TRAWL_WARP(GSWORD_ALLEY, false); }
    } else if (method == GSWORD_WJ) {
        if (trace) { if (cg) GSWORD_TRAWL(GSWORD_WJ, true, true); else GSWORD_TRAWL(GSWORD_WJ, true, false); }
        else { if (cg) GSWORD_TRAWL(GSWORD_WJ, false, true); else GSWORD_TRAWL(GSWORD_WJ, false, false); }
    } else {
        if (trace) { if (cg) GSWORD_TRAWL(GSWORD_ALLEY, true, true); else GSWORD_TRAWL(GSWORD_ALLEY, true, false); }
        else { if (cg) GSWORD_TRAWL(GSWORD_ALLEY, false, true); else GSWORD_TRAWL(GSWORD_ALLEY, false, false); }
    }
#undef GSWORD_TRAWL_WARP
#undef GSWORD_TRAWL
    return cudaGetLastError();
}

// ---------------------------------------------------------------- device-side graph load
// (gsword_load_graph_device: the CSR stays in caller-owned device memory)
__device__ __forceinline__ bool key_less(int32_t la, int32_t a, int32_t lb, int32_t b) {
    return la < lb || (la == lb && a < b);
}

// canonical check: ids in range, no self loop, rows strictly ascending by (label, id), and
// the adjacency symmetric (v found in w's row by binary search on (label, id))
__global__ void dev_validate_kernel(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                                    const int32_t* __restrict__ labels, int64_t n, int32_t n_labels,
                                    int* __restrict__ bad) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t lv = labels ? labels[v] : 0;
        if (lv < 0 || lv >= n_labels) { atomicOr(bad, 1); continue; }
        const int64_t a = row_ptr[v], b = row_ptr[v + 1];
        if (b < a) { atomicOr(bad, 2); continue; }
        int32_t pl = -1, pw = -1;
        for (int64_t i = a; i < b; ++i) {
            const int32_t w = col[i];
            if (w < 0 || w >= n || w == v) { atomicOr(bad, 4); break; }
            const int32_t lw = labels ? labels[w] : 0;
            if (i > a && !key_less(pl, pw, lw, w)) { atomicOr(bad, 8); break; }
            pl = lw;
            pw = w;
            int64_t lo = row_ptr[w], hi = row_ptr[w + 1];
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                const int32_t x = col[mid];
                const int32_t lx = labels ? labels[x] : 0;
                if (key_less(lx, x, lv, (int32_t)v)) lo = mid + 1; else hi = mid;
            }
            if (lo >= row_ptr[w + 1] || col[lo] != (int32_t)v) { atomicOr(bad, 16); break; }
        }
    }
}

__global__ void dev_seg_kernel(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                               const int32_t* __restrict__ labels, int64_t n, int32_t L, uint32_t* __restrict__ seg) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n; v += (int64_t)gridDim.x * blockDim.x) {
        if (v == n) {
            seg[(size_t)n * L] = (uint32_t)row_ptr[n];
            continue;
        }
        const int64_t a = row_ptr[v], b = row_ptr[v + 1];
        int32_t l = 0;
        for (int64_t i = a; i < b; ++i) {
            const int32_t lw = labels ? labels[col[i]] : 0;
            while (l <= lw) seg[(size_t)v * L + l++] = (uint32_t)i;
        }
        while (l < L) seg[(size_t)v * L + l++] = (uint32_t)b;
    }
}

__global__ void label_hist_kernel(const int32_t* __restrict__ labels, int64_t n, unsigned long long* __restrict__ hist) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(hist + (labels ? labels[v] : 0), 1ull);
}

// data adjacency entries per (label, label): block-private histograms in shared memory
__global__ void pair_hist_kernel(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                                 const int32_t* __restrict__ labels, int64_t n, int32_t L,
                                 unsigned long long* __restrict__ hist) {
    extern __shared__ unsigned long long h[];
    const int bins = L * L;
    for (int i = threadIdx.x; i < bins; i += blockDim.x) h[i] = 0ull;
    __syncthreads();
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t lv = labels ? labels[v] : 0;
        if (!labels) {
            atomicAdd(&h[0], (unsigned long long)(row_ptr[v + 1] - row_ptr[v]));
            continue;
        }
        for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; ++i) atomicAdd(&h[lv * L + labels[col[i]]], 1ull);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < bins; i += blockDim.x)
        if (h[i]) atomicAdd(hist + i, h[i]);
}

__global__ void label_count_kernel(const int32_t* __restrict__ labels, int64_t n, int32_t l,
                                   uint32_t* __restrict__ counts) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v <= n; v += (int64_t)gridDim.x * blockDim.x)
        counts[v] = (v < n && labels[v] == l) ? 1u : 0u;
}

__global__ void label_fill_kernel(const int32_t* __restrict__ labels, int64_t n, int32_t l,
                                  const uint32_t* __restrict__ off, int32_t* __restrict__ bucket) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        if (labels[v] == l) bucket[off[v]] = (int32_t)v;
}

cudaError_t launch_dev_validate(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n,
                                int32_t n_labels, int* d_bad, cudaStream_t stream) {
    dev_validate_kernel<<<sm_grid(8), 256, 0, stream>>>(row_ptr, col, labels, n, n_labels, d_bad);
    return cudaGetLastError();
}

cudaError_t launch_dev_seg(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n, int32_t L,
                           uint32_t* seg, cudaStream_t stream) {
    dev_seg_kernel<<<sm_grid(8), 256, 0, stream>>>(row_ptr, col, labels, n, L, seg);
    return cudaGetLastError();
}

cudaError_t launch_label_hist(const int32_t* labels, int64_t n, unsigned long long* hist, cudaStream_t stream) {
    label_hist_kernel<<<sm_grid(4), 256, 0, stream>>>(labels, n, hist);
    return cudaGetLastError();
}

cudaError_t launch_pair_hist(const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int64_t n, int32_t L,
                             unsigned long long* hist, cudaStream_t stream) {
    const size_t smem = sizeof(unsigned long long) * (size_t)L * (size_t)L;
    pair_hist_kernel<<<sm_grid(4), 256, smem, stream>>>(row_ptr, col, labels, n, L, hist);
    return cudaGetLastError();
}

cudaError_t launch_label_bucket(const int32_t* labels, int64_t n, int32_t l, uint32_t* counts,
                                const unsigned long long* d_base, uint32_t* d_tmp, unsigned long long* d_total,
                                int32_t* bucket, cudaStream_t stream) {
    label_count_kernel<<<sm_grid(4), 256, 0, stream>>>(labels, n, l, counts);
    cudaError_t e = launch_scan(counts, n + 1, d_base, d_tmp, d_total, stream);
    if (e != cudaSuccess) return e;
    label_fill_kernel<<<sm_grid(4), 256, 0, stream>>>(labels, n, l, counts, bucket);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- gather roofline (K5)
// Random 4-byte loads, one per 32-byte sector, uniformly over a buffer of `words` u32:
// `inflight` independent chains per thread, each `steps` long (the next index depends on
// the loaded value, like the sampler's dependent gathers).  Measures the sector rate the
// memory system sustains for this access pattern.
__global__ void gather_kernel(const uint32_t* __restrict__ buf, uint64_t words, int steps, int inflight,
                              unsigned long long* __restrict__ sink) {
    const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint32_t acc = 0;
    uint64_t idx[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) idx[c] = (tid * 8 + c) * 0x9E3779B97F4A7C15ull;
    for (int s = 0; s < steps; ++s) {
#pragma unroll
        for (int c = 0; c < 8; ++c) {
            if (c >= inflight) break;
            const uint64_t i = ((idx[c] >> 17) % (words >> 3)) << 3;  // sector-aligned word
            const uint32_t v = __ldg(buf + i);
            acc ^= v;
            idx[c] = (idx[c] + v + 0x632BE59BD9B4E019ull) * 0xD6E8FEB86659FD93ull;
        }
    }
    if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

cudaError_t launch_gather(const uint32_t* buf, uint64_t words, int steps, int inflight, int blocks, int threads,
                          unsigned long long* sink, cudaStream_t stream) {
    gather_kernel<<<blocks, threads, 0, stream>>>(buf, words, steps, inflight, sink);
    return cudaGetLastError();
}

cudaError_t launch_build_bucket_identity(int32_t* bucket, int64_t n, cudaStream_t stream) {
    iota_kernel<<<sm_grid(4), 256, 0, stream>>>(bucket, n);
    return cudaGetLastError();
}

}  // namespace gsword
