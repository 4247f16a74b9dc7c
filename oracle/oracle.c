/*
 * oracle.c — plain, slow, obviously-correct CPU reference for the gSWORD hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_journals_pacmmod_yelsg24_b200/) never links, imports or calls it, and it
 * shares no code, header, table or constant generator with the CUDA path.
 *
 * What it computes (PAPER.md = P:L<line>; readings = DESIGN.md §3):
 *   - Philox4x32-10 counter-based generator (reading A6; Salmon et al. SC'11),
 *     one call per (seed, sample id, depth).
 *   - WanderJoin samples (§2.2; Fig. 19 WJ P:L1756-L1774; Alg. 1):
 *     seed from the global candidate set, each next vertex drawn uniformly from the
 *     smallest local candidate list of the already-matched query neighbours
 *     (GetMinCandidate, Alg. 1 l.8 P:L798), then Validate (DupCheck + IsEdge).
 *   - Alley samples (Fig. 19 AL P:L1775-L1805): the candidate set is the
 *     intersection of all local candidate lists of matched query neighbours, minus
 *     already-matched vertices (reading A5); an empty set ends the sample.
 *   - Horvitz-Thompson value per sample (Eq. 1): Y = prod |C_d| if the
 *     sample is a complete instance, else 0.  Aggregation (sum / n) is done by the
 *     Python wrapper with a correctly rounded sum (math.fsum).
 *   - Exact embedding count by plain backtracking (estimand, reading A1).
 *
 * Every step is written in the paper's order with no blocking, fusion or
 * reordering.  Membership tests use the C library bsearch on ascending lists.
 */
#include <pthread.h>
#include <stdatomic.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_MAX_QV 16

/* ---- per-sample record (layout is the contract of include/gsword.h, restated) ---- */
typedef struct {
    uint64_t sample_id;
    uint8_t valid;
    uint8_t depth_reached;
    uint8_t pad[2];
    uint32_t sectors; /* algorithmic 32-byte sectors of the sample (reading A26, below) */
    int32_t path[OR_MAX_QV];
    uint32_t csize[OR_MAX_QV];
    double weight;
} or_record; /* 152 bytes */

/* ---- Philox4x32-10 (reading A6 / SURVEY R10) ---------------------------------- */
void or_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
    uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int round = 0; round < 10; ++round) {
        uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* r(sid, d, c): key = seed, counter = (sid, d, c); r = x1:x0.  The plain
 * samplers use c = 0; warp streaming (reading A25) uses c = 1 + element index for the
 * per-candidate draws and c = 0x80000000 | chunk for the per-chunk merge draws. */
static uint64_t draw_rc(uint64_t seed, uint64_t sid, uint32_t d, uint32_t c) {
    uint32_t ctr[4] = {(uint32_t)sid, (uint32_t)(sid >> 32), d, c};
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t x[4];
    or_philox4x32_10(ctr, key, x);
    return ((uint64_t)x[1] << 32) | (uint64_t)x[0];
}

static uint64_t draw_r(uint64_t seed, uint64_t sid, uint32_t d) { return draw_rc(seed, sid, d, 0u); }

/* uniform index in [0, c): floor(r * c / 2^64) */
static uint64_t uniform_index(uint64_t r, uint64_t c) {
    return (uint64_t)(((unsigned __int128)r * (unsigned __int128)c) >> 64);
}

uint64_t or_uniform_index(uint64_t seed, uint64_t sid, uint32_t d, uint64_t c) {
    return uniform_index(draw_r(seed, sid, d), c);
}

/* ---- graph / query --------------------------------------------------------------- */
typedef struct {
    int64_t n;
    const int64_t* row_ptr;
    const int32_t* col;
    const int32_t* labels; /* never NULL here: the wrapper passes zeros when unlabelled */
} or_graph;

typedef struct {
    int32_t nq;
    int32_t adj[OR_MAX_QV][OR_MAX_QV]; /* query-vertex adjacency */
    int32_t label[OR_MAX_QV];          /* L_q(u) */
    int32_t order[OR_MAX_QV];          /* phi */
} or_query;

static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

static int contains(const int32_t* list, int64_t len, int32_t x) {
    if (len <= 0) return 0;
    return bsearch(&x, list, (size_t)len, sizeof(int32_t), cmp_i32) != NULL;
}

/* Global candidate sets C(u) (Def. 4): inC[u * n + v] = 1 iff v in C(u).
 * filter 0: label only, C(u) = {v : L(v) = L_q(u)}            (reading A2)
 * filter 1: + degree, deg(v) >= deg_q(u)                       (LDF, reading A21)
 * filter 2: + for every label l, |N_l(v)| >= |N_l^q(u)|         (NLF, reading A21)
 * Each is a superset of the vertices u can map to in an embedding. */
static void candidate_sets(const or_graph* G, const or_query* Q, int filter, uint8_t* inC) {
    for (int u = 0; u < Q->nq; ++u) {
        int deg_q = 0;
        for (int w = 0; w < Q->nq; ++w) deg_q += Q->adj[u][w] ? 1 : 0;
        for (int64_t v = 0; v < G->n; ++v) {
            int ok = G->labels[v] == Q->label[u];
            if (ok && filter >= 1) ok = (G->row_ptr[v + 1] - G->row_ptr[v]) >= deg_q;
            if (ok && filter >= 2) {
                for (int w = 0; w < Q->nq && ok; ++w) {
                    if (!Q->adj[u][w]) continue;
                    int32_t l = Q->label[w];
                    int need = 0;
                    for (int x = 0; x < Q->nq; ++x)
                        if (Q->adj[u][x] && Q->label[x] == l) need += 1;
                    int64_t have = 0;
                    for (int64_t i = G->row_ptr[v]; i < G->row_ptr[v + 1]; ++i)
                        if (G->labels[G->col[i]] == l) have += 1;
                    ok = have >= need;
                }
            }
            inC[(int64_t)u * G->n + v] = (uint8_t)ok;
        }
    }
}

/* Local candidate set C(u', u, v) = N(v) ∩ C(u), ascending id (Def. 4; A2/A4).
 * `inCu` is the membership row of C(u).  Returns its size. */
static int64_t local_candidates(const or_graph* G, int32_t v, const uint8_t* inCu, int32_t* out) {
    int64_t len = 0;
    for (int64_t i = G->row_ptr[v]; i < G->row_ptr[v + 1]; ++i) {
        int32_t w = G->col[i];
        if (inCu[w]) out[len++] = w;
    }
    return len;
}

/* ---- one sample (Alg. 1 inner loop) --------------------------------- */
/* One position d of a sample (method 0 = WanderJoin, 1 = Alley): forms C_d from the
 * matched prefix M[0..d-1], draws M[d] with r(sid, d), multiplies *W by |C_d| (the running
 * product of Eq. 1 in depth order, reading A7; *W starts as |C_0| at d = 0) and validates.
 * Returns 1 if M[0..d] is still a valid partial instance, 0 if the sample died here. */
/* Per-call flags of the sampler (readings A3, A5, A25):
 *   OR_SELECT_STREAM        Alley draws by warp streaming (Alg. 3) instead of count-then-index
 *   OR_WJ_PARENT_FIRST      WanderJoin walks from the FIRST backward position's list instead
 *                           of the smallest (the "previously selected vertex" of P:L538)
 *   OR_ALLEY_DUPCHECK_POST  Alley's refine keeps matched vertices; a drawn matched vertex
 *                           kills the sample (Fig. 19 AL Validate/DupCheck) */
#define OR_SELECT_STREAM 1
#define OR_WJ_PARENT_FIRST 2
#define OR_ALLEY_DUPCHECK_POST 4

/* Alley refine predicate (Fig. 19 AL; reading A5): x of the driver list S[p]
 * lies in every other local list and (unless the DupCheck is deferred to after sampling) is
 * not an already-matched vertex. */
static int alley_keep(int32_t x, int32_t** S, const int64_t* len, int nb, int p, const int32_t* M, int d,
                      int check_matched) {
    for (int b = 0; b < nb; ++b) {
        if (b == p) continue;
        if (!contains(S[b], len[b], x)) return 0;
    }
    if (check_matched)
        for (int j = 0; j < d; ++j)
            if (M[j] == x) return 0;
    return 1;
}

/* Warp streaming (Alg. 3; reading A25): Refine and Sample of one Alley position
 * streamed over the driver list cand[0..clen) with the weighted reservoir of A-Res.  Every
 * candidate has weight w = 1 if it passes refine, else 0, so its A-Res key u^(1/w) is u.
 * Collaborative phase (l.5-17) while at least 32 candidates remain: the 32 "workers" take
 * cand[it .. it+32), the survivor with the largest key is the chunk's pick (ties -> lowest
 * worker), totalW = survivors, curTotalW += totalW, and the pick replaces curV with
 * probability totalW / curTotalW.  Independent phase (l.18-22): one candidate at a time,
 * curTotalW += w, replace with probability w / curTotalW.  "With probability a / b" is
 * mulhi64(u, b) < a for a fresh draw u.  Returns curTotalW (= |C_d|, Theorem 2) and the
 * pick in *v (-1 when curTotalW = 0). */
static int64_t stream_select(uint64_t seed, uint64_t sid, int d, const int32_t* cand, int64_t clen, int32_t** S,
                             const int64_t* len, int nb, int p, const int32_t* M, int check_matched, int32_t* v) {
    int64_t cur_iter = 0;         /* l.1 */
    int32_t cur_v = -1;           /* l.2 (dummy) */
    uint64_t cur_total = 0;       /* l.4 (curW is 1 for every pick: the weights are 0/1) */
    uint32_t chunk = 0;
    while (clen - cur_iter >= 32) {                          /* l.5 */
        int best = -1;
        uint64_t best_key = 0, total = 0;
        for (int t = 0; t < 32; ++t) {                       /* worker t: cand[cur_iter + t] (l.8) */
            int32_t x = cand[cur_iter + t];
            if (!alley_keep(x, S, len, nb, p, M, d, check_matched)) continue;  /* l.9-10: w = 0 */
            total += 1;
            uint64_t key = draw_rc(seed, sid, (uint32_t)d, (uint32_t)(1 + cur_iter + t));  /* l.11 */
            if (best < 0 || key > best_key) { best = t; best_key = key; }                 /* l.12 */
        }
        cur_total += total;                                   /* l.13-15 */
        if (total > 0 &&
            uniform_index(draw_rc(seed, sid, (uint32_t)d, 0x80000000u | chunk), cur_total) < total)  /* l.16 */
            cur_v = cand[cur_iter + best];
        cur_iter += 32;                                       /* l.17 */
        chunk += 1;
    }
    while (cur_iter < clen) {                                 /* l.18 */
        int32_t x = cand[cur_iter];
        if (alley_keep(x, S, len, nb, p, M, d, check_matched)) {  /* l.19-20: w = 1 */
            cur_total += 1;                                   /* l.21 */
            if (uniform_index(draw_rc(seed, sid, (uint32_t)d, (uint32_t)(1 + cur_iter)), cur_total) < 1)
                cur_v = x;                                    /* l.22: with probability 1 / curTotalW */
        }
        cur_iter += 1;
    }
    *v = cur_v;
    return (int64_t)cur_total;
}

/* ---- algorithmic sectors (SURVEY §8(d) measurement; reading A26 of DESIGN.md §3) -----
 * The memory the method itself must read, in 32-byte sectors, counted for every position a
 * sample starts alive (one local-candidate list = one contiguous ascending run of 4-byte ids
 * whose start/end offsets sit in one 8-byte record; a membership question "x in C(u,u',v)?"
 * costs ONE sector: one probe of an exact index, the minimum for a random question):
 *   d = 0      1 sector to read the drawn seed from the stored list C(phi[0]); 0 when
 *              C(phi[0]) is all of V (M[0] = k needs no memory) or empty.
 *   d >= 1     |B(d)| sectors for the offsets of the local lists S_j (GetMinCandidate;
 *              WanderJoin's first-parent variant reads only the parent's: 1).
 *   WanderJoin +1 for the drawn vertex when |C_d| > 0; then, if it passes DupCheck (registers),
 *              +1 per IsEdge question in ascending backward position up to the first "no".
 *   Alley, |B(d)| = 1: if S_p is not empty, +1 per exclusion question "is M[j] in S_p?" for
 *              every matched j != p with L_q(phi[j]) = L_q(phi[d]), except (label-only lists) when
 *              (phi[j], phi[p]) is a query edge: then M[j] lies in S_p because the prefix is a
 *              partial instance; +1 for the selected vertex when |C_d| > 0 (its index follows
 *              from k and the excluded vertices; the list itself is not scanned).
 *   Alley, |B(d)| >= 2 and |S_p| > 0: ceil(|S_p| / 8) sectors to scan the driver list S_p; for
 *              each driver element that is not a matched vertex (registers), +1 per membership
 *              question in the other lists in ascending backward position up to the first "no";
 *              the selected vertex is already in registers (0).
 *   Alley by warp streaming (OR_SELECT_STREAM): not modelled, the record holds 0.
 * Post-draw DupChecks (variant A5) and the HT update cost nothing. */
static uint32_t div_up8(int64_t len) { return (uint32_t)((len + 7) / 8); }

/* One position d of a sample (method 0 = WanderJoin, 1 = Alley): forms C_d from the
 * matched prefix M[0..d-1], draws M[d] with r(sid, d), multiplies *W by |C_d| (the running
 * product of Eq. 1 in depth order, reading A7; *W starts as |C_0| at d = 0) and validates.
 * `flags`: OR_* above (0 = the default sampler).  `filter` is the candidate filter (0 =
 * label only); it only enters the sector count.  Returns 1 if M[0..d] is still a valid
 * partial instance, 0 if the sample died here.  rec->sectors accumulates the model above. */
static int step_at(const or_graph* G, const or_query* Q, int method, int flags, int filter, uint64_t seed,
                   uint64_t sid, int d, const int32_t* C0, int64_t C0_len, const uint8_t* inC, int32_t** S,
                   int32_t* refine, int32_t* M, double* W, or_record* rec) {
    uint32_t sec_unused = 0;
    uint32_t* sec = rec ? &rec->sectors : &sec_unused;
    if (d == 0) {
        /* seed from the global candidate set C(phi[0]) */
        *W = (double)C0_len;
        if (C0_len == 0) return 0;
        uint64_t k = uniform_index(draw_r(seed, sid, 0), (uint64_t)C0_len);
        M[0] = C0[k];
        if (C0_len != G->n) *sec += 1; /* A26: the seed list is read unless it is all of V */
        if (rec) { rec->path[0] = M[0]; rec->csize[0] = (uint32_t)C0_len; }
        return 1;
    }
    int32_t u = Q->order[d];
    /* backward positions B(d) = { j < d : (phi[j], phi[d]) in E_q } */
    int B[OR_MAX_QV], nb = 0;
    for (int j = 0; j < d; ++j)
        if (Q->adj[Q->order[j]][u]) B[nb++] = j;
    /* GetMinCandidate (Alg. 1 l.8): local lists S_j of every matched neighbour,
     * p = the smallest one, ties -> smallest position j (reading A3) */
    int64_t len[OR_MAX_QV];
    int p = 0;
    for (int b = 0; b < nb; ++b) {
        len[b] = local_candidates(G, M[B[b]], inC + (int64_t)u * G->n, S[b]);
        if (len[b] < len[p]) p = b;
    }
    if (method == 0 && (flags & OR_WJ_PARENT_FIRST)) p = 0; /* variant: first backward position */
    /* A26: the offsets of every local list GetMinCandidate compares (first-parent: one) */
    *sec += (method == 0 && (flags & OR_WJ_PARENT_FIRST)) ? 1u : (uint32_t)nb;
    int64_t clen;
    const int32_t* cand = S[p];
    if (method == 0) {
        /* WanderJoin Refine: refine = cand (Fig. 19 WJ) */
        clen = len[p];
        *W = *W * (double)clen;
        if (clen == 0) return 0;
        /* Sample: uniform vertex of refine, prob 1/rlen */
        uint64_t k = uniform_index(draw_r(seed, sid, (uint32_t)d), (uint64_t)clen);
        int32_t v = cand[k];
        M[d] = v;
        *sec += 1; /* A26: the drawn vertex */
        if (rec) { rec->path[d] = v; rec->csize[d] = (uint32_t)clen; }
        /* Validate: DupCheck against all matched vertices, IsEdge for every other
         * matched query neighbour */
        for (int j = 0; j < d; ++j)
            if (M[j] == v) return 0;
        for (int b = 0; b < nb; ++b) {
            if (b == p) continue;
            *sec += 1; /* A26: one IsEdge question */
            if (!contains(S[b], len[b], v)) return 0;
        }
        return 1;
    }
    const int post = (flags & OR_ALLEY_DUPCHECK_POST) != 0;
    int32_t v = -1;
    if (flags & OR_SELECT_STREAM) {
        clen = stream_select(seed, sid, d, cand, len[p], S, len, nb, p, M, !post, &v);
    } else {
        /* Alley Refine: keep each x of cand that lies in every other local list and is not
         * already matched (Fig. 19 AL; reading A5) */
        clen = 0;
        for (int64_t i = 0; i < len[p]; ++i) {
            int32_t x = cand[i];
            if (alley_keep(x, S, len, nb, p, M, d, !post)) refine[clen++] = x;
        }
        if (clen > 0) v = refine[uniform_index(draw_r(seed, sid, (uint32_t)d), (uint64_t)clen)];
        /* A26: sectors of this refine + select */
        if (nb == 1) {
            if (!post && len[p] > 0) /* no question is needed about an empty S_p */
                for (int j = 0; j < d; ++j) {
                    if (j == B[p] || Q->label[Q->order[j]] != Q->label[u]) continue;
                    if (filter == 0 && Q->adj[Q->order[j]][Q->order[B[p]]]) continue; /* M[j] in S_p */
                    *sec += 1; /* exclusion question "is M[j] in S_p?" */
                }
            if (clen > 0) *sec += 1; /* the selected vertex */
        } else if (len[p] > 0) {
            *sec += div_up8(len[p]); /* driver scan */
            for (int64_t i = 0; i < len[p]; ++i) {
                int32_t x = cand[i];
                int matched = 0;
                for (int j = 0; j < d && !post; ++j) matched |= M[j] == x;
                if (matched) continue;
                for (int b = 0; b < nb; ++b) {
                    if (b == p) continue;
                    *sec += 1; /* membership question "is x in S_b?" */
                    if (!contains(S[b], len[b], x)) break;
                }
            }
        }
    }
    *W = *W * (double)clen;
    /* empty refined set: the sample stops */
    if (clen == 0) return 0;
    M[d] = v;
    if (rec) { rec->path[d] = v; rec->csize[d] = (uint32_t)clen; }
    if (post) /* Fig. 19 AL Validate: DupCheck of the drawn vertex */
        for (int j = 0; j < d; ++j)
            if (M[j] == v) return 0;
    return 1;
}

/* Samples positions 0 .. stop-1 (stop = |V_q| for the plain estimator; the trawling
 * prefix length d otherwise).  Returns Y = W if all `stop` positions were matched, else 0;
 * M and W are left in *Mout / *Wout. */
static double walk(const or_graph* G, const or_query* Q, int method, int flags, int filter, uint64_t seed,
                   uint64_t sid, int stop,
                   const int32_t* C0, int64_t C0_len, const uint8_t* inC, int32_t** S, int32_t* refine,
                   or_record* rec, int32_t* Mout, double* Wout) {
    int32_t M[OR_MAX_QV] = {0};
    double W = 0.0;
    int valid = 1, depth_reached = 0;
    if (rec) {
        memset(rec, 0, sizeof(*rec));
        rec->sample_id = sid;
        for (int i = 0; i < OR_MAX_QV; ++i) rec->path[i] = -1;
    }
    for (int d = 0; d < stop && valid; ++d) {
        depth_reached = d;
        valid = step_at(G, Q, method, flags, filter, seed, sid, d, C0, C0_len, inC, S, refine, M, &W, rec);
    }
    if (rec) {
        if (method == 1 && (flags & OR_SELECT_STREAM)) rec->sectors = 0; /* A26: not modelled */
        rec->valid = (uint8_t)valid;
        rec->depth_reached = (uint8_t)depth_reached;
        rec->weight = W;
    }
    if (Mout) memcpy(Mout, M, sizeof(M));
    if (Wout) *Wout = W;
    return valid ? W : 0.0;
}

static double one_sample(const or_graph* G, const or_query* Q, int method, int flags, int filter, uint64_t seed,
                         uint64_t sid,
                         const int32_t* C0, int64_t C0_len, const uint8_t* inC, int32_t** S, int32_t* refine,
                         or_record* rec) {
    return walk(G, Q, method, flags, filter, seed, sid, Q->nq, C0, C0_len, inC, S, refine, rec, NULL, NULL);
}

static int load_query(or_query* Q, int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col,
                      const int32_t* q_labels, const int32_t* order) {
    if (nq < 1 || nq > OR_MAX_QV) return -1;
    memset(Q, 0, sizeof(*Q));
    Q->nq = nq;
    for (int u = 0; u < nq; ++u) {
        Q->label[u] = q_labels[u];
        Q->order[u] = order[u];
        for (int32_t i = q_row_ptr[u]; i < q_row_ptr[u + 1]; ++i) Q->adj[u][q_col[i]] = 1;
    }
    /* every prefix of the matching order must be connected (reading A13) */
    for (int d = 1; d < nq; ++d) {
        int has = 0;
        for (int j = 0; j < d; ++j) has |= Q->adj[Q->order[j]][Q->order[d]];
        if (!has) return -2;
    }
    return 0;
}

/*
 * Run samples [first, first + count).  y_out[i] = Y of sample first+i (may be NULL);
 * rec_out[i] = its record (may be NULL).  Returns 0, or -1 on bad input / OOM.
 */
/* Candidate sets of `filter` for every query vertex: out[u * n + v] (nq * n bytes). */
int or_candidate_sets(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int filter, uint8_t* out) {
    or_graph G = {n, row_ptr, col, labels};
    or_query Q;
    int rc = load_query(&Q, nq, q_row_ptr, q_col, q_labels, order);
    if (rc) return rc;
    candidate_sets(&G, &Q, filter, out);
    return 0;
}

int or_sample_range_f(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                      double* y_out, or_record* rec_out, int filter);

int or_sample_range(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                    int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                    const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                    double* y_out, or_record* rec_out) {
    return or_sample_range_f(n, row_ptr, col, labels, nq, q_row_ptr, q_col, q_labels, order, method, seed, first,
                             count, y_out, rec_out, 0);
}

int or_sample_range_v(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                      double* y_out, or_record* rec_out, int filter, int flags);

int or_sample_range_mt(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                       int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                       const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                       double* y_out, or_record* rec_out, int filter, int flags, int threads, uint64_t chunk);

/* Run samples [first, first + count) with the candidate sets of `filter`. */
int or_sample_range_f(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                      double* y_out, or_record* rec_out, int filter) {
    return or_sample_range_v(n, row_ptr, col, labels, nq, q_row_ptr, q_col, q_labels, order, method, seed, first,
                             count, y_out, rec_out, filter, 0);
}

/* ... and the sampler flags OR_* (streaming selection, readings A3/A5 variants). */
int or_sample_range_v(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                      int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                      double* y_out, or_record* rec_out, int filter, int flags) {
    return or_sample_range_mt(n, row_ptr, col, labels, nq, q_row_ptr, q_col, q_labels, order, method, seed, first,
                              count, y_out, rec_out, filter, flags, 1, count);
}

/* Shared, read-only state of one call: the graph, the query, the candidate sets of the
 * filter and the seed list C(phi[0]) (built once per call), and the dynamic schedule. */
typedef struct {
    or_graph G;
    or_query Q;
    int method, flags, filter;
    uint64_t seed, first, count, chunk;
    const int32_t* C0;
    int64_t C0_len;
    const uint8_t* inC;
    int64_t maxdeg;
    double* y_out;
    or_record* rec_out;
    _Atomic uint64_t next;   /* next unclaimed offset in [0, count) */
    _Atomic int failed;
} range_job;

/* One worker: claims chunks of sample ids in order of the shared counter (the dynamic
 * scheduling of the paper's CPU baselines) and runs each sample plainly. */
static void* range_worker(void* arg) {
    range_job* J = (range_job*)arg;
    int32_t* buf = (int32_t*)malloc(sizeof(int32_t) * (size_t)(J->maxdeg + 1) * (OR_MAX_QV + 1));
    if (!buf) { J->failed = 1; return NULL; }
    int32_t* S[OR_MAX_QV];
    for (int b = 0; b < OR_MAX_QV; ++b) S[b] = buf + (size_t)b * (size_t)(J->maxdeg + 1);
    int32_t* refine = buf + (size_t)OR_MAX_QV * (size_t)(J->maxdeg + 1);
    for (;;) {
        uint64_t a = atomic_fetch_add(&J->next, J->chunk);
        if (a >= J->count) break;
        uint64_t b = a + J->chunk < J->count ? a + J->chunk : J->count;
        for (uint64_t i = a; i < b; ++i) {
            double y = one_sample(&J->G, &J->Q, J->method, J->flags, J->filter, J->seed, J->first + i, J->C0,
                                  J->C0_len, J->inC, S, refine, J->rec_out ? &J->rec_out[i] : NULL);
            if (J->y_out) J->y_out[i] = y;
        }
    }
    free(buf);
    return NULL;
}

/* Run samples [first, first + count) on `threads` host threads, chunks of `chunk` ids. */
int or_sample_range_mt(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                       int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                       const int32_t* order, int method, uint64_t seed, uint64_t first, uint64_t count,
                       double* y_out, or_record* rec_out, int filter, int flags, int threads, uint64_t chunk) {
    range_job J;
    memset(&J, 0, sizeof(J));
    J.G = (or_graph){n, row_ptr, col, labels};
    int rc = load_query(&J.Q, nq, q_row_ptr, q_col, q_labels, order);
    if (rc) return rc;
    if (threads < 1) threads = 1;
    if (threads > 256) threads = 256;
    J.method = method;
    J.flags = flags;
    J.filter = filter;
    J.seed = seed;
    J.first = first;
    J.count = count;
    J.chunk = chunk > 0 ? chunk : 1;
    J.y_out = y_out;
    J.rec_out = rec_out;
    atomic_init(&J.next, 0);
    atomic_init(&J.failed, 0);
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] - row_ptr[v] > J.maxdeg) J.maxdeg = row_ptr[v + 1] - row_ptr[v];
    int32_t* C0 = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    uint8_t* inC = (uint8_t*)malloc((size_t)(n > 0 ? n : 1) * (size_t)nq);
    if (!C0 || !inC) { free(C0); free(inC); return -1; }
    candidate_sets(&J.G, &J.Q, filter, inC);
    /* global candidate set of phi[0], ascending */
    int64_t C0_len = 0;
    const uint8_t* in0 = inC + (int64_t)J.Q.order[0] * n;
    for (int64_t v = 0; v < n; ++v)
        if (in0[v]) C0[C0_len++] = (int32_t)v;
    J.C0 = C0;
    J.C0_len = C0_len;
    J.inC = inC;
    if (threads == 1) {
        range_worker(&J);
    } else {
        pthread_t tid[256];
        int started = 0;
        for (; started < threads; ++started)
            if (pthread_create(&tid[started], NULL, range_worker, &J) != 0) break;
        if (started == 0) range_worker(&J);
        for (int t = 0; t < started; ++t) pthread_join(tid[t], NULL);
    }
    free(inC);
    free(C0);
    return atomic_load(&J.failed) ? -1 : 0;
}

/* ---- exact count of embeddings by plain backtracking (reading A1) --------------- */
typedef struct {
    const or_graph* G;
    const or_query* Q;
    int32_t M[OR_MAX_QV];
    unsigned __int128 count;
    int overflow;
} enum_state;

static int is_edge(const or_graph* G, int32_t a, int32_t b) {
    return contains(G->col + G->row_ptr[a], G->row_ptr[a + 1] - G->row_ptr[a], b);
}

static void extend(enum_state* st, int d) {
    const or_query* Q = st->Q;
    const or_graph* G = st->G;
    if (d == Q->nq) {
        st->count += 1;
        return;
    }
    int32_t u = Q->order[d];
    /* candidates: any vertex with the right label for d = 0; otherwise the neighbours
     * of the first matched query neighbour (every embedding is reached exactly once) */
    int jfirst = -1;
    for (int j = 0; j < d && jfirst < 0; ++j)
        if (Q->adj[Q->order[j]][u]) jfirst = j;
    int64_t lo, hi;
    if (d == 0) { lo = 0; hi = G->n; }
    else { lo = G->row_ptr[st->M[jfirst]]; hi = G->row_ptr[st->M[jfirst] + 1]; }
    for (int64_t i = lo; i < hi; ++i) {
        int32_t v = (d == 0) ? (int32_t)i : G->col[i];
        if (G->labels[v] != Q->label[u]) continue;
        int ok = 1;
        for (int j = 0; j < d && ok; ++j) {
            if (st->M[j] == v) ok = 0;
            else if (Q->adj[Q->order[j]][u] && !is_edge(G, st->M[j], v)) ok = 0;
        }
        if (!ok) continue;
        st->M[d] = v;
        extend(st, d + 1);
    }
}

/* count_out = low 64 bits, count_hi = high 64 bits of the 128-bit count. */
int or_count_embeddings(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                        int32_t nq, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                        const int32_t* order, uint64_t* count_lo, uint64_t* count_hi) {
    or_graph G = {n, row_ptr, col, labels};
    or_query Q;
    int rc = load_query(&Q, nq, q_row_ptr, q_col, q_labels, order);
    if (rc) return rc;
    enum_state st;
    memset(&st, 0, sizeof(st));
    st.G = &G;
    st.Q = &Q;
    extend(&st, 0);
    *count_lo = (uint64_t)st.count;
    *count_hi = (uint64_t)(st.count >> 64);
    return 0;
}

/* ---- trawling (Alg. 4; NEXT-2, reading A23) --------------------------- */
typedef struct {
    uint64_t sample_id;
    uint8_t status; /* 0 prefix died (T = 0), 1 enumerated, 2 enumeration budget exceeded */
    uint8_t d;      /* number of sampled vertices */
    uint8_t pad[6];
    int32_t path[OR_MAX_QV];
    uint32_t csize[OR_MAX_QV];
    double weight;  /* W_d = prod_{j<d} |C_j| (running product) */
    uint64_t count; /* completions of the sampled partial instance */
    uint64_t nodes; /* enumeration nodes visited */
} or_trawl_record; /* 168 bytes */

/* d ~ P(d = j) proportional to 2^-j, j in [3, |V_q|], drawn exactly in integers:
 * weights 2^(nq-j), total 2^(nq-2) - 1, index = mulhi64(r(sid, 31), total). */
static int choose_d(uint64_t seed, uint64_t sid, int nq) {
    if (nq <= 3) return nq;
    uint64_t total = (1ull << (nq - 2)) - 1ull;
    uint64_t k = uniform_index(draw_r(seed, sid, 31u), total);
    uint64_t acc = 0;
    for (int j = 3; j <= nq; ++j) {
        acc += 1ull << (nq - j);
        if (k < acc) return j;
    }
    return nq;
}

typedef struct {
    const or_graph* G;
    const or_query* Q;
    const uint8_t* inC;
    int32_t M[OR_MAX_QV];
    int32_t* buf; /* per (level, backward slot) candidate lists */
    int64_t stride;
    uint64_t count, nodes, budget;
    int timeout;
} trawl_state;

/* Count the completions of M[0..t-1]: every extension keeps a partial instance, so the
 * candidates at t are the Alley refine set (intersection of the local candidate lists of
 * the matched query neighbours, minus matched vertices), enumerated in ascending order. */
static void enumerate_completions(trawl_state* st, int t) {
    const or_query* Q = st->Q;
    if (st->timeout) return;
    if (t == Q->nq) {
        st->count += 1;
        return;
    }
    int32_t u = Q->order[t];
    int B[OR_MAX_QV], nb = 0;
    for (int j = 0; j < t; ++j)
        if (Q->adj[Q->order[j]][u]) B[nb++] = j;
    int64_t len[OR_MAX_QV];
    int32_t* S[OR_MAX_QV];
    int p = 0;
    for (int b = 0; b < nb; ++b) {
        S[b] = st->buf + ((int64_t)t * OR_MAX_QV + b) * st->stride;
        len[b] = local_candidates(st->G, st->M[B[b]], st->inC + (int64_t)u * st->G->n, S[b]);
        if (len[b] < len[p]) p = b;
    }
    for (int64_t i = 0; i < len[p]; ++i) {
        int32_t x = S[p][i];
        int keep = 1;
        for (int b = 0; b < nb && keep; ++b)
            if (b != p && !contains(S[b], len[b], x)) keep = 0;
        for (int j = 0; j < t && keep; ++j)
            if (st->M[j] == x) keep = 0;
        if (!keep) continue;
        if (st->nodes == st->budget) {
            st->timeout = 1;
            return;
        }
        st->nodes += 1;
        st->M[t] = x;
        enumerate_completions(st, t + 1);
        if (st->timeout) return;
    }
}

/* Trawling samples [first, first + count): t_out[i] = T_i = W_d * cnt (0 when the prefix
 * dies), status_out[i] as or_trawl_record.status, rec_out optional. */
int or_trawl_range(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int32_t nq,
                   const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels, const int32_t* order,
                   int method, uint64_t seed, uint64_t first, uint64_t count, uint64_t budget, int filter,
                   double* t_out, uint8_t* status_out, or_trawl_record* rec_out) {
    or_graph G = {n, row_ptr, col, labels};
    or_query Q;
    int rc = load_query(&Q, nq, q_row_ptr, q_col, q_labels, order);
    if (rc) return rc;
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] - row_ptr[v] > maxdeg) maxdeg = row_ptr[v + 1] - row_ptr[v];
    int64_t stride = maxdeg + 1;
    int32_t* C0 = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t* buf = (int32_t*)malloc(sizeof(int32_t) * (size_t)stride * (OR_MAX_QV + 1));
    int32_t* ebuf = (int32_t*)malloc(sizeof(int32_t) * (size_t)stride * OR_MAX_QV * OR_MAX_QV);
    uint8_t* inC = (uint8_t*)malloc((size_t)(n > 0 ? n : 1) * (size_t)nq);
    if (!C0 || !buf || !ebuf || !inC) { free(C0); free(buf); free(ebuf); free(inC); return -1; }
    candidate_sets(&G, &Q, filter, inC);
    int64_t C0_len = 0;
    const uint8_t* in0 = inC + (int64_t)Q.order[0] * n;
    for (int64_t v = 0; v < n; ++v)
        if (in0[v]) C0[C0_len++] = (int32_t)v;
    int32_t* S[OR_MAX_QV];
    for (int b = 0; b < OR_MAX_QV; ++b) S[b] = buf + (size_t)b * (size_t)stride;
    int32_t* refine = buf + (size_t)OR_MAX_QV * (size_t)stride;
    for (uint64_t i = 0; i < count; ++i) {
        uint64_t sid = first + i;
        int d = choose_d(seed, sid, nq);
        or_record r;
        trawl_state st;
        memset(&st, 0, sizeof(st));
        double W = 0.0;
        double y = walk(&G, &Q, method, 0, filter, seed, sid, d, C0, C0_len, inC, S, refine, &r, st.M, &W);
        uint8_t status = 0;
        double t = 0.0;
        if (r.valid) {
            st.G = &G;
            st.Q = &Q;
            st.inC = inC;
            st.buf = ebuf;
            st.stride = stride;
            st.budget = budget;
            enumerate_completions(&st, d);
            status = st.timeout ? 2 : 1;
            t = st.timeout ? 0.0 : y * (double)st.count;
        }
        if (t_out) t_out[i] = t;
        if (status_out) status_out[i] = status;
        if (rec_out) {
            or_trawl_record* o = &rec_out[i];
            memset(o, 0, sizeof(*o));
            o->sample_id = sid;
            o->status = status;
            o->d = (uint8_t)d;
            memcpy(o->path, r.path, sizeof(o->path));
            memcpy(o->csize, r.csize, sizeof(o->csize));
            o->weight = W;
            o->count = st.count;
            o->nodes = st.nodes;
        }
    }
    free(C0);
    free(buf);
    free(ebuf);
    free(inC);
    return 0;
}

int or_trawl_record_size(void) { return (int)sizeof(or_trawl_record); }

/* ---- sample inheritance (Alg. 2; NEXT-3, reading A24) ------------------- */
/* Groups of 32 consecutive sample ids [first + 32g, first + 32g + 32) run in lock step, one
 * position per round (sample synchronisation).  After a round that is not the last,
 * if some group members hold a valid partial sample and others do not, every member without
 * one inherits the valid sample of the lowest such member (the parent, Alg. 2 l.2), and the
 * parent and its k copies all carry W / (k + 1) (the push-down of the recursive estimator,
 * P:L902-L910).  A copy keeps drawing with its own sample id.  group_out[g] = the sum of
 * the weights of the complete instances of group g; *n_complete counts those instances. */
int or_inherit_range_v(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int32_t nq,
                       const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels, const int32_t* order,
                       int method, uint64_t seed, uint64_t first, uint64_t count, int filter, double* group_out,
                       uint64_t* n_complete, int flags);

int or_inherit_range(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int32_t nq,
                     const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels, const int32_t* order,
                     int method, uint64_t seed, uint64_t first, uint64_t count, int filter, double* group_out,
                     uint64_t* n_complete) {
    return or_inherit_range_v(n, row_ptr, col, labels, nq, q_row_ptr, q_col, q_labels, order, method, seed, first,
                              count, filter, group_out, n_complete, 0);
}

/* ... with the sampler flags OR_* (inheritance + warp streaming = the paper's O2). */
int or_inherit_range_v(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* labels, int32_t nq,
                       const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels, const int32_t* order,
                       int method, uint64_t seed, uint64_t first, uint64_t count, int filter, double* group_out,
                       uint64_t* n_complete, int flags) {
    or_graph G = {n, row_ptr, col, labels};
    or_query Q;
    int rc = load_query(&Q, nq, q_row_ptr, q_col, q_labels, order);
    if (rc) return rc;
    int64_t maxdeg = 0;
    for (int64_t v = 0; v < n; ++v)
        if (row_ptr[v + 1] - row_ptr[v] > maxdeg) maxdeg = row_ptr[v + 1] - row_ptr[v];
    int64_t stride = maxdeg + 1;
    int32_t* C0 = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t* buf = (int32_t*)malloc(sizeof(int32_t) * (size_t)stride * (OR_MAX_QV + 1));
    uint8_t* inC = (uint8_t*)malloc((size_t)(n > 0 ? n : 1) * (size_t)nq);
    if (!C0 || !buf || !inC) { free(C0); free(buf); free(inC); return -1; }
    candidate_sets(&G, &Q, filter, inC);
    int64_t C0_len = 0;
    const uint8_t* in0 = inC + (int64_t)Q.order[0] * n;
    for (int64_t v = 0; v < n; ++v)
        if (in0[v]) C0[C0_len++] = (int32_t)v;
    int32_t* S[OR_MAX_QV];
    for (int b = 0; b < OR_MAX_QV; ++b) S[b] = buf + (size_t)b * (size_t)stride;
    int32_t* refine = buf + (size_t)OR_MAX_QV * (size_t)stride;
    uint64_t completes = 0;
    uint64_t g = 0;
    for (uint64_t g0 = 0; g0 < count; g0 += 32, ++g) {
        int L = (int)((count - g0) < 32 ? (count - g0) : 32);
        int32_t M[32][OR_MAX_QV];
        double W[32];
        int alive[32];
        double total = 0.0;
        for (int l = 0; l < L; ++l) alive[l] = 1;
        for (int d = 0; d < nq; ++d) {
            int any = 0;
            for (int l = 0; l < L; ++l) {
                if (!alive[l]) continue;
                alive[l] = step_at(&G, &Q, method, flags, filter, seed, first + g0 + (uint64_t)l, d, C0, C0_len, inC, S,
                                   refine,
                                   M[l], &W[l], NULL);
                any |= alive[l];
            }
            if (!any) break;
            if (d == nq - 1) {
                for (int l = 0; l < L; ++l)
                    if (alive[l]) { total += W[l]; completes += 1; }
                break;
            }
            int parent = -1, k = 0;
            for (int l = 0; l < L; ++l) {
                if (alive[l] && parent < 0) parent = l;
                if (!alive[l]) k += 1;
            }
            if (k > 0) {
                double Wn = W[parent] / (double)(k + 1);
                W[parent] = Wn;
                for (int l = 0; l < L; ++l) {
                    if (alive[l]) continue;
                    memcpy(M[l], M[parent], sizeof(int32_t) * (size_t)(d + 1));
                    W[l] = Wn;
                    alive[l] = 1;
                }
            }
        }
        group_out[g] = total;
    }
    *n_complete = completes;
    free(C0);
    free(buf);
    free(inC);
    return 0;
}

int or_record_size(void) { return (int)sizeof(or_record); }
