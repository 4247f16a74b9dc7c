/*
 * gsword.h — C ABI of the B200-native gSWORD hot path: the WanderJoin / Alley
 * random-walk estimator of the number of embeddings of a labelled query graph q in a
 * labelled data graph G, with Horvitz-Thompson aggregation.
 *
 * Citations: P:L<n> = line n of PAPER.md (the gSWORD paper, PACMMOD 2024);
 * readings A<n> = DESIGN.md §3 (where the paper is silent or garbled).
 *
 * Conventions for every entry point
 *   - Return value: GSWORD_OK (0) on success, a negative gsword_status on error; the
 *     thread-local message of the last error is available from gsword_last_error().
 *   - Host pointers are borrowed for the duration of the call only and are never
 *     written unless documented as outputs.  The context owns every device buffer it
 *     allocates; nothing is freed by the caller.
 *   - A context is bound to one CUDA device and is not thread-safe.  All device work
 *     is issued on the context's stream (gsword_set_stream), in stream order.
 *   - Results are a pure function of (graph, query, matching order, method, seed,
 *     first sample id, sample count); the scheduling of samples onto the GPU does not
 *     change any per-sample result, and aggregates agree to a relative 1e-12.
 */
#ifndef GSWORD_H
#define GSWORD_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GSWORD_MAX_QV 16 /* largest query (P:L1055 uses 4/8/16 vertices; reading A12) */

typedef struct gsword_ctx gsword_ctx; /* opaque */

/* Random-walk estimators (P:L538 WanderJoin, P:L540 Alley). */
typedef enum { GSWORD_WJ = 0, GSWORD_ALLEY = 1 } gsword_method;

/* Comparison variants (GSWORD_OPT_VARIANT bits) of the two passages the paper leaves open:
 *  WJ_PARENT_FIRST (reading A3; "a vertex that has been previously selected"):
 *      WanderJoin draws from the label-filtered list of the FIRST backward position
 *      j = min B(d) instead of the smallest list (GetMinCandidate, Alg. 1 l.8);
 *      the other backward neighbours are validated as usual.
 *  ALLEY_DUPCHECK_POST (reading A5; Fig. 19 AL Validate): Alley's refined
 *      set keeps matched vertices (|C_d| counts them) and a drawn vertex equal to a
 *      matched one kills the sample after the draw (recorded like a WanderJoin
 *      validation failure: path[d] = v, csize[d] = |C_d|, valid = 0).
 * Both variants are unbiased; the per-sample results differ from the default. */
typedef enum { GSWORD_VARIANT_WJ_PARENT_FIRST = 2, GSWORD_VARIANT_ALLEY_DUPCHECK_POST = 4 } gsword_variant;

typedef enum {
    GSWORD_OK = 0,
    GSWORD_EINVAL = -1,   /* bad argument (NULL pointer, unknown method, label out of range) */
    GSWORD_ENOGRAPH = -2, /* no graph loaded */
    GSWORD_ENOQUERY = -3, /* no query loaded (or the graph was reloaded since) */
    GSWORD_EORDER = -4,   /* order is not a permutation, or an order prefix is disconnected (A13) */
    GSWORD_EGRAPH = -5,   /* CSR not canonical: unsorted/duplicate/self loop/asymmetric (A10, A11) */
    GSWORD_ELIMIT = -6,   /* nq > GSWORD_MAX_QV, or |V|, 2|E|, n_labels beyond 32-bit indexing */
    GSWORD_ECUDA = -7,    /* CUDA runtime error (including: no device) */
    GSWORD_ENOMEM = -8,   /* device or host allocation failed */
    GSWORD_EFAULT = -9    /* the kernels' sample accounting does not match the requested range
                             (n != n_samples: a corrupted queue counter or partial); the result
                             is discarded (SURVEY §5 failure detection) */
} gsword_status;

/* Aggregate of a sample range (Eq. 1; readings A8, A9).
 *   estimate = sum / n_samples               (HT estimator, dead samples count in n)
 *   variance = (sumsq - sum^2/n) / (n (n-1))  (variance of the estimate; NaN if n < 2)
 *   sum      = sum_i Y_i,  Y_i = prod_d |C_id| if sample i is a complete instance else 0
 *   sumsq    = sum_i Y_i^2 (Y_i^2 rounded to fp64 per sample)
 *   seconds  = device time of the sampling kernels (CUDA events), 0 if not measured */
typedef struct {
    double estimate;
    double variance;
    double sum;
    double sumsq;
    uint64_t n_samples;
    uint64_t n_valid;
    double seconds;
} gsword_result;

/* One traced sample (152 bytes, little endian, no implicit padding).
 *   path[d]  data vertex drawn at depth d (matching-order position), -1 if none
 *   csize[d] |C_d|, the size of the candidate set drawn from at depth d (0 if unused)
 *   depth_reached: last depth at which a candidate set was formed (nq-1 if complete)
 *   valid    1 iff the sample is a complete instance of q
 *   sectors  algorithmic 32-byte sectors the sample needs under the model of reading A26
 *            (DESIGN.md §3): list offsets, drawn/selected vertices, Alley
 *            driver scans, one sector per membership question; 0 for Alley by warp
 *            streaming (not modelled)
 *   weight   running fp64 product prod_{d <= depth_reached} csize[d] in depth order (A7);
 *            Y = weight if valid else 0.
 * A WanderJoin vertex drawn and then rejected by Validate is recorded (valid = 0);
 * an empty candidate set at depth d gives path[d] = -1, csize[d] = 0, weight 0. */
typedef struct {
    uint64_t sample_id;
    uint8_t valid;
    uint8_t depth_reached;
    uint8_t pad[2];
    uint32_t sectors;
    int32_t path[GSWORD_MAX_QV];
    uint32_t csize[GSWORD_MAX_QV];
    double weight;
} gsword_sample_record;

/* One traced trawling sample (168 bytes; gsword_trace_trawl).
 *   status  0: the sampled prefix died (T = 0); 1: completions enumerated; 2: the node
 *           budget was exceeded (the sample is left out of the estimate)
 *   d       number of sampled vertices (positions 0 .. d-1), the rest enumerated
 *   path/csize/weight as gsword_sample_record for the sampled prefix (W_d)
 *   count   completions of the prefix (T = weight * count when status == 1)
 *   nodes   enumeration nodes visited (vertices placed at positions >= d) */
typedef struct {
    uint64_t sample_id;
    uint8_t status;
    uint8_t d;
    uint8_t pad[6];
    int32_t path[GSWORD_MAX_QV];
    uint32_t csize[GSWORD_MAX_QV];
    double weight;
    uint64_t count;
    uint64_t nodes;
} gsword_trawl_record;

/* Host-side view of a compiled query plan (for inspection / tests).
 *   back_mask[d]  bit j set iff j < d and (phi[j], phi[d]) is a query edge: B(d)
 *   dup_mask[d]   bit j set iff j < d and L_q(phi[j]) == L_q(phi[d]) (injectivity
 *                 checks needed at depth d; SURVEY R5')
 *   label[d]      L_q(phi[d]) */
typedef struct {
    int32_t nq;
    int32_t label[GSWORD_MAX_QV];
    uint32_t back_mask[GSWORD_MAX_QV];
    uint32_t dup_mask[GSWORD_MAX_QV];
} gsword_plan_info;

/* Statistics of the loaded query (gsword_query_info).
 *   candidates[u]  |C(u)| for query vertex u under the filter the query was loaded with
 *   cg_entries     total local-candidate entries of the candidate graph (0 for filter 0)
 *   build_seconds  device time of the candidate-graph build (0 for filter 0)
 *   cg_bytes       device bytes of the candidate graph in the three-CSR format of Fig. 4
 *                  (P:L770-L776): C(u) bitmaps + rank directories, |C(u)| + 1 offsets per
 *                  directed query edge, the local lists and the seed list (0 for filter 0) */
typedef struct {
    int32_t nq;
    int32_t filter;
    uint64_t candidates[GSWORD_MAX_QV];
    uint64_t cg_entries;
    double build_seconds;
    int32_t refill_min[2]; /* refill threshold in use per method (after autotune) */
    int32_t occupancy[2];  /* resident CTAs per SM of the estimate kernel in use   */
                           /* per method (after autotune; GSWORD_OPT_BLOCKS_PER_SM */
                           /* may lower it further)                               */
    uint64_t cg_bytes;
} gsword_query_stats;

/* Tunables for gsword_set_option (defaults chosen by measurement). */
typedef enum {
    GSWORD_OPT_BLOCKS_PER_SM = 0,  /* persistent CTAs per SM; 0 = occupancy maximum  */
    GSWORD_OPT_THREADS = 1,        /* threads per CTA (multiple of 32, 64..256)       */
    GSWORD_OPT_CHUNK = 2,          /* sample ids a warp takes from the queue at once  */
    GSWORD_OPT_L2_PERSIST = 3,     /* L2 access-policy window: 0 none, 1 adjacency,   */
                                   /* 2 (default) edge filter + seg; sets the        */
                                   /* device's persisting-L2 limit                    */
    GSWORD_OPT_COOP_THRESHOLD = 4, /* Alley |S_p| above which the warp refines it in   */
                                   /* 32-element chunks (0..128; below: task pool)    */
    GSWORD_OPT_BLOOM = 5,          /* 1 = edge Bloom pre-test (L2-resident filter)    */
    GSWORD_OPT_EDGE_SET = 6,       /* 1 = exact edge hash set for adjacency tests;    */
                                   /* 0 = binary search in the adjacency run          */
    GSWORD_OPT_SCHEDULE = 8,       /* 0 refill free lanes every round (default);      */
                                   /* 1 sample synchronisation (comparison);  */
                                   /* 2 = 1 + sample inheritance (Alg. 2, NEXT-3,     */
                                   /*   reading A24; estimates only, no traces; the   */
                                   /*   variance uses groups of 32 ids; sumsq of the  */
                                   /*   async output holds squared group totals)      */
    GSWORD_OPT_REFILL_MIN = 9,     /* schedule 0: a warp refills only when at least    */
                                   /* this many lanes are free (1..32; 32 = sample    */
                                   /* synchronisation; default 16); no effect on    */
                                   /* results                                         */
    GSWORD_OPT_AUTOTUNE = 10,      /* 1 (default): gsword_load_query times pilots of   */
                                   /* refill thresholds 8/16/24/28/32 per method and  */
                                   /* keeps the fastest, then times the estimate      */
                                   /* kernel compiled for one CTA/SM less and one     */
                                   /* more (register budget vs occupancy) at that     */
                                   /* threshold; results are unaffected.              */
                                   /* Results are cached per (query arrays, options)  */
                                   /* until the next graph load: reloading the same   */
                                   /* query runs no pilots                            */
    GSWORD_OPT_BLOOM_BITS = 11,    /* edge filter bits per undirected edge (2..64,    */
                                   /* default 16), applied at the next graph load     */
    GSWORD_OPT_STREAMING = 12,     /* 1 = Alley draws by warp streaming (Alg. 3,      */
                                   /* P:L914-L968, NEXT-3 comparison mode, reading    */
                                   /* A25): same C_d and weights, a different vertex  */
                                   /* of C_d than count-then-index; 0 (default) off.  */
                                   /* Applies to estimates and traces with every      */
                                   /* schedule; WanderJoin and count_sectors ignore it */
    GSWORD_OPT_VARIANT = 13,       /* comparison variants of the sampler (bit flags,  */
                                   /* gsword_variant; default 0 = readings A3/A5 as   */
                                   /* in SURVEY R3-R5).  Applies to estimates and     */
                                   /* traces (every schedule, streaming included);    */
                                   /* trawling ignores it                             */
    GSWORD_OPT_OCCUPANCY = 14,     /* estimate-kernel occupancy variant: -1 (default) */
                                   /* the autotuned one; 0 default launch bounds, 1   */
                                   /* one CTA/SM less, 2 one more (forced; for A/B    */
                                   /* and sanitizer runs).  Results are unaffected    */
    GSWORD_OPT_FAULT_QUEUE = 15,   /* fault injection (tests): the next sampling launch */
                                   /* starts its sample queue at this value instead of */
                                   /* 0, as a corrupted counter would (ids skipped);   */
                                   /* one-shot; 0 = off.  Synchronous calls then fail  */
                                   /* with GSWORD_EFAULT                               */
    GSWORD_OPT_TRAWL_WARP = 16,    /* gsword_trawl_range enumeration: 1 (default) the  */
                                   /* warp-cooperative kernel (32 candidates tested   */
                                   /* per round, last-position survivors counted by   */
                                   /* popcount), 0 one lane per sample depth first.   */
                                   /* Same counts and timeouts (the node total of a   */
                                   /* sample's tree decides the timeout); traces     */
                                   /* always use the per-lane kernel                  */
    GSWORD_OPT_FILTER = 7          /* candidate filter applied by the next            */
                                   /* gsword_load_query: 0 label only, 1 LDF, 2 NLF   */
                                   /* (1-2 build the candidate graph, reading A21)    */
} gsword_option;

/* ---- context -------------------------------------------------------------------- */

/* Create a context on CUDA device `cuda_device`.  *out receives the handle.
 * Errors: EINVAL (out NULL), ECUDA (no such device / no driver), ENOMEM. */
int gsword_create(int cuda_device, gsword_ctx** out);

/* Destroy a context and free every device buffer it owns.  NULL is a no-op. */
int gsword_destroy(gsword_ctx* ctx);

/* Issue all later device work on `cuda_stream` (a cudaStream_t, e.g.
 * torch.cuda.Stream.cuda_stream; NULL = the context's own non-blocking stream; the
 * legacy default stream is cudaStreamLegacy, (void*)0x1).  Borrowed, not destroyed.
 * Ordering: work issued after the switch starts only after all work the context issued
 * on the previous stream (an event on the old stream, waited on by the new one), so
 * switching never races the context's reused queue / partial / output buffers. */
int gsword_set_stream(gsword_ctx* ctx, void* cuda_stream);

/* Set a tunable (gsword_option).  Errors: EINVAL for an unknown option or value. */
int gsword_set_option(gsword_ctx* ctx, int option, int64_t value);

/* ---- graph and query -------------------------------------------------------------- */

/* Load the data graph G (P:L404 notation).  Host arrays, copied; the context owns the
 * device copy.  Canonical CSR required (reading A10/A11):
 *   row_ptr  int64[n_vertices+1], row_ptr[0] = 0, non-decreasing
 *   col      int32[row_ptr[n]], each row strictly ascending, no self loop, and the
 *            adjacency symmetric (u in N(v) iff v in N(u))
 *   labels   int32[n_vertices] in [0, n_labels), or NULL = unlabelled (n_labels must be 1)
 * The library re-lays adjacency out sorted by (label, id) so that every label-filtered
 * local candidate set N_l(v) (Def. 4) is one contiguous ascending run.
 * Loading a graph invalidates the loaded query.
 * Errors: EINVAL, EGRAPH, ELIMIT (n_vertices or 2|E| >= 2^31, n_vertices*n_labels >= 2^31),
 * ENOMEM, ECUDA. */
int gsword_load_graph(gsword_ctx* ctx, int64_t n_vertices, const int64_t* row_ptr, const int32_t* col,
                      const int32_t* labels, int32_t n_labels);

/* Load the data graph from DEVICE memory (e.g. torch tensors on the context's device).
 *   d_row_ptr int64[n_vertices+1]  borrowed for the call only
 *   d_col     int32[row_ptr[n]]    borrowed, NOT copied: the caller keeps it alive and
 *                                  unchanged until the next load or gsword_destroy
 *   d_labels  int32[n_vertices] or NULL (n_labels 1); borrowed like d_col
 * Each row must already be sorted by (label, id) (= by id when unlabelled), with no self
 * loop and a symmetric adjacency; this is checked on the device (EGRAPH).  The library
 * derives and owns seg, the label buckets, the Bloom filter and the edge set.
 * Errors: EINVAL, EGRAPH, ELIMIT, ENOMEM, ECUDA. */
int gsword_load_graph_device(gsword_ctx* ctx, int64_t n_vertices, const int64_t* d_row_ptr, const int32_t* d_col,
                             const int32_t* d_labels, int32_t n_labels);

/* Load the query q and its matching order phi (Def. 2).  Host arrays, copied.
 * With GSWORD_OPT_FILTER > 0 this also builds the candidate graph on the device
 * (Def. 5; Fig. 4) and the sampler draws from its local candidate lists:
 *   q_row_ptr int32[n_qv+1], q_col: symmetric query adjacency over vertices 0..n_qv-1
 *   q_labels  int32[n_qv] in [0, n_labels of the loaded graph)
 *   order     int32[n_qv], a permutation of 0..n_qv-1 with every prefix connected
 * Errors: ENOGRAPH, EINVAL, EORDER, ELIMIT (n_qv > GSWORD_MAX_QV). */
int gsword_load_query(gsword_ctx* ctx, int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col,
                      const int32_t* q_labels, const int32_t* order);

/* Statistics of the loaded query: candidate-set sizes and candidate-graph size/build
 * time (Tab. 3 analogue).  Errors: EINVAL, ENOQUERY. */
int gsword_query_info(gsword_ctx* ctx, gsword_query_stats* out);

/* ---- matching order (NEXT-4) --------------------------------- */

typedef enum {
    GSWORD_ORDER_QUICKSI = 0, /* infrequent-edge-first order from data label statistics (A22) */
    GSWORD_ORDER_TRIAL = 1    /* G-CARE-style trial: pilot-estimate candidate orders on the GPU,
                                 keep the smallest single-sample variance        */
} gsword_order_strategy;

/* Host-only QuickSI-style order (reading A22).  Graph arrays as gsword_load_graph (labels
 * may be NULL with n_labels 1); query CSR + labels as gsword_load_query.  order_out receives
 * n_qv query-vertex ids with every prefix connected.  Errors: EINVAL, ELIMIT, EORDER. */
int gsword_quicksi_order(int64_t n_vertices, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                         int32_t n_labels, int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col,
                         const int32_t* q_labels, int32_t* order_out);

/* Choose a matching order for the loaded graph and LOAD the query with it.
 *   GSWORD_ORDER_QUICKSI: as gsword_quicksi_order (no sampling).
 *   GSWORD_ORDER_TRIAL: candidates = the QuickSI order + every directed query edge as the
 *     first two positions completed in QuickSI preference; each is pilot-estimated with
 *     `m`, samples [0, pilot_samples) and `seed`; the smallest variance of one sample wins
 *     (ties: earliest candidate).  score_out (may be NULL) receives it.
 * order_out: n_qv entries.  Errors: ENOGRAPH, EINVAL, EORDER, ELIMIT, ECUDA. */
int gsword_select_order(gsword_ctx* ctx, int strategy, gsword_method m, int32_t n_qv, const int32_t* q_row_ptr,
                        const int32_t* q_col, const int32_t* q_labels, uint64_t pilot_samples, uint64_t seed,
                        int32_t* order_out, double* score_out);

/* ---- estimation ----------------------------------------------------------------------- */

/* Draw samples 0 .. n_samples-1 with `method` and `seed`, return the HT aggregate
 * (Eq. 1).  Synchronous (waits for the context stream).  Same as
 * gsword_estimate_range(ctx, m, 0, n_samples, seed, out).  The kernels count every sample
 * id they run; a count different from n_samples is reported as EFAULT.
 * Errors: ENOGRAPH, ENOQUERY, EINVAL (n_samples == 0, out NULL, bad method), ECUDA, EFAULT. */
int gsword_estimate(gsword_ctx* ctx, gsword_method m, uint64_t n_samples, uint64_t seed, gsword_result* out);

/* Accuracy-targeted estimate: samples 0, 1, 2, ... in doubling batches (first batch
 * min_samples) until the relative standard error sqrt(variance)/estimate <= rel_se_target
 * or max_samples are drawn; the result is identical to gsword_estimate over the same
 * number of samples (batches are sample-id ranges).  A zero estimate never meets the
 * target (the underestimation regime) and runs to max_samples.
 * Errors: as gsword_estimate, EINVAL (target <= 0, min_samples < 2, max < min). */
int gsword_estimate_until(gsword_ctx* ctx, gsword_method m, uint64_t seed, double rel_se_target, uint64_t min_samples,
                          uint64_t max_samples, gsword_result* out);

/* Same for the sample-id range [first_sample_id, first_sample_id + n_samples): the
 * multi-GPU split and checkpoint/resume unit (sample ids are global).
 * The exclusive end first_sample_id + n_samples must fit in u64 (so the largest usable id
 * is 2^64 - 2); a wrapping range is EINVAL here and in every other range-taking call
 * (async, trace, trawl, count_sectors). */
int gsword_estimate_range(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples,
                          uint64_t seed, gsword_result* out);

/* Asynchronous form: enqueue the sampling + reduction kernels on the context stream
 * and write 4 fp64 values {sum, sumsq, n_valid, n_samples} to DEVICE memory d_out4
 * (caller-owned, 32 bytes, 8-byte aligned).  Returns without waiting; the values are
 * valid in stream order.  Used by the multi-GPU layer (all_reduce on the same stream)
 * and by device-side timing.  Counts are exact as fp64 below 2^53. */
int gsword_estimate_async(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples,
                          uint64_t seed, double* d_out4);

/* Trawling estimator (NEXT-2; Alg. 4; reading A23) over samples
 * [first, first + n): each sample draws d ~ P(d = j) proportional to 2^-j, j in [3, |V_q|]
 * (P:L1012), samples positions 0..d-1 with `m` (the same draws as gsword_estimate), counts
 * every completion exactly with a depth-first enumeration of at most node_budget nodes,
 * and contributes T = W_d * count (unbiased).  Samples over budget are left out
 * (P:L1026): out->n_samples counts the finished ones, *n_timeout (may be NULL) the rest;
 * out->n_valid counts T > 0.  Synchronous. */
int gsword_trawl_range(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples, uint64_t seed,
                       uint64_t node_budget, gsword_result* out, uint64_t* n_timeout);

/* Parity entry for trawling: n records in sample-id order.  Synchronous. */
int gsword_trace_trawl(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples, uint64_t seed,
                       uint64_t node_budget, gsword_trawl_record* host_out);

/* Host-only: turn 4 aggregated values {sum, sumsq, n_valid, n_samples} into a result. */
int gsword_finalize(const double* host4, gsword_result* out);

/* Parity entry: run samples [first, first+n) through the same kernel code with a
 * per-sample record writer; host_out receives n records in sample-id order.
 * Synchronous.  Errors as gsword_estimate_range, ENOMEM. */
int gsword_trace_samples(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples,
                         uint64_t seed, gsword_sample_record* host_out);

/* Measurement entry: run [first, first+n) in the counting build of the
 * kernel (the same refine/sample code as the estimate, plus counters) and return, summed
 * over the range:
 *   *sectors_out  the ALGORITHMIC 32-byte sectors of reading A26 (the per-sample `sectors`
 *                 of gsword_sample_record; equal to the oracle's count, tests pin both)
 *   *touched_out  (may be NULL) the sectors this implementation's accesses touch: edge-filter
 *                 words, edge-set buckets (or binary-search probes), list offsets, driver
 *                 chunks of the cooperative refine and re-tests, drawn elements
 * Synchronous.  Ignores GSWORD_OPT_STREAMING. */
int gsword_count_sectors(gsword_ctx* ctx, gsword_method m, uint64_t first_sample_id, uint64_t n_samples,
                         uint64_t seed, double* sectors_out, double* touched_out);

/* Profiling aid: warp-cycles per loop phase summed over all warps, recorded by the last
 * gsword_count_sectors run: [0] refill, [1] draw + GetMinCandidate, [2] WanderJoin step /
 * Alley path selection, [3] Alley task pool, [4] Alley survivor selection, [5] Alley
 * cooperative refine, [6] epilogue, [7] exit.  out8 receives 8 doubles. */
int gsword_phase_cycles(gsword_ctx* ctx, double* out8);

/* Device time (CUDA events on the context stream) of the last sampling-kernel launch
 * alone (without the queue reset and the grid reduction).  Waits for that launch. */
int gsword_last_kernel_seconds(gsword_ctx* ctx, double* seconds);

/* Measurement aid (SURVEY §8(d) "K5"): the random-gather roofline of this device — one
 * 4-byte load per 32-byte sector at uniformly random positions of a buffer_bytes buffer,
 * `inflight` (1..8) independent dependent-load chains per thread, 8 CTAs x 256 threads per
 * SM.  *sectors_per_s receives the sustained sector rate (x 32 B = bytes/s). */
int gsword_gather_roofline(gsword_ctx* ctx, uint64_t buffer_bytes, int inflight, double* sectors_per_s);

/* Launch geometry used by the last estimate: grid CTAs, threads per CTA, kernel
 * launches per estimate.  Any pointer may be NULL. */
int gsword_launch_info(gsword_ctx* ctx, int* grid, int* threads, int* launches_per_estimate);

/* ---- host-only helpers (no device needed) ------------------------------------------- */

/* Check that a CSR is canonical (same rules as gsword_load_graph). */
int gsword_check_graph(int64_t n_vertices, const int64_t* row_ptr, const int32_t* col, const int32_t* labels,
                       int32_t n_labels);

/* Compile a query + order into its plan (the same plan gsword_load_query stages into
 * shared memory); n_labels bounds the labels. */
int gsword_plan_query(int32_t n_qv, const int32_t* q_row_ptr, const int32_t* q_col, const int32_t* q_labels,
                      const int32_t* order, int32_t n_labels, gsword_plan_info* out);

/* Thread-local message for the last failing call on this thread ("" if none). */
const char* gsword_last_error(void);

/* ABI version (major*100 + minor). */
int gsword_version(void);

#ifdef __cplusplus
}
#endif

#endif /* GSWORD_H */
