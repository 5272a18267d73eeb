/*
 * algas.h -- C-ABI of the B200-native ALGAS search library (libalgas.so).
 *
 * ALGAS: Chen et al., "ALGAS: A Low-latency GPU-Based Approximate Nearest
 * Neighbor Search System", IPDPS 2025.  Citations "P:L<n>" point into the
 * paper text; "R<n>" are the readings listed in
 * DESIGN.md §3 where the paper is silent or ambiguous.
 *
 * Problem: given base vectors P (n x dim) and a query q, return the
 * k points of P closest to q under F(a,b).  Search runs greedy/beam search
 * over a fixed-out-degree proximity graph (Alg.1, beam extend
 * P:L200/P:L249), possibly with several CTAs per query,
 * each CTA publishing its own top-k and the host merging them.
 *
 * Conventions for every entry point:
 *  - Distances are "internal" distances, ascending = closer:
 *      ALGAS_L2: squared Euclidean  sum_j (q_j - x_j)^2         (R2)
 *      ALGAS_IP: negated inner product  -sum_j q_j x_j           (R3)
 *  - Ties are broken by point id: order is lexicographic (dist, id) (R4).
 *  - Results are sorted ascending, ids unique, padded with
 *    (ALGAS_SENTINEL, +inf) when fewer than k points were reached (R12).
 *  - Pointers: every array argument may be HOST or DEVICE memory of the
 *    current CUDA device unless stated otherwise; the library detects which
 *    (cudaPointerGetAttributes) and copies as needed.  All arrays are
 *    caller-owned; the library never frees or retains caller memory beyond
 *    the call (except where a function says it copies).
 *  - Return codes: ALGAS_OK (0) or a negative ALGAS_E* code; the message for
 *    the last failing call on this thread is in algas_last_error().
 *  - A CUDA failure is reported as ALGAS_ECUDA, never silently retried and
 *    never answered on the CPU: the library has no CPU fallback.
 */
#ifndef ALGAS_H
#define ALGAS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default) /* the C-ABI is the only exported surface */
#endif

#define ALGAS_SENTINEL 0xFFFFFFFFu
#define ALGAS_MAX_ITOPK 512   /* max candidate-list length L            */
#define ALGAS_MAX_DEGREE 128  /* max graph out-degree R                 */
#define ALGAS_MAX_DIM 2048    /* max dim (must also be a multiple of 4) */
#define ALGAS_MAX_WIDTH 32    /* max parents per beam-extend step       */
#define ALGAS_MAX_CTAS 64     /* max CTAs per query (N_parallel)        */
#define ALGAS_MAX_SEEDS 256   /* max random entry points per CTA        */

/* L2: squared Euclidean; IP: -q.x; COSINE: -(q.x)/(|q||x|), the negated
 * cosine similarity (the paper's cosine datasets; DESIGN.md
 * R29).  COSINE is served as IP on unit rows: algas_index_create normalises
 * its HBM copy of the data, every search kernel normalises the query in
 * shared memory when it is staged; a zero row / query scores 0. */
enum algas_metric { ALGAS_L2 = 0, ALGAS_IP = 1, ALGAS_COSINE = 2 };

enum algas_status {
    ALGAS_OK = 0,
    ALGAS_EINVAL = -1,   /* bad argument (see each function)               */
    ALGAS_ENOMEM = -2,   /* device or pinned host allocation failed        */
    ALGAS_ECUDA = -3,    /* a CUDA call or kernel failed                   */
    ALGAS_EAGAIN = -4,   /* persistent path: no EMPTY slot right now       */
    ALGAS_ESTATE = -5,   /* object in the wrong state (e.g. server closed) */
    ALGAS_ENCCL = -6,    /* reserved for the sharded multi-GPU path        */
    ALGAS_EOVERFLOW = -7 /* a visited table overflowed (result still valid,
                            exploration was cut short; see stats)          */
};

/* Visited-table sharing between the CTAs of one query ("sharing the
 * visited table").  PRIVATE: one exact table per CTA -- deterministic, the
 * parity mode (R9).  SHARED: one table per query, shared by its CTAs (the
 * paper's design; nondeterministic which CTA scores a point). */
enum algas_visited { ALGAS_VISITED_PRIVATE = 0, ALGAS_VISITED_SHARED = 1 };

/* Search parameters.  Field meaning follows P:L213 (TopK, candidate list of
 * max length L, T CTAs) and P:L249 (offset_beam).  Zero / negative values
 * select the documented default.  Fill with algas_params_default(). */
typedef struct algas_params {
    int32_t k;               /* results per query, 1 <= k <= itopk                    */
    int32_t itopk;           /* L: candidate-list length, k <= L <= ALGAS_MAX_ITOPK   */
    int32_t width;           /* w: parents per step once diffusing, 1..32   */
    int32_t offset_beam;     /* off: diffusing starts when the first
                                unchecked position >= off; < 0 -> itopk/4;
                                >= itopk disables beam extend (pure Alg.1)           */
    int32_t ctas_per_query;  /* T = N_parallel; 0 -> adaptive tuner */
    int32_t threads_per_cta; /* 32/64/128/256/512/1024 (1024: dim <= 512); 0 -> tuner */
    int32_t n_seeds;         /* S random entry points per CTA; 0 -> 32      */
    int32_t max_iter;        /* per-CTA step cap (R8); 0 -> 4*itopk + 256            */
    int32_t visited_mode;    /* enum algas_visited                                  */
    int32_t slots;           /* persistent path: B query slots; 0 -> 32     */
    int32_t hash_bits;       /* log2 of the per-CTA shared-memory visited hash; 0 -> tuner */
    int32_t stage_rows;      /* vectors per shared-memory staging buffer (2 buffers); 0 -> tuner */
    int32_t cluster_size;    /* persistent paths: CTAs (SMs) per search as a thread-block
                                cluster sharing the distance gathers through DSMEM;
                                1 = off, 2/4/8 (needs threads_per_cta = 256); 0 -> 1 */
    int32_t host_threads;    /* persistent server: host poller threads, each watching
                                slots q with q % host_threads == its index, merging
                                and refilling them (Fig. 18); 0 -> 1 (measured best on
                                the B200 box: more threads contend for the FIFO/queue locks) */
    int32_t state_mirror;    /* persistent server: 1 = the host mirrors each staged query's
                                state word, params and query into DEVICE memory (stream-
                                ordered async copies from the host thread's private IO
                                stream, P:L255-272's GDRCopy state copy without GDRCopy), so
                                the slots' CTAs poll HBM instead of host memory over PCIe;
                                0 (default) = CTAs poll the host-mapped ring */
    int32_t watchdog_ms;     /* persistent server: a query in a slot longer than this is
                                reported (algas_poll -> ALGAS_ESTATE, the stuck tag in
                                algas_last_error): a hung or dead kernel never leaves the
                                caller waiting silently; 0 -> 10000 ms, < 0 -> off */
    uint64_t seed;           /* entry-point generator seed (R5)                      */
} algas_params;

/* Per-query counters (summed over the query's CTAs unless noted). */
typedef struct algas_query_stats {
    uint32_t iters;       /* steps = candidate-list maintenance operations */
    uint32_t max_iters;   /* max steps over the query's CTAs                       */
    uint32_t parents;     /* expanded candidate points                             */
    uint32_t dist_evals;  /* distance computations (vectors gathered)              */
    uint32_t cap_hits;    /* CTAs stopped by max_iter rather than Finish            */
    uint32_t spills;      /* CTAs whose shared-memory visited hash spilled to HBM   */
    uint32_t overflows;   /* CTAs whose visited table overflowed (should be 0)      */
    uint32_t ctas;        /* T used                                                 */
    uint64_t t_start_ns;  /* device globaltimer at pickup (persistent/dynamic path) */
    uint64_t t_end_ns;    /* device globaltimer when the last CTA published         */
    uint64_t latency_ns;  /* host: submit -> merged result ready (server path)      */
    /* SM cycles spent per search phase (summed over CTAs; the paper's
     * calculation-vs-sorting breakdown, Fig. 3 / Fig. 17) */
    uint64_t cyc_select;  /* parent selection (P:L217 step 1)                    */
    uint64_t cyc_gather;  /* neighbour-id gather + visited filter (steps 1-2)    */
    uint64_t cyc_dist;    /* vector gathers + distances (step 3)                 */
    uint64_t cyc_sort;    /* sort + merge into the candidate list (step 4)       */
    /* device globaltimer (persistent/dynamic path): the first / last of the
     * query's CTAs to enter its search loop (after pickup, query staging,
     * visited reset and seeding), and the last to leave it */
    uint64_t t_loop_first_ns;
    uint64_t t_loop_last_ns;
    uint64_t t_loop_end_ns;
    uint64_t t_entry_last_ns;  /* the last CTA to start its search (query staged) */
    uint64_t queue_ns;    /* host: algas_enqueue -> into a slot (0 for algas_submit) */
    /* candidate updates (P:L219 step 4) by path: the warp-register bitonic
     * merge fused with the next selection, and the CTA-wide rank merge
     * (steps with more than 128 surviving new keys, e.g. while the list
     * fills, or lists longer than the register budget) */
    uint32_t merges_bitonic;
    uint32_t merges_rank;
} algas_query_stats;

/* Optional per-call timing filled by the search entry points. */
typedef struct algas_run_info {
    float kernel_ms;          /* search kernel duration (CUDA events on the launch stream) */
    int32_t grid;             /* CTAs launched                                             */
    int32_t threads_per_cta;
    int32_t ctas_per_query;
    int32_t smem_per_cta;     /* dynamic shared memory bytes                               */
    int32_t blocks_per_sm;    /* occupancy of the search kernel                            */
    int32_t hash_bits;
    int32_t reserved;
    float call_ms;            /* host wall time of the whole call (entry -> outputs written) */
    float merge_ms;           /* host wall time of the TopK merge + output copy    */
} algas_run_info;

typedef struct algas_index algas_index;   /* opaque; immutable after create */
typedef struct algas_server algas_server; /* opaque; owns ring + persistent kernel */

/* Fill *p with defaults: k=10, itopk=64, width=1, offset_beam=-1, T=1,
 * threads=0, n_seeds=32, max_iter=0, PRIVATE, slots=32, seed=0. */
void algas_params_default(algas_params *p);

/* Thread-local description of the last error (never NULL). */
const char *algas_last_error(void);

/* Library version string. */
const char *algas_version(void);

/* ------------------------------------------------------------------ */
/* Index (graph index G=(V,E) over the vectors of P).            */
/* ------------------------------------------------------------------ */
/* Creates an index on the current CUDA device.  The library COPIES data
 * (n x dim fp32, row-major) and graph (n x degree u32, row-major, entries
 * in [0,n) or ALGAS_SENTINEL) into HBM; the caller keeps ownership.
 * graph == NULL builds the graph: exact kNN with 2*degree neighbours
 * (algas_knn) followed by CAGRA-style pruning to `degree` (algas_prune).
 * EINVAL (returns NULL): n < 1 or n >= 2^31, dim < 4, dim % 4 != 0,
 * dim > ALGAS_MAX_DIM, degree < 1 or > ALGAS_MAX_DEGREE, bad metric.
 * metric COSINE: the HBM copy of data is normalised to unit rows (the
 * caller's buffer is untouched) and the built graph is the IP graph of the
 * unit rows (= the cosine kNN graph). */
algas_index *algas_index_create(const float *data, int64_t n, int32_t dim, int32_t metric,
                                const uint32_t *graph, int32_t degree);
int algas_index_destroy(algas_index *idx);
/* Shape query; any out pointer may be NULL.  *dev_data / *dev_graph are
 * device pointers owned by the index (graph row stride = *graph_stride). */
int algas_index_info(const algas_index *idx, int64_t *n, int32_t *dim, int32_t *metric,
                     int32_t *degree, int32_t *graph_stride, const float **dev_data,
                     const uint32_t **dev_graph);

/* ------------------------------------------------------------------ */
/* Static (batch) search: one launch over nq queries (P:L107 batch       */
/* processing; the search procedure of P:L213-223).                      */
/* ------------------------------------------------------------------ */
/* queries: nq x dim fp32.  out_ids / out_dists: nq x k.  Uses
 * algas_params_default() with the given k, itopk, width. */
int algas_search(const algas_index *idx, const float *queries, int64_t nq, int32_t k,
                 int32_t itopk, int32_t width, uint32_t *out_ids, float *out_dists);

/* Full-control batch search.  Query i uses tag = tag0 + i (R23), so a batch
 * result is reproducible through algas_submit with the same tag.
 * out_cta_ids / out_cta_dists (nullable): nq x T x k per-CTA results before
 * the host merge.  out_stats (nullable): nq entries.
 * stream: cudaStream_t to run on (NULL = the legacy default stream); the
 * call is synchronous with respect to the host.  info (nullable): kernel
 * time and launch shape.
 * Returns EOVERFLOW (results still written) if any visited table overflowed. */
int algas_search_ex(const algas_index *idx, const float *queries, int64_t nq,
                    const algas_params *params, uint64_t tag0, uint32_t *out_ids,
                    float *out_dists, uint32_t *out_cta_ids, float *out_cta_dists,
                    algas_query_stats *out_stats, void *stream, algas_run_info *info);

/* Dynamic batching from an HBM-resident query queue: a
 * persistent kernel keeps exactly params->slots queries in flight; a slot
 * takes the next query the moment its CTAs finish (no batch barrier).
 * queries must be DEVICE memory (nq x dim); outputs may be host or device.
 * Per-query stats carry device start/end timestamps (globaltimer). */
int algas_search_dynamic(const algas_index *idx, const float *queries_dev, int64_t nq,
                         const algas_params *params, uint64_t tag0, uint32_t *out_ids,
                         float *out_dists, algas_query_stats *out_stats, void *stream,
                         algas_run_info *info);

/* ------------------------------------------------------------------ */
/* Persistent server: host-mapped slot ring + persistent kernel          */
/* (P:L157-178), host TopK merge.                           */
/* ------------------------------------------------------------------ */
/* Launches the persistent kernel (cooperative launch: all slots x T CTAs
 * co-resident).  params->k / itopk are the per-server maxima; a
 * submit may ask for smaller k/itopk/width.  *out is NULL on failure.
 * Each of the B slots has two ring entries in host-mapped memory: a slot
 * runs one query at a time (B searches in flight) while its next query can
 * already be staged in the other entry, so a slot's CTAs start the next
 * query without waiting for the host (the host merges the finished one
 * meanwhile).  Submitting fills idle slots first.  Host poller threads:
 * params->host_threads. */
int algas_server_create(const algas_index *idx, const algas_params *params, algas_server **out);
/* As algas_server_create, but the persistent kernel is NOT launched: the
 * ring, poller threads and device state exist, and algas_submit may stage
 * up to two queries per slot into the ring (None -> Work) before
 * algas_server_start launches the kernel.  For bounded sessions under tools
 * that serialise kernel launches (profilers, compute-sanitizer), where the
 * host cannot submit while the launch call blocks. */
int algas_server_create_deferred(const algas_index *idx, const algas_params *params,
                                 algas_server **out);
/* TEST HARNESS, not a search: a server whose device side is a host thread
 * that follows the persistent kernel's ring protocol (P:L166-172 states;
 * the kernel's mode-0 loop in kernels.cuh) -- for tests of the host state
 * machine (slot claim, two ring entries per slot, epochs, poller, host merge,
 * recycle, FIFO drain, watchdog, bounded sessions) on machines without a
 * GPU.  No CUDA call is made.  params: slots, ctas_per_query (T), k, itopk,
 * width, host_threads, watchdog_ms are used; dim: query length (multiple of
 * 4).  The emulated device returns a fixed function of each query, not
 * neighbours: CTA r's list entry i is (tag*1000 + i*T + r, q[0] + i*T + r),
 * and for T > 1 CTA 1 repeats CTA 0's first id at a larger distance, so a
 * query's merged result is ids tag*1000 + j, dists q[0] + j, j < k.
 * deferred != 0: the device thread starts with algas_server_start (bounded
 * sessions).  Destroy with algas_server_destroy. */
int algas_server_create_emulated(const algas_params *params, int32_t dim, int32_t deferred, algas_server **out);
/* Emulated server only: the query with this tag is never finished (it stays
 * in its slot; the watchdog reports it).  ALGAS_EINVAL on a real server. */
int algas_server_emulated_stall(algas_server *s, uint64_t tag);
/* Launch a deferred server's kernel.  quit_when_idle != 0 makes it a bounded
 * session: every free ring entry becomes QUIT -- now and whenever a
 * finished query's entry is recycled -- so the kernel exits after the staged
 * queries; submit/enqueue then fail with ALGAS_ESTATE.  Results are still
 * collected with algas_poll.  ALGAS_ESTATE if already started. */
int algas_server_start(algas_server *s, int32_t quit_when_idle);
/* Non-blocking.  query: dim fp32 in HOST memory (copied).  Claims a free
 * ring entry (EMPTY -> READY); ALGAS_EAGAIN if every entry is busy.
 * k <= server k, itopk <= server itopk, width <= 32 (0 -> server value). */
int algas_submit(algas_server *s, const float *query, uint64_t tag, int32_t k, int32_t itopk,
                 int32_t width);
/* Non-blocking batched submit: queries i = 0.. (n x dim fp32, HOST,
 * row-major) with tags tag0 + i are submitted in order until every slot is
 * busy; *n_accepted (required) = how many were (0 when the ring is full --
 * not an error).  Same semantics per query as algas_submit; one library
 * crossing for many queries (the host side of dynamic batching). */
int algas_submit_many(algas_server *s, const float *queries, int64_t n, uint64_t tag0, int32_t k,
                      int32_t itopk, int32_t width, int64_t *n_accepted);
/* Non-blocking.  Moves up to max_results completed queries into caller
 * HOST buffers: tags[i], ids[i*kmax .. ), dists[i*kmax .. ) where kmax is
 * the server's k (rows padded with SENTINEL / +inf), stats[i] (nullable).
 * *n_out = number returned. */
/* Non-blocking, never refuses: queries i = 0.. (n x dim fp32, HOST,
 * row-major; copied) with tags tag0 + i join a host FIFO; as many as there
 * are free slots go in now, the rest enter slots in order as the poller
 * thread recycles them (Done -> None -> Work without a library crossing by
 * the caller: the host side of dynamic batching).
 * Results arrive through algas_poll like submitted ones (stats.queue_ns =
 * FIFO wait, stats.latency_ns = slot in -> merged result).  Queries still in
 * the FIFO at algas_server_destroy are dropped. */
int algas_enqueue(algas_server *s, const float *queries, int64_t n, uint64_t tag0, int32_t k, int32_t itopk,
                  int32_t width);
int algas_poll(algas_server *s, uint64_t *tags, uint32_t *ids, float *dists,
               algas_query_stats *stats, int32_t max_results, int32_t *n_out);
/* Number of submitted-but-not-yet-polled queries. */
int algas_server_inflight(const algas_server *s, int64_t *n);
/* Sets QUIT, joins the kernel and the poller, frees the ring. */
int algas_server_destroy(algas_server *s);

/* ------------------------------------------------------------------ */
/* Host TopK merge & filter, exposed for tests and shard mode.  */
/* ------------------------------------------------------------------ */
/* Merges m (id, dist) HOST entries by (dist, id), drops SENTINEL and
 * repeated ids (keeps the smallest key, R11), writes k (padded).  Returns
 * the number of real entries written. */
int32_t algas_merge_topk(const uint32_t *ids, const float *dists, int32_t m, int32_t k,
                         uint32_t *out_ids, float *out_dists);
/* Row-wise batch form for the sharded layout: nq independent merges of the
 * entries ids[p*stride_part + q*m_per + j] (parts p < nparts, j < m_per):
 * the per-shard [nparts][nq][m_per] results of an all-gather.  HOST arrays;
 * out_ids / out_dists: nq x k.  Returns ALGAS_OK or ALGAS_EINVAL. */
int algas_merge_topk_parts(const uint32_t *ids, const float *dists, int32_t nparts, int64_t nq,
                           int32_t m_per, int32_t k, uint32_t *out_ids, float *out_dists);

/* ------------------------------------------------------------------ */
/* Adaptive tuning.                                        */
/* ------------------------------------------------------------------ */
typedef struct algas_device_props {
    int32_t n_sm;                 /* N_SM                         */
    int32_t max_blocks_per_sm;    /* N_max_block_per_SM           */
    int64_t smem_per_sm;          /* M_per_SM (bytes)             */
    int64_t smem_reserved_per_block; /* driver reservation (bytes) */
    int64_t smem_per_block_optin; /* largest dynamic smem per CTA */
    int32_t max_threads_per_sm;
    int32_t regs_per_sm;
} algas_device_props;

typedef struct algas_tuning {
    int32_t ctas_per_query;   /* N_parallel                 */
    int32_t blocks_per_sm;    /* N_block_per_SM             */
    int64_t smem_avail_per_block; /* M_avail_per_block bound */
    int64_t smem_per_block;   /* bytes the search kernel will use    */
    int32_t threads_per_cta;
    int32_t width;
    int32_t offset_beam;
    int32_t hash_bits;
    int32_t stage_rows;
    int32_t visited_mode;     /* enum algas_visited: SHARED when T > 1 */
} algas_tuning;

/* Properties of the current device (props of P:L280-291 Table II). */
int algas_device_query(algas_device_props *out);
/* The three printed equations, exactly (align() = ceil, R13). */
int32_t algas_tuner_max_parallel(int32_t slots, int32_t n_sm, int32_t max_blocks_per_sm);
int32_t algas_tuner_blocks_per_sm(int32_t n_parallel, int32_t slots, int32_t n_sm);
int64_t algas_tuner_smem_per_block(int64_t smem_per_sm, int32_t blocks_per_sm,
                                   int64_t smem_reserved_per_block);
/* Full tuner: picks T, threads/CTA, width, offset_beam, the visited mode and
 * the visited hash size for `slots` concurrent queries of this shape so that every slot's
 * CTAs are co-resident and the per-block shared memory respects
 * P:L245 with M_reserved sized for the dimension.
 * props NULL -> algas_device_query().  Returns EINVAL if no configuration fits. */
int algas_tune(const algas_device_props *props, int32_t slots, int32_t dim, int32_t degree,
               int32_t itopk, int32_t k, algas_tuning *out);

/* ------------------------------------------------------------------ */
/* Graph construction (supporting code, not the search hot path):        */
/* exact kNN + CAGRA-style pruning (graph named P:L293; ref [25] P:L430). */
/* ------------------------------------------------------------------ */
/* Exact k nearest base points of every query, fp32 distances,
 * (dist,id) order.  self_base >= 0 excludes base id (self_base + i) from
 * query i's answer (kNN graph of the base set: queries = base, self_base=0).
 * k <= 1024.  out_ids/out_dists: nq x k.  base/queries/outputs: host or
 * device pointers (copied as needed; caller keeps ownership).
 * Two paths with identical results: large problems (n*nq >= 1e8, k <= 170)
 * screen candidates with tensor-core 3xTF32 GEMMs (cuBLAS), re-rank them
 * with the exact fp32 direct-form distance and certify each query (bound on
 * the screening error), redoing uncertified queries on the direct CUDA-core
 * path; ALGAS_KNN_MODE=direct|screened forces one.  metric COSINE: IP on
 * unit-row copies of base and queries (R29).  Errors: EINVAL on bad
 * arguments, ENOMEM/ECUDA from the device. */
int algas_knn(const float *base, int64_t n, const float *queries, int64_t nq, int32_t dim,
              int32_t metric, int32_t k, int64_t self_base, uint32_t *out_ids, float *out_dists);
/* Rows screened by the tensor-core path since the last call on this thread;
 * *fallback_rows (nullable) = rows the certificate sent to the direct path.
 * Resets both counters. */
int64_t algas_knn_last_stats(int64_t *fallback_rows);
/* CAGRA-style reading R24: rank-based detour count, keep `degree` edges,
 * add reverse edges, merge.  knn: n x knn_degree (sorted rows, no self).
 * out_graph: n x degree. */
int algas_prune(const uint32_t *knn, int64_t n, int32_t knn_degree, int32_t degree,
                uint32_t *out_graph);
/* algas_knn(self) with knn_degree neighbours, then algas_prune if prune != 0
 * (else the first `degree` kNN columns).  out_graph: n x degree. */
int algas_build_graph(const float *data, int64_t n, int32_t dim, int32_t metric,
                      int32_t knn_degree, int32_t degree, int32_t prune, uint32_t *out_graph);
/* Partitioned approximate kNN of the base set (DESIGN.md
 * R30; the paper builds its graphs with CAGRA [25] P:L293 and gives no
 * build algorithm): centres = rows floor(j*n/n_clusters), j < n_clusters;
 * every point joins the clusters of its `overlap` nearest centres
 * ((dist, centre) order); exact kNN (algas_knn, self excluded) inside each
 * cluster; each point's cluster lists merged by (dist, id), duplicates
 * dropped, first k kept, padded with (SENTINEL, +inf).  n_clusters = 1 is
 * the exact kNN.  out_ids/out_dists: n x k, host or device.  EINVAL: n < 2,
 * k outside [1, 1024], n_clusters outside [1, n], overlap outside
 * [1, n_clusters], bad dim/metric. */
int algas_knn_partitioned(const float *data, int64_t n, int32_t dim, int32_t metric, int32_t k,
                          int32_t n_clusters, int32_t overlap, uint32_t *out_ids, float *out_dists);
/* Neighbour-of-neighbour refinement of an approximate kNN list (DESIGN.md
 * R33, the NN-descent step; not in the paper): `rounds` Jacobi rounds, each
 * giving every point p the first k by (dist, id) of its list and the
 * distances to the ids found in the first `fan` entries of the lists of its
 * first `fan` neighbours (p and ids already listed excluded).  fan < 0:
 * R35 rounds with |fan| -- p's first |fan| REVERSE neighbours (the points r
 * whose first |fan| entries hold p, in (rank, r) order) are candidates
 * themselves and their lists are joined like the forward ones.  ids /
 * dists: n x k in/out (rows sorted by (dist, id), SENTINEL / +inf padded),
 * host or device.  EINVAL: |fan| outside [1, min(k, 64)] (32 for R35),
 * k > 1024, bad dim/metric. */
int algas_knn_refine(const float *data, int64_t n, int32_t dim, int32_t metric, int32_t k, int32_t fan,
                     int32_t rounds, uint32_t *ids, float *dists);
/* algas_build_graph with algas_knn_partitioned (+ refine_rounds rounds of
 * algas_knn_refine with refine_fan, 0 = none; refine_fan < 0: R35 rounds
 * with reverse neighbours) as its kNN step; rows the
 * partition left short (clusters of <= knn_degree points) are completed
 * with the exact kNN of those rows over the whole set before the prune. */
int algas_build_graph_partitioned(const float *data, int64_t n, int32_t dim, int32_t metric,
                                  int32_t knn_degree, int32_t degree, int32_t prune,
                                  int32_t n_clusters, int32_t overlap, int32_t refine_fan,
                                  int32_t refine_rounds, uint32_t *out_graph);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif /* ALGAS_H */
