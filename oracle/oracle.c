/*
 * oracle.c -- plain, slow, single-threaded CPU reference ("oracle") for the
 * ALGAS hot path (Chen et al., IPDPS'25; /root/reference/PAPER.md, cited
 * below as P:L<line>).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load this library.  It
 * shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_ipps_chencyzw025_b200/csrc); neither side includes the other.
 *
 * Build: gcc -O2 -ffp-contract=off -fPIC -shared (no -ffast-math), so every
 * fp32 sum below is evaluated left to right in index order, one rounding per
 * operation, exactly as written.
 *
 * Functions and the passage each follows:
 *   orc_splitmix64 / orc_entry_point  random entry points ("enters
 *                                     random entry point"; Alg.1 `p`)
 *                                     -- counter-based generator, R5
 *   orc_distance                      F(a,b) of the k-NN problem:
 *                                     squared Euclidean or negated inner
 *                                     product (R2, R3)
 *   orc_brute_force  (O1)             exact k-NN by definition
 *   orc_search       (O2)             Algorithm 1 + beam extend
 *                                      + multi-CTA with
 *                                     per-CTA lists +
 *                                     host TopK merge & filter
 *   orc_merge_topk   (A9)             host priority-queue merge
 *   orc_tuner_*                       adaptive tuning equations (P:L231,
 *                                     P:L235)
 *   orc_knn_refine   (f4, R33)        one neighbour-of-neighbour refinement
 *                                     round of an approximate kNN list
 *                                     (R33; not in the paper:
 *                                     parity unpinned by it, pinned by its
 *                                     exact fixed point and a hand example)
 *   orc_knn_refine_rev (f4, R35)      the same round with reverse neighbours
 *                                     joined (R35; not in the paper:
 *                                     parity unpinned by it, pinned by a hand
 *                                     example, fixed point, superset property)
 *   orc_prune        (K10)            CAGRA-style rank-based detour pruning +
 *                                     reverse edges (graph named at P:L293,
 *                                     algorithm from ref [25] P:L430, which is
 *                                     NOT in PAPER.md -> "parity unpinned" by
 *                                     the paper; pinned by hand-worked
 *                                     examples and invariants, R24)
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_SENTINEL 0xFFFFFFFFu
#define ORC_L2 0
#define ORC_IP 1
#define ORC_COSINE 2

/* ------------------------------------------------------------------ */
/* Counter-based generator for entry points (R5).            */
/* splitmix64 (Steele, Lea, Flood 2014): one output step.              */
/* ------------------------------------------------------------------ */
uint64_t orc_splitmix64(uint64_t z)
{
    z = z + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* j-th random entry point of CTA `cta` for query `tag`. */
uint32_t orc_entry_point(uint64_t seed, uint64_t tag, uint32_t cta, uint32_t j, int64_t n)
{
    uint64_t a = orc_splitmix64(((uint64_t)cta << 32) | (uint64_t)j);
    uint64_t b = orc_splitmix64(tag ^ a);
    uint64_t h = orc_splitmix64(seed ^ b);
    return (uint32_t)(h % (uint64_t)n);
}

/* ------------------------------------------------------------------ */
/* F(a,b).  L2: sum_j (q_j - x_j)^2 (squared, no sqrt: R2).     */
/* IP: -sum_j q_j x_j (smaller = more similar: R3).                    */
/* ------------------------------------------------------------------ */
float orc_distance(const float *q, const float *x, int32_t d, int32_t metric)
{
    float acc = 0.0f;
    int32_t j;
    if (metric == ORC_L2) {
        for (j = 0; j < d; j++) {
            float t = q[j] - x[j];
            acc = acc + t * t;
        }
        return acc;
    }
    if (metric == ORC_COSINE) {
        /* COSINE (two of the paper's datasets are "cosine";
         * DESIGN.md R29): -(q.x) / (|q| |x|), the negated cosine similarity,
         * in double; a zero vector has distance 0 to everything. */
        double qx = 0.0, qq = 0.0, xx = 0.0;
        for (j = 0; j < d; j++) {
            qx += (double)q[j] * (double)x[j];
            qq += (double)q[j] * (double)q[j];
            xx += (double)x[j] * (double)x[j];
        }
        if (qq == 0.0 || xx == 0.0) return 0.0f;
        return (float)(-qx / (sqrt(qq) * sqrt(xx)));
    }
    for (j = 0; j < d; j++)
        acc = acc + q[j] * x[j];
    return -acc;
}

/* Lexicographic (dist, id) order (R4). */
static int key_less(float da, uint32_t ia, float db, uint32_t ib)
{
    if (da < db) return 1;
    if (db < da) return 0;
    return ia < ib;
}

/* ------------------------------------------------------------------ */
/* O1: exact k-NN.  For each query, every base point is scored  */
/* and the k smallest by (dist, id) are kept.  If self_base >= 0, base  */
/* point (self_base + query index) is excluded (graph construction:     */
/* "kNN of every base point, excluding itself").  Short rows are padded  */
/* with (SENTINEL, +inf).                                               */
/* ------------------------------------------------------------------ */
void orc_brute_force(const float *X, int64_t n, int32_t d, int32_t metric,
                     const float *Q, int64_t nq, int32_t k, int64_t self_base,
                     uint32_t *out_ids, float *out_d)
{
    int64_t qi, i;
    for (qi = 0; qi < nq; qi++) {
        const float *q = Q + qi * (int64_t)d;
        uint32_t *bi = out_ids + qi * (int64_t)k;
        float *bd = out_d + qi * (int64_t)k;
        int32_t cnt = 0, p;
        for (i = 0; i < n; i++) {
            float di;
            if (self_base >= 0 && i == self_base + qi) continue;
            di = orc_distance(q, X + i * (int64_t)d, d, metric);
            if (cnt == k && !key_less(di, (uint32_t)i, bd[k - 1], bi[k - 1]))
                continue;
            /* insertion into the sorted top-k */
            p = (cnt < k) ? cnt : k - 1;
            while (p > 0 && key_less(di, (uint32_t)i, bd[p - 1], bi[p - 1])) {
                bd[p] = bd[p - 1];
                bi[p] = bi[p - 1];
                p--;
            }
            bd[p] = di;
            bi[p] = (uint32_t)i;
            if (cnt < k) cnt++;
        }
        for (p = cnt; p < k; p++) {
            bi[p] = ORC_SENTINEL;
            bd[p] = __builtin_inff();
        }
    }
}

/* ------------------------------------------------------------------ */
/* Candidate-list entry of Algorithm 1: point id, its distance to q and  */
/* the "checked" mark.                                       */
/* ------------------------------------------------------------------ */
typedef struct {
    float dist;
    uint32_t id;
    int32_t checked;
} orc_cand;

static int cand_cmp(const void *a, const void *b)
{
    const orc_cand *x = (const orc_cand *)a, *y = (const orc_cand *)b;
    if (key_less(x->dist, x->id, y->dist, y->id)) return -1;
    if (key_less(y->dist, y->id, x->dist, x->id)) return 1;
    return 0;
}

/* Visited table = bitmap over all n points ("implemented as a bitmap"). */
static int bm_test(const uint8_t *bm, uint32_t id) { return (bm[id >> 3] >> (id & 7)) & 1; }
static void bm_set(uint8_t *bm, uint32_t id) { bm[id >> 3] = (uint8_t)(bm[id >> 3] | (1u << (id & 7))); }

/* Search parameters (R5-R10). */
typedef struct {
    int32_t k;              /* TopK returned */
    int32_t L;              /* candidate list max length, "itopk" (L >= k P:L219) */
    int32_t w;              /* parents per beam-extend step */
    int32_t off;            /* offset_beam; >= L disables beam extend */
    int32_t T;              /* CTAs per query, N_parallel */
    int32_t S;              /* random entry points per CTA (S=1 is Alg.1's single p) */
    int32_t max_iter;       /* safety cap on steps per CTA (R8) */
    int32_t shared_visited; /* 1: one visited table shared by the query's CTAs */
    uint64_t seed;
} orc_params;

/* Per-query counters (summed over the query's CTAs). */
typedef struct {
    int64_t iters;      /* steps = candidate-list maintenance operations */
    int64_t parents;    /* expanded candidate points */
    int64_t dist_evals; /* distance computations (P:L217 step 3) */
    int64_t cap_hits;   /* CTAs stopped by max_iter instead of P:L217's Finish */
    int64_t max_iters;  /* max steps over the query's CTAs */
} orc_stats;

/* ------------------------------------------------------------------ */
/* A9: host TopK merge & filter.  Merges m (id, dist) entries   */
/* by (dist, id), filters sentinels and duplicate ids (keeps the first   */
/* = smallest key; R11), returns the first k, padded (R12).             */
/* ------------------------------------------------------------------ */
int32_t orc_merge_topk(const uint32_t *ids, const float *dists, int32_t m, int32_t k,
                       uint32_t *out_ids, float *out_d)
{
    orc_cand *all = (orc_cand *)malloc(sizeof(orc_cand) * (size_t)(m > 0 ? m : 1));
    int32_t i, cnt = 0, outn = 0;
    for (i = 0; i < m; i++) {
        if (ids[i] == ORC_SENTINEL) continue;
        all[cnt].dist = dists[i];
        all[cnt].id = ids[i];
        all[cnt].checked = 0;
        cnt++;
    }
    qsort(all, (size_t)cnt, sizeof(orc_cand), cand_cmp);
    for (i = 0; i < cnt && outn < k; i++) {
        {
            /* a duplicate id (the same point found by two CTAs) keeps only
               its first, i.e. smallest-key, copy */
            int32_t t, dup = 0;
            for (t = 0; t < outn; t++)
                if (out_ids[t] == all[i].id) { dup = 1; break; }
            if (dup) continue;
        }
        out_ids[outn] = all[i].id;
        out_d[outn] = all[i].dist;
        outn++;
    }
    for (i = outn; i < k; i++) {
        out_ids[i] = ORC_SENTINEL;
        out_d[i] = __builtin_inff();
    }
    free(all);
    return outn;
}

/* ------------------------------------------------------------------ */
/* O2: reference search for one query.                                   */
/*                                                                       */
/* Per CTA c: own candidate list S_c, S random entry    */
/* points.  Each step (Alg.1 lines 6-18; P:L217 steps 1-4):             */
/*   U = unchecked positions of S_c in list order                         */
/*   Finish if U empty (P:L217 step 1) or steps >= max_iter (R8)          */
/*   diffusing latches when U[0] >= off (R6)                      */
/*   parents P = U[:w] if diffusing else U[:1] (Alg.1 line 6)     */
/*   mark P checked (Alg.1 line 7)                                        */
/*   for each parent, each neighbor (row order): skip sentinel / visited, */
/*     mark visited, score, add (P:L217 steps 1-3, Alg.1 lines 8-13)      */
/*   S_c = first L of sort(S_c + new) by (dist,id)  */
/* The query's CTAs step round-robin in rank order (matters only for the  */
/* shared visited table).  Each CTA pushes its first k (R10);     */
/* the host merges them.                                        */
/*                                                                       */
/* cta_ids / cta_d (nullable): T*k per-CTA results before the merge.     */
/* Returns 0, or -1 on allocation failure / bad arguments.               */
/* ------------------------------------------------------------------ */
int32_t orc_search(const float *X, int64_t n, int32_t d, int32_t metric,
                   const uint32_t *G, int32_t R,
                   const float *q, uint64_t tag, const orc_params *pp,
                   uint32_t *out_ids, float *out_d,
                   uint32_t *cta_ids, float *cta_d, orc_stats *st)
{
    const int32_t T = pp->T, L = pp->L, w = pp->w, k = pp->k;
    const int32_t cap = L + w * R + pp->S; /* list + one step's new points */
    orc_cand **S = (orc_cand **)calloc((size_t)T, sizeof(orc_cand *));
    int32_t *cnt = (int32_t *)calloc((size_t)T, sizeof(int32_t));
    int32_t *iters = (int32_t *)calloc((size_t)T, sizeof(int32_t));
    int32_t *diff = (int32_t *)calloc((size_t)T, sizeof(int32_t));
    int32_t *active = (int32_t *)calloc((size_t)T, sizeof(int32_t));
    int32_t *U = (int32_t *)malloc(sizeof(int32_t) * (size_t)(w > 0 ? w : 1));
    size_t bm_bytes = (size_t)((n + 7) / 8);
    int32_t nvis = pp->shared_visited ? 1 : T;
    uint8_t **V = (uint8_t **)calloc((size_t)nvis, sizeof(uint8_t *));
    uint32_t *all_ids = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)T * (size_t)k);
    float *all_d = (float *)malloc(sizeof(float) * (size_t)T * (size_t)k);
    int32_t c, i, j, nactive, rc = 0;
    orc_stats local;
    memset(&local, 0, sizeof(local));

    if (!S || !cnt || !iters || !diff || !active || !U || !V || !all_ids || !all_d ||
        T < 1 || L < 1 || w < 1 || k < 1 || pp->S < 1 || n < 1) {
        rc = -1;
        goto done;
    }
    for (c = 0; c < nvis; c++) {
        V[c] = (uint8_t *)calloc(bm_bytes, 1);
        if (!V[c]) { rc = -1; goto done; }
    }

    /* Entry: S random points per CTA (Alg.1 line 5 `S.add(p)`).
       A CTA keeps its own (deduplicated) seeds even if another CTA of the
       query already marked them in a shared table (R21). */
    for (c = 0; c < T; c++) {
        uint8_t *Vc = V[pp->shared_visited ? 0 : c];
        S[c] = (orc_cand *)malloc(sizeof(orc_cand) * (size_t)cap);
        if (!S[c]) { rc = -1; goto done; }
        for (j = 0; j < pp->S; j++) {
            uint32_t e = orc_entry_point(pp->seed, tag, (uint32_t)c, (uint32_t)j, n);
            int32_t dup = 0, t;
            for (t = 0; t < cnt[c]; t++)
                if (S[c][t].id == e) { dup = 1; break; }
            if (dup) continue;
            bm_set(Vc, e);
            S[c][cnt[c]].dist = orc_distance(q, X + (int64_t)e * d, d, metric);
            S[c][cnt[c]].id = e;
            S[c][cnt[c]].checked = 0;
            cnt[c]++;
            local.dist_evals++;
        }
        qsort(S[c], (size_t)cnt[c], sizeof(orc_cand), cand_cmp);
        if (cnt[c] > L) cnt[c] = L;
        active[c] = 1;
    }

    nactive = T;
    while (nactive > 0) {
        for (c = 0; c < T; c++) {
            uint8_t *Vc;
            int32_t nu = 0, np, base;
            if (!active[c]) continue;
            Vc = V[pp->shared_visited ? 0 : c];
            /* U = first (up to w) unchecked positions in list order */
            for (i = 0; i < cnt[c] && nu < w; i++)
                if (!S[c][i].checked) U[nu++] = i;
            if (nu == 0 || iters[c] >= pp->max_iter) {
                if (nu > 0) local.cap_hits++;
                active[c] = 0;
                nactive--;
                continue;
            }
            if (U[0] >= pp->off) diff[c] = 1;      /* enter diffusing phase (sticky) */
            np = diff[c] ? nu : 1;                  /* several points at once */
            for (i = 0; i < np; i++) S[c][U[i]].checked = 1;
            base = cnt[c];
            for (i = 0; i < np; i++) {
                uint32_t p = S[c][U[i]].id;
                for (j = 0; j < R; j++) {
                    uint32_t nb = G[(int64_t)p * R + j];
                    if (nb == ORC_SENTINEL) continue;
                    if (bm_test(Vc, nb)) continue;          /* P:L217 step 2 */
                    bm_set(Vc, nb);
                    S[c][base].dist = orc_distance(q, X + (int64_t)nb * d, d, metric);
                    S[c][base].id = nb;
                    S[c][base].checked = 0;
                    base++;
                    local.dist_evals++;
                }
            }
            local.parents += np;
            qsort(S[c], (size_t)base, sizeof(orc_cand), cand_cmp); /* Alg.1 line 15 */
            cnt[c] = base > L ? L : base;                          /* Alg.1 lines 16-18 */
            iters[c]++;
        }
    }

    for (c = 0; c < T; c++) {
        for (i = 0; i < k; i++) {
            if (i < cnt[c]) {
                all_ids[c * k + i] = S[c][i].id;
                all_d[c * k + i] = S[c][i].dist;
            } else {
                all_ids[c * k + i] = ORC_SENTINEL;
                all_d[c * k + i] = __builtin_inff();
            }
        }
        local.iters += iters[c];
        if (iters[c] > local.max_iters) local.max_iters = iters[c];
    }
    if (cta_ids) memcpy(cta_ids, all_ids, sizeof(uint32_t) * (size_t)T * (size_t)k);
    if (cta_d) memcpy(cta_d, all_d, sizeof(float) * (size_t)T * (size_t)k);
    orc_merge_topk(all_ids, all_d, T * k, k, out_ids, out_d);
    if (st) *st = local;

done:
    if (S) for (c = 0; c < T; c++) free(S[c]);
    if (V) for (c = 0; c < nvis; c++) free(V[c]);
    free(S); free(cnt); free(iters); free(diff); free(active); free(U); free(V);
    free(all_ids); free(all_d);
    return rc;
}

/* Batch driver: query qi uses tag = tag0 + qi (R23). */
int32_t orc_search_batch(const float *X, int64_t n, int32_t d, int32_t metric,
                         const uint32_t *G, int32_t R,
                         const float *Q, int64_t nq, uint64_t tag0, const orc_params *pp,
                         uint32_t *out_ids, float *out_d,
                         uint32_t *cta_ids, float *cta_d, orc_stats *st)
{
    int64_t qi;
    for (qi = 0; qi < nq; qi++) {
        int64_t ck = (int64_t)pp->T * pp->k;
        int32_t rc = orc_search(X, n, d, metric, G, R, Q + qi * (int64_t)d, tag0 + (uint64_t)qi, pp,
                                out_ids + qi * pp->k, out_d + qi * pp->k,
                                cta_ids ? cta_ids + qi * ck : NULL,
                                cta_d ? cta_d + qi * ck : NULL,
                                st ? st + qi : NULL);
        if (rc) return rc;
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* Adaptive tuning equations, written out as printed.       */
/* ------------------------------------------------------------------ */
/* N_parallel * slot <= N_SM * N_max_block_per_SM  ->  largest N_parallel */
int32_t orc_tuner_max_parallel(int32_t slots, int32_t n_sm, int32_t max_block_per_sm)
{
    return (int32_t)(((int64_t)n_sm * max_block_per_sm) / slots);
}
/* N_block_per_SM = align(N_parallel * slot / N_SM), align = ceil (R13) */
int32_t orc_tuner_blocks_per_sm(int32_t n_parallel, int32_t slots, int32_t n_sm)
{
    int64_t t = (int64_t)n_parallel * slots;
    return (int32_t)((t + n_sm - 1) / n_sm);
}
/* M_avail_per_block <= M_per_SM / N_block_per_SM - M_reserved_per_block (bytes) */
int64_t orc_tuner_smem_per_block(int64_t m_per_sm, int32_t blocks_per_sm, int64_t m_reserved)
{
    return m_per_sm / blocks_per_sm - m_reserved;
}

/* ------------------------------------------------------------------ */
/* K10 reading (R24): CAGRA-style optimisation of a kNN graph.           */
/*   knn: n x K, each row sorted by (dist,id), no self, no sentinels.    */
/*   1. detour count of edge x->y_j: #{ i < j : y_j occurs among the     */
/*      first j entries of knn[y_i] } (a route x->y_i->y_j whose two     */
/*      ranks are both < j).                                             */
/*   2. pruned P[x]: the K edges ordered by (count, j); keep first R.    */
/*   3. reverse: for each x and rank r < R of P[x], edge P[x][r] -> x    */
/*      with priority (r, x); Rev[y] keeps the R smallest priorities.    */
/*   4. out[x] = P[x][0 .. R/2) ++ Rev[x] (priority order, skipping ids  */
/*      present) ++ P[x][R/2 .. R) (skipping ids present), cut to R;     */
/*      pad with SENTINEL.                                               */
/* ------------------------------------------------------------------ */
typedef struct { int32_t count, j; uint32_t id; } orc_edge;
static int edge_cmp(const void *a, const void *b)
{
    const orc_edge *x = (const orc_edge *)a, *y = (const orc_edge *)b;
    if (x->count != y->count) return x->count < y->count ? -1 : 1;
    if (x->j != y->j) return x->j < y->j ? -1 : 1;
    return 0;
}
typedef struct { int32_t r; uint32_t src; } orc_rev;
static int rev_cmp(const void *a, const void *b)
{
    const orc_rev *x = (const orc_rev *)a, *y = (const orc_rev *)b;
    if (x->r != y->r) return x->r < y->r ? -1 : 1;
    if (x->src != y->src) return x->src < y->src ? -1 : 1;
    return 0;
}

int32_t orc_prune(const uint32_t *knn, int64_t n, int32_t K, int32_t R, uint32_t *out,
                  uint32_t *pruned /* nullable n x R, step 2 output */)
{
    uint32_t *P = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)n * (size_t)R);
    orc_edge *e = (orc_edge *)malloc(sizeof(orc_edge) * (size_t)K);
    int32_t *nrev = (int32_t *)calloc((size_t)n, sizeof(int32_t));
    orc_rev *rev = NULL;
    int64_t x;
    int32_t i, j, t;
    if (!P || !e || !nrev || R > K || R < 1) { free(P); free(e); free(nrev); return -1; }

    for (x = 0; x < n; x++) {
        const uint32_t *row = knn + x * K;
        for (j = 0; j < K; j++) {
            int32_t count = 0;
            for (i = 0; i < j; i++) {
                const uint32_t *ri = knn + (int64_t)row[i] * K;
                for (t = 0; t < j; t++)
                    if (ri[t] == row[j]) { count++; break; }
            }
            e[j].count = count;
            e[j].j = j;
            e[j].id = row[j];
        }
        qsort(e, (size_t)K, sizeof(orc_edge), edge_cmp);
        for (j = 0; j < R; j++) P[x * R + j] = e[j].id;
    }
    if (pruned) memcpy(pruned, P, sizeof(uint32_t) * (size_t)n * (size_t)R);

    /* reverse edges: gather all, then per target keep the R smallest priorities */
    for (x = 0; x < n; x++)
        for (j = 0; j < R; j++) nrev[P[x * R + j]]++;
    {
        int64_t *start = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
        int64_t *fill = (int64_t *)calloc((size_t)n, sizeof(int64_t));
        rev = (orc_rev *)malloc(sizeof(orc_rev) * (size_t)n * (size_t)R);
        if (!start || !fill || !rev) { free(start); free(fill); free(rev); free(P); free(e); free(nrev); return -1; }
        start[0] = 0;
        for (x = 0; x < n; x++) start[x + 1] = start[x] + nrev[x];
        for (x = 0; x < n; x++)
            for (j = 0; j < R; j++) {
                uint32_t y = P[x * R + j];
                rev[start[y] + fill[y]].r = j;
                rev[start[y] + fill[y]].src = (uint32_t)x;
                fill[y]++;
            }
        for (x = 0; x < n; x++) {
            orc_rev *rx = rev + start[x];
            int32_t m = nrev[x], o = 0, h = R / 2;
            uint32_t *ox = out + x * R;
            qsort(rx, (size_t)m, sizeof(orc_rev), rev_cmp);
            if (m > R) m = R;
            for (j = 0; j < h; j++) ox[o++] = P[x * R + j];
            for (i = 0; i < m && o < R; i++) {
                int32_t dup = 0;
                for (t = 0; t < o; t++) if (ox[t] == rx[i].src) { dup = 1; break; }
                if (!dup) ox[o++] = rx[i].src;
            }
            for (j = h; j < R && o < R; j++) {
                int32_t dup = 0;
                for (t = 0; t < o; t++) if (ox[t] == P[x * R + j]) { dup = 1; break; }
                if (!dup) ox[o++] = P[x * R + j];
            }
            for (; o < R; o++) ox[o] = ORC_SENTINEL;
        }
        free(start);
        free(fill);
    }
    free(rev); free(P); free(e); free(nrev);
    return 0;
}

/* ------------------------------------------------------------------ */
/* f4 reading R33: one neighbour-of-neighbour refinement round of an      */
/* approximate kNN list (the NN-descent step).  For every point p, in     */
/* id order, from the INPUT lists only (a Jacobi round):                  */
/*   C(p) = { x = in[q][b] : q = in[p][a], a < fan, b < fan,              */
/*            x != SENTINEL, x != p, x not in in[p] }, each x once        */
/*   out[p] = first k of sort_by_(dist,id)( in[p] u {(F(p,x), x) : x in C} ) */
/*   padded with (SENTINEL, +inf).  F is orc_distance.            */
/* in/out: n x k, rows sorted by (dist, id), SENTINEL-padded.            */
/* Returns 0, or -1 on bad arguments / allocation failure.               */
/* ------------------------------------------------------------------ */
int32_t orc_knn_refine(const float *X, int64_t n, int32_t d, int32_t metric, int32_t k, int32_t fan,
                       const uint32_t *ids_in, const float *d_in, uint32_t *ids_out, float *d_out)
{
    uint8_t *mark;
    orc_cand *c;
    int64_t p;
    int32_t a, b, i, m;
    if (n < 1 || k < 1 || fan < 1 || fan > k) return -1;
    mark = (uint8_t *)calloc((size_t)((n + 7) / 8), 1);
    c = (orc_cand *)malloc(sizeof(orc_cand) * (size_t)(k + fan * fan));
    if (!mark || !c) { free(mark); free(c); return -1; }
    for (p = 0; p < n; p++) {
        m = 0;
        bm_set(mark, (uint32_t)p);
        for (i = 0; i < k; i++) {             /* the current list */
            uint32_t x = ids_in[p * k + i];
            if (x == ORC_SENTINEL) continue;
            bm_set(mark, x);
            c[m].dist = d_in[p * k + i];
            c[m].id = x;
            c[m].checked = 0;
            m++;
        }
        for (a = 0; a < fan; a++) {           /* neighbours of its first fan neighbours */
            uint32_t q = ids_in[p * k + a];
            if (q == ORC_SENTINEL) continue;
            for (b = 0; b < fan; b++) {
                uint32_t x = ids_in[(int64_t)q * k + b];
                if (x == ORC_SENTINEL || bm_test(mark, x)) continue;
                bm_set(mark, x);
                c[m].dist = orc_distance(X + p * (int64_t)d, X + (int64_t)x * d, d, metric);
                c[m].id = x;
                c[m].checked = 0;
                m++;
            }
        }
        qsort(c, (size_t)m, sizeof(orc_cand), cand_cmp);
        for (i = 0; i < k; i++) {
            ids_out[p * k + i] = i < m ? c[i].id : ORC_SENTINEL;
            d_out[p * k + i] = i < m ? c[i].dist : __builtin_inff();
        }
        /* clear the marks of this point */
        mark[p >> 3] = 0;
        for (i = 0; i < m; i++) mark[c[i].id >> 3] = 0;
    }
    free(mark);
    free(c);
    return 0;
}


/* ------------------------------------------------------------------ */
/* f4 reading R35: the R33 round with reverse neighbours (the NN-descent  */
/* local join over forward and reverse lists).  From the INPUT lists:     */
/*   rev(p) = the first fan pairs (a, r), in (a, r) order, with           */
/*            in[r][a] == p, a < fan, r != p  (p's reverse neighbours)    */
/*   N(p)   = { in[p][a] : a < fan } u { r : (a, r) in rev(p) }           */
/*   C(p)   = { r in rev(p) } u { x = in[q][b] : q in N(p), b < fan },    */
/*            x != SENTINEL, x != p, x not in in[p], each x once           */
/*   out[p] = first k of sort_by_(dist,id)( in[p] u {(F(p,x), x) : x in C} ) */
/* padded with (SENTINEL, +inf).  Same layouts and return as            */
/* orc_knn_refine.                                                        */
/* ------------------------------------------------------------------ */
typedef struct {
    int32_t a;
    uint32_t r;
} orc_rv;
static int rv_cmp(const void *x, const void *y)
{
    const orc_rv *u = (const orc_rv *)x, *v = (const orc_rv *)y;
    if (u->a != v->a) return u->a < v->a ? -1 : 1;
    if (u->r != v->r) return u->r < v->r ? -1 : 1;
    return 0;
}

int32_t orc_knn_refine_rev(const float *X, int64_t n, int32_t d, int32_t metric, int32_t k, int32_t fan,
                           const uint32_t *ids_in, const float *d_in, uint32_t *ids_out, float *d_out)
{
    uint8_t *mark;
    orc_cand *c;
    int64_t *cnt, *start, p, r, tot = 0;
    int64_t *fill;
    orc_rv *rv;
    uint32_t *rev;
    int32_t a, b, i, m, nr;
    if (n < 1 || k < 1 || fan < 1 || fan > k) return -1;
    cnt = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    start = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    fill = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    rev = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)n * fan);
    mark = (uint8_t *)calloc((size_t)((n + 7) / 8), 1);
    c = (orc_cand *)malloc(sizeof(orc_cand) * (size_t)(k + 2 * fan * fan + fan));
    if (!cnt || !start || !fill || !rev || !mark || !c) {
        free(cnt); free(start); free(fill); free(rev); free(mark); free(c);
        return -1;
    }
    /* reverse pairs (a, r) of every point, then the first fan by (a, r) */
    for (r = 0; r < n; r++)
        for (a = 0; a < fan; a++) {
            uint32_t q = ids_in[r * k + a];
            if (q != ORC_SENTINEL && (int64_t)q != r) cnt[q]++;
        }
    for (p = 0; p < n; p++) { start[p] = tot; tot += cnt[p]; }
    rv = (orc_rv *)malloc(sizeof(orc_rv) * (size_t)(tot > 0 ? tot : 1));
    if (!rv) { free(cnt); free(start); free(fill); free(rev); free(mark); free(c); return -1; }
    for (r = 0; r < n; r++)
        for (a = 0; a < fan; a++) {
            uint32_t q = ids_in[r * k + a];
            if (q == ORC_SENTINEL || (int64_t)q == r) continue;
            rv[start[q] + fill[q]].a = a;
            rv[start[q] + fill[q]].r = (uint32_t)r;
            fill[q]++;
        }
    for (p = 0; p < n; p++) {
        qsort(rv + start[p], (size_t)cnt[p], sizeof(orc_rv), rv_cmp);
        for (i = 0; i < fan; i++) rev[p * fan + i] = i < cnt[p] ? rv[start[p] + i].r : ORC_SENTINEL;
    }
    for (p = 0; p < n; p++) {
        m = 0;
        bm_set(mark, (uint32_t)p);
        for (i = 0; i < k; i++) {             /* the current list */
            uint32_t x = ids_in[p * k + i];
            if (x == ORC_SENTINEL) continue;
            bm_set(mark, x);
            c[m].dist = d_in[p * k + i];
            c[m].id = x;
            c[m].checked = 0;
            m++;
        }
        for (i = 0; i < fan; i++) {           /* the reverse neighbours themselves */
            uint32_t x = rev[p * fan + i];
            if (x == ORC_SENTINEL || bm_test(mark, x)) continue;
            bm_set(mark, x);
            c[m].dist = orc_distance(X + p * (int64_t)d, X + (int64_t)x * d, d, metric);
            c[m].id = x;
            c[m].checked = 0;
            m++;
        }
        for (nr = 0; nr < 2 * fan; nr++) {    /* lists of the forward, then the reverse neighbours */
            uint32_t q = nr < fan ? ids_in[p * k + nr] : rev[p * fan + (nr - fan)];
            if (q == ORC_SENTINEL) continue;
            for (b = 0; b < fan; b++) {
                uint32_t x = ids_in[(int64_t)q * k + b];
                if (x == ORC_SENTINEL || bm_test(mark, x)) continue;
                bm_set(mark, x);
                c[m].dist = orc_distance(X + p * (int64_t)d, X + (int64_t)x * d, d, metric);
                c[m].id = x;
                c[m].checked = 0;
                m++;
            }
        }
        qsort(c, (size_t)m, sizeof(orc_cand), cand_cmp);
        for (i = 0; i < k; i++) {
            ids_out[p * k + i] = i < m ? c[i].id : ORC_SENTINEL;
            d_out[p * k + i] = i < m ? c[i].dist : __builtin_inff();
        }
        mark[p >> 3] = 0;
        for (i = 0; i < m; i++) mark[c[i].id >> 3] = 0;
    }
    free(cnt); free(start); free(fill); free(rev); free(mark); free(c); free(rv);
    return 0;
}
