// internal.h -- declarations shared by the translation units of libalgas.so.
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <cstdarg>
#include <cstdint>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/algas.h"
#include "search_core.cuh"

namespace algas {

// ------------------------------------------------------------------ errors
int set_error(int code, const char* fmt, ...);
#define ALGAS_CUDA_TRY(expr)                                                                     \
  do {                                                                                           \
    cudaError_t _e = (expr);                                                                     \
    if (_e != cudaSuccess)                                                                       \
      return ::algas::set_error(ALGAS_ECUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e), \
                                __FILE__, __LINE__);                                             \
  } while (0)

bool is_device_ptr(const void* p);

// ------------------------------------------------------------------ index
struct Workspace {
  std::mutex mu;
  unsigned long long* gtab = nullptr;  // epoch-tagged spill tables
  size_t gtab_entries = 0;
  int* counters = nullptr;             // small device scratch (work counters ...)
  uint32_t epoch = 1;                  // next epoch for the spill tables
  void* h_res = nullptr;               // pinned staging of per-CTA results
  size_t h_res_bytes = 0;
  void* h_st = nullptr;                // pinned staging of per-CTA counters
  size_t h_st_bytes = 0;
  // grow-only device scratch of the dynamic-batching path (per-CTA results,
  // counters, control block, SHARED bitmaps): no allocation per call
  void* d_scratch[4] = {nullptr, nullptr, nullptr, nullptr};
  size_t d_scratch_bytes[4] = {0, 0, 0, 0};
  // host-mapped per-CTA results / counters / Finish words of the dynamic
  // path's streaming merge (grow-only)
  void* m_buf = nullptr;
  size_t m_bytes = 0;
  uint32_t call_id = 0;
};

}  // namespace algas

struct algas_index {
  int device = 0;
  int64_t n = 0;
  int32_t dim = 0, d4 = 0, metric = 0, degree = 0, rp_shift = 0;
  float* d_data = nullptr;      // n x dim
  uint32_t* d_graph = nullptr;  // n x (1 << rp_shift), sentinel padded
  algas::Workspace* ws = nullptr;
};

namespace algas {

// ------------------------------------------------------------------ launch plumbing
// Resolved launch configuration for one search call.
struct Plan {
  int nt;          // threads per CTA
  int ccfg;        // chunk config (TL, CPL) index
  int T;           // CTAs per query
  int smem;        // dynamic shared memory bytes
  int blocks_per_sm;
  SearchCfg cfg;   // L/w/off/S/max_iter/hash filled
  int k;
  int visited_mode;
  int metric;
  int cluster;     // CTAs per search (thread-block cluster), persistent paths
  int occ;         // resident CTAs per SM the persistent kernel is built for (1 or 2)
};
int max_active_clusters(const Plan& pl, int* out);
int check_coresident(const Plan& pl, int slots);

int chunk_config_for(int d4);          // -1 if unsupported

// Shared-memory sizing inside a per-CTA budget: staging rows =
// one step's new vectors (w x Rp, <= 128, two buffers within a quarter of the
// budget), then the largest visited hash (<= 2^15) that still fits.  Values
// already > 0 in *hash_bits / *stage_rows are kept (explicit overrides).
inline void choose_smem(int dp4, int L, int ncap, int S, int w, int Rp, int64_t budget, int* hash_bits,
                        int* stage_rows) {
  const int row_bytes = dp4 * 16;
  int sr = *stage_rows;
  if (sr < 0) {
    sr = 0;  // register gather path: no staging buffers
  } else if (sr == 0) {
    sr = 1;
    while (sr < (w * Rp < 128 ? w * Rp : 128)) sr <<= 1;
    while (sr > 4 && (int64_t)2 * sr * row_bytes > budget / 4) sr >>= 1;
  }
  int hb = *hash_bits;
  if (hb <= 0) {
    int hb_min = 6;
    while ((1LL << hb_min) < 2LL * (S + w * Rp)) ++hb_min;
    hb = 15;
    while (hb > hb_min && smem_layout(dp4, L, ncap, hb, sr).total > budget) --hb;
  }
  *hash_bits = hb;
  *stage_rows = sr;
}
int make_plan(const algas_index* idx, const algas_params* p, int slots, Plan* out, bool persistent,
              bool allow_dsmem = true);
int launch_cluster_size(const Plan& pl);

// spill tables: ensure >= entries, returns base pointer (workspace locked by caller)
int ensure_gtab(algas_index* idx, size_t entries);

// kernel launchers (search_kernels.cu)
struct BatchLaunch {
  const float4* queries;
  int64_t nq;
  uint64_t tag0;
  ResultEntry* res;       // nq x T x k (device)
  CtaStats* stats;        // nq x T (device, nullable)
  unsigned long long* gtab;
  uint32_t epoch_base;
  int* work_counter;      // device int, zeroed by the launcher
  int grid;
};
int launch_batch(const Plan& pl, const BatchLaunch& bl, cudaStream_t st);

// persistent kernel arguments (ring and device-queue feeds)
struct alignas(64) RingSlot {
  volatile uint32_t state;  // host-written: (epoch << 8) | {0 EMPTY, 1 READY, 2 QUIT}
  int32_t k, L, w;
  uint64_t tag;
  uint32_t pad[10];
};
enum { kSlotEmpty = 0, kSlotReady = 1, kSlotQuit = 2 };

struct PersistArgs {
  int mode;                 // 0 ring, 1 device queue
  int slots, T, kmax;
  // device queue
  const float4* queries;
  int64_t nq;
  uint64_t tag0;
  int* queue_head;
  ResultEntry* dq_res;      // nq x T x kmax
  CtaStats* dq_stats;       // nq x T
  // streaming merge (host-mapped dq_res / dq_stats): per (query, CTA) Finish
  // word set to call_id with a system-scope release once its list and
  // counters are written, so the host merges a query while the kernel runs
  uint32_t* dq_done;        // nq x T, or null
  uint32_t call_id;
  // host ring (mapped pointers)
  RingSlot* ring;
  const float4* ring_q;     // slots x d4
  ResultEntry* ring_res;    // slots x T x kmax
  CtaStats* ring_stats;     // slots x T
  uint32_t* ring_done;      // slots x T
  // state mirror (algas_params.state_mirror): per ring entry a device copy
  // of the RingSlot line (state word first) followed by the query, written by
  // the host with stream-ordered copies (payload, then state); null = poll
  // the host-mapped ring
  const uint8_t* mir;
  int64_t mir_stride;       // bytes per mirrored entry (64 + dim*4, 16-B multiple)
  // device mailbox
  unsigned long long* mbox; // slots
  float4* qbuf;             // slots x d4
  int4* dparams;            // slots: {k, L, w, 0}
  unsigned long long* dtag; // slots
  unsigned int* slot_fin;   // slots
  unsigned long long* gtab;
  uint32_t epoch_base;
  // SHARED visited mode: two n-bit bitmaps per slot (vbm_words u32 words
  // each, a multiple of 4; zero at launch), or null -> the epoch-tagged
  // per-slot hash in gtab
  uint32_t* vbm;
  int64_t vbm_words;
};
// SHARED-mode bitmap words per slot for n points (0 = too large: use the hash)
inline int64_t shared_bitmap_words(int64_t n) {
  if (n > (int64_t(1) << 22)) return 0;  // > 512 KB per slot and query to clear
  return ((n + 127) / 128) * 4;
}
int launch_persistent(const Plan& pl, const PersistArgs& pa, cudaStream_t st);

// device control block of a persistent launch: queue head | dparams (16-B) |
// mbox | dtag | slot_fin, every array naturally aligned
inline size_t control_bytes(int slots) { return 256 + (size_t)slots * (16 + 8 + 8 + 4) + 64; }
inline void carve_control(uint8_t* cb, int slots, PersistArgs* pa) {
  pa->queue_head = reinterpret_cast<int*>(cb);
  pa->dparams = reinterpret_cast<int4*>(cb + 256);
  pa->mbox = reinterpret_cast<unsigned long long*>(cb + 256 + (size_t)slots * 16);
  pa->dtag = reinterpret_cast<unsigned long long*>(cb + 256 + (size_t)slots * 24);
  pa->slot_fin = reinterpret_cast<unsigned int*>(cb + 256 + (size_t)slots * 32);
}
int max_blocks_per_sm(const Plan& pl, bool persistent, int* out);

// kernel tables, one per thread count (kernels_nt.cu): the batch or
// persistent kernel for (metric, chunk config, cluster size), or null
void* kernel_table_nt32(int metric, int cc, bool persist, int cs, int occ);
void* kernel_table_nt64(int metric, int cc, bool persist, int cs, int occ);
void* kernel_table_nt128(int metric, int cc, bool persist, int cs, int occ);
void* kernel_table_nt256(int metric, int cc, bool persist, int cs, int occ);
void* kernel_table_nt512(int metric, int cc, bool persist, int cs, int occ);
void* kernel_table_nt1024(int metric, int cc, bool persist, int cs, int occ);

// per-query counters from the T per-CTA records
inline void aggregate_cta_stats(const CtaStats* cs, int T, algas_query_stats* q) {
  *q = algas_query_stats{};
  q->ctas = (uint32_t)T;
  unsigned long long t0 = ~0ull, t1 = 0;
  for (int c = 0; c < T; ++c) {
    q->iters += cs[c].iters;
    if (cs[c].iters > q->max_iters) q->max_iters = cs[c].iters;
    q->parents += cs[c].parents;
    q->dist_evals += cs[c].dist_evals;
    q->cap_hits += cs[c].cap_hit;
    q->spills += cs[c].spilled;
    q->overflows += cs[c].overflow;
    q->cyc_select += cs[c].cyc_select;
    q->cyc_gather += cs[c].cyc_gather;
    q->cyc_dist += cs[c].cyc_dist;
    q->cyc_sort += cs[c].cyc_sort;
    if (cs[c].t_start < t0) t0 = cs[c].t_start;
    if (cs[c].t_end > t1) t1 = cs[c].t_end;
    if (c == 0 || cs[c].t_loop0 < q->t_loop_first_ns) q->t_loop_first_ns = cs[c].t_loop0;
    if (cs[c].t_loop0 > q->t_loop_last_ns) q->t_loop_last_ns = cs[c].t_loop0;
    if (cs[c].t_loop1 > q->t_loop_end_ns) q->t_loop_end_ns = cs[c].t_loop1;
    if (cs[c].t_entry > q->t_entry_last_ns) q->t_entry_last_ns = cs[c].t_entry;
    q->merges_bitonic += cs[c].mg_bitonic;
    q->merges_rank += cs[c].mg_rank;
  }
  q->t_start_ns = t0 == ~0ull ? 0 : t0;
  q->t_end_ns = t1;
}

// partitioned graph build (build_part.cu, R30 / R33)
struct ClusterBlock {
  int32_t cluster;  // a CTA of the batched cluster kNN: 64 member rows of one cluster
  int32_t row0;
};
int launch_cluster_knn(const float* X, int d, int metric, const uint32_t* mem, const int64_t* start,
                       const std::vector<ClusterBlock>& blocks, int k, uint64_t* out);
int launch_merge_lists(const uint64_t* lists, const uint32_t* slot_of, int64_t n, int c, int k, uint32_t* out_ids,
                       float* out_d);
int launch_refine(const float* X, int d, int metric, int64_t n, int k, int fan, const uint32_t* in_ids,
                  const float* in_d, const uint32_t* rev, uint32_t* out_ids, float* out_d);
constexpr int kPartMaxKnn = 128;  // list length the batched cluster kNN keeps in shared memory

// graph build's contraction on the tensor cores (knn_tc.cu): D (qb x nb, row
// stride ldD) = Q . X^T from TF32 hi/lo splits (3xTF32), tcgen05 + TMEM
int tc_dot_3xtf32(const float* Qh, const float* Ql, int64_t qb, const float* Xh, const float* Xl, int64_t nb, int d,
                  float* D, int64_t ldD, cudaStream_t st);

// host TopK merge (runtime.cpp)
int32_t merge_cta_lists(const ResultEntry* res, int T, int kin, int k, uint32_t* out_ids, float* out_d);

}  // namespace algas
