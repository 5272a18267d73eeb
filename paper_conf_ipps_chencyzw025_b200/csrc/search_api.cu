// search_api.cu -- C-ABI: errors, index lifetime, planning, batch search
// (algas_search / algas_search_ex) and dynamic batching from an HBM queue
// (algas_search_dynamic).  The host merge of per-CTA results is in
// runtime.cu; graph construction in knn.cu.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <thread>
#include <vector>

#include "internal.h"

namespace algas {

static thread_local std::string g_err = "no error";

int set_error(int code, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    (void)cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

int ensure_gtab(algas_index* idx, size_t entries) {
  Workspace* ws = idx->ws;
  if (ws->gtab_entries >= entries) return ALGAS_OK;
  if (ws->gtab) cudaFree(ws->gtab);
  ws->gtab = nullptr;
  ws->gtab_entries = 0;
  ALGAS_CUDA_TRY(cudaMalloc(&ws->gtab, entries * sizeof(unsigned long long)));
  ALGAS_CUDA_TRY(cudaMemset(ws->gtab, 0, entries * sizeof(unsigned long long)));
  ws->gtab_entries = entries;
  ws->epoch = 1;
  return ALGAS_OK;
}

// grow-only device scratch buffer `i` of the workspace (caller holds ws->mu;
// every user synchronizes its stream before releasing the lock)
static int ensure_scratch(Workspace* ws, int i, size_t bytes, void** out) {
  bytes = std::max<size_t>(bytes, 256);
  if (ws->d_scratch_bytes[i] < bytes) {
    if (ws->d_scratch[i]) {
      ALGAS_CUDA_TRY(cudaDeviceSynchronize());
      cudaFree(ws->d_scratch[i]);
    }
    ws->d_scratch[i] = nullptr;
    ws->d_scratch_bytes[i] = 0;
    ALGAS_CUDA_TRY(cudaMalloc(&ws->d_scratch[i], bytes));
    ws->d_scratch_bytes[i] = bytes;
  }
  *out = ws->d_scratch[i];
  return ALGAS_OK;
}

// Reserve `count` consecutive spill-table epochs; clears the tables on wrap.
static int take_epochs(algas_index* idx, uint64_t count, uint32_t* base, cudaStream_t st) {
  Workspace* ws = idx->ws;
  if ((uint64_t)ws->epoch + count >= 0xFFFFFFF0ull) {
    if (ws->gtab) ALGAS_CUDA_TRY(cudaMemsetAsync(ws->gtab, 0, ws->gtab_entries * 8, st));
    ws->epoch = 1;
  }
  *base = ws->epoch;
  ws->epoch += (uint32_t)count;
  return ALGAS_OK;
}

int make_plan(const algas_index* idx, const algas_params* p, int slots, Plan* out, bool persistent, bool allow_dsmem) {
  Plan pl;
  memset(&pl, 0, sizeof(pl));
  const int L = p->itopk, k = p->k, w = p->width;
  if (k < 1 || L < k || L > ALGAS_MAX_ITOPK)
    return set_error(ALGAS_EINVAL, "need 1 <= k (%d) <= itopk (%d) <= %d", k, L, ALGAS_MAX_ITOPK);
  if (w < 1 || w > ALGAS_MAX_WIDTH) return set_error(ALGAS_EINVAL, "width %d not in [1,%d]", w, ALGAS_MAX_WIDTH);
  if (p->visited_mode != ALGAS_VISITED_PRIVATE && p->visited_mode != ALGAS_VISITED_SHARED)
    return set_error(ALGAS_EINVAL, "bad visited_mode %d", p->visited_mode);
  int S = p->n_seeds > 0 ? p->n_seeds : 32;
  if (S > ALGAS_MAX_SEEDS) return set_error(ALGAS_EINVAL, "n_seeds %d > %d", S, ALGAS_MAX_SEEDS);
  int T = p->ctas_per_query;
  int nt = p->threads_per_cta;
  if (T == 0 || nt == 0) {
    algas_tuning tu;
    int rc = algas_tune(nullptr, slots, idx->dim, idx->degree, L, k, &tu);
    if (rc != ALGAS_OK) return rc;
    if (T == 0) T = tu.ctas_per_query;
    if (nt == 0) nt = tu.threads_per_cta;
  }
  if (T < 1 || T > ALGAS_MAX_CTAS) return set_error(ALGAS_EINVAL, "ctas_per_query %d not in [1,%d]", T, ALGAS_MAX_CTAS);
  if (nt != 32 && nt != 64 && nt != 128 && nt != 256 && nt != 512 && nt != 1024)
    return set_error(ALGAS_EINVAL, "threads_per_cta %d not in {32,64,128,256,512,1024}", nt);
  const int cc = chunk_config_for(idx->d4);
  if (cc < 0) return set_error(ALGAS_EINVAL, "dim %d unsupported", idx->dim);
  const int Rp = 1 << idx->rp_shift;
  const int dp4 = chunk_tl(cc) * chunk_cpl(cc);
  int ncap = 1;
  while (ncap < std::max(S, w * Rp)) ncap <<= 1;
  int optin = 0, dev = 0, smem_sm = 0, reserved = 0, nsm = 0;
  ALGAS_CUDA_TRY(cudaGetDevice(&dev));
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev));
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  // Shared-memory budget per CTA: M_avail = M_per_SM / N_block_per_SM
  // - M_reserved, with N_block_per_SM from P:L235 for a persistent grid of
  // slots x T CTAs, or a target occupancy of 8 CTAs/SM for a static batch.
  const int cs = persistent ? (p->cluster_size > 0 ? p->cluster_size : 1) : 1;
  if (cs != 1 && cs != 2 && cs != 4 && cs != 8) return set_error(ALGAS_EINVAL, "cluster_size %d not in {1,2,4,8}", cs);
  const int bps = persistent ? std::max(1, (int)(((int64_t)slots * T * cs + nsm - 1) / nsm)) : 8;
  const int64_t budget = std::min<int64_t>((int64_t)smem_sm / bps - reserved, (int64_t)optin - reserved);
  // vector-gather path: 0 = LDG.128 into registers (default),
  // 1 = cp.async (LDGSTS) staging, 2 = cp.async.bulk staging, 3 = team-local
  // cp.async staging (every row of a pass in flight, no data registers)
  // (ALGAS_GATHER_MODE)
  const char* gm_env = getenv("ALGAS_GATHER_MODE");
  const int gather_mode = gm_env ? atoi(gm_env) : 0;
  if (gather_mode < 0 || gather_mode > 4) return set_error(ALGAS_EINVAL, "ALGAS_GATHER_MODE must be 0..4");
#if !ALGAS_GATHER_EXPERIMENTS
  if (gather_mode != 0)
    return set_error(ALGAS_EINVAL, "ALGAS_GATHER_MODE %d needs a build with -DALGAS_GATHER_EXPERIMENTS=1", gather_mode);
#endif
  if (cs > 1 && gather_mode != 0) return set_error(ALGAS_EINVAL, "cluster_size > 1 needs the register gather path");
  const char* pf_env = getenv("ALGAS_PREFETCH");  // experiment switch
  const int prefetch = pf_env ? atoi(pf_env) : 8;
  // graph-row cache (prefetch bit 128; 64 rows of <= 64 ids, 32 of 128):
  // reserved first, if the visited hash can still have its minimum size next
  // to it.  Off by default: measured -4 % at the C2 point (the cp.async issue
  // in the distance step costs more than the L2 read it saves)
  int gcbits = (gather_mode == 0 && cs == 1 && (prefetch & 128)) ? (Rp <= 64 ? 6 : 5) : 0;
  int hb = p->hash_bits, sr = gather_mode == 0 ? -1 : p->stage_rows;
  {
    int hb_min = 6;
    while ((1LL << hb_min) < 2LL * (S + w * Rp)) ++hb_min;
    if (gcbits && smem_layout(dp4, L, ncap, hb > 0 ? hb : hb_min, sr < 0 ? 0 : sr, gc_bytes(gcbits, idx->rp_shift))
                          .total > budget)
      gcbits = 0;
  }
  const int gcb = gc_bytes(gcbits, idx->rp_shift);
  // SHARED visited bitmap in distributed shared memory (vis_claim): a
  // persistent grid of single-CTA searches whose T (a power of two <= 8) CTAs
  // of a slot form one thread-block cluster, each holding 1/T of the n-bit
  // bitmap, if that share fits next to a visited hash of >= 2^12 entries;
  // else the slot's bitmap in HBM.  ALGAS_VIS_DSMEM=0 turns it off (A/B).
  int vis_dsmem = 0, vis_words = 0, vis_tshift = 0;
  if (allow_dsmem && persistent && cs == 1 && gather_mode == 0 && p->visited_mode == ALGAS_VISITED_SHARED && T <= 8 &&
      (T & (T - 1)) == 0) {
    const char* ve = getenv("ALGAS_VIS_DSMEM");
    if (!ve || atoi(ve) != 0) {
      while ((1 << vis_tshift) < T) ++vis_tshift;
      const int64_t words = (idx->n + 31) / 32;
      const int64_t share = (((words + T - 1) / T) + 3) & ~int64_t(3);
      int hb_min = 12;
      while ((1LL << hb_min) < 2LL * (S + w * Rp)) ++hb_min;
      if (share * 4 <= (1 << 20) &&
          smem_layout(dp4, L, ncap, p->hash_bits > 0 ? p->hash_bits : hb_min, 0, gcb, (int)share * 4).total <= budget) {
        vis_dsmem = 1;
        vis_words = (int)share;
      }
    }
  }
  const int vsb = vis_dsmem ? vis_words * 4 : 0;
  int team_rows = 0;
  if (gather_mode == 4) {
    // hybrid: one register pass + team_rows staged rows per team in flight
    const int nteams = nt / chunk_tl(cc);
    team_rows = p->stage_rows > 0 ? p->stage_rows : 1;
    sr = (nteams * team_rows + 1) / 2;
  } else if (gather_mode == 3) {
    // rows in flight per team and pass: enough for a step's new rows
    // (<= w * Rp), as many as fit next to the smallest admissible hash;
    // p->stage_rows > 0 forces it (sweeps)
    const int nteams = nt / chunk_tl(cc);
    int hb_min = 6;
    while ((1LL << hb_min) < 2LL * (S + w * Rp)) ++hb_min;
    const int need = (std::min(w * Rp, ncap) + nteams - 1) / nteams;
    team_rows = p->stage_rows > 0 ? p->stage_rows : std::max(1, std::min(need, 8));
    while (team_rows > 1 &&
           smem_layout(dp4, L, ncap, hb > 0 ? hb : hb_min, (nteams * team_rows + 1) / 2, gcb).total > budget)
      --team_rows;
    sr = (nteams * team_rows + 1) / 2;  // smem_layout reserves 2 x sr staging rows
  }
  choose_smem(dp4, L, ncap, S, w, Rp, budget - gcb - vsb, &hb, &sr);
  if (hb < 6 || hb > 16) return set_error(ALGAS_EINVAL, "hash_bits %d not in [6,16]", hb);
  if ((1 << hb) < 2 * (S + w * Rp))
    return set_error(ALGAS_EINVAL, "visited hash 2^%d too small for seeds + one step (%d)", hb, S + w * Rp);
  SmemLayout lay = smem_layout(dp4, L, ncap, hb, sr, gcb, vsb);
  if (lay.total + reserved > optin)
    return set_error(ALGAS_EINVAL, "search needs %d B shared memory per CTA, device allows %d", lay.total, optin);

  pl.nt = nt;
  pl.ccfg = cc;
  pl.T = T;
  pl.k = k;
  pl.smem = lay.total;
  pl.visited_mode = p->visited_mode;
  pl.metric = idx->metric == ALGAS_COSINE ? ALGAS_IP : idx->metric;  // COSINE = IP on unit rows (R29)
  pl.cluster = cs;
  // a persistent grid of more searches than SMs runs two 256/512-thread CTAs
  // per SM (the build with half the registers per thread)
  pl.occ = (persistent && cs == 1 && (nt == 256 || nt == 512) && (int64_t)slots * T > nsm) ? 2 : 1;
  SearchCfg& c = pl.cfg;
  c.data = reinterpret_cast<const float4*>(idx->d_data);
  c.graph = idx->d_graph;
  c.n = (uint64_t)idx->n;
  c.d4 = idx->d4;
  c.dp4 = dp4;
  c.R = idx->degree;
  c.rp_shift = idx->rp_shift;
  c.L = L;
  c.w = w;
  c.off = p->offset_beam < 0 ? std::max(1, L / 4) : std::min(p->offset_beam, L);
  c.S = S;
  c.max_iter = p->max_iter > 0 ? p->max_iter : 4 * L + 256;
  c.hash_bits = hb;
  c.gtab_bits = std::min(20, std::max(16, hb + 2));
  c.ncap = ncap;
  c.stage_rows = sr;
  c.team_rows = team_rows;
  c.gather_mode = gather_mode;
  c.prefetch = prefetch;
  c.gc_bits = gcbits;
  c.seed = p->seed;
  c.cosine = idx->metric == ALGAS_COSINE ? 1 : 0;
  c.shared = p->visited_mode == ALGAS_VISITED_SHARED ? 1 : 0;
  c.vis_dsmem = vis_dsmem;
  c.vis_tshift = vis_tshift;
  c.vis_words = vis_words;
  if (c.shared && cs > 1) return set_error(ALGAS_EINVAL, "SHARED visited mode needs cluster_size 1");
  int nb = 0;
  int rc = max_blocks_per_sm(pl, persistent, &nb);
  if (rc != ALGAS_OK) return rc;
  if (nb < 1) return set_error(ALGAS_EINVAL, "search kernel does not fit on an SM (smem %d)", pl.smem);
  pl.blocks_per_sm = nb;
  if (vis_dsmem && T > 1) {
    // the slots' clusters of T CTAs must all be co-resident; if
    // they are not, plan again with the HBM bitmap
    int ncl = 0;
    rc = max_active_clusters(pl, &ncl);
    if (rc != ALGAS_OK || ncl < slots) {
      (void)cudaGetLastError();
      return make_plan(idx, p, slots, out, persistent, false);
    }
  }
  *out = pl;
  return ALGAS_OK;
}

// CTAs per thread-block cluster of a persistent launch: a cluster-split
// search (cluster_size), or the T CTAs of a slot sharing a DSMEM bitmap
int launch_cluster_size(const Plan& pl) { return pl.cluster > 1 ? pl.cluster : (pl.cfg.vis_dsmem ? pl.T : 1); }

static int num_sms() {
  int dev = 0, n = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n;
}

// Every slot's searches must be co-resident for the persistent kernel to
// make progress (Eq. P:L231 with the measured occupancy).
int check_coresident(const Plan& pl, int slots) {
  if (launch_cluster_size(pl) <= 1) {
    if ((int64_t)slots * pl.T > (int64_t)pl.blocks_per_sm * num_sms())
      return set_error(ALGAS_EINVAL, "%d slots x %d CTAs exceed co-resident capacity %d x %d SMs (P:L231)", slots,
                       pl.T, pl.blocks_per_sm, num_sms());
    return ALGAS_OK;
  }
  int nc = 0;
  int rc = max_active_clusters(pl, &nc);
  if (rc) return rc;
  const int64_t need = pl.cluster > 1 ? (int64_t)slots * pl.T : (int64_t)slots;
  if (need > nc)
    return set_error(ALGAS_EINVAL, "%d slots x %d searches exceed the %d co-resident %d-CTA clusters (P:L231)", slots,
                     pl.T, nc, launch_cluster_size(pl));
  return ALGAS_OK;
}

// RAII device buffer on a stream
struct DevBuf {
  void* p = nullptr;
  cudaStream_t st = nullptr;
  ~DevBuf() {
    if (p) cudaFreeAsync(p, st);
  }
  int alloc(size_t bytes, cudaStream_t s) {
    st = s;
    ALGAS_CUDA_TRY(cudaMallocAsync(&p, std::max<size_t>(bytes, 16), s));
    return ALGAS_OK;
  }
};

// Host merge of nq x T x k per-CTA lists into the caller's outputs.
// run f(lo, hi) over [0, n) on up to 16 host threads (serial for small n)
template <typename F>
static void parallel_for(int64_t n, int64_t grain, F f) {
  const int hw = (int)std::max(1u, std::thread::hardware_concurrency());
  const int nt = (int)std::min<int64_t>(std::min(16, hw), (n + grain - 1) / grain);
  if (nt <= 1) {
    f((int64_t)0, n);
    return;
  }
  std::vector<std::thread> th;
  const int64_t chunk = (n + nt - 1) / nt;
  for (int t = 0; t < nt; ++t) {
    const int64_t lo = t * chunk, hi = std::min(n, lo + chunk);
    if (lo < hi) th.emplace_back([=] { f(lo, hi); });
  }
  for (auto& x : th) x.join();
}

// Host TopK merge of nq x T x kin per-CTA lists into the caller's
// outputs, plus per-query counters; parallel over queries.
static int finish_outputs(const ResultEntry* res, const CtaStats* cst, int64_t nq, int T, int kin, int k,
                          uint32_t* out_ids, float* out_dists, uint32_t* out_cta_ids, float* out_cta_dists,
                          algas_query_stats* out_stats, bool* overflow) {
  const bool dev_ids = is_device_ptr(out_ids), dev_d = is_device_ptr(out_dists);
  std::vector<uint32_t> hid;
  std::vector<float> hd;
  uint32_t* ids = out_ids;
  float* ds = out_dists;
  if (dev_ids) { hid.resize((size_t)nq * k); ids = hid.data(); }
  if (dev_d) { hd.resize((size_t)nq * k); ds = hd.data(); }
  std::atomic<bool> ovf{false};
  parallel_for(nq, 1024, [&](int64_t lo, int64_t hi) {
    bool o = false;
    for (int64_t q = lo; q < hi; ++q) {
      const ResultEntry* r = res + (size_t)q * T * kin;
      if (T == 1) {
        for (int i = 0; i < k; ++i) { ids[q * k + i] = r[i].id; ds[q * k + i] = r[i].dist; }
      } else {
        merge_cta_lists(r, T, kin, k, ids + q * k, ds + q * k);
      }
      algas_query_stats qs;
      aggregate_cta_stats(cst + q * T, T, &qs);
      if (qs.overflows) o = true;
      if (out_stats) out_stats[q] = qs;
    }
    if (o) ovf = true;
  });
  if (dev_ids) ALGAS_CUDA_TRY(cudaMemcpy(out_ids, hid.data(), hid.size() * 4, cudaMemcpyHostToDevice));
  if (dev_d) ALGAS_CUDA_TRY(cudaMemcpy(out_dists, hd.data(), hd.size() * 4, cudaMemcpyHostToDevice));
  if (out_cta_ids || out_cta_dists) {
    const size_t m = (size_t)nq * T * kin;
    std::vector<uint32_t> ci(m);
    std::vector<float> cd(m);
    for (size_t i = 0; i < m; ++i) { ci[i] = res[i].id; cd[i] = res[i].dist; }
    if (out_cta_ids) ALGAS_CUDA_TRY(cudaMemcpy(out_cta_ids, ci.data(), m * 4, cudaMemcpyDefault));
    if (out_cta_dists) ALGAS_CUDA_TRY(cudaMemcpy(out_cta_dists, cd.data(), m * 4, cudaMemcpyDefault));
  }
  *overflow = ovf.load();
  return ALGAS_OK;
}

// pinned host staging for per-CTA results / counters (workspace-cached)
static int ensure_pinned(Workspace* ws, size_t res_bytes, size_t st_bytes) {
  if (ws->h_res_bytes < res_bytes) {
    if (ws->h_res) cudaFreeHost(ws->h_res);
    ws->h_res = nullptr;
    ws->h_res_bytes = 0;
    ALGAS_CUDA_TRY(cudaMallocHost(&ws->h_res, res_bytes));
    ws->h_res_bytes = res_bytes;
  }
  if (ws->h_st_bytes < st_bytes) {
    if (ws->h_st) cudaFreeHost(ws->h_st);
    ws->h_st = nullptr;
    ws->h_st_bytes = 0;
    ALGAS_CUDA_TRY(cudaMallocHost(&ws->h_st, st_bytes));
    ws->h_st_bytes = st_bytes;
  }
  return ALGAS_OK;
}

// queries -> device (copy if host); returns pointer usable by kernels
static int stage_queries(const algas_index* idx, const float* q, int64_t nq, DevBuf& buf, cudaStream_t st,
                         const float4** out) {
  if (is_device_ptr(q)) {
    if (((uintptr_t)q & 15u) != 0) return set_error(ALGAS_EINVAL, "device queries must be 16-B aligned");
    *out = reinterpret_cast<const float4*>(q);
    return ALGAS_OK;
  }
  size_t bytes = (size_t)nq * idx->dim * 4;
  int rc = buf.alloc(bytes, st);
  if (rc) return rc;
  ALGAS_CUDA_TRY(cudaMemcpyAsync(buf.p, q, bytes, cudaMemcpyHostToDevice, st));
  *out = reinterpret_cast<const float4*>(buf.p);
  return ALGAS_OK;
}

struct EventTimer {
  cudaStream_t st;
  cudaEvent_t a = nullptr, b = nullptr;
  explicit EventTimer(cudaStream_t s) : st(s) {}
  ~EventTimer() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
  }
  int start() {
    ALGAS_CUDA_TRY(cudaEventCreate(&a));
    ALGAS_CUDA_TRY(cudaEventCreate(&b));
    ALGAS_CUDA_TRY(cudaEventRecord(a, st));
    return ALGAS_OK;
  }
  int stop() {
    ALGAS_CUDA_TRY(cudaEventRecord(b, st));
    return ALGAS_OK;
  }
  float ms() {
    float m = 0.f;
    if (cudaEventElapsedTime(&m, a, b) != cudaSuccess) (void)cudaGetLastError();
    return m;
  }
};

static void fill_info(algas_run_info* info, const Plan& pl, int grid, float ms) {
  memset(info, 0, sizeof(*info));
  info->kernel_ms = ms;
  info->grid = grid;
  info->threads_per_cta = pl.nt;
  info->ctas_per_query = pl.T;
  info->smem_per_cta = pl.smem;
  info->blocks_per_sm = pl.blocks_per_sm;
  info->hash_bits = pl.cfg.hash_bits;
}

}  // namespace algas

using namespace algas;

extern "C" {

void algas_params_default(algas_params* p) {
  memset(p, 0, sizeof(*p));
  p->k = 10;
  p->itopk = 64;
  p->width = 1;
  p->offset_beam = -1;
  p->ctas_per_query = 1;
  p->threads_per_cta = 0;
  p->n_seeds = 32;
  p->max_iter = 0;
  p->visited_mode = ALGAS_VISITED_PRIVATE;
  p->slots = 32;
  p->hash_bits = 0;
  p->seed = 0;
}

const char* algas_last_error(void) { return g_err.c_str(); }
// COSINE index (R29): one warp per row, v <- v / |v| (fp32; a zero row stays 0)
__global__ void normalize_rows_kernel(float4* x, int64_t n, int d4) {
  const int64_t row = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (row >= n) return;
  float4* r = x + row * d4;
  float ss = 0.f;
  for (int i = lane; i < d4; i += 32) {
    const float4 v = r[i];
    ss = fmaf(v.x, v.x, fmaf(v.y, v.y, fmaf(v.z, v.z, fmaf(v.w, v.w, ss))));
  }
  for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
  if (ss <= 0.f) return;
  const float inv = 1.0f / sqrtf(ss);
  for (int i = lane; i < d4; i += 32) {
    float4 v = r[i];
    v.x *= inv; v.y *= inv; v.z *= inv; v.w *= inv;
    r[i] = v;
  }
}

const char* algas_version(void) { return "algas-b200 0.1 (sm_100a)"; }

algas_index* algas_index_create(const float* data, int64_t n, int32_t dim, int32_t metric, const uint32_t* graph,
                                int32_t degree) {
  if (!data || n < 1 || n >= (1LL << 31) || dim < 4 || dim % 4 != 0 || dim > ALGAS_MAX_DIM || degree < 1 ||
      degree > ALGAS_MAX_DEGREE || (metric != ALGAS_L2 && metric != ALGAS_IP && metric != ALGAS_COSINE)) {
    set_error(ALGAS_EINVAL, "algas_index_create: bad arguments (n=%lld dim=%d degree=%d metric=%d)", (long long)n,
              dim, degree, metric);
    return nullptr;
  }
  algas_index* idx = new algas_index();
  idx->n = n;
  idx->dim = dim;
  idx->d4 = dim / 4;
  idx->metric = metric;
  idx->degree = degree;
  idx->rp_shift = 2;  // graph rows padded to a power-of-two stride (>= 4 ids)
  while ((1 << idx->rp_shift) < degree) ++idx->rp_shift;
  idx->ws = new Workspace();
  cudaGetDevice(&idx->device);
  const size_t dbytes = (size_t)n * dim * 4, gpitch = (size_t)4 << idx->rp_shift;
  auto fail = [&](const char* what, cudaError_t e) -> algas_index* {
    set_error(e == cudaErrorMemoryAllocation ? ALGAS_ENOMEM : ALGAS_ECUDA, "algas_index_create: %s: %s", what,
              cudaGetErrorString(e));
    algas_index_destroy(idx);
    return nullptr;
  };
  cudaError_t e;
  if ((e = cudaMalloc(&idx->d_data, dbytes)) != cudaSuccess) return fail("cudaMalloc data", e);
  if ((e = cudaMemcpy(idx->d_data, data, dbytes, cudaMemcpyDefault)) != cudaSuccess) return fail("copy data", e);
  if (metric == ALGAS_COSINE) {
    // unit rows in HBM: the search (and the graph build) run as IP on them (R29)
    const int64_t warps_per_block = 8;
    normalize_rows_kernel<<<(unsigned)((n + warps_per_block - 1) / warps_per_block), 32 * warps_per_block>>>(
        reinterpret_cast<float4*>(idx->d_data), n, dim / 4);
    if ((e = cudaGetLastError()) != cudaSuccess || (e = cudaDeviceSynchronize()) != cudaSuccess)
      return fail("normalize rows", e);
  }
  if ((e = cudaMalloc(&idx->d_graph, (size_t)n * gpitch)) != cudaSuccess) return fail("cudaMalloc graph", e);
  if ((e = cudaMemset(idx->d_graph, 0xFF, (size_t)n * gpitch)) != cudaSuccess) return fail("memset graph", e);
  std::vector<uint32_t> built;
  const uint32_t* g = graph;
  if (!g) {
    built.resize((size_t)n * degree);
    int rc = algas_build_graph(idx->d_data, n, dim, metric == ALGAS_COSINE ? ALGAS_IP : metric, std::min<int64_t>(2 * degree, std::max<int64_t>(1, n - 1)),
                               degree, 1, built.data());
    if (rc != ALGAS_OK) {
      algas_index_destroy(idx);
      return nullptr;
    }
    g = built.data();
  }
  if ((e = cudaMemcpy2D(idx->d_graph, gpitch, g, (size_t)degree * 4, (size_t)degree * 4, (size_t)n,
                        cudaMemcpyDefault)) != cudaSuccess)
    return fail("copy graph", e);
  return idx;
}

int algas_index_destroy(algas_index* idx) {
  if (!idx) return ALGAS_OK;
  if (idx->d_data) cudaFree(idx->d_data);
  if (idx->d_graph) cudaFree(idx->d_graph);
  if (idx->ws) {
    if (idx->ws->gtab) cudaFree(idx->ws->gtab);
    if (idx->ws->counters) cudaFree(idx->ws->counters);
    if (idx->ws->h_res) cudaFreeHost(idx->ws->h_res);
    if (idx->ws->h_st) cudaFreeHost(idx->ws->h_st);
    if (idx->ws->m_buf) cudaFreeHost(idx->ws->m_buf);
    for (void* p : idx->ws->d_scratch)
      if (p) cudaFree(p);
    delete idx->ws;
  }
  delete idx;
  return ALGAS_OK;
}

int algas_index_info(const algas_index* idx, int64_t* n, int32_t* dim, int32_t* metric, int32_t* degree,
                     int32_t* graph_stride, const float** dev_data, const uint32_t** dev_graph) {
  if (!idx) return set_error(ALGAS_EINVAL, "null index");
  if (n) *n = idx->n;
  if (dim) *dim = idx->dim;
  if (metric) *metric = idx->metric;
  if (degree) *degree = idx->degree;
  if (graph_stride) *graph_stride = 1 << idx->rp_shift;
  if (dev_data) *dev_data = idx->d_data;
  if (dev_graph) *dev_graph = idx->d_graph;
  return ALGAS_OK;
}

int algas_search(const algas_index* idx, const float* queries, int64_t nq, int32_t k, int32_t itopk, int32_t width,
                 uint32_t* out_ids, float* out_dists) {
  algas_params p;
  algas_params_default(&p);
  p.k = k;
  p.itopk = itopk;
  p.width = width;
  return algas_search_ex(idx, queries, nq, &p, 0, out_ids, out_dists, nullptr, nullptr, nullptr, nullptr, nullptr);
}

int algas_search_ex(const algas_index* cidx, const float* queries, int64_t nq, const algas_params* params,
                    uint64_t tag0, uint32_t* out_ids, float* out_dists, uint32_t* out_cta_ids, float* out_cta_dists,
                    algas_query_stats* out_stats, void* stream, algas_run_info* info) {
  algas_index* idx = const_cast<algas_index*>(cidx);
  if (!idx || !params || !queries || !out_ids || !out_dists || nq < 0)
    return set_error(ALGAS_EINVAL, "algas_search_ex: null argument");
  if (nq == 0) return ALGAS_OK;
  if (params->visited_mode != ALGAS_VISITED_PRIVATE)
    return set_error(ALGAS_EINVAL, "algas_search_ex: SHARED visited mode is served by the persistent paths only");
  Plan pl;
  int rc = make_plan(idx, params, 1, &pl, false);
  if (rc) return rc;
  if (nq * pl.T >= (1LL << 31)) return set_error(ALGAS_EINVAL, "nq * T too large");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int64_t items = nq * pl.T;
  const int grid = (int)std::min<int64_t>(items, (int64_t)pl.blocks_per_sm * num_sms());

  std::lock_guard<std::mutex> lk(idx->ws->mu);
  if ((rc = ensure_gtab(idx, (size_t)grid << pl.cfg.gtab_bits))) return rc;
  if (!idx->ws->counters) ALGAS_CUDA_TRY(cudaMalloc(&idx->ws->counters, 4096));
  uint32_t epoch_base = 1;
  if ((rc = take_epochs(idx, (uint64_t)items + 1, &epoch_base, st))) return rc;

  DevBuf qb, rb, sb;
  const float4* dq = nullptr;
  if ((rc = stage_queries(idx, queries, nq, qb, st, &dq))) return rc;
  if ((rc = rb.alloc((size_t)items * pl.k * sizeof(ResultEntry), st))) return rc;
  if ((rc = sb.alloc((size_t)items * sizeof(CtaStats), st))) return rc;
  ALGAS_CUDA_TRY(cudaMemsetAsync(sb.p, 0, (size_t)items * sizeof(CtaStats), st));
  BatchLaunch bl;
  bl.queries = dq;
  bl.nq = nq;
  bl.tag0 = tag0;
  bl.res = (ResultEntry*)rb.p;
  bl.stats = (CtaStats*)sb.p;
  bl.gtab = idx->ws->gtab;
  bl.epoch_base = epoch_base;
  bl.work_counter = idx->ws->counters;
  bl.grid = grid;
  EventTimer tm(st);
  if ((rc = tm.start())) return rc;
  if ((rc = launch_batch(pl, bl, st))) return rc;
  if ((rc = tm.stop())) return rc;
  const size_t res_bytes = (size_t)items * pl.k * sizeof(ResultEntry), st_bytes = (size_t)items * sizeof(CtaStats);
  if ((rc = ensure_pinned(idx->ws, res_bytes, st_bytes))) return rc;
  ResultEntry* res = (ResultEntry*)idx->ws->h_res;
  CtaStats* cst = (CtaStats*)idx->ws->h_st;
  ALGAS_CUDA_TRY(cudaMemcpyAsync(res, rb.p, res_bytes, cudaMemcpyDeviceToHost, st));
  ALGAS_CUDA_TRY(cudaMemcpyAsync(cst, sb.p, st_bytes, cudaMemcpyDeviceToHost, st));
  ALGAS_CUDA_TRY(cudaStreamSynchronize(st));
  ALGAS_CUDA_TRY(cudaGetLastError());
  if (info) fill_info(info, pl, grid, tm.ms());
  bool ovf = false;
  if ((rc = finish_outputs(res, cst, nq, pl.T, pl.k, pl.k, out_ids, out_dists, out_cta_ids, out_cta_dists, out_stats,
                           &ovf)))
    return rc;
  return ovf ? set_error(ALGAS_EOVERFLOW, "a visited table overflowed") : ALGAS_OK;
}

int algas_search_dynamic(const algas_index* cidx, const float* queries_dev, int64_t nq, const algas_params* params,
                         uint64_t tag0, uint32_t* out_ids, float* out_dists, algas_query_stats* out_stats,
                         void* stream, algas_run_info* info) {
  const auto t_entry = std::chrono::steady_clock::now();
  static const bool trace = getenv("ALGAS_TRACE") != nullptr;
  auto mark = [&](const char* what) {
    if (trace)
      fprintf(stderr, "[algas] %-10s %8.3f ms\n", what,
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t_entry).count());
  };
  algas_index* idx = const_cast<algas_index*>(cidx);
  if (!idx || !params || !queries_dev || !out_ids || !out_dists || nq < 0)
    return set_error(ALGAS_EINVAL, "algas_search_dynamic: null argument");
  if (!is_device_ptr(queries_dev)) return set_error(ALGAS_EINVAL, "algas_search_dynamic: queries must be device memory");
  if (nq == 0) return ALGAS_OK;
  if (nq >= (1LL << 31)) return set_error(ALGAS_EINVAL, "nq too large");
  const int slots = params->slots > 0 ? params->slots : 32;
  Plan pl;
  int rc = make_plan(idx, params, slots, &pl, true);
  if (rc) return rc;
  if ((rc = check_coresident(pl, slots))) return rc;
  mark("plan");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int ctas = slots * pl.T * pl.cluster;
  const int64_t items = nq * pl.T;

  std::lock_guard<std::mutex> lk(idx->ws->mu);
  if ((rc = ensure_gtab(idx, (size_t)ctas << pl.cfg.gtab_bits))) return rc;
  // epoch-tagged spill tables: every query of this call gets an epoch above
  // all earlier ones (base + queries served by its CTA), so nothing is cleared
  uint32_t ebase = 1;
  if ((rc = take_epochs(idx, (uint64_t)nq + 1, &ebase, st))) return rc;

  Workspace* ws = idx->ws;
  void* rbp = nullptr;
  void* sbp = nullptr;
  void* ctlp = nullptr;
  if ((rc = ensure_scratch(ws, 0, (size_t)items * pl.k * sizeof(ResultEntry), &rbp))) return rc;
  if ((rc = ensure_scratch(ws, 1, (size_t)items * sizeof(CtaStats), &sbp))) return rc;
  // control block: queue head | mbox[slots] | dparams[slots] | dtag[slots] | slot_fin[slots] | qbuf unused
  const size_t ctl_bytes = control_bytes(slots);
  if ((rc = ensure_scratch(ws, 2, ctl_bytes, &ctlp))) return rc;
  ALGAS_CUDA_TRY(cudaMemsetAsync(ctlp, 0, ctl_bytes, st));
  uint8_t* cb = (uint8_t*)ctlp;
  PersistArgs pa;
  memset(&pa, 0, sizeof(pa));
  pa.mode = 1;
  pa.slots = slots;
  pa.T = pl.T;
  pa.kmax = pl.k;
  pa.queries = reinterpret_cast<const float4*>(queries_dev);
  pa.nq = nq;
  pa.tag0 = tag0;
  carve_control(cb, slots, &pa);
  pa.dq_res = (ResultEntry*)rbp;
  pa.dq_stats = (CtaStats*)sbp;
  pa.gtab = ws->gtab;
  pa.epoch_base = ebase;
  // SHARED visited bitmaps: two per slot (zeroed here; each query's CTAs clear the other one)
  if (pl.cfg.shared && !pl.cfg.vis_dsmem && (pa.vbm_words = shared_bitmap_words(idx->n)) > 0) {
    void* vbp = nullptr;
    if ((rc = ensure_scratch(ws, 3, (size_t)slots * 2 * pa.vbm_words * 4, &vbp))) return rc;
    ALGAS_CUDA_TRY(cudaMemsetAsync(vbp, 0, (size_t)slots * 2 * pa.vbm_words * 4, st));
    pa.vbm = (uint32_t*)vbp;
  }
  mark("alloc");
  const size_t res_bytes = (size_t)items * pl.k * sizeof(ResultEntry), st_bytes = (size_t)items * sizeof(CtaStats);
  // Streaming merge (GPU-CPU cooperation): with host outputs the
  // CTAs write their lists and counters straight into host-mapped memory and
  // raise a per-(query, CTA) Finish word; this thread merges each query the
  // moment its T lists are in, while the kernel keeps running -- the host
  // merge overlaps the search instead of following it.
  const bool stream_merge = !is_device_ptr(out_ids) && !is_device_ptr(out_dists) && getenv("ALGAS_NO_STREAM_MERGE") == nullptr;
  ResultEntry* mres = nullptr;
  CtaStats* mst = nullptr;
  uint32_t* mdone = nullptr;
  if (stream_merge) {
    const size_t done_bytes = (size_t)items * 4;
    const size_t need = res_bytes + st_bytes + done_bytes + 256;
    if (ws->m_bytes < need) {
      if (ws->m_buf) cudaFreeHost(ws->m_buf);
      ws->m_buf = nullptr;
      ws->m_bytes = 0;
      ALGAS_CUDA_TRY(cudaHostAlloc(&ws->m_buf, need, cudaHostAllocMapped | cudaHostAllocPortable));
      memset(ws->m_buf, 0, need);
      ws->m_bytes = need;
    }
    uint8_t* hb = (uint8_t*)ws->m_buf;
    uint8_t* db = nullptr;
    ALGAS_CUDA_TRY(cudaHostGetDevicePointer((void**)&db, ws->m_buf, 0));
    const size_t o_st = (res_bytes + 127) & ~(size_t)127, o_done = (o_st + st_bytes + 127) & ~(size_t)127;
    mres = (ResultEntry*)hb;
    mst = (CtaStats*)(hb + o_st);
    mdone = (uint32_t*)(hb + o_done);
    pa.dq_res = (ResultEntry*)db;
    pa.dq_stats = (CtaStats*)(db + o_st);
    pa.dq_done = (uint32_t*)(db + o_done);
    pa.call_id = ++ws->call_id;
    if (pa.call_id == 0) pa.call_id = ++ws->call_id;  // 0 = never written
    // the Finish words of THIS call's layout: the region may hold an earlier
    // call's results or counters (other T / nq => other offsets), whose
    // values could equal call_id -- clear it before the launch
    memset(mdone, 0, (size_t)items * 4);
  }
  EventTimer tm(st);
  if ((rc = tm.start())) return rc;
  if ((rc = launch_persistent(pl, pa, st))) return rc;
  if ((rc = tm.stop())) return rc;
  mark("launch");
  if (stream_merge) {
    const auto t_merge = std::chrono::steady_clock::now();
    bool ovf = false;
    const uint32_t cid = pa.call_id;
    const int T = pl.T, k = pl.k;
    int spins = 0;
    for (int64_t q = 0; q < nq; ++q) {
      for (int c = 0; c < T; ++c) {
        while (__atomic_load_n(mdone + q * T + c, __ATOMIC_ACQUIRE) != cid) {
          if (++spins >= 4096) {  // a failed kernel is reported, not waited on
            spins = 0;
            const cudaError_t e = cudaStreamQuery(st);
            if (e != cudaSuccess && e != cudaErrorNotReady)
              return set_error(ALGAS_ECUDA, "search kernel failed: %s", cudaGetErrorString(e));
            if (e == cudaSuccess && __atomic_load_n(mdone + q * T + c, __ATOMIC_ACQUIRE) != cid)
              return set_error(ALGAS_ECUDA, "search kernel finished without publishing query %lld", (long long)q);
          }
        }
      }
      const ResultEntry* r = mres + (size_t)q * T * k;
      if (T == 1) {
        for (int i = 0; i < k; ++i) { out_ids[q * k + i] = r[i].id; out_dists[q * k + i] = r[i].dist; }
      } else {
        merge_cta_lists(r, T, k, k, out_ids + q * k, out_dists + q * k);
      }
      algas_query_stats qs;
      aggregate_cta_stats(mst + q * T, T, &qs);
      if (qs.overflows) ovf = true;
      if (out_stats) out_stats[q] = qs;
    }
    ALGAS_CUDA_TRY(cudaStreamSynchronize(st));
    ALGAS_CUDA_TRY(cudaGetLastError());
    mark("merge");
    if (info) {
      fill_info(info, pl, ctas, tm.ms());
      const auto t_end = std::chrono::steady_clock::now();
      info->merge_ms = std::chrono::duration<float, std::milli>(t_end - t_merge).count();
      info->call_ms = std::chrono::duration<float, std::milli>(t_end - t_entry).count();
    }
    return ovf ? set_error(ALGAS_EOVERFLOW, "a visited table overflowed") : ALGAS_OK;
  }
  if ((rc = ensure_pinned(idx->ws, res_bytes, st_bytes))) return rc;
  ResultEntry* res = (ResultEntry*)idx->ws->h_res;
  CtaStats* cst = (CtaStats*)idx->ws->h_st;
  ALGAS_CUDA_TRY(cudaMemcpyAsync(res, rbp, res_bytes, cudaMemcpyDeviceToHost, st));
  ALGAS_CUDA_TRY(cudaMemcpyAsync(cst, sbp, st_bytes, cudaMemcpyDeviceToHost, st));
  ALGAS_CUDA_TRY(cudaStreamSynchronize(st));
  ALGAS_CUDA_TRY(cudaGetLastError());
  mark("sync");
  if (info) fill_info(info, pl, ctas, tm.ms());
  bool ovf = false;
  const auto t_merge = std::chrono::steady_clock::now();
  if ((rc = finish_outputs(res, cst, nq, pl.T, pl.k, pl.k, out_ids, out_dists, nullptr, nullptr, out_stats, &ovf)))
    return rc;
  mark("merge");
  if (info) {
    const auto t_end = std::chrono::steady_clock::now();
    info->merge_ms = std::chrono::duration<float, std::milli>(t_end - t_merge).count();
    info->call_ms = std::chrono::duration<float, std::milli>(t_end - t_entry).count();
  }
  return ovf ? set_error(ALGAS_EOVERFLOW, "a visited table overflowed") : ALGAS_OK;
}

}  // extern "C"
