// knn.cu -- graph construction (supporting code, not the search hot path).
//
//  algas_knn   : exact k-NN by brute force.  Distances are computed
//                in the DIRECT form sum_j (q_j - x_j)^2 / -sum_j q_j x_j in
//                fp32 (no |q|^2+|x|^2-2q.x cancellation, so the result is
//                exact up to fp32 summation order and bit-exact on the
//                integer lattice), tile by tile into an HBM distance block,
//                then a warp-per-row running top-k selection keyed by
//                (dist, id) (R4).
//  algas_prune : CAGRA-style optimisation of the kNN graph, reading R24
//                (rank-based detour count, keep `degree`, reverse edges,
//                merge).  The graph type is named at P:L293; the algorithm
//                is CAGRA's (ref [25]) and not printed in the paper.
#include <cub/cub.cuh>
#include <cublas_v2.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <thread>
#include <cstring>
#include <vector>

#include "internal.h"

namespace algas {

// ------------------------------------------------------------------ distance tiles
constexpr int TQ = 128, TX = 128, TK = 16;

template <int METRIC>
__global__ void __launch_bounds__(256) dist_tile_kernel(const float* __restrict__ Q, int64_t qn,
                                                        const float* __restrict__ X, int64_t xn, int d,
                                                        float* __restrict__ D, int64_t ldD) {
  __shared__ float Qs[TK][TQ + 4];
  __shared__ float Xs[TK][TX + 4];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int64_t q0 = (int64_t)blockIdx.y * TQ, x0 = (int64_t)blockIdx.x * TX;
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  for (int k0 = 0; k0 < d; k0 += TK) {
    // 128 rows x 16 dims = 512 float4 per operand; 256 threads x 2
    for (int t = threadIdx.x; t < TQ * TK / 4; t += 256) {
      const int r = t >> 2, c4 = (t & 3) * 4;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (q0 + r < qn && k0 + c4 < d) v = *reinterpret_cast<const float4*>(Q + (q0 + r) * d + k0 + c4);
      Qs[c4 + 0][r] = v.x; Qs[c4 + 1][r] = v.y; Qs[c4 + 2][r] = v.z; Qs[c4 + 3][r] = v.w;
      float4 u = make_float4(0.f, 0.f, 0.f, 0.f);
      if (x0 + r < xn && k0 + c4 < d) u = *reinterpret_cast<const float4*>(X + (x0 + r) * d + k0 + c4);
      Xs[c4 + 0][r] = u.x; Xs[c4 + 1][r] = u.y; Xs[c4 + 2][r] = u.z; Xs[c4 + 3][r] = u.w;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < TK; ++kk) {
      float a[8], b[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) a[i] = Qs[kk][ty * 8 + i];
#pragma unroll
      for (int j = 0; j < 8; ++j) b[j] = Xs[kk][tx * 8 + j];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          if (METRIC == kL2) {
            float t = a[i] - b[j];
            acc[i][j] = fmaf(t, t, acc[i][j]);
          } else {
            acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
          }
        }
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int64_t r = q0 + ty * 8 + i;
    if (r >= qn) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int64_t c = x0 + tx * 8 + j;
      if (c < xn) D[r * ldD + c] = (METRIC == kL2) ? acc[i][j] : -acc[i][j];
    }
  }
}

// ------------------------------------------------------------------ running top-k selection
constexpr int SEL_WARPS = 4;
constexpr int SEL_BUF = 64;

// one warp per query row; the row's sorted top-k keys live in HBM between
// chunks and in shared memory (double buffered) while a chunk is scanned.
// MODE 0: D holds distances.  MODE 1/2: D holds dot products q.x from the
// tensor-core screen; the key distance is |q|^2 + |x|^2 - 2 q.x (L2, MODE 1)
// or -q.x (IP, MODE 2).
template <int MODE>
__global__ void __launch_bounds__(SEL_WARPS * 32) select_kernel(const float* __restrict__ D, int64_t ldD, int rows,
                                                                int64_t cols, int64_t col0, int64_t row0,
                                                                int64_t self_base, int k,
                                                                unsigned long long* __restrict__ state,
                                                                const float* __restrict__ qnorm,
                                                                const float* __restrict__ xnorm,
                                                                const int64_t* __restrict__ self_ids) {
  extern __shared__ __align__(16) uint8_t sm[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row = blockIdx.x * SEL_WARPS + warp;
  unsigned long long* la = reinterpret_cast<unsigned long long*>(sm) + (size_t)warp * (2 * k + SEL_BUF);
  unsigned long long* lb = la + k;
  unsigned long long* buf = lb + k;
  if (row >= rows) return;
  unsigned long long* st = state + (size_t)row * k;
  for (int i = lane; i < k; i += 32) la[i] = st[i];
  __syncwarp();
  unsigned long long* cur = la;
  unsigned long long* oth = lb;
  int nb = 0;
  const int64_t self = self_ids ? self_ids[row0 + row] : (self_base >= 0 ? self_base + row0 + row : -1);
  const float* dr = D + (size_t)row * ldD;
  const float qn = MODE == 1 ? qnorm[row0 + row] : 0.f;
  auto flush = [&]() {
    // sort buf[0..64) (padded) with a smem bitonic network, then rank-merge
    for (int i = nb + lane; i < SEL_BUF; i += 32) buf[i] = kKeyMax;
    __syncwarp();
    for (int kk = 2; kk <= SEL_BUF; kk <<= 1)
      for (int j = kk >> 1; j > 0; j >>= 1) {
        const int i = lane;  // SEL_BUF/2 == 32 pairs
        const int lo = 2 * j * (i / j) + (i % j), hi = lo + j;
        const bool up = (lo & kk) == 0;
        unsigned long long a = buf[lo], b = buf[hi];
        if ((a > b) == up) { buf[lo] = b; buf[hi] = a; }
        __syncwarp();
      }
    for (int i = lane; i < nb; i += 32) {
      const int pos = i + lower_bound_u64(cur, k, buf[i]);
      if (pos < k) oth[pos] = buf[i];
    }
    for (int j = lane; j < k; j += 32) {
      const int pos = j + lower_bound_u64(buf, nb, cur[j]);
      if (pos < k) oth[pos] = cur[j];
    }
    __syncwarp();
    unsigned long long* t = cur; cur = oth; oth = t;
    nb = 0;
  };
  for (int64_t base = 0; base < cols; base += 32) {
    const int64_t c = base + lane;
    unsigned long long key = kKeyMax;
    if (c < cols) {
      const int64_t id = col0 + c;
      if (id != self) {
        float dv = dr[c];
        if (MODE == 1) dv = qn + xnorm[id] - 2.f * dv;
        if (MODE == 2) dv = -dv;
        key = make_key(dv, (uint32_t)id);
      }
    }
    const unsigned long long thr = cur[k - 1];
    const bool cand = key < thr;
    const unsigned m = __ballot_sync(0xffffffffu, cand);
    if (m == 0) continue;
    const int cnt = __popc(m);
    if (nb + cnt > SEL_BUF) flush();
    if (cand) buf[nb + __popc(m & ((1u << lane) - 1u))] = key;
    nb += cnt;
    __syncwarp();
    if (nb > SEL_BUF - 32) flush();
  }
  if (nb > 0) flush();
  for (int i = lane; i < k; i += 32) st[i] = cur[i];
}

__global__ void init_state_kernel(unsigned long long* s, size_t n) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) s[i] = kKeyMax;
}
__global__ void decode_state_kernel(const unsigned long long* s, size_t n, uint32_t* ids, float* ds) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  unsigned long long k = s[i];
  if (k == kKeyMax) {
    ids[i] = kSentinel;
    ds[i] = __int_as_float(0x7f800000);
  } else {
    ids[i] = key_id(k);
    ds[i] = key_dist(k);
  }
}

// ------------------------------------------------------------------ prune (R24)
// step 1+2: detour counts and the pruned list (CTA per node, K <= 128)
__global__ void detour_prune_kernel(const uint32_t* __restrict__ knn, int64_t n, int K, int R,
                                    uint32_t* __restrict__ pruned) {
  extern __shared__ __align__(16) uint8_t sm[];
  uint32_t* rows = reinterpret_cast<uint32_t*>(sm);  // K x K
  uint32_t* cnt = rows + (size_t)K * K;               // K
  const int64_t x = blockIdx.x;
  const uint32_t* rx = knn + x * K;
  for (int t = threadIdx.x; t < K * K; t += blockDim.x) {
    const int i = t / K, c = t % K;
    rows[t] = knn[(int64_t)rx[i] * K + c];
  }
  __syncthreads();
  const int j = threadIdx.x;
  if (j < K) {
    const uint32_t yj = rx[j];
    int count = 0;
    for (int i = 0; i < j; ++i) {
      const uint32_t* ri = rows + (size_t)i * K;
      for (int t = 0; t < j; ++t)
        if (ri[t] == yj) { ++count; break; }
    }
    cnt[j] = (uint32_t)count;
  }
  __syncthreads();
  if (j < K) {
    const uint32_t cj = cnt[j];
    int rank = 0;
    for (int i = 0; i < K; ++i) {
      const uint32_t ci = cnt[i];
      rank += (ci < cj) || (ci == cj && i < j);
    }
    if (rank < R) pruned[x * R + rank] = rx[j];
  }
}

__global__ void indegree_kernel(const uint32_t* pruned, int64_t n, int R, uint32_t* indeg) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n * R) return;
  atomicAdd(indeg + pruned[t], 1u);
}
__global__ void scatter_rev_kernel(const uint32_t* pruned, int64_t n, int R, const uint64_t* off, uint32_t* fill,
                                   unsigned long long* rev) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n * R) return;
  const uint32_t y = pruned[t];
  const uint64_t x = (uint64_t)(t / R), r = (uint64_t)(t % R);
  const uint64_t pos = off[y] + atomicAdd(fill + y, 1u);
  rev[pos] = (r << 32) | x;  // ordered by (rank, source)
}
__global__ void merge_out_kernel(const uint32_t* pruned, const unsigned long long* rev, const uint64_t* off,
                                 int64_t n, int R, uint32_t* out) {
  int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= n) return;
  const uint32_t* p = pruned + x * R;
  uint32_t* o = out + x * R;
  int m = (int)(off[x + 1] - off[x]);
  if (m > R) m = R;
  const int h = R / 2;
  int cnt = 0;
  auto has = [&](uint32_t v) {
    for (int t = 0; t < cnt; ++t)
      if (o[t] == v) return true;
    return false;
  };
  for (int j = 0; j < h; ++j) o[cnt++] = p[j];
  for (int i = 0; i < m && cnt < R; ++i) {
    const uint32_t v = (uint32_t)(rev[off[x] + i] & 0xFFFFFFFFull);
    if (!has(v)) o[cnt++] = v;
  }
  for (int j = h; j < R && cnt < R; ++j)
    if (!has(p[j])) o[cnt++] = p[j];
  for (; cnt < R; ++cnt) o[cnt] = kSentinel;
}

struct Dev {
  void* p = nullptr;
  ~Dev() {
    if (p) cudaFree(p);
  }
};

static int to_device(const void* src, size_t bytes, Dev& holder, const void** out) {
  if (is_device_ptr(src)) {
    *out = src;
    return ALGAS_OK;
  }
  ALGAS_CUDA_TRY(cudaMalloc(&holder.p, std::max<size_t>(bytes, 16)));
  ALGAS_CUDA_TRY(cudaMemcpy(holder.p, src, bytes, cudaMemcpyHostToDevice));
  *out = holder.p;
  return ALGAS_OK;
}

// Exact kNN on CUDA cores: direct-form distance tiles + running top-k.
// self_ids (device, nq entries, nullable) overrides self_base per query.
static int knn_direct(const float* base, int64_t n, const float* queries, int64_t nq, int32_t dim, int32_t metric,
                      int32_t k, int64_t self_base, const int64_t* self_ids, uint32_t* out_ids, float* out_dists) {
  Dev hx, hq, hstate, hD, hid, hd;
  const float *X = nullptr, *Q = nullptr;
  int rc;
  if ((rc = to_device(base, (size_t)n * dim * 4, hx, (const void**)&X))) return rc;
  if ((rc = to_device(queries, (size_t)nq * dim * 4, hq, (const void**)&Q))) return rc;
  const int64_t QB = std::min<int64_t>(nq, 4096);
  const int64_t NB = std::min<int64_t>((n + 3) & ~int64_t(3), 65536);  // row stride of the distance block: a multiple of 4 (16-B rows for the tcgen05 epilogue)
  ALGAS_CUDA_TRY(cudaMalloc(&hstate.p, (size_t)QB * k * 8));
  ALGAS_CUDA_TRY(cudaMalloc(&hD.p, (size_t)QB * NB * 4));
  const bool dev_out = is_device_ptr(out_ids) && is_device_ptr(out_dists);
  std::vector<uint32_t> hids;
  std::vector<float> hds;
  ALGAS_CUDA_TRY(cudaMalloc(&hid.p, (size_t)QB * k * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hd.p, (size_t)QB * k * 4));
  const int sel_smem = SEL_WARPS * (2 * k + SEL_BUF) * 8;
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(select_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, sel_smem));
  auto* unsafe_D = (float*)hD.p;
  for (int64_t q0 = 0; q0 < nq; q0 += QB) {
    const int64_t qb = std::min<int64_t>(QB, nq - q0);
    const size_t ns = (size_t)qb * k;
    init_state_kernel<<<(unsigned)((ns + 255) / 256), 256>>>((unsigned long long*)hstate.p, ns);
    for (int64_t x0 = 0; x0 < n; x0 += NB) {
      const int64_t nb = std::min<int64_t>(NB, n - x0);
      dim3 grid((unsigned)((nb + TX - 1) / TX), (unsigned)((qb + TQ - 1) / TQ));
      if (metric == ALGAS_L2)
        dist_tile_kernel<kL2><<<grid, 256>>>(Q + q0 * dim, qb, X + x0 * dim, nb, dim, unsafe_D, NB);
      else
        dist_tile_kernel<kIP><<<grid, 256>>>(Q + q0 * dim, qb, X + x0 * dim, nb, dim, unsafe_D, NB);
      select_kernel<0><<<(unsigned)((qb + SEL_WARPS - 1) / SEL_WARPS), SEL_WARPS * 32, sel_smem>>>(
          unsafe_D, NB, (int)qb, nb, x0, q0, self_base, k, (unsigned long long*)hstate.p, nullptr, nullptr, self_ids);
    }
    decode_state_kernel<<<(unsigned)((ns + 255) / 256), 256>>>((unsigned long long*)hstate.p, ns, (uint32_t*)hid.p,
                                                               (float*)hd.p);
    ALGAS_CUDA_TRY(cudaGetLastError());
    ALGAS_CUDA_TRY(cudaMemcpy(out_ids + q0 * k, hid.p, ns * 4, cudaMemcpyDefault));
    ALGAS_CUDA_TRY(cudaMemcpy(out_dists + q0 * k, hd.p, ns * 4, cudaMemcpyDefault));
  }
  (void)dev_out;
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}


// ------------------------------------------------------------------ tensor-core screened kNN
// The kNN distance block is a dense contraction: |q|^2 + |x|^2 - 2 q.x with
// q.x from cuBLAS tensor-core GEMMs in 3xTF32 (hi/lo split, ~fp32 accuracy),
// screening the top K2 = k + margin candidates per query; the candidates are
// re-ranked with the exact direct-form fp32 distance (the same arithmetic as
// knn_direct), and a per-query certificate
//     screened_dist(K2-th) - eps  >  exact_dist(k-th)
// with eps a rigorous bound on |screened - exact| proves that no unscreened
// point can enter the top k; queries failing it are redone by knn_direct.
// The output is therefore identical to knn_direct's.
__device__ __forceinline__ float tf32_hi(float v) {
  uint32_t h;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(h) : "f"(v));
  return __uint_as_float(h);
}
__global__ void split_tf32_kernel(const float* __restrict__ in, size_t count, float* __restrict__ hi,
                                  float* __restrict__ lo) {
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  const float v = in[i];
  const float h = tf32_hi(v);
  hi[i] = h;
  lo[i] = v - h;  // exact: v - h has at most 14 significant bits
}
// squared norms (sequential fp32 FMA over dims, one thread per row) and the
// running maximum (non-negative floats order like their bit patterns)
__global__ void norms_kernel(const float* __restrict__ X, int64_t n, int d, float* __restrict__ out,
                             unsigned int* __restrict__ maxbits) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const float4* r = reinterpret_cast<const float4*>(X + i * d);
  float acc = 0.f;
  for (int j = 0; j < d / 4; ++j) {
    const float4 v = r[j];
    acc = fmaf(v.x, v.x, acc); acc = fmaf(v.y, v.y, acc); acc = fmaf(v.z, v.z, acc); acc = fmaf(v.w, v.w, acc);
  }
  out[i] = acc;
  if (maxbits) atomicMax(maxbits, __float_as_uint(acc));
}
// one warp per query: exact distances of its K2 screened candidates (same
// arithmetic as dist_tile_kernel: sequential FMA over dims), sort, keep k,
// and the certificate.  K2 <= KMAX (power of two, smem bitonic sort).
template <int METRIC, int KMAX>
__global__ void __launch_bounds__(128) rerank_kernel(const float* __restrict__ Q, int64_t qn, const float* __restrict__ X,
                                                     int d, const unsigned long long* __restrict__ state, int K2,
                                                     int k, const float* __restrict__ qnorm, float xmax, float eps_c,
                                                     uint32_t* __restrict__ out_ids, float* __restrict__ out_d,
                                                     int* __restrict__ fail) {
  __shared__ unsigned long long keys[4][KMAX];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t row = (int64_t)blockIdx.x * 4 + warp;
  if (row >= qn) return;
  unsigned long long* kk = keys[warp];
  const unsigned long long* st = state + row * K2;
  const float* q = Q + row * d;
  for (int i = lane; i < KMAX; i += 32) {
    unsigned long long key = kKeyMax;
    if (i < K2 && st[i] != kKeyMax) {
      const uint32_t id = key_id(st[i]);
      const float4* xr = reinterpret_cast<const float4*>(X + (int64_t)id * d);
      const float4* qr = reinterpret_cast<const float4*>(q);
      float acc = 0.f;
      for (int j = 0; j < d / 4; ++j) {
        const float4 a = qr[j], b = xr[j];
        if (METRIC == kL2) {
          float t = a.x - b.x; acc = fmaf(t, t, acc);
          t = a.y - b.y; acc = fmaf(t, t, acc);
          t = a.z - b.z; acc = fmaf(t, t, acc);
          t = a.w - b.w; acc = fmaf(t, t, acc);
        } else {
          acc = fmaf(a.x, b.x, acc); acc = fmaf(a.y, b.y, acc); acc = fmaf(a.z, b.z, acc); acc = fmaf(a.w, b.w, acc);
        }
      }
      key = make_key(METRIC == kL2 ? acc : -acc, id);
    }
    kk[i] = key;
  }
  __syncwarp();
  for (int size = 2; size <= KMAX; size <<= 1)
    for (int j = size >> 1; j > 0; j >>= 1) {
      for (int t = lane; t < KMAX / 2; t += 32) {
        const int lo = 2 * j * (t / j) + (t % j), hi = lo + j;
        const bool up = (lo & size) == 0;
        const unsigned long long a = kk[lo], b = kk[hi];
        if ((a > b) == up) { kk[lo] = b; kk[hi] = a; }
      }
      __syncwarp();
    }
  for (int i = lane; i < k; i += 32) {
    const unsigned long long key = kk[i];
    out_ids[row * k + i] = key == kKeyMax ? kSentinel : key_id(key);
    out_d[row * k + i] = key == kKeyMax ? __int_as_float(0x7f800000) : key_dist(key);
  }
  if (lane == 0) {
    const unsigned long long thr = st[K2 - 1];
    int ok = 1;
    if (thr != kKeyMax) {  // else every point was screened
      const float qq = qnorm[row];
      const float eps = METRIC == kL2 ? eps_c * (qq + xmax) : eps_c * sqrtf(qq) * sqrtf(xmax);
      const unsigned long long kth = kk[k - 1];
      ok = (kth != kKeyMax) && (key_dist(thr) - eps > key_dist(kth));
    }
    fail[row] = !ok;
  }
}
__global__ void gather_rows_kernel(const float* __restrict__ Q, int d, const int64_t* __restrict__ rows, int m,
                                   float* __restrict__ out) {
  const int i = blockIdx.x;
  for (int j = threadIdx.x; j < d; j += blockDim.x) out[(int64_t)i * d + j] = Q[rows[i] * d + j];
}
__global__ void scatter_results_kernel(const uint32_t* __restrict__ ids, const float* __restrict__ ds, int k,
                                       const int64_t* __restrict__ rows, int m, uint32_t* __restrict__ out_ids,
                                       float* __restrict__ out_d) {
  const int i = blockIdx.x;
  for (int j = threadIdx.x; j < k; j += blockDim.x) {
    out_ids[rows[i] * k + j] = ids[(int64_t)i * k + j];
    out_d[rows[i] * k + j] = ds[(int64_t)i * k + j];
  }
}

static std::mutex g_cublas_mu;
static cublasHandle_t cublas_handle() {
  static cublasHandle_t h[64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_cublas_mu);
  if (!h[dev & 63]) cublasCreate(&h[dev & 63]);
  return h[dev & 63];
}
#define ALGAS_CUBLAS_TRY(expr)                                                                   \
  do {                                                                                           \
    cublasStatus_t _s = (expr);                                                                  \
    if (_s != CUBLAS_STATUS_SUCCESS)                                                             \
      return ::algas::set_error(ALGAS_ECUDA, "%s failed: cublas status %d", #expr, (int)_s);     \
  } while (0)

// screened-path statistics of the last call on this thread (tests, bench)
static thread_local int64_t g_knn_screened_rows = 0, g_knn_fallback_rows = 0;

static int knn_screened(const float* X, int64_t n, const float* Q, int64_t nq, int32_t d, int32_t metric, int32_t k,
                        int64_t self_base, uint32_t* out_ids, float* out_dists) {
  const int margin = std::max(32, k / 2);
  const int K2 = (int)std::min<int64_t>(k + margin, 256);
  const int64_t QB = std::min<int64_t>(nq, 4096);
  const int64_t NB = std::min<int64_t>((n + 3) & ~int64_t(3), 65536);  // row stride of the distance block: a multiple of 4 (16-B rows for the tcgen05 epilogue)
  Dev hxh, hxl, hqh, hql, hxn, hqn, hmax, hstate, hD, hid, hd, hfail, hrows, hself, hqf, hfid, hfd;
  ALGAS_CUDA_TRY(cudaMalloc(&hxh.p, (size_t)n * d * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hxl.p, (size_t)n * d * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hqh.p, (size_t)QB * d * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hql.p, (size_t)QB * d * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hxn.p, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hqn.p, (size_t)nq * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hmax.p, 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hstate.p, (size_t)QB * K2 * 8));
  ALGAS_CUDA_TRY(cudaMalloc(&hD.p, (size_t)QB * NB * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hid.p, (size_t)QB * k * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hd.p, (size_t)QB * k * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hfail.p, (size_t)QB * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hrows.p, (size_t)QB * 8));
  float *Xh = (float*)hxh.p, *Xl = (float*)hxl.p, *Qh = (float*)hqh.p, *Ql = (float*)hql.p;
  float *xn = (float*)hxn.p, *qn = (float*)hqn.p;
  ALGAS_CUDA_TRY(cudaMemset(hmax.p, 0, 4));
  const size_t nx = (size_t)n * d;
  split_tf32_kernel<<<(unsigned)((nx + 255) / 256), 256>>>(X, nx, Xh, Xl);
  norms_kernel<<<(unsigned)((n + 255) / 256), 256>>>(X, n, d, xn, (unsigned int*)hmax.p);
  norms_kernel<<<(unsigned)((nq + 255) / 256), 256>>>(Q, nq, d, qn, nullptr);
  unsigned int maxbits = 0;
  ALGAS_CUDA_TRY(cudaMemcpy(&maxbits, hmax.p, 4, cudaMemcpyDeviceToHost));
  float xmax;
  memcpy(&xmax, &maxbits, 4);
  // rigorous screening error bound, relative to |q|^2 + max|x|^2 (L2) or
  // |q| max|x| (IP): operand split/rounding 3 * 2^-22, fp32 accumulation of
  // the GEMMs, the norms and the direct form gamma_(d+8), final roundings
  const double u = std::ldexp(1.0, -24);
  const double gam = (d + 8) * u / (1.0 - (d + 8) * u);
  const float eps_c = (float)(1.05 * (4.0 * gam + 8.0 * std::ldexp(1.0, -22)));
  const char* gemm_env = getenv("ALGAS_KNN_GEMM");
  const bool use_cublas = gemm_env != nullptr && strcmp(gemm_env, "cublas") == 0;
  cublasHandle_t h = use_cublas ? cublas_handle() : nullptr;
  if (use_cublas) ALGAS_CUBLAS_TRY(cublasSetStream(h, 0));
  const int sel_smem = SEL_WARPS * (2 * K2 + SEL_BUF) * 8;
  void* sel = metric == ALGAS_L2 ? (void*)select_kernel<1> : (void*)select_kernel<2>;
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(sel, cudaFuncAttributeMaxDynamicSharedMemorySize, sel_smem));
  float* D = (float*)hD.p;
  const float one = 1.f, zero = 0.f;
  std::vector<int> fail((size_t)QB);
  std::vector<int64_t> frows;
  for (int64_t q0 = 0; q0 < nq; q0 += QB) {
    const int64_t qb = std::min<int64_t>(QB, nq - q0);
    const size_t ns = (size_t)qb * K2;
    init_state_kernel<<<(unsigned)((ns + 255) / 256), 256>>>((unsigned long long*)hstate.p, ns);
    split_tf32_kernel<<<(unsigned)((qb * d + 255) / 256), 256>>>(Q + q0 * d, (size_t)qb * d, Qh, Ql);
    for (int64_t x0 = 0; x0 < n; x0 += NB) {
      const int64_t nb = std::min<int64_t>(NB, n - x0);
      // D (row-major qb x nb, ld NB) = Q_blk . X_blk^T: hi.hi + lo.hi + hi.lo
      if (use_cublas) {
        // library path (A/B: ALGAS_KNN_GEMM=cublas): D^T col-major = X_blk . Q_blk^T
        const float* A[3] = {Xh + x0 * d, Xl + x0 * d, Xh + x0 * d};
        const float* B[3] = {Qh, Qh, Ql};
        for (int g = 0; g < 3; ++g)
          ALGAS_CUBLAS_TRY(cublasGemmEx(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)qb, d, &one, A[g], CUDA_R_32F, d,
                                        B[g], CUDA_R_32F, d, g == 0 ? &zero : &one, D, CUDA_R_32F, (int)NB,
                                        CUBLAS_COMPUTE_32F_FAST_TF32, CUBLAS_GEMM_DEFAULT));
      } else {
        // hand-written tcgen05 kernel (knn_tc.cu)
        int rc = tc_dot_3xtf32(Qh, Ql, qb, Xh + x0 * d, Xl + x0 * d, nb, d, D, NB, 0);
        if (rc) return rc;
      }
      if (metric == ALGAS_L2)
        select_kernel<1><<<(unsigned)((qb + SEL_WARPS - 1) / SEL_WARPS), SEL_WARPS * 32, sel_smem>>>(
            D, NB, (int)qb, nb, x0, q0, self_base, K2, (unsigned long long*)hstate.p, qn, xn, nullptr);
      else
        select_kernel<2><<<(unsigned)((qb + SEL_WARPS - 1) / SEL_WARPS), SEL_WARPS * 32, sel_smem>>>(
            D, NB, (int)qb, nb, x0, q0, self_base, K2, (unsigned long long*)hstate.p, qn, xn, nullptr);
    }
    const unsigned rb = (unsigned)((qb + 3) / 4);
    if (metric == ALGAS_L2)
      rerank_kernel<kL2, 256><<<rb, 128>>>(Q + q0 * d, qb, X, d, (unsigned long long*)hstate.p, K2, k, qn + q0, xmax,
                                            eps_c, (uint32_t*)hid.p, (float*)hd.p, (int*)hfail.p);
    else
      rerank_kernel<kIP, 256><<<rb, 128>>>(Q + q0 * d, qb, X, d, (unsigned long long*)hstate.p, K2, k, qn + q0, xmax,
                                            eps_c, (uint32_t*)hid.p, (float*)hd.p, (int*)hfail.p);
    ALGAS_CUDA_TRY(cudaGetLastError());
    ALGAS_CUDA_TRY(cudaMemcpy(fail.data(), hfail.p, (size_t)qb * 4, cudaMemcpyDeviceToHost));
    frows.clear();
    for (int64_t i = 0; i < qb; ++i)
      if (fail[i]) frows.push_back(i);
    g_knn_screened_rows += qb;
    g_knn_fallback_rows += (int64_t)frows.size();
    if (!frows.empty()) {
      // redo the uncertified queries exactly on CUDA cores
      const int m = (int)frows.size();
      std::vector<int64_t> selfs(m);
      for (int i = 0; i < m; ++i) selfs[i] = self_base >= 0 ? self_base + q0 + frows[i] : -1;
      Dev a, b, c, e, f;
      ALGAS_CUDA_TRY(cudaMalloc(&a.p, (size_t)m * 8));
      ALGAS_CUDA_TRY(cudaMalloc(&b.p, (size_t)m * 8));
      ALGAS_CUDA_TRY(cudaMalloc(&c.p, (size_t)m * d * 4));
      ALGAS_CUDA_TRY(cudaMalloc(&e.p, (size_t)m * k * 4));
      ALGAS_CUDA_TRY(cudaMalloc(&f.p, (size_t)m * k * 4));
      ALGAS_CUDA_TRY(cudaMemcpy(a.p, frows.data(), (size_t)m * 8, cudaMemcpyHostToDevice));
      ALGAS_CUDA_TRY(cudaMemcpy(b.p, selfs.data(), (size_t)m * 8, cudaMemcpyHostToDevice));
      gather_rows_kernel<<<m, 128>>>(Q + q0 * d, d, (const int64_t*)a.p, m, (float*)c.p);
      int rc = knn_direct(X, n, (const float*)c.p, m, d, metric, k, -1, (const int64_t*)b.p, (uint32_t*)e.p,
                          (float*)f.p);
      if (rc) return rc;
      scatter_results_kernel<<<m, 128>>>((const uint32_t*)e.p, (const float*)f.p, k, (const int64_t*)a.p, m,
                                         (uint32_t*)hid.p, (float*)hd.p);
      ALGAS_CUDA_TRY(cudaGetLastError());
    }
    ALGAS_CUDA_TRY(cudaMemcpy(out_ids + q0 * k, hid.p, (size_t)qb * k * 4, cudaMemcpyDefault));
    ALGAS_CUDA_TRY(cudaMemcpy(out_dists + q0 * k, hd.p, (size_t)qb * k * 4, cudaMemcpyDefault));
  }
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}

// COSINE (R29): dst row = src row / |src row| (fp32; a zero row stays 0), one warp per row
__global__ void normalize_copy_kernel(const float4* __restrict__ src, int64_t n, int d4, float4* __restrict__ dst) {
  const int64_t r = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (r >= n) return;
  const int lane = threadIdx.x & 31;
  const float4* a = src + r * d4;
  float4* b = dst + r * d4;
  float ss = 0.f;
  for (int i = lane; i < d4; i += 32) {
    const float4 v = a[i];
    ss = fmaf(v.x, v.x, fmaf(v.y, v.y, fmaf(v.z, v.z, fmaf(v.w, v.w, ss))));
  }
  for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
  const float inv = ss > 0.f ? 1.0f / sqrtf(ss) : 1.0f;
  for (int i = lane; i < d4; i += 32) {
    float4 v = a[i];
    v.x *= inv; v.y *= inv; v.z *= inv; v.w *= inv;
    b[i] = v;
  }
}

// rows idx[0..m) of X (d4 float4 per row) into out, one warp per row
__global__ void gather_rows_kernel(const float4* __restrict__ X, const uint32_t* __restrict__ idx, int64_t m, int d4,
                                   float4* __restrict__ out) {
  const int64_t r = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (r >= m) return;
  const float4* src = X + (int64_t)idx[r] * d4;
  float4* dst = out + r * d4;
  for (int i = threadIdx.x & 31; i < d4; i += 32) dst[i] = src[i];
}

static int gather_rows(const float* X, const uint32_t* d_idx, int64_t m, int dim, float* out) {
  if (m == 0) return ALGAS_OK;
  gather_rows_kernel<<<(unsigned)((m + 7) / 8), 256>>>(reinterpret_cast<const float4*>(X), d_idx, m, dim / 4,
                                                       reinterpret_cast<float4*>(out));
  ALGAS_CUDA_TRY(cudaGetLastError());
  return ALGAS_OK;
}

// kNN lists (device, n x K, sorted rows, no self) -> graph (R24)
static int graph_from_knn(const uint32_t* dk, int64_t n, int K, int degree, int prune, uint32_t* out_graph) {
  const int R = std::min(degree, K);
  std::vector<uint32_t> tmp;
  int rc;
  if (prune) {
    if (R == degree) return algas_prune(dk, n, K, R, out_graph);
    tmp.resize((size_t)n * R);
    if ((rc = algas_prune(dk, n, K, R, tmp.data()))) return rc;
  } else {
    tmp.resize((size_t)n * R);
    ALGAS_CUDA_TRY(cudaMemcpy2D(tmp.data(), (size_t)R * 4, dk, (size_t)K * 4, (size_t)R * 4, (size_t)n,
                                cudaMemcpyDeviceToHost));
    if (R == degree) {
      ALGAS_CUDA_TRY(cudaMemcpy(out_graph, tmp.data(), tmp.size() * 4, cudaMemcpyDefault));
      return ALGAS_OK;
    }
  }
  // fewer than `degree` neighbours exist: pad rows with sentinels
  std::vector<uint32_t> full((size_t)n * degree, kSentinel);
  for (int64_t i = 0; i < n; ++i) std::copy(tmp.begin() + i * R, tmp.begin() + (i + 1) * R, full.begin() + i * degree);
  ALGAS_CUDA_TRY(cudaMemcpy(out_graph, full.data(), full.size() * 4, cudaMemcpyDefault));
  return ALGAS_OK;
}

}  // namespace algas

using namespace algas;

extern "C" {

int algas_knn(const float* base, int64_t n, const float* queries, int64_t nq, int32_t dim, int32_t metric, int32_t k,
              int64_t self_base, uint32_t* out_ids, float* out_dists) {
  if (!base || !queries || !out_ids || !out_dists || n < 1 || n >= (1LL << 31) || nq < 0 || dim < 4 ||
      dim % 4 != 0 || k < 1 || k > 1024 || (metric != ALGAS_L2 && metric != ALGAS_IP && metric != ALGAS_COSINE))
    return set_error(ALGAS_EINVAL, "algas_knn: bad arguments");
  if (nq == 0) return ALGAS_OK;
  Dev hx, hq, hxn, hqn;
  const float *X = nullptr, *Q = nullptr;
  int rc;
  if ((rc = to_device(base, (size_t)n * dim * 4, hx, (const void**)&X))) return rc;
  if ((rc = to_device(queries, (size_t)nq * dim * 4, hq, (const void**)&Q))) return rc;
  if (metric == ALGAS_COSINE) {
    // IP on unit copies of both sides (R29)
    const bool same = X == Q && n == nq;
    ALGAS_CUDA_TRY(cudaMalloc(&hxn.p, (size_t)n * dim * 4));
    normalize_copy_kernel<<<(unsigned)((n + 7) / 8), 256>>>(reinterpret_cast<const float4*>(X), n, dim / 4,
                                                            reinterpret_cast<float4*>(hxn.p));
    if (!same) {
      ALGAS_CUDA_TRY(cudaMalloc(&hqn.p, (size_t)nq * dim * 4));
      normalize_copy_kernel<<<(unsigned)((nq + 7) / 8), 256>>>(reinterpret_cast<const float4*>(Q), nq, dim / 4,
                                                               reinterpret_cast<float4*>(hqn.p));
    }
    ALGAS_CUDA_TRY(cudaGetLastError());
    X = (const float*)hxn.p;
    Q = same ? X : (const float*)hqn.p;
    metric = ALGAS_IP;
  }
  // path: tensor-core screen + exact rerank + certificate (default for large
  // problems), or the direct CUDA-core path; ALGAS_KNN_MODE=direct|screened
  const char* env = getenv("ALGAS_KNN_MODE");
  bool screened = (double)n * (double)nq >= 1e8 && k + std::max(32, k / 2) <= 256;
  if (env && !strcmp(env, "direct")) screened = false;
  if (env && !strcmp(env, "screened")) screened = k + std::max(32, k / 2) <= 256;
  if (screened) return knn_screened(X, n, Q, nq, dim, metric, k, self_base, out_ids, out_dists);
  return knn_direct(X, n, Q, nq, dim, metric, k, self_base, nullptr, out_ids, out_dists);
}

int64_t algas_knn_last_stats(int64_t* fallback_rows) {
  if (fallback_rows) *fallback_rows = g_knn_fallback_rows;
  const int64_t r = g_knn_screened_rows;
  g_knn_screened_rows = g_knn_fallback_rows = 0;
  return r;
}

int algas_prune(const uint32_t* knn, int64_t n, int32_t knn_degree, int32_t degree, uint32_t* out_graph) {
  if (!knn || !out_graph || n < 1 || knn_degree < 1 || knn_degree > 128 || degree < 1 || degree > knn_degree)
    return set_error(ALGAS_EINVAL, "algas_prune: need 1 <= degree <= knn_degree <= 128");
  const int K = knn_degree, R = degree;
  Dev hk, hp, hindeg, hoff, hfill, hrev, hrev2, htmp, hout;
  const uint32_t* dk = nullptr;
  int rc;
  if ((rc = to_device(knn, (size_t)n * K * 4, hk, (const void**)&dk))) return rc;
  ALGAS_CUDA_TRY(cudaMalloc(&hp.p, (size_t)n * R * 4));
  const int threads = K <= 32 ? 32 : (K <= 64 ? 64 : 128);
  const int smem = (K * K + K) * 4;
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(detour_prune_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  detour_prune_kernel<<<(unsigned)n, threads, smem>>>(dk, n, K, R, (uint32_t*)hp.p);
  ALGAS_CUDA_TRY(cudaGetLastError());
  // reverse edges
  ALGAS_CUDA_TRY(cudaMalloc(&hindeg.p, (size_t)(n + 1) * 4));
  ALGAS_CUDA_TRY(cudaMemset(hindeg.p, 0, (size_t)(n + 1) * 4));
  const int64_t E = n * R;
  indegree_kernel<<<(unsigned)((E + 255) / 256), 256>>>((uint32_t*)hp.p, n, R, (uint32_t*)hindeg.p);
  ALGAS_CUDA_TRY(cudaMalloc(&hoff.p, (size_t)(n + 1) * 8));
  {
    // exclusive scan of in-degrees (as u64) -> segment offsets
    std::vector<uint32_t> indeg(n + 1);
    ALGAS_CUDA_TRY(cudaMemcpy(indeg.data(), hindeg.p, (size_t)(n + 1) * 4, cudaMemcpyDeviceToHost));
    std::vector<uint64_t> off(n + 1);
    uint64_t acc = 0;
    for (int64_t i = 0; i <= n; ++i) { off[i] = acc; if (i < n) acc += indeg[i]; }
    ALGAS_CUDA_TRY(cudaMemcpy(hoff.p, off.data(), (size_t)(n + 1) * 8, cudaMemcpyHostToDevice));
  }
  ALGAS_CUDA_TRY(cudaMalloc(&hfill.p, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMemset(hfill.p, 0, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hrev.p, (size_t)E * 8));
  ALGAS_CUDA_TRY(cudaMalloc(&hrev2.p, (size_t)E * 8));
  scatter_rev_kernel<<<(unsigned)((E + 255) / 256), 256>>>((uint32_t*)hp.p, n, R, (uint64_t*)hoff.p,
                                                           (uint32_t*)hfill.p, (unsigned long long*)hrev.p);
  ALGAS_CUDA_TRY(cudaGetLastError());
  {
    size_t tmp = 0;
    const uint64_t* offp = (const uint64_t*)hoff.p;
    ALGAS_CUDA_TRY(cub::DeviceSegmentedSort::SortKeys(nullptr, tmp, (const unsigned long long*)hrev.p,
                                                      (unsigned long long*)hrev2.p, (int)E, (int)n, offp,
                                                      offp + 1));
    ALGAS_CUDA_TRY(cudaMalloc(&htmp.p, std::max<size_t>(tmp, 16)));
    ALGAS_CUDA_TRY(cub::DeviceSegmentedSort::SortKeys(htmp.p, tmp, (const unsigned long long*)hrev.p,
                                                      (unsigned long long*)hrev2.p, (int)E, (int)n, offp,
                                                      offp + 1));
  }
  uint32_t* dout = out_graph;
  const bool dev_out = is_device_ptr(out_graph);
  if (!dev_out) {
    ALGAS_CUDA_TRY(cudaMalloc(&hout.p, (size_t)n * R * 4));
    dout = (uint32_t*)hout.p;
  }
  merge_out_kernel<<<(unsigned)((n + 127) / 128), 128>>>((uint32_t*)hp.p, (unsigned long long*)hrev2.p,
                                                         (uint64_t*)hoff.p, n, R, dout);
  ALGAS_CUDA_TRY(cudaGetLastError());
  if (!dev_out) ALGAS_CUDA_TRY(cudaMemcpy(out_graph, dout, (size_t)n * R * 4, cudaMemcpyDeviceToHost));
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}

int algas_build_graph(const float* data, int64_t n, int32_t dim, int32_t metric, int32_t knn_degree, int32_t degree,
                      int32_t prune, uint32_t* out_graph) {
  if (!data || !out_graph || n < 2 || knn_degree < degree || degree < 1)
    return set_error(ALGAS_EINVAL, "algas_build_graph: bad arguments");
  const int K = (int)std::min<int64_t>(knn_degree, n - 1);
  Dev guard_k, guard_d;
  ALGAS_CUDA_TRY(cudaMalloc(&guard_k.p, (size_t)n * K * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&guard_d.p, (size_t)n * K * 4));
  int rc = algas_knn(data, n, data, n, dim, metric, K, 0, (uint32_t*)guard_k.p, (float*)guard_d.p);
  if (rc) return rc;
  return graph_from_knn((const uint32_t*)guard_k.p, n, K, degree, prune, out_graph);
}

constexpr int kLloyd = 8;

// Partitioned approximate kNN (R30): sampled
// centres, each point assigned to its `overlap` nearest centres, exact kNN
// inside every cluster (algas_knn, self excluded), per-point merge of its
// cluster lists by (dist, id) with duplicates removed.
int algas_knn_partitioned(const float* data, int64_t n, int32_t dim, int32_t metric, int32_t k, int32_t n_clusters,
                          int32_t overlap, uint32_t* out_ids, float* out_dists) {
  if (!data || !out_ids || !out_dists || n < 2 || n >= (1LL << 31) || dim < 4 || dim % 4 != 0 || k < 1 ||
      k > 1024 || n_clusters < 1 || n_clusters > n || overlap < 1 || overlap > n_clusters ||
      (metric != ALGAS_L2 && metric != ALGAS_IP && metric != ALGAS_COSINE))
    return set_error(ALGAS_EINVAL, "algas_knn_partitioned: bad arguments");
  static const bool trace = getenv("ALGAS_TRACE") != nullptr;
  auto t_last = std::chrono::steady_clock::now();
  auto phase = [&](const char* name) {
    if (!trace) return;
    cudaDeviceSynchronize();
    const auto t = std::chrono::steady_clock::now();
    fprintf(stderr, "[algas_knn_partitioned] %s %.3f s\n", name, std::chrono::duration<double>(t - t_last).count());
    t_last = t;
  };
  Dev hx;
  const float* X = nullptr;
  int rc;
  if ((rc = to_device(data, (size_t)n * dim * 4, hx, (const void**)&X))) return rc;
  const int64_t m = n_clusters;
  const int c = overlap;
  // 1. centres: rows floor(j n / m), j < m
  std::vector<uint32_t> cid(m);
  for (int64_t j = 0; j < m; ++j) cid[j] = (uint32_t)((j * n) / m);
  Dev hcid, hC, hmem, hB;
  ALGAS_CUDA_TRY(cudaMalloc(&hcid.p, (size_t)m * 4));
  ALGAS_CUDA_TRY(cudaMemcpy(hcid.p, cid.data(), (size_t)m * 4, cudaMemcpyHostToDevice));
  ALGAS_CUDA_TRY(cudaMalloc(&hC.p, (size_t)m * dim * 4));
  if ((rc = gather_rows(X, (const uint32_t*)hcid.p, m, dim, (float*)hC.p))) return rc;
  // 1b. kLloyd Lloyd iterations on the sample rows floor(i n / ns), ns =
  //     min(n, 32 m): each sample row to its nearest centre, centre = mean of
  //     its rows (double sums in row order, rounded to fp32; an empty
  //     centre stays).  Moves centres off the high-dimensional hubs.
  if (m > 1) {
    const int64_t ns = std::min<int64_t>(n, 32 * m);
    std::vector<uint32_t> sid(ns);
    for (int64_t i = 0; i < ns; ++i) sid[i] = (uint32_t)((i * n) / ns);
    Dev hsid, hS;
    ALGAS_CUDA_TRY(cudaMalloc(&hsid.p, (size_t)ns * 4));
    ALGAS_CUDA_TRY(cudaMemcpy(hsid.p, sid.data(), (size_t)ns * 4, cudaMemcpyHostToDevice));
    ALGAS_CUDA_TRY(cudaMalloc(&hS.p, (size_t)ns * dim * 4));
    if ((rc = gather_rows(X, (const uint32_t*)hsid.p, ns, dim, (float*)hS.p))) return rc;
    std::vector<float> S((size_t)ns * dim), C((size_t)m * dim);
    ALGAS_CUDA_TRY(cudaMemcpy(S.data(), hS.p, S.size() * 4, cudaMemcpyDeviceToHost));
    ALGAS_CUDA_TRY(cudaMemcpy(C.data(), hC.p, C.size() * 4, cudaMemcpyDeviceToHost));
    std::vector<uint32_t> a1(ns);
    std::vector<float> a1d(ns);
    std::vector<double> acc((size_t)m * dim);
    std::vector<int64_t> cnt(m);
    for (int it = 0; it < kLloyd; ++it) {
      if ((rc = algas_knn((const float*)hC.p, m, (const float*)hS.p, ns, dim, metric, 1, -1, a1.data(), a1d.data())))
        return rc;
      std::fill(acc.begin(), acc.end(), 0.0);
      std::fill(cnt.begin(), cnt.end(), 0);
      for (int64_t i = 0; i < ns; ++i) {
        const uint32_t j = a1[i];
        ++cnt[j];
        for (int t = 0; t < dim; ++t) acc[(size_t)j * dim + t] += (double)S[(size_t)i * dim + t];
      }
      for (int64_t j = 0; j < m; ++j)
        if (cnt[j] > 0)
          for (int t = 0; t < dim; ++t) C[(size_t)j * dim + t] = (float)(acc[(size_t)j * dim + t] / (double)cnt[j]);
      ALGAS_CUDA_TRY(cudaMemcpy(hC.p, C.data(), C.size() * 4, cudaMemcpyHostToDevice));
    }
  }
  // 2. assignment under a capacity (hub centres of high-dimensional data
  //    would otherwise take half the points): every point's P nearest
  //    centres in (dist, centre) order; points in id order take the first c
  //    of them that still have room (cap = ceil(2 c n / m), or n when
  //    4 c >= m), else the
  //    lowest-index centres with room (R30)
  const int P = (int)std::min<int64_t>(m, 4 * c + 4);
  std::vector<uint32_t> pref((size_t)n * P);
  std::vector<float> prefd((size_t)n * P);
  if ((rc = algas_knn((const float*)hC.p, m, X, n, dim, metric, P, -1, pref.data(), prefd.data()))) return rc;
  std::vector<uint32_t> asg((size_t)n * c);
  {
    const int64_t cap = 4 * (int64_t)c >= m ? n : (2 * (int64_t)c * n + m - 1) / m;
    std::vector<int64_t> load(m, 0);
    int64_t low = 0;  // every centre below `low` is full
    for (int64_t i = 0; i < n; ++i) {
      uint32_t* a = asg.data() + (size_t)i * c;
      int got = 0;
      for (int e = 0; e < P && got < c; ++e) {
        const uint32_t j = pref[(size_t)i * P + e];
        if (load[j] < cap) { a[got++] = j; ++load[j]; }
      }
      for (int64_t j = low; got < c && j < m; ++j) {
        if (load[j] >= cap) { if (j == low) ++low; continue; }
        bool dup = false;
        for (int r = 0; r < got; ++r) dup |= a[r] == (uint32_t)j;
        if (!dup) { a[got++] = (uint32_t)j; ++load[j]; }
      }
      if (got < c) return set_error(ALGAS_ESTATE, "algas_knn_partitioned: assignment ran out of room");
    }
  }
  phase("assign");
  // 3. members of each cluster, ascending global id
  std::vector<int64_t> start(m + 1, 0);
  for (size_t e = 0; e < asg.size(); ++e) ++start[asg[e] + 1];
  for (int64_t j = 0; j < m; ++j) start[j + 1] += start[j];
  std::vector<uint32_t> mem(asg.size());
  {
    std::vector<int64_t> fill(start.begin(), start.end() - 1);
    for (int64_t i = 0; i < n; ++i)
      for (int r = 0; r < c; ++r) {
        const uint32_t j = asg[(size_t)i * c + r];
        mem[fill[j]++] = (uint32_t)i;
      }
  }
  int64_t smax = 0;
  for (int64_t j = 0; j < m; ++j) smax = std::max(smax, start[j + 1] - start[j]);
  ALGAS_CUDA_TRY(cudaMalloc(&hmem.p, std::max<size_t>(mem.size() * 4, 16)));
  ALGAS_CUDA_TRY(cudaMemcpy(hmem.p, mem.data(), mem.size() * 4, cudaMemcpyHostToDevice));
  if (k <= kPartMaxKnn && getenv("ALGAS_PART_PER_CLUSTER") == nullptr) {
    // 4+5 on the GPU, all clusters in one launch (build_part.cu): a CTA takes
    // 64 member rows of one cluster against all its members (fp32 direct
    // form, running top-k in shared memory; lists keyed by GLOBAL id, so
    // (dist, id) ties resolve as globally; a cluster of s points yields
    // min(k, s - 1) entries, the rest padding); then every point merges its
    // c cluster lists (repeated ids dropped, first k)
    const float* Xm = X;
    int met = metric;
    Dev hxn;
    if (metric == ALGAS_COSINE) {  // IP on unit-row copies (R29)
      ALGAS_CUDA_TRY(cudaMalloc(&hxn.p, (size_t)n * dim * 4));
      normalize_copy_kernel<<<(unsigned)((n + 7) / 8), 256>>>(reinterpret_cast<const float4*>(X), n, dim / 4,
                                                              reinterpret_cast<float4*>(hxn.p));
      ALGAS_CUDA_TRY(cudaGetLastError());
      Xm = (const float*)hxn.p;
      met = ALGAS_IP;
    }
    std::vector<ClusterBlock> blocks;
    for (int64_t j = 0; j < m; ++j)
      for (int64_t r0 = 0; r0 < start[j + 1] - start[j]; r0 += 64) blocks.push_back(ClusterBlock{(int32_t)j, (int32_t)r0});
    std::vector<uint32_t> slot_of((size_t)n * c);
    for (int64_t j = 0; j < m; ++j)
      for (int64_t t = start[j]; t < start[j + 1]; ++t) {
        const uint32_t i = mem[t];
        int r = 0;
        while (asg[(size_t)i * c + r] != (uint32_t)j) ++r;
        slot_of[(size_t)i * c + r] = (uint32_t)t;
      }
    Dev hstart, hlists, hslot, hoi, hod;
    ALGAS_CUDA_TRY(cudaMalloc(&hstart.p, (size_t)(m + 1) * 8));
    ALGAS_CUDA_TRY(cudaMemcpy(hstart.p, start.data(), (size_t)(m + 1) * 8, cudaMemcpyHostToDevice));
    ALGAS_CUDA_TRY(cudaMalloc(&hlists.p, std::max<size_t>(mem.size() * (size_t)k * 8, 16)));
    ALGAS_CUDA_TRY(cudaMalloc(&hslot.p, slot_of.size() * 4));
    ALGAS_CUDA_TRY(cudaMemcpy(hslot.p, slot_of.data(), slot_of.size() * 4, cudaMemcpyHostToDevice));
    phase("members");
    if ((rc = launch_cluster_knn(Xm, dim, met, (const uint32_t*)hmem.p, (const int64_t*)hstart.p, blocks, k,
                                 (uint64_t*)hlists.p)))
      return rc;
    phase("clusters");
    ALGAS_CUDA_TRY(cudaMalloc(&hoi.p, (size_t)n * k * 4));
    ALGAS_CUDA_TRY(cudaMalloc(&hod.p, (size_t)n * k * 4));
    if ((rc = launch_merge_lists((const uint64_t*)hlists.p, (const uint32_t*)hslot.p, n, c, k, (uint32_t*)hoi.p,
                                 (float*)hod.p)))
      return rc;
    phase("merge");
    ALGAS_CUDA_TRY(cudaMemcpy(out_ids, hoi.p, (size_t)n * k * 4, cudaMemcpyDefault));
    ALGAS_CUDA_TRY(cudaMemcpy(out_dists, hod.p, (size_t)n * k * 4, cudaMemcpyDefault));
    return ALGAS_OK;
  }
  // 4. exact kNN inside each cluster, one algas_knn call per cluster (k >
  //    kPartMaxKnn, or ALGAS_PART_PER_CLUSTER): rows gathered contiguously;
  //    local id order == global id order, so (dist, id) ties resolve as globally
  ALGAS_CUDA_TRY(cudaMalloc(&hB.p, (size_t)smax * dim * 4));
  phase("members");
  std::vector<uint32_t> cand((size_t)n * c * k, kSentinel);
  std::vector<float> candd((size_t)n * c * k, INFINITY);
  std::vector<uint32_t> li;
  std::vector<float> ld;
  for (int64_t j = 0; j < m; ++j) {
    const int64_t sj = start[j + 1] - start[j];
    if (sj < 2) continue;
    const int kj = (int)std::min<int64_t>(k, sj - 1);
    if ((rc = gather_rows(X, (const uint32_t*)hmem.p + start[j], sj, dim, (float*)hB.p))) return rc;
    li.resize((size_t)sj * kj);
    ld.resize((size_t)sj * kj);
    const auto tc0 = std::chrono::steady_clock::now();
    if ((rc = algas_knn((const float*)hB.p, sj, (const float*)hB.p, sj, dim, metric, kj, 0, li.data(), ld.data())))
      return rc;
    if (trace && j < 4)
      fprintf(stderr, "[algas_knn_partitioned] cluster %lld size %lld knn %.4f s\n", (long long)j, (long long)sj,
              std::chrono::duration<double>(std::chrono::steady_clock::now() - tc0).count());
    // scatter into each member's candidate block for this cluster
    for (int64_t t = 0; t < sj; ++t) {
      const uint32_t i = mem[start[j] + t];
      int r = 0;
      while (asg[(size_t)i * c + r] != (uint32_t)j) ++r;
      uint32_t* ci = cand.data() + ((size_t)i * c + r) * k;
      float* cd = candd.data() + ((size_t)i * c + r) * k;
      for (int e = 0; e < kj; ++e) {
        const uint32_t l = li[(size_t)t * kj + e];
        ci[e] = l == kSentinel ? kSentinel : mem[start[j] + l];
        cd[e] = ld[(size_t)t * kj + e];
      }
    }
  }
  if (trace) {
    int64_t fb = 0;
    const int64_t sc = algas_knn_last_stats(&fb);
    fprintf(stderr, "[algas_knn_partitioned] m=%lld largest cluster %lld, rows screened %lld, fallback %lld\n",
            (long long)m, (long long)smax, (long long)sc, (long long)fb);
  }
  phase("clusters");
  // 5. per-point merge (dist, id), duplicates dropped, padded to k
  std::vector<uint32_t> oi((size_t)n * k);
  std::vector<float> od((size_t)n * k);
  const int nth = (int)std::max<unsigned>(1, std::min<unsigned>(16, std::thread::hardware_concurrency()));
  std::vector<std::thread> th;
  for (int w = 0; w < nth; ++w)
    th.emplace_back([&, w] {
      for (int64_t i = w; i < n; i += nth)
        algas_merge_topk(cand.data() + (size_t)i * c * k, candd.data() + (size_t)i * c * k, c * k, k,
                         oi.data() + (size_t)i * k, od.data() + (size_t)i * k);
    });
  for (auto& t : th) t.join();
  phase("merge");
  ALGAS_CUDA_TRY(cudaMemcpy(out_ids, oi.data(), oi.size() * 4, cudaMemcpyDefault));
  ALGAS_CUDA_TRY(cudaMemcpy(out_dists, od.data(), od.size() * 4, cudaMemcpyDefault));
  return ALGAS_OK;
}

// Reverse neighbour lists of one R35 round (device, from the round's input
// lists in[n][k]): rev[p][j], j < fan = the first fan pairs (a, r) in (a, r)
// order with in[r][a] == p, a < fan, r != p (SENTINEL-padded) -- counts,
// offsets, a scatter of (a << 32 | r) keys, a segmented sort per point.
__global__ void rev_count_kernel(const uint32_t* in, int64_t n, int k, int fan, uint32_t* cnt) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n * fan) return;
  const int64_t r = i / fan;
  const uint32_t p = in[r * k + i % fan];
  if (p != kSentinel && (int64_t)p != r) atomicAdd(cnt + p, 1u);
}
__global__ void rev_scatter_kernel(const uint32_t* in, int64_t n, int k, int fan, const uint64_t* off,
                                   uint32_t* fill, unsigned long long* keys) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n * fan) return;
  const int64_t r = i / fan;
  const int a = (int)(i % fan);
  const uint32_t p = in[r * k + a];
  if (p == kSentinel || (int64_t)p == r) return;
  keys[off[p] + atomicAdd(fill + p, 1u)] = ((unsigned long long)a << 32) | (unsigned long long)r;
}
__global__ void rev_take_kernel(const unsigned long long* sorted, const uint64_t* off, int64_t n, int fan,
                                uint32_t* rev) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  const uint64_t o = off[p], m = off[p + 1] - o;
  for (int j = 0; j < fan; ++j) rev[p * fan + j] = (uint64_t)j < m ? (uint32_t)sorted[o + j] : kSentinel;
}
int build_rev_lists(const uint32_t* in, int64_t n, int k, int fan, uint32_t* rev) {
  Dev hcnt, hoff, hfill, hk1, hk2, htmp;
  const int64_t E = n * fan;
  ALGAS_CUDA_TRY(cudaMalloc(&hcnt.p, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMemset(hcnt.p, 0, (size_t)n * 4));
  const unsigned g = (unsigned)((E + 255) / 256);
  rev_count_kernel<<<g, 256>>>(in, n, k, fan, (uint32_t*)hcnt.p);
  ALGAS_CUDA_TRY(cudaGetLastError());
  std::vector<uint32_t> cnt(n);
  ALGAS_CUDA_TRY(cudaMemcpy(cnt.data(), hcnt.p, (size_t)n * 4, cudaMemcpyDeviceToHost));
  std::vector<uint64_t> off(n + 1);
  uint64_t acc = 0;
  for (int64_t i = 0; i < n; ++i) { off[i] = acc; acc += cnt[i]; }
  off[n] = acc;
  ALGAS_CUDA_TRY(cudaMalloc(&hoff.p, (size_t)(n + 1) * 8));
  ALGAS_CUDA_TRY(cudaMemcpy(hoff.p, off.data(), (size_t)(n + 1) * 8, cudaMemcpyHostToDevice));
  ALGAS_CUDA_TRY(cudaMalloc(&hfill.p, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMemset(hfill.p, 0, (size_t)n * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&hk1.p, std::max<size_t>((size_t)acc * 8, 16)));
  ALGAS_CUDA_TRY(cudaMalloc(&hk2.p, std::max<size_t>((size_t)acc * 8, 16)));
  rev_scatter_kernel<<<g, 256>>>(in, n, k, fan, (const uint64_t*)hoff.p, (uint32_t*)hfill.p,
                                 (unsigned long long*)hk1.p);
  ALGAS_CUDA_TRY(cudaGetLastError());
  const uint64_t* offp = (const uint64_t*)hoff.p;
  size_t tmp = 0;
  ALGAS_CUDA_TRY(cub::DeviceSegmentedSort::SortKeys(nullptr, tmp, (const unsigned long long*)hk1.p,
                                                    (unsigned long long*)hk2.p, (int)acc, (int)n, offp, offp + 1));
  ALGAS_CUDA_TRY(cudaMalloc(&htmp.p, std::max<size_t>(tmp, 16)));
  ALGAS_CUDA_TRY(cub::DeviceSegmentedSort::SortKeys(htmp.p, tmp, (const unsigned long long*)hk1.p,
                                                    (unsigned long long*)hk2.p, (int)acc, (int)n, offp, offp + 1));
  rev_take_kernel<<<(unsigned)((n + 255) / 256), 256>>>((const unsigned long long*)hk2.p, offp, n, fan, rev);
  ALGAS_CUDA_TRY(cudaGetLastError());
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}

int algas_knn_refine(const float* data, int64_t n, int32_t dim, int32_t metric, int32_t k, int32_t fan_arg,
                     int32_t rounds, uint32_t* ids, float* dists) {
  const bool reverse = fan_arg < 0;  // R35: reverse neighbours joined too
  const int fan = reverse ? -fan_arg : fan_arg;
  if (!data || !ids || !dists || n < 1 || n >= (1LL << 31) || dim < 4 || dim % 4 != 0 || k < 1 || k > 1024 ||
      fan < 1 || fan > k || fan > (reverse ? 32 : 64) || rounds < 0 ||
      (metric != ALGAS_L2 && metric != ALGAS_IP && metric != ALGAS_COSINE))
    return set_error(ALGAS_EINVAL, "algas_knn_refine: bad arguments");
  if (rounds == 0) return ALGAS_OK;
  Dev hx, hxn, a_i, a_d, b_i, b_d;
  const float* X = nullptr;
  int rc;
  if ((rc = to_device(data, (size_t)n * dim * 4, hx, (const void**)&X))) return rc;
  int met = metric;
  if (metric == ALGAS_COSINE) {  // IP on unit-row copies (R29)
    ALGAS_CUDA_TRY(cudaMalloc(&hxn.p, (size_t)n * dim * 4));
    normalize_copy_kernel<<<(unsigned)((n + 7) / 8), 256>>>(reinterpret_cast<const float4*>(X), n, dim / 4,
                                                            reinterpret_cast<float4*>(hxn.p));
    ALGAS_CUDA_TRY(cudaGetLastError());
    X = (const float*)hxn.p;
    met = ALGAS_IP;
  }
  const size_t bytes = (size_t)n * k * 4;
  ALGAS_CUDA_TRY(cudaMalloc(&a_i.p, bytes));
  ALGAS_CUDA_TRY(cudaMalloc(&a_d.p, bytes));
  ALGAS_CUDA_TRY(cudaMalloc(&b_i.p, bytes));
  ALGAS_CUDA_TRY(cudaMalloc(&b_d.p, bytes));
  ALGAS_CUDA_TRY(cudaMemcpy(a_i.p, ids, bytes, cudaMemcpyDefault));
  ALGAS_CUDA_TRY(cudaMemcpy(a_d.p, dists, bytes, cudaMemcpyDefault));
  Dev hrev;
  if (reverse) ALGAS_CUDA_TRY(cudaMalloc(&hrev.p, (size_t)n * fan * 4));
  for (int r = 0; r < rounds; ++r) {  // Jacobi rounds (R33 / R35)
    if (reverse && (rc = build_rev_lists((const uint32_t*)a_i.p, n, k, fan, (uint32_t*)hrev.p))) return rc;
    if ((rc = launch_refine(X, dim, met, n, k, fan, (const uint32_t*)a_i.p, (const float*)a_d.p,
                            reverse ? (const uint32_t*)hrev.p : nullptr, (uint32_t*)b_i.p, (float*)b_d.p)))
      return rc;
    std::swap(a_i.p, b_i.p);
    std::swap(a_d.p, b_d.p);
  }
  ALGAS_CUDA_TRY(cudaMemcpy(ids, a_i.p, bytes, cudaMemcpyDefault));
  ALGAS_CUDA_TRY(cudaMemcpy(dists, a_d.p, bytes, cudaMemcpyDefault));
  return ALGAS_OK;
}

int algas_build_graph_partitioned(const float* data, int64_t n, int32_t dim, int32_t metric, int32_t knn_degree,
                                  int32_t degree, int32_t prune, int32_t n_clusters, int32_t overlap,
                                  int32_t refine_fan, int32_t refine_rounds, uint32_t* out_graph) {
  if (!data || !out_graph || n < 2 || knn_degree < degree || degree < 1 || refine_rounds < 0)
    return set_error(ALGAS_EINVAL, "algas_build_graph_partitioned: bad arguments");
  const int K = (int)std::min<int64_t>(knn_degree, n - 1);
  Dev guard_k, guard_d;
  ALGAS_CUDA_TRY(cudaMalloc(&guard_k.p, (size_t)n * K * 4));
  ALGAS_CUDA_TRY(cudaMalloc(&guard_d.p, (size_t)n * K * 4));
  int rc = algas_knn_partitioned(data, n, dim, metric, K, n_clusters, overlap, (uint32_t*)guard_k.p,
                                 (float*)guard_d.p);
  if (rc) return rc;
  if (refine_rounds > 0) {
    // refine_fan < 0: R35 rounds (reverse neighbours joined too), fan |refine_fan|
    const bool rv = refine_fan < 0;
    const int f = std::min(std::max(rv ? -refine_fan : refine_fan, 1), std::min(K, rv ? 32 : 64));
    if ((rc = algas_knn_refine(data, n, dim, metric, K, rv ? -f : f, refine_rounds, (uint32_t*)guard_k.p,
                               (float*)guard_d.p)))
      return rc;
  }
  // rows the partition left short (clusters of <= K points) are completed by
  // the exact kNN of those rows over the whole set (the prune needs full rows)
  std::vector<uint32_t> hk((size_t)n * K);
  ALGAS_CUDA_TRY(cudaMemcpy(hk.data(), guard_k.p, hk.size() * 4, cudaMemcpyDeviceToHost));
  std::vector<uint32_t> shortr;
  for (int64_t i = 0; i < n; ++i)
    if (hk[(size_t)i * K + K - 1] == kSentinel) shortr.push_back((uint32_t)i);
  if (!shortr.empty()) {
    Dev hx, hs, hq;
    const float* X = nullptr;
    if ((rc = to_device(data, (size_t)n * dim * 4, hx, (const void**)&X))) return rc;
    const int64_t ns = (int64_t)shortr.size();
    const int K1 = (int)std::min<int64_t>(K + 1, n);
    ALGAS_CUDA_TRY(cudaMalloc(&hs.p, (size_t)ns * 4));
    ALGAS_CUDA_TRY(cudaMemcpy(hs.p, shortr.data(), (size_t)ns * 4, cudaMemcpyHostToDevice));
    ALGAS_CUDA_TRY(cudaMalloc(&hq.p, (size_t)ns * dim * 4));
    if ((rc = gather_rows(X, (const uint32_t*)hs.p, ns, dim, (float*)hq.p))) return rc;
    std::vector<uint32_t> ei((size_t)ns * K1);
    std::vector<float> ed((size_t)ns * K1);
    if ((rc = algas_knn(X, n, (const float*)hq.p, ns, dim, metric, K1, -1, ei.data(), ed.data()))) return rc;
    for (int64_t t = 0; t < ns; ++t) {
      uint32_t* row = hk.data() + (size_t)shortr[t] * K;
      int o = 0;
      for (int e = 0; e < K1 && o < K; ++e)
        if (ei[(size_t)t * K1 + e] != shortr[t]) row[o++] = ei[(size_t)t * K1 + e];
    }
    ALGAS_CUDA_TRY(cudaMemcpy(guard_k.p, hk.data(), hk.size() * 4, cudaMemcpyHostToDevice));
  }
  return graph_from_knn((const uint32_t*)guard_k.p, n, K, degree, prune, out_graph);
}

}  // extern "C"
