// build_part.cu -- GPU kernels of the partitioned graph build (SURVEY §8f f4,
// DESIGN.md R30 / R33; supporting code, not the search hot path):
//
//  cluster_knn_kernel : exact kNN inside every cluster of the partition, all
//                       clusters in ONE launch (a CTA = 64 member rows of one
//                       cluster against all members of that cluster, fp32
//                       direct-form distance tiles, per-row running top-k in
//                       shared memory) -- replaces one algas_knn call per
//                       cluster (R30 step 4)
//  merge_lists_kernel : per point, its `overlap` cluster lists merged by
//                       (dist, id), repeated ids dropped, first k (R30 step 5)
//  refine_kernel      : one neighbour-of-neighbour refinement round (R33):
//                       candidates = the first `fan` entries of the lists of
//                       a point's first `fan` neighbours, scored and merged
//                       into its list (a Jacobi round: reads the previous
//                       round's lists, writes new ones)
//
// Keys are the search kernel's u64 (orderable dist << 32 | id << 1), so every
// merge is by (dist, id) (R4).  Nothing here is shared with oracle/.
#include <cstdint>
#include <vector>

#include "internal.h"

namespace algas {

// sorted-block (one key per lane, ascending across lanes, kKeyMax padded)
// insertion into a sorted shared-memory list of k keys, keeping the first k
// (rank merge: a block key lands at lane + #list keys below it, a list key at
// its index + #block keys below it; keys are unique).  tmp: k keys scratch.
__device__ __forceinline__ int lanes_below(uint64_t blk, uint64_t x) {
  // # of block keys < x (the block is sorted across lanes): branchless
  // lower bound over the 32 lanes with shuffles
  int c = 0;
#pragma unroll
  for (int s = 16; s >= 1; s >>= 1) {
    const uint64_t v = __shfl_sync(0xffffffffu, blk, c + s - 1);
    if (v < x) c += s;
  }
  const uint64_t v = __shfl_sync(0xffffffffu, blk, c);
  return c + (v < x ? 1 : 0);
}
__device__ __forceinline__ void warp_insert_block(uint64_t* list, uint64_t* tmp, int k, uint64_t blk, int lane) {
  if (blk != kKeyMax) {
    const int pos = lane + lower_bound_u64(list, k, blk);
    if (pos < k) tmp[pos] = blk;
  }
  for (int i0 = 0; i0 < k; i0 += 32) {  // every lane takes part in the shuffles
    const int i = i0 + lane;
    const uint64_t x = i < k ? list[i] : kKeyMax;
    const int pos = i + lanes_below(blk, x);
    if (i < k && pos < k) tmp[pos] = x;
  }
  __syncwarp();
  for (int i = lane; i < k; i += 32) list[i] = tmp[i];
  __syncwarp();
}
// filter a block of candidate keys against the list's k-th key, sort the
// survivors and insert them (no-op when none can enter)
__device__ __forceinline__ void warp_offer(uint64_t* list, uint64_t* tmp, int k, uint64_t key, int lane) {
  const uint64_t thr = list[k - 1];
  const bool c = key < thr;
  if (__ballot_sync(0xffffffffu, c) == 0u) return;
  const uint64_t blk = warp_bitonic_sort32(c ? key : kKeyMax, lane);
  warp_insert_block(list, tmp, k, blk, lane);
}

// ------------------------------------------------------------------ cluster kNN (R30 step 4)
constexpr int CQ = 64, CX = 64, CK = 32;  // rows per CTA, member columns per tile, dims per stage
constexpr int kPartMaxK = 128;


template <int METRIC>
__global__ void __launch_bounds__(256) cluster_knn_kernel(const float* __restrict__ X, int d,
                                                          const uint32_t* __restrict__ mem,
                                                          const int64_t* __restrict__ start,
                                                          const ClusterBlock* __restrict__ blocks, int k,
                                                          uint64_t* __restrict__ out) {
  extern __shared__ __align__(16) uint8_t sm[];
  float* Qs = reinterpret_cast<float*>(sm);             // [CK][CQ]
  float* Xs = Qs + CK * CQ;                             // [CK][CX]
  float* D = Xs + CK * CX;                              // [CQ][CX + 1]
  uint32_t* xid = reinterpret_cast<uint32_t*>(D + CQ * (CX + 1));  // [CX]
  uint32_t* qid = xid + CX;                             // [CQ]
  uint64_t* lists = reinterpret_cast<uint64_t*>(qid + CQ);         // [CQ][k]
  uint64_t* tmps = lists + (size_t)CQ * k;              // [8 warps][k]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const ClusterBlock b = blocks[blockIdx.x];
  const int64_t s0 = start[b.cluster], sj = start[b.cluster + 1] - s0;
  const int rows = (int)(sj - b.row0 < CQ ? sj - b.row0 : CQ);
  for (int i = tid; i < CQ * k; i += 256) lists[i] = kKeyMax;
  for (int r = tid; r < CQ; r += 256) qid[r] = r < rows ? mem[s0 + b.row0 + r] : kSentinel;
  const int tx = tid & 15, ty = tid >> 4;
  uint64_t* tmp = tmps + (size_t)warp * k;
  for (int64_t c0 = 0; c0 < sj; c0 += CX) {
    const int cols = (int)(sj - c0 < CX ? sj - c0 : CX);
    __syncthreads();
    for (int c = tid; c < CX; c += 256) xid[c] = c < cols ? mem[s0 + c0 + c] : kSentinel;
    float acc[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
    for (int k0 = 0; k0 < d; k0 += CK) {
      __syncthreads();
      // 64 rows x 32 dims of each operand = 512 float4; 256 threads x 2 each
      for (int t = tid; t < CQ * CK / 4; t += 256) {
        const int r = t >> 3, c4 = (t & 7) * 4;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f), u = v;
        if (r < rows && k0 + c4 < d) v = *reinterpret_cast<const float4*>(X + (int64_t)qid[r] * d + k0 + c4);
        if (r < cols && k0 + c4 < d) u = *reinterpret_cast<const float4*>(X + (int64_t)xid[r] * d + k0 + c4);
        Qs[(c4 + 0) * CQ + r] = v.x; Qs[(c4 + 1) * CQ + r] = v.y; Qs[(c4 + 2) * CQ + r] = v.z; Qs[(c4 + 3) * CQ + r] = v.w;
        Xs[(c4 + 0) * CX + r] = u.x; Xs[(c4 + 1) * CX + r] = u.y; Xs[(c4 + 2) * CX + r] = u.z; Xs[(c4 + 3) * CX + r] = u.w;
      }
      __syncthreads();
      const int kk_end = min(CK, d - k0);
      for (int kk = 0; kk < kk_end; ++kk) {
        const float4 a = *reinterpret_cast<const float4*>(Qs + kk * CQ + ty * 4);
        const float4 bb = *reinterpret_cast<const float4*>(Xs + kk * CX + tx * 4);
        const float av[4] = {a.x, a.y, a.z, a.w}, bv[4] = {bb.x, bb.y, bb.z, bb.w};
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            if (METRIC == kL2) {
              const float t = av[i] - bv[j];
              acc[i][j] = fmaf(t, t, acc[i][j]);
            } else {
              acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
            }
          }
      }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) D[(ty * 4 + i) * (CX + 1) + tx * 4 + j] = METRIC == kL2 ? acc[i][j] : -acc[i][j];
    __syncthreads();
    // running top-k: warp w owns rows w, w+8, ...; two 32-column blocks per row
    for (int r = warp; r < rows; r += 8) {
      uint64_t* L = lists + (size_t)r * k;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int c = h * 32 + lane;
        uint64_t key = kKeyMax;
        if (c < cols && xid[c] != qid[r]) key = make_key(D[r * (CX + 1) + c], xid[c]);  // self excluded
        warp_offer(L, tmp, k, key, lane);
      }
    }
  }
  __syncthreads();
  for (int i = tid; i < rows * k; i += 256) out[(s0 + b.row0) * k + i] = lists[i];
}

// ------------------------------------------------------------------ per-point merge (R30 step 5)
// warp per point: its c cluster lists (sorted, each k keys) merged; equal
// keys are the same id scored twice (identical arithmetic in both clusters),
// so dropping repeats keeps the first copy; first k decoded into ids/dists.
__global__ void __launch_bounds__(128) merge_lists_kernel(const uint64_t* __restrict__ lists,
                                                          const uint32_t* __restrict__ slot_of, int64_t n, int c,
                                                          int k, uint32_t* __restrict__ out_ids,
                                                          float* __restrict__ out_d) {
  extern __shared__ __align__(16) uint8_t sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t* acc = reinterpret_cast<uint64_t*>(sm) + (size_t)warp * 3 * k;  // [k] running result
  uint64_t* tmp = acc + k;                                                 // [2k] merged
  const int64_t i = (int64_t)blockIdx.x * 4 + warp;
  if (i >= n) return;
  const uint64_t* l0 = lists + (size_t)slot_of[i * c] * k;
  for (int e = lane; e < k; e += 32) acc[e] = l0[e];
  __syncwarp();
  for (int r = 1; r < c; ++r) {
    const uint64_t* lb = lists + (size_t)slot_of[i * c + r] * k;
    // rank merge of acc (A) and lb (B) into tmp[0..2k): A keys first among equals
    for (int e = lane; e < k; e += 32) {
      const uint64_t a = acc[e], bk = lb[e];
      tmp[e + lower_bound_u64(lb, k, a)] = a;                 // # B keys < a
      int ub = 0, hi = k;                                      // # A keys <= b
      while (ub < hi) {
        const int mid = (ub + hi) >> 1;
        if (acc[mid] <= bk) ub = mid + 1; else hi = mid;
      }
      tmp[e + ub] = bk;
    }
    __syncwarp();
    // drop repeats (a repeated finite key), keep the first k
    int out = 0;
    for (int base = 0; base < 2 * k && out < k; base += 32) {
      const int t = base + lane;
      const uint64_t x = t < 2 * k ? tmp[t] : kKeyMax;
      const bool keep = t < 2 * k && (x == kKeyMax || t == 0 || tmp[t - 1] != x);
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      const int pos = out + __popc(m & ((1u << lane) - 1u));
      if (keep && pos < k) acc[pos] = x;
      out += __popc(m);
    }
    __syncwarp();
  }
  for (int e = lane; e < k; e += 32) {
    const uint64_t x = acc[e];
    out_ids[i * k + e] = x == kKeyMax ? kSentinel : key_id(x);
    out_d[i * k + e] = x == kKeyMax ? __int_as_float(0x7f800000) : key_dist(x);
  }
}

// ------------------------------------------------------------------ refinement round (R33)
// warp per point p (4 per CTA).  Shared memory per warp: the list (k keys),
// merge scratch (k), a visited hash (2^hb u32) and the candidate ids (fan^2).
template <int METRIC>
__global__ void __launch_bounds__(128) refine_kernel(const float4* __restrict__ X, int d4, int64_t n, int k, int fan,
                                                     int hb, int per_warp, const uint32_t* __restrict__ in_ids,
                                                     const float* __restrict__ in_d, const uint32_t* __restrict__ rev,
                                                     uint32_t* __restrict__ out_ids, float* __restrict__ out_d) {
  extern __shared__ __align__(16) uint8_t sm[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // R33: fan x fan candidate slots; R35 (rev != nullptr): fan reverse
  // neighbours, then the lists of the fan forward and the fan reverse ones
  const int hcap = 1 << hb, ncand = rev ? fan + 2 * fan * fan : fan * fan;
  uint8_t* base = sm + (size_t)warp * per_warp;  // 16-B multiple
  uint64_t* L = reinterpret_cast<uint64_t*>(base);
  uint64_t* tmp = L + k;
  uint32_t* hash = reinterpret_cast<uint32_t*>(tmp + k);
  uint32_t* cid = hash + hcap;
  const int64_t p = (int64_t)blockIdx.x * 4 + warp;
  if (p >= n) return;
  for (int i = lane; i < hcap; i += 32) hash[i] = kHashEmpty;
  __syncwarp();
  if (lane == 0) (void)smem_visit(hash, hb, (uint32_t)p);
  __syncwarp();
  for (int e = lane; e < k; e += 32) {
    const uint32_t x = in_ids[p * k + e];
    L[e] = x == kSentinel ? kKeyMax : make_key(in_d[p * k + e], x);
    if (x != kSentinel) (void)smem_visit(hash, hb, x);
  }
  __syncwarp();
  // candidates: in[q][b] for q = in[p][a], a, b < fan, new to this point
  int m = 0;
  for (int t0 = 0; t0 < ncand; t0 += 32) {
    const int t = t0 + lane;
    uint32_t x = kSentinel;
    if (t < ncand) {
      if (rev == nullptr) {
        const uint32_t q = in_ids[p * k + t / fan];
        if (q != kSentinel) x = in_ids[(int64_t)q * k + t % fan];
      } else if (t < fan) {
        x = rev[p * fan + t];  // a reverse neighbour itself
      } else {
        const int u = t - fan, nr = u / fan;
        const uint32_t q = nr < fan ? in_ids[p * k + nr] : rev[p * fan + (nr - fan)];
        if (q != kSentinel) x = in_ids[(int64_t)q * k + u % fan];
      }
    }
    const bool keep = x != kSentinel && smem_visit(hash, hb, x) == kVisNew;
    const unsigned msk = __ballot_sync(0xffffffffu, keep);
    if (keep) cid[m + __popc(msk & ((1u << lane) - 1u))] = x;
    m += __popc(msk);
  }
  __syncwarp();
  // score them: teams of 8 lanes per row, 4 rows per team in flight
  for (int r0 = 0; r0 < m; r0 += 16) {
    const int team = lane >> 3, tl = lane & 7;
    float a[4] = {0.f, 0.f, 0.f, 0.f};
    for (int c = tl; c < d4; c += 8) {
      const float4 qv = X[p * d4 + c];
      float4 v[4];
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        const int r = r0 + b * 4 + team;
        v[b] = r < m ? X[(int64_t)cid[r] * d4 + c] : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        if (METRIC == kL2) {
          const float e0 = qv.x - v[b].x, e1 = qv.y - v[b].y, e2 = qv.z - v[b].z, e3 = qv.w - v[b].w;
          a[b] = fmaf(e0, e0, a[b]); a[b] = fmaf(e1, e1, a[b]); a[b] = fmaf(e2, e2, a[b]); a[b] = fmaf(e3, e3, a[b]);
        } else {
          a[b] = fmaf(qv.x, v[b].x, a[b]); a[b] = fmaf(qv.y, v[b].y, a[b]);
          a[b] = fmaf(qv.z, v[b].z, a[b]); a[b] = fmaf(qv.w, v[b].w, a[b]);
        }
      }
    }
#pragma unroll
    for (int b = 0; b < 4; ++b) {
#pragma unroll
      for (int o = 4; o > 0; o >>= 1) a[b] += __shfl_xor_sync(0xffffffffu, a[b], o);
    }
    // the 16 keys of this pass: lane tl == 0 of team t holds rows r0 + b*4 + t;
    // gather them into one block (lanes 0..15) and offer it to the list
    uint64_t key = kKeyMax;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
      const int src_team = lane & 3, src_b = lane >> 2;  // lane l < 16 takes row r0 + l
      const float v = __shfl_sync(0xffffffffu, a[b], src_team * 8);
      const int r = r0 + lane;
      if (lane < 16 && src_b == b && r < m) key = make_key(METRIC == kL2 ? v : -v, cid[r]);
    }
    warp_offer(L, tmp, k, key, lane);
  }
  for (int e = lane; e < k; e += 32) {
    const uint64_t x = L[e];
    out_ids[p * k + e] = x == kKeyMax ? kSentinel : key_id(x);
    out_d[p * k + e] = x == kKeyMax ? __int_as_float(0x7f800000) : key_dist(x);
  }
}

// ------------------------------------------------------------------ launchers
int launch_cluster_knn(const float* X, int d, int metric, const uint32_t* mem, const int64_t* start,
                       const std::vector<ClusterBlock>& blocks_h, int k, uint64_t* out) {
  if (k > kPartMaxK) return set_error(ALGAS_EINVAL, "cluster kNN: k %d > %d", k, kPartMaxK);
  ClusterBlock* db = nullptr;
  const size_t nb = blocks_h.size();
  if (nb == 0) return ALGAS_OK;
  ALGAS_CUDA_TRY(cudaMalloc(&db, nb * sizeof(ClusterBlock)));
  cudaError_t e = cudaMemcpy(db, blocks_h.data(), nb * sizeof(ClusterBlock), cudaMemcpyHostToDevice);
  const size_t smem = (size_t)(CK * CQ + CK * CX + CQ * (CX + 1)) * 4 + (CX + CQ) * 4 + (size_t)CQ * k * 8 +
                      (size_t)8 * k * 8;
  void* fn = metric == kL2 ? (void*)cluster_knn_kernel<kL2> : (void*)cluster_knn_kernel<kIP>;
  if (e == cudaSuccess) e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  for (size_t b0 = 0; e == cudaSuccess && b0 < nb; b0 += (1u << 30)) {
    const unsigned g = (unsigned)std::min<size_t>(nb - b0, 1u << 30);
    if (metric == kL2)
      cluster_knn_kernel<kL2><<<g, 256, smem>>>(X, d, mem, start, db + b0, k, out);
    else
      cluster_knn_kernel<kIP><<<g, 256, smem>>>(X, d, mem, start, db + b0, k, out);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  cudaFree(db);
  if (e != cudaSuccess) return set_error(ALGAS_ECUDA, "cluster kNN: %s", cudaGetErrorString(e));
  return ALGAS_OK;
}

int launch_merge_lists(const uint64_t* lists, const uint32_t* slot_of, int64_t n, int c, int k,
                       uint32_t* out_ids, float* out_d) {
  const size_t smem = (size_t)4 * 3 * k * 8;
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(merge_lists_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  merge_lists_kernel<<<(unsigned)((n + 3) / 4), 128, smem>>>(lists, slot_of, n, c, k, out_ids, out_d);
  ALGAS_CUDA_TRY(cudaGetLastError());
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}

int launch_refine(const float* X, int d, int metric, int64_t n, int k, int fan, const uint32_t* in_ids,
                  const float* in_d, const uint32_t* rev, uint32_t* out_ids, float* out_d) {
  const int ncand = rev ? fan + 2 * fan * fan : fan * fan;
  int hb = 6;
  while ((1 << hb) < 2 * (k + ncand + 1)) ++hb;
  const size_t per_warp = ((size_t)16 * k + ((size_t)4 << hb) + (size_t)4 * ncand + 15) & ~(size_t)15;
  const size_t smem = 4 * per_warp;
  void* fn = metric == kL2 ? (void*)refine_kernel<kL2> : (void*)refine_kernel<kIP>;
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const unsigned g = (unsigned)((n + 3) / 4);
  if (metric == kL2)
    refine_kernel<kL2><<<g, 128, smem>>>(reinterpret_cast<const float4*>(X), d / 4, n, k, fan, hb, (int)per_warp,
                                         in_ids, in_d, rev, out_ids, out_d);
  else
    refine_kernel<kIP><<<g, 128, smem>>>(reinterpret_cast<const float4*>(X), d / 4, n, k, fan, hb, (int)per_warp,
                                         in_ids, in_d, rev, out_ids, out_d);
  ALGAS_CUDA_TRY(cudaGetLastError());
  ALGAS_CUDA_TRY(cudaDeviceSynchronize());
  return ALGAS_OK;
}

}  // namespace algas
