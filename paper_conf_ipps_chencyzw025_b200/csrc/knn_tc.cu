// knn_tc.cu -- the graph build's dense contraction on the 5th-generation tensor
// cores, hand-written for sm_100a (tcgen05 + TMEM; supporting code, not the
// search hot path).
//
// D[q][x] = sum_k Q[q][k] X[x][k] for a block of queries against a block of
// base points -- the q.x term of |q|^2 + |x|^2 - 2 q.x that the tensor-core
// screen of algas_knn ranks candidates by (the exact re-rank and the
// certificate in knn.cu make the final kNN exact regardless of this
// product's rounding).  3xTF32: every operand is split into a TF32 "hi"
// part and the remainder "lo" (split_tf32_kernel); D accumulates
// hi.hi + lo(X).hi(Q) + hi(X).lo(Q) in fp32 in TMEM, the same product terms
// the cuBLAS path computes (error bound: knn.cu, eps_c).
//
// One CTA = a 128 (queries) x 256 (base points) tile, 128 threads:
//   * per K block of 32 dims (two stage buffers: block kb+1 is staged while
//     the tensor core runs block kb), all threads stage the four operand tiles
//     (Q hi/lo 128 x 32, X hi/lo 256 x 32) into shared memory in the
//     canonical K-major no-swizzle UMMA layout (8-row x 16-byte core
//     matrices: core (g, c) of row group g and 16-byte K chunk c at
//     g * 1024 + c * 128 bytes; LBO = 128 B between the two K chunks of one
//     MMA, SBO = 1024 B between 8-row groups);
//   * thread 0 issues 4 K steps x 3 tcgen05.mma.cta_group::1.kind::tf32
//     (M = 128, N = 256, K = 8) into one TMEM accumulator (128 lanes x 256
//     fp32 columns) and commits them to an mbarrier the CTA waits on before
//     the tiles are overwritten;
//   * epilogue: warp w reads TMEM lanes 32w..32w+31 (its query rows) with
//     tcgen05.ld.32x32b.x32 (32 columns per load) and writes the rows of D.
#include <cstdint>

#include "internal.h"

namespace algas {

namespace {

constexpr int TC_M = 128, TC_N = 256, TC_K = 32;  // tile rows (queries), cols (base), dims per block
constexpr int TC_THREADS = 128;
constexpr uint32_t kTmemCols = 256;

// canonical K-major, no-swizzle tile of R rows x 32 fp32: byte offset of the
// 16-byte chunk c (4 values) of row r
__device__ __forceinline__ uint32_t tile_off(int r, int c) { return (uint32_t)((r >> 3) * 1024 + c * 128 + (r & 7) * 16); }

// shared-memory matrix descriptor (SM100 UMMA): start >> 4 [0,14), LBO >> 4
// [16,30), SBO >> 4 [32,46), version 1 [46,48), swizzle none (0) [61,64)
__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}
// instruction descriptor, kind::tf32: D f32 [4,6) = 1, A/B tf32 [7,10) /
// [10,13) = 2, both K-major, N >> 3 at [17,23), M >> 4 at [24,29)
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(TC_N >> 3) << 17) |
                            ((uint32_t)(TC_M >> 4) << 24);

__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}"
      ::"r"(tmem_d), "l"(a), "l"(b), "r"(kIdesc), "r"(accumulate)
      : "memory");
}

}  // namespace

constexpr int kStageBytes = (TC_M + TC_N) * TC_K * 4 * 2;  // Q hi/lo + X hi/lo tiles of one K block: 96 KB

// stage K block k0 of the four operand tiles into buffer `buf`: 16-B
// cp.async (LDGSTS) per chunk into its canonical-layout slot, zero-filled
// past the matrix edges (src-size 0); nothing is waited for here -- a thread
// has all 48 of its chunk copies in flight (cp.async.commit_group after)
__device__ __forceinline__ void cp16_zfill(uint8_t* dst, const float* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(valid ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ void tc_stage(uint8_t* buf, const float* Qh, const float* Ql, int64_t qb, int64_t q0,
                                         const float* Xh, const float* Xl, int64_t nb, int64_t x0, int d, int k0,
                                         int tid) {
  uint8_t* a_hi = buf;
  uint8_t* a_lo = a_hi + TC_M * TC_K * 4;
  uint8_t* b_hi = a_lo + TC_M * TC_K * 4;
  uint8_t* b_lo = b_hi + TC_N * TC_K * 4;
#pragma unroll 8
  for (int t = tid; t < TC_M * (TC_K / 4); t += TC_THREADS) {
    const int r = t >> 3, c = t & 7;
    const bool ok = q0 + r < qb && k0 + c * 4 < d;
    const int64_t o = ok ? (q0 + r) * d + k0 + c * 4 : 0;
    cp16_zfill(a_hi + tile_off(r, c), Qh + o, ok);
    cp16_zfill(a_lo + tile_off(r, c), Ql + o, ok);
  }
#pragma unroll 8
  for (int t = tid; t < TC_N * (TC_K / 4); t += TC_THREADS) {
    const int r = t >> 3, c = t & 7;
    const bool ok = x0 + r < nb && k0 + c * 4 < d;
    const int64_t o = ok ? (x0 + r) * d + k0 + c * 4 : 0;
    cp16_zfill(b_hi + tile_off(r, c), Xh + o, ok);
    cp16_zfill(b_lo + tile_off(r, c), Xl + o, ok);
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
}

__global__ void __launch_bounds__(TC_THREADS, 1) tc_dot_kernel(const float* __restrict__ Qh, const float* __restrict__ Ql,
                                                               int64_t qb, const float* __restrict__ Xh,
                                                               const float* __restrict__ Xl, int64_t nb, int d,
                                                               float* __restrict__ D, int64_t ldD) {
  // two stage buffers: block kb+1 is staged while the tensor core runs block kb
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t mbar[2];
  __shared__ uint32_t tmem_base_sh;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int64_t q0 = (int64_t)blockIdx.y * TC_M, x0 = (int64_t)blockIdx.x * TC_N;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(kTmemCols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (tid == 0) {
    mbar_init(&mbar[0], 1);
    mbar_init(&mbar[1], 1);
    mbar_fence_init();
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tmem_base_sh;

  uint32_t ph0 = 0, ph1 = 0;  // parity of the next completion of mbar[0] / mbar[1]
  const int nkb = (d + TC_K - 1) / TC_K;
  tc_stage(sm, Qh, Ql, qb, q0, Xh, Xl, nb, x0, d, 0, tid);
  for (int kb = 0; kb < nkb; ++kb) {
    const int b = kb & 1;
    uint8_t* buf = sm + (size_t)b * kStageBytes;
    asm volatile("cp.async.wait_group 0;" ::: "memory");  // this thread's copies of block kb landed
    fence_proxy_async_smem();  // tile writes -> visible to the tensor core (async proxy)
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t a_hi = smem_u32(buf), a_lo = a_hi + TC_M * TC_K * 4;
      const uint32_t b_hi = a_lo + TC_M * TC_K * 4, b_lo = b_hi + TC_N * TC_K * 4;
      // 4 K steps of 8 (two 16-B chunks each) x 3 products
#pragma unroll
      for (int s = 0; s < TC_K / 8; ++s) {
        const uint32_t off = (uint32_t)s * 256;
        const uint64_t ah = smem_desc(a_hi + off, 128, 1024), al = smem_desc(a_lo + off, 128, 1024);
        const uint64_t bh = smem_desc(b_hi + off, 128, 1024), bl = smem_desc(b_lo + off, 128, 1024);
        mma_tf32(tmem, ah, bh, (kb | s) ? 1u : 0u);  // Q hi . X hi
        mma_tf32(tmem, ah, bl, 1u);                  // Q hi . X lo
        mma_tf32(tmem, al, bh, 1u);                  // Q lo . X hi
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                       smem_u32(&mbar[b]))
                   : "memory");
    }
    if (kb + 1 < nkb) {
      // the other buffer was last read by block kb-1's MMAs
      if (kb >= 1) {
        if (b == 0) { mbar_wait(&mbar[1], ph1); ph1 ^= 1u; }
        else        { mbar_wait(&mbar[0], ph0); ph0 ^= 1u; }
      }
      tc_stage(sm + (size_t)(b ^ 1) * kStageBytes, Qh, Ql, qb, q0, Xh, Xl, nb, x0, d, (kb + 1) * TC_K, tid);
    }
  }
  // the last block's commit covers every earlier MMA (they complete in order)
  if (((nkb - 1) & 1) == 0) mbar_wait(&mbar[0], ph0); else mbar_wait(&mbar[1], ph1);
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

  // ---- epilogue: TMEM lanes 32w.. of warp w = its query rows; 32 columns per load
  const int64_t row = q0 + warp * 32 + lane;
  const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16);
  for (int c0 = 0; c0 < TC_N; c0 += 32) {
    uint32_t v[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),
          "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),
          "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),
          "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr + (uint32_t)c0));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    if (row < qb) {
      float* out = D + row * ldD + x0 + c0;
      if (x0 + c0 + 32 <= nb) {
#pragma unroll
        for (int j = 0; j < 32; j += 4)
          *reinterpret_cast<float4*>(out + j) = make_float4(__uint_as_float(v[j]), __uint_as_float(v[j + 1]),
                                                            __uint_as_float(v[j + 2]), __uint_as_float(v[j + 3]));
      } else {
#pragma unroll
        for (int j = 0; j < 32; ++j)
          if (x0 + c0 + j < nb) out[j] = __uint_as_float(v[j]);
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
}

// D (qb x nb, row stride ldD) = Q . X^T in 3xTF32 on the tensor cores.
// Q/X hi/lo: row-major, d columns (d % 4 == 0), 16-B aligned.
int tc_dot_3xtf32(const float* Qh, const float* Ql, int64_t qb, const float* Xh, const float* Xl, int64_t nb, int d,
                  float* D, int64_t ldD, cudaStream_t st) {
  if (qb <= 0 || nb <= 0) return ALGAS_OK;
  if (d % 4 != 0 || ldD % 4 != 0) return set_error(ALGAS_EINVAL, "tc_dot: d and ldD must be multiples of 4");
  const int smem = 2 * kStageBytes;  // two stages of 96 KB
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(tc_dot_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  const dim3 grid((unsigned)((nb + TC_N - 1) / TC_N), (unsigned)((qb + TC_M - 1) / TC_M));
  tc_dot_kernel<<<grid, TC_THREADS, smem, st>>>(Qh, Ql, qb, Xh, Xl, nb, d, D, ldD);
  ALGAS_CUDA_TRY(cudaGetLastError());
  return ALGAS_OK;
}

}  // namespace algas
