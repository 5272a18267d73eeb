// microbench_wave.cu -- latency of one search-step "wave" on B200: a CTA
// gathers M random 512-B rows (a 1 GB table, L2 flushed), every load of the
// wave issued before any use (volatile asm for loads AND uses, so ptxas
// cannot interleave them), then __syncthreads.  This is the distance phase
// of one search step; the per-step cost is the wave's completion time, i.e.
// the tail latency of M concurrent random row reads.
//
// Columns: threads per CTA, rows per wave, CTAs (32 = batch-32 slots, 148 =
// one per SM), cycles per wave (mean over CTAs), implied GB/s per SM.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mbv scripts/microbench_wave.cu && /tmp/mbv
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

__device__ __forceinline__ float4 ldv(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ float vadd(float a, float4 b) {
  float r;
  asm volatile("add.f32 %0, %1, %2;\n\tadd.f32 %0, %0, %3;\n\tadd.f32 %0, %0, %4;\n\tadd.f32 %0, %0, %5;"
               : "=f"(r)
               : "f"(a), "f"(b.x), "f"(b.y), "f"(b.z), "f"(b.w));
  return r;
}

// TL = 8 lanes per row, CPL = 4 chunks of 16 B per lane (as the search kernel
// at dim 128); each thread holds RB rows' chunks in flight.
template <int NT, int RB>
__global__ void __launch_bounds__(NT) wave(const float4* __restrict__ data, const uint32_t* __restrict__ ids, int waves,
                                           int mvalid, unsigned long long* cyc, float* sink) {
  constexpr int M = NT / 8 * RB;  // rows per wave
  __shared__ uint32_t sid[M];
  const int tid = threadIdx.x, team = tid / 8, tl = tid % 8;
  float acc = 0.f;
  unsigned long long total = 0;
  for (int w = 0; w < waves; ++w) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * waves + w) * M;
    for (int i = tid; i < M; i += NT) sid[i] = rid[i];
    __syncthreads();
    long long t0 = clock64();
    float4 v[RB][4];
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      const float4* row = data + (size_t)sid[b * (NT / 8) + team] * 32;
#pragma unroll
      for (int c = 0; c < 4; ++c)  // predicated as in the search kernel (keeps ptxas from interleaving)
        v[b][c] = (b * (NT / 8) + team < mvalid) ? ldv(row + tl + 8 * c) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncwarp();  // as in the search kernel: all loads of the wave before any use
    float a[RB];
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      a[b] = 0.f;
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const float4 x = v[b][c];
        a[b] = fmaf(x.x, x.x, a[b]); a[b] = fmaf(x.y, x.y, a[b]); a[b] = fmaf(x.z, x.z, a[b]); a[b] = fmaf(x.w, x.w, a[b]);
      }
    }
#pragma unroll
    for (int o = 4; o > 0; o >>= 1)
#pragma unroll
      for (int b = 0; b < RB; ++b) a[b] += __shfl_xor_sync(0xffffffffu, a[b], o);
#pragma unroll
    for (int b = 0; b < RB; ++b) acc += a[b];
    __syncthreads();
    total += (unsigned long long)(clock64() - t0);
  }
  if (tid == 0) cyc[blockIdx.x] = total / waves;
  if (acc == 12345.f) sink[0] = acc;
}

static uint64_t rs = 88172645463325252ull;
static uint32_t rnd() { rs ^= rs << 13; rs ^= rs >> 7; rs ^= rs << 17; return (uint32_t)rs; }

template <int NT, int RB>
void run(const float4* data, void* flush, float* sink, unsigned long long* cyc, int grid) {
  constexpr int M = NT / 8 * RB;
  const int waves = 64;
  std::vector<uint32_t> h((size_t)grid * waves * M);
  for (auto& x : h) x = rnd() % (1u << 21);
  uint32_t* ids;
  cudaMalloc(&ids, h.size() * 4);
  cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMemset(flush, 1, 512u << 20);
  wave<NT, RB><<<grid, NT>>>(data, ids, waves, M, cyc, sink);
  cudaDeviceSynchronize();
  std::vector<unsigned long long> c(grid);
  cudaMemcpy(c.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
  double mean = 0;
  for (auto x : c) mean += x;
  mean /= grid;
  printf("threads=%4d rows/wave=%4d ctas=%3d  %7.0f cyc/wave  %6.1f GB/s/SM  %s\n", NT, M, grid, mean,
         M * 512.0 / (mean / 1.965e9) / 1e9, cudaGetErrorString(cudaGetLastError()));
  cudaFree(ids);
}

int main() {
  float4* data;
  cudaMalloc(&data, 1ull << 30);
  cudaMemset(data, 0, 1ull << 30);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  float* sink;
  cudaMalloc(&sink, 4);
  unsigned long long* cyc;
  cudaMalloc(&cyc, 148 * 8);
  for (int grid : {32, 148}) {
    run<256, 1>(data, flush, sink, cyc, grid);
    run<256, 2>(data, flush, sink, cyc, grid);
    run<256, 4>(data, flush, sink, cyc, grid);
    run<512, 1>(data, flush, sink, cyc, grid);
    run<512, 2>(data, flush, sink, cyc, grid);
    run<512, 4>(data, flush, sink, cyc, grid);
    run<1024, 1>(data, flush, sink, cyc, grid);
    run<1024, 2>(data, flush, sink, cyc, grid);
  }
  return 0;
}
