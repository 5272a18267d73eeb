// microbench_warps.cu -- per-SM random 512-B row gather rate on B200 as a
// function of warps per SM, rows in flight per warp and load flavour.
// One CTA per SM (grid 148); rows uniform over a 1 GB table; L2 flushed.
// Finding this answers: is a search CTA's gather rate bound per warp (more
// warps per query help) or per SM (more SMs per query help)?
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mbw scripts/microbench_warps.cu && /tmp/mbw
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

template <int FL>
__device__ __forceinline__ float4 ld(const float4* p) {
  float4 r;
  if (FL == 0) asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else if (FL == 1) asm volatile("ld.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else if (FL == 2) asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}

// TL lanes per row, each lane 4 chunks of 16 B (TL=8: one 128-B line per lane group per chunk)
template <int RPW, int FL, int TL>
__global__ void __launch_bounds__(1024) gather(const float4* __restrict__ data, const uint32_t* __restrict__ ids,
                                               int rows_per_cta, int rounds, float* sink) {
  __shared__ uint32_t sid[4096];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, NW = blockDim.x / 32;
  constexpr int RPI = 32 / TL;          // rows per load instruction
  constexpr int CPL = 32 / TL;          // 16-B chunks per lane (row = 32 chunks)
  float acc = 0.f;
  for (int r = 0; r < rounds; ++r) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * rounds + r) * rows_per_cta;
    __syncthreads();
    for (int i = tid; i < rows_per_cta; i += blockDim.x) sid[i] = rid[i];
    __syncthreads();
    for (int i0 = warp * RPW; i0 < rows_per_cta; i0 += NW * RPW) {
      float4 v[RPW / RPI][CPL];
#pragma unroll
      for (int j = 0; j < RPW / RPI; ++j)
#pragma unroll
        for (int c = 0; c < CPL; ++c)
          v[j][c] = ld<FL>(data + (size_t)sid[i0 + j * RPI + lane / TL] * 32 + (lane % TL) + c * TL);
      __syncwarp();
#pragma unroll
      for (int j = 0; j < RPW / RPI; ++j)
#pragma unroll
        for (int c = 0; c < CPL; ++c) acc += v[j][c].x + v[j][c].y + v[j][c].z + v[j][c].w;
    }
  }
  if (acc == 12345.f) sink[0] = acc;
}

static uint64_t rs = 88172645463325252ull;
static uint32_t rnd() { rs ^= rs << 13; rs ^= rs >> 7; rs ^= rs << 17; return (uint32_t)rs; }

template <int RPW, int FL, int TL>
void run(const float4* data, const uint32_t* ids, void* flush, float* sink, int nt, int rows, int rounds, int grid) {
  gather<RPW, FL, TL><<<grid, nt>>>(data, ids + (size_t)grid * rounds * rows, rows, rounds, sink);
  cudaMemset(flush, 1, 512u << 20);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  gather<RPW, FL, TL><<<grid, nt>>>(data, ids, rows, rounds, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  const char* fl[4] = {"nc.noalloc", "plain", "cg", "nc"};
  double gbs = (double)grid * rounds * rows * 512 / (ms * 1e-3) / 1e9;
  printf("fl=%-10s TL=%2d warps=%2d RPW=%2d grid=%3d  %7.1f GB/s  %6.1f GB/s/SM  %s\n", fl[FL], TL, nt / 32, RPW, grid,
         gbs, gbs / 148 * (grid >= 148 ? 1 : 148.0 / grid), cudaGetErrorString(cudaGetLastError()));
}

int main() {
  float4* data;
  cudaMalloc(&data, 1ull << 30);
  cudaMemset(data, 0, 1ull << 30);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  float* sink;
  cudaMalloc(&sink, 4);
  const int rows = 4096, rounds = 4, grid = 148;
  std::vector<uint32_t> h((size_t)2 * grid * rounds * rows);
  for (auto& x : h) x = rnd() % (1u << 21);
  uint32_t* ids;
  cudaMalloc(&ids, h.size() * 4);
  cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  for (int nt : {128, 256, 512, 1024}) {
    run<4, 0, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<8, 0, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<16, 0, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<8, 0, 8>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<16, 0, 8>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<8, 1, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<8, 2, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
    run<8, 3, 32>(data, ids, flush, sink, nt, rows, rounds, grid);
  }
  // a single SM (latency-bound regime of one query)
  for (int nt : {256, 1024}) {
    run<8, 0, 32>(data, ids, flush, sink, nt, rows, rounds, 1);
    run<16, 0, 8>(data, ids, flush, sink, nt, rows, rounds, 1);
  }
  return 0;
}
