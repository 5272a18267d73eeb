// microbench_ldg.cu -- latency of one "pass" of random 512-B row gathers
// (each warp loads R rows with one 16-B load per lane per row, all issued
// before use) for different load flavours: ld.global (ca), ld.global.cg
// (L2 only), ld.global.nc (read-only path), ld.global.nc.L1::no_allocate.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/mbldg scripts/microbench_ldg.cu && scripts/mbldg
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

template <int F>
__device__ __forceinline__ float4 ld(const float4* p) {
  float4 r;
  if (F == 0) asm volatile("ld.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  if (F == 1) asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  if (F == 2) asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  if (F == 3)
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
                 : "l"(p));
  if (F == 4) asm volatile("ld.global.cv.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}

template <int F, int R>
__global__ void pass(const float4* __restrict__ data, const uint32_t* __restrict__ ids, int rounds,
                     unsigned long long* cyc, float* sink) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, NW = blockDim.x / 32;
  float acc = 0.f;
  unsigned long long tot = 0;
  for (int r = 0; r < rounds; ++r) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * rounds + r) * NW * R + warp * R;
    uint32_t id[R];
#pragma unroll
    for (int j = 0; j < R; ++j) id[j] = rid[j];
    __syncwarp();
    long long t0 = clock64();
    float4 v[R];
#pragma unroll
    for (int j = 0; j < R; ++j) v[j] = ld<F>(data + (size_t)id[j] * 32 + lane);
    __syncwarp();
#pragma unroll
    for (int j = 0; j < R; ++j) acc += v[j].x + v[j].y + v[j].z + v[j].w;
    __syncwarp();
    long long t1 = clock64();
    tot += (unsigned long long)(t1 - t0);
    __syncthreads();
  }
  if (lane == 0) cyc[blockIdx.x * NW + warp] = tot;
  if (acc == 1234.5f) sink[0] = acc;
}

int main() {
  const size_t rows = (1u << 30) / 512;
  float4* data;
  cudaMalloc(&data, rows * 512);
  cudaMemset(data, 0, rows * 512);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  float* sink;
  cudaMalloc(&sink, 4);
  unsigned long long* cyc;
  cudaMalloc(&cyc, 148 * 32 * 8);
  const int rounds = 50, NT = 256;
  const int grids[2] = {1, 148};
  std::vector<uint32_t> h((size_t)148 * rounds * 8 * 16 * 2);
  uint64_t s = 88172645463325252ull;
  for (auto& x : h) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; x = (uint32_t)(s % rows); }
  uint32_t* ids;
  cudaMalloc(&ids, h.size() * 4);
  cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  const char* nm[5] = {"ld.ca", "ld.cg", "ld.nc", "ld.nc.na", "ld.cv"};
  printf("flavour R grid  cycles/pass(avg over warps)\n");
#define RUN(F, R)                                                                                  \
  for (int g : grids) {                                                                            \
    pass<F, R><<<g, NT>>>(data, ids + h.size() / 2, rounds, cyc, sink);                            \
    cudaMemset(flush, F + R, 512u << 20);                                                          \
    pass<F, R><<<g, NT>>>(data, ids, rounds, cyc, sink);                                           \
    std::vector<unsigned long long> c(g * 8);                                                      \
    cudaMemcpy(c.data(), cyc, c.size() * 8, cudaMemcpyDeviceToHost);                               \
    double m = 0;                                                                                  \
    for (auto x : c) m += x;                                                                       \
    m /= c.size() * rounds;                                                                        \
    printf("%-9s %2d %4d %8.0f  %s\n", nm[F], R, g, m, cudaGetErrorString(cudaGetLastError()));    \
  }
  RUN(0, 1) RUN(0, 4) RUN(0, 8) RUN(0, 16)
  RUN(1, 1) RUN(1, 4) RUN(1, 8) RUN(1, 16)
  RUN(2, 1) RUN(2, 4) RUN(2, 8) RUN(2, 16)
  RUN(3, 1) RUN(3, 4) RUN(3, 8) RUN(3, 16)
  RUN(4, 1) RUN(4, 8)
  return 0;
}
