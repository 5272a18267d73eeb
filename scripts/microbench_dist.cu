// microbench_dist.cu -- the search kernel's own distance step (dist_ldg from
// search_core.cuh) timed in isolation on B200: one CTA evaluates M random
// 512-B rows of a 1M x 128 table (L2 flushed before the run) per "wave",
// exactly as one search step does, then __syncthreads.  Reports cycles per
// wave for several CTA widths / wave sizes / grid sizes, which separates the
// DRAM tail latency of a wave from per-warp issue limits.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//      -I paper_conf_ipps_chencyzw025_b200/csrc -o /tmp/mbd scripts/microbench_dist.cu && /tmp/mbd
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "search_core.cuh"

using namespace algas;

template <int NT, int B>
__global__ void __launch_bounds__(NT) dist_wave(SearchCfg cfg, const uint32_t* __restrict__ ids, int M, int waves,
                                                unsigned long long* cyc, unsigned long long* sink) {
  __shared__ uint32_t newid[1024];
  __shared__ uint64_t newk[1024];
  __shared__ int nkeys;
  __shared__ float4 q[32];
  const int tid = threadIdx.x;
  if (tid < 32) q[tid] = make_float4(1.f, 2.f, 3.f, 4.f);
  __syncthreads();
  unsigned long long total = 0, s = 0;
  for (int w = 0; w < waves; ++w) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * waves + w) * M;
    for (int i = tid; i < M; i += NT) newid[i] = rid[i];
    if (tid == 0) nkeys = 0;
    __syncthreads();
    long long t0 = clock64();
    dist_ldg<NT, 8, 4, kL2, B>(cfg, q, M, 0, 1, ~0ull, newid, newk, &nkeys);
    __syncthreads();
    total += (unsigned long long)(clock64() - t0);
    s += newk[tid % M];
  }
  if (tid == 0) cyc[blockIdx.x] = total / waves;
  if (s == 12345) sink[0] = s;
}

static uint64_t rs = 88172645463325252ull;
static uint32_t rnd() { rs ^= rs << 13; rs ^= rs >> 7; rs ^= rs << 17; return (uint32_t)rs; }

template <int NT, int B = 0>
void run(const SearchCfg& cfg, void* flush, unsigned long long* sink, unsigned long long* cyc, int grid, int M,
         uint32_t span = 0) {
  const int waves = 64;
  std::vector<uint32_t> h((size_t)grid * waves * M);
  for (auto& x : h) x = rnd() % (span ? span : (uint32_t)cfg.n);
  if (span) {  // L2-resident: touch the rows once so every wave hits L2
    uint32_t* ids;
    cudaMalloc(&ids, h.size() * 4);
    cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    dist_wave<NT, B><<<grid, NT>>>(cfg, ids, M, waves, cyc, sink);
    cudaDeviceSynchronize();
    std::vector<unsigned long long> c(grid);
    cudaMemcpy(c.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
    double mean = 0;
    for (auto x : c) mean += x;
    printf("[L2-resident %u rows] ", span);
    mean /= grid;
    dist_wave<NT, B><<<grid, NT>>>(cfg, ids, M, waves, cyc, sink);
    cudaDeviceSynchronize();
    cudaMemcpy(c.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
    mean = 0;
    for (auto x : c) mean += x;
    mean /= grid;
    printf("threads=%4d B=%d rows/wave=%4d ctas=%3d  %7.0f cyc/wave\n", NT, B, M, grid, mean);
    cudaFree(ids);
    return;
  }
  uint32_t* ids;
  cudaMalloc(&ids, h.size() * 4);
  cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMemset(flush, 1, 512u << 20);
  dist_wave<NT, B><<<grid, NT>>>(cfg, ids, M, waves, cyc, sink);
  cudaDeviceSynchronize();
  std::vector<unsigned long long> c(grid);
  cudaMemcpy(c.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
  double mean = 0;
  for (auto x : c) mean += x;
  mean /= grid;
  printf("threads=%4d B=%d rows/wave=%4d ctas=%3d  %7.0f cyc/wave  %6.1f GB/s/SM  %s\n", NT, B, M, grid, mean,
         M * 512.0 / (mean / 1.965e9) / 1e9, cudaGetErrorString(cudaGetLastError()));
  cudaFree(ids);
}

int main(int argc, char** argv) {
  const size_t n = 1 << 21;  // 1 GB of 512-B rows
  float4* data;
  cudaMalloc(&data, n * 512);
  cudaMemset(data, 0, n * 512);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  unsigned long long *sink, *cyc;
  cudaMalloc(&sink, 8);
  cudaMalloc(&cyc, 148 * 8);
  SearchCfg cfg = {};
  cfg.data = data;
  cfg.n = n;
  cfg.d4 = 32;
  cfg.dp4 = 32;
  if (argc > 1) {  // one L2-resident configuration (for ncu): M rows, 1024 threads
    const int M = atoi(argv[1]);
    run<1024>(cfg, flush, sink, cyc, 32, M, 1u << 15);
    return 0;
  }
  for (int M : {8, 32, 128}) {
    run<256, 4>(cfg, flush, sink, cyc, 32, M, 1u << 15);
    run<256, 1>(cfg, flush, sink, cyc, 32, M, 1u << 15);
    run<1024, 1>(cfg, flush, sink, cyc, 32, M, 1u << 15);
  }
  for (int M : {32, 64, 128, 256}) {
    run<128, 4>(cfg, flush, sink, cyc, 32, M);
    run<256, 1>(cfg, flush, sink, cyc, 32, M);
    run<256, 2>(cfg, flush, sink, cyc, 32, M);
    run<256, 4>(cfg, flush, sink, cyc, 32, M);
    run<512, 1>(cfg, flush, sink, cyc, 32, M);
    run<512, 2>(cfg, flush, sink, cyc, 32, M);
    run<512, 4>(cfg, flush, sink, cyc, 32, M);
    run<1024, 1>(cfg, flush, sink, cyc, 32, M);
    run<1024, 2>(cfg, flush, sink, cyc, 32, M);
  }
  return 0;
}
