// microbench_gather.cu -- how fast can ONE CTA (one SM) gather M random
// 512-B rows from a 1 GB table into shared memory on B200?  Compares 16-B
// cp.async (LDGSTS), cp.async.bulk per row (TMA engine) and LDG.128 into
// registers, for several M and grid sizes.  Prints cycles per gather round.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mbg scripts/microbench_gather.cu && /tmp/mbg
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void __launch_bounds__(256) gather(const float4* __restrict__ data, const uint32_t* __restrict__ ids,
                                              int M, int rounds, int d4, unsigned long long* cyc, float* sink) {
  extern __shared__ __align__(128) float4 sm[];
  __shared__ __align__(8) uint64_t bar;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, NW = blockDim.x / 32;
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar)), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  uint32_t phase = 0;
  float acc = 0.f;
  long long t0 = clock64();
  for (int r = 0; r < rounds; ++r) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * rounds + r) * M;
    if (MODE == 0) {  // LDGSTS: warp per row, lane per 16 B
      for (int i = warp; i < M; i += NW) {
        const float4* src = data + (size_t)rid[i] * d4;
        for (int c = lane; c < d4; c += 32)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(sm + i * d4 + c)), "l"(src + c));
      }
      asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
      __syncthreads();
    } else if (MODE == 1) {  // bulk per row
      if (warp == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (lane == 0)
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bar)),
                       "r"(M * d4 * 16));
        __syncwarp();
        for (int i = lane; i < M; i += 32)
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                  smem_u32(sm + i * d4)),
              "l"(data + (size_t)rid[i] * d4), "r"(d4 * 16), "r"(smem_u32(&bar))
              : "memory");
      }
      uint32_t done = 0;
      while (!done) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, "
            "p;\n\t}"
            : "=r"(done)
            : "r"(smem_u32(&bar)), "r"(phase)
            : "memory");
      }
      phase ^= 1;
      __syncthreads();
    } else {  // LDG.128 into registers: warp per row, up to 8 rows in flight per warp
      for (int i0 = warp * 8; i0 < M; i0 += NW * 8) {
        float4 v[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int i = i0 + j;
          v[j] = (i < M && lane < d4) ? __ldg(data + (size_t)rid[i] * d4 + lane) : make_float4(0, 0, 0, 0);
        }
        __syncwarp();  // keep all 8 loads ahead of the first use
#pragma unroll
        for (int j = 0; j < 8; ++j) acc += v[j].x + v[j].y + v[j].z + v[j].w;
      }
      __syncthreads();
    }
    acc += ((volatile float*)sm)[tid];
  }
  long long t1 = clock64();
  if (tid == 0) cyc[blockIdx.x] = (unsigned long long)(t1 - t0);
  if (acc == 12345.f) sink[0] = acc;
}

int main() {
  const size_t rows = (1u << 30) / 512;  // 1 GB of 512-B rows
  const int d4 = 32;
  float4* data;
  cudaMalloc(&data, rows * 512);
  cudaMemset(data, 0, rows * 512);
  const int rounds = 40;
  float* sink;
  cudaMalloc(&sink, 4);
  unsigned long long* cyc;
  cudaMalloc(&cyc, 148 * 8);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("mode M grid threads cycles/round ns/round(at %.2f GHz) GB/s_total\n", clk / 1e6);
  for (int grid : {1, 32, 148}) {
    for (int M : {16, 32, 64, 104, 128, 256}) {
      std::vector<uint32_t> h((size_t)2 * grid * rounds * M);
      uint64_t s = 88172645463325252ull;
      for (auto& x : h) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; x = (uint32_t)(s % rows); }
      uint32_t* ids;
      cudaMalloc(&ids, h.size() * 4);
      cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
      for (int mode = 0; mode < 3; ++mode) {
        for (int nt : {64, 256}) {
          const int smem = M * 512;
          void* fn = mode == 0 ? (void*)gather<0> : (mode == 1 ? (void*)gather<1> : (void*)gather<2>);
          cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
          void* args[] = {&data, &ids, (void*)&M, (void*)&rounds, (void*)&d4, &cyc, &sink};
          cudaEvent_t a, b;
          cudaEventCreate(&a);
          cudaEventCreate(&b);
          // warm with the second half of the ids, time on the first half
          // after an L2 flush so every row comes from DRAM
          const uint32_t* ids_warm = ids + (size_t)grid * rounds * M;
          void* wargs[] = {&data, (void*)&ids_warm, (void*)&M, (void*)&rounds, (void*)&d4, &cyc, &sink};
          cudaLaunchKernel(fn, grid, nt, wargs, smem, 0);
          cudaMemset(flush, mode, 512u << 20);
          cudaEventRecord(a);
          cudaLaunchKernel(fn, grid, nt, args, smem, 0);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float ms = 0;
          cudaEventElapsedTime(&ms, a, b);
          std::vector<unsigned long long> c(grid);
          cudaMemcpy(c.data(), cyc, grid * 8, cudaMemcpyDeviceToHost);
          double mean = 0;
          for (auto x : c) mean += x;
          mean /= grid;
          const char* nm[3] = {"ldgsts", "bulk", "ldg128"};
          printf("%-7s M=%3d grid=%3d nt=%3d  %8.0f cyc/round  %7.0f ns  %8.1f GB/s  err=%s\n", nm[mode], M, grid, nt,
                 mean / rounds, ms * 1e6 / rounds, (double)grid * rounds * M * 512 / (ms * 1e-3) / 1e9,
                 cudaGetErrorString(cudaGetLastError()));
        }
      }
      cudaFree(ids);
    }
  }
  return 0;
}
