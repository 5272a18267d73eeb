// microbench_latency.cu -- dependent-load (pointer chase) latency on B200 as
// a function of the footprint the chase wanders over: L2-resident sizes vs
// DRAM sizes, to separate DRAM latency from address-translation cost.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/mbl scripts/microbench_latency.cu && scripts/mbl
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

__global__ void chase(const uint64_t* __restrict__ next, uint64_t start, int steps, unsigned long long* out) {
  uint64_t p = start;
  long long t0 = clock64();
  for (int i = 0; i < steps; ++i) p = __ldcg(next + p);  // L2-cached, L1 bypass
  long long t1 = clock64();
  out[0] = (unsigned long long)(t1 - t0);
  out[1] = p;
}

int main() {
  const size_t max_bytes = 4ull << 30;
  uint64_t* buf;
  cudaMalloc(&buf, max_bytes);
  unsigned long long* out;
  cudaMalloc(&out, 16);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("footprint_MB stride_B steps cycles/load ns/load\n");
  for (size_t mb : {4, 32, 64, 256, 512, 1024, 2048, 4096}) {
    for (size_t stride : {512ul, 4096ul, (size_t)2 << 20}) {
      const size_t n = (mb << 20) / stride;  // nodes, one per stride
      if (n < 64) continue;
      std::vector<uint64_t> idx(n);
      for (size_t i = 0; i < n; ++i) idx[i] = i;
      uint64_t s = 0x2545F4914F6CDD1Dull;
      for (size_t i = n - 1; i > 0; --i) {  // random cycle
        s ^= s << 13; s ^= s >> 7; s ^= s << 17;
        std::swap(idx[i], idx[s % i]);
      }
      const size_t w = stride / 8;  // words per node
      std::vector<uint64_t> h(n * w, 0);
      for (size_t i = 0; i < n; ++i) h[idx[i] * w] = idx[(i + 1) % n] * w;
      cudaMemcpy(buf, h.data(), n * w * 8, cudaMemcpyHostToDevice);
      const int steps = 4000;
      chase<<<1, 1>>>(buf, idx[0] * w, 200, out);  // warm TLB/L2 a little
      cudaMemset(flush, 1, 512u << 20);               // evict L2
      chase<<<1, 1>>>(buf, idx[7] * w, steps, out);
      unsigned long long r[2];
      cudaMemcpy(r, out, 16, cudaMemcpyDeviceToHost);
      printf("%6zu %8zu %6d %8.0f %7.0f\n", mb, stride, steps, (double)r[0] / steps,
             (double)r[0] / steps / (clk / 1e6));
    }
  }
  return 0;
}
