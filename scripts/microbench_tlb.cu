// microbench_tlb.cu -- is the per-SM random-row gather rate on B200 bound by
// DRAM, by loads in flight, or by address translation?
//
// Every warp gathers random 512-B rows (lane = 16 B, LDG.128), RPW rows in
// flight per warp, ids staged in shared memory first (no dependent id load).
// Footprints:
//   dram1g    rows uniform over a 1 GB table (L2 flushed before the timed run)
//   l2dense   rows uniform over a 64 MB contiguous table (L2 resident)
//   l2sparse  64 MB of rows spread as 1024 x 64 KB chunks, one chunk per
//             2 MB page over a 2 GB span (L2 resident, 1024 distinct pages)
//   dram1g_local rows of each warp-batch drawn from one random 2 MB page
//             (same DRAM traffic as dram1g, far fewer pages per batch)
// l2dense vs l2sparse isolates translation cost; dram1g vs dram1g_local
// shows whether page locality buys DRAM-side throughput.
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mbt scripts/microbench_tlb.cu && /tmp/mbt
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

template <int RPW>
__global__ void __launch_bounds__(256) gather(const float4* __restrict__ data, const uint32_t* __restrict__ ids,
                                              int rows_per_cta, int rounds, float* sink) {
  __shared__ uint32_t sid[2048];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, NW = blockDim.x / 32;
  float acc = 0.f;
  for (int r = 0; r < rounds; ++r) {
    const uint32_t* rid = ids + ((size_t)blockIdx.x * rounds + r) * rows_per_cta;
    __syncthreads();
    for (int i = tid; i < rows_per_cta; i += blockDim.x) sid[i] = rid[i];
    __syncthreads();
    for (int i0 = warp * RPW; i0 < rows_per_cta; i0 += NW * RPW) {
      float4 v[RPW];
#pragma unroll
      for (int j = 0; j < RPW; ++j) v[j] = __ldg(data + (size_t)sid[i0 + j] * 32 + lane);
      __syncwarp();
#pragma unroll
      for (int j = 0; j < RPW; ++j) acc += v[j].x + v[j].y + v[j].z + v[j].w;
    }
  }
  if (acc == 12345.f) sink[0] = acc;
}

static uint64_t rs = 88172645463325252ull;
static uint32_t rnd() { rs ^= rs << 13; rs ^= rs >> 7; rs ^= rs << 17; return (uint32_t)rs; }

int main() {
  const size_t span = 4ull << 30;  // 4 GB allocation
  float4* data;
  if (cudaMalloc(&data, span) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMemset(data, 0, span);
  void* flush;
  cudaMalloc(&flush, 512u << 20);
  float* sink;
  cudaMalloc(&sink, 4);
  const int rows_per_cta = 2048, rounds = 8;
  printf("pattern grid threads RPW GB/s\n");
  for (int pat = 0; pat < 4; ++pat) {
    for (int occ : {1, 2, 4, 8}) {
      const int grid = 148 * occ;
      std::vector<uint32_t> h((size_t)grid * rounds * rows_per_cta);
      for (size_t i = 0; i < h.size(); ++i) {
        if (pat == 0) h[i] = rnd() % (1u << 21);                      // 1 GB / 512 B
        else if (pat == 1) h[i] = rnd() % (1u << 17);                 // 64 MB
        else if (pat == 2) h[i] = (rnd() % 1024) * 4096 + rnd() % 128;  // chunk c in page c (2 MB = 4096 rows)
        else {                                                           // one page per 16-row batch
          static uint32_t page = 0;
          if (i % 16 == 0) page = rnd() % 512;
          h[i] = page * 4096 + rnd() % 4096;
        }
      }
      uint32_t* ids;
      cudaMalloc(&ids, h.size() * 4);
      cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
      const char* nm[4] = {"dram1g", "l2dense", "l2sparse", "dram1g_local"};
      for (int rpw : {8, 16}) {
        void (*fn)(const float4*, const uint32_t*, int, int, float*) = rpw == 8 ? gather<8> : gather<16>;
        fn<<<grid, 256>>>(data, ids, rows_per_cta, rounds, sink);  // warm (L2 for patterns 1/2)
        if (pat == 0 || pat == 3) cudaMemset(flush, 1, 512u << 20);
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        cudaEventRecord(a);
        fn<<<grid, 256>>>(data, ids, rows_per_cta, rounds, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        printf("%-12s %5d 256 %2d %8.1f  %s\n", nm[pat], grid, rpw,
               (double)grid * rounds * rows_per_cta * 512 / (ms * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError()));
      }
      cudaFree(ids);
    }
  }
  return 0;
}
