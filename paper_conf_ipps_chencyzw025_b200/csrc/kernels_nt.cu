// kernels_nt.cu -- the search kernels instantiated for ONE thread count
// (-DALGAS_NT=32|64|128|256|512|1024; build.py compiles this file once per
// value, in parallel): every (chunk config, metric) pair of the batch kernel
// and of the persistent kernel (cluster-split variants for 256 threads).
// 1024-thread CTAs (32 warps, <= 64 registers per thread) are built for rows
// of up to 128 float4 chunks (dim <= 512); wider rows need the registers of
// <= 512-thread CTAs.
#include "kernels.cuh"

#ifndef ALGAS_NT
#error "compile with -DALGAS_NT=<threads per CTA>"
#endif

namespace algas {

template <int NT, int TL, int CPL, int M>
static void* sel_kernel(bool persist, int cs) {
  if constexpr (NT >= 1024 && CPL > 4) {
    return nullptr;
  } else {
    if (!persist) return (void*)batch_kernel<NT, TL, CPL, M>;
    switch (cs) {
      case 1: return (void*)persistent_kernel<NT, TL, CPL, M, 1>;
      // cluster-split searches: instantiated for the 256-thread configuration only
      case 2: return NT == 256 ? (void*)persistent_kernel<NT, TL, CPL, M, (NT == 256 ? 2 : 1)> : nullptr;
      case 4: return NT == 256 ? (void*)persistent_kernel<NT, TL, CPL, M, (NT == 256 ? 4 : 1)> : nullptr;
      case 8: return NT == 256 ? (void*)persistent_kernel<NT, TL, CPL, M, (NT == 256 ? 8 : 1)> : nullptr;
    }
    return nullptr;
  }
}
template <int NT, int M>
static void* pick_cc(int cc, bool persist, int cs) {
  switch (cc) {
    case 0: return sel_kernel<NT, 2, 4, M>(persist, cs);
    case 1: return sel_kernel<NT, 4, 4, M>(persist, cs);
    case 2: return sel_kernel<NT, 8, 4, M>(persist, cs);
    case 3: return sel_kernel<NT, 16, 4, M>(persist, cs);
    case 4: return sel_kernel<NT, 32, 4, M>(persist, cs);
    case 5: return sel_kernel<NT, 32, 8, M>(persist, cs);
    case 6: return sel_kernel<NT, 32, 16, M>(persist, cs);
  }
  return nullptr;
}

#define ALGAS_CAT2(a, b) a##b
#define ALGAS_CAT(a, b) ALGAS_CAT2(a, b)
void* ALGAS_CAT(kernel_table_nt, ALGAS_NT)(int metric, int cc, bool persist, int cs) {
  return metric == kL2 ? pick_cc<ALGAS_NT, kL2>(cc, persist, cs) : pick_cc<ALGAS_NT, kIP>(cc, persist, cs);
}

}  // namespace algas
