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
static void* sel_kernel(bool persist, int cs, int occ) {
  if constexpr (NT >= 1024 && CPL > 4) {
    return nullptr;
  } else {
    if (!persist) return (void*)batch_kernel<NT, TL, CPL, M>;
    if (occ == 2) {
      // two resident CTAs per SM (256/512 threads; 512 only for rows of <= 128
      // chunks, like the 1024-thread build)
      if constexpr ((NT == 256 || NT == 512) && !(NT == 512 && CPL > 4))
        return cs == 1 ? (void*)persistent_kernel<NT, TL, CPL, M, 1, 2> : nullptr;
      else
        return nullptr;
    }
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
static void* pick_cc(int cc, bool persist, int cs, int occ) {
  switch (cc) {
    case 0: return sel_kernel<NT, 2, 4, M>(persist, cs, occ);
    case 1: return sel_kernel<NT, 4, 4, M>(persist, cs, occ);
    case 2: return sel_kernel<NT, 8, 4, M>(persist, cs, occ);
    case 3: return sel_kernel<NT, 16, 4, M>(persist, cs, occ);
    case 4: return sel_kernel<NT, 32, 4, M>(persist, cs, occ);
    case 5: return sel_kernel<NT, 32, 8, M>(persist, cs, occ);
    case 6: return sel_kernel<NT, 32, 16, M>(persist, cs, occ);
  }
  return nullptr;
}

#define ALGAS_CAT2(a, b) a##b
#define ALGAS_CAT(a, b) ALGAS_CAT2(a, b)
void* ALGAS_CAT(kernel_table_nt, ALGAS_NT)(int metric, int cc, bool persist, int cs, int occ) {
  return metric == kL2 ? pick_cc<ALGAS_NT, kL2>(cc, persist, cs, occ) : pick_cc<ALGAS_NT, kIP>(cc, persist, cs, occ);
}

}  // namespace algas
