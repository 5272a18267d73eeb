// search_kernels.cu -- launchers of the search kernels and the dispatch over
// the per-thread-count kernel tables (kernels_nt.cu, kernels.cuh).
#include "kernels.cuh"

namespace algas {

// ------------------------------------------------------------------ dispatch
// chunk configs (TL lanes per vector, CPL float4 chunks per lane), see
// chunk_tl()/chunk_cpl() in search_core.cuh
int chunk_config_for(int d4) {
  if (d4 <= 8) return 0;
  if (d4 <= 16) return 1;
  if (d4 <= 32) return 2;
  if (d4 <= 64) return 3;
  if (d4 <= 128) return 4;
  if (d4 <= 256) return 5;
  if (d4 <= 512) return 6;
  return -1;
}

// per-thread-count kernel tables (kernels_nt.cu, one object per NT)
static void* kernel_for(const Plan& pl, int metric, bool persist) {
  const int cs = persist ? pl.cluster : 1;
  switch (pl.nt) {
    case 32: return kernel_table_nt32(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
    case 64: return kernel_table_nt64(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
    case 128: return kernel_table_nt128(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
    case 256: return kernel_table_nt256(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
    case 512: return kernel_table_nt512(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
    case 1024: return kernel_table_nt1024(metric, pl.ccfg, persist, cs, persist ? pl.occ : 1);
  }
  return nullptr;
}

int max_blocks_per_sm(const Plan& pl, bool persistent, int* out) {
  void* fn = kernel_for(pl, pl.metric, persistent);
  if (!fn)
    return set_error(ALGAS_EINVAL, "no kernel for threads=%d chunk=%d cluster=%d (cluster > 1 needs 256 threads)",
                     pl.nt, pl.ccfg, pl.cluster);
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem));
  int nb = 0;
  ALGAS_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, pl.nt, pl.smem));
  *out = nb;
  return ALGAS_OK;
}

int max_active_clusters(const Plan& pl, int* out) {
  void* fn = kernel_for(pl, pl.metric, true);
  if (!fn) return set_error(ALGAS_EINVAL, "no persistent kernel for cluster=%d", pl.cluster);
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem));
  const int csz = launch_cluster_size(pl);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(csz);
  cfg.blockDim = dim3(pl.nt);
  cfg.dynamicSmemBytes = pl.smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = csz;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  ALGAS_CUDA_TRY(cudaOccupancyMaxActiveClusters(&n, fn, &cfg));
  *out = n;
  return ALGAS_OK;
}

int launch_batch(const Plan& pl, const BatchLaunch& bl, cudaStream_t st) {
  void* fn = kernel_for(pl, pl.metric, false);
  if (!fn) return set_error(ALGAS_EINVAL, "no kernel for threads=%d chunk=%d", pl.nt, pl.ccfg);
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem));
  BatchArgs a;
  a.cfg = pl.cfg;
  a.queries = bl.queries;
  a.nq = bl.nq;
  a.T = pl.T;
  a.k = pl.k;
  a.tag0 = bl.tag0;
  a.work_counter = bl.work_counter;
  a.res = bl.res;
  a.stats = bl.stats;
  a.gtab = bl.gtab;
  a.epoch_base = bl.epoch_base;
  ALGAS_CUDA_TRY(cudaMemsetAsync(bl.work_counter, 0, sizeof(int), st));
  void* args[] = {&a};
  ALGAS_CUDA_TRY(cudaLaunchKernel(fn, dim3(bl.grid), dim3(pl.nt), args, pl.smem, st));
  return ALGAS_OK;
}

int launch_persistent(const Plan& pl, const PersistArgs& pa, cudaStream_t st) {
  void* fn = kernel_for(pl, pl.metric, true);
  if (!fn) return set_error(ALGAS_EINVAL, "no kernel for threads=%d chunk=%d cluster=%d", pl.nt, pl.ccfg, pl.cluster);
  ALGAS_CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, pl.smem));
  PKArgs A;
  A.cfg = pl.cfg;
  A.p = pa;
  void* args[] = {&A};
  // cooperative launch: the runtime refuses a grid that cannot be fully
  // co-resident, which a persistent kernel needs for forward progress;
  // cluster dimension = the CTAs of one cluster-split search
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(pa.slots * pa.T * pl.cluster);
  cfg.blockDim = dim3(pl.nt);
  cfg.dynamicSmemBytes = pl.smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  int na = 0;
  // cooperative launch for single-CTA units (the runtime refuses a grid that
  // cannot be co-resident); cluster grids are checked against
  // cudaOccupancyMaxActiveClusters by make_plan / check_coresident instead
  // (a cooperative cluster launch fails under ncu's kernel replay)
  if (launch_cluster_size(pl) <= 1) {
    at[na].id = cudaLaunchAttributeCooperative;
    at[na].val.cooperative = 1;
    ++na;
  }
  if (launch_cluster_size(pl) > 1) {
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = launch_cluster_size(pl);
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    ++na;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  cudaError_t e = cudaLaunchKernelExC(&cfg, fn, args);
  if (e != cudaSuccess) {
    (void)cudaGetLastError();
    return set_error(e == cudaErrorCooperativeLaunchTooLarge ? ALGAS_EINVAL : ALGAS_ECUDA,
                     "persistent launch (%d slots x %d searches x %d-CTA clusters x %d threads, %d B smem) failed: %s",
                     pa.slots, pa.T, pl.cluster, pl.nt, pl.smem, cudaGetErrorString(e));
  }
  return ALGAS_OK;
}

}  // namespace algas
