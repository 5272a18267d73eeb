// kernels.cuh -- the batch (static) and persistent (dynamic batching) search
// kernel templates.  Instantiated once per thread count in kernels_nt.cu
// (compiled with -DALGAS_NT=<threads>, one object per value, in parallel);
// search_kernels.cu holds the launchers and the dispatch table.
//
//  batch_kernel      : static batching -- one launch over nq queries,
//                      each CTA pulls (query, cta_rank) work items from an
//                      atomic counter until the batch is drained.
//  persistent_kernel : dynamic batching -- grid = slots x T
//                      CTAs that never exit; each slot's rank-0 CTA polls for
//                      work (host-mapped ring: "The CTAs in the slot
//                      poll the state", or an HBM query queue), publishes it
//                      through a device mailbox to the slot's other CTAs,
//                      and every CTA publishes its own top-k + a Finish flag
//                      (P:L170).
#pragma once
#include <cooperative_groups.h>

#include "internal.h"

namespace algas {

// ------------------------------------------------------------------ memory-order helpers
__device__ __forceinline__ uint32_t ld_acquire_sys(const volatile uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire_gpu64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned int ld_acquire_gpu32(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int4 ld_volatile_i4(const int4* p) {
  int4 r;
  asm volatile("ld.volatile.global.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p)
               : "memory");
  return r;
}
__device__ __forceinline__ float4 ld_volatile_f4(const float4* p) {
  float4 r;
  asm volatile("ld.volatile.global.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p)
               : "memory");
  return r;
}

// ------------------------------------------------------------------ static batch kernel
struct BatchArgs {
  SearchCfg cfg;
  const float4* queries;
  int64_t nq;
  int32_t T, k;
  uint64_t tag0;
  int* work_counter;
  ResultEntry* res;
  CtaStats* stats;
  unsigned long long* gtab;
  uint32_t epoch_base;
};

template <int NT, int TL, int CPL, int METRIC>
__global__ void __launch_bounds__(NT) batch_kernel(BatchArgs a) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const SmemLayout lay = smem_layout(a.cfg.dp4, a.cfg.L, a.cfg.ncap, a.cfg.hash_bits, a.cfg.stage_rows,
                                       gc_bytes(a.cfg.gc_bits, a.cfg.rp_shift), a.cfg.vis_dsmem * a.cfg.vis_words * 4);
  const Smem s = carve(smem_raw, lay);
  init_cta<NT>(s, a.cfg);
  __shared__ int s_item;
  const int64_t total = a.nq * a.T;
  unsigned long long* gt = a.gtab ? a.gtab + ((uint64_t)blockIdx.x << a.cfg.gtab_bits) : nullptr;
  for (;;) {
    if (threadIdx.x == 0) s_item = atomicAdd(a.work_counter, 1);
    __syncthreads();
    const int64_t item = s_item;
    if (item >= total) break;
    const int64_t qi = item / a.T;
    const int c = (int)(item - qi * a.T);
    const float4* qsrc = a.queries + qi * a.cfg.d4;
    for (int i = threadIdx.x; i < a.cfg.d4; i += NT) s.q[i] = qsrc[i];
    if (a.cfg.cosine) normalize_query<NT>(s.q, a.cfg.d4);
    __syncthreads();
    CtaStats* st = a.stats ? a.stats + item : nullptr;
    search_cta<NT, TL, CPL, METRIC>(a.cfg, qpar_of(a.cfg), s, a.tag0 + (uint64_t)qi, (uint32_t)c, a.k, gt,
                                    a.epoch_base + (uint32_t)item, a.res + item * a.k, st);
    __syncthreads();
  }
}

// ------------------------------------------------------------------ persistent kernel
struct PKArgs {
  SearchCfg cfg;
  PersistArgs p;
};

constexpr unsigned long long kMboxQuit = 0xFFFFFFFFull << 32;
#ifndef ALGAS_FINISH_FENCE
#define ALGAS_FINISH_FENCE 0
#endif

// MINB = resident CTAs per SM the build is for (1, or 2 when a persistent
// grid of slots x T searches exceeds the SM count: half the registers)
template <int NT, int TL, int CPL, int METRIC, int CS, int MINB = 1>
__global__ void __launch_bounds__(NT, MINB) persistent_kernel(PKArgs A) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  const SmemLayout lay = smem_layout(A.cfg.dp4, A.cfg.L, A.cfg.ncap, A.cfg.hash_bits, A.cfg.stage_rows,
                                       gc_bytes(A.cfg.gc_bits, A.cfg.rp_shift), A.cfg.vis_dsmem * A.cfg.vis_words * 4);
  const Smem s = carve(smem_raw, lay);
  init_cta<NT>(s, A.cfg, CS);
  if constexpr (CS > 1) cluster_barrier();  // every CTA's mbarriers exist before any remote arrive
  const PersistArgs& P = A.p;
  // a search unit = one (slot, cta_rank) search = one cluster of CS CTAs
  const int unit = blockIdx.x / CS;
  const int crank = blockIdx.x % CS;  // rank inside the cluster (1-D clusters)
  const int slot = unit / P.T;
  const int rank = unit % P.T;
  const int tid = threadIdx.x;
  // start message of a query: mailbox word, tag, params (32 B, one unit for
  // the DSMEM push of cluster slots)
  struct __align__(16) StartMsg {
    unsigned long long mbox, tag;
    int4 par;
  };
  __shared__ StartMsg s_start;
  __shared__ unsigned long long s_t0;
  unsigned long long& s_mbox = s_start.mbox;
  unsigned long long& s_tag = s_start.tag;
  int4& s_par = s_start.par;

  if constexpr (CS > 1) {
    if (crank != 0) {
      // cluster worker: serve the leader's distance steps until it quits
      uint32_t ph = 0;
      while (worker_step<NT, TL, CPL, METRIC>(A.cfg, s, ph) == kCmdStep) {
      }
      return;
    }
  }

  // HBM visited tables: one per search unit (PRIVATE spill), or one per slot
  // shared by the slot's T CTAs (SHARED)
  unsigned long long* gt =
      P.gtab ? P.gtab + ((uint64_t)(A.cfg.shared ? slot : unit) << A.cfg.gtab_bits) : nullptr;
  // SHARED visited bitmaps: two per slot, query number e (served count) of
  // the slot uses buffer e & 1 (see the clear below)
  uint32_t* vbm2 = (A.cfg.shared && P.vbm) ? P.vbm + (uint64_t)slot * 2 * P.vbm_words : nullptr;
  uint32_t served = 0;  // queries this CTA has finished (= last epoch in devq mode)
  uint32_t last_epoch = 0;
  // host ring: the slot's two ring entries (sub-slots) alternate, 1 first
  // (runtime.cu); the epoch last seen in each tells a stale READY apart
  int sub = 1;
  uint32_t last_ep0 = 0u, last_ep1 = 0u;  // (two scalars: a 2-array indexed by `sub` would live in local memory)

  for (;;) {
    // ---------------- acquire work (rank 0) and publish it to the slot's CTAs
    if (rank == 0) {
      if (tid == 0) {
        unsigned long long mb;
        // every CTA of the slot finished the previous query (per-slot HBM
        // finish counter) before the next one is staged: the slot's HBM
        // query buffer, params and mailbox are rewritten only after all T
        // CTAs consumed them, and in SHARED mode the bitmap share a CTA
        // clears at its next pickup is no longer in use by a slower CTA
        // (R26).  Wrap-safe difference of u32 counters.
        // (DSMEM-bitmap slots: the first cluster barrier below gives the same
        // guarantee)
        if (!A.cfg.vis_dsmem)
          while ((int)(ld_acquire_gpu32(P.slot_fin + slot) - served * (uint32_t)P.T) < 0) __nanosleep(32);
        if (P.mode == 0) {
          // host ring: poll the slot state in host memory, or its
          // device mirror in HBM (state_mirror: no PCIe read while polling)
          uint32_t st;
          unsigned ns = 64;
          const uint32_t* mstate =
              P.mir ? reinterpret_cast<const uint32_t*>(P.mir + (size_t)(2 * slot + sub) * P.mir_stride) : nullptr;
          for (;;) {
            st = mstate ? ld_acquire_gpu32(mstate) : ld_acquire_sys(&P.ring[2 * slot + sub].state);
            uint32_t kind = st & 0xFFu, ep = st >> 8;
            if (kind == kSlotQuit) break;
            if (kind == kSlotReady && ep != (sub ? last_ep1 : last_ep0)) break;
            __nanosleep(ns);
            if (ns < 256) ns <<= 1;
          }
          if ((st & 0xFFu) == kSlotQuit) {
            mb = kMboxQuit;
          } else {
            const uint32_t ep = st >> 8;
            mb = ((unsigned long long)ep << 32) | (unsigned long long)slot;
          }
        } else {
          int item = atomicAdd(P.queue_head, 1);
          if (item >= P.nq) {
            mb = kMboxQuit;
          } else {
            const uint32_t ep = served + 1;
            mb = ((unsigned long long)ep << 32) | (unsigned long long)(uint32_t)item;
          }
        }
        s_mbox = mb;
        s_t0 = globaltimer();
      }
      __syncthreads();
      if (A.cfg.vis_dsmem) {
        // cluster slot: the query, params and tag go to this CTA's shared
        // memory only; the other CTAs receive them through DSMEM below
        if (s_mbox != kMboxQuit) {
          if (P.mode == 0) {
            const uint8_t* ment = P.mir ? P.mir + (size_t)(2 * slot + sub) * P.mir_stride : nullptr;
            const RingSlot* rs = ment ? reinterpret_cast<const RingSlot*>(ment) : &P.ring[2 * slot + sub];
            const float4* src = ment ? reinterpret_cast<const float4*>(ment + sizeof(RingSlot))
                                     : P.ring_q + (uint64_t)(2 * slot + sub) * A.cfg.d4;
            for (int i = tid; i < A.cfg.d4; i += NT) s.q[i] = ld_volatile_f4(src + i);
            if (tid == NT - 1) {
              const int4 sp4 = ld_volatile_i4(reinterpret_cast<const int4*>(rs));
              s_par = make_int4(sp4.y, sp4.z, sp4.w, 0);
            }
            if (tid == NT - 2) s_tag = *((const volatile unsigned long long*)&rs->tag);
          } else {
            const uint32_t item = (uint32_t)s_mbox;
            const float4* qsrc = P.queries + (uint64_t)item * A.cfg.d4;
            for (int i = tid; i < A.cfg.d4; i += NT) s.q[i] = qsrc[i];
            if (tid == 0) {
              s_par = make_int4(P.kmax, A.cfg.L, A.cfg.w, 0);
              s_tag = P.tag0 + (uint64_t)item;
            }
          }
          if (A.cfg.cosine) normalize_query<NT>(s.q, A.cfg.d4);  // COSINE (R29): pushed normalised
        }
      } else if (s_mbox != kMboxQuit && P.mode == 0) {
        // payload from mapped host memory in ONE PCIe round trip: the query
        // chunks, {state, k, L, w} and the tag are read by different threads
        // at once (volatile: never a stale line; ordered after thread 0's
        // acquire of the state by the barrier), staged into the slot's HBM
        // buffer for the other CTAs and into this CTA's shared memory
        const uint8_t* ment = P.mir ? P.mir + (size_t)(2 * slot + sub) * P.mir_stride : nullptr;
        const RingSlot* rs = ment ? reinterpret_cast<const RingSlot*>(ment) : &P.ring[2 * slot + sub];
        const float4* src = ment ? reinterpret_cast<const float4*>(ment + sizeof(RingSlot))
                                 : P.ring_q + (uint64_t)(2 * slot + sub) * A.cfg.d4;
        float4* dst = P.qbuf + (uint64_t)slot * A.cfg.d4;
        for (int i = tid; i < A.cfg.d4; i += NT) {
          const float4 v = ld_volatile_f4(src + i);
          dst[i] = v;
          s.q[i] = v;
        }
        if (tid == NT - 1) {
          const int4 sp4 = ld_volatile_i4(reinterpret_cast<const int4*>(rs));
          P.dparams[slot] = make_int4(sp4.y, sp4.z, sp4.w, 0);
        }
        if (tid == NT - 2) P.dtag[slot] = *((const volatile unsigned long long*)&rs->tag);
      }
      __syncthreads();
      if (tid == 0 && !A.cfg.vis_dsmem) {
        __threadfence();
        st_release_gpu64(P.mbox + slot, s_mbox);
      }
    } else if (!A.cfg.vis_dsmem) {
      if (tid == 0) {
        unsigned long long mb;
        for (;;) {
          mb = ld_acquire_gpu64(P.mbox + slot);
          if (mb == kMboxQuit) break;
          if ((uint32_t)(mb >> 32) != last_epoch && (uint32_t)(mb >> 32) != 0u) break;
          __nanosleep(32);
        }
        s_mbox = mb;
        s_t0 = globaltimer();
      }
      __syncthreads();
    }
    if (A.cfg.vis_dsmem) {
      // cluster slot start: barrier 1 -- every CTA finished the previous
      // query (so no share is claimed into and no query buffer is read any
      // more) and rank 0 holds the next item; rank 0 then writes {mailbox,
      // params, tag} and the query into the other CTAs' shared memory
      // (DSMEM), every CTA clears its bitmap share; barrier 2 publishes both.
      // Barrier 1 needs no release: the previous query's DSMEM claims all
      // returned their words (performed), and the shared-memory data rank 0
      // pushes was ordered by its own __syncthreads; the results still in
      // flight to host memory are ordered by their Finish word's release.
      cluster_barrier_relaxed();
      if (tid == 0) s_t0 = globaltimer();  // the slot is free: the query starts now
      if (rank == 0) {
        const int nq4 = A.cfg.d4 + 2;  // query chunks + the 32-B start message
        for (int i = tid; i < nq4 * (P.T - 1); i += NT) {
          const int r = 1 + i / nq4, c = i % nq4;
          const uint4* lp = c < A.cfg.d4 ? reinterpret_cast<const uint4*>(s.q + c)
                                          : reinterpret_cast<const uint4*>(&s_start) + (c - A.cfg.d4);
          uint32_t ra;
          asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(lp)), "r"(r));
          const uint4 v = *lp;
          asm volatile("st.shared::cluster.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(ra), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                       : "memory");
        }
      }
      uint4* v4 = reinterpret_cast<uint4*>(s.vsh);
      const uint4 z = make_uint4(0u, 0u, 0u, 0u);
      for (int i = tid; i < (A.cfg.vis_words >> 2); i += NT) v4[i] = z;
      cluster_barrier();
    }
    const unsigned long long mb = s_mbox;
    if (mb == kMboxQuit) {
      if constexpr (CS > 1) post_quit<CS>(s);
      break;  // (cluster slots: no CTA addresses another's shared memory after barrier 2)
    }
    const uint32_t epoch = (uint32_t)(mb >> 32);
    const uint32_t item = (uint32_t)mb;
    int4 par;
    uint64_t tag;
    if (A.cfg.vis_dsmem) {
      par = s_par;  // delivered with the query (cluster slot start)
      tag = s_tag;
    } else if (P.mode == 0) {
      // host ring: per-query params published by rank 0 with the mailbox
      if (tid == 0) {
        const volatile int* vp = reinterpret_cast<const volatile int*>(P.dparams + slot);
        s_par = make_int4(vp[0], vp[1], vp[2], vp[3]);
        s_tag = *((volatile unsigned long long*)(P.dtag + slot));
      }
      __syncthreads();
      par = s_par;
      tag = s_tag;
    } else {
      // device queue: the launch's params; the tag follows from the item
      par = make_int4(P.kmax, A.cfg.L, A.cfg.w, 0);
      tag = P.tag0 + (uint64_t)item;
    }

    // ---------------- stage the query into shared memory (rank 0 of a ring
    // slot already holds it from the PCIe read)
    if (A.cfg.vis_dsmem) {
      // (the query is in s.q already, normalised for COSINE)
    } else if (P.mode == 1) {
      const float4* qsrc = P.queries + (uint64_t)item * A.cfg.d4;
      for (int i = tid; i < A.cfg.d4; i += NT) s.q[i] = qsrc[i];
    } else if (rank != 0) {
      const float4* qsrc = P.qbuf + (uint64_t)slot * A.cfg.d4;
      for (int i = tid; i < A.cfg.d4; i += NT) s.q[i] = ld_volatile_f4(qsrc + i);
    }
    uint32_t* vbm = nullptr;
    if (vbm2) {
      // SHARED visited bitmap ("each CTA initializes a part of the
      // visited table"): this query uses buffer served & 1, and
      // every CTA clears its 1/T share of the OTHER buffer now, for the
      // slot's next query, off the critical path of this one.  That buffer's
      // last user (the previous query) is complete in every CTA: rank 0
      // publishes a query only after the slot's finish counter shows all T
      // CTAs done with the previous one (both feeds), and these stores are
      // ordered before the next query's first claim by this CTA's finish
      // (fence + counter increment) -> rank 0's acquire -> mailbox release.
      vbm = vbm2 + (uint64_t)(served & 1u) * P.vbm_words;
      uint4* o4 = reinterpret_cast<uint4*>(vbm2 + (uint64_t)((served & 1u) ^ 1u) * P.vbm_words);
      const int64_t n4 = P.vbm_words / 4, lo = n4 * rank / P.T, hi = n4 * (rank + 1) / P.T;
      const uint4 z = make_uint4(0u, 0u, 0u, 0u);
      for (int64_t i = lo + tid; i < hi; i += NT) o4[i] = z;
    }
    if (!A.cfg.vis_dsmem) {
      if (A.cfg.cosine) normalize_query<NT>(s.q, A.cfg.d4);  // COSINE (R29), before the cluster push
      if constexpr (CS > 1) push_query<NT, CS>(s, A.cfg.d4);  // released by the first step signal
      __syncthreads();
    }

    const QPar qp{par.y, par.z, A.cfg.off < par.y ? A.cfg.off : par.y};
    const int k = par.x;
    ResultEntry* out;
    CtaStats* stp;
    if (P.mode == 0) {
      out = P.ring_res + ((uint64_t)(2 * slot + sub) * P.T + rank) * P.kmax;
      stp = P.ring_stats + (uint64_t)(2 * slot + sub) * P.T + rank;
    } else {
      out = P.dq_res + ((uint64_t)item * P.T + rank) * P.kmax;
      stp = P.dq_stats + (uint64_t)item * P.T + rank;
    }
    CtaStats local;
    search_cta<NT, TL, CPL, METRIC, CS, MINB>(A.cfg, qp, s, tag, (uint32_t)rank, k, gt, P.epoch_base + served, out,
                                              &local, vbm);
    __syncthreads();
    if (tid == 0) {
      local.t_start = s_t0;
      local.t_end = globaltimer();
      *stp = local;
    }
    served++;
    last_epoch = epoch;
    __syncthreads();
    // ---------------- Finish
    // device-scope finish count, which gates the slot's next pickup: thread 0
    if (tid == 0 && !A.cfg.vis_dsmem) {  // (cluster slots start on a cluster barrier instead)
      __threadfence();
      atomicAdd(P.slot_fin + slot, 1u);
    }
    // host-visible Finish word: the CTA's list and counters (written by its
    // threads before the barrier above) are released at system scope -- the
    // ring's per-CTA Finish flag, or the streaming merge's (query, CTA) word.
    // Issued by the LAST warp, so its release overlaps the next pickup
    // instead of delaying thread 0's polling.  st.release.sys alone orders
    // the CTA's earlier writes (ordered before it by the barrier, release is
    // cumulative) before the flag; ALGAS_FINISH_FENCE=1 builds add a full
    // fence.sc.sys in front (A/B).
    if (tid == NT - 32) {
#if ALGAS_FINISH_FENCE
      if (P.mode == 0 || P.dq_done) __threadfence_system();
#endif
      if (P.mode == 0) {
        st_release_sys(P.ring_done + (uint64_t)(2 * slot + sub) * P.T + rank, epoch);
      } else if (P.dq_done) {
        st_release_sys(P.dq_done + (uint64_t)item * P.T + rank, P.call_id);
      }
    }
    if (P.mode == 0) {  // the slot's next query is in its other ring entry
      if (sub) last_ep1 = epoch; else last_ep0 = epoch;
      sub ^= 1;
    }
  }
}

}  // namespace algas
