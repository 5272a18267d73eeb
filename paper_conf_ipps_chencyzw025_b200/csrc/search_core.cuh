// search_core.cuh -- the per-CTA greedy/beam graph search of ALGAS on sm_100a.
//
// One CTA runs one (query, cta_rank) search:
//   select  : first unchecked candidate(s) of the sorted list            (P:L217 step 1, Alg.1 l.6)
//             -- w parents at once after the list offset reaches off   (beam extend)
//   gather  : the parents' neighbour ids (one id per thread)             (P:L217 step 1)
//   filter  : test-and-set in a shared-memory visited hash               (P:L217 step 2)
//   distance: the surviving neighbours' vectors are copied into shared
//             memory asynchronously (16-B cp.async per lane, or one
//             cp.async.bulk per row on an mbarrier) so every row of a step
//             is in flight at once without holding registers; a team of TL
//             lanes per row reduces (q-x)^2 / q.x with a shuffle tree    (P:L217 step 3, Alg.1 l.9-12)
//   update  : keys that cannot enter the list are dropped; survivors are
//             MERGED into the sorted list by rank (position = rank among
//             the new keys + lower bound in the list), keeping the first L,
//             with no re-sort of the list                                (P:L219 step 4, Alg.1 l.15-18)
//   finish  : all L entries checked (or the max_iter cap)                ("Finish")
// The CTA then writes its first k (id, dist).
//
// Keys are u64: (order-preserving fp32 distance << 32) | (id << 1) | checked.
// Ids are < 2^31, so comparing keys compares (dist, id) lexicographically
// (R4) and the "checked" bit never decides an order (ids in a list are
// unique).  Nothing here is shared with oracle/: it is an independent
// implementation of the same paper passages.
#pragma once

#include <cooperative_groups.h>
#include <cstdint>
#include <cuda_runtime.h>

namespace algas {

constexpr uint32_t kSentinel = 0xFFFFFFFFu;
constexpr uint32_t kHashEmpty = 0xFFFFFFFFu;
constexpr uint64_t kKeyMax = ~0ull;

enum { kL2 = 0, kIP = 1 };

// ------------------------------------------------------------------ keys
__device__ __forceinline__ uint32_t dist_to_ord(float f) {
  if (f == 0.0f) f = 0.0f;  // -0 and +0 compare equal: canonicalise
  uint32_t u = __float_as_uint(f);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float ord_to_dist(uint32_t u) {
  return __uint_as_float((u & 0x80000000u) ? (u & 0x7FFFFFFFu) : ~u);
}
__device__ __forceinline__ uint64_t make_key(float d, uint32_t id) {
  return ((uint64_t)dist_to_ord(d) << 32) | ((uint64_t)id << 1);
}
__device__ __forceinline__ uint32_t key_id(uint64_t k) { return (uint32_t)(k >> 1) & 0x7FFFFFFFu; }
__device__ __forceinline__ float key_dist(uint64_t k) { return ord_to_dist((uint32_t)(k >> 32)); }

// ------------------------------------------------------------------ entry points (R5)
// splitmix64 output step; the same counter-based generator the oracle
// implements independently (R5).
__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint32_t entry_point(uint64_t seed, uint64_t tag, uint32_t cta, uint32_t j,
                                                uint64_t n) {
  uint64_t a = splitmix64(((uint64_t)cta << 32) | (uint64_t)j);
  uint64_t b = splitmix64(tag ^ a);
  return (uint32_t)(splitmix64(seed ^ b) % n);
}

// ------------------------------------------------------------------ memory helpers
__device__ __forceinline__ uint4 ldg_u4(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
// graph rows are re-read by every query (hub neighbourhoods): keep them in L2
// with an evict_last policy while the vector gathers stream past
__device__ __forceinline__ uint64_t l2_evict_last_policy() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint32_t ldg_u32_hint(const uint32_t* p, uint64_t pol) {
  uint32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
// mbarrier + bulk async copy (TMA engine, non-tensor), CTA scope
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(phase)
        : "memory");
  }
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}

// ------------------------------------------------------------------ configuration
// Distance "chunk configs": TL lanes per vector, CPL 16-B chunks per lane.
// A vector of d4 = dim/4 chunks is stored in shared memory padded to
// dp4 = TL*CPL chunks (zero tail) so the distance loop needs no masks.
// Four 16-B chunks per lane (64 B of a row) keep the shuffle tree short
// (log2 TL levels) while a warp-wide load still covers whole 128-B lines.
//   cc: 0      1      2      3      4       5       6
//   d4: <=8   <=16   <=32   <=64   <=128   <=256   <=512
__host__ __device__ inline int chunk_tl(int cc) { const int t[7] = {2, 4, 8, 16, 32, 32, 32}; return t[cc]; }
__host__ __device__ inline int chunk_cpl(int cc) { const int t[7] = {4, 4, 4, 4, 4, 8, 16}; return t[cc]; }
__device__ __forceinline__ float4 ldg_f4_stream(const float4* p) {
  float4 r;
  // volatile: keeps every gather load of a pass ahead of the first use (the
  // scheduler otherwise interleaves loads with the FMAs of earlier rows and
  // serialises the DRAM round trips)
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}

// Row gathers of the distance step.  Volatile (strong, sys-scope) loads:
// ptxas keeps volatile memory operations in program order, so every row
// load of a pass is issued before the (volatile) query reads that the FMAs
// depend on -- the only robust way to keep all loads of a wave in flight
// (plain loads get interleaved with FMAs by the scheduler, serialising the
// round trips).  Device memory: served by L2 like .cg.
#ifndef ALGAS_ROWLOAD
#define ALGAS_ROWLOAD 0  // A/B builds: 1 = ld.relaxed.gpu, 2 = ld.relaxed.cta, 3 = ld.global.nc (asm volatile)
#endif
__device__ __forceinline__ float4 ld_row_f4(const float4* p) {
  float4 r;
#if ALGAS_ROWLOAD == 1
  asm volatile("ld.relaxed.gpu.global.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
#elif ALGAS_ROWLOAD == 2
  asm volatile("ld.relaxed.cta.global.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
#elif ALGAS_ROWLOAD == 3
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
#else
  asm volatile("ld.volatile.global.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
#endif
  return r;
}
__device__ __forceinline__ float4 lds_f4_ordered(const float4* p) {
  float4 r;
  asm volatile("ld.volatile.shared.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "r"(smem_u32(p)));
  return r;
}

struct SearchCfg {
  const float4* data;    // n x d4 float4 (row-major, 16-B aligned rows)
  const uint32_t* graph; // n x Rp u32 (Rp = 1 << rp_shift, padded with sentinels)
  uint64_t n;
  int32_t d4;            // dim / 4
  int32_t dp4;           // padded row length in shared memory (TL*CPL)
  int32_t R;             // out-degree
  int32_t rp_shift;      // log2 of the graph row stride
  int32_t L, w, off, S, max_iter;
  int32_t hash_bits;     // shared-memory visited hash: 2^hash_bits u32
  int32_t gtab_bits;     // HBM spill table per CTA: 2^gtab_bits u64
  int32_t ncap;          // capacity of the new-key buffer
  int32_t stage_rows;    // vectors per shared-memory staging buffer (2 buffers)
  int32_t team_rows;     // gather_mode 3: rows in flight per team and pass (its staging slots)
  int32_t gather_mode;   // 0: LDG.128 into registers, many rows in flight per warp (default)
                         // 1: 16-B cp.async (LDGSTS) staging, 2: cp.async.bulk staging (mbarrier)
                         // 3: team-local cp.async: each lane copies the 16-B chunks of its team's
                         //    rows it will itself reduce into the team's staging slots, so every
                         //    row of a pass is in flight without holding registers and without a
                         //    CTA barrier between landing and use (team_rows rows per team)
  int32_t prefetch;      // bits: 1 L2 prefetch of each surviving row at filter time, 2 of the
                         // likely next parents' graph rows at select, 4 evict_last graph loads,
                         // 8 (default) graph rows of keys entering the list, at distance time,
                         // 16 each row new to the CTA, before the shared claim;
                         // 64 (experiment switch) disables the fused warp merge+select;
                         // 128 enables the shared-memory graph-row cache (gc_bits)
  int32_t gc_bits;       // log2 entries of the shared-memory graph-row cache (0: off): rows of
                         //    keys entering the list are copied (cp.async) into it during the
                         //    distance step, so the next step's parents' neighbour ids are
                         //    read from shared memory instead of L2
  int32_t shared;        // 1: SHARED visited mode -- the HBM table passed to search_cta is the
                         //    query's table, shared by its T CTAs; the shared-memory
                         //    hash is this CTA's cache of it
  int32_t cosine;        // 1: COSINE index (unit data rows, METRIC = kIP): the staged query is
                         //    normalised in shared memory (normalize_query) before the search
  int32_t vis_dsmem;     // 1: SHARED visited bitmap in distributed shared memory -- the query's
                         //    T CTAs form a thread-block cluster and CTA r holds bitmap words
                         //    w with w % T == r (vis_words u32 each); claims are DSMEM atomics
  int32_t vis_tshift;    //    log2 T (T = 1, 2, 4, 8)
  int32_t vis_words;     //    u32 words of this CTA's share (multiple of 4)
  uint64_t seed;
};

struct CtaStats {
  uint32_t iters, parents, dist_evals, cap_hit, spilled, overflow;
  unsigned long long t_start, t_end;  // globaltimer (persistent paths)
  unsigned long long cyc_select, cyc_gather, cyc_dist, cyc_sort;  // SM cycles per phase
  unsigned long long t_loop0, t_loop1;  // globaltimer: search loop entered / left
  unsigned long long t_entry;           // globaltimer: search_cta entered (query staged)
  uint32_t mg_bitonic, mg_rank;         // candidate updates: warp bitonic merge / rank merge
};

struct ResultEntry {
  uint32_t id;
  float dist;
};

struct Ctrl {
  int cnt, np, done, diffusing, vis_count, spilled, overflow, cur;
  // per-step counters, double-buffered by step parity so that the fused
  // merge+select of warp 0 can reset the next step's while the other warps
  // still read this step's
  int nnew[2], nkeys[2];
  uint32_t gc_stamp;  // step stamp of the graph-row cache (claims one copy per slot and step)
  uint32_t iters, parents, dist_evals, cap_hit;
  uint32_t mg_bitonic, mg_rank;  // candidate updates by the warp bitonic merge / by the rank merge
  uint32_t phase;  // bit b: parity of staging barrier b (b=2: step-ready, b=3: keys)
  uint64_t worst;  // prefilter key of the current step
  unsigned long long cyc[4];  // per-phase SM cycles (thread 0)
  long long tp;               // clock64 at the last phase boundary
  // cluster worker mailbox (written remotely by the leader before it arrives
  // on the worker's step-ready barrier)
  int w_cmd;       // kCmdStep / kCmdQuit
  int w_m;         // rows of this worker in the step
  uint64_t w_worst;
};
enum { kCmdStep = 1, kCmdQuit = 2 };

// Shared-memory carve-up (bytes, all 16-B aligned).
// scratch ints for the merge's partial rank counts (>= the widest CTA)
constexpr int kMergeParts = 1024;

struct SmemLayout {
  int off_q, off_listA, off_listB, off_newk, off_newid, off_sel, off_part, off_hash, off_stage, off_bar, off_ctrl,
      off_gc, off_vsh, total;
};
// bytes of a graph-row cache of 2^gc_bits rows of Rp ids + tag + stamp per row
__host__ __device__ inline int gc_bytes(int gc_bits, int rp_shift) {
  return gc_bits > 0 ? (1 << gc_bits) * ((4 << rp_shift) + 8) : 0;
}
__host__ __device__ inline int align16(int x) { return (x + 15) & ~15; }
__host__ __device__ inline SmemLayout smem_layout(int dp4, int L, int ncap, int hash_bits, int stage_rows,
                                                   int gcb = 0, int vsh_bytes = 0) {
  SmemLayout s;
  int o = 0;
  s.off_stage = o; o += 2 * stage_rows * dp4 * 16;  // 128-B aligned at offset 0
  s.off_q = o;     o += align16(dp4 * 16);
  s.off_listA = o; o += align16(L * 8);
  s.off_listB = o; o += align16(L * 8);
  s.off_newk = o;  o += align16(ncap * 8);
  s.off_newid = o; o += align16(ncap * 4);
  s.off_sel = o;   o += align16(64 * 4);
  s.off_part = o;  o += kMergeParts * 4;  // partial ranks of the split merge
  s.off_hash = o;  o += align16((1 << hash_bits) * 4);
  s.off_bar = o;   o += 32;
  s.off_ctrl = o;  o += align16((int)sizeof(Ctrl));
  s.off_gc = o;    o += align16(gcb);
  s.off_vsh = o;   o += align16(vsh_bytes);
  s.total = o;
  return s;
}

struct Smem {
  float4* q;
  uint64_t* list[2];
  uint64_t* newk;
  uint32_t* newid;
  int* sel;         // [0,32): selected positions, [32,64): parent ids
  int* part;        // kMergeParts partial rank counts (merge)
  uint32_t* hash;
  float4* stage;    // 2 x stage_rows x dp4
  uint64_t* bar;    // 2 mbarriers
  Ctrl* ctrl;
  uint32_t* gcache; // graph-row cache: rows [2^gc_bits][Rp], then tags, then stamps
  uint32_t* vsh;    // vis_dsmem: this CTA's share of the query's SHARED visited bitmap
};
__device__ __forceinline__ Smem carve(uint8_t* base, const SmemLayout& l) {
  Smem s;
  s.q = reinterpret_cast<float4*>(base + l.off_q);
  s.list[0] = reinterpret_cast<uint64_t*>(base + l.off_listA);
  s.list[1] = reinterpret_cast<uint64_t*>(base + l.off_listB);
  s.newk = reinterpret_cast<uint64_t*>(base + l.off_newk);
  s.newid = reinterpret_cast<uint32_t*>(base + l.off_newid);
  s.sel = reinterpret_cast<int*>(base + l.off_sel);
  s.part = reinterpret_cast<int*>(base + l.off_part);
  s.hash = reinterpret_cast<uint32_t*>(base + l.off_hash);
  s.stage = reinterpret_cast<float4*>(base + l.off_stage);
  s.bar = reinterpret_cast<uint64_t*>(base + l.off_bar);
  s.gcache = reinterpret_cast<uint32_t*>(base + l.off_gc);
  s.ctrl = reinterpret_cast<Ctrl*>(base + l.off_ctrl);
  s.vsh = reinterpret_cast<uint32_t*>(base + l.off_vsh);
  return s;
}
// once per CTA lifetime (kernel start): staging barriers; zero staging and
// query buffers so the padded tail chunks of every row read as 0
// bar[0..1]: staging buffers; bar[2]: "step ready" (cluster worker, 1
// arrival from the leader); bar[3]: "keys delivered" (cluster leader, CS-1
// arrivals).
template <int NT>
__device__ __forceinline__ void init_cta(const Smem& s, const SearchCfg& cfg, int cs = 1) {
  const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int i = threadIdx.x; i < 2 * cfg.stage_rows * cfg.dp4; i += NT) s.stage[i] = z;
  for (int i = threadIdx.x; i < cfg.dp4; i += NT) s.q[i] = z;
  if (threadIdx.x == 0) {
    mbar_init(s.bar + 0, 1);
    mbar_init(s.bar + 1, 1);
    mbar_init(s.bar + 2, 1);
    mbar_init(s.bar + 3, cs > 1 ? cs - 1 : 1);
    mbar_fence_init();
    s.ctrl->phase = 0;
    s.ctrl->gc_stamp = 0;
  }
  if (cfg.gc_bits > 0) {  // rows are immutable: the cache stays valid across queries
    uint32_t* tags = s.gcache + ((1u << cfg.gc_bits) << cfg.rp_shift);
    for (int i = threadIdx.x; i < (2 << cfg.gc_bits); i += NT) tags[i] = i < (1 << cfg.gc_bits) ? 0xFFFFFFFFu : 0u;
  }
  __syncthreads();
}

// ------------------------------------------------------------------ visited set
enum { kVisNew = 0, kVisSeen = 1, kVisFull = 2 };

__device__ __forceinline__ uint32_t hash_slot(uint32_t id, int bits) {
  return (id * 0x9E3779B1u) >> (32 - bits);
}
// test-and-set in the shared-memory open-addressing table
__device__ __forceinline__ int smem_visit(uint32_t* tab, int bits, uint32_t id) {
  const uint32_t mask = (1u << bits) - 1u;
  uint32_t h = hash_slot(id, bits);
  for (uint32_t p = 0; p <= mask; ++p) {
    uint32_t old = atomicCAS(tab + h, kHashEmpty, id);
    if (old == kHashEmpty) return kVisNew;
    if (old == id) return kVisSeen;
    h = (h + 1) & mask;
  }
  return kVisFull;
}
__device__ __forceinline__ bool smem_contains(const uint32_t* tab, int bits, uint32_t id) {
  const uint32_t mask = (1u << bits) - 1u;
  uint32_t h = hash_slot(id, bits);
  for (uint32_t p = 0; p <= mask; ++p) {
    uint32_t v = tab[h];
    if (v == id) return true;
    if (v == kHashEmpty) return false;
    h = (h + 1) & mask;
  }
  return false;
}
// SHARED visited bitmap: atomic test-and-set of id's bit in the
// query's bitmap; true if this call set it.  vis_dsmem: the bitmap is spread
// over the shared memory of the query's T CTAs (one thread-block cluster),
// word w in CTA w % T -- one DSMEM atomic (~200 cycles) instead of an L2
// atomic that queues behind the step's row traffic; else the slot's HBM
// bitmap (vbm).
__device__ __forceinline__ bool vis_claim(const SearchCfg& cfg, uint32_t* vsh, uint32_t* vbm, uint32_t id) {
  const uint32_t bit = 1u << (id & 31), w = id >> 5;
  if (cfg.vis_dsmem) {
    const uint32_t owner = w & ((1u << cfg.vis_tshift) - 1u), lw = w >> cfg.vis_tshift;
    uint32_t ra, old;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(vsh + lw)), "r"(owner));
    asm volatile("atom.relaxed.cluster.shared::cluster.or.b32 %0, [%1], %2;" : "=r"(old) : "r"(ra), "r"(bit) : "memory");
    return (old & bit) == 0u;
  }
  return (atomicOr(vbm + w, bit) & bit) == 0u;
}

// epoch-tagged HBM table: entry = (epoch << 32) | id; an entry of another
// epoch counts as empty, so the table never needs clearing.
__device__ __forceinline__ int gmem_visit(unsigned long long* tab, int bits, uint32_t epoch, uint32_t id) {
  const uint32_t mask = (1u << bits) - 1u;
  const unsigned long long mine = ((unsigned long long)epoch << 32) | id;
  uint32_t h = hash_slot(id, bits);
  for (uint32_t p = 0; p <= mask; ++p) {
    unsigned long long cur = *((volatile unsigned long long*)(tab + h));
    while ((uint32_t)(cur >> 32) != epoch) {
      unsigned long long old = atomicCAS(tab + h, cur, mine);
      if (old == cur) return kVisNew;
      cur = old;
    }
    if (cur == mine) return kVisSeen;
    h = (h + 1) & mask;
  }
  return kVisFull;
}

template <typename K>
__device__ __forceinline__ int lower_bound_u64(const K* a, int n, K x) {
  int lo = 0, hi = n;
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// ------------------------------------------------------------------ distance (P:L217 step 3)
template <int TL, int CPL>
struct QueryRegs {
  float4 q[CPL];
  __device__ __forceinline__ void load(const float4* qs, int tl) {
#pragma unroll
    for (int c = 0; c < CPL; ++c) q[c] = qs[tl + c * TL];  // padded with zeros
  }
};

// partial sum of one team lane over a (zero-padded) row in shared memory
template <int TL, int CPL, int METRIC>
__device__ __forceinline__ float team_partial_smem(const QueryRegs<TL, CPL>& Q, const float4* x, int tl) {
  float acc = 0.f;
#pragma unroll
  for (int c = 0; c < CPL; ++c) {
    const float4 v = x[tl + c * TL];
    if (METRIC == kL2) {
      float a = Q.q[c].x - v.x, b = Q.q[c].y - v.y, e = Q.q[c].z - v.z, f = Q.q[c].w - v.w;
      acc = fmaf(a, a, acc); acc = fmaf(b, b, acc); acc = fmaf(e, e, acc); acc = fmaf(f, f, acc);
    } else {
      acc = fmaf(Q.q[c].x, v.x, acc); acc = fmaf(Q.q[c].y, v.y, acc);
      acc = fmaf(Q.q[c].z, v.z, acc); acc = fmaf(Q.q[c].w, v.w, acc);
    }
  }
  return acc;
}

// copies of rows [r0, r0+cnt) of newid into staging buffer b.
// gather_mode 0: each warp takes rows, its lanes issue 16-B cp.async
// (LDGSTS) chunks, one commit group for the CTA.  gather_mode 1: warp 0's
// lanes issue one cp.async.bulk per row, all completing on mbarrier b.
template <int NT>
__device__ __forceinline__ void stage_issue(const SearchCfg& cfg, const Smem& s, int b, int r0, int cnt, int warp,
                                            int lane) {
  float4* dst = s.stage + (size_t)b * cfg.stage_rows * cfg.dp4;
  if (cfg.gather_mode == 1) {
    constexpr int NW = NT / 32;
    for (int r = warp; r < cnt; r += NW) {
      const uint32_t id = s.newid[r0 + r];
      const float4* src = cfg.data + (uint64_t)id * cfg.d4;
      float4* d = dst + (size_t)r * cfg.dp4;
      for (int c = lane; c < cfg.d4; c += 32) cp_async16(d + c, src + c);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  } else if (warp == 0) {
    const uint32_t row_bytes = (uint32_t)cfg.d4 * 16u;
    fence_proxy_async_smem();
    if (lane == 0) mbar_arrive_expect_tx(s.bar + b, row_bytes * (uint32_t)cnt);
    __syncwarp();
    for (int r = lane; r < cnt; r += 32) {
      const uint32_t id = s.newid[r0 + r];
      bulk_g2s(dst + (size_t)r * cfg.dp4, cfg.data + (uint64_t)id * cfg.d4, row_bytes, s.bar + b);
    }
  }
}

// ------------------------------------------------------------------ the search
// ------------------------------------------------------------------ cluster helpers (CS > 1)
// One search may be spread over a thread-block cluster of CS CTAs (one per
// SM): CTA rank 0 (the leader) owns the candidate list and visited set and
// runs select / gather / filter / merge; the distance step's vector gathers
// are split over all CS CTAs, which read the step's ids from the leader's
// shared memory and deliver keys into it through distributed shared memory.
// A single SM sustains only ~10 GB/s of random 512-B row gathers
// (profiles/gather_microbench.txt); CS SMs multiply the gather rate of one
// query.
__device__ __forceinline__ void cluster_barrier() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// the same barrier without release semantics on the arrive: a thread's
// earlier writes (e.g. results still on their way to host memory) need not
// be performed before it arrives
__device__ __forceinline__ void cluster_barrier_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
}
template <typename T>
__device__ __forceinline__ T* rank_ptr(T* local, int rank) {
  // generic address of the same shared-memory object in cluster CTA `rank`
  return cooperative_groups::this_cluster().map_shared_rank(local, (unsigned)rank);
}
template <typename T>
__device__ __forceinline__ T* leader_ptr(T* local) {
  return rank_ptr(local, 0);
}
// Point-to-point cluster signalling on mbarriers (cheaper than a full
// barrier.cluster: only the signalling thread and the waiters take part).
// The sender's prior writes (by any thread of its CTA, ordered before it by
// __syncthreads) are released at cluster scope by fence + arrive.release.
__device__ __forceinline__ void fence_cluster() { asm volatile("fence.acq_rel.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_remote_arrive(uint64_t* bar, int rank) {
  uint32_t ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(bar)), "r"(rank));
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(ra) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}

// Distance step for rows r = r0, r0+rstep, ... < M of newid (P:L217 step 3):
// LDG.128 straight into registers, each team keeping B rows in flight
// (NT/TL*B rows per CTA and pass), interleaved shuffle-tree reductions,
// prefilter against `worst`, ballot compaction + one atomic per warp to
// append the surviving keys to newk.  newid/newk/nkeys may live in another
// CTA's shared memory (cluster leader).
//
// A step's wave of row reads is latency-bound, and its fixed cost is
// instruction issue (profiles/dist_wave_microbench*.txt): warps with no row
// in a pass skip it entirely (warp-uniform test), and the compaction is one
// ballot per row group instead of a warp scan.
#ifndef ALGAS_GATHER_EXPERIMENTS
#define ALGAS_GATHER_EXPERIMENTS 0  // 1: compile gather modes 1-4 (A/B builds, ALGAS_GATHER_MODE)
#endif
#ifndef ALGAS_QCHUNK
#define ALGAS_QCHUNK 0  // A/B builds: 1 = query chunk loaded per chunk inside the FMA loop
#endif
#ifndef ALGAS_DIST_BW1024
#define ALGAS_DIST_BW1024 4  // A/B builds: 16-B chunks per lane in flight at 1024 resident threads
#endif
template <int NT, int TL, int CPL, int MINB = 1>
struct DistRows {
  // rows in flight per team and pass: the wave's rows all in flight at once
  // within the register budget (<= 64 registers per thread at 1024 resident
  // threads per SM -- one 1024-thread CTA or two 512-thread CTAs -- <= 128
  // at 512)
  static constexpr int BW = NT * MINB >= 1024 ? ALGAS_DIST_BW1024 : 16;
  static constexpr int B = CPL >= BW ? 1 : BW / CPL;
};
// claim_vbm (SHARED mode with the query's bitmap): the rows are
// claimed HERE -- lane 0 of the team issues the row's atomicOr right before
// the row's loads, so the claim's L2 round trip overlaps the row's DRAM
// fetch; a row another CTA of the query claimed first is gathered but its
// key dropped (the node is scored by exactly one CTA, as with a claim at
// filter time, which costs a separate round trip before the wave).
template <int NT, int TL, int CPL, int METRIC, int BOVR = 0>
__device__ __forceinline__ void dist_ldg(const SearchCfg& cfg, const float4* qs, int M, int r0, int rstep,
                                         uint64_t worst, const uint32_t* newid, uint64_t* newk, int* nkeys,
                                         uint32_t* gcache = nullptr, uint32_t gc_stamp = 0,
                                         uint32_t* claim_vbm = nullptr) {
  const int tid = threadIdx.x, lane = tid & 31;
  constexpr int NTEAMS = NT / TL;
  constexpr int TPW = 32 / TL;  // teams per warp
  const int team = tid / TL, tl = tid % TL;
  const int wteam0 = (tid >> 5) * TPW;  // first team of this warp
  constexpr int B = BOVR > 0 ? BOVR : DistRows<NT, TL, CPL>::B;
  constexpr int PASS = NTEAMS * B;
  const int Mc = M > r0 ? (rstep == 1 ? M - r0 : (M - r0 + rstep - 1) / rstep) : 0;  // rows of this CTA
  for (int base = 0; base < Mc; base += PASS) {
    // row groups of this pass that hold any row of THIS warp (warp-uniform):
    // loads, FMAs, shuffles and compaction of empty groups are skipped
    const int nbw = (Mc - base - wteam0 + NTEAMS - 1) / NTEAMS;
    if (nbw <= 0) continue;
    float4 v[B][CPL];
    uint32_t ids[B];
    uint32_t lost[B];  // claim_vbm: another CTA claimed the row first
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int j = base + b * NTEAMS + team;
      ids[b] = j < Mc ? newid[r0 + j * rstep] : 0u;
      lost[b] = 0u;
      if (claim_vbm != nullptr && tl == 0 && b < nbw && j < Mc) {
        const uint32_t bit = 1u << (ids[b] & 31);
        lost[b] = atomicOr(claim_vbm + (ids[b] >> 5), bit) & bit;
      }
    }
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int j = base + b * NTEAMS + team;
      const float4* row = cfg.data + (uint64_t)ids[b] * cfg.d4;
#pragma unroll
      for (int c = 0; c < CPL; ++c) {
        const int chn = tl + c * TL;
        v[b][c] = (b < nbw && j < Mc && chn < cfg.d4) ? ld_row_f4(row + chn) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
    // the query chunks are read (volatile) only after every row load of the
    // pass was issued; the FMAs depend on them, so no FMA can be scheduled
    // between the row loads (which would serialise the DRAM round trips)
    float acc[B];
#if ALGAS_QCHUNK
    // one query chunk in registers at a time (chunk-outer, row-inner): with
    // B > 1 rows per team the query would otherwise hold CPL float4 next to
    // the B x CPL row chunks.  Each row's sum runs in the same order as below.
#pragma unroll
    for (int b = 0; b < B; ++b) acc[b] = 0.f;
#pragma unroll
    for (int c = 0; c < CPL; ++c) {
      const float4 q = lds_f4_ordered(qs + tl + c * TL);
#pragma unroll
      for (int b = 0; b < B; ++b) {
        if (b >= nbw) continue;
        const float4 x = v[b][c];
        float a = acc[b];
        if (METRIC == kL2) {
          float d0 = q.x - x.x, d1 = q.y - x.y, d2 = q.z - x.z, d3 = q.w - x.w;
          a = fmaf(d0, d0, a); a = fmaf(d1, d1, a); a = fmaf(d2, d2, a); a = fmaf(d3, d3, a);
        } else {
          a = fmaf(q.x, x.x, a); a = fmaf(q.y, x.y, a);
          a = fmaf(q.z, x.z, a); a = fmaf(q.w, x.w, a);
        }
        acc[b] = a;
      }
    }
#else
    QueryRegs<TL, CPL> Q;
#pragma unroll
    for (int c = 0; c < CPL; ++c) Q.q[c] = lds_f4_ordered(qs + tl + c * TL);
#pragma unroll
    for (int b = 0; b < B; ++b) {
      float a = 0.f;
      if (b >= nbw) {
        acc[b] = 0.f;
        continue;
      }
#pragma unroll
      for (int c = 0; c < CPL; ++c) {
        const float4 x = v[b][c];
        if (METRIC == kL2) {
          float d0 = Q.q[c].x - x.x, d1 = Q.q[c].y - x.y, d2 = Q.q[c].z - x.z, d3 = Q.q[c].w - x.w;
          a = fmaf(d0, d0, a); a = fmaf(d1, d1, a); a = fmaf(d2, d2, a); a = fmaf(d3, d3, a);
        } else {
          a = fmaf(Q.q[c].x, x.x, a); a = fmaf(Q.q[c].y, x.y, a);
          a = fmaf(Q.q[c].z, x.z, a); a = fmaf(Q.q[c].w, x.w, a);
        }
      }
      acc[b] = a;
    }
#endif
#pragma unroll
    for (int o = TL >> 1; o > 0; o >>= 1)
#pragma unroll
      for (int b = 0; b < B; ++b)
        if (b < nbw) acc[b] += __shfl_xor_sync(0xffffffffu, acc[b], o);
    // compaction: one ballot per row group; lane 0 reserves the warp's slots
    unsigned m[B];
    int tot = 0;
#pragma unroll
    for (int b = 0; b < B; ++b) {
      const int j = base + b * NTEAMS + team;
      uint64_t key = kKeyMax;
      if (b < nbw && tl == 0 && j < Mc && !lost[b]) key = make_key((METRIC == kL2) ? acc[b] : -acc[b], ids[b]);
      m[b] = b < nbw ? __ballot_sync(0xffffffffu, key < worst) : 0u;
      tot += __popc(m[b]);
      // a key that enters the list is a likely parent of the next step(s):
      // pull its graph row into L2 now (prefetch bit 8, on by default;
      // results unaffected)
      if (gcache != nullptr && key < worst) {
        // graph-row cache: the row of a key entering the list goes to shared
        // memory now (16-B cp.async by this lane, waited for before the
        // step's last barrier), one copy per cache slot and step
        const uint32_t slot = hash_slot(ids[b], cfg.gc_bits);
        uint32_t* tags = gcache + ((1u << cfg.gc_bits) << cfg.rp_shift);
        if (atomicExch(tags + (1u << cfg.gc_bits) + slot, gc_stamp) != gc_stamp) {
          tags[slot] = ids[b];
          const uint32_t* src = cfg.graph + ((uint64_t)ids[b] << cfg.rp_shift);
          uint32_t* dst = gcache + (slot << cfg.rp_shift);
          for (int c = 0; c < (1 << cfg.rp_shift); c += 4) cp_async16(dst + c, src + c);
          asm volatile("cp.async.commit_group;" ::: "memory");
        }
      } else if ((cfg.prefetch & 8) && key < worst)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.graph + ((uint64_t)ids[b] << cfg.rp_shift)),
                     "r"(4u << cfg.rp_shift)
                     : "memory");
      acc[b] = __uint_as_float((uint32_t)(key >> 32));  // keep the key's high word (id is in ids[b])
    }
    if (tot > 0) {
      int wbase = 0;
      if (lane == 0) wbase = atomicAdd(nkeys, tot);
      wbase = __shfl_sync(0xffffffffu, wbase, 0);
      const unsigned lt = (1u << lane) - 1u;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        if (m[b] & (1u << lane))
          newk[wbase + __popc(m[b] & lt)] = ((uint64_t)__float_as_uint(acc[b]) << 32) | ((uint64_t)ids[b] << 1);
        wbase += __popc(m[b]);
      }
    }
  }
}

// Distance step, gather mode 3 (P:L217 step 3): like dist_ldg, but the rows
// of a pass land in shared memory through 16-B cp.async (LDGSTS) issued by
// the lanes that will reduce them -- team t owns staging slots [t*BS, t*BS+BS),
// lane tl copies chunks tl, tl+TL, ... of each of its team's rows -- so a pass
// holds NTEAMS*BS rows in flight with no data registers (the register path's
// rows per pass are capped by the 64-register budget of a 1024-thread CTA),
// and a lane only waits for its own copies (cp.async.wait_group), no CTA
// barrier.  Padded tail chunks of a slot are never written (zero since
// init_cta).  Keys < worst are appended to newk (ballot + one atomic per
// warp and row group).
template <int NT, int TL, int CPL, int METRIC>
__device__ __forceinline__ void dist_async(const SearchCfg& cfg, const float4* qs, float4* stage, int M,
                                           uint64_t worst, const uint32_t* newid, uint64_t* newk, int* nkeys) {
  const int tid = threadIdx.x, lane = tid & 31;
  constexpr int NTEAMS = NT / TL;
  constexpr int TPW = 32 / TL;  // teams per warp
  const int team = tid / TL, tl = tid % TL;
  const int wteam0 = (tid >> 5) * TPW;
  const int BS = cfg.team_rows;
  const int PASS = NTEAMS * BS;
  QueryRegs<TL, CPL> Q;
  Q.load(qs, tl);
  for (int base = 0; base < M; base += PASS) {
    int nb = (M - base - wteam0 + NTEAMS - 1) / NTEAMS;  // row groups holding rows of this warp
    if (nb <= 0) continue;
    if (nb > BS) nb = BS;
    for (int b = 0; b < nb; ++b) {
      const int j = base + b * NTEAMS + team;
      if (j < M) {
        const float4* row = cfg.data + (uint64_t)newid[j] * cfg.d4;
        float4* dst = stage + (size_t)(team * BS + b) * cfg.dp4;
#pragma unroll
        for (int c = 0; c < CPL; ++c) {
          const int chn = tl + c * TL;
          if (chn < cfg.d4) cp_async16(dst + chn, row + chn);
        }
      }
    }
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
    for (int b = 0; b < nb; ++b) {
      const int j = base + b * NTEAMS + team;
      float a = team_partial_smem<TL, CPL, METRIC>(Q, stage + (size_t)(team * BS + b) * cfg.dp4, tl);
#pragma unroll
      for (int o = TL >> 1; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
      uint64_t key = kKeyMax;
      uint32_t id = 0;
      if (tl == 0 && j < M) {
        id = newid[j];
        key = make_key((METRIC == kL2) ? a : -a, id);
      }
      const bool keep = key < worst;
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      if (keep && (cfg.prefetch & 8))  // its graph row: a likely parent of the next step(s)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.graph + ((uint64_t)id << cfg.rp_shift)),
                     "r"(4u << cfg.rp_shift)
                     : "memory");
      if (m) {
        int wbase = 0;
        if (lane == 0) wbase = atomicAdd(nkeys, __popc(m));
        wbase = __shfl_sync(0xffffffffu, wbase, 0);
        if (keep) newk[wbase + __popc(m & ((1u << lane) - 1u))] = key;
      }
    }
  }
}

// Distance step, gather mode 4 (hybrid): the rows beyond the first register
// pass (rows NTEAMS .. NTEAMS*(1+BS)) are put in flight FIRST as team-local
// cp.async copies into shared memory, then the first NTEAMS rows go through
// the register pass (dist_ldg), then each lane waits for its own copies and
// reduces the staged rows -- the two waves' memory latencies overlap instead
// of following each other.  Rows past both waves: further register passes.
template <int NT, int TL, int CPL, int METRIC, int MINB>
__device__ __forceinline__ void dist_hybrid(const SearchCfg& cfg, const float4* qs, float4* stage, int M,
                                            uint64_t worst, const uint32_t* newid, uint64_t* newk, int* nkeys) {
  const int tid = threadIdx.x, lane = tid & 31;
  constexpr int B1 = DistRows<NT, TL, CPL, MINB>::B;  // rows per team of the register wave
  constexpr int NTEAMS = NT / TL;
  constexpr int W1 = NTEAMS * B1;                     // rows of the register wave
  constexpr int TPW = 32 / TL;
  const int team = tid / TL, tl = tid % TL;
  const int wteam0 = (tid >> 5) * TPW;
  const int BS = cfg.team_rows;
  // wave 2 in flight first (no registers held)
  for (int b = 0; b < BS; ++b) {
    const int j = W1 + b * NTEAMS + team;
    if (j < M) {
      const float4* row = cfg.data + (uint64_t)newid[j] * cfg.d4;
      float4* dst = stage + (size_t)(team * BS + b) * cfg.dp4;
#pragma unroll
      for (int c = 0; c < CPL; ++c) {
        const int chn = tl + c * TL;
        if (chn < cfg.d4) cp_async16(dst + chn, row + chn);
      }
    }
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
  // wave 1: the register pass over rows [0, W1)
  dist_ldg<NT, TL, CPL, METRIC, B1>(cfg, qs, M < W1 ? M : W1, 0, 1, worst, newid, newk, nkeys);
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  QueryRegs<TL, CPL> Q;
  Q.load(qs, tl);
  for (int b = 0; b < BS; ++b) {
    if (W1 + b * NTEAMS + wteam0 >= M) break;  // warp-uniform: no row of this warp left
    const int j = W1 + b * NTEAMS + team;
    float a = team_partial_smem<TL, CPL, METRIC>(Q, stage + (size_t)(team * BS + b) * cfg.dp4, tl);
#pragma unroll
    for (int o = TL >> 1; o > 0; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
    uint64_t key = kKeyMax;
    uint32_t id = 0;
    if (tl == 0 && j < M) {
      id = newid[j];
      key = make_key((METRIC == kL2) ? a : -a, id);
    }
    const bool keep = key < worst;
    const unsigned m = __ballot_sync(0xffffffffu, keep);
    if (keep && (cfg.prefetch & 8))
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.graph + ((uint64_t)id << cfg.rp_shift)),
                   "r"(4u << cfg.rp_shift)
                   : "memory");
    if (m) {
      int wbase = 0;
      if (lane == 0) wbase = atomicAdd(nkeys, __popc(m));
      wbase = __shfl_sync(0xffffffffu, wbase, 0);
      if (keep) newk[wbase + __popc(m & ((1u << lane) - 1u))] = key;
    }
  }
  // rows past both waves (large steps): more register passes
  const int done = W1 + NTEAMS * BS;
  if (M > done) dist_ldg<NT, TL, CPL, METRIC, B1>(cfg, qs, M, done, 1, worst, newid, newk, nkeys);
}

// Warp-level bitonic merge ("parallel-friendly bitonic sort", the
// beam-extend candidate update of BASELINE north_star (2)): the sorted list
// (cnt <= 32 keys, one per lane) absorbs nk unsorted new keys 32 at a time --
// bitonic sort of the block in registers, reversed, lane-wise min against
// the list (the 32 smallest of the union, a bitonic sequence), 5-stage
// bitonic merge.  Writes the first L (<= 32) keys to dst.  Warp-uniform.
constexpr int kWarpMergeMax = 128;  // new keys: one block per warp of warps 0..3
__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a < b ? b : a; }
// bitonic sort of one key per lane, ascending across the warp
__device__ __forceinline__ uint64_t warp_bitonic_sort32(uint64_t x, int lane) {
#pragma unroll
  for (int kk = 2; kk <= 32; kk <<= 1) {
#pragma unroll
    for (int j = kk >> 1; j > 0; j >>= 1) {
      const uint64_t y = __shfl_xor_sync(0xffffffffu, x, j);
      const bool keep_min = ((lane & j) == 0) == ((lane & kk) == 0);
      x = keep_min ? umin64(x, y) : umax64(x, y);
    }
  }
  return x;
}
// merge an ascending block (one key per lane) into the ascending list (one
// key per lane): reverse the block, lane-wise min (the 32 smallest of the
// union, bitonic), 5-stage bitonic merge -> the first 32 of the union
__device__ __forceinline__ uint64_t warp_bitonic_merge32(uint64_t list, uint64_t sorted_block, int lane) {
  uint64_t m = umin64(list, __shfl_sync(0xffffffffu, sorted_block, 31 - lane));
#pragma unroll
  for (int j = 16; j > 0; j >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, m, j);
    m = ((lane & j) == 0) ? umin64(m, y) : umax64(m, y);
  }
  return m;
}

// ---- select (P:L217 step 1) from the registers of warp 0 (list striped:
// lane l, register e = position 32e + l): the first w unchecked keys in list
// order (one under greedy search), R6/R7, marked checked; the first L keys
// are written to dst and the step's control words updated.
template <int E>
__device__ __forceinline__ void warp_select_store(const SearchCfg& cfg, const Smem& s, Ctrl* C, int lane,
                                                  uint64_t (&x)[E], uint64_t* dst, int L, int W, int OFF, int sp,
                                                  uint32_t liters, int cur, int lcnt) {
  int tot = 0, first_un = -1;
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const unsigned um = __ballot_sync(0xffffffffu, 32 * e + lane < lcnt && !(x[e] & 1ull));
    if (first_un < 0 && um) first_un = 32 * e + __ffs(um) - 1;
    tot += __popc(um);
  }
  const int diff0 = __shfl_sync(0xffffffffu, lane == 0 ? C->diffusing : 0, 0);
  int done = 0, np = 0, diff = diff0;
  if (tot == 0) {
    done = 1;
  } else if ((int)liters >= cfg.max_iter) {
    done = 1;
    if (lane == 0) C->cap_hit = 1;
  } else {
    if (first_un >= OFF) diff = 1;        // P:L249 (sticky, R6)
    np = diff ? (tot < W ? tot : W) : 1;
    int base = 0;
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const bool un = 32 * e + lane < lcnt && !(x[e] & 1ull);
      const unsigned um = __ballot_sync(0xffffffffu, un);
      const int rank = base + __popc(um & ((1u << lane) - 1u));
      if (un && rank < np) {
        s.sel[32 + rank] = (int)key_id(x[e]);
        x[e] |= 1ull;                           // mark checked (Alg.1 l.7)
      }
      base += __popc(um);
    }
  }
#pragma unroll
  for (int e = 0; e < E; ++e)
    if (32 * e + lane < L) dst[32 * e + lane] = x[e];
  if (lane == 0) {
    C->diffusing = diff;
    C->done = done;
    C->np = np;
    C->nnew[sp ^ 1] = 0;
    C->nkeys[sp ^ 1] = 0;
    if (!done) C->parents += np;
    C->cur = cur;
    C->cnt = lcnt;
  }
}

// Candidate update of the fused path ("parallel-friendly bitonic
// sort ... merges the candidate list and expand list"), for lists of up to
// Lp = 32*E keys: warp 0 holds the sorted list in registers, STRIPED (lane l,
// register e = list position 32*e + l), and absorbs the step's new keys one
// sorted block of 32 at a time (block 0 sorted here, blocks 1.. by warps
// 1.. meanwhile).  Inserting block B: C[i] = min(A[i], B'[Lp-1-i]) with B'
// = B padded by +inf -- only the last register row changes, and C holds the
// Lp smallest keys of A u B as a bitonic sequence -- then a bitonic merge
// network sorts C: strides 32m (m = E/2 .. 1) compare registers e, e|m of a
// lane, strides 16 .. 1 compare lanes (shuffle xor).  A block whose
// smallest key is >= the list's Lp-th key cannot enter and is skipped.
// Then the next step's parents are selected from the registers (P:L217 step
// 1, R6/R7) and the first L keys are written to dst.  Warp-uniform; only
// lane 0 reads/writes the Ctrl fields it owns.
template <int E, int NT>
__device__ __forceinline__ void warp_merge_select(const SearchCfg& cfg, const Smem& s, Ctrl* C, int lane, int cnt,
                                                  int nk, int nblk, const uint64_t* sorted2, int L, int W, int OFF,
                                                  int sp, uint32_t& liters, int np_step, int& cur, int& lcnt) {
  const uint64_t* src = cur ? s.list[1] : s.list[0];
  uint64_t* dst = cur ? s.list[0] : s.list[1];
  uint64_t x[E];
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int i = 32 * e + lane;
    x[e] = i < cnt ? src[i] : kKeyMax;
  }
  if (nk > 0) {
    for (int b = 0; b < nblk; ++b) {
      uint64_t blk;
      if (b == 0 || NT < 128) {
        blk = warp_bitonic_sort32(32 * b + lane < nk ? s.newk[32 * b + lane] : kKeyMax, lane);
      } else {
        if (b == 1) asm volatile("bar.sync 1, %0;" ::"r"(32 * nblk) : "memory");
        blk = sorted2[32 * b + lane];
      }
      const uint64_t last = __shfl_sync(0xffffffffu, x[E - 1], 31);
      if (__shfl_sync(0xffffffffu, blk, 0) >= last) continue;  // nothing of it can enter
      x[E - 1] = umin64(x[E - 1], __shfl_sync(0xffffffffu, blk, 31 - lane));
#pragma unroll
      for (int m = E >> 1; m > 0; m >>= 1) {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          if (!(e & m)) {
            const uint64_t a = x[e], c = x[e | m];
            x[e] = umin64(a, c);
            x[e | m] = umax64(a, c);
          }
        }
      }
#pragma unroll
      for (int j = 16; j > 0; j >>= 1) {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const uint64_t y = __shfl_xor_sync(0xffffffffu, x[e], j);
          x[e] = (lane & j) ? umax64(x[e], y) : umin64(x[e], y);
        }
      }
    }
    cur ^= 1;
    lcnt = (cnt + nk) < L ? cnt + nk : L;
  } else {
    dst = const_cast<uint64_t*>(src);
  }
  liters += np_step > 0 ? 1 : 0;
  warp_select_store<E>(cfg, s, C, lane, x, dst, L, W, OFF, sp, liters, cur, lcnt);
}

// Candidate update for lists of <= 32*E keys, fused with the next
// select: a merge BY RANK in parallel warps instead of warp 0's bitonic
// networks.  New key i goes to position #(new keys < it) + #(list keys < it)
// (a lower bound in the sorted list), list key j to j + #(new keys < it);
// keys are unique, so the positions are a permutation and the first L form
// the merged list -- the same list the bitonic merge produces.  Warps
// 0..nblk-1 place the new keys (32 each, <= 128), warps nblk..nblk+E-1 the
// list keys (32 each), each comparison a shared-memory broadcast read; one
// named barrier, then warp 0 selects from the merged list.  Needs
// NT >= 32 * (4 + E).
template <int E, int NT>
__device__ __forceinline__ void rank_merge_select(const SearchCfg& cfg, const Smem& s, Ctrl* C, int warp, int lane,
                                                  int cnt, int nk, int L, int W, int OFF, int sp, uint32_t& liters,
                                                  int np_step, int& cur, int& lcnt) {
  const uint64_t* src = cur ? s.list[1] : s.list[0];
  uint64_t* dst = cur ? s.list[0] : s.list[1];
  const int nblk = (nk + 31) >> 5;
  const int nlw = (cnt + 31) >> 5;  // list warps (<= E)
  if (nk > 0 && warp < nblk + nlw) {
    if (warp < nblk) {
      const int i = 32 * warp + lane;
      if (i < nk) {
        const uint64_t key = s.newk[i];
        int r = lower_bound_u64(src, cnt, key);
        for (int j = 0; j < nk; ++j) r += (s.newk[j] < key) ? 1 : 0;
        if (r < L) dst[r] = key;
      }
    } else {
      const int i = 32 * (warp - nblk) + lane;
      if (i < cnt) {
        const uint64_t key = src[i];
        int r = i;
        for (int j = 0; j < nk; ++j) r += (s.newk[j] < key) ? 1 : 0;
        if (r < L) dst[r] = key;
      }
    }
    asm volatile("bar.sync 1, %0;" ::"r"(32 * (nblk + nlw)) : "memory");
  }
  if (warp == 0) {
    if (nk > 0) {
      cur ^= 1;
      lcnt = (cnt + nk) < L ? cnt + nk : L;
    } else {
      dst = const_cast<uint64_t*>(src);
    }
    liters += np_step > 0 ? 1 : 0;
    uint64_t x[E];
#pragma unroll
    for (int e = 0; e < E; ++e) x[e] = 32 * e + lane < lcnt ? dst[32 * e + lane] : kKeyMax;
    warp_select_store<E>(cfg, s, C, lane, x, dst, L, W, OFF, sp, liters, cur, lcnt);
  }
}

// COSINE (R29): q <- q / |q| in shared memory, by warp 0, between two CTA
// barriers (the staging threads' stores are visible to warp 0 after the
// first; everyone reads the unit query after the second).  Every CTA of a
// query computes the same fp32 value in the same order.  Zero query: kept.
template <int NT>
__device__ __forceinline__ void normalize_query(float4* q, int d4) {
  __syncthreads();
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    float ss = 0.f;
    for (int i = lane; i < d4; i += 32) {
      const float4 v = q[i];
      ss = fmaf(v.x, v.x, fmaf(v.y, v.y, fmaf(v.z, v.z, fmaf(v.w, v.w, ss))));
    }
    for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
    if (ss > 0.f) {
      const float inv = 1.0f / sqrtf(ss);
      for (int i = lane; i < d4; i += 32) {
        float4 v = q[i];
        v.x *= inv; v.y *= inv; v.z *= inv; v.w *= inv;
        q[i] = v;
      }
    }
  }
  __syncthreads();
}

// Per-query search parameters that may differ from the launch's SearchCfg
// (a server query can ask for a smaller L / w): passed by value so the
// SearchCfg itself stays in the kernel's parameter space (a local copy of the
// whole struct would occupy registers for the life of the kernel).
struct QPar {
  int L, w, off;
};
__host__ __device__ inline QPar qpar_of(const SearchCfg& c) { return QPar{c.L, c.w, c.off}; }

// Preconditions: s.q holds the query (d4 float4, zero tail); init_cta() ran.
// Writes min(k, |list|) results to out[0..k) (rest padded) and the CTA's
// counters to *st.  CS > 1: this CTA is the leader of a cluster whose
// other CTAs run search_worker() in lock step (two cluster barriers per step).
template <int NT, int TL, int CPL, int METRIC, int CS = 1, int MINB = 1>
__device__ void search_cta(const SearchCfg& cfg, const QPar qp, const Smem& s, uint64_t tag, uint32_t cta_rank,
                           int k, unsigned long long* gtab, uint32_t epoch, ResultEntry* out, CtaStats* st,
                           uint32_t* vbm = nullptr) {
  const int tid = threadIdx.x;
  const int lane = tid & 31;
  const int warp = tid >> 5;
  constexpr int NTEAMS = NT / TL;
  const int team = tid / TL;
  const int tl = tid % TL;
  Ctrl* C = s.ctrl;
  const int L = qp.L, W = qp.w, OFF = qp.off;
  const int hbits = cfg.hash_bits;
  const int hcap = 1 << hbits;
  const int Rp = 1 << cfg.rp_shift;
  const int step_max_new = W * Rp;

  if (tid == 0 && st) st->t_entry = globaltimer();
  // ---- reset per-query state (16-B stores)
  {
    uint4* h4 = reinterpret_cast<uint4*>(s.hash);
    const uint4 e = make_uint4(kHashEmpty, kHashEmpty, kHashEmpty, kHashEmpty);
    for (int i = tid; i < (hcap >> 2); i += NT) h4[i] = e;
  }
  if (tid == 0) {
    C->cnt = 0; C->nnew[0] = C->nnew[1] = 0; C->nkeys[0] = C->nkeys[1] = 0; C->np = 0; C->done = 0;
    C->diffusing = 0;
    C->vis_count = 0; C->spilled = 0; C->overflow = 0; C->cur = 0;
    C->iters = 0; C->parents = 0; C->dist_evals = 0; C->cap_hit = 0; C->mg_bitonic = 0; C->mg_rank = 0;
  }
  uint32_t phase = C->phase;  // staging-barrier parities carried across queries
  __syncthreads();

  // ---- entry points (Alg.1 l.5): S seeds, duplicates dropped.
  // One thread per seed, all inserted at once: the shared-memory hash's
  // test-and-set lets exactly one copy of a repeated id through, so the
  // visited set and the new-id list hold the deduplicated seed set (its
  // order in newid is irrelevant: the merge places keys by value).
  for (int j = tid; j < ((cfg.S + 31) & ~31); j += NT) {
    bool keep = false;
    uint32_t e = kSentinel;
    if (j < cfg.S) {
      e = entry_point(cfg.seed, tag, cta_rank, (uint32_t)j, cfg.n);
      keep = smem_visit(s.hash, hbits, e) == kVisNew;
      // SHARED: a CTA keeps its own seeds even when another CTA of the
      // query claimed them first (R21), but marks them for the others
      if (keep && cfg.shared && (vbm || cfg.vis_dsmem)) {
        // (the returned word is consumed: the claim is performed before this
        // thread reaches the next query's relaxed start barrier)
        const bool c = vis_claim(cfg, s.vsh, vbm, e);
        asm volatile("" ::"r"((int)c));
      }
      else if (keep && cfg.shared && gtab) (void)gmem_visit(gtab, cfg.gtab_bits, epoch, e);
    }
    const unsigned m = __ballot_sync(0xffffffffu, keep);
    if (m) {
      int wbase = 0;
      if (lane == 0) wbase = atomicAdd(&C->nnew[0], __popc(m));
      wbase = __shfl_sync(0xffffffffu, wbase, 0);
      if (keep) s.newid[wbase + __popc(m & ((1u << lane) - 1u))] = e;
    }
  }
  __syncthreads();
  if (tid == 0) C->vis_count = C->nnew[0];

  if (tid == 0 && st) st->t_loop0 = globaltimer();
  // per-phase SM cycles (thread 0; the paper's calc/sort split, Fig. 3/17),
  // kept in shared memory: registers held across the whole search loop
  // would spill under the 64-register budget of a 1024-thread CTA
  if (tid == 0) {
    C->cyc[0] = C->cyc[1] = C->cyc[2] = C->cyc[3] = 0;  // select, gather+filter, distance, merge
    C->tp = clock64();
  }
  auto lap = [&](int ph) {
    if (tid == 0) {
      const long long t = clock64();
      C->cyc[ph] += (unsigned long long)(t - C->tp);
      C->tp = t;
    }
  };

  int cur = 0;
  int lcnt = 0;            // list length (uniform register copy in every thread)
  uint32_t liters = 0;     // steps taken
  bool first = true;
  int sp = 0;              // step parity: which nnew/nkeys counters this step uses (0 for clusters)
  bool pre = false;        // the next step's parents were already selected (fused path)
  int np_step = 0;         // parents of the current step
  // graph-row cache (single-CTA searches on the register gather path)
  uint32_t* const gcache = (CS == 1 && cfg.gc_bits > 0 && cfg.gather_mode == 0) ? s.gcache : nullptr;
  uint32_t gstamp = C->gc_stamp;  // read after the seeding barrier; advanced per step

  // ---- select (warp 0, P:L217 step 1): the first w unchecked candidates of
  // the list (one under greedy search), marked checked; resets the step
  // counters [ri] of the step it selects for
  auto select_parents = [&](int ri) {
    const int cnt = lcnt;
    uint64_t* list = cur ? s.list[1] : s.list[0];
    // also look past the parents: the next few unchecked candidates are
    // the likely parents of the next step, whose graph rows are
    // prefetched into L2 now (prefetch bit 1; results are unaffected)
    const int pf = (cfg.prefetch & 2) ? (W < 16 ? W : 32 - W) : 0;
    const int want = W + pf;
    int found = 0;
    for (int base = 0; base < cnt && found < want; base += 32) {
      int i = base + lane;
      bool un = (i < cnt) && !(list[i] & 1ull);
      unsigned m = __ballot_sync(0xffffffffu, un);
      int rank = found + __popc(m & ((1u << lane) - 1u));
      if (un && rank < want) s.sel[rank] = i;
      found += __popc(m);
    }
    const int found_all = found < want ? found : want;
    if (found > W) found = W;
    __syncwarp();
    int done = 0, np = 0;
    if (found == 0) {
      done = 1;
    } else if ((int)liters >= cfg.max_iter) {
      done = 1;
      if (lane == 0) C->cap_hit = 1;
    } else {
      int diff = __shfl_sync(0xffffffffu, lane == 0 ? C->diffusing : 0, 0);  // lane 0 owns the word
      if (s.sel[0] >= OFF) diff = 1;              // P:L249 (sticky, R6)
      np = diff ? found : 1;
      if (lane < np) {
        int pos = s.sel[lane];
        uint64_t kk = list[pos];
        list[pos] = kk | 1ull;                    // mark checked (Alg.1 l.7)
        s.sel[32 + lane] = (int)key_id(kk);
      } else if (lane < found_all) {
        const uint32_t nid = key_id(list[s.sel[lane]]);
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.graph + ((uint64_t)nid << cfg.rp_shift)),
                     "r"(4u << cfg.rp_shift)
                     : "memory");
      }
      if (lane == 0) C->diffusing = diff;
    }
    if (lane == 0) {
      C->done = done;
      C->np = np;
      C->nnew[ri] = 0;
      C->nkeys[ri] = 0;
      if (!done) { C->parents += np; }
      // switch to the HBM spill table before the shared one gets too full
      if (!C->spilled && gtab != nullptr && C->vis_count + step_max_new > (hcap * 3) / 4) C->spilled = 1;
    }
  };

  for (;;) {
    // ================= select (warp 0) =================
    if (!first) {
      if (CS == 1) sp ^= 1;
      if (!pre) {
        if (warp == 0) select_parents(sp);
        __syncthreads();
      }
      pre = false;
      lap(0);
      if (C->done) break;

      // ================= gather + visited filter (P:L217 steps 1-2) =================
      {
        const int np = C->np;
        np_step = np;
        const int spilled = C->spilled;
        const int total = np << cfg.rp_shift;  // one neighbour id per thread and pass
        // SHARED with the query's bitmap: no CTA-local hash in the step
        // (prefetch bit 2048 keeps it as a filter in front of the claim, A/B)
        const bool bitmap_only =
            cfg.shared && (cfg.vis_dsmem || (vbm != nullptr && !(cfg.prefetch & 256))) && !(cfg.prefetch & 2048);
        for (int base = 0; base < total; base += NT) {
          const int idx = base + tid;
          uint32_t id = kSentinel;
          if (idx < total) {
            const uint32_t parent = (uint32_t)s.sel[32 + (idx >> cfg.rp_shift)];
            const uint32_t slot = gcache ? hash_slot(parent, cfg.gc_bits) : 0u;
            if (gcache && gcache[((1u << cfg.gc_bits) << cfg.rp_shift) + slot] == parent) {
              id = gcache[(slot << cfg.rp_shift) + (idx & (Rp - 1))];  // cached row (shared memory)
            } else {
              const uint32_t* gp = cfg.graph + ((uint64_t)parent << cfg.rp_shift) + (idx & (Rp - 1));
              id = (cfg.prefetch & 4) ? ldg_u32_hint(gp, l2_evict_last_policy()) : __ldg(gp);
            }
          }
          bool keep = false;
          if (id != kSentinel) {
            if (bitmap_only) {
              // SHARED bitmap: it holds every point this CTA has
              // visited too (own seeds included, R21), so it alone is the
              // visited set -- one atomic, no shared-memory hash probe
              // (measured ~900 cycles per step, the ATOMS.CAS test-and-set)
              keep = vis_claim(cfg, s.vsh, vbm, id);
            } else if (!spilled) {
              const int r = smem_visit(s.hash, hbits, id);
              keep = (r == kVisNew);
              if (r == kVisFull) atomicOr(&C->overflow, 1);
              // bit 16: the row of an id new to this CTA is pulled into L2
              // now, so its DRAM fetch overlaps the shared claim, the
              // compaction and the barrier (wasted only if another CTA
              // claimed it first)
              if (keep && (cfg.prefetch & 16))
                asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.data + (uint64_t)id * cfg.d4),
                             "r"((uint32_t)cfg.d4 * 16u)
                             : "memory");
              if (keep && (cfg.prefetch & 32)) {  // same with plain per-line L2 prefetches
                const char* rp = reinterpret_cast<const char*>(cfg.data + (uint64_t)id * cfg.d4);
                for (int o = 0; o < cfg.d4 * 16; o += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(rp + o));
              }
              if (keep && cfg.shared) {  // new to this CTA: claim it in the query's table (P:L211, P:L217 step 2)
                if (vbm || cfg.vis_dsmem) {  // the paper's bitmap: one atomic, no probing --
                  if (!(cfg.prefetch & 256) || cfg.vis_dsmem) {  // (A/B, bit 256: with the row's loads in dist_ldg instead --
                                                  //  measured slower: the rows other CTAs won cost more
                                                  //  than the round trip saved, profiles/round2_ab.md)
                    keep = vis_claim(cfg, s.vsh, vbm, id);
                  }
                } else {
                  const int g = gmem_visit(gtab, cfg.gtab_bits, epoch, id);
                  keep = (g == kVisNew);
                  if (g == kVisFull) atomicOr(&C->overflow, 1);
                }
              }
            } else if (vbm || cfg.vis_dsmem) {
              if (!smem_contains(s.hash, hbits, id)) keep = vis_claim(cfg, s.vsh, vbm, id);
            } else if (!smem_contains(s.hash, hbits, id)) {
              const int r = gmem_visit(gtab, cfg.gtab_bits, epoch, id);
              keep = (r == kVisNew);
              if (r == kVisFull) atomicOr(&C->overflow, 1);
            }
          }
          if (keep && (cfg.prefetch & 1)) {
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(cfg.data + (uint64_t)id * cfg.d4),
                         "r"((uint32_t)cfg.d4 * 16u)
                         : "memory");
          }
          const unsigned m = __ballot_sync(0xffffffffu, keep);
          if (m) {
            int wbase = 0;
            if (lane == 0) wbase = atomicAdd(&C->nnew[sp], __popc(m));
            wbase = __shfl_sync(0xffffffffu, wbase, 0);
            if (keep) s.newid[wbase + __popc(m & ((1u << lane) - 1u))] = id;
          }
        }
        __syncthreads();
        if (tid == 0 && !spilled) C->vis_count += C->nnew[sp];
        lap(1);
      }
    }
    const bool first_pass = first;  // the seeding pass: its ids are the CTA's seeds
    first = false;

    // ================= distances (P:L217 step 3) + prefilter =================
    {
      const int M = C->nnew[sp];
      const int cnt = lcnt;
      const uint64_t worst = (cnt >= L) ? (cur ? s.list[1] : s.list[0])[L - 1] : kKeyMax;
      if (cfg.gather_mode == 0) {
        if constexpr (CS > 1) {
          // hand worker c the rows r = c, c+CS, ... (ids pushed into its shared
          // memory), its row count and the prefilter key, then signal it
          for (int r = tid; r < M; r += NT) {
            const int c = r % CS;
            if (c) rank_ptr(s.newid, c)[r / CS] = s.newid[r];
          }
          __syncthreads();
          if (tid < CS - 1) {  // one thread per worker
            const int c = tid + 1;
            Ctrl* wc = rank_ptr(C, c);
            wc->w_cmd = kCmdStep;
            wc->w_m = M > c ? (M - c + CS - 1) / CS : 0;
            wc->w_worst = worst;
            fence_cluster();
            mbar_remote_arrive(s.bar + 2, c);
          }
          dist_ldg<NT, TL, CPL, METRIC, DistRows<NT, TL, CPL, MINB>::B>(cfg, s.q, M, 0, CS, worst, s.newid, s.newk,
                                                                        &C->nkeys[0]);
          mbar_wait_cluster(s.bar + 3, (phase >> 3) & 1u);  // all workers' keys delivered
          phase ^= 8u;
          __syncthreads();
        } else {
          ++gstamp;
          // prefetch bit 256 (A/B): SHARED bitmap claims ride with the row
          // loads (not for the seeds: a CTA keeps its own seeds, R21; not
          // after a spill, whose filter claims at filter time)
          uint32_t* claim = (vbm != nullptr && !first_pass && !C->spilled && (cfg.prefetch & 256)) ? vbm : nullptr;
          dist_ldg<NT, TL, CPL, METRIC, DistRows<NT, TL, CPL, MINB>::B>(cfg, s.q, M, 0, 1, worst, s.newid, s.newk,
                                                                      &C->nkeys[sp], gcache, gstamp, claim);
          __syncthreads();
        }
      }
#if ALGAS_GATHER_EXPERIMENTS
      // measured alternatives of the vector gather (compiled
      // only into A/B builds: their code paths cost the production kernel
      // registers)
      else if (cfg.gather_mode == 3) {
        dist_async<NT, TL, CPL, METRIC>(cfg, s.q, s.stage, M, worst, s.newid, s.newk, &C->nkeys[sp]);
        __syncthreads();
      } else if (cfg.gather_mode == 4) {
        dist_hybrid<NT, TL, CPL, METRIC, MINB>(cfg, s.q, s.stage, M, worst, s.newid, s.newk, &C->nkeys[sp]);
        __syncthreads();
      }
      const int SR = cfg.stage_rows;
      const int nchunks = (cfg.gather_mode == 1 || cfg.gather_mode == 2) ? (M + SR - 1) / SR : 0;
      if (nchunks > 0) stage_issue<NT>(cfg, s, 0, 0, M < SR ? M : SR, warp, lane);
      QueryRegs<TL, CPL> Q;  // staged paths: the query in registers for the chunk loop
      if (nchunks > 0) Q.load(s.q, tl);
      for (int ch = 0; ch < nchunks; ++ch) {
        const int b = ch & 1;
        if (ch + 1 < nchunks) {
          const int r1 = (ch + 1) * SR;
          stage_issue<NT>(cfg, s, b ^ 1, r1, (M - r1) < SR ? (M - r1) : SR, warp, lane);
        }
        if (cfg.gather_mode == 2) {
          mbar_wait(s.bar + b, (phase >> b) & 1u);
          phase ^= (1u << b);
        } else {
          if (ch + 1 < nchunks) asm volatile("cp.async.wait_group 1;" ::: "memory");
          else asm volatile("cp.async.wait_group 0;" ::: "memory");
          __syncthreads();
        }
        const int r0 = ch * SR;
        const int rows = (M - r0) < SR ? (M - r0) : SR;
        const float4* buf = s.stage + (size_t)b * SR * cfg.dp4;
        // each team reduces RB rows at once (independent shuffle trees
        // interleave); rows past `rows` compute garbage that is masked
        constexpr int RB = (CPL <= 4) ? 4 : (CPL <= 8 ? 2 : 1);
        for (int base = 0; base < rows; base += NTEAMS * RB) {
          float acc[RB];
#pragma unroll
          for (int j = 0; j < RB; ++j) {
            const int r = base + team + j * NTEAMS;
            const int rr = r < SR ? r : SR - 1;
            acc[j] = team_partial_smem<TL, CPL, METRIC>(Q, buf + (size_t)rr * cfg.dp4, tl);
          }
#pragma unroll
          for (int o = TL >> 1; o > 0; o >>= 1)
#pragma unroll
            for (int j = 0; j < RB; ++j) acc[j] += __shfl_xor_sync(0xffffffffu, acc[j], o);
#pragma unroll
          for (int j = 0; j < RB; ++j) {
            const int r = base + team + j * NTEAMS;
            const bool valid = (tl == 0) && (r < rows);
            uint64_t key = kKeyMax;
            if (valid) key = make_key((METRIC == kL2) ? acc[j] : -acc[j], s.newid[r0 + r]);
            const bool keep = valid && (key < worst);
            const unsigned m = __ballot_sync(0xffffffffu, keep);
            if (m) {
              int wbase = 0;
              if (lane == 0) wbase = atomicAdd(&C->nkeys[sp], __popc(m));
              wbase = __shfl_sync(0xffffffffu, wbase, 0);
              if (keep) s.newk[wbase + __popc(m & ((1u << lane) - 1u))] = key;
            }
          }
        }
        __syncthreads();  // buffer b fully read before it is re-issued (chunk ch+2)
      }
#endif
      if (tid == 0) C->dist_evals += M;
      lap(2);
    }

    // ================= merge the new keys into the list (P:L219 step 4) =================
    // position of a new key = its rank among the new keys + the number of
    // list keys below it; position of a list key = its index + the number
    // of new keys below it.  Keys are unique, so positions are unique; the
    // first L positions form the new list (a merge, not a re-sort).
    {
      const int nk = C->nkeys[sp];
      const int cnt = lcnt;
      // fused path: register bitonic merge + next select by warp 0 (lists of
      // up to 32*kMaxE keys, <= kWarpMergeMax new keys: the common step --
      // the bulk first steps of a query, when the list is still filling,
      // take the rank merge below)
      constexpr int kMaxE = (NT * MINB >= 1024) ? 4 : 16;  // list registers within the thread budget
      if (CS == 1 && L <= 32 * kMaxE && nk <= kWarpMergeMax && !(cfg.prefetch & (64 | 2))) {
        uint64_t* sorted2 = reinterpret_cast<uint64_t*>(s.part);  // blocks 1..3, sorted
        const int nblk = (nk + 31) >> 5;
        // merge by rank in parallel warps (lists of <= 128 keys; <= 32 with
        // prefetch bit 16384, A/B) -- prefetch bit 4096: warp 0's bitonic
        // networks instead (A/B)
        const int rank_lmax = (cfg.prefetch & 16384) ? 32 : 128;
        const bool by_rank = (NT >= 256) && L <= rank_lmax && !(cfg.prefetch & 4096);
        if (by_rank) {
          if constexpr (NT >= 256) {
            if (tid == 0) C->mg_bitonic++;
            if (L <= 32)
              rank_merge_select<1, NT>(cfg, s, C, warp, lane, cnt, nk, L, W, OFF, sp, liters, np_step, cur, lcnt);
            else if (L <= 64)
              rank_merge_select<2, NT>(cfg, s, C, warp, lane, cnt, nk, L, W, OFF, sp, liters, np_step, cur, lcnt);
            else
              rank_merge_select<4, NT>(cfg, s, C, warp, lane, cnt, nk, L, W, OFF, sp, liters, np_step, cur, lcnt);
          }
        }
        if constexpr (NT >= 128) {
          if (!by_rank && warp >= 1 && warp < nblk) {
            const uint64_t x = (32 * warp + lane < nk) ? s.newk[32 * warp + lane] : kKeyMax;
            sorted2[32 * warp + lane] = warp_bitonic_sort32(x, lane);
            __threadfence_block();
            asm volatile("bar.arrive 1, %0;" ::"r"(32 * nblk) : "memory");
          }
        }
        if (warp == 0 && !by_rank) {
          if (tid == 0) C->mg_bitonic++;
          if (L <= 32)
            warp_merge_select<1, NT>(cfg, s, C, lane, cnt, nk, nblk, sorted2, L, W, OFF, sp, liters, np_step, cur, lcnt);
          else if (L <= 64)
            warp_merge_select<2, NT>(cfg, s, C, lane, cnt, nk, nblk, sorted2, L, W, OFF, sp, liters, np_step, cur, lcnt);
          else if (L <= 128)
            warp_merge_select<4, NT>(cfg, s, C, lane, cnt, nk, nblk, sorted2, L, W, OFF, sp, liters, np_step, cur, lcnt);
          else if (L <= 256)
            warp_merge_select<8, NT>(cfg, s, C, lane, cnt, nk, nblk, sorted2, L, W, OFF, sp, liters, np_step, cur, lcnt);
          else if constexpr (kMaxE >= 16)
            warp_merge_select<16, NT>(cfg, s, C, lane, cnt, nk, nblk, sorted2, L, W, OFF, sp, liters, np_step, cur, lcnt);
          if (tid == 0 && !C->spilled && gtab != nullptr && C->vis_count + step_max_new > (hcap * 3) / 4)
            C->spilled = 1;
        }
        if (gcache) asm volatile("cp.async.wait_all;" ::: "memory");  // cached rows landed (in warp 0's shadow)
        __syncthreads();
        cur = C->cur;
        lcnt = C->cnt;
        pre = true;
        lap(3);
        continue;
      }
      if (tid == 0) C->mg_rank++;
      if (nk > 0) {
        const uint64_t* src = cur ? s.list[1] : s.list[0];
        uint64_t* dst = cur ? s.list[0] : s.list[1];
        // the nk x (nk + cnt) comparisons are split over `parts` threads per
        // key so no thread loops over all nk new keys: partial counts go to
        // s.part, then one thread per key sums them and writes its key
        const int nu = nk + cnt;  // keys to place: new keys, then list keys
        int parts = NT / nu;
        parts = parts < 1 ? 1 : (parts > 16 ? 16 : parts);
        if (parts * nu > kMergeParts) parts = kMergeParts / nu > 0 ? kMergeParts / nu : 1;
        if (parts > 1) {
          if (tid < parts * nu) {
            const int u = tid % nu, part = tid / nu;
            const uint64_t key = u < nk ? s.newk[u] : src[u - nk];
            const int j0 = part * nk / parts, j1 = (part + 1) * nk / parts;
            int rn = 0;
            for (int j = j0; j < j1; ++j) rn += (s.newk[j] < key) ? 1 : 0;
            if (part == 0) rn += u < nk ? lower_bound_u64(src, cnt, key) : u - nk;
            s.part[tid] = rn;
          }
          __syncthreads();
          if (tid < nu) {
            int pos = 0;
            for (int p = 0; p < parts; ++p) pos += s.part[p * nu + tid];
            if (pos < L) dst[pos] = tid < nk ? s.newk[tid] : src[tid - nk];
          }
        } else {
          for (int i = tid; i < nk; i += NT) {
            const uint64_t key = s.newk[i];
            int rn = 0;
            for (int j = 0; j < nk; ++j) rn += (s.newk[j] < key) ? 1 : 0;
            const int pos = rn + lower_bound_u64(src, cnt, key);
            if (pos < L) dst[pos] = key;
          }
          for (int j = tid; j < cnt; j += NT) {
            const uint64_t key = src[j];
            int rn = 0;
            for (int i = 0; i < nk; ++i) rn += (s.newk[i] < key) ? 1 : 0;
            const int pos = j + rn;
            if (pos < L) dst[pos] = key;
          }
        }
        cur ^= 1;
        lcnt = (cnt + nk) < L ? cnt + nk : L;
      }
      liters += np_step > 0 ? 1 : 0;
      if (gcache) asm volatile("cp.async.wait_all;" ::: "memory");
      __syncthreads();
      lap(3);
    }
  }

  // ================= publish the first k =================
  if (gcache) asm volatile("cp.async.wait_all;" ::: "memory");
  if (tid == 0) {
    C->gc_stamp = gstamp + 1;
    if (st) st->t_loop1 = globaltimer();
    C->iters = liters;
  }
  const int cnt = lcnt;
  const uint64_t* fin = cur ? s.list[1] : s.list[0];
  for (int i = tid; i < k; i += NT) {
    ResultEntry r;
    if (i < cnt) {
      uint64_t key = fin[i];
      r.id = key_id(key);
      r.dist = key_dist(key);
    } else {
      r.id = kSentinel;
      r.dist = __int_as_float(0x7f800000);
    }
    out[i] = r;
  }
  if (tid == 0) {
    C->phase = phase;
    if (st) {
      st->iters = C->iters;
      st->parents = C->parents;
      st->dist_evals = C->dist_evals;
      st->cap_hit = C->cap_hit;
      st->spilled = C->spilled;
      st->overflow = C->overflow;
      st->cyc_select = C->cyc[0];
      st->cyc_gather = C->cyc[1];
      st->cyc_dist = C->cyc[2];
      st->cyc_sort = C->cyc[3];
      st->mg_bitonic = C->mg_bitonic;
      st->mg_rank = C->mg_rank;
    }
  }
}

// Cluster worker (CTA rank crank > 0): mirrors the leader's two cluster
// barriers per step and evaluates its share (rows crank, crank+CS, ...) of
// every distance step, reading ids from and delivering keys into the
// leader's shared memory.  Preconditions: s.q holds the query.
// One command from the leader: wait on the step-ready barrier, evaluate this
// CTA's rows (ids in its own shared memory, the query in s.q as pushed by the
// leader at query start), deliver the keys into the leader's newk, signal.
// Returns the command (kCmdStep or kCmdQuit).
template <int NT, int TL, int CPL, int METRIC>
__device__ int worker_step(const SearchCfg& cfg, const Smem& s, uint32_t& phase) {
  mbar_wait_cluster(s.bar + 2, (phase >> 2) & 1u);
  phase ^= 4u;
  const int cmd = *((volatile int*)&s.ctrl->w_cmd);
  if (cmd != kCmdStep) return cmd;
  const int M = *((volatile int*)&s.ctrl->w_m);
  const uint64_t worst = *((volatile uint64_t*)&s.ctrl->w_worst);
  Ctrl* LC = leader_ptr(s.ctrl);
  dist_ldg<NT, TL, CPL, METRIC>(cfg, s.q, M, 0, 1, worst, s.newid, leader_ptr(s.newk), &LC->nkeys[0]);
  __syncthreads();
  if (threadIdx.x == 0) {
    fence_cluster();
    mbar_remote_arrive(s.bar + 3, 0);
  }
  return cmd;
}
// leader: push the query into every worker's shared memory (released by the
// next step signal)
template <int NT, int CS>
__device__ __forceinline__ void push_query(const Smem& s, int d4) {
  for (int c = 1; c < CS; ++c) {
    float4* wq = rank_ptr(s.q, c);
    for (int i = threadIdx.x; i < d4; i += NT) wq[i] = s.q[i];
  }
}
// leader: tell every worker to leave
template <int CS>
__device__ __forceinline__ void post_quit(const Smem& s) {
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int c = 1; c < CS; ++c) rank_ptr(s.ctrl, c)->w_cmd = kCmdQuit;
    fence_cluster();
    for (int c = 1; c < CS; ++c) mbar_remote_arrive(s.bar + 2, c);
  }
}

}  // namespace algas
