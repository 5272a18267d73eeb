// search_core.cuh -- the per-CTA greedy/beam graph search of ALGAS on sm_100a.
//
// One CTA runs one (query, cta_rank) search:
//   select  : first unchecked candidate(s) of the sorted list            (P:L217 step 1, Alg.1 l.6)
//             -- w parents at once after the list offset reaches off   (beam extend)
//   gather  : the parents' neighbour ids, 16-B vector loads of graph rows (P:L217 step 1)
//   filter  : test-and-set in a shared-memory visited hash               (P:L217 step 2)
//   distance: coalesced 16-B gathers of the neighbour vectors, a team of
//             TL lanes per vector, shuffle-tree reduction                (P:L217 step 3, Alg.1 l.9-12)
//   update  : keys that cannot enter the list are dropped, survivors are
//             bitonic-sorted and MERGED (rank merge, no re-sort) into the
//             sorted list, keeping the first L                           (P:L219 step 4, Alg.1 l.15-18)
//   finish  : all L entries checked (or the max_iter cap)                ("Finish")
// The CTA then writes its first k (id, dist).
//
// Keys are u64: (order-preserving fp32 distance << 32) | (id << 1) | checked.
// Ids are < 2^31, so comparing keys compares (dist, id) lexicographically
// (R4) and the "checked" bit never decides an order (ids in a list are
// unique).  Nothing here is shared with oracle/: it is an independent
// implementation of the same paper passages.
#pragma once

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
__device__ __forceinline__ float4 ldg_stream(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ldg_u4(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// ------------------------------------------------------------------ configuration
struct SearchCfg {
  const float4* data;    // n x d4 float4 (row-major, 16-B aligned rows)
  const uint4* graph;    // n x rp4 uint4 (row stride Rp = 4*rp4, padded with sentinels)
  uint64_t n;
  int32_t d4;            // dim / 4
  int32_t R;             // out-degree
  int32_t rp4;           // padded row length / 4
  int32_t L, w, off, S, max_iter;
  int32_t hash_bits;     // shared-memory visited hash: 2^hash_bits u32
  int32_t gtab_bits;     // HBM spill table per CTA: 2^gtab_bits u64
  int32_t ncap;          // capacity of the new-key buffer (power of two)
  uint64_t seed;
};

struct CtaStats {
  uint32_t iters, parents, dist_evals, cap_hit, spilled, overflow;
  unsigned long long t_start, t_end;  // globaltimer (persistent paths)
};

struct ResultEntry {
  uint32_t id;
  float dist;
};

struct Ctrl {
  int cnt, nnew, nkeys, np, done, diffusing, vis_count, spilled, overflow, cur;
  uint32_t iters, parents, dist_evals, cap_hit;
};

// Shared-memory carve-up (bytes, all 16-B aligned).
struct SmemLayout {
  int off_q, off_listA, off_listB, off_newk, off_newid, off_sel, off_hash, off_ctrl, total;
};
__host__ __device__ inline int align16(int x) { return (x + 15) & ~15; }
__host__ __device__ inline SmemLayout smem_layout(int d4, int L, int ncap, int hash_bits) {
  SmemLayout s;
  int o = 0;
  s.off_q = o;     o += align16(d4 * 16);
  s.off_listA = o; o += align16(L * 8);
  s.off_listB = o; o += align16(L * 8);
  s.off_newk = o;  o += align16(ncap * 8);
  s.off_newid = o; o += align16(ncap * 4);
  s.off_sel = o;   o += align16(64 * 4);
  s.off_hash = o;  o += align16((1 << hash_bits) * 4);
  s.off_ctrl = o;  o += align16((int)sizeof(Ctrl));
  s.total = o;
  return s;
}

struct Smem {
  float4* q;
  uint64_t* list[2];
  uint64_t* newk;
  uint32_t* newid;
  int* sel;         // [0,32): selected positions, [32,64): parent ids
  uint32_t* hash;
  Ctrl* ctrl;
};
__device__ __forceinline__ Smem carve(uint8_t* base, const SmemLayout& l) {
  Smem s;
  s.q = reinterpret_cast<float4*>(base + l.off_q);
  s.list[0] = reinterpret_cast<uint64_t*>(base + l.off_listA);
  s.list[1] = reinterpret_cast<uint64_t*>(base + l.off_listB);
  s.newk = reinterpret_cast<uint64_t*>(base + l.off_newk);
  s.newid = reinterpret_cast<uint32_t*>(base + l.off_newid);
  s.sel = reinterpret_cast<int*>(base + l.off_sel);
  s.hash = reinterpret_cast<uint32_t*>(base + l.off_hash);
  s.ctrl = reinterpret_cast<Ctrl*>(base + l.off_ctrl);
  return s;
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

// ------------------------------------------------------------------ sorting
// ascending bitonic sort of one u64 per lane
__device__ __forceinline__ uint64_t warp_bitonic32(uint64_t v, int lane) {
#pragma unroll
  for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      uint64_t o = __shfl_xor_sync(0xffffffffu, v, j);
      bool up = (lane & k) == 0;
      bool lower = (lane & j) == 0;
      bool keep_min = (lower == up);
      v = keep_min ? (o < v ? o : v) : (o > v ? o : v);
    }
  }
  return v;
}
// ascending bitonic sort of s[0..P), P power of two; all NT threads call
template <int NT>
__device__ __forceinline__ void cta_bitonic(uint64_t* s, int P, int tid) {
  for (int k = 2; k <= P; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = tid; i < (P >> 1); i += NT) {
        int lo = 2 * j * (i / j) + (i % j);
        int hi = lo + j;
        bool up = (lo & k) == 0;
        uint64_t a = s[lo], b = s[hi];
        if ((a > b) == up) { s[lo] = b; s[hi] = a; }
      }
      __syncthreads();
    }
  }
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
template <int TL, int CPL, int METRIC>
struct QueryRegs {
  float4 q[CPL];
  __device__ __forceinline__ void load(const float4* qs, int d4, int tl) {
#pragma unroll
    for (int c = 0; c < CPL; ++c) {
      int ch = tl + c * TL;
      q[c] = (ch < d4) ? qs[ch] : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
};

template <int TL, int CPL, int METRIC>
__device__ __forceinline__ float team_partial(const QueryRegs<TL, CPL, METRIC>& Q, const float4* x, int d4,
                                              int tl) {
  float4 v[CPL];
#pragma unroll
  for (int c = 0; c < CPL; ++c) {
    int ch = tl + c * TL;
    v[c] = (ch < d4) ? ldg_stream(x + ch) : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  float acc = 0.f;
#pragma unroll
  for (int c = 0; c < CPL; ++c) {
    if (METRIC == kL2) {
      float a = Q.q[c].x - v[c].x, b = Q.q[c].y - v[c].y, e = Q.q[c].z - v[c].z, f = Q.q[c].w - v[c].w;
      acc = fmaf(a, a, acc); acc = fmaf(b, b, acc); acc = fmaf(e, e, acc); acc = fmaf(f, f, acc);
    } else {
      acc = fmaf(Q.q[c].x, v[c].x, acc); acc = fmaf(Q.q[c].y, v[c].y, acc);
      acc = fmaf(Q.q[c].z, v[c].z, acc); acc = fmaf(Q.q[c].w, v[c].w, acc);
    }
  }
  return acc;
}
template <int TL>
__device__ __forceinline__ float team_reduce(float acc) {
#pragma unroll
  for (int o = TL >> 1; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  return acc;
}

// ------------------------------------------------------------------ the search
// Preconditions: s.q holds the query (d4 float4).  Writes min(k, |list|)
// results to out[0..k) (rest padded) and the CTA's counters to *st.
template <int NT, int TL, int CPL, int METRIC>
__device__ void search_cta(const SearchCfg& cfg, const Smem& s, uint64_t tag, uint32_t cta_rank, int k,
                           unsigned long long* gtab, uint32_t epoch, ResultEntry* out, CtaStats* st) {
  const int tid = threadIdx.x;
  const int lane = tid & 31;
  const int warp = tid >> 5;
  constexpr int NTEAMS = NT / TL;
  const int team = tid / TL;
  const int tl = tid % TL;
  Ctrl* C = s.ctrl;
  const int L = cfg.L;
  const int hbits = cfg.hash_bits;
  const int hcap = 1 << hbits;
  const int step_max_new = cfg.w * cfg.rp4 * 4;

  // ---- reset per-query state
  for (int i = tid; i < hcap; i += NT) s.hash[i] = kHashEmpty;
  if (tid == 0) {
    C->cnt = 0; C->nnew = 0; C->nkeys = 0; C->np = 0; C->done = 0; C->diffusing = 0;
    C->vis_count = 0; C->spilled = 0; C->overflow = 0; C->cur = 0;
    C->iters = 0; C->parents = 0; C->dist_evals = 0; C->cap_hit = 0;
  }
  QueryRegs<TL, CPL, METRIC> Q;
  Q.load(s.q, cfg.d4, tl);
  __syncthreads();

  // ---- entry points (Alg.1 l.5): S seeds, duplicates dropped
  // Seeds are inserted sequentially by warp 0 in j order so the visited set
  // sees exactly the deduplicated seed set.
  if (warp == 0) {
    for (int j0 = 0; j0 < cfg.S; j0 += 32) {
      int j = j0 + lane;
      uint32_t e = (j < cfg.S) ? entry_point(cfg.seed, tag, cta_rank, (uint32_t)j, cfg.n) : kSentinel;
      for (int l = 0; l < 32; ++l) {
        uint32_t el = __shfl_sync(0xffffffffu, e, l);
        if (el == kSentinel) continue;
        if (lane == 0) {
          int r = smem_visit(s.hash, hbits, el);
          if (r == kVisNew) { s.newid[C->nnew] = el; C->nnew++; C->vis_count++; }
        }
        __syncwarp();
      }
    }
  }
  __syncthreads();

  int cur = 0;
  bool first = true;
  for (;;) {
    // ================= select (warp 0) =================
    if (!first) {
      if (warp == 0) {
        const int cnt = C->cnt;
        const uint64_t* list = (cur ? s.list[1] : s.list[0]);
        int found = 0;
        for (int base = 0; base < cnt && found < cfg.w; base += 32) {
          int i = base + lane;
          bool un = (i < cnt) && !(list[i] & 1ull);
          unsigned m = __ballot_sync(0xffffffffu, un);
          int rank = found + __popc(m & ((1u << lane) - 1u));
          if (un && rank < cfg.w) s.sel[rank] = i;
          found += __popc(m);
        }
        if (found > cfg.w) found = cfg.w;
        __syncwarp();
        int done = 0, np = 0;
        if (found == 0) {
          done = 1;
        } else if ((int)C->iters >= cfg.max_iter) {
          done = 1;
          if (lane == 0) C->cap_hit = 1;
        } else {
          int diff = C->diffusing;
          if (s.sel[0] >= cfg.off) diff = 1;          // P:L249 (sticky, R6)
          np = diff ? found : 1;
          if (lane < np) {
            int pos = s.sel[lane];
            uint64_t kk = (cur ? s.list[1] : s.list[0])[pos];
            (cur ? s.list[1] : s.list[0])[pos] = kk | 1ull;              // mark checked (Alg.1 l.7)
            s.sel[32 + lane] = (int)key_id(kk);
          }
          if (lane == 0) C->diffusing = diff;
        }
        if (lane == 0) {
          C->done = done;
          C->np = np;
          C->nnew = 0;
          C->nkeys = 0;
          if (!done) { C->parents += np; }
          // switch to the HBM spill table before the shared one gets too full
          if (!C->spilled && gtab != nullptr && C->vis_count + step_max_new > (hcap * 3) / 4) C->spilled = 1;
        }
      }
      __syncthreads();
      if (C->done) break;

      // ================= gather + visited filter (P:L217 steps 1-2) =================
      {
        const int np = C->np;
        const int spilled = C->spilled;
        const int per_row = cfg.rp4;
        const int total = np * per_row;
        for (int base = 0; base < total; base += NT) {
          int idx = base + tid;
          uint32_t ids[4] = {kSentinel, kSentinel, kSentinel, kSentinel};
          if (idx < total) {
            int p = idx / per_row;
            int c = idx - p * per_row;
            uint32_t parent = (uint32_t)s.sel[32 + p];
            uint4 v = ldg_u4(cfg.graph + (uint64_t)parent * per_row + c);
            ids[0] = v.x; ids[1] = v.y; ids[2] = v.z; ids[3] = v.w;
          }
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            bool keep = false;
            uint32_t id = ids[e];
            if (id != kSentinel) {
              if (!spilled) {
                int r = smem_visit(s.hash, hbits, id);
                keep = (r == kVisNew);
                if (r == kVisFull) atomicOr(&C->overflow, 1);
              } else if (!smem_contains(s.hash, hbits, id)) {
                int r = gmem_visit(gtab, cfg.gtab_bits, epoch, id);
                keep = (r == kVisNew);
                if (r == kVisFull) atomicOr(&C->overflow, 1);
              }
            }
            unsigned m = __ballot_sync(0xffffffffu, keep);
            int wbase = 0;
            if (lane == 0 && m) wbase = atomicAdd(&C->nnew, __popc(m));
            wbase = __shfl_sync(0xffffffffu, wbase, 0);
            if (keep) s.newid[wbase + __popc(m & ((1u << lane) - 1u))] = id;
          }
        }
        __syncthreads();
        if (tid == 0 && !spilled) C->vis_count += C->nnew;
      }
    }
    first = false;

    // ================= distances (P:L217 step 3) + prefilter =================
    {
      const int M = C->nnew;
      const int cnt = C->cnt;
      const uint64_t worst = (cnt >= L) ? (cur ? s.list[1] : s.list[0])[L - 1] : kKeyMax;
      // warp-uniform trip count: every lane joins the team shuffles
      for (int base = 0; base < M; base += NTEAMS) {
        const int i = base + team;
        const bool valid = i < M;
        const uint32_t id = valid ? s.newid[i] : 0u;
        float acc = 0.f;
        if (valid) acc = team_partial<TL, CPL, METRIC>(Q, cfg.data + (uint64_t)id * cfg.d4, cfg.d4, tl);
        acc = team_reduce<TL>(acc);
        if (valid && tl == 0) {
          float d = (METRIC == kL2) ? acc : -acc;
          uint64_t key = make_key(d, id);
          if (key < worst) {
            int pos = atomicAdd(&C->nkeys, 1);
            s.newk[pos] = key;
          }
        }
      }
      __syncthreads();
      if (tid == 0) C->dist_evals += M;
    }

    // ================= sort new keys + merge into the list (P:L219 step 4) =================
    {
      const int nk = C->nkeys;
      const int cnt = C->cnt;
      if (nk > 0) {
        int P = 1;
        while (P < nk) P <<= 1;
        if (P <= 32) {
          if (warp == 0) {
            uint64_t v = (lane < nk) ? s.newk[lane] : kKeyMax;
            v = warp_bitonic32(v, lane);
            if (lane < nk) s.newk[lane] = v;
          }
          __syncthreads();
        } else {
          for (int i = nk + tid; i < P; i += NT) s.newk[i] = kKeyMax;
          __syncthreads();
          cta_bitonic<NT>(s.newk, P, tid);
        }
        const uint64_t* src = (cur ? s.list[1] : s.list[0]);
        uint64_t* dst = (cur ? s.list[0] : s.list[1]);
        for (int i = tid; i < nk; i += NT) {
          uint64_t key = s.newk[i];
          int pos = i + lower_bound_u64(src, cnt, key);
          if (pos < L) dst[pos] = key;
        }
        for (int j = tid; j < cnt; j += NT) {
          uint64_t key = src[j];
          int pos = j + lower_bound_u64(s.newk, nk, key);
          if (pos < L) dst[pos] = key;
        }
        cur ^= 1;
        __syncthreads();
        if (tid == 0) {
          int nc = cnt + nk;
          C->cnt = nc < L ? nc : L;
        }
      }
      if (tid == 0) C->iters += (C->np > 0) ? 1 : 0;
      __syncthreads();
    }
  }

  // ================= publish the first k =================
  const int cnt = C->cnt;
  for (int i = tid; i < k; i += NT) {
    ResultEntry r;
    if (i < cnt) {
      uint64_t key = (cur ? s.list[1] : s.list[0])[i];
      r.id = key_id(key);
      r.dist = key_dist(key);
    } else {
      r.id = kSentinel;
      r.dist = __int_as_float(0x7f800000);
    }
    out[i] = r;
  }
  if (tid == 0 && st) {
    st->iters = C->iters;
    st->parents = C->parents;
    st->dist_evals = C->dist_evals;
    st->cap_hit = C->cap_hit;
    st->spilled = C->spilled;
    st->overflow = C->overflow;
  }
}

}  // namespace algas
