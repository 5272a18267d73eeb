// runtime.cu -- host runtime of ALGAS:
//   * TopK merge & filter on the host (A9): a priority queue over
//     the T sorted per-CTA lists of one query, sentinels and repeated ids
//     filtered out;
//   * adaptive tuning;
//   * the persistent server: host-mapped slot ring with per-slot state
//     machine, host poller threads that watch the per-CTA
//     Finish flags in host memory (local polling), merges and
//     recycles the slot (Done -> None).
#include <algorithm>
#include <chrono>
#include <cstring>
#include <deque>
#include <limits>
#include <memory>
#include <queue>
#include <thread>
#include <vector>

#include "internal.h"

namespace algas {

// ------------------------------------------------------------------ A9 merge
int32_t merge_cta_lists(const ResultEntry* res, int T, int kin, int k, uint32_t* out_ids, float* out_d) {
  // binary min-heap on (dist, id) over the T list heads, in a per-thread
  // buffer (the poller merges every query: no allocation on this path)
  struct H {
    float d;
    uint32_t id;
    int c, p;
  };
  auto less = [](const H& a, const H& b) { return a.d < b.d || (a.d == b.d && a.id < b.id); };
  thread_local std::vector<H> heap;
  if ((int)heap.size() < T) heap.resize(T);
  int hn = 0;
  auto push = [&](H h) {
    int i = hn++;
    while (i > 0) {
      const int par = (i - 1) >> 1;
      if (!less(h, heap[par])) break;
      heap[i] = heap[par];
      i = par;
    }
    heap[i] = h;
  };
  auto pop_top = [&]() {
    const H last = heap[--hn];
    int i = 0;
    for (;;) {
      int c = 2 * i + 1;
      if (c >= hn) break;
      if (c + 1 < hn && less(heap[c + 1], heap[c])) ++c;
      if (!less(heap[c], last)) break;
      heap[i] = heap[c];
      i = c;
    }
    heap[i] = last;
  };
  for (int c = 0; c < T; ++c) {
    const ResultEntry& e = res[(size_t)c * kin];
    if (kin > 0 && e.id != kSentinel) push(H{e.dist, e.id, c, 0});
  }
  int n = 0;
  // repeated ids (R11): a linear scan of the emitted ids for small k, an
  // open-addressing set for large k (k = 100 would cost k^2/2 compares)
  const bool use_set = k > 32;
  uint32_t set_bits = 6;
  while ((1u << set_bits) < 2u * (uint32_t)k) ++set_bits;
  thread_local std::vector<uint32_t> set;
  if (use_set) set.assign((size_t)1 << set_bits, kSentinel);
  auto seen_insert = [&](uint32_t id) -> bool {  // true if id was already emitted
    const uint32_t mask = (1u << set_bits) - 1u;
    uint32_t h = (id * 0x9E3779B1u) >> (32 - set_bits);
    for (;; h = (h + 1) & mask) {
      if (set[h] == id) return true;
      if (set[h] == kSentinel) { set[h] = id; return false; }
    }
  };
  while (hn > 0 && n < k) {
    const H h = heap[0];
    pop_top();
    bool dup = false;
    if (use_set) {
      dup = seen_insert(h.id);
    } else {
      for (int i = 0; i < n; ++i)
        if (out_ids[i] == h.id) { dup = true; break; }
    }
    if (!dup) {
      out_ids[n] = h.id;
      out_d[n] = h.d;
      ++n;
    }
    if (h.p + 1 < kin) {
      const ResultEntry& e = res[(size_t)h.c * kin + h.p + 1];
      if (e.id != kSentinel) push(H{e.dist, e.id, h.c, h.p + 1});
    }
  }
  for (int i = n; i < k; ++i) {
    out_ids[i] = kSentinel;
    out_d[i] = std::numeric_limits<float>::infinity();
  }
  return n;
}

}  // namespace algas

using namespace algas;

// ------------------------------------------------------------------ server
struct algas_server {
  algas_index* idx = nullptr;
  Plan plan;
  int slots = 0, T = 0, kmax = 0, dim = 0, d4 = 0;
  cudaStream_t stream = nullptr;
  // host-mapped ring (host pointer / device alias)
  RingSlot* ring_h = nullptr;
  RingSlot* ring_d = nullptr;
  float* ringq_h = nullptr;
  float4* ringq_d = nullptr;
  ResultEntry* res_h = nullptr;
  ResultEntry* res_d = nullptr;
  CtaStats* st_h = nullptr;
  CtaStats* st_d = nullptr;
  uint32_t* done_h = nullptr;
  uint32_t* done_d = nullptr;
  // device mailbox
  void* ctl = nullptr;
  float4* qbuf = nullptr;
  unsigned long long* gtab = nullptr;  // the server's own HBM spill tables
  uint32_t* vbm = nullptr;             // SHARED visited bitmaps, two per slot
  // Every slot has TWO ring entries ("sub-slots", index u = 2*slot + b):
  // the slot's queries alternate between them (b = 1, 0, 1, ...), so the
  // host can stage a slot's next query while its current one runs, and the
  // slot's CTAs start it without a host round trip (dynamic batching keeps
  // B searches running; the staged ones wait in host memory like the FIFO).
  // Host-side bookkeeping per sub-slot (host owns: EMPTY/claimed/in-flight):
  std::vector<std::atomic<int>>* hstate = nullptr;  // 0 free, 1 claimed, 2 in flight
  std::vector<uint32_t> epoch;   // per sub-slot: epoch of its query
  std::vector<uint32_t> next_ep; // per slot: epoch of its next query
  std::vector<int> next_sub;     // per slot: sub-slot of its next query
  std::unique_ptr<std::atomic<int>[]> slot_lock;  // per slot: claim lock
  std::unique_ptr<std::atomic<int>[]> slot_busy;  // per slot: sub-slots not free (0..2)
  std::atomic<int> n_idle_slots{0};               // slots with both sub-slots free
  std::vector<uint64_t> tags;
  std::vector<int> kq;
  std::vector<std::chrono::steady_clock::time_point> t_submit;
  std::atomic<int> next_slot{0};
  std::vector<std::thread> pollers;
  std::atomic<bool> stop{false};
  std::atomic<bool> kernel_ok{true};
  // bounded session (algas_server_start with quit_when_idle): no new work is
  // accepted, and every ring entry that becomes free is set to QUIT, so the
  // persistent kernel exits once the staged queries are done
  std::atomic<bool> quit_when_idle{false};
  // watchdog: a query in a slot longer than watchdog_ns marks the server failed
  int64_t watchdog_ns = 0;
  std::atomic<bool> stuck{false};
  std::atomic<uint64_t> stuck_tag{0};
  bool launched = false;
  PersistArgs pa;  // launch arguments (kept for a deferred launch)
  // state mirror: host staging of every ring entry (RingSlot line
  // + query) in pinned memory and its device copy the CTAs poll; each host
  // thread writes through its own IO stream ("private IO streams")
  bool mirror = false;
  uint8_t* mir_h = nullptr;
  uint8_t* mir_d = nullptr;
  int64_t mir_stride = 0;
  uint64_t uid = 0;  // server identity for the per-thread stream cache
  std::mutex io_mu;
  std::vector<cudaStream_t> io_streams;
  // emulated ring device (algas_server_create_emulated; protocol tests on
  // hosts without a GPU): a host thread in place of the persistent kernel
  bool emulated = false;
  std::thread emu;
  std::atomic<uint64_t> emu_stall_tag{~0ull};  // a query with this tag is never finished
  std::mutex cq_mu;
  struct Done {
    uint64_t tag;
    std::vector<uint32_t> ids;
    std::vector<float> d;
    algas_query_stats st;
  };
  std::deque<Done> cq;
  std::vector<Done> done_pool;  // recycled completion records (their vectors keep their capacity)
  std::atomic<int64_t> inflight{0};
  // host FIFO of enqueued queries not yet in a slot (algas_enqueue): the
  // poller thread moves the head into a slot the moment one is recycled
  struct Pending {
    uint64_t tag;
    int32_t k, L, w;
    std::chrono::steady_clock::time_point t_enq;
    std::shared_ptr<const std::vector<float>> blk;  // the enqueue call's copy of its queries
    int64_t off;                                    // this query's offset in blk
  };
  std::mutex pq_mu;
  std::deque<Pending> pending;
  std::atomic<int64_t> n_pending{0};
  std::vector<uint64_t> queue_ns;  // per sub-slot: FIFO wait of its query
};

namespace {
std::atomic<uint64_t> g_server_uid{1};

// the calling thread's private IO stream for server s (created on first use,
// destroyed with the server)
cudaStream_t io_stream(algas_server* s) {
  thread_local std::vector<std::pair<uint64_t, cudaStream_t>> cache;
  for (auto& e : cache)
    if (e.first == s->uid) return e.second;
  cudaStream_t st = nullptr;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  {
    std::lock_guard<std::mutex> lk(s->io_mu);
    s->io_streams.push_back(st);
  }
  if (cache.size() > 64) cache.erase(cache.begin());
  cache.emplace_back(s->uid, st);
  return st;
}

// state mirror: publish host staging entry u's state word `state` to the
// device copy -- the payload (params + query) first, the state word last,
// both stream-ordered on the calling thread's IO stream (with_payload = 0:
// state only, e.g. QUIT)
void mirror_publish(algas_server* s, int u, uint32_t state, bool with_payload) {
  uint8_t* h = s->mir_h + (size_t)u * s->mir_stride;
  uint8_t* d = s->mir_d + (size_t)u * s->mir_stride;
  __atomic_store_n(reinterpret_cast<uint32_t*>(h), state, __ATOMIC_RELEASE);
  cudaStream_t st = io_stream(s);
  if (with_payload) cudaMemcpyAsync(d + 4, h + 4, (size_t)s->mir_stride - 4, cudaMemcpyHostToDevice, st);
  cudaMemcpyAsync(d, h, 4, cudaMemcpyHostToDevice, st);
}

// None -> Work of a claimed sub-slot u (epoch already assigned):
// payload first, state word last (release)
void write_slot(algas_server* s, int u, const float* query, uint64_t tag, int32_t k, int32_t itopk, int32_t width) {
  s->tags[u] = tag;
  s->kq[u] = k;
  s->t_submit[u] = std::chrono::steady_clock::now();
  (*s->hstate)[u].store(2, std::memory_order_release);
  const uint32_t state = (s->epoch[u] << 8) | kSlotReady;
  if (s->mirror) {
    uint8_t* h = s->mir_h + (size_t)u * s->mir_stride;
    RingSlot* rs = reinterpret_cast<RingSlot*>(h);
    rs->k = k;
    rs->L = itopk;
    rs->w = width;
    rs->tag = tag;
    memcpy(h + sizeof(RingSlot), query, (size_t)s->dim * 4);
    mirror_publish(s, u, state, true);
    return;
  }
  memcpy(s->ringq_h + (size_t)u * s->dim, query, (size_t)s->dim * 4);
  RingSlot* rs = &s->ring_h[u];
  rs->k = k;
  rs->L = itopk;
  rs->w = width;
  rs->tag = tag;
  __atomic_store_n(&rs->state, state, __ATOMIC_RELEASE);
}
// claim the next sub-slot of a slot whose next sub-slot is free (host state
// 0 -> 1) and give it the slot's next epoch, scanning slots from `start`, a
// slot with nothing in flight first; returns the sub-slot index or -1
int claim_slot(algas_server* s, int start) {
  // pass 0 (a slot with nothing in flight) only while such a slot exists:
  // under load every slot is busy and the scan would cost the poller ~1 us
  // per query (the count is advisory: a stale value only changes placement)
  for (int pass = s->n_idle_slots.load(std::memory_order_relaxed) > 0 ? 0 : 1; pass < 2; ++pass) {
    for (int i = 0; i < s->slots; ++i) {
      const int q = (start + i) % s->slots;
      int unlocked = 0;
      if (!s->slot_lock[q].compare_exchange_strong(unlocked, 1, std::memory_order_acquire)) continue;
      const int u = 2 * q + s->next_sub[q];
      const bool idle = (*s->hstate)[u ^ 1].load(std::memory_order_acquire) == 0;
      int expect = 0;
      if ((pass == 1 || idle) && (*s->hstate)[u].compare_exchange_strong(expect, 1, std::memory_order_acq_rel)) {
        s->epoch[u] = s->next_ep[q];
        const uint32_t ne = (s->next_ep[q] + 1) & 0xFFFFFFu;
        s->next_ep[q] = ne == 0 ? 1 : ne;
        s->next_sub[q] ^= 1;
        if (s->slot_busy[q].fetch_add(1, std::memory_order_relaxed) == 0)
          s->n_idle_slots.fetch_sub(1, std::memory_order_relaxed);
        s->slot_lock[q].store(0, std::memory_order_release);
        return u;
      }
      s->slot_lock[q].store(0, std::memory_order_release);
    }
  }
  return -1;
}
// move FIFO heads into free slots (caller thread or poller)
void drain_pending(algas_server* s, int start) {
  if (s->n_pending.load(std::memory_order_acquire) == 0) return;
  std::lock_guard<std::mutex> lk(s->pq_mu);
  while (!s->pending.empty()) {
    const int q = claim_slot(s, start);
    if (q < 0) break;
    algas_server::Pending& p = s->pending.front();
    s->queue_ns[q] = (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
                         std::chrono::steady_clock::now() - p.t_enq).count();
    write_slot(s, q, p.blk->data() + p.off, p.tag, p.k, p.L, p.w);
    s->pending.pop_front();
    s->n_pending.fetch_sub(1, std::memory_order_acq_rel);
    start = q / 2 + 1;
  }
}
}  // namespace

// poller thread `me` of `nth`: watches slots q = me, me + nth, ...
static void poller_main(algas_server* s, int me, int nth) {
  const int T = s->T;
  std::vector<uint32_t> ids(s->kmax);
  std::vector<float> ds(s->kmax);
  int idle = 0;
  uint64_t sweep = 0;
  while (!s->stop.load(std::memory_order_acquire)) {
    bool any = false;
    int watching = 0;  // this poller's queries in flight
    for (int q = 0; q < 2 * s->slots; ++q) {  // sub-slots of this poller's slots
      if ((q >> 1) % nth != me) continue;
      if ((*s->hstate)[q].load(std::memory_order_acquire) != 2) continue;
      ++watching;
      const uint32_t ep = s->epoch[q];
      bool all = true;
      for (int c = 0; c < T; ++c) {
        // local polling of host memory: no PCIe traffic
        uint32_t v = __atomic_load_n(&s->done_h[(size_t)q * T + c], __ATOMIC_ACQUIRE);
        if (v != ep) { all = false; break; }
      }
      if (!all) {
        // watchdog: checked every 1024 sweeps (a steady_clock read per sweep would cost the merge path)
        if (s->watchdog_ns > 0 && (sweep & 1023) == 0 && !s->stuck.load(std::memory_order_relaxed)) {
          const int64_t age = std::chrono::duration_cast<std::chrono::nanoseconds>(
                                  std::chrono::steady_clock::now() - s->t_submit[q]).count();
          if (age > s->watchdog_ns) {
            s->stuck_tag.store(s->tags[q], std::memory_order_relaxed);
            s->stuck.store(true, std::memory_order_release);
          }
        }
        continue;
      }
      any = true;
      algas_server::Done d;
      {
        std::lock_guard<std::mutex> lk(s->cq_mu);
        if (!s->done_pool.empty()) {
          d = std::move(s->done_pool.back());
          s->done_pool.pop_back();
        }
      }
      d.tag = s->tags[q];
      const int k = s->kq[q];
      const ResultEntry* r = s->res_h + (size_t)q * T * s->kmax;
      d.ids.assign(s->kmax, kSentinel);
      d.d.assign(s->kmax, std::numeric_limits<float>::infinity());
      if (T == 1) {
        for (int i = 0; i < k; ++i) { d.ids[i] = r[i].id; d.d[i] = r[i].dist; }
      } else {
        merge_cta_lists(r, T, s->kmax, k, d.ids.data(), d.d.data());
      }
      aggregate_cta_stats(s->st_h + (size_t)q * T, T, &d.st);
      d.st.latency_ns = (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
                            std::chrono::steady_clock::now() - s->t_submit[q])
                            .count();
      d.st.queue_ns = s->queue_ns[q];
      // Done -> None: host owns the slot again, and the next
      // enqueued query (if any) goes straight into it -- before the result
      // is handed to the caller's completion queue (whose lock a polling
      // caller may hold)
      const bool quit = s->quit_when_idle.load(std::memory_order_acquire) &&
                        s->n_pending.load(std::memory_order_acquire) == 0;
      __atomic_store_n(&s->ring_h[q].state, quit ? (uint32_t)kSlotQuit : (ep << 8) | kSlotEmpty, __ATOMIC_RELEASE);
      if (quit && s->mirror) mirror_publish(s, q, kSlotQuit, false);
      s->queue_ns[q] = 0;
      if (s->slot_busy[q >> 1].fetch_sub(1, std::memory_order_relaxed) == 1)
        s->n_idle_slots.fetch_add(1, std::memory_order_relaxed);
      (*s->hstate)[q].store(0, std::memory_order_release);
      drain_pending(s, q >> 1);
      {
        std::lock_guard<std::mutex> lk(s->cq_mu);
        s->cq.push_back(std::move(d));
      }
    }
    // spin while queries are in flight (a yield can cost several us of
    // rescheduling latency on the merge path); back off only when idle
    ++sweep;
    if (!any && watching == 0) {
      if (++idle > 64) {
        std::this_thread::yield();
        idle = 0;
      }
    } else {
      idle = 0;
    }
  }
}

// host-side bookkeeping of a server's ring (both the real and the emulated device)
static void init_host_state(algas_server* s, int slots, const algas_params* params) {
  const int nsub = 2 * slots;
  s->uid = g_server_uid.fetch_add(1);
  s->watchdog_ns =
      params->watchdog_ms < 0 ? 0 : (int64_t)(params->watchdog_ms > 0 ? params->watchdog_ms : 10000) * 1000000;
  for (auto& a : *s->hstate) a.store(0);
  s->epoch.assign(nsub, 0);
  s->tags.assign(nsub, 0);
  s->kq.assign(nsub, s->kmax);
  s->t_submit.resize(nsub);
  s->queue_ns.assign(nsub, 0);
  s->next_ep.assign(slots, 1);
  s->next_sub.assign(slots, 1);  // the kernel serves sub-slot 1 first, then alternates
  s->slot_lock.reset(new std::atomic<int>[slots]);
  for (int q = 0; q < slots; ++q) s->slot_lock[q].store(0);
  s->slot_busy.reset(new std::atomic<int>[slots]);
  for (int q = 0; q < slots; ++q) s->slot_busy[q].store(0);
  s->n_idle_slots.store(slots);
}

// Emulated ring device: the persistent kernel's side of the host-mapped ring
// protocol (kernels.cuh, mode 0) run by a host thread, for state-machine
// tests without a GPU.  Per slot it serves sub-slot 1 first, then alternates;
// it takes an entry when its state reads READY with an epoch other than the
// one it last served from that entry (or QUIT: the slot stops), and finishes
// a query by writing T per-CTA lists and releasing each CTA's Finish word
// (= the epoch) -- the same words, in the same order, as the kernel.  The
// lists are a fixed function of the staged query and tag, NOT a search: CTA
// r's entry i is (id = tag*1000 + i*T + r, dist = q[0] + i*T + r), plus, for
// T > 1, a repeat of CTA 0's first id at a larger distance (the host merge
// must drop it).  A query whose tag equals emu_stall_tag is never finished
// (watchdog tests).
static void emu_device_main(algas_server* s) {
  const int slots = s->slots, T = s->T, kmax = s->kmax;
  std::vector<int> sub(slots, 1), quit(slots, 0);
  std::vector<uint32_t> last(2 * slots, 0);
  for (;;) {
    int live = 0, progress = 0;
    for (int q = 0; q < slots; ++q) {
      if (quit[q]) continue;
      ++live;
      const int u = 2 * q + sub[q];
      const uint32_t st = __atomic_load_n(&s->ring_h[u].state, __ATOMIC_ACQUIRE);
      const uint32_t kind = st & 0xFFu, ep = st >> 8;
      if (kind == kSlotQuit) { quit[q] = 1; continue; }
      if (kind != kSlotReady || ep == last[u]) continue;
      const RingSlot& rs = s->ring_h[u];
      if (rs.tag == s->emu_stall_tag.load(std::memory_order_relaxed)) continue;
      const int k = rs.k;
      const float q0 = s->ringq_h[(size_t)u * s->dim];
      for (int r = 0; r < T; ++r) {
        ResultEntry* out = s->res_h + ((size_t)u * T + r) * kmax;
        for (int i = 0; i < kmax; ++i) {
          if (i < k) {
            out[i].id = (uint32_t)((rs.tag * 1000ull + (uint64_t)i * T + r) & 0x7FFFFFFFull);
            out[i].dist = q0 + (float)(i * T + r);
          } else {
            out[i].id = kSentinel;
            out[i].dist = std::numeric_limits<float>::infinity();
          }
        }
        if (r == 1 && k >= 2) {  // CTA 0's first id again, farther: a duplicate to drop
          out[k - 1].id = (uint32_t)((rs.tag * 1000ull) & 0x7FFFFFFFull);
          out[k - 1].dist = q0 + (float)(k * T + 7);
        }
        CtaStats& cs = s->st_h[(size_t)u * T + r];
        memset(&cs, 0, sizeof(cs));
        cs.iters = 1;
        __atomic_store_n(&s->done_h[(size_t)u * T + r], ep, __ATOMIC_RELEASE);  // Finish
      }
      last[u] = ep;
      sub[q] ^= 1;
      ++progress;
    }
    if (live == 0) return;
    if (!progress) std::this_thread::yield();
  }
}

extern "C" {

static int server_create(const algas_index* cidx, const algas_params* params, algas_server** out, bool launch);

int algas_server_create_emulated(const algas_params* params, int32_t dim, int32_t deferred, algas_server** out) {
  if (!out || !params) return set_error(ALGAS_EINVAL, "null argument");
  *out = nullptr;
  const int slots = params->slots > 0 ? params->slots : 32;
  const int T = params->ctas_per_query > 0 ? params->ctas_per_query : 1;
  const int k = params->k, L = params->itopk, w = params->width;
  if (dim < 4 || dim % 4 || slots < 1 || T < 1 || T > ALGAS_MAX_CTAS || k < 1 || L < k || w < 1)
    return set_error(ALGAS_EINVAL, "emulated server: bad dim/slots/T/k/itopk/width");
  algas_server* s = new algas_server();
  s->emulated = true;
  s->slots = slots;
  s->T = T;
  s->kmax = k;
  s->dim = dim;
  s->d4 = dim / 4;
  s->plan.T = T;
  s->plan.k = k;
  s->plan.cfg.L = L;
  s->plan.cfg.w = w;
  const int nsub = 2 * slots;
  s->ring_h = (RingSlot*)calloc(nsub, sizeof(RingSlot));
  s->ringq_h = (float*)calloc((size_t)nsub * dim, 4);
  s->res_h = (ResultEntry*)calloc((size_t)nsub * T * k, sizeof(ResultEntry));
  s->st_h = (CtaStats*)calloc((size_t)nsub * T, sizeof(CtaStats));
  s->done_h = (uint32_t*)calloc((size_t)nsub * T, sizeof(uint32_t));
  s->hstate = new std::vector<std::atomic<int>>(nsub);
  if (!s->ring_h || !s->ringq_h || !s->res_h || !s->st_h || !s->done_h) {
    algas_server_destroy(s);
    return set_error(ALGAS_ENOMEM, "emulated server: out of host memory");
  }
  init_host_state(s, slots, params);
  if (!deferred) {
    s->emu = std::thread(emu_device_main, s);
    s->launched = true;
  }
  const int nth = std::max(1, std::min(params->host_threads > 0 ? params->host_threads : 1, slots));
  for (int t = 0; t < nth; ++t) s->pollers.emplace_back(poller_main, s, t, nth);
  *out = s;
  return ALGAS_OK;
}

int algas_server_emulated_stall(algas_server* s, uint64_t tag) {
  if (!s || !s->emulated) return set_error(ALGAS_EINVAL, "not an emulated server");
  s->emu_stall_tag.store(tag);
  return ALGAS_OK;
}

int algas_server_create(const algas_index* cidx, const algas_params* params, algas_server** out) {
  return server_create(cidx, params, out, true);
}

int algas_server_create_deferred(const algas_index* cidx, const algas_params* params, algas_server** out) {
  return server_create(cidx, params, out, false);
}

int algas_server_start(algas_server* s, int32_t quit_when_idle) {
  if (!s) return set_error(ALGAS_EINVAL, "null server");
  if (s->launched) return set_error(ALGAS_ESTATE, "server already started");
  if (quit_when_idle) {
    // every free ring entry becomes QUIT: a slot stops after its staged queries
    s->quit_when_idle.store(true, std::memory_order_release);
    for (int u = 0; u < 2 * s->slots; ++u)
      if ((*s->hstate)[u].load(std::memory_order_acquire) == 0) {
        __atomic_store_n(&s->ring_h[u].state, (uint32_t)kSlotQuit, __ATOMIC_RELEASE);
        if (s->mirror) mirror_publish(s, u, kSlotQuit, false);
      }
    if (s->mirror) cudaStreamSynchronize(io_stream(s));
  }
  // staged queries: their time in the slot (latency, watchdog) starts now
  const auto now = std::chrono::steady_clock::now();
  for (int u = 0; u < 2 * s->slots; ++u)
    if ((*s->hstate)[u].load(std::memory_order_acquire) == 2) s->t_submit[u] = now;
  if (s->emulated) {
    s->emu = std::thread(emu_device_main, s);
    s->launched = true;
    return ALGAS_OK;
  }
  const int rc = launch_persistent(s->plan, s->pa, s->stream);
  if (rc) return rc;
  s->launched = true;
  return ALGAS_OK;
}

static int server_create(const algas_index* cidx, const algas_params* params, algas_server** out, bool launch) {
  if (!out) return set_error(ALGAS_EINVAL, "null out");
  *out = nullptr;
  algas_index* idx = const_cast<algas_index*>(cidx);
  if (!idx || !params) return set_error(ALGAS_EINVAL, "null argument");
  const int slots = params->slots > 0 ? params->slots : 32;
  algas_server* s = new algas_server();
  s->idx = idx;
  int rc = make_plan(idx, params, slots, &s->plan, true);
  if (rc) { delete s; return rc; }
  s->slots = slots;
  s->T = s->plan.T;
  s->kmax = s->plan.k;
  s->dim = idx->dim;
  s->d4 = idx->d4;
  if ((rc = check_coresident(s->plan, slots))) {
    delete s;
    return rc;
  }
  auto cleanup = [&](int code) {
    algas_server_destroy(s);
    return code;
  };
  const unsigned fl = cudaHostAllocMapped | cudaHostAllocPortable;
  cudaError_t e;
#define SRV_ALLOC(hp, dp, bytes)                                                       \
  if ((e = cudaHostAlloc((void**)&hp, (bytes), fl)) != cudaSuccess)                    \
    return cleanup(set_error(ALGAS_ENOMEM, "cudaHostAlloc: %s", cudaGetErrorString(e))); \
  memset(hp, 0, (bytes));                                                              \
  if ((e = cudaHostGetDevicePointer((void**)&dp, hp, 0)) != cudaSuccess)               \
    return cleanup(set_error(ALGAS_ECUDA, "cudaHostGetDevicePointer: %s", cudaGetErrorString(e)));
  const int nsub = 2 * slots;  // two ring entries per slot (sub-slots)
  SRV_ALLOC(s->ring_h, s->ring_d, sizeof(RingSlot) * nsub);
  SRV_ALLOC(s->ringq_h, s->ringq_d, (size_t)nsub * s->dim * 4);
  SRV_ALLOC(s->res_h, s->res_d, sizeof(ResultEntry) * (size_t)nsub * s->T * s->kmax);
  SRV_ALLOC(s->st_h, s->st_d, sizeof(CtaStats) * (size_t)nsub * s->T);
  SRV_ALLOC(s->done_h, s->done_d, sizeof(uint32_t) * (size_t)nsub * s->T);
#undef SRV_ALLOC
  s->mirror = params->state_mirror != 0;
  if (s->mirror) {
    s->mir_stride = (int64_t)sizeof(RingSlot) + (int64_t)s->dim * 4;  // 16-B multiple (dim % 4 == 0)
    if ((e = cudaHostAlloc((void**)&s->mir_h, (size_t)nsub * s->mir_stride, cudaHostAllocPortable)) != cudaSuccess)
      return cleanup(set_error(ALGAS_ENOMEM, "cudaHostAlloc mirror staging: %s", cudaGetErrorString(e)));
    memset(s->mir_h, 0, (size_t)nsub * s->mir_stride);
    if ((e = cudaMalloc(&s->mir_d, (size_t)nsub * s->mir_stride)) != cudaSuccess)
      return cleanup(set_error(ALGAS_ENOMEM, "cudaMalloc state mirror: %s", cudaGetErrorString(e)));
    cudaMemset(s->mir_d, 0, (size_t)nsub * s->mir_stride);
  }
  s->hstate = new std::vector<std::atomic<int>>(nsub);
  init_host_state(s, slots, params);
  const size_t ctl_bytes = control_bytes(slots);
  if ((e = cudaMalloc(&s->ctl, ctl_bytes)) != cudaSuccess)
    return cleanup(set_error(ALGAS_ENOMEM, "cudaMalloc: %s", cudaGetErrorString(e)));
  cudaMemset(s->ctl, 0, ctl_bytes);
  if ((e = cudaMalloc(&s->qbuf, (size_t)slots * s->dim * 4)) != cudaSuccess)
    return cleanup(set_error(ALGAS_ENOMEM, "cudaMalloc: %s", cudaGetErrorString(e)));
  if ((e = cudaStreamCreateWithFlags(&s->stream, cudaStreamNonBlocking)) != cudaSuccess)
    return cleanup(set_error(ALGAS_ECUDA, "stream: %s", cudaGetErrorString(e)));
  // a server owns its spill tables (the index workspace serves batch searches)
  const size_t gent = ((size_t)slots * s->T) << s->plan.cfg.gtab_bits;
  if ((e = cudaMalloc(&s->gtab, gent * 8)) != cudaSuccess)
    return cleanup(set_error(ALGAS_ENOMEM, "cudaMalloc spill tables: %s", cudaGetErrorString(e)));
  cudaMemset(s->gtab, 0, gent * 8);
  const int64_t vw = (s->plan.cfg.shared && !s->plan.cfg.vis_dsmem) ? shared_bitmap_words(idx->n) : 0;
  if (vw > 0 && (e = cudaMalloc(&s->vbm, (size_t)slots * 2 * vw * 4)) != cudaSuccess)
    return cleanup(set_error(ALGAS_ENOMEM, "cudaMalloc visited bitmaps: %s", cudaGetErrorString(e)));
  if (vw > 0) cudaMemset(s->vbm, 0, (size_t)slots * 2 * vw * 4);
  uint8_t* cb = (uint8_t*)s->ctl;
  PersistArgs pa;
  memset(&pa, 0, sizeof(pa));
  pa.mode = 0;
  pa.slots = slots;
  pa.T = s->T;
  pa.kmax = s->kmax;
  pa.ring = s->ring_d;
  pa.ring_q = s->ringq_d;
  pa.ring_res = s->res_d;
  pa.ring_stats = s->st_d;
  pa.ring_done = s->done_d;
  carve_control(cb, slots, &pa);
  pa.qbuf = s->qbuf;
  pa.gtab = s->gtab;
  pa.epoch_base = 1;
  pa.vbm = s->vbm;
  pa.vbm_words = vw;
  pa.mir = s->mir_d;
  pa.mir_stride = s->mir_stride;
  cudaDeviceSynchronize();
  s->pa = pa;
  if (launch) {
    rc = launch_persistent(s->plan, pa, s->stream);
    if (rc) return cleanup(rc);
    s->launched = true;
  }
  const int nth = std::max(1, std::min(params->host_threads > 0 ? params->host_threads : 1, slots));
  for (int t = 0; t < nth; ++t) s->pollers.emplace_back(poller_main, s, t, nth);
  *out = s;
  return ALGAS_OK;
}

int algas_submit(algas_server* s, const float* query, uint64_t tag, int32_t k, int32_t itopk, int32_t width) {
  if (!s || !query) return set_error(ALGAS_EINVAL, "null argument");
  if (s->stop.load()) return set_error(ALGAS_ESTATE, "server is shutting down");
  if (s->quit_when_idle.load()) return set_error(ALGAS_ESTATE, "bounded session: no new work after start");
  if (k <= 0) k = s->kmax;
  if (itopk <= 0) itopk = s->plan.cfg.L;
  if (width <= 0) width = s->plan.cfg.w;
  if (k > s->kmax || itopk > s->plan.cfg.L || k > itopk || width > s->plan.cfg.w)
    return set_error(ALGAS_EINVAL, "submit: k=%d itopk=%d width=%d exceed server limits (%d,%d,%d)", k, itopk, width,
                     s->kmax, s->plan.cfg.L, s->plan.cfg.w);
  const int start = s->next_slot.fetch_add(1, std::memory_order_relaxed);
  const int q = claim_slot(s, start);
  if (q < 0) return ALGAS_EAGAIN;
  s->queue_ns[q] = 0;
  s->inflight.fetch_add(1);
  write_slot(s, q, query, tag, k, itopk, width);
  return ALGAS_OK;
}

int algas_submit_many(algas_server* s, const float* queries, int64_t n, uint64_t tag0, int32_t k, int32_t itopk,
                      int32_t width, int64_t* n_accepted) {
  if (!n_accepted) return set_error(ALGAS_EINVAL, "null n_accepted");
  *n_accepted = 0;
  if (!s || (!queries && n > 0) || n < 0) return set_error(ALGAS_EINVAL, "null argument");
  int64_t i = 0;
  for (; i < n; ++i) {
    const int rc = algas_submit(s, queries + i * (int64_t)s->dim, tag0 + (uint64_t)i, k, itopk, width);
    if (rc == ALGAS_EAGAIN) break;
    if (rc != ALGAS_OK) {
      *n_accepted = i;
      return rc;
    }
  }
  *n_accepted = i;
  return ALGAS_OK;
}

int algas_enqueue(algas_server* s, const float* queries, int64_t n, uint64_t tag0, int32_t k, int32_t itopk,
                  int32_t width) {
  if (!s || (!queries && n > 0) || n < 0) return set_error(ALGAS_EINVAL, "null argument");
  if (s->stop.load()) return set_error(ALGAS_ESTATE, "server is shutting down");
  if (s->quit_when_idle.load()) return set_error(ALGAS_ESTATE, "bounded session: no new work after start");
  if (k <= 0) k = s->kmax;
  if (itopk <= 0) itopk = s->plan.cfg.L;
  if (width <= 0) width = s->plan.cfg.w;
  if (k > s->kmax || itopk > s->plan.cfg.L || k > itopk || width > s->plan.cfg.w)
    return set_error(ALGAS_EINVAL, "enqueue: k=%d itopk=%d width=%d exceed server limits (%d,%d,%d)", k, itopk, width,
                     s->kmax, s->plan.cfg.L, s->plan.cfg.w);
  if (n == 0) return ALGAS_OK;
  const auto now = std::chrono::steady_clock::now();
  // one copy of the whole call (the caller keeps ownership of `queries`)
  auto blk = std::make_shared<const std::vector<float>>(queries, queries + n * (int64_t)s->dim);
  {
    std::lock_guard<std::mutex> lk(s->pq_mu);
    for (int64_t i = 0; i < n; ++i) {
      algas_server::Pending p;
      p.tag = tag0 + (uint64_t)i;
      p.k = k;
      p.L = itopk;
      p.w = width;
      p.t_enq = now;
      p.blk = blk;
      p.off = i * (int64_t)s->dim;
      s->pending.push_back(std::move(p));
    }
    s->inflight.fetch_add(n);
    s->n_pending.fetch_add(n, std::memory_order_acq_rel);
  }
  drain_pending(s, s->next_slot.fetch_add(1, std::memory_order_relaxed));
  return ALGAS_OK;
}

int algas_poll(algas_server* s, uint64_t* tags, uint32_t* ids, float* dists, algas_query_stats* stats,
               int32_t max_results, int32_t* n_out) {
  if (!s || !n_out) return set_error(ALGAS_EINVAL, "null argument");
  *n_out = 0;
  if (max_results <= 0) return ALGAS_OK;
  // a persistent kernel that died is reported, not silently waited on
  if (!s->emulated) {
    cudaError_t e = cudaStreamQuery(s->stream);
    if (e != cudaSuccess && e != cudaErrorNotReady)
      return set_error(ALGAS_ECUDA, "persistent kernel failed: %s", cudaGetErrorString(e));
  }
  if (s->stuck.load(std::memory_order_acquire))
    return set_error(ALGAS_ESTATE, "watchdog: query tag %llu has been in its slot for more than %lld ms",
                     (unsigned long long)s->stuck_tag.load(), (long long)(s->watchdog_ns / 1000000));
  std::lock_guard<std::mutex> lk(s->cq_mu);
  int n = 0;
  while (n < max_results && !s->cq.empty()) {
    algas_server::Done& d = s->cq.front();
    if (tags) tags[n] = d.tag;
    if (ids) memcpy(ids + (size_t)n * s->kmax, d.ids.data(), sizeof(uint32_t) * s->kmax);
    if (dists) memcpy(dists + (size_t)n * s->kmax, d.d.data(), sizeof(float) * s->kmax);
    if (stats) stats[n] = d.st;
    if (s->done_pool.size() < 4096) s->done_pool.push_back(std::move(d));  // keep its buffers for the poller
    s->cq.pop_front();
    ++n;
  }
  s->inflight.fetch_sub(n);
  *n_out = n;
  return ALGAS_OK;
}

int algas_server_inflight(const algas_server* s, int64_t* n) {
  if (!s || !n) return set_error(ALGAS_EINVAL, "null argument");
  *n = s->inflight.load();
  return ALGAS_OK;
}

int algas_server_destroy(algas_server* s) {
  if (!s) return ALGAS_OK;
  int rc = ALGAS_OK;
  if (s->emulated) {
    // Quit every slot, let the emulated device drain and exit, stop the pollers
    if (s->ring_h)
      for (int u = 0; u < 2 * s->slots; ++u) __atomic_store_n(&s->ring_h[u].state, (uint32_t)kSlotQuit, __ATOMIC_RELEASE);
    if (s->emu.joinable()) s->emu.join();
    s->stop.store(true);
    for (auto& th : s->pollers)
      if (th.joinable()) th.join();
    free(s->ring_h);
    free(s->ringq_h);
    free(s->res_h);
    free(s->st_h);
    free(s->done_h);
    delete s->hstate;
    delete s;
    return ALGAS_OK;
  }
  if (s->ring_h && s->stream && s->launched) {
    // Quit: every slot, then wait for the kernel to exit
    for (int u = 0; u < 2 * s->slots; ++u) {
      __atomic_store_n(&s->ring_h[u].state, (uint32_t)kSlotQuit, __ATOMIC_RELEASE);
      if (s->mirror) mirror_publish(s, u, kSlotQuit, false);
    }
    auto t0 = std::chrono::steady_clock::now();
    for (;;) {
      cudaError_t e = cudaStreamQuery(s->stream);
      if (e == cudaSuccess) break;
      if (e != cudaErrorNotReady) {
        rc = set_error(ALGAS_ECUDA, "persistent kernel failed: %s", cudaGetErrorString(e));
        break;
      }
      if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(30)) {
        rc = set_error(ALGAS_ESTATE, "persistent kernel did not quit within 30 s");
        break;
      }
      std::this_thread::sleep_for(std::chrono::microseconds(50));
    }
  }
  s->stop.store(true);
  for (auto& th : s->pollers)
    if (th.joinable()) th.join();
  if (rc == ALGAS_OK) {
    if (s->gtab) cudaFree(s->gtab);
    if (s->vbm) cudaFree(s->vbm);
    if (s->ctl) cudaFree(s->ctl);
    if (s->qbuf) cudaFree(s->qbuf);
    if (s->ring_h) cudaFreeHost(s->ring_h);
    if (s->ringq_h) cudaFreeHost(s->ringq_h);
    if (s->res_h) cudaFreeHost(s->res_h);
    if (s->st_h) cudaFreeHost(s->st_h);
    if (s->done_h) cudaFreeHost(s->done_h);
    if (s->mir_h) cudaFreeHost(s->mir_h);
    if (s->mir_d) cudaFree(s->mir_d);
    for (cudaStream_t st : s->io_streams) cudaStreamDestroy(st);
    if (s->stream) cudaStreamDestroy(s->stream);
    delete s->hstate;
    delete s;
  }
  return rc;
}

int32_t algas_merge_topk(const uint32_t* ids, const float* dists, int32_t m, int32_t k, uint32_t* out_ids,
                         float* out_dists) {
  if (m < 0 || k < 1 || (m > 0 && (!ids || !dists)) || !out_ids || !out_dists)
    return set_error(ALGAS_EINVAL, "algas_merge_topk: bad arguments");
  std::vector<ResultEntry> all;
  all.reserve(m);
  for (int i = 0; i < m; ++i)
    if (ids[i] != kSentinel) all.push_back(ResultEntry{ids[i], dists[i]});
  std::sort(all.begin(), all.end(), [](const ResultEntry& a, const ResultEntry& b) {
    if (a.dist != b.dist) return a.dist < b.dist;
    return a.id < b.id;
  });
  // one sorted list; reuse the T-way merge with T = 1 for the filtering rule
  std::vector<ResultEntry> one(all.size() + 1, ResultEntry{kSentinel, 0.f});
  std::copy(all.begin(), all.end(), one.begin());
  return merge_cta_lists(one.data(), 1, (int)all.size() + 1, k, out_ids, out_dists);
}

int algas_merge_topk_parts(const uint32_t* ids, const float* dists, int32_t nparts, int64_t nq, int32_t m_per,
                           int32_t k, uint32_t* out_ids, float* out_dists) {
  if (!ids || !dists || !out_ids || !out_dists || nparts < 1 || nq < 0 || m_per < 1 || k < 1)
    return set_error(ALGAS_EINVAL, "algas_merge_topk_parts: bad arguments");
  // each part's row is sorted (a shard's TopK): the T-way heap merge applies
  std::vector<ResultEntry> rows((size_t)nparts * m_per);
  for (int64_t q = 0; q < nq; ++q) {
    for (int p = 0; p < nparts; ++p)
      for (int j = 0; j < m_per; ++j) {
        const size_t src = ((size_t)p * nq + q) * m_per + j;
        rows[(size_t)p * m_per + j] = ResultEntry{ids[src], dists[src]};
      }
    merge_cta_lists(rows.data(), nparts, m_per, k, out_ids + q * k, out_dists + q * k);
  }
  return ALGAS_OK;
}

// ------------------------------------------------------------------ tuner
int32_t algas_tuner_max_parallel(int32_t slots, int32_t n_sm, int32_t max_blocks_per_sm) {
  if (slots < 1) return 0;
  return (int32_t)(((int64_t)n_sm * max_blocks_per_sm) / slots);
}
int32_t algas_tuner_blocks_per_sm(int32_t n_parallel, int32_t slots, int32_t n_sm) {
  if (n_sm < 1) return 0;
  const int64_t t = (int64_t)n_parallel * slots;
  return (int32_t)((t + n_sm - 1) / n_sm);  // P:L235, align() = ceil (R13)
}
int64_t algas_tuner_smem_per_block(int64_t smem_per_sm, int32_t blocks_per_sm, int64_t smem_reserved_per_block) {
  if (blocks_per_sm < 1) return 0;
  return smem_per_sm / blocks_per_sm - smem_reserved_per_block;
}

int algas_device_query(algas_device_props* out) {
  if (!out) return set_error(ALGAS_EINVAL, "null out");
  int dev = 0;
  ALGAS_CUDA_TRY(cudaGetDevice(&dev));
  int v = 0;
  memset(out, 0, sizeof(*out));
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev));
  out->n_sm = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMaxBlocksPerMultiprocessor, dev));
  out->max_blocks_per_sm = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
  out->smem_per_sm = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrReservedSharedMemoryPerBlock, dev));
  out->smem_reserved_per_block = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  out->smem_per_block_optin = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMaxThreadsPerMultiProcessor, dev));
  out->max_threads_per_sm = v;
  ALGAS_CUDA_TRY(cudaDeviceGetAttribute(&v, cudaDevAttrMaxRegistersPerMultiprocessor, dev));
  out->regs_per_sm = v;
  return ALGAS_OK;
}

// Full tuner.  Policy ("tuner"), matched to the measured
// optimum of the bench sweeps (profiles/round2_tuner.md):
//  * threads/CTA: the paper fixes one warp.  On B200 a search step
//    is latency-bound (dependent select -> gather -> distance -> merge) and a
//    step's wave of row reads completes fastest with all its rows in flight:
//    1024 threads (the widest CTA, dim <= 512 under its 64-register budget),
//    512 for wider vectors (C3's 960-d rows).
//  * N_parallel: the largest T allowed by P:L231 -- with N_max_block_per_SM
//    = 1, the occupancy of a wide search CTA (its registers fill the SM) --
//    whose per-block shared memory fits P:L245 (with M_reserved grown for
//    wide vectors), capped at T_cap = 8.
//  * width / offset_beam: beam extend from the first step
//    (offset_beam = 1): a step has a fixed latency of ~2 DRAM round
//    trips plus barriers, so fewer, wider steps win on B200 at equal recall;
//    w = 12 for short lists (L <= 32), 16 above.
//  * visited table: SHARED (one per query) when T > 1 -- it removes
//    the multi-CTA redundant evaluations that PRIVATE tables repeat.
int algas_tune(const algas_device_props* props, int32_t slots, int32_t dim, int32_t degree, int32_t itopk, int32_t k,
               algas_tuning* out) {
  if (!out || slots < 1 || dim < 4 || degree < 1 || itopk < 1 || k < 1)
    return set_error(ALGAS_EINVAL, "algas_tune: bad arguments");
  algas_device_props dp;
  if (!props) {
    int rc = algas_device_query(&dp);
    if (rc) return rc;
    props = &dp;
  }
  const int nt = (dim <= 512 && props->max_threads_per_sm >= 1024) ? 1024 : 512;
  const int search_blocks_per_sm = 1;  // occupancy of one wide search CTA
  const int w = std::min(itopk, itopk <= 32 ? 12 : 16);
  int Rp = 4;
  while (Rp < degree) Rp <<= 1;
  const int S = 32;
  int ncap = 1;
  while (ncap < std::max(S, w * Rp)) ncap <<= 1;
  const int cc = chunk_config_for(dim / 4);
  if (cc < 0) return set_error(ALGAS_EINVAL, "algas_tune: dim %d unsupported", dim);
  const int dp4 = chunk_tl(cc) * chunk_cpl(cc);
  // M_reserved_per_block: driver reservation + extra L1 for wide rows
  const int64_t reserved = props->smem_reserved_per_block + (dim > 256 ? 8 * 1024 : 0);
  const int tmax_eq = algas_tuner_max_parallel(slots, props->n_sm, std::min(props->max_blocks_per_sm, search_blocks_per_sm));
  const int tcap = std::min(8, ALGAS_MAX_CTAS);
  int best = 0, best_bps = 0, best_hb = 0, best_sr = 0;
  int64_t best_avail = 0, best_smem = 0;
  for (int T = std::min(tmax_eq, tcap); T >= 1; --T) {
    const int bps = algas_tuner_blocks_per_sm(T, slots, props->n_sm);
    if (bps > props->max_blocks_per_sm) continue;
    if ((int64_t)bps * nt > props->max_threads_per_sm) continue;
    const int64_t avail = algas_tuner_smem_per_block(props->smem_per_sm, bps, reserved);
    int hb = 0, sr = 0;
    choose_smem(dp4, itopk, ncap, S, w, Rp, avail, &hb, &sr);
    const int64_t smem = smem_layout(dp4, itopk, ncap, hb, sr).total;
    if (smem <= avail && smem <= props->smem_per_block_optin - props->smem_reserved_per_block) {
      best = T;
      best_bps = bps;
      best_avail = avail;
      best_hb = hb;
      best_sr = sr;
      best_smem = smem;
      break;
    }
  }
  if (best == 0) return set_error(ALGAS_EINVAL, "algas_tune: no N_parallel fits %d slots", slots);
  memset(out, 0, sizeof(*out));
  out->ctas_per_query = best;
  out->blocks_per_sm = best_bps;
  out->smem_avail_per_block = best_avail;
  out->smem_per_block = best_smem;
  out->threads_per_cta = nt;
  out->width = w;
  out->offset_beam = 1;
  out->hash_bits = best_hb;
  out->stage_rows = best_sr;
  out->visited_mode = best > 1 ? ALGAS_VISITED_SHARED : ALGAS_VISITED_PRIVATE;
  (void)k;
  return ALGAS_OK;
}

}  // extern "C"
