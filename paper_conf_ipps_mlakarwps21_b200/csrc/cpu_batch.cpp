// cpu_batch.cpp -- SURVEY.md §8(f) NEXT-4: the paper's CPU-BATCH, i.e. the
// batch-based RCM of Alg. 5 with its signalling chain run by
// std::thread workers ("each worker ... draws batches from the
// queue"), for host-side context of the paper's multicore numbers
// (Fig. 6).  Not a fallback of the GPU library (include/rcm_cpu.h).
//
// One chain per connected component (C-6 seed order).  Per batch t:
//   s_early = Discovered received?                          (ln 2)
//   discover: owner[c] <- min(owner[c], key(p)), key(p) = pos(p) + 1    (ln 3, C-4)
//   s_mid = Discovered received?                            (ln 4)
//   if s_early or s_mid: forward Discovered, rediscover, try signalCount (ln 5-12)
//   sort each parent's children by (valence, id)            (ln 13, C-1)
//   else: wait Discovered, forward it, rediscover           (ln 14-19)
//   wait Counted, signalCount: successor gets (out_off + count, q_off + nb)
//   output o[out_off ...], generate batches at q_off ... (greedy B_s / T cuts,
//   P:L644-667), empty slots for the rest of the nb reserved.
// Termination: the batch whose output completes the graph, or a
// batch after which no slot is reserved (the component is exhausted).
// Overhang forwarding is a performance option and is not used.
#include "../../include/rcm_cpu.h"

#include <algorithm>
#include <atomic>
#include <memory>
#include <new>
#include <thread>
#include <vector>

namespace {

constexpr uint32_t kUnowned = 0xFFFFFFFFu;

inline void cpu_relax() {
#if defined(__x86_64__) || defined(__i386__)
  __builtin_ia32_pause();
#else
  std::this_thread::yield();
#endif
}

struct Slot {                       // queue slot t = batch descriptor + the signals t receives
  std::atomic<uint32_t> pub{0};     // chain tag when [b, e) is published
  int32_t b = 0, e = 0;
  std::atomic<uint32_t> disc{0};    // chain tag when Discovered was received
  std::atomic<uint32_t> cnt{0};     // chain tag when Counted was received (payload below)
  int32_t out_off = 0, q_off = 0;
};

struct Shared {
  int32_t n = 0;
  const int32_t* rp = nullptr;
  const int32_t* ci = nullptr;
  std::vector<int32_t> deg;                      // valence, P:L209 (C-2)
  std::unique_ptr<std::atomic<uint32_t>[]> owner;  // parent-rank key of the claiming parent
  std::vector<int32_t> o;                        // CM order
  int64_t B = 256, T = 4096;
  int64_t qcap = 0;
  std::unique_ptr<Slot[]> q;
  // per chain
  uint32_t tag = 0;
  int32_t chain_pos0 = 0;
  std::atomic<int32_t> head{0};
  std::atomic<int32_t> done{0};
  std::atomic<int32_t> error{0};
  std::atomic<int32_t> ordered{0};               // nodes placed when the chain ended
  // pool
  std::atomic<uint32_t> gen{0};
  std::atomic<int32_t> finished{0};
  std::atomic<int32_t> shutdown{0};
  // stats
  std::atomic<int64_t> executed{0}, empty{0}, early{0}, late{0}, removed{0};
};

struct Scratch {                                  // one worker's temporary memory
  std::vector<std::vector<uint64_t>> cand;        // children per parent: valence << 32 | id
  std::vector<int32_t> out;
};

inline uint64_t vkey(const Shared& S, int32_t v) { return ((uint64_t)(uint32_t)S.deg[v] << 32) | (uint32_t)v; }

// Wait until `flag` carries the chain tag; false if the chain ended meanwhile.
inline bool wait_tag(const Shared& S, const std::atomic<uint32_t>& flag) {
  for (int it = 0; flag.load(std::memory_order_acquire) != S.tag; ++it) {
    if (S.done.load(std::memory_order_relaxed)) return false;
    if (it < 256) cpu_relax(); else std::this_thread::yield();
  }
  return true;
}

// signalCount: the successor's output offset and queue offset.
// nb = floor(N/B) + max(1, ceil(2V/T)) reserved slots.
void signal_count(Shared& S, int32_t t, int32_t count, int64_t V, int32_t& out_off, int32_t& q_off, int32_t& nb,
                  bool& chain_end) {
  Slot& me = S.q[t];
  out_off = me.out_off;
  q_off = me.q_off;
  nb = 0;
  if (count > 0) {
    const int64_t v2 = (2 * V + S.T - 1) / S.T;
    nb = (int32_t)(count / S.B + (v2 > 1 ? v2 : 1));
  }
  if ((int64_t)q_off + nb + 1 > S.qcap) {
    S.error.store(5);
    S.done.store(1);
    nb = 0;
  }
  Slot& succ = S.q[t + 1];
  succ.out_off = out_off + count;
  succ.q_off = q_off + nb;
  succ.cnt.store(S.tag, std::memory_order_release);
  chain_end = (q_off + nb == t + 1);   // nothing reserved after t: component exhausted
}

void forward_discovered(Shared& S, int32_t t) { S.q[t + 1].disc.store(S.tag, std::memory_order_release); }

// Alg. 4 rediscover: keep n iff it is still owned by p's key.
int64_t rediscover(Shared& S, Scratch& W, int32_t b, int32_t np) {
  int64_t removed = 0;
  for (int32_t i = 0; i < np; ++i) {
    const uint32_t key = (uint32_t)b + 1 + (uint32_t)i;
    auto& c = W.cand[i];
    const size_t before = c.size();
    c.erase(std::remove_if(c.begin(), c.end(),
                           [&](uint64_t k) {
                             return S.owner[(uint32_t)k].load(std::memory_order_relaxed) != key;
                           }),
            c.end());
    removed += (int64_t)(before - c.size());
  }
  return removed;
}

void process_batch(Shared& S, Scratch& W, int32_t t) {
  Slot& me = S.q[t];
  const int32_t b = me.b, e = me.e, np = e - b;
  if (np == 0) {   // empty slot: pass both signals on unchanged
    S.empty.fetch_add(1, std::memory_order_relaxed);
    if (!wait_tag(S, me.disc)) return;
    forward_discovered(S, t);
    if (!wait_tag(S, me.cnt)) return;
    int32_t out_off, q_off, nb;
    bool chain_end;
    signal_count(S, t, 0, 0, out_off, q_off, nb, chain_end);
    if (chain_end) {
      S.ordered.store(out_off);
      S.done.store(1);
    }
    return;
  }
  if ((int32_t)W.cand.size() < np) W.cand.resize(np);
  const bool s_early = me.disc.load(std::memory_order_acquire) == S.tag;   // ln 2
  // ln 3: speculative discovery with parent-rank keys (C-4)
  bool steal = false;
  const uint32_t klast = (uint32_t)e;
  for (int32_t i = 0; i < np; ++i) {
    const int32_t p = S.o[b + i];
    const uint32_t key = (uint32_t)b + 1 + (uint32_t)i;
    auto& c = W.cand[i];
    c.clear();
    for (int32_t x = S.rp[p]; x < S.rp[p + 1]; ++x) {
      const int32_t ch = S.ci[x];
      uint32_t old = S.owner[ch].load(std::memory_order_relaxed);
      while (old > key && !S.owner[ch].compare_exchange_weak(old, key, std::memory_order_relaxed)) {
      }
      if (old > key) {
        c.push_back(vkey(S, ch));
        steal |= old <= klast;   // taken from a sibling parent of this batch
      }
    }
  }
  std::atomic_thread_fence(std::memory_order_release);
  const bool s_mid = me.disc.load(std::memory_order_acquire) == S.tag;   // ln 4
  bool rediscovered = false, counted = false, chain_end = false;
  const bool early_path = s_early || s_mid;
  int32_t out_off = 0, q_off = 0, nb = 0, count = 0;
  int64_t V = 0;
  auto tally = [&] {
    count = 0;
    V = 0;
    for (int32_t i = 0; i < np; ++i) {
      count += (int32_t)W.cand[i].size();
      for (uint64_t k : W.cand[i]) V += std::min<int64_t>((int64_t)(k >> 32), S.T);
    }
  };
  if (s_early || s_mid) {   // ln 5-12: forward Discovered, rediscover before sorting
    forward_discovered(S, t);
    if (!s_early || steal) S.removed.fetch_add(rediscover(S, W, b, np), std::memory_order_relaxed);
    rediscovered = true;
    tally();
    if (me.cnt.load(std::memory_order_acquire) == S.tag) {
      signal_count(S, t, count, V, out_off, q_off, nb, chain_end);
      counted = true;
    }
  }
  for (int32_t i = 0; i < np; ++i) std::sort(W.cand[i].begin(), W.cand[i].end());   // ln 13 (C-1)
  if (!rediscovered) {   // ln 14-19
    if (!wait_tag(S, me.disc)) return;
    forward_discovered(S, t);
    S.removed.fetch_add(rediscover(S, W, b, np), std::memory_order_relaxed);
    tally();
  }
  if (!counted) {   // ln 20-22
    if (!wait_tag(S, me.cnt)) return;
    signal_count(S, t, count, V, out_off, q_off, nb, chain_end);
  }
  // ln 23-26: output in parent order, each parent's children sorted
  int32_t pos = out_off;
  for (int32_t i = 0; i < np; ++i)
    for (uint64_t k : W.cand[i]) S.o[pos++] = (int32_t)(uint32_t)k;
  // generation: greedy cuts at B_s nodes / T summed clamped valence
  int32_t emitted = 0, start = out_off, cnt = 0;
  int64_t val = 0;
  auto close = [&](int32_t end) {
    Slot& d = S.q[q_off + emitted];
    d.b = start;
    d.e = end;
    d.pub.store(S.tag, std::memory_order_release);
    ++emitted;
    start = end;
    cnt = 0;
    val = 0;
  };
  for (int32_t k = out_off; k < out_off + count; ++k) {
    const int64_t cv = std::min<int64_t>(S.deg[S.o[k]], S.T);
    if (cnt > 0 && (cnt + 1 > S.B || val + cv > S.T)) close(k);
    ++cnt;
    val += cv;
  }
  if (cnt > 0) close(out_off + count);
  for (; emitted < nb; ++emitted) {   // unused reservations: empty batches
    Slot& d = S.q[q_off + emitted];
    d.b = d.e = 0;
    d.pub.store(S.tag, std::memory_order_release);
  }
  // early/late tallied with `executed`, so a batch abandoned at termination
  // (it returns at a wait above) counts in none of them
  (early_path ? S.early : S.late).fetch_add(1, std::memory_order_relaxed);
  S.executed.fetch_add(1, std::memory_order_relaxed);
  if (out_off + count == S.n || chain_end) {   // termination
    S.ordered.store(out_off + count);
    S.done.store(1);
  }
}

void worker_loop(Shared& S, Scratch& W) {
  while (!S.done.load(std::memory_order_relaxed)) {
    const int32_t t = S.head.fetch_add(1, std::memory_order_relaxed);
    if (t + 1 >= S.qcap) {   // only after a capacity error
      S.error.store(5);
      S.done.store(1);
      return;
    }
    if (!wait_tag(S, S.q[t].pub)) return;
    process_batch(S, W, t);
  }
}

// BFS levels from r over r's component (GL finder); returns #levels, lev[] set.
int32_t bfs_levels(const Shared& S, int32_t r, std::vector<int32_t>& lev, std::vector<int32_t>& fifo,
                   std::vector<int32_t>& touched) {
  for (int32_t v : touched) lev[v] = -1;
  touched.clear();
  fifo.clear();
  fifo.push_back(r);
  lev[r] = 0;
  touched.push_back(r);
  int32_t nl = 1;
  for (size_t h = 0; h < fifo.size(); ++h) {
    const int32_t p = fifo[h];
    for (int32_t x = S.rp[p]; x < S.rp[p + 1]; ++x) {
      const int32_t c = S.ci[x];
      if (lev[c] < 0) {
        lev[c] = lev[p] + 1;
        nl = std::max(nl, lev[c] + 1);
        fifo.push_back(c);
        touched.push_back(c);
      }
    }
  }
  return nl;
}

// GL pseudo-peripheral finder (C-5): restart from the lowest
// (valence, id) node of the last level until the level count stops growing;
// return the last root.
int32_t gl_finder(const Shared& S, int32_t r, std::vector<int32_t>& lev) {
  std::vector<int32_t> fifo, touched;
  int32_t nl = bfs_levels(S, r, lev, fifo, touched);
  for (;;) {
    int32_t x = -1;
    uint64_t best = ~0ull;
    for (int32_t v : fifo)
      if (lev[v] == nl - 1 && vkey(S, v) < best) { best = vkey(S, v); x = v; }
    const int32_t nx = bfs_levels(S, x, lev, fifo, touched);
    if (nx <= nl) {
      for (int32_t v : touched) lev[v] = -1;
      return x;
    }
    nl = nx;
  }
}

}  // namespace

extern "C" int rcm_cpu_batch(int32_t n, const int32_t* row_ptr, const int32_t* col_idx, int32_t mode, int32_t start,
                             int32_t threads, int32_t batch_nodes, int32_t temp_elems, int32_t* perm,
                             rcm_cpu_stats_t* stats) {
  if (n < 0 || !row_ptr || !perm || mode < 0 || mode > 2 || batch_nodes < 0 || temp_elems < 0) return 1;
  if (n == 0) return 0;
  if (row_ptr[n] > 0 && !col_idx) return 1;
  if (mode == 0 && (start < 0 || start >= n)) return 1;
  int nt = threads > 0 ? threads : (int)std::thread::hardware_concurrency();
  if (nt < 1) nt = 1;
  Shared S;
  try {
    S.n = n;
    S.rp = row_ptr;
    S.ci = col_idx;
    S.B = batch_nodes ? batch_nodes : 256;
    S.T = temp_elems ? temp_elems : 4096;
    S.deg.resize(n);
    for (int32_t v = 0; v < n; ++v) S.deg[v] = row_ptr[v + 1] - row_ptr[v];
    S.owner.reset(new std::atomic<uint32_t>[n]);
    for (int32_t v = 0; v < n; ++v) S.owner[v].store(kUnowned, std::memory_order_relaxed);
    S.o.assign(n, -1);
    const int64_t nnz = row_ptr[n];
    S.qcap = 2 * (int64_t)n + n / S.B + 2 * (nnz / S.T + 1) + 64;
    S.q.reset(new Slot[S.qcap]);
  } catch (const std::bad_alloc&) {
    return 2;
  }
  std::vector<Scratch> scratch(nt);
  // worker pool: threads 1..nt-1 join each chain released by `gen`
  std::vector<std::thread> pool;
  for (int w = 1; w < nt; ++w) {
    pool.emplace_back([&S, &scratch, w] {
      uint32_t seen = 0;
      for (;;) {
        uint32_t g;
        for (int it = 0; (g = S.gen.load(std::memory_order_acquire)) == seen; ++it) {
          if (S.shutdown.load(std::memory_order_relaxed)) return;
          if (it < 1024) cpu_relax(); else std::this_thread::yield();
        }
        seen = g;
        worker_loop(S, scratch[w]);
        S.finished.fetch_add(1, std::memory_order_acq_rel);
      }
    });
  }
  // C-6 seed order: ascending (valence, id)
  std::vector<uint64_t> order(n);
  for (int32_t v = 0; v < n; ++v) order[v] = vkey(S, v);
  std::sort(order.begin(), order.end());
  std::vector<int32_t> lev(mode == 2 ? n : 0, -1);
  int32_t len = 0, cursor = 0, chains = 0;
  bool first = true;
  while (len < n && !S.error.load()) {
    int32_t s;
    if (first && mode == 0) {
      s = start;
    } else {
      while (S.owner[(int32_t)(uint32_t)order[cursor]].load(std::memory_order_relaxed) != kUnowned) ++cursor;
      s = (int32_t)(uint32_t)order[cursor];
      if (mode == 2) s = gl_finder(S, s, lev);
    }
    first = false;
    S.owner[s].store((uint32_t)len, std::memory_order_relaxed);   // root key: smaller than every parent key
    S.o[len] = s;
    if (S.deg[s] == 0) {   // isolated node: nothing to traverse
      ++len;
      continue;
    }
    // chain set-up: slot 0 = the seed batch, its virtual predecessor has
    // Discovered and Counted with out_off = len + 1, q_off = 1
    ++chains;
    S.tag = (uint32_t)chains;
    S.chain_pos0 = len;
    S.q[0].b = len;
    S.q[0].e = len + 1;
    S.q[0].out_off = len + 1;
    S.q[0].q_off = 1;
    S.q[0].disc.store(S.tag, std::memory_order_relaxed);
    S.q[0].cnt.store(S.tag, std::memory_order_relaxed);
    S.q[0].pub.store(S.tag, std::memory_order_relaxed);
    S.head.store(0);
    S.done.store(0);
    S.ordered.store(len + 1);
    S.finished.store(0);
    S.gen.fetch_add(1, std::memory_order_acq_rel);   // release the pool
    worker_loop(S, scratch[0]);
    while (S.finished.load(std::memory_order_acquire) < nt - 1) std::this_thread::yield();
    len = S.ordered.load();
  }
  S.shutdown.store(1);
  for (auto& th : pool) th.join();
  if (S.error.load()) return S.error.load();
  for (int32_t k = 0; k < n; ++k) perm[k] = S.o[n - 1 - k];   // reverse(o)
  if (stats) {
    stats->batches_executed = S.executed.load();
    stats->batches_empty = S.empty.load();
    stats->rediscover_early = S.early.load();
    stats->rediscover_late = S.late.load();
    stats->candidates_removed = S.removed.load();
    stats->chains = chains;
  }
  return 0;
}
