// rcm_batch.cuh -- per-batch work of the batch-based RCM (one persistent thread
// block = one worker): parent load, speculative discovery,
// rediscovery, per-parent (valence, id) sort, output with fused reverse, and
// batch generation with work aggregation.  Citations P:L<n> = PAPER.md line n.
#pragma once
#include "rcm_device.cuh"

namespace rcm {

// Kernel-wide parameters (passed by value to every kernel).
struct KParams {
  const int32_t* row_ptr;
  const int32_t* col_idx;
  unsigned long long* word;   // per node: owner key (hi 32) | valence (lo 32)
  int32_t* o;                 // CM order (matrix-local ids at matrix-local positions)
  int32_t* perm;              // output, new -> old
  int32_t* iperm;             // nullable, old -> new (single graph)
  Desc* desc;                 // batch queue
  Sig* sig;                   // per-slot signals (qcap + 1)
  Ctl* ctl;
  Stats* stats;
  const Problem* chains;
  const Problem* solos;
  unsigned long long* spill;  // oversize scratch: [0, spill_cap) keys, [spill_cap, 2*spill_cap) temp
  int64_t spill_cap;
  int32_t qcap;
  int32_t BS;                 // B_s capacity (shared-memory layout)
  int32_t T;                  // temp-element capacity per batch (shared memory)
  int32_t Bg;                 // B_s used to cut new batches (<= BS)
  int32_t Tg;                 // valence budget used to cut new batches (<= T)
  int32_t flags;
  int32_t collect_stats;
  int32_t nblocks;
  int32_t* dbg;               // per-block progress (8 ints per block), always written
  unsigned long long* trace;  // nullable: per-slot event times (collect_stats == 3)
  int32_t trace_cap;          // slots traced
  uint32_t* fwdv;             // look-back chain, per slot that forwards its output: [2t] count, [2t+1] valence
};

// Per-slot event trace (collect_stats == 3), kTraceW words per slot:
// %globaltimer at dequeue (0), parents loaded (1), discovery done (2),
// Discovered known (3), aggregate published (4), before the prefix look-back
// (5), prefix known (6), output written (7), batches published (8);
// [kTraceW-1] = generator slot << 32 | block.  Thread 0 only.
constexpr int kTraceW = 16;
static __device__ __noinline__ void trace_ev_slow(unsigned long long* trace, int cap, int slot, int ev) {
  if (trace && slot >= 0 && slot < cap) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    trace[(size_t)slot * kTraceW + ev] = t;
  }
}
// Compiled in only with -DRCM_TRACE (the extra code changes the inlining and
// register allocation of the persistent kernel).
__device__ __forceinline__ void trace_ev(const KParams& kp, int slot, int ev) {
#ifdef RCM_TRACE
  if (kp.collect_stats == 3 && threadIdx.x == 0) trace_ev_slow(kp.trace, kp.trace_cap, slot, ev);
#endif
}

// Per-block progress beacon: phase, slot, aux, SM clock -- polled by the host
// while the kernel runs (rcm_debug_state) to diagnose stalls.  Thread 0 only.
// Store-only: a read-modify-write here would put a memory round trip on the
// block's critical path at every call.
__device__ __forceinline__ void beacon(const KParams& kp, int phase, int slot, int aux) {
  if (threadIdx.x == 0) {
    volatile int32_t* d = kp.dbg + blockIdx.x * 8;
    d[0] = phase;
    d[1] = slot;
    d[2] = aux;
    d[3] = (int32_t)clock();
  }
}

enum : int32_t { F_NO_OVERHANG = 1, F_NO_EARLY = 2, F_NO_SORT = 4, F_FORCE_CHAIN = 8, F_SERIAL_CHAIN = 16,
                 F_LEVELED = 32, F_MULTI_BATCH = 64 };


// Dynamic shared memory of one worker.  The layout is recomputed from the
// kernel parameters (constant bank) at every use instead of being held in
// registers:
//   cand  T+1 candidate keys (valence << 32 | id); reused for prefixes
//   lpof  T local parent id of every edge slot (u16)
//   p_v   BS parent ids
//   p_rs  BS row starts (local, add ci_base)
//   p_eo  BS+1 edge-slot offsets (exclusive prefix of row lengths)
//   p_cnt BS slots used (claims) per parent
extern __shared__ __align__(16) unsigned char rcm_dsm[];
// multi-batch execution (F_MULTI_BATCH): byte offset of the current batch
// context's scratch (0 or the context size); always 0 otherwise
__shared__ uint32_t rcm_ctx_base;
struct SmemPtrs {};
__device__ __forceinline__ unsigned char* sm_base(const KParams& kp) {
  return rcm_dsm + rcm_ctx_base;
}
__device__ __forceinline__ unsigned long long* sm_cand(const KParams& kp) {
  return reinterpret_cast<unsigned long long*>(sm_base(kp));
}
__device__ __forceinline__ uint16_t* sm_lpof(const KParams& kp) {
  return reinterpret_cast<uint16_t*>(sm_base(kp) + 8 * ((size_t)kp.T + 1));
}
__device__ __forceinline__ int32_t* sm_ip(const KParams& kp) {
  return reinterpret_cast<int32_t*>(sm_base(kp) + ((8 * ((size_t)kp.T + 1) + 2 * (size_t)kp.T + 15) & ~size_t(15)));
}
__device__ __forceinline__ int32_t* sm_p_v(const KParams& kp) { return sm_ip(kp); }
__device__ __forceinline__ int32_t* sm_p_rs(const KParams& kp) { return sm_ip(kp) + kp.BS; }
__device__ __forceinline__ int32_t* sm_p_eo(const KParams& kp) { return sm_ip(kp) + 2 * kp.BS; }        // BS + 1
__device__ __forceinline__ int32_t* sm_p_cnt(const KParams& kp) { return sm_ip(kp) + 3 * kp.BS + 1; }

__host__ __device__ inline size_t smem_bytes(int BS, int T) {
  return sizeof(unsigned long long) * (size_t)(T + 1) + 2 * (size_t)T + 16 +
         sizeof(int32_t) * (size_t)(4 * BS + 2) + 64;
}

// Leveled traversal (rcm_leveled.cuh): shared memory after the batch layout --
// the ids of the children the block wrote last, its output buffer, and the
// long rows of its discovery.
constexpr int kLvStage = 1024;   // children ids staged per block
constexpr int kLvOut = 2048;     // children buffered per block before HBM scratch
constexpr int kLvBig = 256;      // long rows expanded by the whole block (per D pass)
__host__ __device__ inline size_t lv_smem_base(int BS, int T) { return (smem_bytes(BS, T) + 15) & ~size_t(15); }
constexpr size_t kLvExtraBytes = 4 * ((size_t)kLvStage + kLvOut + 3 * (size_t)kLvBig + 1);

// Static shared state of one worker.
constexpr int kLvList = 32;   // leveled traversal: output regions per block and round
struct ShState {
  unsigned long long wtmp64[kWarps + 1];
  long long wtmp64b[kWarps + 1];
  int32_t wtmp32[kWarps + 1];
  long long wtmpll[kWarps + 1];
  int32_t t, o_begin, o_end, next;
  int32_t nP, E, steal, removed;
  int32_t s_early, s_mid, counted, aborted;
  int32_t mb, mb_it;           // multi-batch execution: phase (PH_*) and poll counter of this context
  unsigned long long sigw;     // last signal word read from this batch's slot
  int32_t out_off, q_off, ovh_n, ovh_t;
  int32_t fwd, nb, count, chain_end;
  long long V;
  int32_t k, written, pos, big_n;
  unsigned long long minkey;
  int64_t spill_base;
  uint32_t* ovbits;            // oversize claims bitmap (shared memory, or HBM scratch for long rows)
  int32_t big_list[256];
  int32_t lv_off[kLvList], lv_cnt[kLvList], lv_n, lv_outn, lv_cap;   // leveled traversal: this block's output list
  long long clk[10];           // per-stage cycle accumulators (thread 0)
  long long tclk;
  Problem prob;                // the problem being traversed (chain or solo)
};

// Stage clock: attribute the cycles since the last mark to stage i (thread 0).
__device__ __forceinline__ void clk_mark(const KParams& kp, ShState& sh, int i) {
  if (kp.collect_stats == 2 && threadIdx.x == 0) {
    const long long now = clock64();
    sh.clk[i] += now - sh.tclk;
    sh.tclk = now;
  }
}

__device__ __forceinline__ void latch_error(Ctl* ctl, int32_t code) {
  atomicCAS(&ctl->status, 0, code);
  atomicExch(&ctl->done, 1);
}

// Watchdog expiry: record where (site) and on what, then latch RCM_ERR_HANG.
__device__ __forceinline__ void latch_hang(Ctl* ctl, int site, long long a, long long b, long long c) {
  if (atomicCAS(&ctl->status, 0, ST_HANG) == 0) {
    ctl->dbg[0] = site; ctl->dbg[1] = a; ctl->dbg[2] = b; ctl->dbg[3] = c;
    ctl->dbg[4] = blockIdx.x;
  }
  atomicExch(&ctl->done, 1);
}

// ---------------------------------------------------------------- signals
// One acquire load returns state + payload (Sig::word).
__device__ __forceinline__ unsigned long long load_sig(const Sig* s) { return ld_acquire_u64(&s->word); }

__device__ __forceinline__ void send_sig(Sig* s, unsigned long long w) { st_release_u64(&s->word, w); }

// Busy wait: tight polling first, then sleep back-off.  Returns
// the signal word, or 0 if the chain was terminated (done) or the watchdog fired.
static __device__ unsigned long long wait_sig(const Sig* s, uint32_t need, Ctl* ctl) {
  unsigned long long w = load_sig(s);
  if (sig_state(w) >= need) return w;
  uint64_t t0 = 0;
  unsigned ns = 0;
  for (int it = 0;; ++it) {
    if (ld_relaxed_s32(&ctl->done)) return 0;
    if (it >= 64) {
      __nanosleep(ns);
      if (ns < 256) ns = ns ? ns * 2 : 32;
    }
    w = load_sig(s);
    if (sig_state(w) >= need) return w;
    if ((it & 1023) == 1023) {
      if (t0 == 0) t0 = globaltimer();
      else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(ctl, 5, need, (long long)w, 0); return 0; }
    }
  }
}

// ----------------------------------------------------------- parent load
// Load the parents o[o_base + o_begin + lp], lp < nP, their row starts and the
// exclusive prefix of their row lengths into p_eo.  If cut_T, shrink nP to the
// longest prefix whose edge count fits T (at least one parent) -- the solo
// worker's batch formation.  Returns nP; sh.E = edge slots.
static __device__ int load_parents(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                            int o_begin, int nP, bool cut_T) {
  for (int lp = threadIdx.x; lp < nP; lp += kThreads) {
    int v = ld_cg_s32(kp.o + P.o_base + o_begin + lp);
    const int32_t* rp = kp.row_ptr + P.rp_base + v;
    int rs = __ldg(rp), re = __ldg(rp + 1);
    sm_p_v(kp)[lp] = v;
    sm_p_rs(kp)[lp] = rs;
    sm_p_eo(kp)[lp] = re - rs;
  }
  __syncthreads();
  int E = block_scan_array<int32_t>(sm_p_eo(kp), nP, sh.wtmp32);
  sm_p_eo(kp)[nP] = E;   // (visible after the barrier below)
  __syncthreads();
  if (cut_T && E > kp.T && nP > 1) {
    // largest nP' with p_eo[nP'] <= T (p_eo is non-decreasing); at least 1.
    if (threadIdx.x == 0) {
      int lo = 1, hi = nP;   // p_eo[lo] may exceed T when the first row alone is oversize
      while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (sm_p_eo(kp)[mid] <= kp.T) lo = mid; else hi = mid - 1;
      }
      sh.nP = lo;
    }
    __syncthreads();
    nP = sh.nP;
    E = sm_p_eo(kp)[nP];
  }
  if (threadIdx.x == 0) { sh.nP = nP; sh.E = E; }
  // local parent of every edge slot, one warp per parent (discovery and the
  // later passes read it instead of searching p_eo per slot)
  if (E <= kp.T) {
    const int lane = threadIdx.x & 31;
    for (int lp = threadIdx.x >> 5; lp < nP; lp += kWarps) {
      const int eb = sm_p_eo(kp)[lp], ee = sm_p_eo(kp)[lp + 1];
      for (int j = eb + lane; j < ee; j += 32) sm_lpof(kp)[j] = (uint16_t)lp;
    }
  }
  __syncthreads();
  return nP;
}

// largest lp in [lo, nP) with p_eo[lp] <= e
__device__ __forceinline__ int find_parent(const int32_t* p_eo, int lo, int nP, int e) {
  int hi = nP - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (p_eo[mid] <= e) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// -------------------------------------------------- speculative discovery
// Alg. 4 discover with parent-rank keys (C-4):
// key(p) = pos(p) + 1; m_n <- atomicMin(word[n], key); n is a candidate of p
// iff the old owner was larger.  The valence comes back in the same 64-bit word
// ("immediately compute the valence").  Candidates go to p's segment
// of the scratchpad ("atomicAdd to reserve a unique spot").
static __device__ void discover(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                         int o_begin, int nP, int E) {
  for (int lp = threadIdx.x; lp < nP; lp += kThreads) sm_p_cnt(kp)[lp] = 0;
  __syncthreads();
  const uint32_t kfirst = (uint32_t)o_begin + 1, klast = (uint32_t)o_begin + (uint32_t)nP;
  int steal = 0, claims = 0;
  unsigned long long* word = kp.word + P.node_base;
  const int32_t* col = kp.col_idx + P.ci_base;
  // kDiscU edges per thread per round, each memory step issued for all of them
  // before any result is used: the three dependent round trips (column,
  // owner word, atomicMin) are paid once per round instead of once per edge.
  for (int e0 = threadIdx.x; e0 < E; e0 += kThreads * kDiscU) {
    // the local parent of a slot is re-read from shared memory (lpof) where it
    // is needed instead of being held in registers across the three steps
    int c[kDiscU];
    unsigned long long w[kDiscU];
#pragma unroll
    for (int u = 0; u < kDiscU; ++u) {
      const int e = e0 + u * kThreads;
      c[u] = -1;
      if (e < E) {
        const int lp = sm_lpof(kp)[e];
        c[u] = __ldg(col + sm_p_rs(kp)[lp] + (e - sm_p_eo(kp)[lp]));
      }
    }
#pragma unroll
    for (int u = 0; u < kDiscU; ++u) w[u] = c[u] >= 0 ? ld_weak_u64(word + c[u]) : 0ull;   // prefilter
#pragma unroll
    for (int u = 0; u < kDiscU; ++u) {
      if (c[u] < 0) continue;
      const uint32_t key = kfirst + (uint32_t)sm_lpof(kp)[e0 + u * kThreads];
      if ((uint32_t)(w[u] >> 32) > key)
        w[u] = atomicMin(word + c[u], ((unsigned long long)key << 32) | (w[u] & 0xffffffffull));
      else
        c[u] = -1;
    }
#pragma unroll
    for (int u = 0; u < kDiscU; ++u) {
      if (c[u] < 0) continue;
      const int lp = sm_lpof(kp)[e0 + u * kThreads];
      const uint32_t key = kfirst + (uint32_t)lp;
      const uint32_t ow = (uint32_t)(w[u] >> 32);
      if (ow > key) {
        int slot = sm_p_eo(kp)[lp] + atomicAdd(&sm_p_cnt(kp)[lp], 1);
        sm_cand(kp)[slot] = ((w[u] & 0xffffffffull) << 32) | (uint32_t)c[u];
        steal |= (ow <= klast);   // taken from a sibling parent of this batch
        ++claims;
      }
    }
  }
  if (__syncthreads_or(steal) && threadIdx.x == 0) sh.steal = 1;
  if (kp.collect_stats) {
    int tot = block_reduce_sum<int32_t>(claims, sh.wtmp32);
    if (threadIdx.x == 0 && tot) atomicAdd(&kp.stats->cand_spec, (unsigned long long)tot);
  }
  __syncthreads();
}

// ------------------------------------------------------------ rediscovery
// Alg. 4 rediscover fused with the count of the batch's outputs:
// if `check`, drop n from c when a predecessor (or a sibling parent with a
// smaller key) owns it now -- keep iff owner(n) == key(p); removed candidates
// become kKeyMax.  Then sh.count = kept children and sh.V = the sum of their
// valences clamped to Tg (oversize valences are clamped, they get
// their own batch).  One combined block reduction.
static __device__ void rediscover_count(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                                 int o_begin, int E, bool check) {
  const unsigned long long* word = kp.word + P.node_base;
  long long kr = 0, val = 0;   // kept << 32 | removed, clamped valence sum
  // kDiscU owner re-reads per thread in flight (see discover); only the owner
  // keys stay in registers, the slots are re-read from shared memory
  for (int e0 = threadIdx.x; e0 < E; e0 += kThreads * kDiscU) {
    uint32_t ow[kDiscU];
    if (check) {
#pragma unroll
      for (int u = 0; u < kDiscU; ++u) {
        const int e = e0 + u * kThreads;
        ow[u] = 0;
        if (e < E) {
          const int lp = sm_lpof(kp)[e];
          const unsigned long long k = sm_cand(kp)[e];
          if (e - sm_p_eo(kp)[lp] < sm_p_cnt(kp)[lp] && k != kKeyMax)
            ow[u] = (uint32_t)(ld_weak_u64(word + (uint32_t)k) >> 32);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < kDiscU; ++u) {
      const int e = e0 + u * kThreads;
      if (e >= E) continue;
      const int lp = sm_lpof(kp)[e];
      const unsigned long long k = sm_cand(kp)[e];
      if (e - sm_p_eo(kp)[lp] >= sm_p_cnt(kp)[lp] || k == kKeyMax) continue;
      if (check && ow[u] != (uint32_t)o_begin + 1 + (uint32_t)lp) {
        sm_cand(kp)[e] = kKeyMax;
        kr += 1;
      } else {
        const long long d = (long long)(k >> 32);
        kr += 1ll << 32;
        val += d < kp.Tg ? d : kp.Tg;
      }
    }
  }
  block_reduce_sum2(kr, val, sh.wtmpll, sh.wtmp64b);
  if (threadIdx.x == 0) {
    sh.count = (int)(kr >> 32);
    sh.V = val;
    sh.removed = (int)(kr & 0xffffffffll);
    if (kp.collect_stats && sh.removed) atomicAdd(&kp.stats->cand_removed, (unsigned long long)sh.removed);
  }
  __syncthreads();
}

// ------------------------------------------------------------------ sort
// Ascending sort of keys a[0..n) with a bitonic network in which every
// comparator places the minimum at the lower index (the "flip" formulation), so
// virtual +inf padding beyond n needs no storage.  Executed by `nthr` threads
// (tid = rank in the group); `sync()` is the group barrier.
template <typename Sync>
__device__ __forceinline__ void bitonic_sort_flip(unsigned long long* a, int n, int tid, int nthr,
                                                  Sync sync) {
  int N = 1;
  while (N < n) N <<= 1;
  for (int k = 2; k <= N; k <<= 1) {
    // flip stage: compare i with the mirrored partner inside each k-block
    for (int i = tid; i < N / 2; i += nthr) {
      int blk = i / (k / 2);
      int off = i % (k / 2);
      int lo = blk * k + off;
      int hi = blk * k + k - 1 - off;
      if (hi < n) {
        unsigned long long x = a[lo], y = a[hi];
        if (y < x) { a[lo] = y; a[hi] = x; }
      }
    }
    sync();
    for (int j = k / 4; j > 0; j >>= 1) {
      for (int i = tid; i < N / 2; i += nthr) {
        int blk = i / j;
        int off = i % j;
        int lo = blk * 2 * j + off;
        int hi = lo + j;
        if (hi < n) {
          unsigned long long x = a[lo], y = a[hi];
          if (y < x) { a[lo] = y; a[hi] = x; }
        }
      }
      sync();
    }
  }
}

// Sort every parent's segment cand[p_eo[lp] .. p_eo[lp] + p_cnt[lp]) by
// (valence, id) -- Alg. 1 ln 14 "sort(c)" per parent, equivalently the
// GPU key (local parent, valence) of P:L778-781 with the id tie-break of C-1.
// Tiny segments: one thread (insertion sort); medium: one warp; large: block.
static __device__ void sort_segments(const KParams& kp, const SmemPtrs& sm, ShState& sh, int nP) {
  if (threadIdx.x == 0) sh.big_n = 0;
  __syncthreads();
  for (int lp = threadIdx.x; lp < nP; lp += kThreads) {
    int n = sm_p_cnt(kp)[lp];
    if (n <= 1) continue;
    unsigned long long* a = sm_cand(kp) + sm_p_eo(kp)[lp];
    if (n <= 16) {
      for (int i = 1; i < n; ++i) {
        unsigned long long x = a[i];
        int j = i - 1;
        while (j >= 0 && a[j] > x) { a[j + 1] = a[j]; --j; }
        a[j + 1] = x;
      }
    } else {
      int idx = atomicAdd(&sh.big_n, 1);
      if (idx < 256) sh.big_list[idx] = lp;
    }
  }
  __syncthreads();
  int nbig = sh.big_n;
  if (nbig == 0) return;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (nbig <= 256) {
    // warp-level for segments <= 4096, the rest block-level below
    for (int b = wid; b < nbig; b += kWarps) {
      int lp = sh.big_list[b];
      int n = sm_p_cnt(kp)[lp];
      if (n > 4096) continue;
      bitonic_sort_flip(sm_cand(kp) + sm_p_eo(kp)[lp], n, lane, 32, [] { __syncwarp(); });
    }
    __syncthreads();
    for (int b = 0; b < nbig; ++b) {
      int lp = sh.big_list[b];
      int n = sm_p_cnt(kp)[lp];
      if (n <= 4096) continue;
      bitonic_sort_flip(sm_cand(kp) + sm_p_eo(kp)[lp], n, threadIdx.x, kThreads, [] { __syncthreads(); });
    }
  } else {
    // too many large segments for the list: one warp per segment, scanning all
    for (int lp = wid; lp < nP; lp += kWarps) {
      int n = sm_p_cnt(kp)[lp];
      if (n <= 16 || n > 4096) continue;
      bitonic_sort_flip(sm_cand(kp) + sm_p_eo(kp)[lp], n, lane, 32, [] { __syncwarp(); });
    }
    __syncthreads();
    for (int lp = 0; lp < nP; ++lp) {
      int n = sm_p_cnt(kp)[lp];
      if (n <= 4096) continue;
      bitonic_sort_flip(sm_cand(kp) + sm_p_eo(kp)[lp], n, threadIdx.x, kThreads, [] { __syncthreads(); });
    }
  }
  __syncthreads();
}

// Output (Alg. 5 ln 24-27): the kept children in array order
// (parent segments in parent order, each sorted) at o[out_off ...]; the RCM
// permutation is written reversed in the same pass (perm[N-1-pos] = o[pos],
// P:L219) and optionally its inverse.  Kept = inside the parent's claims and
// not removed (kKeyMax), so removed children need no re-sort.  One block scan
// of (kept << 40 | clamped valence) over contiguous per-thread chunks gives
// the positions; with `gen` the scan is also left in cand[0..E] for batch
// generation (gen_chunk): cand[i] = exclusive prefix of slot i, cand[E] = total.
static __device__ void write_output(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                             int E, int out_off, bool gen) {
  const int per = (E + kThreads - 1) / kThreads;
  const int b = threadIdx.x * per, e = min(E, b + per);
  const unsigned long long Tg = (unsigned long long)kp.Tg;
  unsigned long long s = 0;
  for (int i = b; i < e; ++i) {
    const int lp = sm_lpof(kp)[i];
    const unsigned long long k = sm_cand(kp)[i];
    if (i - sm_p_eo(kp)[lp] < sm_p_cnt(kp)[lp] && k != kKeyMax) {
      const unsigned long long d = k >> 32;
      s += (1ull << 40) | (d < Tg ? d : Tg);
    }
  }
  unsigned long long tot;
  unsigned long long run = block_exclusive_scan<unsigned long long>(s, sh.wtmp64, tot);
  int32_t* o = kp.o + P.o_base;
  int32_t* perm = kp.perm + P.perm_base;
  const int last = P.mat_n - 1;
  for (int i = b; i < e; ++i) {
    const int lp = sm_lpof(kp)[i];
    const unsigned long long k = sm_cand(kp)[i];
    unsigned long long x = 0;
    if (i - sm_p_eo(kp)[lp] < sm_p_cnt(kp)[lp] && k != kKeyMax) {
      const unsigned long long d = k >> 32;
      x = (1ull << 40) | (d < Tg ? d : Tg);
      const int pos = out_off + (int)(run >> 40);
      const int v = (int)(uint32_t)k;
      o[pos] = v;
      perm[last - pos] = v;
      if (kp.iperm) kp.iperm[P.node_base + v] = last - pos;
    }
    if (gen) sm_cand(kp)[i] = run;
    run += x;
  }
  if (gen && threadIdx.x == 0) sm_cand(kp)[E] = tot;
  __syncthreads();
}

// ------------------------------------------------------ batch generation
// Greedy cut of the ordered output (after an incoming overhang) into batches of
// at most B_s nodes and at most T summed (clamped) valence; a node whose
// valence reaches T gets a single-node batch.  `nb` slots were
// reserved at q_off by signalCount (early generation); unused ones
// are published as empty batches and skipped by the `next` link of
// the last real batch.
struct GenState {
  int start;       // matrix-local position where the open batch starts
  int cnt;         // nodes in the open batch
  long long val;   // clamped valence sum of the open batch
  int emitted;     // batches written so far
  int pend_b, pend_e;  // last closed batch, not yet written (its `next` is unknown)
  int has_pend;
  int defer;       // 1: write descriptor fields only; the caller fences and writes the tags
};

__device__ __forceinline__ void publish_desc(Desc* d, int b, int e, int next, uint32_t epoch) {
  d->o_begin = b;
  d->o_end = e;
  d->next = next;
  st_release_u32(&d->tag, epoch);   // release: orders the fields above (and, cumulatively, what the block wrote before its last barrier)
}

__device__ __forceinline__ void write_desc(const GenState& g, Desc* d, int b, int e, int next, uint32_t epoch) {
  if (g.defer) { d->o_begin = b; d->o_end = e; d->next = next; }
  else publish_desc(d, b, e, next, epoch);
}

__device__ __forceinline__ void gen_close(const KParams& kp, GenState& g, int end, int q_off,
                                          int nb, uint32_t epoch) {
  if (g.has_pend) {
    if (g.emitted < nb)   // never exceeded; guarded anyway
      write_desc(g, kp.desc + q_off + g.emitted, g.pend_b, g.pend_e, q_off + g.emitted + 1, epoch);
    else
      latch_error(kp.ctl, ST_CAPACITY);
    ++g.emitted;
  }
  g.pend_b = g.start;
  g.pend_e = end;
  g.has_pend = 1;
  g.start = end;
  g.cnt = 0;
  g.val = 0;
}

// Consume one chunk of ordered nodes.  pre[i] (i <= m) = exclusive prefix over
// the chunk's slots of (count << 40 | clamped valence); slot i's node sits at
// matrix-local position base + (pre[i] >> 40).  Thread 0 only.
static __device__ void gen_chunk(const KParams& kp, GenState& g, const unsigned long long* pre, int m,
                          int base, int q_off, int nb, uint32_t epoch) {
  const unsigned long long kMaskV = (1ull << 40) - 1;
  int a = 0;   // first slot not yet assigned
  while (true) {
    unsigned long long pa = pre[a];
    unsigned long long pm = pre[m];
    int ca = (int)(pa >> 40), cm = (int)(pm >> 40);
    if (cm == ca) return;   // chunk exhausted
    // largest slot s in (a, m] with cnt + (c(s)-c(a)) <= BS and val + (v(s)-v(a)) <= T
    int lo = a, hi = m;
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      unsigned long long p = pre[mid];
      int c = (int)(p >> 40) - ca;
      long long v = (long long)((p & kMaskV) - (pa & kMaskV));
      if (g.cnt + c <= kp.Bg && g.val + v <= kp.Tg) lo = mid; else hi = mid - 1;
    }
    int taken = (int)(pre[lo] >> 40) - ca;
    if (taken == 0) {
      // the next node does not fit the open batch: close it (never empty here
      // because a single node always fits an empty batch: clamped valence <= T)
      gen_close(kp, g, base + ca, q_off, nb, epoch);
      continue;
    }
    g.cnt += taken;
    g.val += (long long)((pre[lo] & kMaskV) - (pa & kMaskV));
    a = lo;
    // advance a past holes (slots contributing nothing)
    if ((int)(pre[lo] >> 40) == cm) return;
    gen_close(kp, g, base + (int)(pre[lo] >> 40), q_off, nb, epoch);
  }
}

static __device__ void gen_finish(const KParams& kp, GenState& g, int end, int q_off, int nb,
                           uint32_t epoch) {
  if (g.cnt > 0) gen_close(kp, g, end, q_off, nb, epoch);
  if (g.has_pend) {
    if (g.emitted < nb) write_desc(g, kp.desc + q_off + g.emitted, g.pend_b, g.pend_e, q_off + nb, epoch);
    else latch_error(kp.ctl, ST_CAPACITY);
    ++g.emitted;
    g.has_pend = 0;
  }
}

// Publish empty batches q_off + [from, nb) (all threads of warp 0).
static __device__ void publish_empties(const KParams& kp, int q_off, int from, int nb, uint32_t epoch) {
  if (threadIdx.x < 32) {
    for (int i = from + threadIdx.x; i < nb; i += 32) publish_desc(kp.desc + q_off + i, 0, 0, q_off + i + 1, epoch);
  }
}

}  // namespace rcm
