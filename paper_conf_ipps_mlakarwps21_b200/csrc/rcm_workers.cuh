// rcm_workers.cuh -- the persistent workers: the multi-block signalling chain
// (Alg. 5) and the single-block "solo" worker for small
// components / matrices, plus the oversize single-node batch.
#pragma once
#include "rcm_batch.cuh"

namespace rcm {

// ------------------------------------------------------------- utilities
__device__ __forceinline__ void stat_add(const KParams& kp, unsigned long long* c, unsigned long long v) {
  if (kp.collect_stats && v) atomicAdd(c, v);
}

// Seed a component: o[pos] = s, perm[N-1-pos] = s, owner(s) = 0 (the root key,
// smaller than every parent key pos+1).  Thread 0 only.
static __device__ void place_root(const KParams& kp, const Problem& P, int s, int pos) {
  kp.o[P.o_base + pos] = s;
  kp.perm[P.perm_base + P.mat_n - 1 - pos] = s;
  if (kp.iperm) kp.iperm[P.node_base + s] = P.mat_n - 1 - pos;
  unsigned long long* wp = kp.word + P.node_base + s;
  unsigned long long w = ld_relaxed_u64(wp);
  atomicMin(wp, w & 0xffffffffull);
}

static __device__ void grid_barrier(const KParams& kp) {
  beacon(kp, 11, -1, ld_relaxed_s32(&kp.ctl->gbar_gen));
  __syncthreads();
  if (threadIdx.x == 0) {
    // the generation this barrier ends: a relaxed read cannot return an older
    // value than the one this thread observed at the previous barrier, and the
    // count cannot complete without this block
    const int gen = ld_relaxed_s32(&kp.ctl->gbar_gen);
    int arrived;   // acq_rel: releases this block's writes (after bar.sync), acquires the earlier arrivals
    asm volatile("atom.add.acq_rel.gpu.global.s32 %0, [%1], 1;" : "=r"(arrived) : "l"(&kp.ctl->gbar_count) : "memory");
    if (arrived == kp.nblocks - 1) {
      if (kp.trace) kp.ctl->dbg[7] = (long long)globaltimer();   // last arrival (leveled trace)
      st_relaxed_s32(&kp.ctl->gbar_count, 0);
      st_release_s32(&kp.ctl->gbar_gen, gen + 1);
    } else {
      // relaxed polling + one acquire fence (an ld.acquire per poll would drop the SM's L1 each time)
      uint64_t t0 = globaltimer();
      while (ld_relaxed_s32(&kp.ctl->gbar_gen) == gen) {
        __nanosleep(32);
        if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 4, gen, 0, 0); break; }
      }
      fence_acquire_gpu();
    }
  }
  __syncthreads();
}

// ---------------------------------------------------- block radix sort (global)
// Stable LSD radix sort (8-bit digits) of a[0..n) in global memory by one
// block, temp buffer tmp[0..n); digits that are equal in all keys are skipped.
// `scratch` is >= (1 + kWarps) * 256 ints of shared memory.
static __device__ void block_radix_sort_global(unsigned long long* a, unsigned long long* tmp, int n,
                                        int32_t* scratch, ShState& sh, int lo_shift = 0) {
  if (n <= 1) return;
  unsigned long long first = __ldcg(a);
  unsigned long long diff = 0;
  for (int i = threadIdx.x; i < n; i += kThreads) diff |= __ldcg(a + i) ^ first;
  // OR-reduce
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) diff |= __shfl_xor_sync(0xffffffffu, diff, d);
  if ((threadIdx.x & 31) == 0) sh.wtmp64[threadIdx.x >> 5] = diff;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long x = 0;
    for (int w = 0; w < kWarps; ++w) x |= sh.wtmp64[w];
    sh.wtmp64[kWarps] = x;
  }
  __syncthreads();
  diff = sh.wtmp64[kWarps];
  __syncthreads();
  int32_t* off = scratch;             // 256 running digit offsets
  int32_t* wcnt = scratch + 256;      // kWarps x 256 per-warp digit counts
  unsigned long long* src = a;
  unsigned long long* dst = tmp;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const unsigned lt = (1u << lane) - 1;
  for (int shift = lo_shift; shift < 64; shift += 8) {   // digits below lo_shift already in order
    if (((diff >> shift) & 0xffull) == 0) continue;
    for (int i = threadIdx.x; i < 256; i += kThreads) off[i] = 0;
    __syncthreads();
    for (int i = threadIdx.x; i < n; i += kThreads) atomicAdd(&off[(__ldcg(src + i) >> shift) & 0xff], 1);
    __syncthreads();
    if (threadIdx.x < 32) {   // exclusive scan of 256 counters by warp 0
      int v[8], s = 0;
#pragma unroll
      for (int j = 0; j < 8; ++j) { v[j] = off[threadIdx.x * 8 + j]; s += v[j]; }
      int x = s;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) { int y = __shfl_up_sync(0xffffffffu, x, d); if (threadIdx.x >= d) x += y; }
      int run = x - s;
#pragma unroll
      for (int j = 0; j < 8; ++j) { off[threadIdx.x * 8 + j] = run; run += v[j]; }
    }
    __syncthreads();
    for (int base = 0; base < n; base += kThreads) {
      int i = base + threadIdx.x;
      bool valid = i < n;
      unsigned long long k = valid ? __ldcg(src + i) : 0ull;
      int d = valid ? (int)((k >> shift) & 0xff) : 256;
      unsigned peers = __match_any_sync(0xffffffffu, d);
      int rank = __popc(peers & lt);
      for (int j = threadIdx.x; j < kWarps * 256; j += kThreads) wcnt[j] = 0;
      __syncthreads();
      if (valid && rank == 0) wcnt[wid * 256 + d] = __popc(peers);
      __syncthreads();
      // per digit: exclusive prefix over warps, then advance the running offset
      for (int dg = threadIdx.x; dg < 256; dg += kThreads) {
        int run = off[dg];
        for (int w = 0; w < kWarps; ++w) { int c = wcnt[w * 256 + dg]; wcnt[w * 256 + dg] = run; run += c; }
        off[dg] = run;
      }
      __syncthreads();
      if (valid) dst[wcnt[wid * 256 + d] + rank] = k;
      __syncthreads();
    }
    unsigned long long* t = src; src = dst; dst = t;
  }
  if (src != a) {
    __threadfence_block();
    for (int i = threadIdx.x; i < n; i += kThreads) a[i] = __ldcg(src + i);
  }
  __threadfence();
  __syncthreads();
}

// ------------------------------------------------------- oversize batches
// A single parent whose row exceeds the scratchpad.  Discovery
// claims are kept in a shared-memory bitmap over the row; after rediscovery the
// kept children are gathered into plan-owned HBM scratch, sorted by
// (valence, id) there, written out, and cut into batches chunk by chunk.
static __device__ bool oversize_discover(const KParams& kp, const Problem& P, const SmemPtrs& sm,
                                  ShState& sh, uint32_t key, int rs, int D) {
  const int nw = (D + 31) >> 5;
  if (threadIdx.x == 0) {
    sh.ovbits = reinterpret_cast<uint32_t*>(sm_cand(kp));
    if (nw > 2 * (kp.T + 1)) {   // row longer than the shared-memory bitmap: HBM scratch
      const long long base = atomicAdd(&kp.ctl->spill_cursor, (nw + 1) >> 1);
      if (base + ((nw + 1) >> 1) > kp.spill_cap) { latch_error(kp.ctl, ST_CAPACITY); sh.ovbits = nullptr; }
      else sh.ovbits = reinterpret_cast<uint32_t*>(kp.spill + base);
    }
  }
  __syncthreads();
  uint32_t* bits = sh.ovbits;
  if (!bits) return false;
  for (int i = threadIdx.x; i < nw; i += kThreads) bits[i] = 0;
  __threadfence_block();
  __syncthreads();
  unsigned long long* word = kp.word + P.node_base;
  const int32_t* col = kp.col_idx + P.ci_base + rs;
  int claims = 0;
  for (int e = threadIdx.x; e < D; e += kThreads) {
    int c = __ldg(col + e);
    unsigned long long w = ld_relaxed_u64(word + c);
    if ((uint32_t)(w >> 32) > key) {
      unsigned long long old = atomicMin(word + c, ((unsigned long long)key << 32) | (w & 0xffffffffull));
      if ((uint32_t)(old >> 32) > key) { atomicOr(&bits[e >> 5], 1u << (e & 31)); ++claims; }
    }
  }
  if (kp.collect_stats) {
    int tot = block_reduce_sum<int32_t>(claims, sh.wtmp32);
    if (threadIdx.x == 0) stat_add(kp, &kp.stats->cand_spec, tot);
  }
  __threadfence_block();
  __syncthreads();
  return true;
}

// bitmap word i (shared memory, or HBM written by atomics: read through L2)
__device__ __forceinline__ uint32_t ov_word(const KParams& kp, const uint32_t* bits, int i) {
  return __isShared(bits) ? bits[i] : __ldcg(bits + i);
}

// Rediscover (keep iff owner == key), then count and clamped valence sum.
static __device__ void oversize_rediscover_count(const KParams& kp, const Problem& P, const SmemPtrs& sm,
                                          ShState& sh, uint32_t key, int rs, int D) {
  uint32_t* bits = sh.ovbits;
  const int nw = (D + 31) >> 5;
  const unsigned long long* word = kp.word + P.node_base;
  const int32_t* col = kp.col_idx + P.ci_base + rs;
  int cnt = 0, removed = 0;
  long long val = 0;
  for (int i = threadIdx.x; i < nw; i += kThreads) {
    uint32_t b = ov_word(kp, bits, i), keep = b;
    while (b) {
      int j = __ffs(b) - 1;
      b &= b - 1;
      int c = __ldg(col + i * 32 + j);
      unsigned long long w = ld_relaxed_u64(word + c);
      if ((uint32_t)(w >> 32) != key) { keep &= ~(1u << j); ++removed; }
      else { ++cnt; long long d = (long long)(w & 0xffffffffull); val += d < kp.Tg ? d : kp.Tg; }
    }
    bits[i] = keep;
  }
  __threadfence_block();
  int C = block_reduce_sum<int32_t>(cnt, sh.wtmp32);
  long long V = block_reduce_sum<long long>(val, sh.wtmpll);
  int R = block_reduce_sum<int32_t>(removed, sh.wtmp32);
  if (threadIdx.x == 0) {
    sh.count = C;
    sh.V = V;
    stat_add(kp, &kp.stats->cand_removed, R);
  }
  __syncthreads();
}

// Gather kept children into spill, sort them.  Returns false on capacity error.
static __device__ bool oversize_gather_sort(const KParams& kp, const Problem& P, const SmemPtrs& sm,
                                     ShState& sh, int rs, int D) {
  const uint32_t* bits = sh.ovbits;
  const int nw = (D + 31) >> 5;
  const int C = sh.count;
  if (threadIdx.x == 0) {
    long long base = atomicAdd(&kp.ctl->spill_cursor, C);
    if (base + C > kp.spill_cap) { latch_error(kp.ctl, ST_CAPACITY); base = -1; }
    sh.spill_base = base;
  }
  __syncthreads();
  if (sh.spill_base < 0) return false;
  unsigned long long* out = kp.spill + sh.spill_base;
  const unsigned long long* word = kp.word + P.node_base;
  const int32_t* col = kp.col_idx + P.ci_base + rs;
  // contiguous word ranges per thread keep id order within the row (stable)
  const int per = (nw + kThreads - 1) / kThreads;
  const int b = threadIdx.x * per, e = min(nw, b + per);
  int mine = 0;
  for (int i = b; i < e; ++i) mine += __popc(ov_word(kp, bits, i));
  int tot;
  int run = block_exclusive_scan<int32_t>(mine, sh.wtmp32, tot);
  for (int i = b; i < e; ++i) {
    uint32_t x = ov_word(kp, bits, i);
    while (x) {
      int j = __ffs(x) - 1;
      x &= x - 1;
      int c = __ldg(col + i * 32 + j);
      unsigned long long w = ld_relaxed_u64(word + c);
      out[run++] = ((w & 0xffffffffull) << 32) | (uint32_t)c;
    }
  }
  __threadfence_block();
  __syncthreads();
  // sort by (valence, id); the bitmap area is free now.  The gather is stable in
  // row order, so when the row's kept ids ascend (sorted columns, the usual
  // case) a stable sort on the valence half alone gives (valence, id) order --
  // the paper's direct copy of a single-valence bin in id order
  int unsorted = 0;
  for (int i = threadIdx.x; i + 1 < C; i += kThreads)
    unsorted |= (uint32_t)__ldcg(out + i) >= (uint32_t)__ldcg(out + i + 1);
  unsorted = __syncthreads_or(unsorted);
  block_radix_sort_global(out, kp.spill + kp.spill_cap + sh.spill_base, C,
                          reinterpret_cast<int32_t*>(sm_cand(kp)), sh, unsorted ? 0 : 32);
  return true;
}

// Write the sorted children at out_off and cut them into batches.
// Thread-0 generation state g must be initialised by the caller (overhang).
static __device__ void oversize_output(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                                int out_off, bool generate, GenState& g, int q_off, int nb,
                                uint32_t epoch) {
  const int C = sh.count;
  const unsigned long long* src = kp.spill + sh.spill_base;
  int32_t* o = kp.o + P.o_base;
  int32_t* perm = kp.perm + P.perm_base;
  const int last = P.mat_n - 1;
  for (int i = threadIdx.x; i < C; i += kThreads) {
    int v = (int)(uint32_t)__ldcg(src + i);
    o[out_off + i] = v;
    perm[last - out_off - i] = v;
    if (kp.iperm) kp.iperm[P.node_base + v] = last - out_off - i;
  }
  __threadfence();
  __syncthreads();
  if (!generate) return;
  // chunked prefix over (1, clamped valence) in output order
  for (int c0 = 0; c0 < C; c0 += kp.T) {
    const int m = min(kp.T, C - c0);
    const int per = (m + kThreads - 1) / kThreads;
    const int b = threadIdx.x * per, e = min(m, b + per);
    unsigned long long s = 0;
    for (int i = b; i < e; ++i) {
      unsigned long long d = __ldcg(src + c0 + i) >> 32;
      s += (1ull << 40) | (d < (unsigned long long)kp.Tg ? d : (unsigned long long)kp.Tg);
    }
    unsigned long long tot;
    unsigned long long run = block_exclusive_scan<unsigned long long>(s, sh.wtmp64, tot);
    for (int i = b; i < e; ++i) {
      unsigned long long d = __ldcg(src + c0 + i) >> 32;
      sm_cand(kp)[i] = run;
      run += (1ull << 40) | (d < (unsigned long long)kp.Tg ? d : (unsigned long long)kp.Tg);
    }
    if (threadIdx.x == 0) sm_cand(kp)[m] = tot;
    __syncthreads();
    if (threadIdx.x == 0) gen_chunk(kp, g, sm_cand(kp), m, out_off + c0, q_off, nb, epoch);
    __syncthreads();
  }
}

// ------------------------------------------------------------ chain worker
// signalCount (Alg. 5 ln 31-40): with the exact output count known
// and the predecessor's output position received (signal word `w`), forward the
// position, the queue offset and possibly an overhang to the successor.
// Thread 0 only.
static __device__ void signal_count(const KParams& kp, ShState& sh, const Sig* mine, unsigned long long w,
                             Sig* succ_sig, int succ) {
  const int out_off = sig_out(w);
  const int q_off = sig_q(w);
  int ovh_n = 0, ovh_t = 0;
  if (sig_has_ovh(w)) {
    const unsigned long long ov = ld_relaxed_u64(&mine->ovh);   // ordered after the acquire of w
    ovh_n = (int)(ov >> 32);
    ovh_t = (int)(uint32_t)ov;
  }
  const int Np = ovh_n + sh.count;
  const long long Vp = (long long)ovh_t + sh.V;
  // combine with next: below half a batch in nodes and temp
  // elements, and a successor slot already exists (else nobody would receive it)
  const bool fwd = !(kp.flags & F_NO_OVERHANG) && Np > 0 && 2 * Np < kp.Bg &&
                   2 * Vp < (long long)kp.Tg && succ < q_off;
  int nb = 0;
  if (fwd) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(&succ_sig->ovh),
                 "l"(((unsigned long long)(uint32_t)Np << 32) | (uint32_t)Vp) : "memory");
    send_sig(succ_sig, sig_pack(out_off + sh.count, q_off, 1, S_COUNTED));
    stat_add(kp, &kp.stats->ovh_forwards, 1);
  } else {
    if (Np > 0) {
      // safe over-estimate of the greedy batch count:
      // floor(N/B_s) + max(1, ceil(2V/T))  (P:L800-809 uses 2x the ideal count)
      const long long v2 = (2 * Vp + kp.Tg - 1) / kp.Tg;
      nb = Np / kp.Bg + (int)(v2 > 1 ? v2 : 1);
    }
    if ((long long)q_off + nb > kp.qcap) {
      latch_error(kp.ctl, ST_CAPACITY);
      nb = 0;
    }
    send_sig(succ_sig, sig_pack(out_off + sh.count, q_off + nb, 0, S_COMPLETED));  // Alg. 5 ln 39
    if (nb) atomicMax(&kp.ctl->qtail, q_off + nb);
    stat_add(kp, &kp.stats->generated, nb);
  }
  sh.sigw = w;
  sh.out_off = out_off;
  sh.q_off = q_off;
  sh.ovh_n = ovh_n;
  sh.ovh_t = ovh_t;
  sh.fwd = fwd;
  sh.nb = nb;
  sh.chain_end = (!fwd && nb == 0 && succ == q_off);
  sh.counted = 1;
}

// Dequeue the next non-empty batch in queue order.
// Look-back chain end without termination (a disconnected graph): every
// reserved slot has finished, so nothing will ever be published again.  A slot
// counts itself (and the empties it generated) in `completed` only after its
// reservation raised `qtail` (release), and every reserved slot is counted
// exactly once, so completed == qtail read in this order (acquire) implies no
// slot is still running.  Polled by blocks idling in dequeue.
static __device__ __noinline__ bool lb_chain_exhausted(const KParams& kp) {
  // relaxed polls first: an ld.acquire.gpu invalidates the whole SM's L1 (the
  // other resident block's cached rows included), so idle blocks only pay for
  // the acquire when the counters look equal
  if (ld_relaxed_s32(&kp.ctl->completed) != ld_relaxed_s32(&kp.ctl->qtail)) return false;
  const int c = ld_acquire_s32(&kp.ctl->completed);
  if (c != ld_acquire_s32(&kp.ctl->qtail)) return false;
  kp.ctl->incomplete = 1;   // idempotent: several idle blocks may get here
  __threadfence();
  atomicExch(&kp.ctl->done, 1);
  return true;
}

// Thread 0; returns false when the chain is done.
static __device__ bool dequeue(const KParams& kp, ShState& sh, uint32_t epoch) {
  for (;;) {
    if (ld_relaxed_s32(&kp.ctl->done)) return false;
    const int t = atomicAdd(&kp.ctl->head, 1);
    trace_ev(kp, t, 9);   // slot claimed (before its descriptor is seen)
    beacon(kp, 1, t, 0);
    if (t >= kp.qcap) {   // only possible after a capacity error; wait for done
      while (!ld_relaxed_s32(&kp.ctl->done)) __nanosleep(1000);
      return false;
    }
    const Desc* d = kp.desc + t;
    uint64_t t0 = 0;
    unsigned ns = 0;
    for (int it = 0; ld_relaxed_u32(&d->tag) != epoch; ++it) {   // relaxed poll, acquire below
      if (ld_relaxed_s32(&kp.ctl->done)) return false;
      if (it >= 32) {
        __nanosleep(ns);
        if (ns < RCM_DQ_SLEEP_MAX) ns = ns ? ns * 2 : 32;
      }
      if ((it & 15) == 15 && !(kp.flags & F_SERIAL_CHAIN) && lb_chain_exhausted(kp)) return false;
      if ((it & 255) == 255) {
        if (t0 == 0) t0 = globaltimer();
        else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 1, t, ld_relaxed_s32(&kp.ctl->head), 0); return false; }
      }
    }
    (void)ld_acquire_u32(&d->tag);   // acquire the publication (one L1 invalidation per dequeue)
    const int b = ld_relaxed_s32(&d->o_begin), e = ld_relaxed_s32(&d->o_end), nx = ld_relaxed_s32(&d->next);
    stat_add(kp, &kp.stats->dequeued, 1);
    if (b == e) { stat_add(kp, &kp.stats->empty, 1); continue; }
    trace_ev(kp, t, 0);
    sh.t = t;
    sh.o_begin = b;
    sh.o_end = e;
    sh.next = nx;
    return true;
  }
}

// Process one dequeued batch of the chain: Alg. 5 BatchRCM.
__device__ __forceinline__ void chain_batch(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                            uint32_t epoch) {
  const int t = sh.t, o_begin = sh.o_begin, succ = sh.next;
  Sig* mine = kp.sig + t;
  Sig* succ_sig = kp.sig + succ;
  int nP = load_parents(kp, P, sm, sh, o_begin, sh.o_end - o_begin, false);
  const int E = sh.E;
  if (threadIdx.x == 0) {
    sh.steal = 0;
    sh.counted = 0;
    sh.aborted = 0;
    sh.s_early = (kp.flags & F_NO_EARLY) ? S_NONE : sig_state(load_sig(mine));   // ln 2
  }
  __syncthreads();
  const bool oversize = E > kp.T;   // only single-node batches (batch generation)
  const uint32_t key0 = (uint32_t)o_begin + 1;
  if (oversize) {
    if (!oversize_discover(kp, P, sm, sh, key0, sm_p_rs(kp)[0], E)) return;
  } else {
    discover(kp, P, sm, sh, o_begin, nP, E);                                    // ln 3
  }
  if (threadIdx.x == 0) { sh.sigw = load_sig(mine); sh.s_mid = sig_state(sh.sigw); }  // ln 4
  __syncthreads();
  const int s_early = sh.s_early, s_mid = sh.s_mid;
  bool rediscovered = false;
  if (!oversize && (s_early >= S_DISCOVERED || s_mid >= S_DISCOVERED)) {
    // ln 5-12: every predecessor has discovered; forward Discovered right after
    // our own discovery, rediscover before sorting (dense array after sorting).
    if (threadIdx.x == 0) {
      __threadfence();   // the block's atomicMin marks before the signal
      send_sig(succ_sig, S_DISCOVERED);
    }
    rediscover_count(kp, P, sm, sh, o_begin, E, s_early < S_DISCOVERED || sh.steal);
    if (threadIdx.x == 0 && s_early < S_DISCOVERED) stat_add(kp, &kp.stats->redisc_early, 1);
    rediscovered = true;
    if (threadIdx.x == 0) {
      const unsigned long long w = load_sig(mine);
      if (sig_state(w) >= S_COUNTED) signal_count(kp, sh, mine, w, succ_sig, succ);
    }
    __syncthreads();
  }
  if (!oversize) {
    if (!(kp.flags & F_NO_SORT)) sort_segments(kp, sm, sh, nP);                // ln 13
  }
  if (!rediscovered) {
    // ln 14-19: late discovery -- wait for Discovered, forward it, rediscover
    if (threadIdx.x == 0) {
      if (sig_state(wait_sig(mine, S_DISCOVERED, kp.ctl)) < S_DISCOVERED) sh.aborted = 1;
      else { __threadfence(); send_sig(succ_sig, S_DISCOVERED); }
    }
    __syncthreads();
    if (sh.aborted) return;
    if (oversize) {
      oversize_rediscover_count(kp, P, sm, sh, key0, sm_p_rs(kp)[0], E);
    } else {
      rediscover_count(kp, P, sm, sh, o_begin, E, true);   // removed: flagged, no re-sort
    }
    if (threadIdx.x == 0) {
      stat_add(kp, &kp.stats->redisc_late, 1);
      const unsigned long long w = load_sig(mine);
      if (sig_state(w) >= S_COUNTED) signal_count(kp, sh, mine, w, succ_sig, succ);
    }
    __syncthreads();
  }
  if (!sh.counted) {                                                            // ln 20-22
    if (threadIdx.x == 0) {
      const unsigned long long w = wait_sig(mine, S_COUNTED, kp.ctl);
      if (sig_state(w) < S_COUNTED) sh.aborted = 1;
      else signal_count(kp, sh, mine, w, succ_sig, succ);
    }
    __syncthreads();
    if (sh.aborted) return;
  }
  // ln 23-26: output (dense: segments are sorted, removed children at the end)
  const int out_off = sh.out_off;
  GenState g;
  if (threadIdx.x == 0) {
    g.start = out_off - sh.ovh_n;
    g.cnt = sh.ovh_n;
    g.val = sh.ovh_t;
    g.emitted = 0;
    g.has_pend = 0;
    g.defer = 0;
  }
  const bool gen = !sh.fwd && sh.nb > 0;
  // wait(Completed) before publishing batches that reference an overhang, or
  // before forwarding Completed for an overhang we passed on (ln 27-29)
  const bool need_completed = sh.fwd || sh.ovh_n > 0;
  if (oversize) {
    if (!oversize_gather_sort(kp, P, sm, sh, sm_p_rs(kp)[0], E)) return;
    if (threadIdx.x == 0 && need_completed && sig_state(sh.sigw) < S_COMPLETED) {
      if (sig_state(wait_sig(mine, S_COMPLETED, kp.ctl)) < S_COMPLETED) sh.aborted = 1;
    }
    __syncthreads();
    if (sh.aborted) return;
    oversize_output(kp, P, sm, sh, out_off, gen, g, sh.q_off, sh.nb, epoch);
    if (threadIdx.x == 0) stat_add(kp, &kp.stats->oversize, 1);
  } else {
    write_output(kp, P, sm, sh, E, out_off, gen);
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0 && need_completed && sig_state(sh.sigw) < S_COMPLETED) {
      if (sig_state(wait_sig(mine, S_COMPLETED, kp.ctl)) < S_COMPLETED) sh.aborted = 1;
    }
    __syncthreads();
    if (sh.aborted) return;
    if (gen && threadIdx.x == 0) gen_chunk(kp, g, sm_cand(kp), E, out_off, sh.q_off, sh.nb, epoch);
  }
  if (threadIdx.x == 0) {
    if (sh.fwd) send_sig(succ_sig, sig_pack(out_off + sh.count, sh.q_off, 1, S_COMPLETED));
    if (gen) {
      gen_finish(kp, g, out_off + sh.count, sh.q_off, sh.nb, epoch);           // ln 30
      if (g.emitted > sh.nb) latch_error(kp.ctl, ST_CAPACITY);
    }
    sh.k = gen ? g.emitted : 0;
    stat_add(kp, &kp.stats->executed, 1);
  }
  __syncthreads();
  if (gen) publish_empties(kp, sh.q_off, sh.k, sh.nb, epoch);
  if (threadIdx.x == 0) {
    const int total = out_off + sh.count;
    if (total == P.pos0 + P.size) {               // early termination
      kp.ctl->chain_total = total;
      __threadfence();
      atomicExch(&kp.ctl->done, 1);
    } else if (sh.chain_end) {                    // queue ran dry: component exhausted
      kp.ctl->chain_total = total;
      kp.ctl->incomplete = 1;
      __threadfence();
      atomicExch(&kp.ctl->done, 1);
    }
  }
  __syncthreads();
}

// Chain set-up (a2): slot 0 = the seed batch [pos0, pos0+1) whose virtual
// predecessor is Completed with out_off = pos0+1 and queue tail 1.  Thread 0 of
// block 0, before a grid barrier.
static __device__ void chain_init(const KParams& kp, const Problem& P) {
  const uint32_t ep = atomicAdd(&kp.ctl->epoch, 1u) + 1u;
  kp.ctl->head = 0;
  kp.ctl->done = 0;
  kp.ctl->qtail = 1;
  kp.ctl->completed = 0;
  place_root(kp, P, P.seed, P.pos0);
  kp.sig[0].ovh = 0;
  // serial chain: the virtual predecessor of slot 0 has Completed with
  // out_off = pos0+1 and queue tail 1; look-back chain: slot 0 starts empty
  kp.sig[0].word = (kp.flags & F_SERIAL_CHAIN) ? sig_pack(P.pos0 + 1, 1, 0, S_COMPLETED) : 0ull;
  Desc* d0 = kp.desc;
  d0->o_begin = P.pos0;
  d0->o_end = P.pos0 + 1;
  d0->next = 1;
  d0->tag = ep;
  stat_add(kp, &kp.stats->components, 1);
  __threadfence();
}

// After a chain run (all blocks, between grid barriers): zero the signal slots
// it used so the next run starts from S_NONE without an epoch in the word.
static __device__ void chain_reset_signals(const KParams& kp) {
  const int qt = min(ld_cg_s32(&kp.ctl->qtail) + 2, kp.qcap + 1);
  for (int i = blockIdx.x * kThreads + threadIdx.x; i < qt; i += kp.nblocks * kThreads) {
    kp.sig[i].word = 0;
    kp.sig[i].ovh = 0;
  }
}

// ------------------------------------------------------------- solo worker
// Block-level BFS inside one component for the pseudo-peripheral finder
// (P:L365-375): the queue lives in the component's still-unwritten output
// range q[], levels in lev[] (-1 = unvisited; reset before returning).
// Returns the number of levels; sh.minkey = min (valence, id) of the last level.
static __device__ int block_bfs(const KParams& kp, const Problem& P, int32_t* q, int32_t* lev, int r, ShState& sh) {
  int32_t* lv = lev + P.node_base;
  const int32_t* rp = kp.row_ptr + P.rp_base;
  const int32_t* col = kp.col_idx + P.ci_base;
  if (threadIdx.x == 0) { q[0] = r; lv[r] = 0; sh.written = 1; }
  __syncthreads();
  int head = 0, tail = 1, level = 0, lb = 0;
  for (;;) {
    for (int i = head + threadIdx.x; i < tail; i += kThreads) {
      const int p = q[i];
      for (int e = __ldg(rp + p); e < __ldg(rp + p + 1); ++e) {
        const int c = __ldg(col + e);
        if (ld_cg_s32(lv + c) < 0 && atomicCAS(lv + c, -1, level + 1) == -1) q[atomicAdd(&sh.written, 1)] = c;
      }
    }
    __syncthreads();
    const int nt = sh.written;
    __syncthreads();
    if (nt == tail) break;
    lb = tail;
    head = tail;
    tail = nt;
    ++level;
  }
  unsigned long long best = kKeyMax;
  const unsigned long long* word = kp.word + P.node_base;
  for (int i = lb + threadIdx.x; i < tail; i += kThreads) {
    const int v = q[i];
    const unsigned long long k = ((ld_relaxed_u64(word + v) & 0xffffffffull) << 32) | (uint32_t)v;
    best = k < best ? k : best;
  }
  best = warp_min_u64(best);
  if ((threadIdx.x & 31) == 0) sh.wtmp64[threadIdx.x >> 5] = best;
  __syncthreads();
  if (threadIdx.x < 32) {
    unsigned long long b = threadIdx.x < kWarps ? sh.wtmp64[threadIdx.x] : kKeyMax;
    b = warp_min_u64(b);
    if (threadIdx.x == 0) sh.minkey = b;
  }
  for (int i = threadIdx.x; i < tail; i += kThreads) lv[q[i]] = -1;
  __syncthreads();
  return level + 1;
}

// GL finder (C-5) from r inside its component, block-level.
static __device__ int block_gl(const KParams& kp, const Problem& P, int32_t* q, int32_t* lev, int r, ShState& sh) {
  int nl = block_bfs(kp, P, q, lev, r, sh);
  int x = (int)(uint32_t)sh.minkey;
  __syncthreads();
  for (;;) {
    const int nx = block_bfs(kp, P, q, lev, x, sh);
    if (nx <= nl) return x;   // same level count: "use the last node"
    nl = nx;
    x = (int)(uint32_t)sh.minkey;
    __syncthreads();
  }
}

// One block orders a whole (small) component of a large graph with the same
// batch steps but without the signalling chain: batches are consecutive output
// ranges.  (Batched matrices and small graphs use rcm_solo.cuh instead.)
__device__ __forceinline__ void run_solo(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh, int32_t* lev) {
  int seed = P.seed;
  if (P.flags & 2) seed = block_gl(kp, P, kp.o + P.o_base + P.pos0, lev, seed, sh);
  if (threadIdx.x == 0) {
    place_root(kp, P, seed, P.pos0);
    stat_add(kp, &kp.stats->solo_problems, 1);
    stat_add(kp, &kp.stats->components, 1);
  }
  int pos = P.pos0, written = P.pos0 + 1;
  const int end = P.pos0 + P.size;
  __syncthreads();
  for (;;) {
    if (pos == written) {
      if (written >= end) break;
      // a component problem whose declared size exceeds what its BFS reaches:
      // the pattern is not symmetric (C-9)
      if (threadIdx.x == 0) latch_error(kp.ctl, ST_NOT_SYM);
      break;
    }
    int nP = load_parents(kp, P, sm, sh, pos, min(kp.BS, written - pos), true);
    const int E = sh.E;
    if (E > kp.T) {
      const uint32_t key = (uint32_t)pos + 1;
      if (!oversize_discover(kp, P, sm, sh, key, sm_p_rs(kp)[0], E)) break;
      oversize_rediscover_count(kp, P, sm, sh, key, sm_p_rs(kp)[0], E);
      if (!oversize_gather_sort(kp, P, sm, sh, sm_p_rs(kp)[0], E)) break;
      GenState g;
      oversize_output(kp, P, sm, sh, written, false, g, 0, 0, 0);
      if (threadIdx.x == 0) stat_add(kp, &kp.stats->oversize, 1);
      written += sh.count;
    } else {
      if (threadIdx.x == 0) sh.steal = 0;
      discover(kp, P, sm, sh, pos, nP, E);
      rediscover_count(kp, P, sm, sh, pos, E, sh.steal != 0);
      const int c = sh.count;
      if (!(kp.flags & F_NO_SORT)) sort_segments(kp, sm, sh, nP);
      write_output(kp, P, sm, sh, E, written, false);
      written += c;
    }
    if (threadIdx.x == 0) stat_add(kp, &kp.stats->executed, 1);
    pos += nP;
    __syncthreads();
  }
  __syncthreads();
}

}  // namespace rcm
