// rcm_lookback.cuh -- the default B200 chain: Alg. 5's signalling chain with
// the two signals (Discovered, Counted) turned into per-slot status words that a
// batch publishes about ITSELF as early as possible, and that a successor reads
// with a decoupled look-back over a 32-slot window per round trip (one warp),
// instead of one predecessor -> successor hand-off per batch.
//
//   Discovered: slot j has LOCAL once its own discovery is done and
//     DINCL once it knows every slot <= j is discovered.  Batch t may rediscover
//     when every slot < t is LOCAL up to the nearest DINCL slot.
//   Counted: slot j has AGG(count_j, nb_j) once its exact
//     output count is known (after rediscovery, before sorting -- the paper's
//     early Counted), and INCL(out_end_j, q_end_j) once its prefix is known.
//     Batch t's output position / queue offset = nearest INCL + sum of AGGs.
//
// Result-neutral: the keys, rediscovery rule and per-parent sort are those of
// the serial chain (C-4, C-11).  Work aggregation by overhang
// forwarding is a sequential decision and is not used here; the
// generator batches its own outputs only.
#pragma once
#include "rcm_workers.cuh"

namespace rcm {

// Sig::word: Discovered flags, release stores (they order the block's
// atomicMin marks, cumulatively, before the flag).
constexpr unsigned long long LB_LOCAL = 1, LB_DINCL = 2;
// set by a slot that forwarded its output once that output is written (the
// receiver publishes batches over it only after seeing this flag)
constexpr unsigned long long LB_OUTDONE = 4;
// Sig::ovh holds the Counted facts, plain values (relaxed stores, no fence):
//   AGG  = 2 | count << 2 (31 bit) | nb << 33 (30 bit)
//   INCL = 1 | out_end << 2 (31 bit) | q_end << 33 (30 bit), replaces AGG
// A successor reads one word per slot; nothing it reads depends on other data.
constexpr unsigned long long LB_INCL = 1, LB_AGG = 2;
// INCL bit 63: this slot forwarded its output to the next slot (work
// aggregation); its count and valence sum are in KParams::fwdv
constexpr unsigned long long LB_FWD = 1ull << 63;
__device__ __forceinline__ unsigned long long lb_pfx(unsigned long long kind, long long a, long long b) {
  return kind | ((unsigned long long)(uint32_t)a << 2) | ((unsigned long long)(uint32_t)b << 33);
}
__device__ __forceinline__ void st_relaxed_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void lb_spin(unsigned& ns, int it) {
  if (it >= 16) {
    __nanosleep(ns);
    if (ns < RCM_LB_SLEEP_MAX) ns = ns ? ns * 2 : 32;
  }
}

// Warp 0: wait until every slot < t is discovered.  Returns false on error.
// try_only: give up (return false, *ready = 0) instead of spinning.
static __device__ bool lb_wait_discovered(const KParams& kp, int t, bool try_only, int* ready) {
  const int lane = threadIdx.x & 31;
  int j = t - 1;
  unsigned ns = 0;
  uint64_t t0 = 0;
  for (int it = 0; j >= 0; ++it) {
    const int idx = j - lane;
    const unsigned long long a = idx >= 0 ? ld_relaxed_u64(&kp.sig[idx].word) : (LB_LOCAL | LB_DINCL);
    const unsigned incl = __ballot_sync(0xffffffffu, (a & LB_DINCL) != 0);
    const unsigned loc = __ballot_sync(0xffffffffu, (a & LB_LOCAL) != 0);
    const int stop = incl ? __ffs(incl) - 1 : 32;
    const unsigned need = stop == 32 ? 0xffffffffu : ((1u << stop) - 1);
    if ((loc & need) == need) {
      if (stop < 32) break;
      j -= 32;
      continue;
    }
    j -= __ffs(~loc & need) - 1;   // verified-LOCAL slots stay LOCAL (monotone)
    if (lane == 0 && (it & 63) == 63) { volatile int32_t* d = kp.dbg + blockIdx.x * 8; d[4] = j; d[5] = (int)a; d[6] = it; }
    // A batch still waiting for Discovered has no aggregate yet, so it is a
    // successor of the batch that completed the order (which saw every
    // predecessor's aggregate): after early termination it has nothing to
    // output and may be abandoned -- and must be, since a slot it waits on may
    // have been abandoned at dequeue.
    // every exit decision is taken warp-uniformly (lane 0's view, broadcast):
    // lanes that left the loop on their own would strand the others in the
    // full-mask ballots above
    int quit = lane == 0 && (ld_relaxed_s32(&kp.ctl->status) || ld_relaxed_s32(&kp.ctl->done));
    if ((it & 1023) == 1023 && lane == 0) {
      if (t0 == 0) t0 = globaltimer();
      else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 2, t, j, (long long)a); quit = 1; }
    }
    if (__shfl_sync(0xffffffffu, quit, 0)) return false;
    // try mode gives up only after the termination check above: a batch that
    // must be abandoned is, even when it is only polled
    if (try_only && it >= 2) { *ready = 0; return true; }
    lb_spin(ns, it);
  }
  // the flags were polled relaxed: one acquire fence orders this block's
  // rediscovery loads (after the caller's barrier) behind the predecessors'
  // LOCAL/DINCL releases, i.e. behind their atomicMin marks
  fence_acquire_gpu();
  *ready = 1;
  return true;
}

// Warp 0: output position and queue offset of slot t (exclusive prefix).
// try_only: give up (return true, *ready = 0) after a short poll instead of spinning.
static __device__ bool lb_prefix(const KParams& kp, const Problem& P, int t, int count, int& out_off, int& q_off,
                          bool try_only, int* ready) {
  const int lane = threadIdx.x & 31;
  long long sc = 0, sn = 0;
  int j = t - 1;
  long long base_out = P.pos0 + 1, base_q = 1;   // the virtual predecessor of slot 0
  unsigned ns = 0;
  uint64_t t0 = 0;
  for (int it = 0; j >= 0; ++it) {
    if (lane == 0 && (it & 63) == 63) { volatile int32_t* d = kp.dbg + blockIdx.x * 8; d[4] = j; d[6] = it; }
    const int idx = j - lane;
    const bool valid = idx >= 0;
    // relaxed: the prefix needs only the values carried in the status words
    const unsigned long long b = valid ? ld_relaxed_u64(&kp.sig[idx].ovh) : 0ull;
    const unsigned incl = __ballot_sync(0xffffffffu, !valid || (b & LB_INCL));
    const unsigned agg = __ballot_sync(0xffffffffu, valid && (b & LB_AGG));
    const int stop = incl ? __ffs(incl) - 1 : 32;
    const unsigned need = stop == 32 ? 0xffffffffu : ((1u << stop) - 1);
    unsigned take = need;
    const bool complete = (agg & need) == need;
    if (!complete) take = (1u << (__ffs(~agg & need) - 1)) - 1;   // AGG prefix of the window
    // accumulate the AGG lanes in `take`
    long long c = ((take >> lane) & 1) ? (long long)((b >> 2) & 0x7fffffffull) : 0;
    long long q = ((take >> lane) & 1) ? (long long)(b >> 33) : 0;
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
      c += __shfl_xor_sync(0xffffffffu, c, d);
      q += __shfl_xor_sync(0xffffffffu, q, d);
    }
    sc += c;
    sn += q;
    if (complete) {
      if (stop < 32) {
        const unsigned long long bs = __shfl_sync(0xffffffffu, b, stop);
        const int vs = __shfl_sync(0xffffffffu, (int)valid, stop);
        if (vs) { base_out = (long long)((bs >> 2) & 0x7fffffffull); base_q = (long long)((bs >> 33) & 0x3fffffffull); }
        j = -1;
        break;
      }
      j -= 32;
      continue;
    }
    j -= __popc(take);
    // after early termination only batches without output may give up (a batch
    // with output precedes the terminating batch, whose look-back saw all of
    // its predecessors' aggregates, so this loop finishes)
    int quit = lane == 0 && (ld_relaxed_s32(&kp.ctl->status) || (count == 0 && ld_relaxed_s32(&kp.ctl->done)));
    if ((it & 1023) == 1023 && lane == 0) {
      if (t0 == 0) t0 = globaltimer();
      else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 3, t, j, (long long)b); quit = 1; }
    }
    if (__shfl_sync(0xffffffffu, quit, 0)) return false;   // warp-uniform exit
    if (try_only && it >= 2) { *ready = 0; return true; }  // after the termination check
    lb_spin(ns, it);
  }
  out_off = (int)(base_out + sc);
  q_off = (int)(base_q + sn);
  *ready = 1;
  return true;
}

__device__ __forceinline__ int lb_nb(const KParams& kp, int N, long long V) {
  if (N <= 0) return 0;
  // safe over-estimate of the greedy batch count
  const long long v2 = (2 * V + kp.Tg - 1) / kp.Tg;
  return N / kp.Bg + (int)(v2 > 1 ? v2 : 1);
}

// One dequeued batch with the look-back chain, in three phases separated by
// its two waits (Alg. 5 wait points): lb_phase_a runs up to the
// Discovered wait, lb_phase_d up to the Counted (prefix) wait, lb_phase_c to
// the end.  The phases return PH_* (next phase); with try_only a wait that is
// not yet satisfied returns the same phase (multi-batch execution).
enum : int32_t { PH_IDLE = 0, PH_CLAIMED = 1, PH_A = 2, PH_D = 3, PH_C = 4, PH_ABORT = 5 };

__device__ __forceinline__ int lb_phase_a(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh) {
  const int t = sh.t, o_begin = sh.o_begin;
  Sig* mine = kp.sig + t;
  clk_mark(kp, sh, 0);
  beacon(kp, 2, t, 0);
  const int nP = load_parents(kp, P, sm, sh, o_begin, sh.o_end - o_begin, false);
  trace_ev(kp, t, 1);
  const int E = sh.E;
  const bool oversize = E > kp.T;
  const uint32_t key0 = (uint32_t)o_begin + 1;
  if (threadIdx.x == 0) { sh.steal = 0; sh.aborted = 0; sh.s_early = 0; }
  __syncthreads();
  clk_mark(kp, sh, 1);
  if (oversize) {
    if (!oversize_discover(kp, P, sm, sh, key0, sm_p_rs(kp)[0], E)) return PH_ABORT;
  } else {
    discover(kp, P, sm, sh, o_begin, nP, E);
  }
  clk_mark(kp, sh, 2);
  beacon(kp, 4, t, 0);
  trace_ev(kp, t, 2);
  // own discovery done: LOCAL.  The release store orders the block's atomicMin
  // marks (performed before discover's closing barrier) ahead of the flag.
  if (threadIdx.x == 0) st_release_u64(&mine->word, LB_LOCAL);
  // early Discovered: all predecessors already discovered?  Warp 1 looks back
  // while thread 0 (warp 0) waits out the release fence of LOCAL.
  if (threadIdx.x >= 32 && threadIdx.x < 64 && !oversize && !(kp.flags & F_NO_EARLY)) {
    int ready = 0;
    if (!lb_wait_discovered(kp, t, true, &ready)) ready = -1;
    if (threadIdx.x == 32) { sh.s_early = ready; if (ready < 0) sh.aborted = 1; }
  }
  __syncthreads();
  clk_mark(kp, sh, 3);
  if (sh.aborted) return PH_ABORT;
  if (sh.s_early == 1) {
    trace_ev(kp, t, 3);
    if (threadIdx.x == 0) st_release_u64(&mine->word, LB_LOCAL | LB_DINCL);
    rediscover_count(kp, P, sm, sh, o_begin, E, true);   // before sorting: removed sort to the end
    if (threadIdx.x == 0) {
      sh.nb = lb_nb(kp, sh.count, sh.V);
      st_relaxed_u64(&mine->ovh, lb_pfx(LB_AGG, sh.count, sh.nb));   // early Counted
      stat_add(kp, &kp.stats->redisc_early, 1);
    }
    trace_ev(kp, t, 4);
    clk_mark(kp, sh, 4);
    if (!(kp.flags & F_NO_SORT)) sort_segments(kp, sm, sh, nP);
    clk_mark(kp, sh, 5);
    return PH_C;
  }
  if (!oversize && !(kp.flags & F_NO_SORT)) sort_segments(kp, sm, sh, nP);   // speculative sort
  clk_mark(kp, sh, 5);
  beacon(kp, 6, t, 0);
  return PH_D;
}

__device__ __forceinline__ int lb_phase_d(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                                          bool try_only) {
  const int t = sh.t, o_begin = sh.o_begin, E = sh.E;
  Sig* mine = kp.sig + t;
  if (threadIdx.x < 32) {
    int ready = 0;
    const bool ok = lb_wait_discovered(kp, t, try_only, &ready);
    if (threadIdx.x == 0) { sh.aborted = ok ? 0 : 1; sh.s_mid = ready; }
  }
  __syncthreads();
  if (sh.aborted) return PH_ABORT;
  if (!sh.s_mid) return PH_D;
  clk_mark(kp, sh, 3);
  trace_ev(kp, t, 3);
  if (threadIdx.x == 0) st_release_u64(&mine->word, LB_LOCAL | LB_DINCL);
  if (E > kp.T) {
    oversize_rediscover_count(kp, P, sm, sh, (uint32_t)o_begin + 1, sm_p_rs(kp)[0], E);
  } else {
    rediscover_count(kp, P, sm, sh, o_begin, E, true);   // removed: flagged, no re-sort
  }
  if (threadIdx.x == 0) {
    sh.nb = lb_nb(kp, sh.count, sh.V);
    st_relaxed_u64(&mine->ovh, lb_pfx(LB_AGG, sh.count, sh.nb));
    stat_add(kp, &kp.stats->redisc_late, 1);
  }
  trace_ev(kp, t, 4);
  clk_mark(kp, sh, 4);
  return PH_C;
}

__device__ __forceinline__ int lb_phase_c(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                                          uint32_t epoch, bool try_only) {
  const int t = sh.t, E = sh.E;
  const bool oversize = E > kp.T;
  Sig* mine = kp.sig + t;
  // Counted: prefix over the predecessors' aggregates
  beacon(kp, 8, t, sh.count);
  trace_ev(kp, t, 5);
  if (threadIdx.x < 32) {
    int out_off = 0, q_off = 0, ready = 0;
    const bool ok = lb_prefix(kp, P, t, sh.count, out_off, q_off, try_only, &ready);
    if (threadIdx.x == 0) {
      sh.s_mid = ready;
      if (!ok) {
        sh.aborted = 1;
      } else if (ready) {
        sh.aborted = 0;
        sh.out_off = out_off;
        sh.q_off = q_off;
        if ((long long)q_off + sh.nb > kp.qcap) { latch_error(kp.ctl, ST_CAPACITY); sh.nb = 0; sh.aborted = 1; }
        // Work aggregation without a sequential decision chain: an
        // even slot whose output is below half a batch (nodes and valence)
        // forwards it to slot t+1 when t+1 is already a published non-empty
        // batch; odd slots never forward, so an overhang is one slot deep and
        // fits the receiver's first batch.  The receiver cuts the combined range
        // into the slots both reserved (next-fit: NF(A ++ B) <= NF(A) + NF(B)).
        bool fwd = false;
        if (!(kp.flags & (F_NO_OVERHANG | F_MULTI_BATCH)) && !(t & 1) && !oversize && sh.count > 0 &&
            2 * sh.count < kp.Bg && 2 * sh.V < (long long)kp.Tg && t + 1 < kp.qcap && !sh.aborted) {
          const Desc* d1 = kp.desc + t + 1;
          if (ld_acquire_u32(&d1->tag) == epoch)
            fwd = ld_relaxed_s32(&d1->o_begin) < ld_relaxed_s32(&d1->o_end);
        }
        if (fwd) {
          kp.fwdv[2 * t] = (uint32_t)sh.count;
          kp.fwdv[2 * t + 1] = (uint32_t)sh.V;
          __threadfence();
          stat_add(kp, &kp.stats->ovh_forwards, 1);
        }
        sh.fwd = fwd;
        st_relaxed_u64(&mine->ovh, lb_pfx(LB_INCL, out_off + sh.count, q_off + sh.nb) | (fwd ? LB_FWD : 0ull));
        atomicMax(&kp.ctl->qtail, q_off + sh.nb);
        atomicMax(&kp.ctl->chain_total, out_off + sh.count);
        stat_add(kp, &kp.stats->generated, sh.nb);
        // receiver: an odd slot takes the overhang of slot t-1 if it forwarded
        sh.ovh_n = 0;
        sh.ovh_t = 0;
        if ((t & 1) && !(kp.flags & (F_NO_OVERHANG | F_MULTI_BATCH)) && !sh.aborted) {
          uint64_t t0 = 0;
          for (int it = 0;; ++it) {
            const unsigned long long b = ld_relaxed_u64(&kp.sig[t - 1].ovh);
            if ((b & 3) == LB_AGG && ((b >> 2) & 0x7fffffffull) == 0) break;   // empty / no output: no forward
            if ((b & 3) == LB_INCL) {
              if (b & LB_FWD) {
                fence_acquire_gpu();
                sh.ovh_n = (int)__ldcg(kp.fwdv + 2 * (t - 1));
                sh.ovh_t = (int)__ldcg(kp.fwdv + 2 * (t - 1) + 1);
              }
              break;
            }
            if (ld_relaxed_s32(&kp.ctl->done)) break;   // terminated: nothing left to batch
            if ((it & 1023) == 1023) {
              if (t0 == 0) t0 = globaltimer();
              else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 7, t, (long long)b, 0); sh.aborted = 1; break; }
            }
          }
        }
      } else {
        sh.aborted = 0;
      }
    }
  }
  __syncthreads();
  if (sh.aborted) return PH_ABORT;
  if (!sh.s_mid) return PH_C;
  clk_mark(kp, sh, 6);
  const int out_off = sh.out_off;
  // batches are cut over [out_off - overhang, out_off + count) into the slots
  // reserved by the forwarder and by this batch (contiguous in the queue);
  // a forwarder generates nothing and publishes none of its reserved slots
  const int onb = sh.ovh_n > 0 ? lb_nb(kp, sh.ovh_n, sh.ovh_t) : 0;
  const int q_off = sh.q_off - onb;
  const int nb = sh.fwd ? 0 : sh.nb + onb;
  beacon(kp, 9, t, out_off);
  trace_ev(kp, t, 6);
  GenState g;
  if (threadIdx.x == 0) {
    g.start = out_off - sh.ovh_n; g.cnt = sh.ovh_n; g.val = sh.ovh_t;
    g.emitted = 0; g.has_pend = 0; g.defer = !oversize;
  }
  if (oversize) {
    if (!oversize_gather_sort(kp, P, sm, sh, sm_p_rs(kp)[0], E)) return PH_ABORT;
    oversize_output(kp, P, sm, sh, out_off, nb > 0, g, q_off, nb, epoch);
    if (threadIdx.x == 0) stat_add(kp, &kp.stats->oversize, 1);
  } else {
    // write_output ends with a block barrier: the block's o[] writes precede
    // thread 0's fence below, which publishes them cumulatively
    write_output(kp, P, sm, sh, E, out_off, nb > 0);
    clk_mark(kp, sh, 7);
    trace_ev(kp, t, 7);
    if (nb > 0 && threadIdx.x == 0) gen_chunk(kp, g, sm_cand(kp), E, out_off, q_off, nb, epoch);
  }
  if (threadIdx.x == 0) {
    int emitted = 0;
    if (nb > 0) {
      gen_finish(kp, g, out_off + sh.count, q_off, nb, epoch);   // descriptor fields only (deferred tags)
      if (g.emitted > nb) latch_error(kp.ctl, ST_CAPACITY);
      emitted = min(g.emitted, nb);
    }
    // empty slots: discovered, zero aggregate (values only)
    for (int i = emitted; i < nb; ++i) {
      st_relaxed_u64(&kp.sig[q_off + i].word, LB_LOCAL);
      st_relaxed_u64(&kp.sig[q_off + i].ovh, lb_pfx(LB_AGG, 0, 0));
      Desc* d = kp.desc + q_off + i;
      d->o_begin = 0; d->o_end = 0; d->next = q_off + i + 1;
    }
    stat_add(kp, &kp.stats->executed, 1);
    const int total = out_off + sh.count;
    if (sh.ovh_n > 0) {   // the forwarder's o[] entries must be visible before our batches cover them
      uint64_t t0 = 0;
      for (int it = 0; !(ld_relaxed_u64(&kp.sig[t - 1].word) & LB_OUTDONE); ++it) {
        if (ld_relaxed_s32(&kp.ctl->done)) break;
        if ((it & 1023) == 1023) {
          if (t0 == 0) t0 = globaltimer();
          else if (globaltimer() - t0 > kWatchdogNs) { latch_hang(kp.ctl, 8, t, 0, 0); break; }
        }
      }
    }
    // one fence publishes the o[] writes and every descriptor's fields; the
    // tags (and the completion count) are then relaxed stores (release pattern)
    fence_acquire_gpu();
    if (sh.fwd) st_relaxed_u64(&mine->word, LB_LOCAL | LB_DINCL | LB_OUTDONE);
    for (int i = 0; i < nb; ++i) st_relaxed_u32(&kp.desc[q_off + i].tag, epoch);
    if (total == P.pos0 + P.size) {             // early termination
      atomicExch(&kp.ctl->done, 1);
    } else {
      // count this slot and the empties it generated as finished (each slot
      // reserves before it counts itself).  Fire-and-forget: chain end without
      // termination (completed == qtail) is detected by the idle dequeuers
      // (lb_chain_exhausted), off this block's critical path.
      red_relaxed_add_s32(&kp.ctl->completed, 1 + (nb - emitted));   // a forwarder: nb = 0
    }
  }
  trace_ev(kp, t, 8);
#ifdef RCM_TRACE
  if (kp.collect_stats == 3 && threadIdx.x == 0 && kp.trace && t < kp.trace_cap) {
    kp.trace[(size_t)t * kTraceW + 10] = (unsigned long long)(uint32_t)ld_relaxed_s32(&kp.ctl->head);
    kp.trace[(size_t)t * kTraceW + 11] = (unsigned long long)(uint32_t)q_off;
  }
  if (kp.collect_stats == 3 && threadIdx.x == 0 && kp.trace && nb > 0)
    for (int i = 0; i < nb && q_off + i < kp.trace_cap; ++i)
      kp.trace[(size_t)(q_off + i) * kTraceW + kTraceW - 1] = ((unsigned long long)(uint32_t)t << 32) | blockIdx.x;
#endif
  __syncthreads();
  clk_mark(kp, sh, 8);
  return PH_IDLE;
}

// Process one dequeued batch with the look-back chain, waiting in place.
__device__ __forceinline__ void lb_batch(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                                         uint32_t epoch) {
  int ph = lb_phase_a(kp, P, sm, sh);
  if (ph == PH_D) ph = lb_phase_d(kp, P, sm, sh, false);
  if (ph == PH_C) lb_phase_c(kp, P, sm, sh, epoch, false);
}

// Multi-batch execution: thread 0 polls the claimed slot of a
// context once.  Returns PH_A (published batch), PH_IDLE (published empty slot,
// consumed), PH_CLAIMED (not yet published) or PH_ABORT (chain over).
static __device__ int mb_poll(const KParams& kp, ShState& s, uint32_t epoch) {
  const int t = s.t;
  if (t >= kp.qcap || ld_relaxed_s32(&kp.ctl->done)) return PH_ABORT;
  const Desc* d = kp.desc + t;
  if (ld_relaxed_u32(&d->tag) != epoch) {
    if ((++s.mb_it & 15) == 0 && lb_chain_exhausted(kp)) return PH_ABORT;
    return PH_CLAIMED;
  }
  (void)ld_acquire_u32(&d->tag);
  const int b = ld_relaxed_s32(&d->o_begin), e = ld_relaxed_s32(&d->o_end);
  stat_add(kp, &kp.stats->dequeued, 1);
  if (b == e) { stat_add(kp, &kp.stats->empty, 1); return PH_IDLE; }
  trace_ev(kp, t, 0);
  s.o_begin = b;
  s.o_end = e;
  return PH_A;
}

// Multi-batch execution (RCM_FLAG_MULTI_BATCH, SURVEY.md §8(f) NEXT-2,
// P:L719-731): every block keeps two batch contexts (own shared scratch and
// state).  Instead of waiting for Discovered or Counted, the block checks the
// signal once and moves on to the other context, which may draw a new batch
// from the queue.  Batches of one block can finish out of order; later ones
// never overtake earlier ones for Discovered (the look-back enforces it).
static __device__ __noinline__ void chain_worker_mb(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh0, ShState& sh1,
                                uint32_t epoch) {
  const uint32_t cbytes = (uint32_t)((smem_bytes(kp.BS, kp.T) + 15) & ~size_t(15));
  if (threadIdx.x == 0) {
    sh0.mb = PH_IDLE;
    sh1.mb = PH_IDLE;
    for (int i = 0; i < 10; ++i) sh0.clk[i] = sh1.clk[i] = 0;
    sh0.tclk = sh1.tclk = clock64();
  }
  __syncthreads();
  uint64_t t_idle = 0;   // thread 0: start of the current stretch without progress (watchdog)
  unsigned ns = 0;
  for (;;) {
    bool progress = false;
    for (int c = 0; c < 2; ++c) {
      ShState& s = c ? sh1 : sh0;
      if (threadIdx.x == 0) rcm_ctx_base = c ? cbytes : 0u;
      __syncthreads();
      const int ph = s.mb;
      // every thread has read the phase before thread 0 may overwrite it below
      // (compute-sanitizer racecheck: a late reader could otherwise follow the
      // new phase into a different sequence of block barriers)
      __syncthreads();
      int nx = ph;
      if (ph == PH_IDLE) {
        if (threadIdx.x == 0) {
          if (ld_relaxed_s32(&kp.ctl->done)) {
            nx = PH_ABORT;
          } else {
            s.t = atomicAdd(&kp.ctl->head, 1);
            s.mb_it = 0;
            trace_ev(kp, s.t, 9);
            nx = PH_CLAIMED;
          }
        }
      } else if (ph == PH_CLAIMED) {
        if (threadIdx.x == 0) nx = mb_poll(kp, s, epoch);
      } else if (ph == PH_A) {
        nx = lb_phase_a(kp, P, sm, s);
      } else if (ph == PH_D) {
        nx = lb_phase_d(kp, P, sm, s, true);
      } else if (ph == PH_C) {
        nx = lb_phase_c(kp, P, sm, s, epoch, true);
      }
      if (threadIdx.x == 0) s.mb = nx;
      __syncthreads();
      progress |= s.mb != ph;
    }
    if (threadIdx.x == 0) {   // progress beacon of both contexts (rcm_debug_state)
      volatile int32_t* d = kp.dbg + blockIdx.x * 8;
      d[4] = sh0.t;
      d[5] = sh1.t;
      d[6] = sh0.mb * 8 + sh1.mb;
    }
    if (sh0.mb == PH_ABORT && sh1.mb == PH_ABORT) break;
    if (threadIdx.x == 0) {
      if (progress) {
        t_idle = 0;
        ns = 0;
      } else {
        __nanosleep(ns);
        if (ns < 128) ns = ns ? ns * 2 : 16;
        const uint64_t now = globaltimer();
        if (!t_idle) t_idle = now;
        else if (now - t_idle > kWatchdogNs) { latch_hang(kp.ctl, 6, sh0.t, sh1.t, sh0.mb * 8 + sh1.mb); }
      }
    }
  }
  if (threadIdx.x == 0) rcm_ctx_base = 0;
  if (kp.collect_stats == 2 && threadIdx.x == 0)
    for (int i = 0; i < 10; ++i) atomicAdd(&kp.stats->stage[i], (unsigned long long)(sh0.clk[i] + sh1.clk[i]));
  __syncthreads();
}

__device__ __forceinline__ void chain_worker(const KParams& kp, const Problem& P, const SmemPtrs& sm, ShState& sh,
                             uint32_t epoch) {
  if (threadIdx.x == 0) {
    for (int i = 0; i < 10; ++i) sh.clk[i] = 0;
    sh.tclk = clock64();
  }
  for (;;) {
    if (threadIdx.x == 0) sh.aborted = dequeue(kp, sh, epoch) ? 0 : 1;
    __syncthreads();
    if (sh.aborted) break;
    if (kp.flags & F_SERIAL_CHAIN) chain_batch(kp, P, sm, sh, epoch);   // Alg. 5 hand-off chain
    else lb_batch(kp, P, sm, sh, epoch);                                 // look-back chain
  }
  clk_mark(kp, sh, 0);
  beacon(kp, 12, -1, 0);
  if (kp.collect_stats == 2 && threadIdx.x == 0)
    for (int i = 0; i < 10; ++i) atomicAdd(&kp.stats->stage[i], (unsigned long long)sh.clk[i]);
  __syncthreads();
}

}  // namespace rcm
