// rcm_leveled.cuh -- NEXT-3: level-synchronous RCM on the B200 (Alg. 2,
// the paper's GPU-RCM baseline), producing the same
// permutation as serial RCM and as the batch chain.  It runs inside the
// persistent kernel; a BFS level costs two grid barriers:
//
//   D  discover (Alg. 4 ln 4-9): every node x the block just wrote claims its
//      unplaced neighbours n with m_n <- atomicMin(word[n], pos(x)+1) -- the
//      parent-rank key of the chain (C-4), so after all claims of the level
//      the owner of n is the earliest parent in o that sees it (Alg. 1 ln 8-12,
//      P:L202-212).  Warp-cooperative, load-balanced expansion
//      (rcm_expand.cuh); rows above kLvWarpRow edges go to one block-wide pass.
//   == grid barrier (every claim of the level is final: the paper's
//      "Discovered" for all batches of the level at once)
//   R  rediscover + sort + count over an even share of the level, in batches of
//      <= B_s parents / <= T edge slots (the chain's segments and sort_segments): a
//      child n is kept by parent p iff owner(n) == pos(p)+1 (Alg. 5 ln 16-17);
//      each parent's children sorted by (valence, id) (C-1); duplicate
//      entries of a row collapse after the sort (C-8).  Kept ids are buffered
//      in shared memory (HBM scratch past kLvOut).
//   == grid barrier (every block's child count is published)
//   W  prefix of the block counts (the paper's Counted), output with fused
//      reverse, then D of the children this block wrote (their ids
//      kept in shared memory; D stores their row starts and valences by
//      position, so R of the next level loads a parent with one round trip).
//
// A level wider than nblocks x B_s parents runs in rounds (R..D per round).  If
// one block's output is far above the mean, that D is spread over all blocks
// behind one more barrier.
#pragma once
#include "rcm_components.cuh"

namespace rcm {

constexpr int kLvU = 4;            // edges per lane in flight (D)
constexpr int kLvWarpRow = 64;     // rows longer than this are expanded block-wide (D)
static_assert(kLvBig <= kThreads, "one long row per thread in the block scan");

__device__ __forceinline__ int32_t* lv_sm(const KParams& kp) {
  return reinterpret_cast<int32_t*>(rcm_dsm + lv_smem_base(kp.BS, kp.T));
}
__device__ __forceinline__ int32_t* lv_st_v(const KParams& kp) { return lv_sm(kp); }
__device__ __forceinline__ int32_t* lv_out(const KParams& kp) { return lv_sm(kp) + kLvStage; }
__device__ __forceinline__ int32_t* lv_bg_rs(const KParams& kp) { return lv_out(kp) + kLvOut; }
__device__ __forceinline__ int32_t* lv_bg_key(const KParams& kp) { return lv_bg_rs(kp) + kLvBig; }
__device__ __forceinline__ int32_t* lv_bg_pre(const KParams& kp) { return lv_bg_key(kp) + kLvBig; }   // kLvBig + 1

__device__ __forceinline__ void lv_claim(unsigned long long* word, int c, unsigned long long wv, uint32_t k) {
  if (c >= 0 && (uint32_t)(wv >> 32) > k) atomicMin(word + c, ((unsigned long long)k << 32) | (wv & 0xffffffffull));
}

// D over the nodes at matrix-local positions [x0, x0 + cnt): claim every
// neighbour whose owner key is larger than pos + 1.  `staged`: the ids are in
// lv_st_v (written by W), else in o[].  Row starts / valences are stored by
// position (prs, pdeg) for R.  Block-local work, no barrier.
static __device__ void lv_discover(const KParams& kp, const Problem& P, const CompWS& w, ShState& sh, int x0, int cnt,
                                   bool staged) {
  if (cnt <= 0) return;   // block-uniform
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int32_t* o = kp.o + P.o_base;
  const int32_t* rp = kp.row_ptr + P.rp_base;
  const int32_t* col = kp.col_idx + P.ci_base;
  unsigned long long* word = kp.word + P.node_base;
  if (threadIdx.x == 0) sh.big_n = 0;
  __syncthreads();
  const int per = min(32, max(1, (cnt + kWarps - 1) / kWarps));
  for (int i0 = wid * per; i0 < cnt; i0 += kWarps * per) {
    const int i = i0 + lane;
    int rs = 0, d = 0;
    uint32_t key = 0;
    if (lane < per && i < cnt) {
      const int v = staged ? lv_st_v(kp)[i] : ld_cg_s32(o + x0 + i);
      rs = __ldg(rp + v);
      d = __ldg(rp + v + 1) - rs;
      key = (uint32_t)(x0 + i) + 1u;
      w.front0[P.o_base + x0 + i] = rs;   // prs
      w.front1[P.o_base + x0 + i] = d;    // pdeg
      if (d > kLvWarpRow) {
        const int k = atomicAdd(&sh.big_n, 1);
        if (k < kLvBig) { lv_bg_rs(kp)[k] = rs; lv_bg_key(kp)[k] = (int)key; lv_bg_pre(kp)[k] = d; d = 0; }
        // else: expanded here by the warp
      }
    }
    WarpRows R;
    R.init(rs, d);
    for (int b = 0; b < R.E; b += 32 * kLvU) {
      int c[kLvU], j[kLvU];
      R.cols<kLvU>(col, b, c, j);
      unsigned long long wv[kLvU];
#pragma unroll
      for (int u = 0; u < kLvU; ++u) wv[u] = c[u] >= 0 ? ld_weak_u64(word + c[u]) : 0ull;   // prefilter
#pragma unroll
      for (int u = 0; u < kLvU; ++u) lv_claim(word, c[u], wv[u], __shfl_sync(kFull, key, j[u] & 31));
    }
  }
  __syncthreads();
  const int nbig = min(sh.big_n, kLvBig);
  if (nbig == 0) return;
  // long rows: one block-wide flattened pass over all of them
  int tot;
  const int len = threadIdx.x < nbig ? lv_bg_pre(kp)[threadIdx.x] : 0;
  const int ex = block_exclusive_scan<int32_t>(len, sh.wtmp32, tot);
  if (threadIdx.x < nbig) lv_bg_pre(kp)[threadIdx.x] = ex;
  if (threadIdx.x == 0) lv_bg_pre(kp)[nbig] = tot;
  __syncthreads();
  for (int e0 = threadIdx.x; e0 < tot; e0 += kThreads * kLvU) {
    int c[kLvU], jj[kLvU];
#pragma unroll
    for (int u = 0; u < kLvU; ++u) {
      const int e = e0 + u * kThreads;
      c[u] = -1;
      jj[u] = 0;
      if (e < tot) {
        int lo = 0, hi = nbig - 1;   // last row with pre <= e
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (lv_bg_pre(kp)[mid] <= e) lo = mid; else hi = mid - 1;
        }
        jj[u] = lo;
        c[u] = __ldg(col + lv_bg_rs(kp)[lo] + (e - lv_bg_pre(kp)[lo]));
      }
    }
    unsigned long long wv[kLvU];
#pragma unroll
    for (int u = 0; u < kLvU; ++u) wv[u] = c[u] >= 0 ? ld_weak_u64(word + c[u]) : 0ull;
#pragma unroll
    for (int u = 0; u < kLvU; ++u) lv_claim(word, c[u], wv[u], c[u] >= 0 ? (uint32_t)lv_bg_key(kp)[jj[u]] : 0u);
  }
  __syncthreads();
}

// HBM scratch for output past the shared buffer: w.ckey viewed as 2n ints
// (idle during a traversal), cursor per level parity.  A block reserves it in
// chunks that double with its overflow so far (>= 1,024 ids) and appends
// consecutive emits to its last chunk: a block's overflow is a few regions,
// and the level's reservations stay within 2n.
__device__ __forceinline__ int32_t* lv_ovf(const CompWS& w) { return reinterpret_cast<int32_t*>(w.ckey); }
__device__ __forceinline__ int lv_alloc(const KParams& kp, long long cap, int32_t* cur, int cnt) {
  const int base = atomicAdd(cur, cnt);
  if ((long long)base + cnt > cap) { latch_error(kp.ctl, ST_CAPACITY); return -1; }
  return base;
}
// Thread 0: room for `cnt` more overflow ids of this block; returns the write
// offset in lv_ovf (or -1 on a latched capacity error).  The last entry is
// extended or a new one opened; the caller writes the ids.
__device__ __forceinline__ int lv_ovf_reserve(const KParams& kp, const CompWS& w, ShState& sh, int32_t* gcur, int cnt) {
  if (sh.lv_n > 0 && sh.lv_cnt[sh.lv_n - 1] + cnt <= sh.lv_cap) {
    const int at = sh.lv_off[sh.lv_n - 1] + sh.lv_cnt[sh.lv_n - 1];
    sh.lv_cnt[sh.lv_n - 1] += cnt;
    return at;
  }
  if (sh.lv_n == kLvList) { latch_error(kp.ctl, ST_CAPACITY); return -1; }
  int so_far = 0;
  for (int j = 0; j < sh.lv_n; ++j) so_far += sh.lv_cnt[j];
  const int chunk = max(cnt, max(1024, so_far));
  const int base = lv_alloc(kp, 2 * w.cap, gcur, chunk);
  if (base < 0) return -1;
  sh.lv_off[sh.lv_n] = base;
  sh.lv_cnt[sh.lv_n] = cnt;
  sh.lv_cap = chunk;
  ++sh.lv_n;
  return base;
}

// Exclusive block scan with ONE barrier (warp totals in sh.wtmp32, read by
// every warp after the barrier).  The caller guarantees a full barrier between
// two calls (every R step has several), so one buffer suffices.
__device__ __forceinline__ int lv_scan1(int v, ShState& sh, int& total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int x = warp_incl_scan(v);
  if (lane == 31) sh.wtmp32[wid] = x;
  __syncthreads();
  int wv = lane < kWarps ? sh.wtmp32[lane] : 0;
#pragma unroll
  for (int d = 1; d < kWarps; d <<= 1) {
    const int y = __shfl_up_sync(kFull, wv, d);
    if (lane >= d) wv += y;
  }
  total = __shfl_sync(kFull, wv, kWarps - 1);
  const int base = __shfl_sync(kFull, wv, (wid + 31) & 31);
  return (wid ? base : 0) + x - v;
}

// The sorted, kept children of a batch (segments cand[p_eo[lp] .. + p_cnt[lp]))
// in slot order, duplicates (adjacent after the sort) dropped: appended to the
// block's shared-memory output buffer while it fits and no HBM entry exists
// yet, else to HBM scratch as the next entry of the block's list.
static __device__ void lv_emit(const KParams& kp, const CompWS& w, ShState& sh, int32_t* gcur, int E) {
  const int per = (E + kThreads - 1) / kThreads;
  const int b0 = min(E, threadIdx.x * per), b1 = min(E, b0 + per);
  const unsigned long long* cand = sm_cand(kp);
  auto valid = [&](int e) {
    const int lp = sm_lpof(kp)[e];
    const int i = e - sm_p_eo(kp)[lp];
    return i < sm_p_cnt(kp)[lp] && (i == 0 || cand[e] != cand[e - 1]);
  };
  // read before the scan's barrier; thread 0 updates lv_outn after it, and the
  // caller's end-of-batch barrier orders that before the next batch's read
  const int outn = sh.lv_outn, nlist = sh.lv_n;
  int k = 0;
  for (int e = b0; e < b1; ++e) k += valid(e);
  int tot;
  int r = lv_scan1(k, sh, tot);
  if (tot == 0) return;
  if (nlist == 0 && outn + tot <= kLvOut) {
    for (int e = b0; e < b1; ++e)
      if (valid(e)) lv_out(kp)[outn + r++] = (int)(uint32_t)cand[e];
    if (threadIdx.x == 0) sh.lv_outn = outn + tot;
    return;
  }
  __syncthreads();
  if (threadIdx.x == 0) sh.count = lv_ovf_reserve(kp, w, sh, gcur, tot);
  __syncthreads();
  const int base = sh.count;
  if (base >= 0)
    for (int e = b0; e < b1; ++e)
      if (valid(e)) lv_ovf(w)[base + r++] = (int)(uint32_t)cand[e];
  __syncthreads();
}

// A parent with more than T edges: its kept children counted,
// collected (shared memory when they fit T, else HBM scratch), sorted by one
// block, de-duplicated and emitted.
static __device__ void lv_oversize(const KParams& kp, const Problem& P, const CompWS& w, ShState& sh,
                                   int32_t* gcur, int32_t* scur, int q) {
  const int32_t* rp = kp.row_ptr + P.rp_base;
  const int32_t* col = kp.col_idx + P.ci_base;
  const unsigned long long* word = kp.word + P.node_base;
  const int v = ld_cg_s32(kp.o + P.o_base + q);
  const int rs = __ldg(rp + v), re = __ldg(rp + v + 1);
  const uint32_t key = (uint32_t)q + 1u;
  int k = 0;
  for (int e = rs + threadIdx.x; e < re; e += kThreads) k += (uint32_t)(ld_weak_u64(word + __ldg(col + e)) >> 32) == key;
  const int K = block_reduce_sum<int32_t>(k, sh.wtmp32);
  if (K == 0) return;
  const bool gm = K > kp.T;
  if (threadIdx.x == 0) {
    sh.count = 0;
    sh.spill_base = 0;
    if (gm) {
      const int sb = atomicAdd(scur, K);
      if ((long long)sb + K > kp.spill_cap) { latch_error(kp.ctl, ST_CAPACITY); sh.spill_base = -1; }
      else sh.spill_base = sb;
    }
  }
  __syncthreads();
  if (sh.spill_base < 0) return;
  unsigned long long* a = gm ? kp.spill + sh.spill_base : sm_cand(kp);
  for (int e = rs + threadIdx.x; e < re; e += kThreads) {
    const int c = __ldg(col + e);
    const unsigned long long wv = ld_weak_u64(word + c);
    if ((uint32_t)(wv >> 32) == key) a[atomicAdd(&sh.count, 1)] = ((wv & 0xffffffffull) << 32) | (uint32_t)c;
  }
  __syncthreads();
  if (gm) block_radix_sort_global(a, kp.spill + kp.spill_cap + sh.spill_base, K,
                                  reinterpret_cast<int32_t*>(sm_cand(kp)), sh);
  else bitonic_sort_flip(a, K, threadIdx.x, kThreads, [] { __syncthreads(); });
  __syncthreads();
  // de-duplicate (equal keys adjacent): count, one allocation, emit in rounds of kThreads
  auto key_at = [&](int i) { return gm ? __ldcg(a + i) : a[i]; };
  int u = 0;
  for (int i = threadIdx.x; i < K; i += kThreads) u += i == 0 || key_at(i) != key_at(i - 1);
  const int U = block_reduce_sum<int32_t>(u, sh.wtmp32);
  if (threadIdx.x == 0) sh.k = lv_ovf_reserve(kp, w, sh, gcur, U);
  __syncthreads();
  const int base = sh.k;
  if (base < 0) return;
  int run = 0;
  for (int i0 = 0; i0 < K; i0 += kThreads) {
    const int i = i0 + threadIdx.x;
    const unsigned long long x = i < K ? key_at(i) : 0ull;
    const bool ok = i < K && (i == 0 || x != key_at(i - 1));
    int tot;
    const int r = block_exclusive_scan<int32_t>(ok ? 1 : 0, sh.wtmp32, tot);
    if (ok) lv_ovf(w)[base + run + r] = (int)(uint32_t)x;
    run += tot;
  }
  __syncthreads();
  if (threadIdx.x == 0) stat_add(kp, &kp.stats->oversize, 1);
}

// load_parents (rcm_batch.cuh) for the parents at positions [q0, q0 + nP):
// id, row start and valence in one round trip (o[], and prs / pdeg written by
// D).  Cuts at T edge slots; sh.E = slots.
static __device__ int lv_parents(const KParams& kp, const Problem& P, const CompWS& w, ShState& sh, int q0, int nP) {
  if (nP <= kThreads) {   // one parent per thread: one-barrier scan, the T cut by a barrier count
    const int t = threadIdx.x;
    int rs = 0, d = 0;
    if (t < nP) {
      const int64_t x = P.o_base + q0 + t;
      sm_p_v(kp)[t] = ld_cg_s32(kp.o + x);
      rs = ld_cg_s32(w.front0 + x);
      d = ld_cg_s32(w.front1 + x);
    }
    int E;
    const int eo = lv_scan1(d, sh, E);
    const bool fit = t < nP && (t == 0 || eo + d <= kp.T);   // the first parent always (oversize alone)
    if (t < nP) {
      sm_p_rs(kp)[t] = rs;
      sm_p_eo(kp)[t] = eo;
      sm_p_eo(kp)[t + 1] = eo + d;   // == the next parent's offset; the last one ends the slots
      sm_p_cnt(kp)[t] = 0;
    }
    nP = __syncthreads_count(fit);
    E = sm_p_eo(kp)[nP];
    if (t == 0) { sh.nP = nP; sh.E = E; }
    if (E <= kp.T) {
      const int lane = t & 31;
      for (int lp = t >> 5; lp < nP; lp += kWarps) {
        const int eb = sm_p_eo(kp)[lp], ee = sm_p_eo(kp)[lp + 1];
        for (int j = eb + lane; j < ee; j += 32) sm_lpof(kp)[j] = (uint16_t)lp;
      }
    }
    __syncthreads();
    return nP;
  }
  for (int lp = threadIdx.x; lp < nP; lp += kThreads) {
    const int64_t x = P.o_base + q0 + lp;
    sm_p_v(kp)[lp] = ld_cg_s32(kp.o + x);
    sm_p_rs(kp)[lp] = ld_cg_s32(w.front0 + x);
    sm_p_eo(kp)[lp] = ld_cg_s32(w.front1 + x);
  }
  __syncthreads();
  int E = block_scan_array<int32_t>(sm_p_eo(kp), nP, sh.wtmp32);
  sm_p_eo(kp)[nP] = E;
  __syncthreads();
  if (E > kp.T && nP > 1) {   // longest prefix whose edges fit T (at least one parent)
    if (threadIdx.x == 0) {
      int lo = 1, hi = nP;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (sm_p_eo(kp)[mid] <= kp.T) lo = mid; else hi = mid - 1;
      }
      sh.nP = lo;
    }
    __syncthreads();
    nP = sh.nP;
    E = sm_p_eo(kp)[nP];
  }
  if (threadIdx.x == 0) { sh.nP = nP; sh.E = E; }
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

// R over the parents at positions [x0, x0 + cnt): batches of <= Bg parents /
// <= T edge slots, each rediscovered, sorted and emitted.  Returns the block's
// child count.
static __device__ int lv_rediscover(const KParams& kp, const Problem& P, const CompWS& w, const SmemPtrs& sm,
                                    ShState& sh, int32_t* gcur, int32_t* scur, int x0, int cnt) {
  const int32_t* col = kp.col_idx + P.ci_base;
  const unsigned long long* word = kp.word + P.node_base;
  if (threadIdx.x == 0) { sh.lv_n = 0; sh.lv_outn = 0; }
  __syncthreads();
  for (int ob = 0; ob < cnt;) {
    const int nP = lv_parents(kp, P, w, sh, x0 + ob, min(kp.Bg, cnt - ob));
    const int E = sh.E;
    if (E > kp.T) {   // nP == 1, oversize
      lv_oversize(kp, P, w, sh, gcur, scur, x0 + ob);
      ob += 1;
      __syncthreads();
      continue;
    }
    if (min(kp.Bg, cnt - ob) > kThreads) {   // (the one-parent-per-thread load zeroed them)
      for (int lp = threadIdx.x; lp < nP; lp += kThreads) sm_p_cnt(kp)[lp] = 0;
      __syncthreads();
    }
    // rediscovery (Alg. 5 ln 16-17): keep n iff owner(n) == key(p)
    const uint32_t kfirst = (uint32_t)(x0 + ob) + 1u;
    for (int e0 = threadIdx.x; e0 < E; e0 += kThreads * kDiscU) {
      int c[kDiscU];
#pragma unroll
      for (int u = 0; u < kDiscU; ++u) {
        const int e = e0 + u * kThreads;
        c[u] = -1;
        if (e < E) {
          const int lp = sm_lpof(kp)[e];
          c[u] = __ldg(col + sm_p_rs(kp)[lp] + (e - sm_p_eo(kp)[lp]));
        }
      }
      unsigned long long wv[kDiscU];
#pragma unroll
      for (int u = 0; u < kDiscU; ++u) wv[u] = c[u] >= 0 ? ld_weak_u64(word + c[u]) : 0ull;
#pragma unroll
      for (int u = 0; u < kDiscU; ++u) {
        if (c[u] < 0) continue;
        const int lp = sm_lpof(kp)[e0 + u * kThreads];
        if ((uint32_t)(wv[u] >> 32) == kfirst + (uint32_t)lp) {
          const int slot = sm_p_eo(kp)[lp] + atomicAdd(&sm_p_cnt(kp)[lp], 1);
          sm_cand(kp)[slot] = ((wv[u] & 0xffffffffull) << 32) | (uint32_t)c[u];
        }
      }
    }
    __syncthreads();
    sort_segments(kp, sm, sh, nP);   // (valence, id) per parent; duplicates end up adjacent
    lv_emit(kp, w, sh, gcur, E);
    if (threadIdx.x == 0) stat_add(kp, &kp.stats->executed, 1);
    ob += nP;
    __syncthreads();
  }
  int myc = sh.lv_outn;
  for (int j = 0; j < sh.lv_n; ++j) myc += sh.lv_cnt[j];
  return myc;
}

static __device__ void leveled_chain(const KParams& kp, const MainArgs& a, const Problem& P, const SmemPtrs& sm,
                                     ShState& sh) {
  const CompWS& w = a.w;
  const int nb = kp.nblocks, b = blockIdx.x;
  int32_t* o = kp.o + P.o_base;
  int32_t* perm = kp.perm + P.perm_base;
  int32_t* btot = w.hist;          // [2][kMaxBlocks]: per-block child counts, parity by round
  int32_t* gcur = w.sctl + 8;      // [2]: overflow scratch cursors, parity by round
  int32_t* scur = w.sctl + 10;     // [2]: oversize spill cursors, parity by round
  if (gtid() == 0) {
    place_root(kp, P, P.seed, P.pos0);
    gcur[0] = gcur[1] = scur[0] = scur[1] = 0;
    stat_add(kp, &kp.stats->components, 1);
  }
  if (b == 0 && threadIdx.x == 0) lv_st_v(kp)[0] = P.seed;
  __syncthreads();
  lv_discover(kp, P, w, sh, P.pos0, b == 0 ? 1 : 0, true);
  grid_barrier(kp);
  // per-round timeline of block 0 (collect_stats == 3): R start, R end, after
  // barrier 1, output written, D done, after the level barrier; children,
  // level, max block output
  int nround = (b == 0 && threadIdx.x == 0) ? (int)kp.ctl->dbg[6] : 0;   // across the problems of a call
  auto tr = [&](int k, unsigned long long v) {
    if (kp.trace && b == 0 && threadIdx.x == 0 && nround < kp.trace_cap) kp.trace[(size_t)nround * kTraceW + k] = v;
  };
  int lb = P.pos0, le = P.pos0 + 1, par = 0, rnd = 0;
  const int per_round = nb * kp.Bg;
  for (int level = 0;; ++level) {
    int le_next = le;
    for (int rb = lb; rb < le; rb += per_round) {
      // ---- R: an even share of the round
      const int re_ = min(le, rb + per_round);
      const int m = (re_ - rb + nb - 1) / nb;
      const int cb = min(re_, rb + b * m), ce = min(re_, cb + m);
      tr(0, globaltimer());
      // the other parity's scratch was last allocated in round - 1 (before its
      // barrier) and is read in W of round - 1: only its cursor is reset here,
      // its space is reused after this round's barrier
      if (gtid() == 0) { gcur[(rnd + 1) & 1] = 0; scur[(rnd + 1) & 1] = 0; }
      const int myc = lv_rediscover(kp, P, w, sm, sh, gcur + (rnd & 1), scur + (rnd & 1), cb, ce - cb);
      if (threadIdx.x == 0) st_relaxed_s32(btot + par * kMaxBlocks + b, myc);
      tr(1, globaltimer());
      grid_barrier(kp);
      tr(2, globaltimer());
      tr(6, (unsigned long long)kp.ctl->dbg[7]);
      // ---- W: prefix of the block counts, output with fused reverse
      int total = 0, mx = 0;
      for (int i0 = 0; i0 < nb; i0 += kThreads) {
        const int i = i0 + threadIdx.x;
        const int bc = i < nb ? ld_cg_s32(btot + par * kMaxBlocks + i) : 0;
        int tot;
        const int ex = block_exclusive_scan<int32_t>(bc, sh.wtmp32, tot);
        if (i == b) sh.written = total + ex;
        total += tot;
        mx = max(mx, bc);
      }
      mx = __reduce_max_sync(kFull, mx);
      if ((threadIdx.x & 31) == 0) sh.wtmp64b[threadIdx.x >> 5] = mx;
      __syncthreads();
      long long maxc = 0;
      for (int i = 0; i < kWarps; ++i) maxc = max(maxc, sh.wtmp64b[i]);
      const int xw = le_next + sh.written;
      auto put = [&](int i, int c) {
        const int x = xw + i;
        if (x >= P.mat_n) { latch_error(kp.ctl, ST_CAPACITY); return; }   // only after a latched scratch error
        o[x] = c;
        perm[P.mat_n - 1 - x] = c;
        if (kp.iperm) kp.iperm[P.node_base + c] = P.mat_n - 1 - x;
        if (i < kLvStage) lv_st_v(kp)[i] = c;
      };
      const int outn = sh.lv_outn;
      for (int i = threadIdx.x; i < outn; i += kThreads) put(i, lv_out(kp)[i]);
      int run = outn;
      for (int j = 0; j < sh.lv_n; ++j) {
        const int off = sh.lv_off[j], n = sh.lv_cnt[j];
        for (int i = threadIdx.x; i < n; i += kThreads) put(run + i, __ldcg(lv_ovf(w) + off + i));
        run += n;
      }
      __syncthreads();
      tr(3, globaltimer());
      // ---- D of the next level
      const long long mean = (total + nb - 1) / nb;
      if (maxc <= 4 * mean + 256) {
        lv_discover(kp, P, w, sh, xw, myc, myc <= kLvStage);   // the children this block wrote
      } else {                                                  // skewed: spread over all blocks
        grid_barrier(kp);
        const int mm = (int)mean;
        const int d0 = min(total, b * mm), d1 = min(total, d0 + mm);
        lv_discover(kp, P, w, sh, le_next + d0, d1 - d0, false);
      }
      tr(4, globaltimer());
      tr(8, (unsigned long long)total);
      tr(9, (unsigned long long)level);
      tr(10, (unsigned long long)maxc);
      le_next += total;
      par ^= 1;
      ++nround;
      ++rnd;
    }
    grid_barrier(kp);
    if (nround > 0) { --nround; tr(5, globaltimer()); tr(7, (unsigned long long)kp.ctl->dbg[7]); ++nround; }
    if (le_next == le) break;
    lb = le;
    le = le_next;
  }
  if (gtid() == 0) {
    kp.ctl->dbg[6] = nround;
    kp.ctl->chain_total = le;
    if (le < P.pos0 + P.size) kp.ctl->incomplete = 1;   // component exhausted, others remain
  }
  grid_barrier(kp);
}

}  // namespace rcm
