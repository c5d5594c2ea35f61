// rcm_leveled.cuh -- NEXT-3: level-synchronous RCM on the B200 (Alg. 2,
// the paper's GPU-RCM baseline), producing the same
// permutation as serial RCM and as the batch chain.  It runs inside the
// persistent kernel; a BFS level costs two grid barriers:
//
//   D  discover (Alg. 4 ln 4-9): every node x of the new level
//      claims its unplaced neighbours n with m_n <- atomicMin(word[n], pos(x)+1)
//      -- the parent-rank key of the chain (C-4), so after all claims of the
//      level the owner of n is the earliest parent in o that sees it (Alg. 1
//      ln 8-12).  Warp-cooperative, load-balanced expansion
//      (rcm_expand.cuh); rows above kLvBigRow edges are expanded by the block.
//   == grid barrier (every claim of the level is final: the paper's
//      "Discovered" for all batches of the level at once)
//   R  rediscover + sort + count, per batch of <= B_s parents / <= T edge slots
//      (the chain's load_parents / sort_segments): a child n is kept by parent
//      p iff owner(n) == pos(p)+1 (Alg. 5 ln 16-17); each parent's children
//      sorted by (valence, id) (C-1); duplicate entries of a row
//      collapse after the sort (C-8).  Kept ids go to HBM scratch in order.
//   == grid barrier (every block's child count is published)
//   W  prefix of the block counts (the paper's Counted), output with fused
//      reverse, then D of the children this block just wrote.
//
// A level wider than nblocks x B_s parents runs in rounds (R == W per round).
// If one block's output is far above the mean, the next D is re-balanced
// over all blocks behind one more barrier.
#pragma once
#include "rcm_components.cuh"

namespace rcm {

constexpr int kLvU = 4;            // edges per lane in flight (D)
constexpr int kLvBigRow = 2048;    // rows longer than this are expanded by the whole block (D)

// D over the nodes at matrix-local positions [x0, x1): claim every neighbour
// whose owner key is larger than pos + 1.  Block-local work, no barrier.
static __device__ void lv_discover(const KParams& kp, const Problem& P, ShState& sh, int x0, int x1) {
  const int cnt = x1 - x0;
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
      const int v = ld_cg_s32(o + x0 + i);
      rs = __ldg(rp + v);
      d = __ldg(rp + v + 1) - rs;
      key = (uint32_t)(x0 + i) + 1u;
      if (d > kLvBigRow) {
        const int k = atomicAdd(&sh.big_n, 1);
        if (k < 256) { sh.big_list[k] = i; d = 0; }   // else: expanded here by the warp
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
      for (int u = 0; u < kLvU; ++u) {
        const uint32_t k = __shfl_sync(kFull, key, j[u] & 31);
        if (c[u] >= 0 && (uint32_t)(wv[u] >> 32) > k)
          atomicMin(word + c[u], ((unsigned long long)k << 32) | (wv[u] & 0xffffffffull));
      }
    }
  }
  __syncthreads();
  const int nbig = min(sh.big_n, 256);
  for (int bi = 0; bi < nbig; ++bi) {   // long rows: the whole block, kLvU edges per thread in flight
    const int i = sh.big_list[bi];
    const int v = ld_cg_s32(o + x0 + i);
    const int rs = __ldg(rp + v), re = __ldg(rp + v + 1);
    const uint32_t k = (uint32_t)(x0 + i) + 1u;
    for (int e0 = rs + threadIdx.x; e0 < re; e0 += kThreads * kLvU) {
      int c[kLvU];
      unsigned long long wv[kLvU];
#pragma unroll
      for (int u = 0; u < kLvU; ++u) {
        const int e = e0 + u * kThreads;
        c[u] = e < re ? __ldg(col + e) : -1;
      }
#pragma unroll
      for (int u = 0; u < kLvU; ++u) wv[u] = c[u] >= 0 ? ld_weak_u64(word + c[u]) : 0ull;
#pragma unroll
      for (int u = 0; u < kLvU; ++u)
        if (c[u] >= 0 && (uint32_t)(wv[u] >> 32) > k)
          atomicMin(word + c[u], ((unsigned long long)k << 32) | (wv[u] & 0xffffffffull));
    }
  }
  __syncthreads();
}

// Append `cnt` ids (already in order) as the next entry of this block's output
// list; when the list is full its entries are first merged into one region.
__device__ __forceinline__ int lv_alloc(const KParams& kp, const CompWS& w, int32_t* gcur, int cnt) {
  const int base = atomicAdd(gcur, cnt);
  if ((long long)base + cnt > w.cap) { latch_error(kp.ctl, ST_CAPACITY); return -1; }
  return base;
}
static __device__ void lv_list_push(const KParams& kp, const CompWS& w, ShState& sh, int32_t* gcur, int base, int cnt) {
  // called by all threads; sh.lv_* updated by thread 0
  if (sh.lv_n == kLvList) {   // merge the list into one contiguous region
    int tot = 0;
    for (int j = 0; j < kLvList; ++j) tot += sh.lv_cnt[j];
    __syncthreads();
    if (threadIdx.x == 0) sh.k = lv_alloc(kp, w, gcur, tot);
    __syncthreads();
    const int nb = sh.k;
    if (nb >= 0) {
      int run = 0;
      for (int j = 0; j < kLvList; ++j) {
        for (int i = threadIdx.x; i < sh.lv_cnt[j]; i += kThreads) w.vals1[nb + run + i] = __ldcg(w.vals1 + sh.lv_off[j] + i);
        run += sh.lv_cnt[j];
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) { sh.lv_off[0] = nb; sh.lv_cnt[0] = tot; sh.lv_n = 1; }
    __syncthreads();
  }
  if (threadIdx.x == 0) { sh.lv_off[sh.lv_n] = base; sh.lv_cnt[sh.lv_n] = cnt; ++sh.lv_n; }
  __syncthreads();
}

// The sorted, kept children of a batch (segments cand[p_eo[lp] .. + p_cnt[lp]))
// -> HBM scratch in slot order, duplicates (adjacent after the sort) dropped.
static __device__ void lv_emit(const KParams& kp, const CompWS& w, ShState& sh, int32_t* gcur, int E) {
  const int per = (E + kThreads - 1) / kThreads;
  const int b0 = min(E, threadIdx.x * per), b1 = min(E, b0 + per);
  const unsigned long long* cand = sm_cand(kp);
  auto valid = [&](int e) {
    const int lp = sm_lpof(kp)[e];
    const int i = e - sm_p_eo(kp)[lp];
    return i < sm_p_cnt(kp)[lp] && (i == 0 || cand[e] != cand[e - 1]);
  };
  int k = 0;
  for (int e = b0; e < b1; ++e) k += valid(e);
  int tot;
  int r = block_exclusive_scan<int32_t>(k, sh.wtmp32, tot);
  if (tot == 0) return;
  if (threadIdx.x == 0) sh.k = lv_alloc(kp, w, gcur, tot);
  __syncthreads();
  const int base = sh.k;
  if (base >= 0)
    for (int e = b0; e < b1; ++e)
      if (valid(e)) w.vals1[base + r++] = (int)(uint32_t)cand[e];
  lv_list_push(kp, w, sh, gcur, base < 0 ? 0 : base, base < 0 ? 0 : tot);
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
  if (threadIdx.x == 0) sh.k = lv_alloc(kp, w, gcur, U);
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
    if (ok) w.vals1[base + run + r] = (int)(uint32_t)x;
    run += tot;
  }
  lv_list_push(kp, w, sh, gcur, base, U);
  if (threadIdx.x == 0) stat_add(kp, &kp.stats->oversize, 1);
}

// R over this block's parents [cb, ce) of the current level: batches of
// <= Bg parents / <= T edge slots, each rediscovered, sorted and emitted.
static __device__ void lv_rediscover(const KParams& kp, const Problem& P, const CompWS& w, const SmemPtrs& sm,
                                     ShState& sh, int32_t* gcur, int32_t* scur, int cb, int ce) {
  const int32_t* col = kp.col_idx + P.ci_base;
  const unsigned long long* word = kp.word + P.node_base;
  for (int ob = cb; ob < ce;) {
    const int nP = load_parents(kp, P, sm, sh, ob, min(kp.Bg, ce - ob), true);
    const int E = sh.E;
    if (E > kp.T) {   // nP == 1, oversize
      lv_oversize(kp, P, w, sh, gcur, scur, ob);
      ob += 1;
      __syncthreads();
      continue;
    }
    for (int lp = threadIdx.x; lp < nP; lp += kThreads) sm_p_cnt(kp)[lp] = 0;
    __syncthreads();
    // rediscovery (Alg. 5 ln 16-17): keep n iff owner(n) == key(p)
    const uint32_t kfirst = (uint32_t)ob + 1u;
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
}

static __device__ void leveled_chain(const KParams& kp, const MainArgs& a, const Problem& P, const SmemPtrs& sm,
                                     ShState& sh) {
  const CompWS& w = a.w;
  const int nb = kp.nblocks, b = blockIdx.x;
  int32_t* o = kp.o + P.o_base;
  int32_t* perm = kp.perm + P.perm_base;
  int32_t* btot = w.hist;          // [2][kMaxBlocks]: per-block child counts, parity by round
  int32_t* gcur = w.sctl + 8;      // [2]: scratch cursors (children ids), parity by level
  int32_t* scur = w.sctl + 10;     // [2]: oversize spill cursors, parity by level
  if (gtid() == 0) {
    place_root(kp, P, P.seed, P.pos0);
    gcur[0] = gcur[1] = scur[0] = scur[1] = 0;
    stat_add(kp, &kp.stats->components, 1);
  }
  grid_barrier(kp);
  if (b == 0) lv_discover(kp, P, sh, P.pos0, P.pos0 + 1);
  grid_barrier(kp);
  int lb = P.pos0, le = P.pos0 + 1, par = 0;
  const int per_round = nb * kp.Bg;
  // per-round timeline of block 0 (collect_stats == 3): R start, R end, after
  // barrier 1, output written, D done, after the level barrier; children, level
  int nround = (b == 0 && threadIdx.x == 0) ? (int)kp.ctl->dbg[6] : 0;   // across the problems of a call
  auto tr = [&](int k, unsigned long long v) {
    if (kp.trace && b == 0 && threadIdx.x == 0 && nround < kp.trace_cap) kp.trace[(size_t)nround * kTraceW + k] = v;
  };
  for (int level = 0;; ++level) {
    int32_t* gc = gcur + (level & 1);
    int32_t* sc = scur + (level & 1);
    int le_next = le;
    for (int rb = lb; rb < le; rb += per_round) {
      // ---- R: this block's share of the round
      const int re_ = min(le, rb + per_round);
      const int m = (re_ - rb + nb - 1) / nb;
      const int cb = min(re_, rb + b * m), ce = min(re_, cb + m);
      if (threadIdx.x == 0) sh.lv_n = 0;
      __syncthreads();
      tr(0, globaltimer());
      lv_rediscover(kp, P, w, sm, sh, gc, sc, cb, ce);
      tr(1, globaltimer());
      int myc = 0;
      for (int j = 0; j < sh.lv_n; ++j) myc += sh.lv_cnt[j];
      if (threadIdx.x == 0) st_relaxed_s32(btot + par * kMaxBlocks + b, myc);
      grid_barrier(kp);
      tr(2, globaltimer());
      // ---- W: prefix of the block counts, output with fused reverse
      if (gtid() == 0) { gcur[(level + 1) & 1] = 0; scur[(level + 1) & 1] = 0; }
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
      const int x0 = le_next + sh.written;
      // flattened copy of the block's list: position x0 + i
      int run = 0;
      for (int j = 0; j < sh.lv_n; ++j) {
        const int off = sh.lv_off[j], cnt = sh.lv_cnt[j];
        for (int i = threadIdx.x; i < cnt; i += kThreads) {
          const int c = __ldcg(w.vals1 + off + i);
          const int x = x0 + run + i;
          o[x] = c;
          perm[P.mat_n - 1 - x] = c;
          if (kp.iperm) kp.iperm[P.node_base + c] = P.mat_n - 1 - x;
        }
        run += cnt;
      }
      __syncthreads();
      tr(3, globaltimer());
      // ---- D of the next level
      const long long mean = (total + nb - 1) / nb;
      if (maxc <= 4 * mean + 256) {
        lv_discover(kp, P, sh, x0, x0 + myc);     // the children this block wrote
      } else {                                      // skewed: spread the claims over all blocks
        grid_barrier(kp);
        const int mm = (total + nb - 1) / nb;
        const int d0 = min(total, b * mm), d1 = min(total, d0 + mm);
        lv_discover(kp, P, sh, le_next + d0, le_next + d1);
      }
      tr(4, globaltimer());
      tr(8, (unsigned long long)total);
      tr(9, (unsigned long long)level);
      tr(10, (unsigned long long)maxc);
      le_next += total;
      par ^= 1;
      ++nround;
    }
    grid_barrier(kp);
    if (nround > 0) { --nround; tr(5, globaltimer()); ++nround; }
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
