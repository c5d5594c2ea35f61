// rcm_components.cuh -- the device phases around the traversal that the paper
// leaves implicit, all executed inside the one persistent kernel (grid
// barriers between phases, all blocks co-resident):
//   * connected components of a disconnected graph, ordered by the C-6 rule (a13)
//   * a grid-wide stable LSD radix sort used to order components / matrices
//   * the pseudo-peripheral start finder of P:L365-375 (level-synchronous BFS)
#pragma once
#include <cuda_runtime.h>

#include "../../include/rcm.h"
#include "rcm_lookback.cuh"
#include "rcm_expand.cuh"

namespace rcm {

constexpr int kSortTile = 8 * kThreads;   // keys per tile of a radix pass (8 per thread)

struct CompWS {
  int32_t* label;              // union-find parent (-1: already ordered)
  unsigned long long* ckey;    // per root: min (deg << 32 | id)
  int32_t* csize;              // per root: component size
  unsigned long long* keys0;   // radix ping-pong buffers
  unsigned long long* keys1;
  int32_t* vals0;
  int32_t* vals1;
  long long* offs;             // component output offsets
  int32_t* hist;               // radix: 256 x tiles
  int32_t* sctl;               // [0] count, [1] current buffer, [2] skip flag
  int32_t* lev;                // GL levels
  int32_t* front0;
  int32_t* front1;
  int32_t* gctl;               // GL: [0] next frontier size
  unsigned long long* gkey;    // GL: [0] argmin of the last level
  int64_t cap;
};

// Arguments of one k_main launch.
struct MainArgs {
  CompWS w;
  int n;                // single graph: nodes
  long long nnz;
  int mode;
  int start;
  int validate;
  int vec;              // row_ptr 16-byte aligned
  int thr;              // solo threshold for components
  long long prob_cap;
  int idbits;
  int gl_only;          // rcm_find_pseudo_peripheral
  int gl_start;
  int32_t* gl_out;
};

__device__ __forceinline__ int gtid() { return blockIdx.x * kThreads + threadIdx.x; }
__device__ __forceinline__ int gthreads(const KParams& kp) { return kp.nblocks * kThreads; }

__device__ __forceinline__ void stamp(const KParams& kp, int i) {
  if (blockIdx.x == 0 && threadIdx.x == 0) kp.ctl->ts[i] = globaltimer();
}

// ============================================================ radix sort
// Grid-wide stable LSD radix sort of (key, val) pairs by bits [lo_bit, hi_bit)
// (8-bit digits; the order of equal keys -- and thus of bits below lo_bit when
// the input is already ordered by them -- is preserved).  Count in w.sctl[0]; w.sctl[1] = buffer holding the data.
// A digit that is equal in all keys is skipped.  `scratch`: >= 17 KB smem.
static __device__ void radix_sort_phase(const KParams& kp, const CompWS& w, int lo_bit, int hi_bit, int32_t* scratch,
                                 ShState& sh) {
  const int count = ld_cg_s32(w.sctl);
  if (count <= 1) return;
  const int tiles = (count + kSortTile - 1) / kSortTile;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const unsigned lt = (1u << lane) - 1;
  int32_t* off = scratch;           // 256
  int32_t* wcnt = scratch + 256;    // kWarps x 256
  for (int shift = lo_bit; shift < hi_bit; shift += 8) {
    const int cur = ld_cg_s32(w.sctl + 1);
    const unsigned long long* sk = cur ? w.keys1 : w.keys0;
    const int32_t* sv = cur ? w.vals1 : w.vals0;
    unsigned long long* dk = cur ? w.keys0 : w.keys1;
    int32_t* dv = cur ? w.vals0 : w.vals1;
    // 1. per-tile digit histograms
    for (int b = blockIdx.x; b < tiles; b += kp.nblocks) {
      for (int i = threadIdx.x; i < 256; i += kThreads) off[i] = 0;
      __syncthreads();
      for (int i = b * kSortTile + threadIdx.x; i < min(count, (b + 1) * kSortTile); i += kThreads)
        atomicAdd(&off[(__ldcg(sk + i) >> shift) & 0xff], 1);
      __syncthreads();
      for (int i = threadIdx.x; i < 256; i += kThreads) w.hist[i * tiles + b] = off[i];
      __syncthreads();
    }
    grid_barrier(kp);
    // 2. block 0: skip test + exclusive scan over (digit, tile)
    if (blockIdx.x == 0) {
      int skip = 0;
      for (int d = threadIdx.x; d < 256; d += kThreads) {
        long long s = 0;
        for (int t = 0; t < tiles; ++t) s += __ldcg(w.hist + d * tiles + t);
        if (s == count) skip = 1;
      }
      skip = __syncthreads_or(skip);
      if (!skip) {
        const int total = 256 * tiles;
        const int per = (total + kThreads - 1) / kThreads;
        const int b0 = threadIdx.x * per, e0 = min(total, b0 + per);
        int s = 0;
        for (int i = b0; i < e0; ++i) s += __ldcg(w.hist + i);
        int tot;
        int run = block_exclusive_scan<int32_t>(s, sh.wtmp32, tot);
        for (int i = b0; i < e0; ++i) { int x = __ldcg(w.hist + i); w.hist[i] = run; run += x; }
      }
      if (threadIdx.x == 0) w.sctl[2] = skip;
    }
    grid_barrier(kp);
    if (ld_cg_s32(w.sctl + 2)) continue;   // constant digit: no pass, no swap
    // 3. stable scatter, tile by tile
    for (int b = blockIdx.x; b < tiles; b += kp.nblocks) {
      for (int i = threadIdx.x; i < 256; i += kThreads) off[i] = __ldcg(w.hist + i * tiles + b);
      for (int j = 0; j < kSortTile / kThreads; ++j) {
        const int i = b * kSortTile + j * kThreads + threadIdx.x;
        const bool valid = i < count;
        const unsigned long long k = valid ? __ldcg(sk + i) : 0ull;
        const int v = valid ? __ldcg(sv + i) : 0;
        const int d = valid ? (int)((k >> shift) & 0xff) : 256;
        const unsigned peers = __match_any_sync(0xffffffffu, d);
        const int rank = __popc(peers & lt);
        for (int q = threadIdx.x; q < kWarps * 256; q += kThreads) wcnt[q] = 0;
        __syncthreads();
        if (valid && rank == 0) wcnt[wid * 256 + d] = __popc(peers);
        __syncthreads();
        for (int dg = threadIdx.x; dg < 256; dg += kThreads) {
          int run = off[dg];
          for (int ww = 0; ww < kWarps; ++ww) { int c = wcnt[ww * 256 + dg]; wcnt[ww * 256 + dg] = run; run += c; }
          off[dg] = run;
        }
        __syncthreads();
        if (valid) {
          const int pos = wcnt[wid * 256 + d] + rank;
          dk[pos] = k;
          dv[pos] = v;
        }
        __syncthreads();
      }
    }
    grid_barrier(kp);
    if (blockIdx.x == 0 && threadIdx.x == 0) w.sctl[1] = cur ^ 1;
    grid_barrier(kp);
  }
}

// ====================================================== connected components
// Union-find (hook the larger root under the smaller, path halving) over the
// nodes the chain-first pass left unvisited; components are then ordered by
// their minimum (valence, id) member (C-6) and laid out by a prefix sum.
__device__ __forceinline__ int uf_find(int32_t* label, int x) {
  int p = ld_cg_s32(label + x);
  while (p != x) {
    int gp = ld_cg_s32(label + p);
    if (gp != p) label[x] = gp;   // path halving (benign race)
    x = p;
    p = gp;
  }
  return x;
}

// Union two nodes: hook the larger root under the smaller (ECL-CC style).
__device__ __forceinline__ void uf_unite(int32_t* label, int u, int c) {
  for (;;) {
    int x = uf_find(label, u), y = uf_find(label, c);
    if (x == y) return;
    if (x > y) { int t = x; x = y; y = t; }
    if (atomicCAS(label + y, y, x) == y) return;
  }
}

// Grid-wide ordered scan helper: block b owns [b*C, min(n,(b+1)*C)).
__device__ __forceinline__ void chunk_of(const KParams& kp, long long n, long long& b, long long& e) {
  const long long C = (n + kp.nblocks - 1) / kp.nblocks;
  b = min(n, (long long)blockIdx.x * C);
  e = min(n, b + C);
}

static __device__ void cc_phase(const KParams& kp, const MainArgs& a, const SmemPtrs& sm, ShState& sh) {
  const CompWS& w = a.w;
  const int n = a.n;
  const int G = gthreads(kp);
  const int lane = threadIdx.x & 31;
  const int gwarp = gtid() >> 5, nwarps = G >> 5;
  // init
  for (int v = gtid(); v < n; v += G) {
    const bool unv = (uint32_t)(ld_relaxed_u64(kp.word + v) >> 32) == kInf;
    w.label[v] = unv ? v : -1;
    w.ckey[v] = kKeyMax;
    w.csize[v] = 0;
  }
  if (gtid() == 0) { w.gctl[1] = 0; w.gctl[2] = 0; w.gctl[3] = -1; }
  grid_barrier(kp);
  // Sampling (Afforest, Sutton et al. IPDPS'18): hook every unvisited node to
  // its first kSample unvisited neighbours, so that the giant component is
  // (mostly) one tree before the full pass.  Its members -- flagged in csize,
  // a snapshot that stays fixed during the full pass -- then skip their rows;
  // an edge between a member and a non-member is hooked from the non-member
  // side, an edge between two members is already inside one tree.
#ifndef RCM_CC_SAMPLE
#define RCM_CC_SAMPLE 4
#endif
  constexpr int kSample = RCM_CC_SAMPLE;
  for (int u = gtid(); u < n; u += G) {
    if (ld_cg_s32(w.label + u) < 0) continue;
    const int rs = __ldg(kp.row_ptr + u), re = __ldg(kp.row_ptr + u + 1);
    int k = 0;
    for (int e = rs, ee = min(re, rs + 4 * kSample); e < ee && k < kSample; ++e) {   // bounded scan (hub rows)
      const int c = __ldg(kp.col_idx + e);
      if (c != u && ld_cg_s32(w.label + c) >= 0) { uf_unite(w.label, u, c); ++k; }
    }
  }
  grid_barrier(kp);
  if (blockIdx.x == 0) {   // giant = most frequent root among kThreads spread samples
    int32_t* s_root = reinterpret_cast<int32_t*>(sm_cand(kp));
    unsigned long long* s_best = reinterpret_cast<unsigned long long*>(s_root + kThreads);
    const int v = (int)(((long long)threadIdx.x * n) / kThreads);
    const int r = ld_cg_s32(w.label + v) >= 0 ? uf_find(w.label, v) : -1;
    s_root[threadIdx.x] = r;
    if (threadIdx.x == 0) *s_best = 0;
    __syncthreads();
    int cnt = 0;
    for (int i = 0; i < kThreads; ++i) cnt += s_root[i] == r;
    if (r >= 0) atomicMax(s_best, ((unsigned long long)cnt << 32) | (uint32_t)r);
    __syncthreads();
    if (threadIdx.x == 0 && *s_best) w.gctl[3] = (int)(uint32_t)*s_best;
  }
  grid_barrier(kp);
  const int giant = ld_cg_s32(w.gctl + 3);
  for (int v = gtid(); v < n; v += G) {   // compress + member snapshot
    if (ld_cg_s32(w.label + v) < 0) continue;
    const int r = uf_find(w.label, v);
    w.label[v] = r;
    w.csize[v] = r == giant;
  }
  grid_barrier(kp);
  // hook every remaining edge (c < u: the pattern is symmetric; or c a member)
  // -- thread / warp / block per row by degree so that hub rows are split
  // across many threads; rows above 32 entries are listed during the thread
  // pass (front0 / front1)
  for (int u = gtid(); u < n; u += G) {
    const int rs = __ldg(kp.row_ptr + u), re = __ldg(kp.row_ptr + u + 1);
    if (ld_cg_s32(w.label + u) < 0 || __ldcg(w.csize + u)) continue;
    if (re - rs > 32) {
      if (re - rs > 4096) w.front1[atomicAdd(w.gctl + 2, 1)] = u;
      else w.front0[atomicAdd(w.gctl + 1, 1)] = u;
      continue;
    }
    for (int e = rs; e < re; ++e) {
      const int c = __ldg(kp.col_idx + e);
      if ((c < u || __ldcg(w.csize + c)) && ld_cg_s32(w.label + c) >= 0) uf_unite(w.label, u, c);
    }
  }
  grid_barrier(kp);
  const int nmed = ld_cg_s32(w.gctl + 1), nbig = ld_cg_s32(w.gctl + 2);
  for (int i = gwarp; i < nmed; i += nwarps) {
    const int u = __ldcg(w.front0 + i);
    const int rs = __ldg(kp.row_ptr + u), re = __ldg(kp.row_ptr + u + 1);
    for (int e = rs + lane; e < re; e += 32) {
      const int c = __ldg(kp.col_idx + e);
      if ((c < u || __ldcg(w.csize + c)) && ld_cg_s32(w.label + c) >= 0) uf_unite(w.label, u, c);
    }
  }
  for (int i = blockIdx.x; i < nbig; i += kp.nblocks) {
    const int u = __ldcg(w.front1 + i);
    const int rs = __ldg(kp.row_ptr + u), re = __ldg(kp.row_ptr + u + 1);
    for (int e = rs + threadIdx.x; e < re; e += kThreads) {
      const int c = __ldg(kp.col_idx + e);
      if ((c < u || __ldcg(w.csize + c)) && ld_cg_s32(w.label + c) >= 0) uf_unite(w.label, u, c);
    }
  }
  grid_barrier(kp);
  for (int v = gtid(); v < n; v += G) w.csize[v] = 0;   // member flags -> sizes
  grid_barrier(kp);
  // compress; per root: minimum (valence, id) member and size
  // warp-aggregated per root: the giant component's nodes would otherwise all
  // hit one address with atomics
  for (int base = blockIdx.x * kThreads; base < n; base += G) {
    const int v = base + threadIdx.x;
    int r = -1;
    unsigned long long k = kKeyMax;
    if (v < n && ld_cg_s32(w.label + v) >= 0) {
      r = uf_find(w.label, v);
      w.label[v] = r;
      k = ((ld_relaxed_u64(kp.word + v) & 0xffffffffull) << 32) | (uint32_t)v;
    }
    const unsigned peers = __match_any_sync(0xffffffffu, r);
    unsigned long long m;
    int cnt;
    {   // reduce over the peer group (lanes with the same root)
      unsigned rest = peers;
      unsigned long long mm = kKeyMax;
      while (rest) {
        const int l = __ffs(rest) - 1;
        rest &= rest - 1;
        const unsigned long long x = __shfl_sync(peers, k, l);
        mm = x < mm ? x : mm;
      }
      m = mm;
      cnt = __popc(peers);
    }
    if (r >= 0 && lane == __ffs(peers) - 1) {
      atomicMin(w.ckey + r, m);
      atomicAdd(w.csize + r, cnt);
    }
  }
  grid_barrier(kp);
  // ordered compaction of component representatives (the min (valence, id)
  // member): the list comes out in id order, so a stable sort on the valence
  // bits alone yields (valence, id) order (C-6)
  long long cb, ce;
  chunk_of(kp, n, cb, ce);
  {
    int cnt = 0;
    // isolated nodes (valence 0, C-2) are components of their own whose C-6 key
    // (0, id) precedes every other: they take the first positions in id order
    // directly and stay out of the sort (C4: 2.18 M of its 2.19 M components)
    int iso = 0;
    for (long long v = cb + threadIdx.x; v < ce; v += kThreads) {
      const int r = __ldcg(w.label + v);
      if (r >= 0) {
        const unsigned long long k = __ldcg(w.ckey + r);
        const bool rep = (int)(uint32_t)k == (int)v;
        cnt += rep && (k >> 32) != 0;
        iso += rep && (k >> 32) == 0;
      }
    }
    cnt = block_reduce_sum<int32_t>(cnt, sh.wtmp32);
    iso = block_reduce_sum<int32_t>(iso, sh.wtmp32);
    if (threadIdx.x == 0) { w.hist[blockIdx.x] = cnt; w.hist[2 * kp.nblocks + blockIdx.x] = iso; }
  }
  grid_barrier(kp);
  if (blockIdx.x == 0) {
    const int tot = block_scan_partials<int32_t>(w.hist, w.hist + kp.nblocks, kp.nblocks, sh.wtmp32);
    const int niso = block_scan_partials<int32_t>(w.hist + 2 * kp.nblocks, w.hist + 3 * kp.nblocks, kp.nblocks,
                                                  sh.wtmp32);
    if (threadIdx.x == 0) { w.sctl[0] = tot; w.sctl[1] = 0; w.sctl[4] = niso; }
  }
  grid_barrier(kp);
  {
    int run = __ldcg(w.hist + kp.nblocks + blockIdx.x);
    int irun = ld_cg_s32(&kp.ctl->chain_total) + __ldcg(w.hist + 3 * kp.nblocks + blockIdx.x);
    for (long long base = cb; base < ce; base += kThreads) {
      const long long v = base + threadIdx.x;
      int r = -1, f = 0, fi = 0;
      unsigned long long k = 0;
      if (v < ce) {
        r = __ldcg(w.label + v);
        if (r >= 0) {
          k = __ldcg(w.ckey + r);
          const bool rep = (int)(uint32_t)k == (int)v;
          f = rep && (k >> 32) != 0;
          fi = rep && (k >> 32) == 0;
        }
      }
      int tot, itot;
      const int ex = block_exclusive_scan<int32_t>(f, sh.wtmp32, tot);
      const int iex = block_exclusive_scan<int32_t>(fi, sh.wtmp32, itot);
      if (f) {
        w.keys0[run + ex] = ((k >> 32) << a.idbits) | (k & 0xffffffffull);
        w.vals0[run + ex] = r;
      }
      if (fi) {   // an isolated node: its position now
        const int pos = irun + iex;
        kp.o[pos] = (int)v;
        kp.perm[n - 1 - pos] = (int)v;
        if (kp.iperm) kp.iperm[v] = n - 1 - pos;
      }
      run += tot;
      irun += itot;
    }
    if (kp.collect_stats) {
      const int mine = __ldcg(w.hist + 2 * kp.nblocks + blockIdx.x);
      if (threadIdx.x == 0 && mine) atomicAdd(&kp.stats->components, (unsigned long long)mine);
    }
  }
  grid_barrier(kp);
  stamp(kp, 5);
  int maxdeg = ld_cg_s32(&kp.ctl->maxdeg);
  int dbits = 0;
  while (dbits < 32 && (1ll << dbits) <= maxdeg) ++dbits;
  radix_sort_phase(kp, w, a.idbits, a.idbits + dbits, reinterpret_cast<int32_t*>(sm_cand(kp)), sh);
  // offsets: exclusive scan of sizes in key order, after the chain-first total
  const int count = ld_cg_s32(w.sctl);
  const int cur = ld_cg_s32(w.sctl + 1);
  const int32_t* vals = cur ? w.vals1 : w.vals0;
  chunk_of(kp, count, cb, ce);
  {
    long long s = 0;
    for (long long i = cb + threadIdx.x; i < ce; i += kThreads) s += __ldcg(w.csize + __ldcg(vals + i));
    s = block_reduce_sum<long long>(s, sh.wtmpll);
    if (threadIdx.x == 0) w.offs[blockIdx.x] = s;   // offs[] as per-block scratch first
  }
  grid_barrier(kp);
  if (blockIdx.x == 0) {
    // block bases (counts < 2^31)
    block_scan_partials<long long, int32_t>(w.offs, w.hist, kp.nblocks, sh.wtmpll);
    if (threadIdx.x == 0) {
      kp.ctl->n_comp = count;
      kp.ctl->n_chain = 0;
      kp.ctl->n_solo = 0;
      kp.ctl->solo_next = 0;
    }
  }
  grid_barrier(kp);
  // problems: singletons written directly, small ones to solo, large to chains
  Problem* chains = const_cast<Problem*>(kp.chains);
  Problem* solos = const_cast<Problem*>(kp.solos);
  int singles = 0;
  {
    long long run = (long long)ld_cg_s32(&kp.ctl->chain_total) + ld_cg_s32(w.sctl + 4) + __ldcg(w.hist + blockIdx.x);
    for (long long base = cb; base < ce; base += kThreads) {
      const long long i = base + threadIdx.x;
      int root = -1, size = 0;
      if (i < ce) { root = __ldcg(vals + i); size = __ldcg(w.csize + root); }
      long long tot;
      const long long ex = block_exclusive_scan<long long>((long long)size, sh.wtmpll, tot);
      if (i < ce) {
        const int seed = (int)(uint32_t)__ldcg(w.ckey + root);
        const int pos = (int)(run + ex);
        if (size == 1) {
          kp.o[pos] = seed;
          kp.perm[n - 1 - pos] = seed;
          if (kp.iperm) kp.iperm[seed] = n - 1 - pos;
          ++singles;
        } else {
          Problem P;
          P.node_base = 0; P.rp_base = 0; P.ci_base = 0; P.o_base = 0; P.perm_base = 0;
          P.mat_n = n; P.pos0 = pos; P.size = size; P.seed = seed; P.pad = 0;
          P.flags = a.mode == RCM_START_PSEUDO_PERIPHERAL ? 2 : 0;
          if (a.thr > 0 && size <= a.thr) {
            const int j = atomicAdd(&kp.ctl->n_solo, 1);
            if (j < a.prob_cap) solos[j] = P; else latch_error(kp.ctl, ST_CAPACITY);
          } else {
            const int j = atomicAdd(&kp.ctl->n_chain, 1);
            if (j < a.prob_cap) chains[j] = P; else latch_error(kp.ctl, ST_CAPACITY);
          }
        }
      }
      run += tot;
    }
  }
  if (kp.collect_stats) {
    singles = block_reduce_sum<int32_t>(singles, sh.wtmp32);
    if (threadIdx.x == 0 && singles) atomicAdd(&kp.stats->components, (unsigned long long)singles);
  }
  grid_barrier(kp);
  stamp(kp, 6);
}

// =============================================== pseudo-peripheral finder
// P:L365-375 with reading C-5: BFS from r; x = min (valence, id) node of the
// last level; BFS from x; continue while the level count grows; return x.
// Level-synchronous BFS, frontier queues in HBM, grid barrier per level.
static __device__ int gl_bfs(const KParams& kp, const CompWS& w, int n, int r, ShState& sh) {
  const int G = gthreads(kp);
  const int lane = threadIdx.x & 31;
  const int gwarp = gtid() >> 5, nwarps = G >> 5;
  constexpr int kU = 4;          // edges per lane in flight
  constexpr int kChunk = 1024;   // rows longer than this are split into kChunk-edge items, one warp each
  // per-level counters rotate over three slots (next-frontier size, long-row
  // items at gctl[8 + i], [16 + i]): level L counts into slot L % 3 and clears
  // slot (L + 1) % 3, last read before the barrier of level L - 1 -- one grid
  // barrier per level (two when the level has rows above kChunk)
  int32_t* cnt = w.gctl + 8;
  int32_t* cbig = w.gctl + 16;
  for (int v = gtid(); v < n; v += G) w.lev[v] = -1;
  grid_barrier(kp);
  if (gtid() == 0) {
    w.lev[r] = 0;
    w.front0[0] = r;
    cnt[0] = cbig[0] = 0;
    w.gkey[0] = kKeyMax;
  }
  grid_barrier(kp);
  int32_t* cur = w.front0;
  int32_t* nxt = w.front1;
  int ncur = 1, level = 0;
  for (;;) {
    const int sl = level % 3;
    if (gtid() == 0) { const int s1 = (level + 1) % 3; cnt[s1] = 0; cbig[s1] = 0; }
    // the kU column loads of a lane, then kU level loads, then the CASes; the
    // newly reached nodes are appended with one atomicAdd per warp and round
    auto visit = [&](const int (&c)[kU]) {
      int lv[kU];
#pragma unroll
      for (int u = 0; u < kU; ++u) lv[u] = c[u] >= 0 ? ld_cg_s32(w.lev + c[u]) : 0;
      bool nw[kU];
      int k = 0;
#pragma unroll
      for (int u = 0; u < kU; ++u) {
        nw[u] = c[u] >= 0 && lv[u] < 0 && atomicCAS(w.lev + c[u], -1, level + 1) == -1;
        k += nw[u];
      }
      const int incl = warp_incl_scan(k);
      const int tot = __shfl_sync(kFull, incl, 31);
      if (tot) {
        int base = 0;
        if (lane == 31) base = atomicAdd(cnt + sl, tot);
        base = __shfl_sync(kFull, base, 31) + incl - k;
#pragma unroll
        for (int u = 0; u < kU; ++u)
          if (nw[u]) nxt[base++] = c[u];
      }
    };
    // frontier nodes per warp: spread a narrow level over all warps
    const int per = min(32, max(1, (ncur + nwarps - 1) / nwarps));
    for (int i0 = gwarp * per; i0 < ncur; i0 += nwarps * per) {
      const int i = i0 + lane;
      int p = -1, rs = 0, d = 0;
      if (lane < per && i < ncur) {
        p = __ldcg(cur + i);
        rs = __ldg(kp.row_ptr + p);
        d = __ldg(kp.row_ptr + p + 1) - rs;
      }
      const int nit = d > kChunk ? (d + kChunk - 1) / kChunk : 0;   // long row -> items
      const int iincl = warp_incl_scan(nit);
      const int itot = __shfl_sync(kFull, iincl, 31);
      if (itot) {
        int base = 0;
        if (lane == 31) base = atomicAdd(cbig + sl, itot);
        base = __shfl_sync(kFull, base, 31);
        if (base + itot > w.cap) {
          if (lane == 0) latch_error(kp.ctl, ST_CAPACITY);
        } else {
          for (int k = 0; k < nit; ++k) {
            w.vals0[base + iincl - nit + k] = p;
            w.vals1[base + iincl - nit + k] = k;
          }
        }
      }
      WarpRows R;
      R.init(rs, nit ? 0 : d);
      for (int b = 0; b < R.E; b += 32 * kU) {
        int c[kU], j[kU];
        R.cols<kU>(kp.col_idx, b, c, j);
        visit(c);
      }
    }
    grid_barrier(kp);
    // items past a latched capacity error were never written: none are read then
    const int nbig = ld_cg_s32(&kp.ctl->status) ? 0 : ld_cg_s32(cbig + sl);
    if (nbig) {   // uniform: read after the barrier
      for (int it = gwarp; it < nbig; it += nwarps) {
        const int p = __ldcg(w.vals0 + it), k = __ldcg(w.vals1 + it);
        const int rs = __ldg(kp.row_ptr + p) + k * kChunk;
        const int re = min(__ldg(kp.row_ptr + p + 1), rs + kChunk);
        for (int b = rs; b < re; b += 32 * kU) {
          int c[kU];
#pragma unroll
          for (int u = 0; u < kU; ++u) {
            const int e = b + u * 32 + lane;
            c[u] = e < re ? __ldg(kp.col_idx + e) : -1;
          }
          visit(c);
        }
      }
      grid_barrier(kp);
    }
    const int nn = ld_cg_s32(cnt + sl);
    if (nn == 0) break;
    ++level;
    int32_t* t = cur; cur = nxt; nxt = t;
    ncur = nn;
  }
  unsigned long long best = kKeyMax;
  for (int i = gtid(); i < ncur; i += G) {
    const int v = __ldcg(cur + i);
    const unsigned long long k = ((ld_relaxed_u64(kp.word + v) & 0xffffffffull) << 32) | (uint32_t)v;
    best = k < best ? k : best;
  }
  best = warp_min_u64(best);
  if ((threadIdx.x & 31) == 0 && best != kKeyMax) atomicMin(w.gkey, best);
  grid_barrier(kp);
  return level + 1;
}

// Not inlined: with the warp-flattened BFS inlined, k_main<2,0>'s register
// allocation moved spills into the chain's hot loop (ncu local-memory sectors
// on C2 0.36 M -> 9.1 M; noinline: 4.2 M, C2 3.44 -> 3.40 ms, tools/gpu_spill.sh).
static __device__ __noinline__ int gl_phase(const KParams& kp, const CompWS& w, int n, int r, ShState& sh) {
  int nl = gl_bfs(kp, w, n, r, sh);
  for (;;) {
    const int x = (int)(uint32_t)__ldcg(w.gkey);
    const int nx = gl_bfs(kp, w, n, x, sh);
    if (nx > nl) { nl = nx; continue; }
    return x;   // "use the last node"
  }
}

}  // namespace rcm
