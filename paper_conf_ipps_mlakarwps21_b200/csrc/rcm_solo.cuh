// rcm_solo.cuh -- the batched / small-graph path: one matrix (or one small
// graph) per thread block, many blocks per SM, no inter-block signalling.
//
// Inside one block the batches of the paper's method (Alg. 5) run
// one after the other, so the speculation / rediscovery / chain of the
// multi-block path is not needed: when a batch starts, every earlier batch is
// complete.  What remains of a batch is:
//   parents    the next nP <= B_s nodes of the CM order o, whose summed
//              valence fits the T edge slots; held with their row
//              start and valence in a shared-memory ring, so a batch does not
//              re-read o[] or row_ptr for its parents;
//   discover   every edge (p, c) of the batch with c not yet placed (a
//              shared-memory VISITED BITMAP, one bit per node of the matrix,
//              replaces the owner-word prefilter of the multi-block path)
//              inserts (c, edge slot e) into a shared-memory CLAIM TABLE that
//              keeps, per child c, the minimum edge slot.  Edge slots are laid
//              out parent by parent, so the minimum slot is the earliest parent
//              in o (Alg. 1 ln 8-12: the first parent to see c claims it,
//              P:L202-212) and, within one parent, the first of duplicate
//              entries (C-8).  The child's valence r[c+1]-r[c] and row
//              start are loaded while the claims are inserted;
//   sort       the winners of each parent, by (valence, id) (C-1);
//   output     at the next positions of o, written reversed into perm
//              and appended to the ring as future parents.
// There is no global atomic and no owner word: per batch two dependent global
// round trips remain (the batch's columns, then the children's row_ptr).
//
// Seeds follow C-6 (min (valence, id) over the unplaced nodes, found with a
// cursor that only moves forward because that minimum never decreases), FIXED
// starts, and the GL finder (C-5) by a block-level BFS.  A parent
// whose valence exceeds T is processed in chunks of T edges; its
// children are sorted in plan-owned HBM scratch by a block radix sort.
// Matrices above the shared-memory bitmap capacity keep their bitmaps in HBM
// (same code, global atomics).  DESIGN.md §2.6.
#pragma once
#include "rcm_batch.cuh"
#include "rcm_expand.cuh"

// Read-only CSR loads: through the non-coherent path from HBM, or plain loads
// when the whole CSR of a small graph was staged in shared memory (k_solo_sm).
#ifdef RCM_SOLO_SMEM_CSR
#define SO_LD(p) (*(p))
#define SO_LDS(p) (*(p))
#else
#define SO_LD(p) __ldg(p)
// a parent's row is read once: streaming load (evict-first), so the
// children's row_ptr lines keep their place in L2 (C5 31.3 -> 30.2 ms)
#define SO_LDS(p) __ldcs(p)
#endif

namespace rcm {

#ifndef RCM_SOLO_NT
#define RCM_SOLO_NT 256
#endif
#ifndef RCM_SOLO_U
#define RCM_SOLO_U 3
#endif
#ifndef RCM_SOLO_Q
#define RCM_SOLO_Q 256
#endif
#ifndef RCM_SOLO_PEND
#define RCM_SOLO_PEND 1
#endif
constexpr bool kSoloPend = RCM_SOLO_PEND != 0;     // ring overflow kept as (row start, valence)
constexpr int kSoloNT = RCM_SOLO_NT;                // threads per block
constexpr int kSoloNW = kSoloNT / 32;
constexpr int kSoloU = RCM_SOLO_U;                  // edge slots per thread per batch
constexpr int kSoloT = kSoloNT * kSoloU;            // T: edge slots of a batch
// claim-table slots: the power of two >= T (a batch has at most T distinct
// children, so linear probing always finds a free slot; load <= T / H)
constexpr int kSoloHBits = 32 - __builtin_clz((unsigned)kSoloT - 1u);
constexpr int kSoloH = 1 << kSoloHBits;
constexpr int kSoloQ = RCM_SOLO_Q;                  // ring of pending parents (power of two)
constexpr int kSoloNMax = (1 << 17) - 1;            // shared-memory bitmap capacity (nodes)
constexpr int kSoloVisW = (kSoloNMax >> 5) + 1;     // bitmap words
static_assert(kSoloT <= 32767 && (kSoloH & (kSoloH - 1)) == 0 && kSoloHBits <= 15, "claim table packing");
static_assert((kSoloQ & (kSoloQ - 1)) == 0 && kSoloQ >= 256, "ring size");
constexpr uint32_t kEmpty32 = 0xFFFFFFFFu;          // (c:17 | e:15) never reaches it: c < 2^17 - 1
constexpr int kSoloGrp = 64;                        // output-group ring (stats only)

// Arguments of the solo kernels (one launch of k_solo_order + one of k_solo).
struct SoloArgs {
  const int32_t* row_ptr;     // batched: per matrix n_k + 1 local offsets, concatenated
  const int32_t* col_idx;     // local column ids
  int32_t* perm;              // output (new -> old, local ids)
  int32_t* iperm;             // nullable (single graph only)
  const int64_t* node_off;    // nullable: single graph of n nodes / nnz entries
  const int64_t* nnz_off;
  const int32_t* starts;      // nullable: per-matrix FIXED starts
  int32_t* order;             // matrix processing order (largest first)
  uint32_t* gvis;             // HBM bitmaps for matrices above kSoloNMax: 2 x gvis_words
  long long gvis_words;
  unsigned long long* spill;  // oversize scratch: keys [0, cap), radix temp [cap, 2 cap)
  int2* pend;                 // per output position: (row start, valence) of a node that did
                              // not fit the ring, read back coalesced when it becomes a parent
                              // (valence -1: not recorded, re-read row_ptr)
  long long spill_cap;
  Ctl* ctl;
  Stats* stats;
  int num_mats;
  int n;                      // single graph
  long long nnz;
  int mode;
  int start;                  // single graph FIXED start
  int validate;
  int collect_stats;
  int flags;
  int BS;                     // B_s (<= kSoloNT)
  int chunk;                  // 0: a call's first launch (resets status, stats, timers);
                              // > 0: a later chunk of rcm_reorder_batched_host
};

// Shared-memory layout (bytes), dynamic.
constexpr size_t kSoOffVis = 0;
constexpr size_t kSoOffRing = kSoOffVis + 4 * (size_t)kSoloVisW;
constexpr size_t kSoOffPar = kSoOffRing + 12 * (size_t)kSoloQ;                 // 3 int arrays of kSoloNT + 1
constexpr size_t kSoOffLpof = kSoOffPar + 3 * 4 * (size_t)(kSoloNT + 1) + 4;             // u16 per edge slot
constexpr size_t kSoOffFlp = kSoOffLpof + 2 * (size_t)kSoloT;                            // u16 per thread
constexpr size_t kSoOffCand = (kSoOffFlp + 2 * (size_t)kSoloNT + 15) & ~size_t(15);
constexpr size_t kSoOffHash = kSoOffCand + 8 * (size_t)kSoloT;
constexpr size_t kSoOffRsv = kSoOffHash + 4 * (size_t)kSoloH;                  // big matrices: 8 B entries over hash+rsv
constexpr size_t kSoOffRdeg = kSoOffRsv + 4 * (size_t)kSoloH;                 // valence per table slot
constexpr size_t kSoloSmem = kSoOffRdeg + 4 * (size_t)kSoloH;
static_assert(kSoloSmem - kSoOffRing >= 4 * (size_t)kSoloVisW, "GL bitmap overlays ring..rdeg");

struct SoloSh {
  int32_t wtmp[kSoloNW + 1];
  int32_t wscan[2][kSoloNW];   // one-barrier scans alternate between the two buffers
  int32_t nbig[2];             // segments above 16 children, per batch parity
  long long wtmpll[kSoloNW + 1];
  unsigned long long wtmp64[kSoloNW + 1];
  int32_t k, pos, written, rhi, nP, E, cnt, tail, found, big_n;
  int32_t cur_deg, cur_id, bad;
  unsigned long long minkey;
  long long st_exec, st_comp, st_over, st_claim, st_comb;
  // start positions of the pending output groups (one per batch), for the
  // work-aggregation counter: a batch whose parents span several groups
  // combines the outputs of several earlier batches
  int32_t grp[kSoloGrp];
  int32_t grp_h, grp_t;
};

// Matrix geometry.
struct SoloMat {
  const int32_t* rp;   // local row_ptr (n + 1)
  const int32_t* col;  // local columns (add rp values)
  int32_t* perm;       // local perm (n)
  long long node_base;
  int n;
  int nnz;
  uint32_t* vis;       // placed bitmap (smem or HBM)
  uint32_t* bvis;      // GL BFS bitmap (smem overlay or HBM)
  int b0;              // bit of local node 0 in the first word (HBM bitmaps are packed
                       // over all nodes, so neighbouring matrices may share a word)
  bool gmem;           // bitmaps in HBM
};

__device__ __forceinline__ uint8_t* so_base() { return rcm_dsm; }
__device__ __forceinline__ int32_t* so_ring_v() { return reinterpret_cast<int32_t*>(so_base() + kSoOffRing); }
__device__ __forceinline__ int32_t* so_ring_rs() { return so_ring_v() + kSoloQ; }
__device__ __forceinline__ int32_t* so_ring_d() { return so_ring_v() + 2 * kSoloQ; }
// per parent of the batch: row start, first edge slot (+ end), children filed
__device__ __forceinline__ int32_t* so_p_rs() { return reinterpret_cast<int32_t*>(so_base() + kSoOffPar); }
__device__ __forceinline__ int32_t* so_p_eo() { return so_p_rs() + (kSoloNT + 1); }
__device__ __forceinline__ int32_t* so_p_cnt() { return so_p_rs() + 2 * (kSoloNT + 1); }
__device__ __forceinline__ uint16_t* so_lpof() { return reinterpret_cast<uint16_t*>(so_base() + kSoOffLpof); }
// segments above 16 children (sort phase), over the slot->parent table, which
// is dead after the file phase
__device__ __forceinline__ int32_t* so_big_list() { return reinterpret_cast<int32_t*>(so_base() + kSoOffLpof); }
static_assert(2 * kSoloT >= 4 * kSoloNT || kSoloU < 2, "big-segment list overlays lpof");
__device__ __forceinline__ uint16_t* so_flp() { return reinterpret_cast<uint16_t*>(so_base() + kSoOffFlp); }
__device__ __forceinline__ unsigned long long* so_cand() {
  return reinterpret_cast<unsigned long long*>(so_base() + kSoOffCand);
}
__device__ __forceinline__ uint32_t* so_hash() { return reinterpret_cast<uint32_t*>(so_base() + kSoOffHash); }
__device__ __forceinline__ unsigned long long* so_hash64() {
  return reinterpret_cast<unsigned long long*>(so_base() + kSoOffHash);
}
__device__ __forceinline__ int32_t* so_rsv() { return reinterpret_cast<int32_t*>(so_base() + kSoOffRsv); }
__device__ __forceinline__ int32_t* so_rdeg() { return reinterpret_cast<int32_t*>(so_base() + kSoOffRdeg); }

// ------------------------------------------------------------- block helpers
template <typename T>
__device__ __forceinline__ T so_scan(T v, T* wtmp, T& total) {   // exclusive, kSoloNT threads
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  T x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T y = __shfl_up_sync(0xffffffffu, x, d);
    if (lane >= d) x += y;
  }
  if (lane == 31) wtmp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T w = lane < kSoloNW ? wtmp[lane] : T(0);
    T s = w;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      T y = __shfl_up_sync(0xffffffffu, s, d);
      if (lane >= d) s += y;
    }
    if (lane < kSoloNW) wtmp[lane] = s - w;
    if (lane == kSoloNW - 1) wtmp[kSoloNW] = s;
  }
  __syncthreads();
  const T r = wtmp[wid] + x - v;
  total = wtmp[kSoloNW];
  __syncthreads();
  return r;
}

__device__ __forceinline__ unsigned long long so_min_u64(unsigned long long v, SoloSh& sh) {
  v = warp_min_u64(v);
  if ((threadIdx.x & 31) == 0) sh.wtmp64[threadIdx.x >> 5] = v;
  __syncthreads();
  if (threadIdx.x < 32) {
    unsigned long long b = threadIdx.x < kSoloNW ? sh.wtmp64[threadIdx.x] : kKeyMax;
    b = warp_min_u64(b);
    if (threadIdx.x == 0) sh.minkey = b;
  }
  __syncthreads();
  const unsigned long long r = sh.minkey;
  __syncthreads();
  return r;
}

__device__ __forceinline__ unsigned long long so_or_u64(unsigned long long v, SoloSh& sh) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) v |= __shfl_xor_sync(0xffffffffu, v, d);
  if ((threadIdx.x & 31) == 0) sh.wtmp64[threadIdx.x >> 5] = v;
  __syncthreads();
  unsigned long long r = 0;
#pragma unroll
  for (int w = 0; w < kSoloNW; ++w) r |= sh.wtmp64[w];
  __syncthreads();
  return r;
}

__device__ __forceinline__ bool so_test(const SoloMat& M, int v) {
  v += M.b0;
  const uint32_t w = M.gmem ? __ldcg(M.vis + (v >> 5)) : M.vis[v >> 5];
  return (w >> (v & 31)) & 1u;
}
template <bool kBig>
__device__ __forceinline__ bool so_placed(const SoloMat& M, int v) {
  uint32_t w;
  if constexpr (kBig) { v += M.b0; w = __ldcg(M.vis + (v >> 5)); }
  else w = reinterpret_cast<const uint32_t*>(so_base() + kSoOffVis)[v >> 5];
  return (w >> (v & 31)) & 1u;
}
__device__ __forceinline__ void so_set(const SoloMat& M, uint32_t* bits, int v) {
  v += M.b0;
  atomicOr(bits + (v >> 5), 1u << (v & 31));
}
// placed-bit set on the hot path: the shared-memory bitmap addressed as shared
// (ATOMS) for small matrices, the HBM bitmap otherwise
template <bool kBig>
__device__ __forceinline__ void so_place(const SoloMat& M, int v) {
  if constexpr (kBig) so_set(M, M.vis, v);
  else atomicOr(reinterpret_cast<uint32_t*>(so_base() + kSoOffVis) + (v >> 5), 1u << (v & 31));
}
// test-and-set, true if this call set the bit
__device__ __forceinline__ bool so_claim_bit(const SoloMat& M, uint32_t* bits, int v) {
  v += M.b0;
  const uint32_t b = 1u << (v & 31);
  return !(atomicOr(bits + (v >> 5), b) & b);
}

// Clear bits [b0, b0 + n): whole words with stores, a word shared with a
// neighbouring matrix (HBM bitmaps) with an atomic AND of this matrix's bits.
__device__ __forceinline__ void so_zero_bits(const SoloMat& M, uint32_t* bits) {
  const int lo = M.b0, hi = M.b0 + M.n;       // bit range
  const int w0 = lo >> 5, w1 = (hi - 1) >> 5;  // word range (inclusive)
  for (int i = w0 + threadIdx.x; i <= w1; i += kSoloNT) {
    const int bl = max(lo, i << 5) - (i << 5), bh = min(hi, (i << 5) + 32) - (i << 5);   // [bl, bh) in word i
    if (bl == 0 && bh == 32) bits[i] = 0u;
    else atomicAnd(bits + i, ~((bh == 32 ? 0xffffffffu : ((1u << bh) - 1u)) & ~((1u << bl) - 1u)));
  }
}

__device__ __forceinline__ uint32_t so_hslot(uint32_t c) { return (c * 2654435761u) >> (32 - kSoloHBits); }

// Insert claim (c, e) into the table: per child the minimum edge slot (small
// matrices: one 32-bit word c:17 | e:15; large: c:32 | e:32).  Returns the
// slot; *ins = this call created the entry (exactly one claimer per child).
template <bool kBig>
__device__ __forceinline__ int so_claim(uint32_t c, uint32_t e, bool* ins) {
  uint32_t s = so_hslot(c);
  if constexpr (!kBig) {
    volatile uint32_t* h = so_hash();
    const uint32_t want = (c << 15) | e;
    for (;;) {
      uint32_t cur = h[s];
      if (cur == kEmpty32) {
        cur = atomicCAS(const_cast<uint32_t*>(h) + s, kEmpty32, want);
        if (cur == kEmpty32) { *ins = true; return (int)s; }
      }
      if ((cur >> 15) == c) { atomicMin(const_cast<uint32_t*>(h) + s, want); *ins = false; return (int)s; }
      s = (s + 1) & (kSoloH - 1);
    }
  } else {
    volatile unsigned long long* h = so_hash64();
    const unsigned long long want = ((unsigned long long)c << 32) | e;
    for (;;) {
      unsigned long long cur = h[s];
      if (cur == kKeyMax) {
        cur = atomicCAS(const_cast<unsigned long long*>(h) + s, kKeyMax, want);
        if (cur == kKeyMax) { *ins = true; return (int)s; }
      }
      if ((uint32_t)(cur >> 32) == c) {
        atomicMin(const_cast<unsigned long long*>(h) + s, want);
        *ins = false;
        return (int)s;
      }
      s = (s + 1) & (kSoloH - 1);
    }
  }
}
// Winning (minimum) edge slot of the child in table slot s.
template <bool kBig>
__device__ __forceinline__ int so_winner(int s) {
  if constexpr (!kBig) return (int)(so_hash()[s] & 0x7fffu);
  else return (int)(uint32_t)so_hash64()[s];
}
// Local parent of edge slot e: the largest lp with p_eo[lp] <= e.
__device__ __forceinline__ int so_find_lp(int e, int nP) {
  const int32_t* eo = so_p_eo();
  int lo = 0, hi = nP - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (eo[mid] <= e) lo = mid; else hi = mid - 1;
  }
  return lo;
}
template <bool kBig>
__device__ __forceinline__ void so_unclaim(int s) {
  if constexpr (!kBig) so_hash()[s] = kEmpty32;
  else so_hash64()[s] = kKeyMax;
}

// Every claim-table slot empty (after the GL bitmap or the radix scratch
// overlaid the table).
template <bool kBig>
__device__ __forceinline__ void so_hash_reset() {
  if constexpr (!kBig) for (int i = threadIdx.x; i < kSoloH; i += kSoloNT) so_hash()[i] = kEmpty32;
  else for (int i = threadIdx.x; i < kSoloH; i += kSoloNT) so_hash64()[i] = kKeyMax;
  __syncthreads();
}

// Stable LSD radix sort (8-bit digits, constant digits skipped) of a[0..n) in
// HBM by one block, temp tmp[0..n).  Used for an oversize parent's children.
static __device__ void so_radix_sort_global(unsigned long long* a, unsigned long long* tmp, int n, SoloSh& sh) {
  if (n <= 1) return;
  int32_t* off = reinterpret_cast<int32_t*>(so_cand());       // 256 digit offsets
  int32_t* wcnt = off + 256;                                  // kSoloNW x 256
  const unsigned long long first = __ldcg(a);
  unsigned long long diff = 0;
  for (int i = threadIdx.x; i < n; i += kSoloNT) diff |= __ldcg(a + i) ^ first;
  diff = so_or_u64(diff, sh);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const unsigned lt = (1u << lane) - 1;
  unsigned long long* src = a;
  unsigned long long* dst = tmp;
  for (int shift = 0; shift < 64; shift += 8) {
    if (((diff >> shift) & 0xffull) == 0) continue;
    for (int i = threadIdx.x; i < 256; i += kSoloNT) off[i] = 0;
    __syncthreads();
    for (int i = threadIdx.x; i < n; i += kSoloNT) atomicAdd(&off[(__ldcg(src + i) >> shift) & 0xff], 1);
    __syncthreads();
    if (threadIdx.x < 32) {
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
    for (int base = 0; base < n; base += kSoloNT) {
      const int i = base + threadIdx.x;
      const bool valid = i < n;
      const unsigned long long k = valid ? __ldcg(src + i) : 0ull;
      const int d = valid ? (int)((k >> shift) & 0xff) : 256;
      const unsigned peers = __match_any_sync(0xffffffffu, d);
      const int rank = __popc(peers & lt);
      for (int j = threadIdx.x; j < kSoloNW * 256; j += kSoloNT) wcnt[j] = 0;
      __syncthreads();
      if (valid && rank == 0) wcnt[wid * 256 + d] = __popc(peers);
      __syncthreads();
      for (int dg = threadIdx.x; dg < 256; dg += kSoloNT) {
        int run = off[dg];
        for (int w = 0; w < kSoloNW; ++w) { const int c = wcnt[w * 256 + dg]; wcnt[w * 256 + dg] = run; run += c; }
        off[dg] = run;
      }
      __syncthreads();
      if (valid) dst[wcnt[wid * 256 + d] + rank] = k;
      __syncthreads();
    }
    unsigned long long* t = src; src = dst; dst = t;
  }
  if (src != a)
    for (int i = threadIdx.x; i < n; i += kSoloNT) a[i] = __ldcg(src + i);
  __syncthreads();
}

// --------------------------------------------------------------- seeds / GL
// Valence of local node v.
__device__ __forceinline__ int so_deg(const SoloMat& M, int v) { return SO_LD(M.rp + v + 1) - SO_LD(M.rp + v); }

// Block-level BFS over the (wholly unplaced) component of r for the GL finder:
// the queue lives in the not-yet-written part of perm, visited bits in M.bvis.
// Returns the number of levels; *minkey = min (valence, id) of the last level.
static __device__ int so_bfs(const SoloMat& M, int written, int r, unsigned long long* minkey, SoloSh& sh) {
  constexpr int kU = 4;                       // edges per lane in flight
  int32_t* q = M.perm;                        // entries [0, n - written) are free
  so_zero_bits(M, M.bvis);
  __syncthreads();
  if (threadIdx.x == 0) { q[0] = r; so_claim_bit(M, M.bvis, r); sh.tail = 1; }
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int head = 0, tail = 1, levels = 1;
  for (;;) {
    // warp-cooperative expansion: a warp takes up to 32 frontier nodes and
    // walks their rows as one flattened edge list (rcm_expand.cuh), kU column
    // loads per lane in flight; new nodes appended with one atomic per warp
    const int cnt = tail - head;
    const int per = min(32, max(1, (cnt + kSoloNW - 1) / kSoloNW));
    for (int i0 = wid * per; i0 < cnt; i0 += kSoloNW * per) {
      int rs = 0, d = 0;
      if (lane < per && i0 + lane < cnt) {
        const int p = __ldcg(q + head + i0 + lane);
        rs = SO_LD(M.rp + p);
        d = SO_LD(M.rp + p + 1) - rs;
      }
      const int incl = warp_incl_scan(d), excl = incl - d;
      const int E = __shfl_sync(kFull, incl, 31);
      for (int b = 0; b < E; b += 32 * kU) {
        int c[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
          const int e = b + u * 32 + lane;
          const int jj = warp_edge_lane(e, incl) & 31;
          const int r0 = __shfl_sync(kFull, rs, jj), x0 = __shfl_sync(kFull, excl, jj);
          c[u] = e < E ? SO_LD(M.col + r0 + (e - x0)) : -1;
        }
        int k = 0;
        bool nw[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) { nw[u] = c[u] >= 0 && so_claim_bit(M, M.bvis, c[u]); k += nw[u]; }
        const int ki = warp_incl_scan(k);
        const int kt = __shfl_sync(kFull, ki, 31);
        if (kt) {
          int base = 0;
          if (lane == 31) base = atomicAdd(&sh.tail, kt);
          base = __shfl_sync(kFull, base, 31) + ki - k;
#pragma unroll
          for (int u = 0; u < kU; ++u)
            if (nw[u]) q[base++] = c[u];
        }
      }
    }
    __syncthreads();
    const int nt = sh.tail;
    __syncthreads();
    if (nt == tail) break;
    head = tail;
    tail = nt;
    ++levels;
  }
  unsigned long long best = kKeyMax;
  for (int i = head + threadIdx.x; i < tail; i += kSoloNT) {
    const int v = __ldcg(q + i);
    const unsigned long long k = ((unsigned long long)(uint32_t)so_deg(M, v) << 32) | (uint32_t)v;
    best = k < best ? k : best;
  }
  *minkey = so_min_u64(best, sh);
  return levels;
}

// GL finder (C-5): BFS from r, next root = min (valence, id) of the
// last level, repeat while the level count grows, return the last root.
// Not inlined: keeps the warp-flattened BFS out of k_solo's register allocation.
static __device__ __noinline__ int so_gl(const SoloMat& M, int written, int r, SoloSh& sh) {
  unsigned long long key;
  int nl = so_bfs(M, written, r, &key, sh);
  int x = (int)(uint32_t)key;
  for (;;) {
    const int nx = so_bfs(M, written, x, &key, sh);
    if (nx <= nl) break;
    nl = nx;
    x = (int)(uint32_t)key;
  }
  if (!M.gmem) so_hash_reset<false>();   // the BFS bitmap overlaid the claim table
  return x;
}

// Next C-6 seed: min (valence, id) over the unplaced nodes.  The minimum never
// decreases as nodes get placed, so a cursor (cur_deg, cur_id) scans forward:
// first the ids after cur_id with valence cur_deg, then the next larger
// valence present.  O(n) per distinct valence, not per component.
static __device__ int so_next_seed(const SoloMat& M, SoloSh& sh) {
  for (;;) {
    const int d = sh.cur_deg;
    for (int base = sh.cur_id + 1; base < M.n; base += kSoloNT) {
      const int v = base + threadIdx.x;
      const bool f = v < M.n && !so_test(M, v) && so_deg(M, v) == d;
      if (threadIdx.x == 0) sh.found = 0x7fffffff;
      __syncthreads();
      if (f) atomicMin(&sh.found, v);
      __syncthreads();
      const int s = sh.found;
      __syncthreads();
      if (s != 0x7fffffff) {
        if (threadIdx.x == 0) sh.cur_id = s;
        __syncthreads();
        return s;
      }
    }
    unsigned long long best = kKeyMax;   // smallest valence above d among unplaced
    for (int v = threadIdx.x; v < M.n; v += kSoloNT) {
      if (so_test(M, v)) continue;
      const int dv = so_deg(M, v);
      if (dv > d) {
        const unsigned long long k = ((unsigned long long)(uint32_t)dv << 32) | (uint32_t)v;
        best = k < best ? k : best;
      }
    }
    best = so_min_u64(best, sh);
    if (best == kKeyMax) return -1;
    if (threadIdx.x == 0) { sh.cur_deg = (int)(best >> 32); sh.cur_id = (int)(uint32_t)best; }
    __syncthreads();
    return (int)(uint32_t)best;
  }
}

// Place a root at position q: perm, iperm, placed bit (thread 0) and the ring
// entry if the ring is contiguous up to q (rhi == q; every thread updates its
// copy of rhi).
__device__ __forceinline__ void so_place_root(const SoloArgs& a, const SoloMat& M, int s, int q, int& rhi) {
  if (threadIdx.x == 0) {
    M.perm[M.n - 1 - q] = s;
    if (a.iperm) a.iperm[M.node_base + s] = M.n - 1 - q;
    so_set(M, M.vis, s);
    if (rhi == q) {
      so_ring_v()[q & (kSoloQ - 1)] = s;
      so_ring_rs()[q & (kSoloQ - 1)] = SO_LD(M.rp + s);
      so_ring_d()[q & (kSoloQ - 1)] = so_deg(M, s);
    } else if (kSoloPend) {
      a.pend[M.node_base + q] = make_int2(0, -1);
    }
  }
  if (rhi == q) rhi = q + 1;
}

// ------------------------------------------------------------ validation
// validate >= 1: r[0] = 0, non-decreasing, r[n] = nnz, 0 <= col < n;
// validate == 2: every (u, c) has (c, u) (binary search in sorted rows, linear
// scan otherwise).  Returns true if the matrix is well formed.
static __device__ bool so_validate(const SoloArgs& a, const SoloMat& M, SoloSh& sh) {
  int bad = 0;
  if (threadIdx.x == 0) bad = (SO_LD(M.rp) != 0) || (SO_LD(M.rp + M.n) != M.nnz);
  for (int v = threadIdx.x; v < M.n; v += kSoloNT) bad |= SO_LD(M.rp + v + 1) < SO_LD(M.rp + v);
  bad = __syncthreads_or(bad);
  if (!bad)
    for (int i = threadIdx.x; i < M.nnz; i += kSoloNT) {
      const int c = SO_LD(M.col + i);
      bad |= (c < 0 || c >= M.n);
    }
  bad = __syncthreads_or(bad);
  if (bad) {
    if (threadIdx.x == 0) atomicCAS(&a.ctl->status, 0, ST_BAD_CSR);
    return false;
  }
  if (a.validate < 2) return true;
  int asym = 0;
  for (int u = threadIdx.x; u < M.n && !asym; u += kSoloNT) {   // thread per row
    for (int e = SO_LD(M.rp + u), re = SO_LD(M.rp + u + 1); e < re && !asym; ++e) {
      const int c = SO_LD(M.col + e);
      int lo = SO_LD(M.rp + c), hi = SO_LD(M.rp + c + 1) - 1;
      const int b0 = lo, b1 = hi;
      bool found = false;
      while (lo <= hi) {   // sorted row: O(log deg)
        const int mid = (lo + hi) >> 1;
        const int x = SO_LD(M.col + mid);
        if (x == u) { found = true; break; }
        if (x < u) lo = mid + 1; else hi = mid - 1;
      }
      for (int f = b0; f <= b1 && !found; ++f) found = SO_LD(M.col + f) == u;   // unsorted row
      asym |= !found;
    }
  }
  asym = __syncthreads_or(asym);
  if (asym && threadIdx.x == 0) atomicCAS(&a.ctl->status, 0, ST_NOT_SYM);
  return !asym;
}

// ---------------------------------------------------------------- batches
// Exclusive block scan with ONE barrier: warp totals go to buffer `buf`,
// consecutive calls alternate buffers (a buffer is rewritten only after every
// thread has passed the other buffer's barrier).
__device__ __forceinline__ int so_scan1(int v, int32_t* buf, int& total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, d);
    if (lane >= d) x += y;
  }
  if (lane == 31) buf[wid] = x;
  __syncthreads();
  // the kSoloNW warp totals, scanned in the first lanes of every warp
  int wv = lane < kSoloNW ? buf[lane] : 0;
#pragma unroll
  for (int d = 1; d < kSoloNW; d <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, wv, d);
    if (lane >= d) wv += y;
  }
  total = __shfl_sync(0xffffffffu, wv, kSoloNW - 1);
  const int base = __shfl_sync(0xffffffffu, wv, (wid + 31) & 31);   // inclusive total of warps < wid
  return (wid ? base : 0) + x - v;
}

// Traversal state, block-uniform, held in registers by every thread.
struct SoloPos {
  int pos;      // next parent position of o
  int written;  // next output position of o
  int rhi;      // the ring holds positions [pos, rhi) (small matrices; -1: unused)
  int par;      // batch parity (scan / counter buffers)
};

// A parent whose valence exceeds T: its row in chunks of T edge
// slots, children to HBM scratch, one block radix sort by (valence, id).
template <bool kBig>
static __device__ void so_oversize(const SoloArgs& a, const SoloMat& M, SoloSh& sh, SoloPos& S, int rs, int D) {
  unsigned long long* keys = a.spill + M.node_base;
  if (threadIdx.x == 0) sh.cnt = 0;
  __syncthreads();
  for (int c0 = 0; c0 < D; c0 += kSoloT) {
    int cc[kSoloU], slot[kSoloU], crs[kSoloU], cre[kSoloU];
    bool ins[kSoloU];
#pragma unroll
    for (int u = 0; u < kSoloU; ++u) {
      const int e = c0 + threadIdx.x * kSoloU + u;
      cc[u] = e < D ? SO_LD(M.col + rs + e) : -1;
      ins[u] = false;
    }
#pragma unroll
    for (int u = 0; u < kSoloU; ++u) {
      if (cc[u] >= 0 && !so_placed<kBig>(M, cc[u])) {
        slot[u] = so_claim<kBig>((uint32_t)cc[u], (uint32_t)(threadIdx.x * kSoloU + u), &ins[u]);
        if (ins[u]) { crs[u] = SO_LD(M.rp + cc[u]); cre[u] = SO_LD(M.rp + cc[u] + 1); }
      }
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kSoloU; ++u) {
      if (ins[u]) {   // one parent: every child is kept, once (duplicates share the entry)
        const int idx = atomicAdd(&sh.cnt, 1);
        keys[idx] = ((unsigned long long)(uint32_t)(cre[u] - crs[u]) << 32) | (uint32_t)cc[u];
        so_place<kBig>(M, cc[u]);
        so_unclaim<kBig>(slot[u]);
      }
    }
    __syncthreads();
  }
  const int C = sh.cnt;
  if (!(a.flags & F_NO_SORT)) {
    so_radix_sort_global(keys, a.spill + a.spill_cap + M.node_base, C, sh);
    so_hash_reset<kBig>();   // the sort's digit counters overlaid the table
  }
  const int last = M.n - 1;
  for (int i = threadIdx.x; i < C; i += kSoloNT) {
    const int c = (int)(uint32_t)__ldcg(keys + i);
    M.perm[last - S.written - i] = c;
    if (a.iperm) a.iperm[M.node_base + c] = last - S.written - i;
    if (!kBig && kSoloPend) a.pend[M.node_base + S.written + i] = make_int2(0, -1);   // row start not kept: re-read
  }
  if (threadIdx.x == 0) { ++sh.st_exec; ++sh.st_over; }
  S.pos += 1;
  S.written += C;   // the ring is not extended: these parents are refilled from perm
  __syncthreads();
}

// One batch (P:L749-792 on one block): parents [pos, pos + nP) from the ring,
// the longest prefix (<= B_s) whose valences fit the T edge slots; thread t
// owns edge slots [U t, U t + U).  The first claimer of a child (exactly one
// per child) loads its row_ptr and files it under the winning (minimum edge
// slot = earliest) parent; thread lp sorts parent lp's children and writes
// them out.  Six block barriers per batch.
template <bool kBig>
static __device__ void so_step(const SoloArgs& a, const SoloMat& M, SoloSh& sh, SoloPos& S) {
  const int last = M.n - 1;
  const int t = threadIdx.x;
  // ---- refill the ring from perm when it runs low
  int rhi = S.rhi;
  if (kBig || (rhi < S.written && rhi - S.pos < a.BS)) {
    const int lo = kBig ? S.pos : rhi;
    const int hi = min(S.written, S.pos + kSoloQ);
    for (int q = lo + t; q < hi; q += kSoloNT) {
      const int v = __ldcs(M.perm + last - q);   // read once (streaming)
      int2 rd = (kBig || !kSoloPend) ? make_int2(0, -1) : __ldcs(a.pend + M.node_base + q);   // coalesced
      if (rd.y < 0) { rd.x = SO_LD(M.rp + v); rd.y = SO_LD(M.rp + v + 1) - rd.x; }
      so_ring_v()[q & (kSoloQ - 1)] = v;
      so_ring_rs()[q & (kSoloQ - 1)] = rd.x;
      so_ring_d()[q & (kSoloQ - 1)] = rd.y;
    }
    rhi = hi;
    if (!kBig) S.rhi = hi;
    __syncthreads();
  }
  // ---- parents
  const int pos = S.pos, written = S.written;
  const int avail = min(a.BS, rhi - pos);
  const int d = t < avail ? so_ring_d()[(pos + t) & (kSoloQ - 1)] : 0;
  int E;
  const int eo = so_scan1(d, sh.wscan[0], E);
  const bool fit = t < avail && eo + d <= kSoloT;
  if (fit) {
    so_p_rs()[t] = so_ring_rs()[(pos + t) & (kSoloQ - 1)];
    so_p_eo()[t] = eo;
    so_p_eo()[t + 1] = eo + d;   // == the next parent's offset; the last one ends the slots
    so_p_cnt()[t] = 0;
    // owner of the first slot of every U-slot group this parent covers
    for (int g = (eo + kSoloU - 1) / kSoloU; g * kSoloU < eo + d; ++g) so_flp()[g] = (uint16_t)t;
  }
  const int nP = __syncthreads_count(fit);
  if (nP == 0) {   // the first parent alone exceeds T
    so_oversize<kBig>(a, M, sh, S, so_ring_rs()[pos & (kSoloQ - 1)], so_ring_d()[pos & (kSoloQ - 1)]);
    return;
  }
  E = so_p_eo()[nP];
  if (t == 0 && a.collect_stats) {   // does this batch combine the outputs of several earlier batches?
    while (sh.grp_h < sh.grp_t && sh.grp[sh.grp_h & (kSoloGrp - 1)] <= pos) ++sh.grp_h;
    if (sh.grp_h < sh.grp_t && sh.grp[sh.grp_h & (kSoloGrp - 1)] < pos + nP) ++sh.st_comb;
  }
  // ---- discover: columns, placed test, claims; first claimers load the child's row_ptr
  const int e0 = t * kSoloU;
  int cc[kSoloU], slot[kSoloU];   // slot >= 0: this thread created the child's table entry
  if (e0 < E) {
    // the parent of the thread's first slot, then advance: its row start and
    // slot range stay in registers across the kSoloU slots
    int lp = so_flp()[t];
    int se = so_p_eo()[lp], nx = so_p_eo()[lp + 1], rs = so_p_rs()[lp];
#pragma unroll
    for (int u = 0; u < kSoloU; ++u) {
      const int e = e0 + u;
      cc[u] = -1;
      if (e < E) {
        while (nx <= e) { ++lp; se = nx; nx = so_p_eo()[lp + 1]; rs = so_p_rs()[lp]; }
        so_lpof()[e] = (uint16_t)lp;
        cc[u] = SO_LDS(M.col + rs + (e - se));
      }
    }
  } else {
#pragma unroll
    for (int u = 0; u < kSoloU; ++u) cc[u] = -1;
  }
#pragma unroll
  for (int u = 0; u < kSoloU; ++u) {
    slot[u] = -1;
    if (cc[u] >= 0 && !so_placed<kBig>(M, cc[u])) {   // placed nodes (self-loops included) are skipped
      bool ins;
      const int sl = so_claim<kBig>((uint32_t)cc[u], (uint32_t)(e0 + u), &ins);
      if (ins) {
        const int r0 = SO_LD(M.rp + cc[u]);
        if constexpr (!kBig) so_rsv()[sl] = r0;   // (big matrices: the 8 B entries overlay rsv)
        so_rdeg()[sl] = SO_LD(M.rp + cc[u] + 1) - r0;
        slot[u] = sl;
      }
    }
  }
  __syncthreads();
  // ---- file every child under the minimum edge slot's parent
  int won = 0;
#pragma unroll
  for (int u = 0; u < kSoloU; ++u) {
    const int sl = slot[u];
    if (sl >= 0) {
      int c, ew;
      if constexpr (!kBig) { const uint32_t h = so_hash()[sl]; c = (int)(h >> 15); ew = (int)(h & 0x7fffu); }
      else { const unsigned long long h = so_hash64()[sl]; c = (int)(h >> 32); ew = (int)(uint32_t)h; }
      const int lp = so_lpof()[ew];
      const int idx = atomicAdd(&so_p_cnt()[lp], 1);
      const unsigned long long dg = (unsigned long long)(uint32_t)so_rdeg()[sl];
      unsigned long long key;
      if constexpr (!kBig) key = (dg << 32) | ((unsigned long long)(uint32_t)c << 15) | (uint32_t)sl;
      else key = (dg << 32) | (uint32_t)c;
      so_cand()[so_p_eo()[lp] + idx] = key;
      so_place<kBig>(M, c);
      so_unclaim<kBig>(sl);   // each entry is read by its creator only
      ++won;
    }
  }
  __syncthreads();
  // ---- thread lp: sort parent lp's children by (valence, id) (C-1)
  const int par = S.par;
  const int mycnt = t < nP ? so_p_cnt()[t] : 0;
  unsigned long long* seg = so_cand() + (t < nP ? so_p_eo()[t] : 0);
  if (mycnt > 1 && !(a.flags & F_NO_SORT)) {
    if (mycnt <= 16) {
      for (int i = 1; i < mycnt; ++i) {
        const unsigned long long x = seg[i];
        int j = i - 1;
        while (j >= 0 && seg[j] > x) { seg[j + 1] = seg[j]; --j; }
        seg[j + 1] = x;
      }
    } else {
      so_big_list()[atomicAdd(&sh.nbig[par], 1)] = t;
    }
  }
  // ---- output positions: exclusive prefix of the per-parent counts
  int tot;
  const int pf = so_scan1(mycnt, sh.wscan[1], tot);
  const int nbig = sh.nbig[par];
  if (nbig) {   // segments above 16 children: one warp each
    const int lane = t & 31, wid = t >> 5;
    for (int b = wid; b < nbig; b += kSoloNW) {
      const int lp = so_big_list()[b];
      bitonic_sort_flip(so_cand() + so_p_eo()[lp], so_p_cnt()[lp], lane, 32, [] { __syncwarp(); });
    }
    __syncthreads();
  }
  const int pos_new = pos + nP;
  const bool ring_ok = !kBig && S.rhi == written;
  for (int j = 0; j < mycnt; ++j) {
    const unsigned long long key = seg[j];
    const int q = written + pf + j;
    int c;
    if constexpr (!kBig) c = (int)((key >> 15) & 0x1ffffu);
    else c = (int)(uint32_t)key;
    M.perm[last - q] = c;
    if (a.iperm) a.iperm[M.node_base + c] = last - q;
    if constexpr (!kBig) {
      const int r0 = so_rsv()[key & 0x7fffu];
      if (ring_ok && q < pos_new + kSoloQ) {
        so_ring_v()[q & (kSoloQ - 1)] = c;
        so_ring_rs()[q & (kSoloQ - 1)] = r0;
        so_ring_d()[q & (kSoloQ - 1)] = (int)(key >> 32);
      } else if (kSoloPend) {
        a.pend[M.node_base + q] = make_int2(r0, (int)(key >> 32));
      }
    }
  }
  if (a.collect_stats && won) atomicAdd(reinterpret_cast<unsigned long long*>(&sh.st_claim), (unsigned long long)won);
  if (t == 0) {
    sh.nbig[par ^ 1] = 0;   // the next batch's counter (this one is read above)
    ++sh.st_exec;
    if (a.collect_stats && tot > 0 && sh.grp_t - sh.grp_h < kSoloGrp) sh.grp[(sh.grp_t++) & (kSoloGrp - 1)] = written;
  }
  S.pos = pos_new;
  S.written = written + tot;
  if (ring_ok) S.rhi = min(written + tot, pos_new + kSoloQ);
  S.par = par ^ 1;
  __syncthreads();
}

template <bool kBig>
static __device__ void so_traverse(const SoloArgs& a, const SoloMat& M, SoloSh& sh, int seed) {
  SoloPos S;
  S.pos = 0;
  S.written = 0;
  S.rhi = kBig ? -1 : 0;
  S.par = 0;
  if (threadIdx.x == 0) {
    sh.grp_h = sh.grp_t = 0;
    sh.nbig[0] = sh.nbig[1] = 0;
    ++sh.st_comp;
  }
  so_place_root(a, M, seed, 0, S.rhi);
  S.written = 1;
  __syncthreads();
  for (;;) {
    if (S.pos == S.written) {   // component exhausted (C-6)
      if (S.written >= M.n) break;
      int s = so_next_seed(M, sh);
      if (s < 0) { if (threadIdx.x == 0) atomicCAS(&a.ctl->status, 0, ST_BAD_CSR); break; }
      if (a.mode == RCM_START_PSEUDO_PERIPHERAL) s = so_gl(M, S.written, s, sh);
      so_place_root(a, M, s, S.written, S.rhi);
      S.written += 1;
      if (threadIdx.x == 0) ++sh.st_comp;
      __syncthreads();
      continue;
    }
    so_step<kBig>(a, M, sh, S);
  }
}

// One matrix: validation, seed (C-5 / C-6 / FIXED), traversal.
static __device__ void so_matrix(const SoloArgs& a, int k, SoloSh& sh) {
  SoloMat M;
  long long rp_base = 0, ci_base = 0;
  if (a.node_off) {
    M.node_base = __ldg(a.node_off + k);
    M.n = (int)(__ldg(a.node_off + k + 1) - M.node_base);
    ci_base = __ldg(a.nnz_off + k);
    M.nnz = (int)(__ldg(a.nnz_off + k + 1) - ci_base);
    rp_base = M.node_base + k;
  } else {
    M.node_base = 0;
    M.n = a.n;
    M.nnz = (int)a.nnz;
  }
  if (M.n <= 0) return;
  M.rp = a.row_ptr + rp_base;
  M.col = a.col_idx + ci_base;
  M.perm = a.perm + M.node_base;
  M.gmem = M.n > kSoloNMax;
  M.b0 = 0;
  if (M.gmem) {
    M.vis = a.gvis + (M.node_base >> 5);
    M.bvis = a.gvis + a.gvis_words + (M.node_base >> 5);
    M.b0 = (int)(M.node_base & 31);
  } else {
    M.vis = reinterpret_cast<uint32_t*>(so_base() + kSoOffVis);
    // overlays the ring and the batch scratch: the GL finder runs only when no
    // parent is pending (matrix start, component restart)
    M.bvis = reinterpret_cast<uint32_t*>(so_base() + kSoOffRing);
  }
  if (a.validate && !so_validate(a, M, sh)) return;
  int seed;
  if (a.mode == RCM_START_FIXED) seed = a.node_off ? (a.starts ? __ldg(a.starts + k) : 0) : a.start;
  else seed = 0;
  if (seed < 0 || seed >= M.n) {   // FIXED start out of range (checked always: ADVICE r1)
    if (threadIdx.x == 0) atomicCAS(&a.ctl->status, 0, ST_BAD_CSR);
    return;
  }
  // prologue: argmin (valence, id) -- the MIN_DEGREE seed and the C-6 cursor
  unsigned long long best = kKeyMax;
  for (int v = threadIdx.x; v < M.n; v += kSoloNT) {
    const unsigned long long key = ((unsigned long long)(uint32_t)so_deg(M, v) << 32) | (uint32_t)v;
    best = key < best ? key : best;
  }
  so_zero_bits(M, M.vis);
  // claim table starts empty (every batch restores it)
  if (!M.gmem) so_hash_reset<false>();
  else so_hash_reset<true>();
  best = so_min_u64(best, sh);
  if (a.mode != RCM_START_FIXED) seed = (int)(uint32_t)best;
  if (threadIdx.x == 0) {
    sh.cur_deg = (int)(best >> 32);
    sh.cur_id = a.mode == RCM_START_FIXED ? -1 : seed;
  }
  __syncthreads();
  if (a.mode == RCM_START_PSEUDO_PERIPHERAL) seed = so_gl(M, 0, seed, sh);
  if (M.gmem) so_traverse<true>(a, M, sh, seed);
  else so_traverse<false>(a, M, sh, seed);
}

}  // namespace rcm
