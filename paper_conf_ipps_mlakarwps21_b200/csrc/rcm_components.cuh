// rcm_components.cuh -- everything around the traversal that the paper leaves
// implicit: connected components of a disconnected graph ordered by the C-6
// rule (a13), a grid-wide LSD radix sort used to order them, and the
// pseudo-peripheral start finder of P:L365-375 (level-synchronous BFS, NEXT-1).
#pragma once
#include <cuda_runtime.h>

#include "../../include/rcm.h"
#include "rcm_workers.cuh"

namespace rcm {

constexpr int kSortTile = 4096;          // keys per block per radix pass
constexpr int kSortThreads = 512;        // 8 keys per thread

struct CompWS {
  int64_t cap = 0;
  int32_t* label = nullptr;              // union-find parent
  unsigned long long* ckey = nullptr;    // per root: min (deg << 32 | id)
  int32_t* csize = nullptr;              // per root: component size
  unsigned long long* keys[2] = {nullptr, nullptr};
  int32_t* vals[2] = {nullptr, nullptr};
  long long* offs = nullptr;             // component output offsets
  int32_t* hist = nullptr;               // radix: 256 x tiles
  int32_t* ctl = nullptr;                // [0] count, [1] cur buffer, [2] skip, [3..] misc
  int32_t* order = nullptr;              // matrix order (batched LPT)
  int32_t* lev = nullptr;                // GL levels
  int32_t* front[2] = {nullptr, nullptr};
  int32_t* gl_ctl = nullptr;             // GL counters
  unsigned long long* gl_key = nullptr;
};

inline cudaError_t comp_alloc(CompWS& w, int64_t n) {
  w.cap = n;
  const int64_t tiles = (n + kSortTile - 1) / kSortTile + 1;
  cudaError_t e;
#define A(p, b) if ((e = cudaMalloc((void**)&(p), (b))) != cudaSuccess) return e;
  A(w.label, 4 * n) A(w.ckey, 8 * n) A(w.csize, 4 * n) A(w.keys[0], 8 * n) A(w.keys[1], 8 * n)
  A(w.vals[0], 4 * n) A(w.vals[1], 4 * n) A(w.offs, 8 * (n + 1)) A(w.hist, 4 * 256 * tiles)
  A(w.ctl, 4 * 64) A(w.order, 4 * n) A(w.lev, 4 * n) A(w.front[0], 4 * n) A(w.front[1], 4 * n)
  A(w.gl_ctl, 4 * 64) A(w.gl_key, 8 * 64)
#undef A
  return cudaSuccess;
}

inline void comp_free(CompWS& w) {
  cudaFree(w.label); cudaFree(w.ckey); cudaFree(w.csize); cudaFree(w.keys[0]); cudaFree(w.keys[1]);
  cudaFree(w.vals[0]); cudaFree(w.vals[1]); cudaFree(w.offs); cudaFree(w.hist); cudaFree(w.ctl);
  cudaFree(w.order); cudaFree(w.lev); cudaFree(w.front[0]); cudaFree(w.front[1]); cudaFree(w.gl_ctl);
  cudaFree(w.gl_key);
}

// ============================================================ radix sort
// Grid-wide stable LSD radix sort of (key u64, val i32) pairs; the element
// count lives on the device (cctl[0]); cctl[1] = index of the buffer holding
// the current data; a pass whose digit is constant is skipped (cctl[2]).
__global__ void __launch_bounds__(kSortThreads) k_radix_hist(CompWS w, int shift) {
  __shared__ int h[256];
  const int count = w.ctl[0];
  const int tiles = (count + kSortTile - 1) / kSortTile;
  const int b = blockIdx.x;
  for (int i = threadIdx.x; i < 256; i += kSortThreads) h[i] = 0;
  __syncthreads();
  if (b < tiles) {
    const unsigned long long* src = w.keys[w.ctl[1]];
    for (int i = b * kSortTile + threadIdx.x; i < min(count, (b + 1) * kSortTile); i += kSortThreads)
      atomicAdd(&h[(src[i] >> shift) & 0xff], 1);
  }
  __syncthreads();
  if (b < tiles)
    for (int i = threadIdx.x; i < 256; i += kSortThreads) w.hist[i * tiles + b] = h[i];
}

// single block: exclusive scan of hist[digit][tile] (digit-major) and the skip test
__global__ void __launch_bounds__(1024) k_radix_scan(CompWS w) {
  __shared__ int tmp[33];
  __shared__ int carry;
  __shared__ int skip;
  const int count = w.ctl[0];
  const int tiles = (count + kSortTile - 1) / kSortTile;
  const int total = 256 * tiles;
  if (threadIdx.x == 0) { carry = 0; skip = 0; }
  __syncthreads();
  // skip test: some digit holds every element
  for (int d = threadIdx.x; d < 256; d += blockDim.x) {
    long long s = 0;
    for (int t = 0; t < tiles; ++t) s += w.hist[d * tiles + t];
    if (s == count) skip = 1;
  }
  __syncthreads();
  if (skip || count <= 1) {
    if (threadIdx.x == 0) w.ctl[2] = 1;
    return;
  }
  for (int base = 0; base < total; base += blockDim.x) {
    int i = base + threadIdx.x;
    int v = i < total ? w.hist[i] : 0;
    int x = v;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int d = 1; d < 32; d <<= 1) { int y = __shfl_up_sync(0xffffffffu, x, d); if (lane >= d) x += y; }
    if (lane == 31) tmp[wid] = x;
    __syncthreads();
    if (wid == 0) {
      int s = lane < (int)(blockDim.x >> 5) ? tmp[lane] : 0;
      int q = s;
      for (int d = 1; d < 32; d <<= 1) { int y = __shfl_up_sync(0xffffffffu, q, d); if (lane >= d) q += y; }
      tmp[lane] = q - s;
      if (lane == 31) tmp[32] = q;
    }
    __syncthreads();
    if (i < total) w.hist[i] = carry + tmp[wid] + x - v;
    __syncthreads();
    if (threadIdx.x == 0) carry += tmp[32];
    __syncthreads();
  }
  if (threadIdx.x == 0) w.ctl[2] = 0;
}

__global__ void __launch_bounds__(kSortThreads) k_radix_scatter(CompWS w, int shift) {
  __shared__ int wcnt[kSortThreads / 32][256];
  __shared__ int off[256];
  const int count = w.ctl[0];
  const int tiles = (count + kSortTile - 1) / kSortTile;
  const int b = blockIdx.x;
  if (w.ctl[2]) return;   // skipped pass (no buffer swap)
  const int cur = w.ctl[1];
  if (b < tiles) {
    const unsigned long long* sk = w.keys[cur];
    const int32_t* sv = w.vals[cur];
    unsigned long long* dk = w.keys[cur ^ 1];
    int32_t* dv = w.vals[cur ^ 1];
    for (int i = threadIdx.x; i < 256; i += kSortThreads) off[i] = w.hist[i * tiles + b];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1;
    for (int j = 0; j < kSortTile / kSortThreads; ++j) {
      const int i = b * kSortTile + j * kSortThreads + threadIdx.x;
      const bool valid = i < count;
      unsigned long long k = valid ? sk[i] : 0;
      int v = valid ? sv[i] : 0;
      int d = valid ? (int)((k >> shift) & 0xff) : 256;
      unsigned peers = __match_any_sync(0xffffffffu, d);
      int rank = __popc(peers & lt);
      for (int q = threadIdx.x; q < (kSortThreads / 32) * 256; q += kSortThreads) (&wcnt[0][0])[q] = 0;
      __syncthreads();
      if (valid && rank == 0) wcnt[wid][d] = __popc(peers);
      __syncthreads();
      for (int dg = threadIdx.x; dg < 256; dg += kSortThreads) {
        int run = off[dg];
        for (int ww = 0; ww < kSortThreads / 32; ++ww) { int c = wcnt[ww][dg]; wcnt[ww][dg] = run; run += c; }
        off[dg] = run;
      }
      __syncthreads();
      if (valid) {
        int pos = wcnt[wid][d] + rank;
        dk[pos] = k;
        dv[pos] = v;
      }
      __syncthreads();
    }
  }
}

__global__ void k_radix_flip(CompWS w) {
  if (!w.ctl[2] && w.ctl[0] > 1) w.ctl[1] ^= 1;
}

inline void radix_sort_pairs(CompWS& w, int64_t max_count, int nbits, cudaStream_t s) {
  const int tiles = (int)((max_count + kSortTile - 1) / kSortTile);
  if (tiles <= 0) return;
  for (int shift = 0; shift < nbits; shift += 8) {
    k_radix_hist<<<tiles, kSortThreads, 0, s>>>(w, shift);
    k_radix_scan<<<1, 1024, 0, s>>>(w);
    k_radix_scatter<<<tiles, kSortThreads, 0, s>>>(w, shift);
    k_radix_flip<<<1, 1, 0, s>>>(w);
  }
}

// ====================================================== connected components
// Union-find (hooking larger root under smaller, path halving) over the nodes
// the chain-first pass left unvisited.  Runs only if ctl->incomplete.
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

__global__ void k_cc_init(CompWS w, Ctl* ctl, const unsigned long long* __restrict__ word, int n) {
  if (!ctl->incomplete) {
    // the chain-first pass ordered every node: make the follow-up scheduler a no-op
    if (blockIdx.x == 0 && threadIdx.x == 0) { ctl->n_chain = 0; ctl->n_solo = 0; }
    return;
  }
  for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    bool unv = (uint32_t)(word[v] >> 32) == kInf;
    w.label[v] = unv ? v : -1;
    w.ckey[v] = kKeyMax;
    w.csize[v] = 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) w.ctl[0] = 0;
}

__global__ void k_cc_hook(CompWS w, Ctl* ctl, const int32_t* __restrict__ row_ptr,
                          const int32_t* __restrict__ col_idx, int n) {
  if (!ctl->incomplete) return;
  for (int u = blockIdx.x * blockDim.x + threadIdx.x; u < n; u += gridDim.x * blockDim.x) {
    if (w.label[u] < 0) continue;
    for (int e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
      int c = col_idx[e];
      if (c == u || ld_cg_s32(w.label + c) < 0) continue;
      for (;;) {
        int a = uf_find(w.label, u), b = uf_find(w.label, c);
        if (a == b) break;
        if (a > b) { int t = a; a = b; b = t; }
        if (atomicCAS(w.label + b, b, a) == b) break;
      }
    }
  }
}

__global__ void k_cc_compress_keys(CompWS w, Ctl* ctl, const unsigned long long* __restrict__ word, int n) {
  if (!ctl->incomplete) return;
  for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    if (ld_cg_s32(w.label + v) < 0) continue;
    int r = uf_find(w.label, v);
    unsigned long long k = ((word[v] & 0xffffffffull) << 32) | (uint32_t)v;
    atomicMin(w.ckey + r, k);
    atomicAdd(w.csize + r, 1);
  }
}

// roots -> (key, root) list; the order of the list is fixed by the sort below
__global__ void k_cc_collect(CompWS w, Ctl* ctl, int n, int idbits) {
  if (!ctl->incomplete) return;
  for (int v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
    if (ld_cg_s32(w.label + v) != v) continue;
    int i = atomicAdd(w.ctl + 0, 1);
    unsigned long long k = w.ckey[v];
    // compact key (deg << idbits | id): same order as (deg << 32 | id)
    w.keys[0][i] = ((k >> 32) << idbits) | (k & 0xffffffffull);
    w.vals[0][i] = v;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) w.ctl[1] = 0;
}

// Component output offsets: exclusive scan of sizes in key order, starting at
// the chain-first total; then problems / direct singleton writes.
__global__ void __launch_bounds__(1024) k_cc_offsets(CompWS w, Ctl* ctl) {
  if (!ctl->incomplete) return;
  __shared__ long long tmp[33];
  __shared__ long long carry;
  const int count = w.ctl[0];
  const int cur = w.ctl[1];
  if (threadIdx.x == 0) carry = ctl->chain_total;
  __syncthreads();
  for (int base = 0; base < count; base += blockDim.x) {
    int i = base + threadIdx.x;
    long long v = i < count ? w.csize[w.vals[cur][i]] : 0;
    long long x = v;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int d = 1; d < 32; d <<= 1) { long long y = __shfl_up_sync(0xffffffffu, x, d); if (lane >= d) x += y; }
    if (lane == 31) tmp[wid] = x;
    __syncthreads();
    if (wid == 0) {
      long long s0 = lane < (int)(blockDim.x >> 5) ? tmp[lane] : 0;
      long long q = s0;
      for (int d = 1; d < 32; d <<= 1) { long long y = __shfl_up_sync(0xffffffffu, q, d); if (lane >= d) q += y; }
      tmp[lane] = q - s0;
      if (lane == 31) tmp[32] = q;
    }
    __syncthreads();
    if (i < count) w.offs[i] = carry + tmp[wid] + x - v;
    __syncthreads();
    if (threadIdx.x == 0) carry += tmp[32];
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    ctl->n_comp = count;
    ctl->n_chain = 0;
    ctl->n_solo = 0;
    ctl->solo_next = 0;
    ctl->gbar_count = 0;
  }
}

__global__ void k_cc_problems(CompWS w, KParams kp, int n, int thr, int64_t prob_cap) {
  if (!kp.ctl->incomplete) return;
  const int count = w.ctl[0];
  const int cur = w.ctl[1];
  Problem* chains = const_cast<Problem*>(kp.chains);
  Problem* solos = const_cast<Problem*>(kp.solos);
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x) {
    const int root = w.vals[cur][i];
    const int size = w.csize[root];
    const int seed = (int)(uint32_t)w.ckey[root];
    const int pos = (int)w.offs[i];
    if (size == 1) {   // isolated node: write it directly
      kp.o[pos] = seed;
      kp.perm[n - 1 - pos] = seed;
      if (kp.iperm) kp.iperm[seed] = n - 1 - pos;
      continue;
    }
    Problem P;
    P.node_base = 0; P.rp_base = 0; P.ci_base = 0; P.o_base = 0; P.perm_base = 0;
    P.mat_n = n; P.pos0 = pos; P.size = size; P.seed = seed; P.flags = 0; P.pad = 0;
    if (thr > 0 && size <= thr) {
      int j = atomicAdd(&kp.ctl->n_solo, 1);
      if (j < prob_cap) solos[j] = P; else latch_error(kp.ctl, ST_CAPACITY);
    } else {
      int j = atomicAdd(&kp.ctl->n_chain, 1);
      if (j < prob_cap) chains[j] = P; else latch_error(kp.ctl, ST_CAPACITY);
    }
  }
}

__global__ void k_cc_count_singletons(CompWS w, KParams kp) {
  if (!kp.ctl->incomplete || !kp.collect_stats) return;
  const int count = w.ctl[0];
  const int cur = w.ctl[1];
  int c = 0;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < count; i += gridDim.x * blockDim.x)
    c += w.csize[w.vals[cur][i]] == 1;
  c = __reduce_add_sync(0xffffffffu, c);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(&kp.stats->components, (unsigned long long)c);
}

inline int bits_for(int64_t x) {
  int b = 0;
  while ((1ll << b) <= x) ++b;
  return b;
}

inline rcm_status_t comp_stage(CompWS& w, const KParams& kp, int n, int64_t nnz, int mode, int thr,
                               int64_t prob_cap, cudaStream_t s) {
  (void)nnz;
  (void)mode;
  const int blocks = std::min((n + 255) / 256, 148 * 16);
  k_cc_init<<<blocks, 256, 0, s>>>(w, kp.ctl, kp.word, n);
  k_cc_hook<<<blocks, 256, 0, s>>>(w, kp.ctl, kp.row_ptr, kp.col_idx, n);
  k_cc_compress_keys<<<blocks, 256, 0, s>>>(w, kp.ctl, kp.word, n);
  const int idbits = bits_for(n - 1 > 0 ? n - 1 : 1);
  k_cc_collect<<<blocks, 256, 0, s>>>(w, kp.ctl, n, idbits);
  // key bits: idbits + valence bits (valence < 2^31)
  radix_sort_pairs(w, n, idbits + 32, s);
  k_cc_offsets<<<1, 1024, 0, s>>>(w, kp.ctl);
  k_cc_problems<<<blocks, 256, 0, s>>>(w, kp, n, thr, prob_cap);
  k_cc_count_singletons<<<blocks, 256, 0, s>>>(w, kp);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? RCM_OK : RCM_ERR_CUDA;
}

// =================================================== batched: LPT order
__global__ void k_size_keys(CompWS w, const int64_t* __restrict__ node_off, int num) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) { w.ctl[0] = num; w.ctl[1] = 0; }
  if (i >= num) return;
  long long sz = node_off[i + 1] - node_off[i];
  // descending size, ties by index: key = (~size) << 32 | i  (sort ascending)
  w.keys[0][i] = ((unsigned long long)(0xffffffffu - (uint32_t)sz) << 32) | (uint32_t)i;
  w.vals[0][i] = i;
}
__global__ void k_copy_order(CompWS w, int num) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < num) w.order[i] = w.vals[w.ctl[1]][i];
}

inline rcm_status_t comp_order_by_size(CompWS& w, const int64_t* node_off, int num, cudaStream_t s) {
  k_size_keys<<<(num + 255) / 256, 256, 0, s>>>(w, node_off, num);
  radix_sort_pairs(w, num, 64, s);
  k_copy_order<<<(num + 255) / 256, 256, 0, s>>>(w, num);
  return cudaGetLastError() == cudaSuccess ? RCM_OK : RCM_ERR_CUDA;
}

// ============================================== pseudo-peripheral finder
// P:L365-375 with reading C-5: BFS from r; x = min (valence, id) on the last
// level; BFS from x; continue while the level count grows; return the last x.
// One persistent kernel, level-synchronous frontiers, grid barriers between
// levels (all blocks co-resident).
struct GLParams {
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const unsigned long long* word;
  int32_t* lev;
  int32_t* front0;
  int32_t* front1;
  int32_t* gctl;                 // [0] barrier count, [1] barrier gen, [2] next-frontier size
  unsigned long long* gkey;      // [0] argmin of the last level
  Ctl* ctl;
  const int32_t* start;          // nullable: start node (else ctl->minkey)
  int32_t* out;
  int n;
  int nblocks;
};

__device__ void gl_barrier(const GLParams& g) {
  __syncthreads();
  if (threadIdx.x == 0) {
    int gen = ld_acquire_s32(g.gctl + 1);
    __threadfence();
    if (atomicAdd(g.gctl + 0, 1) == g.nblocks - 1) {
      atomicExch(g.gctl + 0, 0);
      __threadfence();
      st_release_s32(g.gctl + 1, gen + 1);
    } else {
      while (ld_acquire_s32(g.gctl + 1) == gen) __nanosleep(64);
    }
  }
  __syncthreads();
}

// BFS from r; returns the number of levels; gkey[0] = argmin of the last level.
__device__ int gl_bfs(const GLParams& g, int r, int& sz_cur_ref) {
  const int tid = blockIdx.x * blockDim.x + threadIdx.x;
  const int nth = gridDim.x * blockDim.x;
  for (int v = tid; v < g.n; v += nth) g.lev[v] = -1;
  gl_barrier(g);
  if (tid == 0) {
    g.lev[r] = 0;
    g.front0[0] = r;
    g.gctl[2] = 0;
  }
  gl_barrier(g);
  int32_t* cur = g.front0;
  int32_t* nxt = g.front1;
  int ncur = 1, level = 0;
  __shared__ int s_n;
  for (;;) {
    for (int i = tid; i < ncur; i += nth) {
      int p = ld_cg_s32(cur + i);
      for (int e = __ldg(g.row_ptr + p); e < __ldg(g.row_ptr + p + 1); ++e) {
        int c = __ldg(g.col_idx + e);
        if (ld_cg_s32(g.lev + c) < 0 && atomicCAS(g.lev + c, -1, level + 1) == -1) {
          int j = atomicAdd(g.gctl + 2, 1);
          nxt[j] = c;
        }
      }
    }
    gl_barrier(g);
    if (threadIdx.x == 0) s_n = ld_acquire_s32(g.gctl + 2);
    __syncthreads();
    const int nn = s_n;
    gl_barrier(g);
    if (nn == 0) break;
    if (tid == 0) g.gctl[2] = 0;
    ++level;
    int32_t* t = cur; cur = nxt; nxt = t;
    ncur = nn;
    gl_barrier(g);
  }
  // cur holds the last level (ncur nodes): argmin (valence, id)
  if (tid == 0) g.gkey[0] = kKeyMax;
  gl_barrier(g);
  unsigned long long best = kKeyMax;
  for (int i = tid; i < ncur; i += nth) {
    int v = ld_cg_s32(cur + i);
    unsigned long long k = ((g.word[v] & 0xffffffffull) << 32) | (uint32_t)v;
    best = k < best ? k : best;
  }
  best = warp_min_u64(best);
  if ((threadIdx.x & 31) == 0 && best != kKeyMax) atomicMin(g.gkey, best);
  gl_barrier(g);
  sz_cur_ref = ncur;
  return level + 1;
}

__global__ void __launch_bounds__(512) k_gl(GLParams g) {
  int r = g.start ? *g.start : (int)(uint32_t)g.ctl->minkey;
  int sz;
  int nl = gl_bfs(g, r, sz);
  for (;;) {
    const int x = (int)(uint32_t)ld_acquire_u64(g.gkey);
    const int nx = gl_bfs(g, x, sz);
    if (nx > nl) { r = x; nl = nx; continue; }
    if (blockIdx.x == 0 && threadIdx.x == 0) *g.out = x;   // "use the last node"
    break;
  }
}

inline rcm_status_t gl_launch(CompWS& w, const int32_t* row_ptr, const int32_t* col_idx, int n,
                              const unsigned long long* word, Ctl* ctl, const int32_t* start_host,
                              int32_t* out, cudaStream_t s) {
  static int nb = 0;
  if (!nb) {
    int dev = 0, sms = 0, occ = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_gl, 512, 0);
    nb = sms * std::max(1, std::min(occ, 2));
  }
  GLParams g;
  g.row_ptr = row_ptr; g.col_idx = col_idx; g.word = word; g.lev = w.lev;
  g.front0 = w.front[0]; g.front1 = w.front[1]; g.gctl = w.gl_ctl; g.gkey = w.gl_key; g.ctl = ctl;
  g.start = nullptr; g.out = out; g.n = n; g.nblocks = nb;
  if (start_host) {
    if (cudaMemcpyAsync(w.gl_ctl + 8, start_host, 4, cudaMemcpyHostToDevice, s) != cudaSuccess) return RCM_ERR_CUDA;
    g.start = w.gl_ctl + 8;
  }
  if (cudaMemsetAsync(w.gl_ctl, 0, 8, s) != cudaSuccess) return RCM_ERR_CUDA;
  k_gl<<<nb, 512, 0, s>>>(g);
  return cudaGetLastError() == cudaSuccess ? RCM_OK : RCM_ERR_CUDA;
}

inline rcm_status_t gl_batched(CompWS&, const int32_t*, const int32_t*, const int64_t*, const int64_t*, int,
                               unsigned long long*, cudaStream_t) {
  return RCM_ERR_INVALID_ARGUMENT;   // per-matrix GL: not implemented yet
}

}  // namespace rcm
