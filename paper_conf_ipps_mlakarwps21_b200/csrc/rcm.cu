// rcm.cu -- kernels and the C ABI (include/rcm.h) of the B200 batch-RCM library.
// Citations P:L<n> = /root/reference/PAPER.md line n; C-k = DESIGN.md readings.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>

#include "../../include/rcm.h"
#include "rcm_components.cuh"
#include "rcm_workers.cuh"

using namespace rcm;

// ===================================================================== kernels
// a1 -- prologue: valence = row_ptr diff, owner word init, argmin of
// (valence, id) (C-6 / MIN_DEGREE seed), max valence, optional CSR checks.
// Four nodes per thread with an int4 row_ptr load and a one-element halo.
__global__ void __launch_bounds__(256) k_prologue(const int32_t* __restrict__ row_ptr, int n,
                                                  long long nnz, unsigned long long* __restrict__ word,
                                                  Ctl* ctl, int validate, int vec) {
  __shared__ unsigned long long smin[8];
  __shared__ int smax[8];
  __shared__ int sbad[8];
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  const int v0 = t * 4;
  unsigned long long best = kKeyMax;
  int mx = 0, bad = 0;
  if (v0 < n) {
    int r[5];
    if (vec && v0 + 4 <= n) {
      int4 q = __ldg(reinterpret_cast<const int4*>(row_ptr + v0));
      r[0] = q.x; r[1] = q.y; r[2] = q.z; r[3] = q.w;
      r[4] = __ldg(row_ptr + v0 + 4);
    } else {
      for (int j = 0; j < 5; ++j) r[j] = (v0 + j <= n) ? __ldg(row_ptr + v0 + j) : 0;
    }
    const int m = min(4, n - v0);
    unsigned long long w[4];
    for (int j = 0; j < 4; ++j) {
      if (j < m) {
        int d = r[j + 1] - r[j];
        if (d < 0) { bad = 1; d = 0; }
        w[j] = ((unsigned long long)kInf << 32) | (uint32_t)d;
        unsigned long long k = ((unsigned long long)(uint32_t)d << 32) | (uint32_t)(v0 + j);
        best = k < best ? k : best;
        mx = max(mx, d);
      }
    }
    if (m == 4) {
      reinterpret_cast<ulonglong2*>(word + v0)[0] = make_ulonglong2(w[0], w[1]);
      reinterpret_cast<ulonglong2*>(word + v0)[1] = make_ulonglong2(w[2], w[3]);
    } else {
      for (int j = 0; j < m; ++j) word[v0 + j] = w[j];
    }
    if (validate) {
      if (v0 == 0 && r[0] != 0) bad = 1;
      if (v0 + m == n && (long long)r[m] != nnz) bad = 1;
    }
  }
  best = warp_min_u64(best);
  for (int d = 16; d > 0; d >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, d));
  bad = __any_sync(0xffffffffu, bad);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) { smin[wid] = best; smax[wid] = mx; sbad[wid] = bad; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int i = 1; i < (int)(blockDim.x >> 5); ++i) {
      best = smin[i] < best ? smin[i] : best;
      mx = max(mx, smax[i]);
      bad |= sbad[i];
    }
    if (best != kKeyMax) atomicMin(&ctl->minkey, best);
    if (mx) atomicMax(&ctl->maxdeg, mx);
    if (bad) atomicCAS(&ctl->status, 0, ST_BAD_CSR);
  }
}

// validate >= 1: every column index in range.
__global__ void k_validate_cols(const int32_t* __restrict__ col_idx, long long nnz, int n, Ctl* ctl) {
  int bad = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < nnz;
       i += (long long)gridDim.x * blockDim.x) {
    int c = __ldg(col_idx + i);
    bad |= (c < 0 || c >= n);
  }
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicCAS(&ctl->status, 0, ST_BAD_CSR);
}

// validate == 2: structural symmetry -- for every (u, c) the row of c holds u.
__global__ void k_validate_sym(const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                               int n, Ctl* ctl) {
  int bad = 0;
  for (int u = blockIdx.x * blockDim.x + threadIdx.x; u < n; u += gridDim.x * blockDim.x) {
    for (int e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
      int c = col_idx[e];
      if (c < 0 || c >= n) { bad = 1; continue; }
      bool found = false;
      for (int f = row_ptr[c]; f < row_ptr[c + 1] && !found; ++f) found = col_idx[f] == u;
      bad |= !found;
    }
  }
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicCAS(&ctl->status, 0, ST_NOT_SYM);
}

// Batched prologue: per matrix k, local valences and the per-matrix argmin.
__global__ void __launch_bounds__(256) k_prologue_batched(const int32_t* __restrict__ rp_local,
                                                          const int64_t* __restrict__ node_off,
                                                          int num, long long total,
                                                          unsigned long long* __restrict__ word,
                                                          unsigned long long* __restrict__ pm_key,
                                                          Ctl* ctl) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long base = (long long)blockIdx.x * blockDim.x; base < total; base += stride) {
    const long long g = base + threadIdx.x;   // warp-uniform loop; lanes past the end idle
    const bool valid = g < total;
    int k = 0;
    unsigned long long key = kKeyMax;
    if (valid) {
      // matrix of g: largest k with node_off[k] <= g
      int lo = 0, hi = num - 1;
      while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (__ldg(node_off + mid) <= g) lo = mid; else hi = mid - 1;
      }
      k = lo;
      const int v = (int)(g - __ldg(node_off + k));
      const int d = max(__ldg(rp_local + g + k + 1) - __ldg(rp_local + g + k), 0);
      word[g] = ((unsigned long long)kInf << 32) | (uint32_t)d;
      key = ((unsigned long long)(uint32_t)d << 32) | (uint32_t)v;
    } else {
      k = -1;
    }
    // warp-aggregated min per matrix: lanes of one matrix are contiguous, so a
    // segmented shuffle-down min leaves the segment minimum in its first lane
    const unsigned peers = __match_any_sync(0xffffffffu, k);
    unsigned long long m = key;
    const int lane = threadIdx.x & 31;
    for (int off = 1; off < 32; off <<= 1) {
      unsigned long long o2 = __shfl_down_sync(0xffffffffu, m, off);
      int ko = __shfl_down_sync(0xffffffffu, k, off);
      if (lane + off < 32 && ko == k && o2 < m) m = o2;
    }
    if (valid && (int)(threadIdx.x & 31) == __ffs(peers) - 1) atomicMin(pm_key + k, m);
  }
}

// Problem set-up for one graph: the chain-first pass (or one solo problem).
__global__ void k_setup_single(Problem* chains, Problem* solos, Ctl* ctl, int n, int mode, int start,
                               int solo, const int32_t* gl_seed) {
  Problem P;
  P.node_base = 0; P.rp_base = 0; P.ci_base = 0; P.o_base = 0; P.perm_base = 0;
  P.mat_n = n; P.pos0 = 0; P.size = n;
  P.seed = mode == RCM_START_FIXED ? start
         : (gl_seed ? *gl_seed : (int)(uint32_t)ctl->minkey);
  P.flags = solo ? 1 : 0;
  P.pad = 0;
  if (solo) { solos[0] = P; ctl->n_solo = 1; ctl->n_chain = 0; }
  else { chains[0] = P; ctl->n_chain = 1; ctl->n_solo = 0; }
  ctl->solo_next = 0;
  ctl->spill_cursor = 0;
  ctl->incomplete = 0;
  ctl->chain_total = 0;
  ctl->gbar_count = 0;
}

// Problem set-up for a batch of matrices: one solo problem per matrix (C5).
__global__ void k_setup_batched(Problem* solos, Ctl* ctl, const int64_t* __restrict__ node_off,
                                const int64_t* __restrict__ nnz_off, int num, int mode,
                                const int32_t* __restrict__ starts,
                                const unsigned long long* __restrict__ pm_key,
                                const int32_t* __restrict__ order) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) {
    ctl->n_solo = num; ctl->n_chain = 0; ctl->solo_next = 0; ctl->spill_cursor = 0;
    ctl->incomplete = 0; ctl->chain_total = 0; ctl->gbar_count = 0;
  }
  if (i >= num) return;
  const int k = order ? order[i] : i;
  Problem P;
  P.node_base = node_off[k];
  P.rp_base = node_off[k] + k;
  P.ci_base = nnz_off[k];
  P.o_base = node_off[k];
  P.perm_base = node_off[k];
  P.mat_n = (int)(node_off[k + 1] - node_off[k]);
  P.pos0 = 0;
  P.size = P.mat_n;
  P.seed = (mode == RCM_START_FIXED && starts) ? starts[k] : (int)(uint32_t)pm_key[k];
  P.flags = 1;
  P.pad = 0;
  solos[i] = P;
}

// The persistent scheduler: every chain problem in turn on all blocks (grid
// barrier between chains), then the solo problems, one per block at a time.
__global__ void __launch_bounds__(kThreads, 2) k_scheduler(KParams kp) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ ShState sh;
  SmemPtrs sm = carve_smem(dsm, kp.BS, kp.T);
  const int nchain = ld_relaxed_s32(&kp.ctl->n_chain);
  for (int c = 0; c < nchain; ++c) {
    if (blockIdx.x == 0 && threadIdx.x == 0) chain_init(kp, kp.chains[c]);
    grid_barrier(kp);
    if (ld_relaxed_s32(&kp.ctl->status)) return;
    const uint32_t epoch = ld_acquire_u32(&kp.ctl->epoch);
    const Problem P = kp.chains[c];
    chain_worker(kp, P, sm, sh, epoch);
    grid_barrier(kp);
  }
  const int nsolo = ld_relaxed_s32(&kp.ctl->n_solo);
  for (;;) {
    if (threadIdx.x == 0) sh.k = atomicAdd(&kp.ctl->solo_next, 1);
    __syncthreads();
    const int k = sh.k;
    __syncthreads();
    if (k >= nsolo || ld_relaxed_s32(&kp.ctl->status)) break;
    const Problem P = kp.solos[k];
    if (P.size > 0) run_solo(kp, P, sm, sh);
  }
}

// ======================================================================= host
struct rcm_plan {
  int64_t n_max = 0, nnz_max = 0;
  rcm_options_t opt{};
  int device = 0, num_sms = 0, nblocks = 0, BS = 512, T = 0;
  size_t smem = 0;
  int64_t qcap = 0, prob_cap = 0, spill_cap = 0;
  unsigned long long* word = nullptr;
  int32_t* o = nullptr;
  Desc* desc = nullptr;
  Sig* sig = nullptr;
  Ctl* ctl = nullptr;
  Stats* stats = nullptr;
  Problem* chains = nullptr;
  Problem* solos = nullptr;
  unsigned long long* pm_key = nullptr;
  unsigned long long* spill = nullptr;
  CompWS comp{};
  int32_t* gl_out = nullptr;
  int32_t last_status = 0;
};

static rcm_status_t cuda_fail(cudaError_t e) {
  if (e == cudaErrorMemoryAllocation) return RCM_ERR_OUT_OF_MEMORY;
  return RCM_ERR_CUDA;
}
#define CK(x)                                   \
  do {                                          \
    cudaError_t _e = (x);                       \
    if (_e != cudaSuccess) return cuda_fail(_e); \
  } while (0)

extern "C" void rcm_default_options(rcm_options_t* opt) {
  if (opt) std::memset(opt, 0, sizeof(*opt));
}

extern "C" const char* rcm_status_string(rcm_status_t st) {
  switch (st) {
    case RCM_OK: return "ok";
    case RCM_ERR_INVALID_ARGUMENT: return "invalid argument";
    case RCM_ERR_BAD_CSR: return "malformed CSR";
    case RCM_ERR_NOT_SYMMETRIC: return "pattern not structurally symmetric";
    case RCM_ERR_OUT_OF_MEMORY: return "out of device memory";
    case RCM_ERR_CAPACITY: return "queue or scratch capacity exceeded";
    case RCM_ERR_HANG: return "spin watchdog expired";
    case RCM_ERR_CUDA: return "CUDA error";
    case RCM_ERR_NCCL: return "NCCL error";
  }
  return "unknown status";
}

extern "C" void rcm_plan_destroy(rcm_plan_t p) {
  if (!p) return;
  cudaFree(p->word); cudaFree(p->o); cudaFree(p->desc); cudaFree(p->sig); cudaFree(p->ctl);
  cudaFree(p->stats); cudaFree(p->chains); cudaFree(p->solos); cudaFree(p->pm_key);
  cudaFree(p->spill); cudaFree(p->gl_out);
  comp_free(p->comp);
  delete p;
}

extern "C" rcm_status_t rcm_plan_create(rcm_plan_t* out, int64_t n_max, int64_t nnz_max,
                                        const rcm_options_t* opt_in) {
  if (!out || n_max <= 0 || nnz_max < 0 || n_max >= (1ll << 31) - 2) return RCM_ERR_INVALID_ARGUMENT;
  *out = nullptr;
  rcm_plan* p = new (std::nothrow) rcm_plan();
  if (!p) return RCM_ERR_OUT_OF_MEMORY;
  if (opt_in) p->opt = *opt_in;
  rcm_options_t& o = p->opt;
  if (o.batch_nodes < 0 || o.batch_nodes > kMaxBatchNodes || o.temp_elems < 0 || o.blocks_per_sm < 0 ||
      o.validate < 0 || o.validate > 2 || o.queue_capacity < 0) {
    delete p;
    return RCM_ERR_INVALID_ARGUMENT;
  }
  p->n_max = n_max;
  p->nnz_max = nnz_max;
  cudaError_t e = cudaGetDevice(&p->device);
  if (e != cudaSuccess) { delete p; return RCM_ERR_CUDA; }
  cudaDeviceGetAttribute(&p->num_sms, cudaDevAttrMultiProcessorCount, p->device);
  int smem_optin = 0;
  cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, p->device);
  int smem_sm = 0;
  cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, p->device);
  p->BS = o.batch_nodes ? o.batch_nodes : 512;
  int bps = o.blocks_per_sm ? o.blocks_per_sm : 2;
  const size_t static_sh = sizeof(ShState) + 64;
  // T from the shared-memory budget of `bps` blocks per SM (1 KB reserved per block)
  size_t per_block = std::min<size_t>((size_t)smem_sm / bps - 1024 - static_sh, (size_t)smem_optin - static_sh);
  int T = o.temp_elems;
  if (!T) {
    size_t fixed = smem_bytes(p->BS, 0);
    T = (int)((per_block - fixed) / 10);
    T = T / 256 * 256;
  }
  if (T < 2304 || smem_bytes(p->BS, T) > (size_t)smem_optin - static_sh) {
    delete p;
    return RCM_ERR_INVALID_ARGUMENT;
  }
  p->T = T;
  p->smem = smem_bytes(p->BS, T);
  e = cudaFuncSetAttribute(k_scheduler, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->smem);
  if (e != cudaSuccess) { delete p; return RCM_ERR_CUDA; }
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_scheduler, kThreads, p->smem);
  if (occ <= 0) { delete p; return RCM_ERR_CUDA; }
  p->nblocks = std::min(occ, bps) * p->num_sms;
  // queue bound: sum over generating batches of floor(N/B) + max(1, ceil(2V/T))
  int64_t qb = 2 * n_max + n_max / p->BS + 2 * (nnz_max / T + 1) + 64;
  p->qcap = o.queue_capacity ? o.queue_capacity : std::min<int64_t>(qb, (1ll << 31) - 2);
  p->prob_cap = std::max<int64_t>(1, n_max / 2 + 1);
  p->spill_cap = n_max;
  rcm_status_t st = RCM_OK;
#define AL(ptr, bytes)                                                  \
  do {                                                                  \
    cudaError_t _e = cudaMalloc((void**)&(ptr), (bytes));               \
    if (_e != cudaSuccess) { st = cuda_fail(_e); goto fail; }           \
  } while (0)
  AL(p->word, sizeof(unsigned long long) * n_max);
  AL(p->o, sizeof(int32_t) * n_max);
  AL(p->desc, sizeof(Desc) * p->qcap);
  AL(p->sig, sizeof(Sig) * (p->qcap + 1));
  AL(p->ctl, sizeof(Ctl));
  AL(p->stats, sizeof(Stats));
  AL(p->chains, sizeof(Problem) * p->prob_cap);
  AL(p->solos, sizeof(Problem) * p->prob_cap);
  AL(p->pm_key, sizeof(unsigned long long) * p->prob_cap);
  AL(p->spill, sizeof(unsigned long long) * 2 * p->spill_cap);
  AL(p->gl_out, sizeof(int32_t) * 4);
  if (comp_alloc(p->comp, n_max) != cudaSuccess) { st = RCM_ERR_OUT_OF_MEMORY; goto fail; }
#undef AL
  // descriptors / signals start with tag 0 (epochs start at 1)
  if (cudaMemset(p->desc, 0, sizeof(Desc) * p->qcap) != cudaSuccess ||
      cudaMemset(p->sig, 0, sizeof(Sig) * (p->qcap + 1)) != cudaSuccess ||
      cudaMemset(p->ctl, 0, sizeof(Ctl)) != cudaSuccess || cudaMemset(p->stats, 0, sizeof(Stats)) != cudaSuccess ||
      cudaDeviceSynchronize() != cudaSuccess) {
    st = RCM_ERR_CUDA;
    goto fail;
  }
  *out = p;
  return RCM_OK;
fail:
  rcm_plan_destroy(p);
  return st;
}

static KParams make_kparams(rcm_plan* p, const int32_t* row_ptr, const int32_t* col_idx, int32_t* perm,
                            int32_t* iperm) {
  KParams kp;
  kp.row_ptr = row_ptr;
  kp.col_idx = col_idx;
  kp.word = p->word;
  kp.o = p->o;
  kp.perm = perm;
  kp.iperm = iperm;
  kp.desc = p->desc;
  kp.sig = p->sig;
  kp.ctl = p->ctl;
  kp.stats = p->stats;
  kp.chains = p->chains;
  kp.solos = p->solos;
  kp.spill = p->spill;
  kp.spill_cap = p->spill_cap;
  kp.qcap = (int32_t)p->qcap;
  kp.BS = p->BS;
  kp.T = p->T;
  kp.flags = p->opt.flags;
  kp.collect_stats = p->opt.collect_stats;
  kp.nblocks = p->nblocks;
  return kp;
}

// Reset the per-call parts of the control block (keeps the epoch counter).
__global__ void k_reset_ctl(Ctl* ctl, Stats* stats) {
  ctl->minkey = kKeyMax;
  ctl->maxdeg = 0;
  ctl->status = 0;
  ctl->head = 0;
  ctl->done = 0;
  ctl->chain_total = 0;
  ctl->gbar_count = 0;
  ctl->solo_next = 0;
  ctl->n_chain = 0;
  ctl->n_solo = 0;
  ctl->n_comp = 0;
  ctl->spill_cursor = 0;
  ctl->incomplete = 0;
  if (stats) *stats = Stats{};
}

static rcm_status_t launch_scheduler(rcm_plan* p, const KParams& kp, cudaStream_t s) {
  k_scheduler<<<p->nblocks, kThreads, p->smem, s>>>(kp);
  CK(cudaGetLastError());
  return RCM_OK;
}

extern "C" rcm_status_t rcm_reorder(rcm_plan_t p, int32_t n, int64_t nnz, const int32_t* row_ptr,
                                    const int32_t* col_idx, rcm_start_t mode, int32_t start,
                                    int32_t* perm, int32_t* iperm, void* stream) {
  if (!p || !row_ptr || !perm || n <= 0 || nnz < 0 || (nnz > 0 && !col_idx)) return RCM_ERR_INVALID_ARGUMENT;
  if (n > p->n_max || nnz > p->nnz_max || nnz >= (1ll << 31)) return RCM_ERR_INVALID_ARGUMENT;
  if (mode < RCM_START_FIXED || mode > RCM_START_PSEUDO_PERIPHERAL) return RCM_ERR_INVALID_ARGUMENT;
  if (mode == RCM_START_FIXED && (start < 0 || start >= n)) return RCM_ERR_INVALID_ARGUMENT;
  cudaStream_t s = (cudaStream_t)stream;
  KParams kp = make_kparams(p, row_ptr, col_idx, perm, iperm);
  k_reset_ctl<<<1, 1, 0, s>>>(p->ctl, p->stats);
  const int vec = ((reinterpret_cast<uintptr_t>(row_ptr) & 15) == 0) ? 1 : 0;
  const int nthr4 = (n + 3) / 4;
  k_prologue<<<(nthr4 + 255) / 256, 256, 0, s>>>(row_ptr, n, nnz, p->word, p->ctl, p->opt.validate, vec);
  if (p->opt.validate >= 1 && nnz > 0)
    k_validate_cols<<<std::min<long long>((nnz + 255) / 256, 4096), 256, 0, s>>>(col_idx, nnz, n, p->ctl);
  if (p->opt.validate == 2)
    k_validate_sym<<<std::min((n + 255) / 256, 4096), 256, 0, s>>>(row_ptr, col_idx, n, p->ctl);
  const int32_t* gl_seed = nullptr;
  if (mode == RCM_START_PSEUDO_PERIPHERAL) {
    rcm_status_t st = gl_launch(p->comp, row_ptr, col_idx, n, p->word, p->ctl, nullptr, p->gl_out, s);
    if (st != RCM_OK) return st;
    gl_seed = p->gl_out;
  }
  const int thr = p->opt.solo_threshold == 0 ? 4096 : p->opt.solo_threshold;
  const int solo = (!(p->opt.flags & RCM_FLAG_FORCE_CHAIN) && thr > 0 && n <= thr) ? 1 : 0;
  k_setup_single<<<1, 1, 0, s>>>(p->chains, p->solos, p->ctl, n, (int)mode, start, solo, gl_seed);
  CK(cudaGetLastError());
  rcm_status_t st = launch_scheduler(p, kp, s);
  if (st != RCM_OK) return st;
  if (!solo) {
    // a13: components left over by the chain-first pass (C-6).  All kernels of
    // this stage exit immediately when the first pass ordered every node.
    st = comp_stage(p->comp, kp, n, nnz, (int)mode, thr, p->prob_cap, s);
    if (st != RCM_OK) return st;
    st = launch_scheduler(p, kp, s);
    if (st != RCM_OK) return st;
  }
  return RCM_OK;
}

extern "C" rcm_status_t rcm_reorder_batched(rcm_plan_t p, int32_t num_mats, int64_t total_nodes,
                                            int64_t total_nnz, const int64_t* node_off,
                                            const int64_t* nnz_off, const int32_t* row_ptr_local,
                                            const int32_t* col_idx_local, rcm_start_t mode,
                                            const int32_t* starts, int32_t* perm_local, void* stream) {
  if (!p || num_mats <= 0 || !node_off || !nnz_off || !row_ptr_local || !perm_local || total_nodes <= 0 ||
      total_nnz < 0 || (total_nnz > 0 && !col_idx_local))
    return RCM_ERR_INVALID_ARGUMENT;
  if (total_nodes > p->n_max || total_nnz > p->nnz_max || num_mats > p->prob_cap) return RCM_ERR_INVALID_ARGUMENT;
  if (mode < RCM_START_FIXED || mode > RCM_START_PSEUDO_PERIPHERAL) return RCM_ERR_INVALID_ARGUMENT;
  if (mode == RCM_START_FIXED && !starts) return RCM_ERR_INVALID_ARGUMENT;
  cudaStream_t s = (cudaStream_t)stream;
  KParams kp = make_kparams(p, row_ptr_local, col_idx_local, perm_local, nullptr);
  k_reset_ctl<<<1, 1, 0, s>>>(p->ctl, p->stats);
  CK(cudaMemsetAsync(p->pm_key, 0xff, sizeof(unsigned long long) * num_mats, s));
  const long long blocks = std::min<long long>((total_nodes + 255) / 256, 65535);
  k_prologue_batched<<<(int)blocks, 256, 0, s>>>(row_ptr_local, node_off, num_mats, total_nodes, p->word,
                                                 p->pm_key, p->ctl);
  const int32_t* order = nullptr;
  if (num_mats > 1) {
    // LPT: largest matrices first (the solo workers dequeue in this order)
    rcm_status_t st = comp_order_by_size(p->comp, node_off, num_mats, s);
    if (st != RCM_OK) return st;
    order = p->comp.order;
  }
  if (mode == RCM_START_PSEUDO_PERIPHERAL) {
    rcm_status_t st = gl_batched(p->comp, row_ptr_local, col_idx_local, node_off, nnz_off, num_mats,
                                 p->pm_key, s);
    if (st != RCM_OK) return st;
  }
  k_setup_batched<<<(num_mats + 255) / 256, 256, 0, s>>>(p->solos, p->ctl, node_off, nnz_off, num_mats,
                                                         (int)mode, starts, p->pm_key, order);
  CK(cudaGetLastError());
  return launch_scheduler(p, kp, s);
}

extern "C" rcm_status_t rcm_find_pseudo_peripheral(rcm_plan_t p, int32_t n, int64_t nnz,
                                                   const int32_t* row_ptr, const int32_t* col_idx,
                                                   int32_t start, int32_t* out, void* stream) {
  if (!p || !row_ptr || !out || n <= 0 || start < 0 || start >= n || nnz < 0 || (nnz > 0 && !col_idx))
    return RCM_ERR_INVALID_ARGUMENT;
  if (n > p->n_max || nnz > p->nnz_max) return RCM_ERR_INVALID_ARGUMENT;
  cudaStream_t s = (cudaStream_t)stream;
  k_reset_ctl<<<1, 1, 0, s>>>(p->ctl, nullptr);
  const int vec = ((reinterpret_cast<uintptr_t>(row_ptr) & 15) == 0) ? 1 : 0;
  k_prologue<<<((n + 3) / 4 + 255) / 256, 256, 0, s>>>(row_ptr, n, nnz, p->word, p->ctl, 0, vec);
  return gl_launch(p->comp, row_ptr, col_idx, n, p->word, p->ctl, &start, out, s);
}

extern "C" rcm_status_t rcm_sync_status(rcm_plan_t p, void* stream) {
  if (!p) return RCM_ERR_INVALID_ARGUMENT;
  CK(cudaStreamSynchronize((cudaStream_t)stream));
  int32_t st = 0;
  CK(cudaMemcpy(&st, &p->ctl->status, sizeof(int32_t), cudaMemcpyDeviceToHost));
  p->last_status = st;
  return (rcm_status_t)st;
}

extern "C" rcm_status_t rcm_get_stats(rcm_plan_t p, rcm_stats_t* out) {
  if (!p || !out) return RCM_ERR_INVALID_ARGUMENT;
  Stats s;
  CK(cudaMemcpy(&s, p->stats, sizeof(Stats), cudaMemcpyDeviceToHost));
  out->batches_generated = (int64_t)s.generated + 0;
  out->batches_dequeued = (int64_t)s.dequeued;
  out->batches_executed = (int64_t)s.executed;
  out->batches_empty = (int64_t)s.empty;
  out->rediscover_early = (int64_t)s.redisc_early;
  out->rediscover_late = (int64_t)s.redisc_late;
  out->candidates_speculative = (int64_t)s.cand_spec;
  out->candidates_removed = (int64_t)s.cand_removed;
  out->oversize_batches = (int64_t)s.oversize;
  out->components = (int64_t)s.components;
  out->overhang_forwards = (int64_t)s.ovh_forwards;
  out->solo_problems = (int64_t)s.solo_problems;
  return RCM_OK;
}

extern "C" rcm_status_t rcm_plan_info(rcm_plan_t p, int64_t* out6) {
  if (!p || !out6) return RCM_ERR_INVALID_ARGUMENT;
  out6[0] = p->nblocks;
  out6[1] = kThreads;
  out6[2] = p->BS;
  out6[3] = p->T;
  out6[4] = (int64_t)p->smem;
  out6[5] = p->qcap;
  return RCM_OK;
}
