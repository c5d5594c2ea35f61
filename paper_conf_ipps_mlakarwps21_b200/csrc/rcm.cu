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
#include "rcm_solo.cuh"

using namespace rcm;

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
  uint32_t* fwdv = nullptr;
  Ctl* ctl = nullptr;
  Stats* stats = nullptr;
  Problem* chains = nullptr;
  Problem* solos = nullptr;
  unsigned long long* spill = nullptr;
  int32_t* dbg = nullptr;
  unsigned long long* trace = nullptr;
  int32_t trace_cap = 0;
  const void* kernel = nullptr;
  CompWS w{};
  // batched / small-graph path (rcm_solo.cuh)
  int solo_blocks = 0;
  size_t solo_smem = 0;
  int64_t mats_cap = 0, gvis_words = 0;
  int32_t* order = nullptr;
  uint32_t* gvis = nullptr;
  int2* pend = nullptr;
  int solo_BS = 256;
  bool batched_only = false;
  cudaStream_t s_copy = nullptr, s_kern = nullptr, s_back = nullptr;   // rcm_reorder_batched_host
  size_t smem_optin = 0;   // largest dynamic shared memory of one block
};

static rcm_status_t cuda_fail(cudaError_t e) {
  if (e == cudaErrorMemoryAllocation) return RCM_ERR_OUT_OF_MEMORY;
  return RCM_ERR_CUDA;
}
#define CK(x)                                    \
  do {                                           \
    cudaError_t _e = (x);                        \
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

static void free_all(rcm_plan* p) {
  void* ptrs[] = {p->fwdv, p->pend, p->order, p->gvis, p->trace, p->dbg, p->word, p->o, p->desc, p->sig, p->ctl, p->stats, p->chains, p->solos, p->spill,
                  p->w.label, p->w.ckey, p->w.csize, p->w.keys0, p->w.keys1, p->w.vals0, p->w.vals1,
                  p->w.offs, p->w.hist, p->w.sctl, p->w.lev, p->w.front0, p->w.front1,
                  p->w.gctl, p->w.gkey};
  for (void* q : ptrs) cudaFree(q);
}

extern "C" void rcm_plan_destroy(rcm_plan_t p) {
  if (!p) return;
  for (cudaStream_t s : {p->s_copy, p->s_kern, p->s_back})
    if (s) cudaStreamDestroy(s);
  free_all(p);
  delete p;
}

// k_main instantiations (k_main_inst.cu, one translation unit each): 1 or 2
// resident blocks per SM (register budget 64K / (bps * kThreads)), with or
// traversal mode 0 chain / 1 multi-batch chain / 2 leveled.
extern "C" const void* rcm_kmain_ptr_1_0();
extern "C" const void* rcm_kmain_ptr_2_0();
extern "C" const void* rcm_kmain_ptr_1_1();
extern "C" const void* rcm_kmain_ptr_2_1();
extern "C" const void* rcm_kmain_ptr_1_2();
extern "C" const void* rcm_kmain_ptr_2_2();
extern "C" const void* rcm_ksolo_order_ptr();
extern "C" const void* rcm_ksolo_ptr();
extern "C" size_t rcm_ksolo_smem();
extern "C" int rcm_ksolo_threads();
extern "C" int rcm_ksolo_nmax();
extern "C" const void* rcm_ksolo_sm_ptr();
static const void* pick_kernel(int bps, bool mb, bool lv) {
  static_assert(1024 / kThreads >= 2, "two 512-thread blocks per SM");
  if (lv) return bps >= 2 ? rcm_kmain_ptr_2_2() : rcm_kmain_ptr_1_2();
  if (mb) return bps >= 2 ? rcm_kmain_ptr_2_1() : rcm_kmain_ptr_1_1();
  return bps == 2 ? rcm_kmain_ptr_2_0() : rcm_kmain_ptr_1_0();
}

static rcm_status_t plan_alloc(rcm_plan* p) {
  const rcm_options_t& o = p->opt;
  const int64_t n = p->n_max;
#define AL(ptr, bytes)                                          \
  do {                                                          \
    cudaError_t _e = cudaMalloc((void**)&(ptr), (size_t)(bytes)); \
    if (_e != cudaSuccess) return cuda_fail(_e);                \
  } while (0)
  // shared by both paths
  AL(p->ctl, sizeof(Ctl));
  AL(p->stats, sizeof(Stats));
  AL(p->dbg, 4 * 8 * 1024);
  AL(p->spill, 8 * 2 * p->spill_cap);
  // batched / small-graph path (rcm_solo.cuh)
  AL(p->order, 4 * p->mats_cap);
  AL(p->gvis, 4 * 2 * p->gvis_words);
  AL(p->pend, 8 * n);
  if (!p->batched_only) {   // multi-block chain + components + GL finder
    const int64_t tiles = (n + kSortTile - 1) / kSortTile + 1;
    AL(p->word, 8 * n);
    AL(p->o, 4 * n);
    AL(p->desc, sizeof(Desc) * p->qcap);
    AL(p->sig, sizeof(Sig) * (p->qcap + 1));
    AL(p->fwdv, 8 * (p->qcap + 1));
    AL(p->chains, sizeof(Problem) * p->prob_cap);
    AL(p->solos, sizeof(Problem) * p->prob_cap);
    if (o.collect_stats == 3) {
      p->trace_cap = (int32_t)std::min<int64_t>(p->qcap, 1 << 20);
      AL(p->trace, 8 * kTraceW * (size_t)p->trace_cap);
    }
    AL(p->w.label, 4 * n); AL(p->w.ckey, 8 * n); AL(p->w.csize, 4 * n);
    AL(p->w.keys0, 8 * n); AL(p->w.keys1, 8 * n); AL(p->w.vals0, 4 * n); AL(p->w.vals1, 4 * n);
    AL(p->w.offs, 8 * (n + 1 + 1024)); AL(p->w.hist, 4 * std::max<int64_t>(256 * tiles, 4 * kMaxBlocks));
    AL(p->w.sctl, 4 * 64);
    AL(p->w.lev, 4 * n); AL(p->w.front0, 4 * n); AL(p->w.front1, 4 * n);
    AL(p->w.gctl, 4 * 64); AL(p->w.gkey, 8 * 64);
    p->w.cap = n;
    // descriptors / signals start with tag 0 (epochs start at 1)
    CK(cudaMemset(p->desc, 0, sizeof(Desc) * p->qcap));
    CK(cudaMemset(p->sig, 0, sizeof(Sig) * (p->qcap + 1)));
  }
#undef AL
  CK(cudaMemset(p->ctl, 0, sizeof(Ctl)));
  CK(cudaMemset(p->stats, 0, sizeof(Stats)));
  CK(cudaMemset(p->dbg, 0, 4 * 8 * 1024));
  CK(cudaDeviceSynchronize());
  return RCM_OK;
}

extern "C" rcm_status_t rcm_plan_create(rcm_plan_t* out, int64_t n_max, int64_t nnz_max,
                                        const rcm_options_t* opt_in) {
  if (!out || n_max <= 0 || nnz_max < 0 || n_max >= (1ll << 31) - 2) return RCM_ERR_INVALID_ARGUMENT;
  *out = nullptr;
  rcm_plan* p = new (std::nothrow) rcm_plan();
  if (!p) return RCM_ERR_OUT_OF_MEMORY;
  if (opt_in) p->opt = *opt_in;
  const rcm_options_t& o = p->opt;
  if (o.batch_nodes < 0 || o.batch_nodes > kMaxBatchNodes || o.temp_elems < 0 || o.blocks_per_sm < 0 ||
      o.blocks_per_sm > 4 || o.validate < 0 || o.validate > 2 || o.queue_capacity < 0) {
    delete p;
    return RCM_ERR_INVALID_ARGUMENT;
  }
  p->n_max = n_max;
  p->nnz_max = nnz_max;
  p->batched_only = (o.flags & RCM_FLAG_BATCHED_ONLY) != 0;
  if (cudaGetDevice(&p->device) != cudaSuccess) { delete p; return RCM_ERR_CUDA; }
  cudaDeviceGetAttribute(&p->num_sms, cudaDevAttrMultiProcessorCount, p->device);
  int smem_optin = 0, smem_sm = 0;
  cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, p->device);
  cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, p->device);
  // ---- batched / small-graph path: many blocks per SM, shared-memory bitmap
  p->solo_smem = rcm_ksolo_smem();
  if (cudaFuncSetAttribute(rcm_ksolo_ptr(), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->solo_smem) !=
      cudaSuccess) {
    delete p;
    return RCM_ERR_CUDA;
  }
  int occ_s = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_s, rcm_ksolo_ptr(), rcm_ksolo_threads(), p->solo_smem);
  if (occ_s <= 0) { delete p; return RCM_ERR_CUDA; }
  p->solo_blocks = occ_s * p->num_sms;
  p->smem_optin = (size_t)smem_optin - 4096;   // room for the kernel's static shared memory
  if (cudaFuncSetAttribute(rcm_ksolo_sm_ptr(), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->smem_optin) !=
      cudaSuccess) {
    delete p;
    return RCM_ERR_CUDA;
  }
  p->solo_BS = o.batch_nodes ? std::min(o.batch_nodes, rcm_ksolo_threads()) : rcm_ksolo_threads();
  p->mats_cap = n_max + 1;
  p->gvis_words = n_max / 32 + 2;   // bitmaps packed over all nodes (one bit each)
  // oversize scratch: children of oversize parents (<= n) + claims bitmaps of
  // rows longer than the shared-memory bitmap (<= nnz / 64 u64 words)
  p->spill_cap = n_max + (p->batched_only ? 0 : nnz_max / 64 + 64);
  // ---- multi-block chain path
  if (!p->batched_only) {
    const bool dense = !o.temp_elems && !o.batch_nodes && nnz_max >= 20 * n_max;
    // dense rows (FEM-like): smaller batches shorten the critical generation
    // chain
    p->BS = o.batch_nodes ? o.batch_nodes : dense ? 192 : 256;
    const int bps = o.blocks_per_sm ? o.blocks_per_sm : 2;
    const size_t static_sh = 2 * sizeof(ShState) + 64;
    const int nctx = (o.flags & RCM_FLAG_MULTI_BATCH) ? 2 : 1;   // batch contexts per block
    // T from the shared-memory budget of `bps` blocks per SM (1 KB reserved per
    // block), 10 B per slot (candidate key, local parent id)
    const size_t per_block =
        std::min<size_t>((size_t)smem_sm / bps - 1024 - static_sh, (size_t)smem_optin - static_sh);
    int T = o.temp_elems;
    if (!T) T = (int)((per_block / nctx - 16 - smem_bytes(p->BS, 0)) / 10) / 256 * 256;
    // dense: B_s rows of ~27 fit; the shared memory left over serves as L1
    if (dense) T = std::min(T, 6144);
    // sparse rows at the default occupancy: a budget past ~7.7 k candidates buys
    // few extra parents per batch but takes the SM's L1 (r01d sweep, DESIGN.md
    // "batch limits": C3 10.9 -> 9.6 ms, C4 unchanged)
    else if (!o.temp_elems && !o.blocks_per_sm && nctx == 1) T = std::min(T, 7680);
    if (T < 2304 || smem_bytes(p->BS, T) > (size_t)smem_optin - static_sh) {
      delete p;
      return RCM_ERR_INVALID_ARGUMENT;
    }
    p->T = T;
    p->smem = nctx == 1 ? smem_bytes(p->BS, T) : nctx * ((smem_bytes(p->BS, T) + 15) & ~size_t(15));
    if (o.flags & RCM_FLAG_LEVELED) p->smem = lv_smem_base(p->BS, T) + kLvExtraBytes;   // + staging (rcm_leveled.cuh)
    // one block per SM: the 128-register build (no spills); more: the 64-register build
    p->kernel = pick_kernel(bps, nctx == 2, (o.flags & RCM_FLAG_LEVELED) != 0);
    if (cudaFuncSetAttribute(p->kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)p->smem) != cudaSuccess) {
      delete p;
      return RCM_ERR_CUDA;
    }
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, p->kernel, kThreads, p->smem);
    if (occ <= 0) { delete p; return RCM_ERR_CUDA; }
    p->nblocks = std::min(occ, bps) * p->num_sms;   // persistent: every block co-resident
    if (p->nblocks > kMaxBlocks) p->nblocks = kMaxBlocks / p->num_sms * p->num_sms;   // beacon / scratch sizing
    // queue bound: sum over generating batches of floor(N/B) + max(1, ceil(2V/T))
    const int64_t qb = 2 * n_max + n_max / p->BS + 2 * (nnz_max / T + 1) + 64;
    // the Counted payload packs queue offsets in 30 bits (rcm_device.cuh sig_pack,
    // rcm_lookback.cuh lb_pfx): the queue never exceeds 2^30 - 1 slots
    p->qcap = std::min<int64_t>(o.queue_capacity ? o.queue_capacity : qb, (1ll << 30) - 1);
    p->prob_cap = std::max<int64_t>(1, n_max / 2 + 1);
  }
  if (cudaStreamCreateWithFlags(&p->s_copy, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&p->s_kern, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&p->s_back, cudaStreamNonBlocking) != cudaSuccess) {
    rcm_plan_destroy(p);
    return RCM_ERR_CUDA;
  }
  const rcm_status_t st = plan_alloc(p);
  if (st != RCM_OK) {
    rcm_plan_destroy(p);
    return st;
  }
  *out = p;
  return RCM_OK;
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
  kp.Bg = p->BS;
  kp.Tg = p->T;
  kp.flags = p->opt.flags;
  kp.collect_stats = p->opt.collect_stats;
  kp.nblocks = p->nblocks;
  kp.dbg = p->dbg;
  kp.trace = p->trace;
  kp.trace_cap = p->trace_cap;
  kp.fwdv = p->fwdv;
  return kp;
}

static MainArgs make_args(rcm_plan* p) {
  MainArgs a;
  std::memset(&a, 0, sizeof(a));
  a.w = p->w;
  a.prob_cap = p->prob_cap;
  a.validate = p->opt.validate;
  a.thr = p->opt.solo_threshold == 0 ? 4096 : p->opt.solo_threshold;
  return a;
}

static int bits_for(int64_t x) {
  int b = 0;
  while (b < 62 && (1ll << b) <= x) ++b;
  return b;
}

// Cooperative launch: the runtime guarantees every block of the persistent
// grid is co-resident (grid barriers and spin-waits rely on it) or fails.
static rcm_status_t launch_main(rcm_plan* p, const KParams& kp, const MainArgs& a, cudaStream_t s) {
  if (p->trace) CK(cudaMemsetAsync(p->trace, 0, 8 * kTraceW * (size_t)p->trace_cap, s));
  KParams kpc = kp;
  MainArgs ac = a;
  void* args[] = {&kpc, &ac};
  CK(cudaLaunchCooperativeKernel(p->kernel, dim3(p->nblocks), dim3(kThreads), args, p->smem, s));
  return RCM_OK;
}

// The batched / small-graph path: k_solo_order (reset + largest-first order)
// then k_solo on every SM (rcm_solo.cuh).  Regular launches: no block waits
// for another, so co-residency is not required.
static rcm_status_t launch_solo(rcm_plan* p, SoloArgs& sa, cudaStream_t s) {
  sa.order = p->order;
  sa.gvis = p->gvis;
  sa.gvis_words = p->gvis_words;
  sa.spill = p->spill;
  sa.spill_cap = p->spill_cap;
  sa.pend = p->pend;
  sa.ctl = p->ctl;
  sa.stats = p->stats;
  sa.validate = p->opt.validate;
  sa.collect_stats = p->opt.collect_stats;
  sa.flags = p->opt.flags;
  sa.BS = p->solo_BS;
  void* args[] = {&sa};
  CK(cudaLaunchKernel(rcm_ksolo_order_ptr(), dim3(1), dim3(1024), args, 0, s));
  CK(cudaLaunchKernel(rcm_ksolo_ptr(), dim3(p->solo_blocks), dim3(rcm_ksolo_threads()), args, p->solo_smem, s));
  return RCM_OK;
}

extern "C" rcm_status_t rcm_reorder(rcm_plan_t p, int32_t n, int64_t nnz, const int32_t* row_ptr,
                                    const int32_t* col_idx, rcm_start_t mode, int32_t start,
                                    int32_t* perm, int32_t* iperm, void* stream) {
  if (!p || !row_ptr || !perm || n <= 0 || nnz < 0 || (nnz > 0 && !col_idx)) return RCM_ERR_INVALID_ARGUMENT;
  if (n > p->n_max || nnz > p->nnz_max || nnz >= (1ll << 31)) return RCM_ERR_INVALID_ARGUMENT;
  if (mode < RCM_START_FIXED || mode > RCM_START_PSEUDO_PERIPHERAL) return RCM_ERR_INVALID_ARGUMENT;
  if (mode == RCM_START_FIXED && (start < 0 || start >= n)) return RCM_ERR_INVALID_ARGUMENT;
  const int thr = p->opt.solo_threshold == 0 ? 4096 : p->opt.solo_threshold;
  const bool solo = !(p->opt.flags & RCM_FLAG_FORCE_CHAIN) && thr > 0 && n <= thr;
  if (solo) {   // one block orders the whole graph (small graphs, e.g. config 1)
    SoloArgs sa;
    std::memset(&sa, 0, sizeof(sa));
    sa.row_ptr = row_ptr;
    sa.col_idx = col_idx;
    sa.perm = perm;
    sa.iperm = iperm;
    sa.num_mats = 1;
    sa.n = n;
    sa.nnz = nnz;
    sa.mode = (int)mode;
    sa.start = start;
    // the whole CSR fits in shared memory next to the batch scratch: one block,
    // no global round trip per batch (k_solo_sm)
    const size_t csr = 4 * (((size_t)n + 1 + 3) / 4 * 4) + 4 * (size_t)nnz;
    if (p->solo_smem + csr <= p->smem_optin && n <= rcm_ksolo_nmax()) {
      sa.order = p->order; sa.gvis = p->gvis; sa.gvis_words = p->gvis_words; sa.spill = p->spill;
      sa.spill_cap = p->spill_cap; sa.pend = p->pend; sa.ctl = p->ctl; sa.stats = p->stats;
      sa.validate = p->opt.validate; sa.collect_stats = p->opt.collect_stats; sa.flags = p->opt.flags;
      sa.BS = p->solo_BS;
      void* args[] = {&sa};
      CK(cudaLaunchKernel(rcm_ksolo_sm_ptr(), dim3(1), dim3(rcm_ksolo_threads()), args, p->solo_smem + csr,
                          (cudaStream_t)stream));
      return RCM_OK;
    }
    return launch_solo(p, sa, (cudaStream_t)stream);
  }
  if (p->batched_only) return RCM_ERR_INVALID_ARGUMENT;   // no chain workspace in this plan
  KParams kp = make_kparams(p, row_ptr, col_idx, perm, iperm);
  if (!p->opt.batch_nodes && !p->opt.temp_elems && nnz >= 20ll * n) {
    // dense rows (FEM-like, average valence >= 20) on a plan sized for sparser
    // graphs: cut smaller batches
    kp.Bg = std::min(kp.BS, 192);
    kp.Tg = std::min(kp.T, 6144);
  }
  MainArgs a = make_args(p);
  a.n = n;
  a.nnz = nnz;
  a.mode = (int)mode;
  a.start = start;
  a.vec = ((reinterpret_cast<uintptr_t>(row_ptr) & 15) == 0) ? 1 : 0;
  a.idbits = bits_for(n - 1 > 0 ? n - 1 : 1);
  return launch_main(p, kp, a, (cudaStream_t)stream);
}

extern "C" rcm_status_t rcm_reorder_batched(rcm_plan_t p, int32_t num_mats, int64_t total_nodes,
                                            int64_t total_nnz, const int64_t* node_off,
                                            const int64_t* nnz_off, const int32_t* row_ptr_local,
                                            const int32_t* col_idx_local, rcm_start_t mode,
                                            const int32_t* starts, int32_t* perm_local, void* stream) {
  if (!p || num_mats <= 0 || !node_off || !nnz_off || !row_ptr_local || !perm_local || total_nodes < 0 ||
      total_nnz < 0 || (total_nnz > 0 && !col_idx_local))
    return RCM_ERR_INVALID_ARGUMENT;
  if (total_nodes > p->n_max || total_nnz > p->nnz_max || num_mats > p->mats_cap - 1)
    return RCM_ERR_INVALID_ARGUMENT;
  if (mode < RCM_START_FIXED || mode > RCM_START_PSEUDO_PERIPHERAL) return RCM_ERR_INVALID_ARGUMENT;
  if (mode == RCM_START_FIXED && !starts) return RCM_ERR_INVALID_ARGUMENT;
  SoloArgs sa;
  std::memset(&sa, 0, sizeof(sa));
  sa.row_ptr = row_ptr_local;
  sa.col_idx = col_idx_local;
  sa.perm = perm_local;
  sa.node_off = node_off;
  sa.nnz_off = nnz_off;
  sa.starts = starts;
  sa.num_mats = num_mats;
  sa.mode = (int)mode;
  return launch_solo(p, sa, (cudaStream_t)stream);
}

// Host-resident batch with copy/compute overlap: the batch is cut into
// `chunks` ranges of matrices of about equal nnz; the H2D copy of range g+1
// (copy stream) runs while range g is ordered (kernel stream), and range g's
// permutations go back on a third stream.  Everything is ordered after the
// work already enqueued on `stream`, and `stream` waits for all of it.
extern "C" rcm_status_t rcm_reorder_batched_host(rcm_plan_t p, int32_t num_mats, const int64_t* node_off_h,
                                                 const int64_t* nnz_off_h, const int32_t* row_ptr_h,
                                                 const int32_t* col_idx_h, rcm_start_t mode, const int32_t* starts_h,
                                                 int32_t* perm_h, int64_t* node_off_d, int64_t* nnz_off_d,
                                                 int32_t* row_ptr_d, int32_t* col_idx_d, int32_t* starts_d,
                                                 int32_t* perm_d, int32_t chunks, void* stream) {
  if (!p || num_mats <= 0 || !node_off_h || !nnz_off_h || !row_ptr_h || !perm_h || !node_off_d || !nnz_off_d ||
      !row_ptr_d || !perm_d || chunks <= 0)
    return RCM_ERR_INVALID_ARGUMENT;
  const int64_t total = node_off_h[num_mats], total_nnz = nnz_off_h[num_mats];
  if (total < 0 || total_nnz < 0 || (total_nnz > 0 && (!col_idx_h || !col_idx_d))) return RCM_ERR_INVALID_ARGUMENT;
  if (total > p->n_max || total_nnz > p->nnz_max || num_mats > p->mats_cap - 1) return RCM_ERR_INVALID_ARGUMENT;
  if (mode < RCM_START_FIXED || mode > RCM_START_PSEUDO_PERIPHERAL) return RCM_ERR_INVALID_ARGUMENT;
  if (mode == RCM_START_FIXED && (!starts_h || !starts_d)) return RCM_ERR_INVALID_ARGUMENT;
  chunks = std::min(chunks, std::min<int32_t>(num_mats, 64));
  cudaStream_t cs = p->s_copy, ks = p->s_kern, bs = p->s_back, us = (cudaStream_t)stream;
  cudaEvent_t ev[2 * 64 + 4];
  int nev = 0;
  auto mk = [&]() -> cudaEvent_t {
    cudaEvent_t e = nullptr;
    cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    ev[nev++] = e;
    return e;
  };
  cudaEvent_t e0 = mk();
  CK(cudaEventRecord(e0, us));
  CK(cudaStreamWaitEvent(cs, e0, 0));
  CK(cudaStreamWaitEvent(ks, e0, 0));
  CK(cudaStreamWaitEvent(bs, e0, 0));
  CK(cudaMemcpyAsync(node_off_d, node_off_h, 8 * (size_t)(num_mats + 1), cudaMemcpyHostToDevice, cs));
  CK(cudaMemcpyAsync(nnz_off_d, nnz_off_h, 8 * (size_t)(num_mats + 1), cudaMemcpyHostToDevice, cs));
  if (starts_h && starts_d) CK(cudaMemcpyAsync(starts_d, starts_h, 4 * (size_t)num_mats, cudaMemcpyHostToDevice, cs));
  int32_t m0 = 0;
  for (int g = 0; g < chunks; ++g) {
    // end of range g: the first matrix whose nnz prefix reaches (g+1)/chunks of the total
    int32_t m1 = num_mats;
    if (g + 1 < chunks) {
      const int64_t target = total_nnz / chunks * (g + 1);
      m1 = (int32_t)(std::lower_bound(nnz_off_h, nnz_off_h + num_mats + 1, target) - nnz_off_h);
      m1 = std::max(m1, m0 + 1);
      m1 = std::min(m1, num_mats - (chunks - 1 - g));
    }
    const int64_t r0 = node_off_h[m0] + m0, r1 = node_off_h[m1] + m1;   // row_ptr entries
    const int64_t c0 = nnz_off_h[m0], c1 = nnz_off_h[m1];
    CK(cudaMemcpyAsync(row_ptr_d + r0, row_ptr_h + r0, 4 * (size_t)(r1 - r0), cudaMemcpyHostToDevice, cs));
    if (c1 > c0) CK(cudaMemcpyAsync(col_idx_d + c0, col_idx_h + c0, 4 * (size_t)(c1 - c0), cudaMemcpyHostToDevice, cs));
    cudaEvent_t ec = mk();
    CK(cudaEventRecord(ec, cs));
    CK(cudaStreamWaitEvent(ks, ec, 0));
    SoloArgs sa;
    std::memset(&sa, 0, sizeof(sa));
    sa.col_idx = col_idx_d;
    sa.perm = perm_d;
    sa.node_off = node_off_d + m0;
    sa.nnz_off = nnz_off_d + m0;
    sa.starts = starts_d ? starts_d + m0 : nullptr;
    sa.num_mats = m1 - m0;
    sa.mode = (int)mode;
    sa.chunk = g;
    // matrix k of the range is global matrix m0 + k: its row_ptr starts at
    // node_off[m0 + k] + m0 + k -- shift the row_ptr base by m0 for the kernel's
    // node_off[k] + k indexing
    sa.row_ptr = row_ptr_d + m0;
    const rcm_status_t st = launch_solo(p, sa, ks);
    if (st != RCM_OK) return st;
    cudaEvent_t ek = mk();
    CK(cudaEventRecord(ek, ks));
    CK(cudaStreamWaitEvent(bs, ek, 0));
    const int64_t n0 = node_off_h[m0], n1 = node_off_h[m1];
    if (n1 > n0) CK(cudaMemcpyAsync(perm_h + n0, perm_d + n0, 4 * (size_t)(n1 - n0), cudaMemcpyDeviceToHost, bs));
    m0 = m1;
  }
  cudaEvent_t eb = mk(), ek = mk();
  CK(cudaEventRecord(eb, bs));
  CK(cudaEventRecord(ek, ks));
  CK(cudaStreamWaitEvent(us, eb, 0));
  CK(cudaStreamWaitEvent(us, ek, 0));
  for (int i = 0; i < nev; ++i) cudaEventDestroy(ev[i]);   // released once completed
  return RCM_OK;
}

extern "C" rcm_status_t rcm_find_pseudo_peripheral(rcm_plan_t p, int32_t n, int64_t nnz,
                                                   const int32_t* row_ptr, const int32_t* col_idx,
                                                   int32_t start, int32_t* out, void* stream) {
  if (!p || !row_ptr || !out || n <= 0 || start < 0 || start >= n || nnz < 0 || (nnz > 0 && !col_idx))
    return RCM_ERR_INVALID_ARGUMENT;
  if (n > p->n_max || nnz > p->nnz_max || p->batched_only) return RCM_ERR_INVALID_ARGUMENT;
  KParams kp = make_kparams(p, row_ptr, col_idx, nullptr, nullptr);
  MainArgs a = make_args(p);
  a.n = n;
  a.nnz = nnz;
  a.mode = RCM_START_PSEUDO_PERIPHERAL;
  a.vec = ((reinterpret_cast<uintptr_t>(row_ptr) & 15) == 0) ? 1 : 0;
  a.gl_only = 1;
  a.gl_start = start;
  a.gl_out = out;
  a.validate = 0;
  return launch_main(p, kp, a, (cudaStream_t)stream);
}

extern "C" rcm_status_t rcm_sync_status(rcm_plan_t p, void* stream) {
  if (!p) return RCM_ERR_INVALID_ARGUMENT;
  CK(cudaStreamSynchronize((cudaStream_t)stream));
  int32_t st = 0;
  CK(cudaMemcpy(&st, &p->ctl->status, sizeof(int32_t), cudaMemcpyDeviceToHost));
  return (rcm_status_t)st;
}

extern "C" rcm_status_t rcm_get_stats(rcm_plan_t p, rcm_stats_t* out) {
  if (!p || !out) return RCM_ERR_INVALID_ARGUMENT;
  Stats s;
  CK(cudaMemcpy(&s, p->stats, sizeof(Stats), cudaMemcpyDeviceToHost));
  out->batches_generated = (int64_t)s.generated;
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
  for (int i = 0; i < 10; ++i) out->stage_cycles[i] = (int64_t)s.stage[i];
  return RCM_OK;
}

extern "C" rcm_status_t rcm_get_timing(rcm_plan_t p, double* out_ms) {
  if (!p || !out_ms) return RCM_ERR_INVALID_ARGUMENT;
  unsigned long long ts[8];
  CK(cudaMemcpy(ts, p->ctl->ts, sizeof(ts), cudaMemcpyDeviceToHost));
  // [prologue, seed + set-up, traversal, components + their traversal, total,
  //  component labelling, component sort + layout]
  auto d = [&](int a, int b) { return ts[b] >= ts[a] ? (double)(ts[b] - ts[a]) * 1e-6 : 0.0; };
  const bool cc = ts[5] >= ts[3] && ts[6] >= ts[5] && ts[4] >= ts[6];
  out_ms[0] = d(0, 1);
  out_ms[1] = d(1, 2);
  out_ms[2] = d(2, 3);
  out_ms[3] = d(3, 4);
  out_ms[4] = d(0, 4);
  out_ms[5] = cc ? d(3, 5) : 0.0;
  out_ms[6] = cc ? d(5, 6) : 0.0;
  return RCM_OK;
}

// Watchdog diagnostics of the last call (8 host int64): site (1 dequeue,
// 2 look-back Discovered, 3 look-back prefix, 4 grid barrier, 5 serial chain
// wait), slot, index, word, block.  Not part of the public header.
extern "C" rcm_status_t rcm_debug_info(rcm_plan_t p, long long* out8) {
  if (!p || !out8) return RCM_ERR_INVALID_ARGUMENT;
  CK(cudaMemcpy(out8, p->ctl->dbg, 8 * sizeof(long long), cudaMemcpyDeviceToHost));
  return RCM_OK;
}

// Per-block progress beacons (nblocks x 8 int32: phase, slot, aux, count,
// look-back j, word, iterations), copied on a private non-blocking stream so
// it can be read while a launch is still running.  Not in the public header.
extern "C" rcm_status_t rcm_debug_state(rcm_plan_t p, int32_t* host_out, int32_t* nblocks) {
  if (!p || !host_out) return RCM_ERR_INVALID_ARGUMENT;
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaError_t e = cudaMemcpyAsync(host_out, p->dbg, 4 * 8 * p->nblocks, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaStreamDestroy(s);
  if (nblocks) *nblocks = p->nblocks;
  return e == cudaSuccess ? RCM_OK : RCM_ERR_CUDA;
}

// Per-slot event trace of the last call (collect_stats == 3): copies
// min(cnt, trace_cap) * kTraceW u64.  Debug / analysis only.
extern "C" rcm_status_t rcm_debug_trace(rcm_plan_t p, int32_t cnt, unsigned long long* host_out) {
  if (!p || !host_out || !p->trace) return RCM_ERR_INVALID_ARGUMENT;
  const int32_t c = std::min(cnt, p->trace_cap);
  CK(cudaMemcpy(host_out, p->trace, 8 * kTraceW * (size_t)c, cudaMemcpyDeviceToHost));
  return RCM_OK;
}

// Raw chain slot state (desc + both status words) for slots [lo, lo+cnt):
// 6 int64 per slot.  Debug only; copied on a private stream.
extern "C" rcm_status_t rcm_debug_slots(rcm_plan_t p, int32_t lo, int32_t cnt, long long* host_out) {
  if (!p || !host_out || !p->sig || lo < 0 || cnt <= 0 || lo + cnt > p->qcap) return RCM_ERR_INVALID_ARGUMENT;
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  Sig* sg = (Sig*)malloc(sizeof(Sig) * cnt);
  Desc* dd = (Desc*)malloc(sizeof(Desc) * cnt);
  cudaMemcpyAsync(sg, p->sig + lo, sizeof(Sig) * cnt, cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(dd, p->desc + lo, sizeof(Desc) * cnt, cudaMemcpyDeviceToHost, s);
  Ctl c;
  cudaMemcpyAsync(&c, p->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s);
  cudaError_t e = cudaStreamSynchronize(s);
  cudaStreamDestroy(s);
  for (int i = 0; i < cnt; ++i) {
    host_out[6 * i + 0] = (long long)sg[i].word;
    host_out[6 * i + 1] = (long long)sg[i].ovh;
    host_out[6 * i + 2] = dd[i].o_begin;
    host_out[6 * i + 3] = dd[i].o_end;
    host_out[6 * i + 4] = dd[i].next;
    host_out[6 * i + 5] = dd[i].tag;
  }
  host_out[6 * cnt] = c.head; host_out[6 * cnt + 1] = c.done; host_out[6 * cnt + 2] = c.qtail;
  host_out[6 * cnt + 3] = c.completed; host_out[6 * cnt + 4] = c.epoch; host_out[6 * cnt + 5] = c.status;
  free(sg); free(dd);
  return e == cudaSuccess ? RCM_OK : RCM_ERR_CUDA;
}

extern "C" rcm_status_t rcm_plan_info(rcm_plan_t p, int64_t* out8) {
  if (!p || !out8) return RCM_ERR_INVALID_ARGUMENT;
  out8[0] = p->nblocks;
  out8[1] = kThreads;
  out8[2] = p->BS;
  out8[3] = p->T;
  out8[4] = (int64_t)p->smem;
  out8[5] = p->qcap;
  out8[6] = p->solo_blocks;
  out8[7] = (int64_t)p->solo_smem;
  return RCM_OK;
}
