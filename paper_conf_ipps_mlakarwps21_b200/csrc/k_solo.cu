// k_solo.cu -- kernels of the batched / small-graph path (rcm_solo.cuh):
//   k_solo_order  one block: per-call reset of the control block and the
//                 processing order of the matrices, largest first (LPT by
//                 size class, so the longest traversals start first);
//   k_solo        persistent blocks, each dequeues matrices in that order and
//                 orders one matrix at a time.
#include "../../include/rcm.h"
#include "rcm_solo.cuh"

namespace rcm {

#ifndef RCM_SOLO_MINB
#define RCM_SOLO_MINB 5
#endif

__global__ void __launch_bounds__(1024) k_solo_order(const __grid_constant__ SoloArgs a) {
  __shared__ int32_t hist[33];
  if (threadIdx.x == 0) {
    Ctl* c = a.ctl;
    c->solo_next = 0;
    if (a.chunk == 0) {
      c->ts[0] = globaltimer();
      c->ts[1] = c->ts[0];
      c->ts[2] = ~0ull;
      c->ts[3] = c->ts[4] = c->ts[5] = c->ts[6] = 0;
      c->status = 0;
      c->done = 0;
      c->n_chain = 0;
      c->n_solo = 0;
      if (a.collect_stats) *a.stats = Stats{};
    }
  }
  if (threadIdx.x < 33) hist[threadIdx.x] = 0;
  __syncthreads();
  const int M = a.num_mats;
  // size class c = bit length of n_k (1..32, 0 for an empty matrix); bucket
  // 32 - c puts the largest classes first
  auto bucket = [&](int k) -> int {
    const long long n = a.node_off ? a.node_off[k + 1] - a.node_off[k] : a.n;
    return n > 0 ? 32 - (64 - __clzll(n)) : 32;
  };
  for (int k = threadIdx.x; k < M; k += blockDim.x) atomicAdd(&hist[max(0, bucket(k))], 1);
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int b = 0; b < 33; ++b) { const int x = hist[b]; hist[b] = run; run += x; }
  }
  __syncthreads();
  for (int k = threadIdx.x; k < M; k += blockDim.x) a.order[atomicAdd(&hist[max(0, bucket(k))], 1)] = k;
}

__global__ void __launch_bounds__(kSoloNT, RCM_SOLO_MINB) k_solo(const __grid_constant__ SoloArgs a) {
  __shared__ SoloSh sh;
  if (threadIdx.x == 0) {
    sh.st_exec = sh.st_comp = sh.st_over = sh.st_claim = sh.st_comb = 0;
    atomicMin(&a.ctl->ts[2], globaltimer());
  }
  long long mats = 0;
  for (;;) {
    if (threadIdx.x == 0) {
      int i = atomicAdd(&a.ctl->solo_next, 1);
      if (i < a.num_mats && ld_relaxed_s32(&a.ctl->status)) i = a.num_mats;   // an error ends the call
      sh.k = i < a.num_mats ? __ldcg(a.order + i) : -1;
    }
    __syncthreads();
    const int k = sh.k;
    __syncthreads();
    if (k < 0) break;
    so_matrix(a, k, sh);
    ++mats;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    if (a.collect_stats) {
      Stats* s = a.stats;
      if (sh.st_exec) atomicAdd(&s->executed, (unsigned long long)sh.st_exec);
      if (sh.st_exec) atomicAdd(&s->dequeued, (unsigned long long)sh.st_exec);
      if (sh.st_exec) atomicAdd(&s->generated, (unsigned long long)sh.st_exec);
      if (sh.st_comp) atomicAdd(&s->components, (unsigned long long)sh.st_comp);
      if (sh.st_over) atomicAdd(&s->oversize, (unsigned long long)sh.st_over);
      if (sh.st_claim) atomicAdd(&s->cand_spec, (unsigned long long)sh.st_claim);
      if (sh.st_comb) atomicAdd(&s->ovh_forwards, (unsigned long long)sh.st_comb);
      if (mats) atomicAdd(&s->solo_problems, (unsigned long long)mats);
    }
    const unsigned long long t = globaltimer();
    atomicMax(&a.ctl->ts[3], t);
    atomicMax(&a.ctl->ts[4], t);
  }
}

}  // namespace rcm

extern "C" const void* rcm_ksolo_order_ptr() { return (const void*)rcm::k_solo_order; }
extern "C" const void* rcm_ksolo_ptr() { return (const void*)rcm::k_solo; }
extern "C" size_t rcm_ksolo_smem() { return rcm::kSoloSmem; }
extern "C" int rcm_ksolo_threads() { return rcm::kSoloNT; }
extern "C" int rcm_ksolo_nmax() { return rcm::kSoloNMax; }
