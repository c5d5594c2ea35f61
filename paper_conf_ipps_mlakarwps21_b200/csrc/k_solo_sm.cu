// k_solo_sm.cu -- one small graph on one block with its whole CSR staged in
// shared memory (rcm_reorder on graphs of <= solo_threshold nodes whose CSR
// fits next to the batch scratch, e.g. config 1: 97 KB).  Same code as k_solo
// (rcm_solo.cuh) with every row_ptr / column read served from shared memory,
// so a batch has no global round trip left but the output stores.
#define RCM_SOLO_SMEM_CSR 1
#include "../../include/rcm.h"
#include "rcm_solo.cuh"

namespace rcm {

// TMA bulk copy global -> shared (cp.async.bulk), completion on an mbarrier.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* mbar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   (uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src), "r"(bytes), "r"((uint32_t)__cvta_generic_to_shared(mbar))
               : "memory");
}

// Stage n32 int32 from global into (16-byte aligned) shared memory: a
// 16-byte-aligned source's body of whole 16-byte chunks by one TMA bulk copy
// (issued by thread 0), everything else by plain loads.
__device__ __forceinline__ void stage_i32(int32_t* dst, const int32_t* src, long long n32, uint32_t body_bytes,
                                          uint64_t* mbar, bool issue) {
  for (long long i = body_bytes / 4 + threadIdx.x; i < n32; i += kSoloNT) dst[i] = __ldg(src + i);
  if (body_bytes > 0 && issue) bulk_g2s(dst, src, body_bytes, mbar);
}

__global__ void __launch_bounds__(kSoloNT, 1) k_solo_sm(const __grid_constant__ SoloArgs a) {
  __shared__ SoloSh sh;
  int32_t* srp = reinterpret_cast<int32_t*>(so_base() + kSoloSmem);
  int32_t* scol = srp + ((a.n + 1 + 3) & ~3);
  if (threadIdx.x == 0) {
    Ctl* c = a.ctl;
    c->ts[0] = c->ts[1] = c->ts[2] = globaltimer();
    c->ts[3] = c->ts[4] = c->ts[5] = c->ts[6] = 0;
    c->status = 0;
    c->solo_next = 0;
    c->done = 0;
    if (a.collect_stats) *a.stats = Stats{};
    sh.st_exec = sh.st_comp = sh.st_over = sh.st_claim = sh.st_comb = 0;
  }
  // stage the CSR: TMA bulk copies of the 16-byte-aligned bodies (one thread),
  // the rest by plain loads; an mbarrier tracks the bulk bytes
  __shared__ __align__(8) uint64_t mbar;
  const uint32_t m = (uint32_t)__cvta_generic_to_shared(&mbar);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(m));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const bool lead = threadIdx.x == 0;
  const uint32_t body_rp = ((uintptr_t)a.row_ptr & 15) == 0 ? (uint32_t)(4 * ((a.n + 1) / 4 * 4)) : 0u;
  const uint32_t body_col = ((uintptr_t)a.col_idx & 15) == 0 ? (uint32_t)(4 * (a.nnz / 4 * 4)) : 0u;
  if (lead) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(m), "r"(body_rp + body_col)
                         : "memory");
  stage_i32(srp, a.row_ptr, a.n + 1, body_rp, &mbar, lead);
  if (a.nnz > 0) stage_i32(scol, a.col_idx, a.nnz, body_col, &mbar, lead);
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra WAIT_%=;\n}" ::"r"(m)
      : "memory");
  __syncthreads();
  SoloArgs la = a;
  la.row_ptr = srp;
  la.col_idx = scol;
  so_matrix(la, 0, sh);
  __syncthreads();
  if (threadIdx.x == 0) {
    if (a.collect_stats) {
      Stats* s = a.stats;
      s->executed = s->dequeued = s->generated = (unsigned long long)sh.st_exec;
      s->components = (unsigned long long)sh.st_comp;
      s->oversize = (unsigned long long)sh.st_over;
      s->cand_spec = (unsigned long long)sh.st_claim;
      s->ovh_forwards = (unsigned long long)sh.st_comb;
      s->solo_problems = 1;
    }
    a.ctl->ts[3] = a.ctl->ts[4] = globaltimer();
  }
}

}  // namespace rcm

extern "C" const void* rcm_ksolo_sm_ptr() { return (const void*)rcm::k_solo_sm; }
