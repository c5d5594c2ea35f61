// k_probe.cu -- the chain-latency bound of SURVEY.md §8(d): the cost of one
// hand-off between two thread blocks on different SMs, measured with the same
// primitives the chain uses (st.release.gpu of a flag, relaxed polling +
// fence.acq_rel on the receiver, "explicit non-locally cached
// writes").  Two blocks, pinned to SMs a and b by their %smid, bounce a
// counter `iters` times; t_hop = elapsed / (2 * iters).
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/rcm.h"
#include "rcm_device.cuh"

namespace rcm {

struct ProbeCtl {
  int32_t role_taken[2];
  int32_t ready;
  int32_t pad;
  uint32_t flag;          // ping-pong counter
  uint32_t pad2[31];      // flag on its own 128 B line
  unsigned long long t0, t1;
};

__device__ __forceinline__ uint32_t smid() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

__global__ void k_probe_hop(ProbeCtl* c, int sm_a, int sm_b, int iters) {
  if (threadIdx.x != 0) return;
  const uint32_t me = smid();
  int role = -1;
  if ((int)me == sm_a && atomicCAS(&c->role_taken[0], 0, 1) == 0) role = 0;
  else if ((int)me == sm_b && atomicCAS(&c->role_taken[1], 0, 1) == 0) role = 1;
  if (role < 0) return;
  // both roles present (bounded wait: the launch has more blocks than SMs)
  atomicAdd(&c->ready, 1);
  const uint64_t tw = globaltimer();
  while (ld_relaxed_s32(&c->ready) < 2) {
    if (globaltimer() - tw > 2000000000ull) return;
  }
  const uint32_t mine = (uint32_t)role;   // role 0 waits for even values, role 1 for odd
  if (role == 0) c->t0 = globaltimer();
  for (int i = 0; i < iters; ++i) {
    const uint32_t want = 2u * (uint32_t)i + mine;
    const uint64_t ts = globaltimer();
    while (ld_relaxed_u32(&c->flag) != want) {
      if (globaltimer() - ts > 1000000000ull) return;
    }
    fence_acquire_gpu();
    st_release_u32(&c->flag, want + 1);
  }
  if (role == 0) c->t1 = globaltimer();
}

}  // namespace rcm

// Host: one-way hand-off latency (ns) between SMs a and b, averaged over
// `iters` round trips; writes -1 if the two roles could not be placed.
extern "C" rcm_status_t rcm_probe_hop(int32_t sm_a, int32_t sm_b, int32_t iters, double* out_ns) {
  using rcm::ProbeCtl;
  if (!out_ns || iters <= 0 || sm_a == sm_b) return RCM_ERR_INVALID_ARGUMENT;
  int dev = 0, nsm = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return RCM_ERR_CUDA;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  ProbeCtl* c = nullptr;
  if (cudaMalloc(&c, sizeof(ProbeCtl)) != cudaSuccess) return RCM_ERR_OUT_OF_MEMORY;
  cudaMemset(c, 0, sizeof(ProbeCtl));
  rcm::k_probe_hop<<<4 * nsm, 32>>>(c, sm_a, sm_b, iters);
  ProbeCtl h;
  cudaError_t e = cudaMemcpy(&h, c, sizeof(ProbeCtl), cudaMemcpyDeviceToHost);
  cudaFree(c);
  if (e != cudaSuccess) return RCM_ERR_CUDA;
  *out_ns = (h.t1 > h.t0 && h.ready == 2) ? (double)(h.t1 - h.t0) / (2.0 * iters) : -1.0;
  return RCM_OK;
}
