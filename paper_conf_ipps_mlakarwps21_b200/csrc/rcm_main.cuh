// rcm_main.cuh -- the persistent kernel k_main (one cooperative launch per
// rcm_* call) and its phases: prologue, seeding, traversal scheduling,
// components.  Instantiated once per (blocks-per-SM, chain / multi-batch / leveled) variant in
// k_main_inst.cu (separate translation units, compiled in parallel).
// Citations P:L<n> = /root/reference/PAPER.md line n; C-k = DESIGN.md readings.
#pragma once
#include "rcm_lookback.cuh"
#include "rcm_components.cuh"
#include "rcm_leveled.cuh"

namespace rcm {

// ===================================================================== phases
// a1 -- prologue: valence = row_ptr diff, owner word init, argmin of
// (valence, id) (C-6 / MIN_DEGREE seed), max valence, optional CSR checks.
// Four nodes per thread with an int4 row_ptr load and a one-element halo.
static __device__ void prologue_phase(const KParams& kp, const MainArgs& a, ShState& sh) {
  const int n = a.n;
  unsigned long long best = kKeyMax;
  int mx = 0, bad = 0;
  const int G = gthreads(kp);
  for (int t = gtid(); t * 4 < n; t += G) {
    const int v0 = t * 4;
    int r[5];
    if (a.vec && v0 + 4 <= n) {
      int4 q = __ldg(reinterpret_cast<const int4*>(kp.row_ptr + v0));
      r[0] = q.x; r[1] = q.y; r[2] = q.z; r[3] = q.w;
      r[4] = __ldg(kp.row_ptr + v0 + 4);
    } else {
      for (int j = 0; j < 5; ++j) r[j] = (v0 + j <= n) ? __ldg(kp.row_ptr + v0 + j) : 0;
    }
    const int m = min(4, n - v0);
    unsigned long long w[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (j < m) {
        int d = r[j + 1] - r[j];
        if (d < 0) { bad = 1; d = 0; }
        w[j] = ((unsigned long long)kInf << 32) | (uint32_t)d;
        const unsigned long long k = ((unsigned long long)(uint32_t)d << 32) | (uint32_t)(v0 + j);
        best = k < best ? k : best;
        mx = max(mx, d);
      }
    }
    if (m == 4) {
      reinterpret_cast<ulonglong2*>(kp.word + v0)[0] = make_ulonglong2(w[0], w[1]);
      reinterpret_cast<ulonglong2*>(kp.word + v0)[1] = make_ulonglong2(w[2], w[3]);
    } else {
      for (int j = 0; j < m; ++j) kp.word[v0 + j] = w[j];
    }
    if (a.validate) {
      if (v0 == 0 && r[0] != 0) bad = 1;
      if (v0 + m == n && (long long)r[m] != a.nnz) bad = 1;
    }
  }
  if (a.validate >= 1) {   // every column index in range
    for (long long i = gtid(); i < a.nnz; i += G) {
      const int c = __ldg(kp.col_idx + i);
      bad |= (c < 0 || c >= n);
    }
  }
  best = warp_min_u64(best);
  for (int d = 16; d > 0; d >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, d));
  bad = __any_sync(0xffffffffu, bad);
  if ((threadIdx.x & 31) == 0) {
    if (best != kKeyMax) atomicMin(&kp.ctl->minkey, best);
    if (mx) atomicMax(&kp.ctl->maxdeg, mx);
    if (bad) atomicCAS(&kp.ctl->status, 0, ST_BAD_CSR);
  }
}

// validate == 2: structural symmetry -- for every (u, c) the row of c holds u.
// Binary search (sorted rows: O(nnz log deg)), linear scan only when the
// search misses (unsorted rows).
static __device__ void validate_sym_phase(const KParams& kp, int n) {
  int bad = 0;
  for (int u = gtid(); u < n; u += gthreads(kp)) {
    for (int e = __ldg(kp.row_ptr + u); e < __ldg(kp.row_ptr + u + 1); ++e) {
      const int c = __ldg(kp.col_idx + e);
      if (c < 0 || c >= n) { bad = 1; continue; }
      const int b0 = __ldg(kp.row_ptr + c), b1 = __ldg(kp.row_ptr + c + 1) - 1;
      int lo = b0, hi = b1;
      bool found = false;
      while (lo <= hi) {
        const int mid = (lo + hi) >> 1;
        const int x = __ldg(kp.col_idx + mid);
        if (x == u) { found = true; break; }
        if (x < u) lo = mid + 1; else hi = mid - 1;
      }
      for (int f = b0; f <= b1 && !found; ++f) found = __ldg(kp.col_idx + f) == u;
      bad |= !found;
    }
  }
  if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) atomicCAS(&kp.ctl->status, 0, ST_NOT_SYM);
}

// The scheduling phase: every chain problem in turn on all blocks (grid
// barrier between chains), then the solo problems, one per block at a time.
// kMode: 0 look-back / serial chain, 1 multi-batch chain, 2 leveled (NEXT-3);
// one kernel instantiation each, so no variant pays the others' registers.
template <int kMode>
__device__ __forceinline__ void schedule_phase(const KParams& kp, const MainArgs& a, const SmemPtrs& sm, ShState& sh,
                                               ShState& sh2) {
  const int nchain = ld_cg_s32(&kp.ctl->n_chain);
  for (int c = 0; c < nchain; ++c) {
    if (kp.chains[c].flags & 2) {   // PSEUDO_PERIPHERAL component: GL seed first (C-5)
      const int x = gl_phase(kp, a.w, a.n, kp.chains[c].seed, sh);
      if (blockIdx.x == 0 && threadIdx.x == 0) const_cast<Problem*>(kp.chains)[c].seed = x;
      grid_barrier(kp);
    }
    if constexpr (kMode == 2) {      // NEXT-3: Alg. 2 level-synchronous traversal
      const Problem PL = kp.chains[c];
      leveled_chain(kp, a, PL, sm, sh);
      continue;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) chain_init(kp, kp.chains[c]);
    grid_barrier(kp);
    const uint32_t epoch = ld_acquire_u32(&kp.ctl->epoch);
    // the problem lives in shared memory: its fields are re-read on use (LDS)
    // instead of pinning 16 registers across the whole traversal
    if (threadIdx.x == 0) sh.prob = kp.chains[c];
    __syncthreads();
    if constexpr (kMode == 1) chain_worker_mb(kp, sh.prob, sm, sh, sh2, epoch);
    else if constexpr (kMode == 0) chain_worker(kp, sh.prob, sm, sh, epoch);
    grid_barrier(kp);
    chain_reset_signals(kp);
    grid_barrier(kp);
  }
  const int nsolo = ld_cg_s32(&kp.ctl->n_solo);
  for (;;) {
    if (threadIdx.x == 0) {
      sh.k = atomicAdd(&kp.ctl->solo_next, 1);
      if (ld_cg_s32(&kp.ctl->status)) sh.k = nsolo;   // block-uniform exit decision
    }
    __syncthreads();
    const int k = sh.k;
    __syncthreads();
    if (k >= nsolo) break;
    if (threadIdx.x == 0) sh.prob = kp.solos[k];
    __syncthreads();
    if (sh.prob.size > 0) run_solo(kp, sh.prob, sm, sh, a.w.lev);
    __syncthreads();
  }
}

// One launch per call: reset -> prologue -> seed / problem set-up ->
// traversal -> (components -> traversal).  Grid barriers between phases.
template <int kMinBlocks, int kMode>
__global__ void __launch_bounds__(kThreads, kMinBlocks) k_main(const __grid_constant__ KParams kp, const __grid_constant__ MainArgs a) {
  __shared__ ShState sh;
  __shared__ ShState sh2;   // second batch context (multi-batch execution, kMB only)
  SmemPtrs sm;   // layout accessors sm_*(kp) (rcm_batch.cuh)
  if (threadIdx.x == 0) rcm_ctx_base = 0;
  const int G = gthreads(kp);
  // ---- phase 0: reset the per-call control state
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    Ctl* c = kp.ctl;
    c->ts[0] = globaltimer();
    c->ts[5] = c->ts[6] = 0;
    for (int i = 0; i < 8; ++i) c->dbg[i] = 0;
    c->minkey = kKeyMax; c->maxdeg = 0; c->status = 0; c->head = 0; c->done = 0; c->chain_total = 0;
    c->solo_next = 0; c->n_chain = 0; c->n_solo = 0; c->n_comp = 0; c->spill_cursor = 0; c->incomplete = 0;
    if (kp.collect_stats) *kp.stats = Stats{};
  }
  if (a.mode == RCM_START_PSEUDO_PERIPHERAL && !a.gl_only)
    for (long long v = gtid(); v < a.n; v += G) a.w.lev[v] = -1;
  grid_barrier(kp);
  // ---- phase 1: prologue (a1)
  prologue_phase(kp, a, sh);
  if (a.validate == 2) validate_sym_phase(kp, a.n);
  grid_barrier(kp);
  stamp(kp, 1);
  if (ld_cg_s32(&kp.ctl->status)) return;   // read after a barrier: uniform across blocks
  if (a.gl_only) {   // rcm_find_pseudo_peripheral
    const int x = gl_phase(kp, a.w, a.n, a.gl_start, sh);
    if (gtid() == 0) *a.gl_out = x;
    stamp(kp, 4);
    return;
  }
  // ---- phase 2: problems
  int seed = a.mode == RCM_START_FIXED ? a.start : (int)(uint32_t)__ldcg(&kp.ctl->minkey);
  if (a.mode == RCM_START_PSEUDO_PERIPHERAL) seed = gl_phase(kp, a.w, a.n, seed, sh);
  if (gtid() == 0) {
    Problem P;
    P.node_base = 0; P.rp_base = 0; P.ci_base = 0; P.o_base = 0; P.perm_base = 0;
    P.mat_n = a.n; P.pos0 = 0; P.size = a.n; P.seed = seed; P.pad = 0;
    P.flags = 0;
    const_cast<Problem*>(kp.chains)[0] = P;
    kp.ctl->n_chain = 1;
  }
  grid_barrier(kp);
  stamp(kp, 2);
  // ---- phase 3: the traversal (a2-a12)
  schedule_phase<kMode>(kp, a, sm, sh, sh2);
  grid_barrier(kp);
  stamp(kp, 3);
  // ---- phase 4: components left over by the chain-first pass (a13)
  if (ld_cg_s32(&kp.ctl->incomplete) && !ld_cg_s32(&kp.ctl->status)) {
    cc_phase(kp, a, sm, sh);
    schedule_phase<kMode>(kp, a, sm, sh, sh2);
    grid_barrier(kp);
  }
  stamp(kp, 4);
}


}  // namespace rcm
