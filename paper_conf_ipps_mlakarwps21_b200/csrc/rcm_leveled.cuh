// rcm_leveled.cuh -- NEXT-3: Leveled RCM (Alg. 2) on the
// B200, the paper's GPU-RCM baseline and an independent second GPU
// implementation of the same permutation.  Level-synchronous, inside the
// persistent kernel (grid barriers between the steps of a level):
//   expand  : per parent p of level i and neighbour n:
//             m_n <- atomicMin(m[n], i+1)                    (Alg. 2 ln 8)
//             if m_n >= i+1: atomicMin(s[n], pos(p))          (ln 9-10, lowest source)
//             if m_n >  i+1: c <- c + {n}                      (ln 11-13, first time)
//   sort    : c by (lowest source position, valence, id)      (ln 14, C-1 tie-break)
//   write   : o[next level] <- c                              (ln 15), perm reversed (C-7)
// m is the owner field of word[] (hi 32 bits; the valence stays in the low 32),
// s[] reuses the component-label array, c and its sort use the radix buffers.
#pragma once
#include "rcm_components.cuh"

namespace rcm {

static __device__ void leveled_chain(const KParams& kp, const MainArgs& a, const Problem& P, const SmemPtrs& sm,
                              ShState& sh) {
  const CompWS& w = a.w;
  const int G = gthreads(kp);
  const int n = P.mat_n;
  int32_t* src = w.label;
  unsigned long long* word = kp.word + P.node_base;
  int32_t* o = kp.o + P.o_base;
  int32_t* perm = kp.perm + P.perm_base;
  for (int v = gtid(); v < n; v += G) src[v] = 0x7fffffff;
  if (gtid() == 0) {
    place_root(kp, P, P.seed, P.pos0);    // level 0
    stat_add(kp, &kp.stats->components, 1);
  }
  grid_barrier(kp);
  const int idbits = a.idbits;
  int dbits = 0;
  while (dbits < 32 && (1ll << dbits) <= ld_cg_s32(&kp.ctl->maxdeg)) ++dbits;
  int lb = P.pos0, le = P.pos0 + 1;
  const int lane = threadIdx.x & 31, gwarp = gtid() >> 5, nwarps = G >> 5;
  for (uint32_t level = 0;; ++level) {
    const int W = le - lb;
    if (gtid() == 0) w.sctl[0] = 0;
    grid_barrier(kp);
    // expand: one warp per parent, lanes stride the row
    const uint32_t nl = level + 1;
    for (int i = gwarp; i < W; i += nwarps) {
      const int p = __ldcg(o + lb + i);
      const int rs = __ldg(kp.row_ptr + P.rp_base + p), re = __ldg(kp.row_ptr + P.rp_base + p + 1);
      for (int base = rs; base < re; base += 32) {
        const int e = base + lane;
        bool first = false;
        int c = 0;
        if (e < re) {
          c = __ldg(kp.col_idx + P.ci_base + e);
          unsigned long long wv = ld_relaxed_u64(word + c);
          if ((uint32_t)(wv >> 32) >= nl) {
            const unsigned long long old = atomicMin(word + c, ((unsigned long long)nl << 32) | (wv & 0xffffffffull));
            const uint32_t mn = (uint32_t)(old >> 32);
            if (mn >= nl) atomicMin(src + c, lb + i);
            first = mn > nl;
          }
        }
        const unsigned bal = __ballot_sync(0xffffffffu, first);
        int slot0 = 0;
        if (bal && lane == 0) slot0 = atomicAdd(w.sctl, __popc(bal));
        slot0 = __shfl_sync(0xffffffffu, slot0, 0);
        if (first) w.vals0[slot0 + __popc(bal & ((1u << lane) - 1))] = c;
      }
    }
    grid_barrier(kp);
    const int cnt = ld_cg_s32(w.sctl);
    if (cnt == 0) break;
    // keys (source position in the level, valence, id): one 64-bit radix key
    int wbits = 0;
    while ((1ll << wbits) < W) ++wbits;
    const int tot = wbits + dbits + idbits;
    if (tot > 64) {
      if (gtid() == 0) latch_error(kp.ctl, ST_CAPACITY);
      grid_barrier(kp);
      break;
    }
    for (int i = gtid(); i < cnt; i += G) {
      const int c = __ldcg(w.vals0 + i);
      const unsigned long long s = (unsigned long long)(ld_cg_s32(src + c) - lb);
      const unsigned long long d = ld_relaxed_u64(word + c) & 0xffffffffull;
      w.keys0[i] = (s << (dbits + idbits)) | (d << idbits) | (unsigned long long)(uint32_t)c;
    }
    if (gtid() == 0) w.sctl[1] = 0;
    grid_barrier(kp);
    radix_sort_phase(kp, w, 0, tot, reinterpret_cast<int32_t*>(sm_cand(kp)), sh);   // parallelSort (ln 14)
    const unsigned long long* keys = ld_cg_s32(w.sctl + 1) ? w.keys1 : w.keys0;
    const unsigned long long idmask = (1ull << idbits) - 1;
    for (int i = gtid(); i < cnt; i += G) {                                     // parallelWrite (ln 15)
      const int c = (int)(__ldcg(keys + i) & idmask);
      o[le + i] = c;
      perm[P.mat_n - 1 - (le + i)] = c;
      if (kp.iperm) kp.iperm[P.node_base + c] = P.mat_n - 1 - (le + i);
    }
    if (gtid() == 0 && kp.collect_stats) atomicAdd(&kp.stats->executed, 1ull);
    grid_barrier(kp);
    lb = le;
    le += cnt;
  }
  if (gtid() == 0) {
    kp.ctl->chain_total = le;
    if (le < P.pos0 + P.size) kp.ctl->incomplete = 1;   // component exhausted, others remain
  }
  grid_barrier(kp);
}

}  // namespace rcm
