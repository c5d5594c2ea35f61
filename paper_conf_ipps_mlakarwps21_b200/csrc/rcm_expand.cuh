// rcm_expand.cuh -- warp-cooperative, load-balanced row expansion for the
// level-synchronous phases (GL finder P:L365-375, leveled traversal).
//
// A warp holds up to 32 rows, one per lane (row start rs, length d; d = 0 for
// an idle lane).  The rows' edges are numbered 0..E-1 in lane order (an
// inclusive warp scan of d), and lane l takes edges base + u*32 + l, so every
// lane does the same amount of work whatever the mix of row lengths, and
// kU independent column loads per lane are in flight before any is used.
// The row an edge belongs to is found by a 5-step binary search over the
// scanned lengths (warp shuffles, no shared memory).
#pragma once
#include "rcm_device.cuh"

namespace rcm {

constexpr unsigned kFull = 0xffffffffu;

__device__ __forceinline__ int warp_incl_scan(int x) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int s = 1; s < 32; s <<= 1) {
    const int y = __shfl_up_sync(kFull, x, s);
    if (lane >= s) x += y;
  }
  return x;
}

// Lane holding edge e (< total): the number of lanes whose inclusive prefix is <= e.
__device__ __forceinline__ int warp_edge_lane(int e, int incl) {
  int pos = 0;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    const int v = __shfl_sync(kFull, incl, pos + s - 1);
    if (v <= e) pos += s;
  }
  return pos;
}

// Rows of the warp, scanned once: `incl` (inclusive prefix of d), `excl`, E.
struct WarpRows {
  int rs, incl, excl, E;
  __device__ __forceinline__ void init(int rs_, int d) {
    rs = rs_;
    incl = warp_incl_scan(d);
    excl = incl - d;
    E = __shfl_sync(kFull, incl, 31);
  }
  // Column of edge e (< 0 past the end) and the lane (row) it belongs to.
  template <int kU>
  __device__ __forceinline__ void cols(const int32_t* col, int base, int (&c)[kU], int (&j)[kU]) const {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int u = 0; u < kU; ++u) {
      const int e = base + u * 32 + lane;
      const int jj = warp_edge_lane(e, incl);
      const int r0 = __shfl_sync(kFull, rs, jj & 31);
      const int x0 = __shfl_sync(kFull, excl, jj & 31);
      j[u] = jj;
      c[u] = e < E ? __ldg(col + r0 + (e - x0)) : -1;
    }
  }
};

// Warp-aggregated append of the lanes with `take` set to list[atomicAdd(cnt)].
__device__ __forceinline__ void warp_append(bool take, int v, int32_t* cnt, int32_t* list) {
  const unsigned bal = __ballot_sync(kFull, take);
  if (!bal) return;
  const int lane = threadIdx.x & 31;
  const int leader = __ffs(bal) - 1;
  int base = 0;
  if (lane == leader) base = atomicAdd(cnt, __popc(bal));
  base = __shfl_sync(kFull, base, leader);
  if (take) list[base + __popc(bal & ((1u << lane) - 1u))] = v;
}

}  // namespace rcm
