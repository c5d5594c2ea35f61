// rcm_device.cuh -- device-side data structures and primitives of the batch-RCM
// library (sm_100a).  Citations P:L<n> = /root/reference/PAPER.md line n.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace rcm {

#ifndef RCM_THREADS
#define RCM_THREADS 512
#endif
constexpr int kThreads = RCM_THREADS;       // threads per persistent worker block
constexpr int kWarps = kThreads / 32;
static_assert(kThreads % 32 == 0 && kThreads >= 256 && kThreads <= 1024, "block size");
#ifndef RCM_DISC_U
#define RCM_DISC_U 4
#endif
constexpr int kDiscU = RCM_DISC_U;
          // edge slots per thread in flight in discovery
// spin back-off caps (ns): dequeue polling, look-back polling
#ifndef RCM_DQ_SLEEP_MAX
#define RCM_DQ_SLEEP_MAX 512
#endif
#ifndef RCM_LB_SLEEP_MAX
#define RCM_LB_SLEEP_MAX 256
#endif
constexpr int kMaxBlocks = 1024;            // persistent workers per launch (beacon / scratch sizing)
constexpr int kMaxBatchNodes = 1024;        // B_s upper bound (u16 local parent ids)
constexpr uint32_t kInf = 0xFFFFFFFFu;      // "unmarked" owner
constexpr uint64_t kKeyMax = ~0ull;         // removed / padding sort key

// Signal states a batch receives from its predecessor (Alg. 5).
enum : uint32_t { S_NONE = 0, S_DISCOVERED = 1, S_COUNTED = 2, S_COMPLETED = 3 };

// Status codes (mirror rcm_status_t)
enum : int32_t { ST_OK = 0, ST_BAD_CSR = 2, ST_NOT_SYM = 3, ST_CAPACITY = 5, ST_HANG = 6 };

// Batch descriptor: a contiguous range [o_begin, o_end) of matrix-local output
// positions.  `next` is the queue index of the chain successor
// (skip-link over trailing empty batches).  `tag` = chain epoch,
// written last with release semantics: tag == epoch <=> published.
struct __align__(16) Desc {
  int32_t o_begin, o_end, next;
  uint32_t tag;
};

// Signal a batch receives from its chain predecessor,
// packed so that one acquire load returns the state AND the Counted payload:
//   word = out_off << 33 | q_off << 3 | has_ovh << 2 | state
//   out_off: matrix-local output position of this batch's first child (31 bit)
//   q_off:   queue index where this batch's generated batches go (30 bit)
//   ovh:     overhang forwarded to this batch, nodes << 32 | clamped valence
//            sum, written before `word`, read iff has_ovh.
// Slots are zeroed after every chain run, so 0 == S_NONE.
struct __align__(16) Sig {
  unsigned long long word;
  unsigned long long ovh;
};
__host__ __device__ __forceinline__ unsigned long long sig_pack(int out_off, int q_off, int has_ovh,
                                                                 uint32_t st) {
  return ((unsigned long long)(uint32_t)out_off << 33) | ((unsigned long long)(uint32_t)q_off << 3) |
         ((unsigned long long)(has_ovh & 1) << 2) | st;
}
__host__ __device__ __forceinline__ uint32_t sig_state(unsigned long long w) { return (uint32_t)(w & 3); }
__host__ __device__ __forceinline__ int sig_out(unsigned long long w) { return (int)(w >> 33); }
__host__ __device__ __forceinline__ int sig_q(unsigned long long w) { return (int)((w >> 3) & 0x3fffffffu); }
__host__ __device__ __forceinline__ int sig_has_ovh(unsigned long long w) { return (int)((w >> 2) & 1); }

// One independent unit of work: a connected component of one matrix.
struct Problem {
  int64_t node_base;  // word[] index of local node 0
  int64_t rp_base;    // row_ptr index of local node 0
  int64_t ci_base;    // added to row_ptr values to index col_idx
  int64_t o_base;     // o[] index of matrix-local position 0
  int64_t perm_base;  // perm[] index of matrix-local position 0
  int32_t mat_n;      // matrix size (perm[perm_base + mat_n-1-pos] = o[pos])
  int32_t pos0;       // first matrix-local position of this problem
  int32_t size;       // nodes to order (component size, or mat_n when unknown)
  int32_t seed;       // local id of the seed
  int32_t flags;      // bit0: may contain several components (solo restart allowed)
  int32_t pad;
};

// Device control block (one per plan, persistent across launches).
struct Ctl {
  unsigned long long minkey;   // prologue: min (deg << 32 | id)
  int32_t maxdeg;
  int32_t status;              // latched error (0 = ok)
  int32_t head;                // chain dequeue counter
  int32_t done;                // chain early-termination flag
  int32_t chain_total;         // nodes ordered after the chain-first pass
  uint32_t epoch;              // chain epoch counter (descriptor / signal tags)
  int32_t gbar_count;          // grid barrier
  int32_t gbar_gen;
  int32_t solo_next;           // solo problem dequeue counter
  int32_t n_chain;             // number of chain problems in the list
  int32_t n_solo;              // number of solo problems in the list
  int32_t n_comp;              // number of components found (CC pass)
  int32_t spill_cursor;        // oversize scratch allocation cursor
  int32_t chain_cur;           // chain index currently processed
  int32_t incomplete;          // 1 if the chain-first pass did not order every node
  int32_t qtail;               // highest queue slot reserved by the current chain
  int32_t completed;           // look-back chain: slots finished (chain-end detection)
  int32_t pad[1];
  unsigned long long ts[8];    // phase timestamps (%globaltimer ns) of the last call
  long long dbg[8];            // watchdog diagnostics: site, slot, index, word, ...
};

struct Stats {
  unsigned long long generated, dequeued, executed, empty, redisc_early, redisc_late,
      cand_spec, cand_removed, oversize, components, ovh_forwards, solo_problems;
  // per-stage SM cycles summed over workers (collect_stats == 2), the GPU
  // analogue of the paper's Fig. 6 stage breakdown:
  // dequeue, parents, discover, wait-Discovered, rediscover+count, sort,
  // wait-Counted (prefix), output, generate, other
  unsigned long long stage[10];
};

// ----------------------------------------------------------------- memory ops
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_acquire_s32(const int32_t* p) {
  int32_t v;
  asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_relaxed_s32(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Acquire side of a relaxed polling loop.  On sm_100a every ld.acquire.gpu is
// an LDG.STRONG followed by CCTL.IVALL, which drops the whole SM's L1 (the
// other resident block's cached lines and spill slots included), so spin
// loops poll with relaxed loads and pay for one acquire fence after they exit
// (PTX memory model: relaxed load observing a release + fence.acq_rel = acquire
// pattern).
__device__ __forceinline__ void fence_acquire_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void st_release_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void red_release_add_s32(int32_t* p, int32_t v) {
  asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed_add_s32(int32_t* p, int32_t v) {
  asm volatile("red.relaxed.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_s32(int32_t* p, int32_t v) {
  asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_s32(int32_t* p, int32_t v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// Owner-word load the compiler may schedule freely (a plain ld.global.cg, L2,
// not volatile): for prefilters and rediscovery re-reads, where a batch of
// independent loads is issued before any result is used.  Owner keys only
// decrease (atomicMin), so a stale value is never below the current one; it
// stays ordered by barriers and fences like any other load.
__device__ __forceinline__ unsigned long long ld_weak_u64(const unsigned long long* p) { return __ldcg(p); }
// L2-coherent load for data written by other blocks during this launch.
__device__ __forceinline__ int32_t ld_cg_s32(const int32_t* p) { return __ldcg(p); }

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// Spin-wait budget before the watchdog latches RCM_ERR_HANG (ns).
constexpr uint64_t kWatchdogNs = 20ull * 1000 * 1000 * 1000;

// --------------------------------------------------------------- block scan
// Exclusive block-wide prefix sum of one value per thread (kThreads threads).
// `warp_tmp` must hold kWarps + 1 elements of T in shared memory.
template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* warp_tmp, T& total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  T x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T y = __shfl_up_sync(0xffffffffu, x, d);
    if (lane >= d) x += y;
  }
  if (lane == 31) warp_tmp[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T w = (lane < kWarps) ? warp_tmp[lane] : T(0);
    T s = w;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      T y = __shfl_up_sync(0xffffffffu, s, d);
      if (lane >= d) s += y;
    }
    if (lane < kWarps) warp_tmp[lane] = s - w;
    if (lane == kWarps - 1) warp_tmp[kWarps] = s;
  }
  __syncthreads();
  T res = warp_tmp[wid] + x - v;
  total = warp_tmp[kWarps];
  __syncthreads();
  return res;
}

template <typename T>
__device__ __forceinline__ T block_reduce_sum(T v, T* warp_tmp) {
  T tot;
  block_exclusive_scan<T>(v, warp_tmp, tot);
  return tot;
}

// Block-wide sums of two values with one pair of barriers (all threads get both).
__device__ __forceinline__ void block_reduce_sum2(long long& a, long long& b, long long* ta, long long* tb) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, d);
    b += __shfl_xor_sync(0xffffffffu, b, d);
  }
  if (lane == 0) { ta[wid] = a; tb[wid] = b; }
  __syncthreads();
  a = 0;
  b = 0;
#pragma unroll
  for (int w = 0; w < kWarps; ++w) { a += ta[w]; b += tb[w]; }   // broadcast reads
  __syncthreads();
}

// Exclusive scan of m per-block partials in global memory (in[] and out[]
// distinct), by one block in chunks of kThreads (m may exceed the block size).
// Returns the total.
template <typename T, typename U = T>
__device__ __forceinline__ T block_scan_partials(const T* in, U* out, int m, T* warp_tmp) {
  T carry = 0;
  for (int base = 0; base < m; base += kThreads) {
    const int i = base + threadIdx.x;
    const T x = i < m ? __ldcg(in + i) : T(0);
    T tot;
    const T ex = block_exclusive_scan<T>(x, warp_tmp, tot);
    if (i < m) out[i] = (U)(carry + ex);
    carry += tot;
  }
  return carry;
}

// Exclusive scan, in place, of a[0..len) in shared memory; returns the total.
// Each thread scans a contiguous chunk (few block barriers).
template <typename T>
__device__ __forceinline__ T block_scan_array(T* a, int len, T* warp_tmp) {
  const int per = (len + kThreads - 1) / kThreads;
  const int b = threadIdx.x * per;
  const int e = min(len, b + per);
  T s = 0;
  for (int i = b; i < e; ++i) s += a[i];
  T tot;
  T run = block_exclusive_scan<T>(s, warp_tmp, tot);
  for (int i = b; i < e; ++i) {
    T x = a[i];
    a[i] = run;
    run += x;
  }
  __syncthreads();
  return tot;
}

__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long v) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) {
    unsigned long long o = __shfl_xor_sync(0xffffffffu, v, d);
    v = o < v ? o : v;
  }
  return v;
}

}  // namespace rcm
