/* rcm_cpu.h -- host CPU-BATCH: the paper's batch-based RCM on CPU threads
 * (Mlakar et al., IPDPS'21, Alg. 5 with the signalling chain of Sec. IV-B/C,
 * P:L376-839, run on std::thread workers as in the paper's CPU evaluation,
 * P:L863-865).  SURVEY.md §8(f) NEXT-4.
 *
 * This is a second implementation of the method for comparison on the host
 * (the paper's "CPU-BATCH" column), NOT a fallback of the GPU library: the
 * product path (rcm.h) never calls it.  All pointers are HOST pointers.
 *
 * Result: identical to serial RCM (Alg. 1 + the component rule C-6), like the
 * GPU path; readings C-1..C-11 of DESIGN.md apply.
 */
#ifndef RCM_CPU_H
#define RCM_CPU_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int64_t batches_executed;      /* non-empty batches processed                    */
  int64_t batches_empty;         /* empty slots processed (over-reservation)       */
  int64_t rediscover_early;      /* Discovered known right after discovery (ln 5-12) */
  int64_t rediscover_late;       /* Discovered waited for after sorting (ln 14-19) */
  int64_t candidates_removed;    /* speculative claims dropped by rediscovery      */
  int64_t chains;                /* signalling chains run (components with edges)  */
} rcm_cpu_stats_t;

/* Reorder one graph (CSR, structurally symmetric, 0 <= col < n) on `threads`
 * host threads (<= 0: hardware concurrency).
 *   mode:  0 FIXED (first seed = start), 1 MIN_DEGREE, 2 PSEUDO_PERIPHERAL
 *          (as rcm_start_t in rcm.h; later components by C-6)
 *   batch_nodes (B_s, 0 = 256) and temp_elems (T, 0 = 4096): batch cut limits,
 *          result-neutral (C-11)
 *   perm:  n entries, new -> old (perm[k] = o[n-1-k])
 *   stats: nullable.
 * Returns 0 on success, 1 on invalid arguments, 2 on allocation failure,
 * 5 if the batch queue overflowed (cannot happen with the bound of DESIGN.md §4).
 * Blocking; no state survives the call. */
int rcm_cpu_batch(int32_t n, const int32_t* row_ptr, const int32_t* col_idx, int32_t mode, int32_t start,
                  int32_t threads, int32_t batch_nodes, int32_t temp_elems, int32_t* perm,
                  rcm_cpu_stats_t* stats);

#ifdef __cplusplus
}
#endif
#endif /* RCM_CPU_H */
