/* include/bgpq_apps.h — C ABI of the paper's applications on BGPQ (§6.5):
 * persistent kernels whose CTAs loop DELETEMIN(K) -> expand -> prune -> INSERT on one heap
 * through the device API (include/bgpq_dev.cuh).  All pointers are DEVICE pointers, calls are
 * asynchronous on `stream` (cudaStream_t as void*).  Heaps must be created with
 * BGPQ_FLAG_VALUES and K in {64, 1024}.  Return BGPQ_OK or a negative BGPQ_E* code.
 *
 * state: 8 uint64 words owned by the caller, read / written by the kernels:
 *   [0] incumbent   knapsack: best profit found (initialise 0); A*: best cost to the target
 *                   found (initialise 0xFFFFFFFF)            — all-reduced between GPUs
 *   [1] pending     search nodes in the heap or being expanded; the caller sets it to the
 *                   number of entries in the heap before every run (bgpq_size)
 *   [2] expanded    [3] inserted   [4] pops (non-empty DELETEMINs)   [5] error flags
 *   [6] pruned (popped and discarded)   [7] empty DELETEMINs
 * A run ends when pending reaches 0 (search complete on this heap) or when every CTA has
 * done `budget` DELETEMINs (the heap then holds the unfinished frontier).
 */
#ifndef BGPQ_APPS_H
#define BGPQ_APPS_H

#include <stdint.h>

#include "bgpq.h"

#ifdef __cplusplus
extern "C" {
#endif

/* 0-1 knapsack (R23).  The caller allocates w, p (n entries) and Wp, Pp
 * (n + 1 uint64 entries) on the device; bgpq_ks_prepare fills them from the item arrays
 * w_in / p_in (device): items in profit/weight-descending order, prefix sums of weights and
 * profits.  n <= 1023, C < 2^22 (entry value packing (level << 22) | weight). */
typedef struct {
  uint32_t n;
  uint64_t C;
  uint32_t* w;
  uint32_t* p;
  uint64_t* Wp;
  uint64_t* Pp;
} bgpq_ks_t;
int bgpq_ks_prepare(uint32_t n, const uint32_t* w_in, const uint32_t* p_in, uint64_t C, bgpq_ks_t* ks,
                    void* stream);
/* The root node's queue entry (key = 0xFFFFFFFF - Dantzig bound, value 0) to key[0] / val[0]. */
int bgpq_ks_root(const bgpq_ks_t* ks, uint32_t* key, uint32_t* val, void* stream);
/* One run of the branch-and-bound kernel on heap q. */
int bgpq_ks_run(bgpq_t* q, const bgpq_ks_t* ks, uint64_t* state, uint32_t budget, void* stream);

/* A* on an N x M grid (R24): grid = N*M bytes row-major (1 = obstacle),
 * g = N*M uint32 scratch (best known cost per cell), target (tr, tc).  8 moves, orthogonal
 * cost 1, diagonal cost 2, Manhattan heuristic; N + M < 2^16. */
typedef struct {
  uint32_t N, M;
  const uint8_t* grid;
  uint32_t* g;
  uint32_t tr, tc;
} bgpq_astar_t;
/* Reset g to +inf, set g[start] = 0 and write the start entry to key[0] / val[0]. */
int bgpq_astar_init(const bgpq_astar_t* as, uint32_t sr, uint32_t sc, uint32_t* key, uint32_t* val,
                    void* stream);
int bgpq_astar_run(bgpq_t* q, const bgpq_astar_t* as, uint64_t* state, uint32_t budget, void* stream);

#ifdef __cplusplus
}
#endif

#endif /* BGPQ_APPS_H */
