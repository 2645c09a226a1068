/* include/bgpq.h — C ABI of the B200-native BGPQ batched-heap priority queue.
 *
 * The operations are those of the paper's problem statement (BGPQ, Chen et al., ICPP'21,
 * /root/reference/PAPER.md, cited as P:<line>):
 *   - the priority-queue ADT: INSERT of (key, value) pairs and DELETEMIN returning the pair
 *     with the smallest key (§2);
 *   - batched: one INSERT carries 1..k keys, one DELETEMIN returns the 1..k smallest keys,
 *     or every key left if fewer remain (§3.2);
 *   - linearizable: every operation takes effect at a point while it holds the root lock
 *     (§5).
 *
 * Conventions common to every call
 *   - Keys and values are uint32; keys are ordered as unsigned integers ("32-bit keys").
 *   - All key / value / count pointers are DEVICE pointers unless the name ends in _host.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Calls are
 *     asynchronous and stream-ordered; caller buffers must stay valid until the stream has
 *     reached the call (as with cudaMemcpyAsync).  One handle must not be used from two
 *     streams concurrently: concurrency lives INSIDE a call (many CTAs execute its batch
 *     operations at once) and in bgpq_run_mixed.
 *   - The handle owns the heap storage; the caller owns every other buffer.
 *   - Return values: BGPQ_OK (0) or a negative BGPQ_E* code.  bgpq_create returns NULL on
 *     failure; bgpq_last_error() then says why (thread-local).
 *   - There is no CPU fallback: if no sm_100 device is present the calls fail with
 *     BGPQ_ECUDA.
 */
#ifndef BGPQ_H
#define BGPQ_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bgpq bgpq_t;

enum {
  BGPQ_OK = 0,
  BGPQ_EINVAL = -1, /* bad argument (K not a power of two in 64..4096, NULL pointer, ...) */
  BGPQ_ENOMEM = -2, /* device allocation failed                                          */
  BGPQ_EFULL = -3,  /* sticky: an INSERT needed a node beyond the capacity; op dropped   */
  BGPQ_ECUDA = -4   /* a CUDA runtime call or kernel launch failed                       */
};

/* bgpq_create_ex flags */
enum {
  BGPQ_FLAG_VALUES = 1u, /* store a uint32 value with every key (w = 8 B per entry)        */
  BGPQ_FLAG_SERIAL = 2u, /* execute operations one at a time on a single CTA (test mode:
                            the node layout then equals the sequential Alg.1-3 model)     */
  BGPQ_FLAG_LOCKS = 4u   /* per-node-lock execution of every call (the mixed-call engine,
                            used for insert-only and deletemin-only calls too)              */
};
/* Default execution (no flag):
 *  - bgpq_insert: a level pipeline — one CTA per heap depth applies that depth's
 *    INSERT_HEAPIFY steps (Alg.1 l.30-34) in call order, the root stage runs PARTIAL_INSERT
 *    (l.15-29), sorter CTAs run Sort(items) (l.2); the heap after the call equals the
 *    sequential Alg.1 model node for node;
 *  - bgpq_deletemin: a top CTA keeps the root, the pBuffer and depths 1-2 in shared memory,
 *    runs every root section (Alg.2) and the depth-0..2 steps of Alg.3 in call order, and
 *    hands the walk below depth 3 (node still locked) to walker CTAs that take the paper's
 *    per-node locks top-down hand over hand;
 *  - bgpq_run_mixed: every CTA of a persistent grid executes whole operations (Alg.1,
 *    Alg.2+3) with per-node locks, a lock warp per CTA taking the next level's locks ahead. */

/* Create an empty heap able to hold `capacity` keys with node capacity K (§3.1:
 * every non-root node holds K sorted keys; k > 1).  K must be a power of two in 64..4096
 * (4096: keys only — a node pair with values exceeds the 227 KB of shared memory of a CTA;
 * the paper stopped at 1K for the same reason on its GPU).  Allocates ceil(capacity/K)+2 node slots of K entries in device memory of the
 * current device.  bgpq_create stores keys and values (flags = BGPQ_FLAG_VALUES). */
bgpq_t* bgpq_create(uint64_t capacity, uint32_t K);
bgpq_t* bgpq_create_ex(uint64_t capacity, uint32_t K, uint32_t flags);

/* Free the handle and its device memory (synchronizes the device first). */
void bgpq_destroy(bgpq_t* q);

/* INSERT n keys (Alg.1 BGPQ_INSERT): executed as ceil(n/K) batch INSERTs of
 * the consecutive K-slices keys[j*K, min(n,(j+1)*K)), linearized in some order.
 * keys: device, n entries.  vals: device, n entries, or NULL (values then undefined; a
 * handle without BGPQ_FLAG_VALUES ignores vals).  n = 0 is a no-op.
 * Capacity overflow sets the sticky BGPQ_EFULL reported by bgpq_size(); the overflowing
 * batch is dropped. */
int bgpq_insert(bgpq_t* q, const uint32_t* keys, const uint32_t* vals, uint64_t n, void* stream);

/* DELETEMIN n keys (Alg.2+3): executed as ceil(n/K) batch DELETEMINs.  The
 * batch that takes linearization ticket t of this call asks for min(K, n - t*K) keys and
 * writes them at out_keys[t*K ...], so the output is compact and ascending when no INSERT
 * runs concurrently.  Writes min(n, current size) entries in total; if d_count != NULL
 * (device uint64) that count is ADDED to *d_count.  out_vals may be NULL. */
int bgpq_deletemin(bgpq_t* q, uint32_t* out_keys, uint32_t* out_vals, uint64_t n,
                   uint64_t* d_count, void* stream);

/* Number of keys in the heap (|root| + |pBuffer| + K*(heapSize-1)).  Synchronizes
 * `stream`.  Returns BGPQ_EFULL if a capacity overflow happened since creation. */
int bgpq_size(bgpq_t* q, uint64_t* out_size, void* stream);

/* Same as bgpq_insert / bgpq_deletemin with HOST buffers (pinned memory gives full
 * PCIe bandwidth): the host->device and device->host copies are part of the call and are
 * ordered on `stream`; the call returns after the results are in the host buffers.
 * out_count_host (nullable) receives the number of entries written. */
int bgpq_insert_host(bgpq_t* q, const uint32_t* keys_host, const uint32_t* vals_host, uint64_t n,
                     void* stream);
int bgpq_deletemin_host(bgpq_t* q, uint32_t* out_keys_host, uint32_t* out_vals_host, uint64_t n,
                        uint64_t* out_count_host, void* stream);

/* Test / bench extension: run an arbitrary stream of n_ops batch operations concurrently
 * on the persistent CTAs (op j: op_types[j] 0 = INSERT, 1 = DELETEMIN; op_sizes[j] in 1..K).
 * INSERT j reads op_sizes[j] keys at in_keys[in_off[j]]; DELETEMIN j writes at
 * out_keys[j*K] and its entry count to op_count[j].  lin_ticket[j] (nullable) receives
 * the global linearization ticket taken under the root lock.  All device.
 * An op size outside 1..K skips the op (op_count = 0 for a DELETEMIN) and sets the sticky
 * BGPQ_EINVAL reported by the next bgpq_size(). */
int bgpq_run_mixed(bgpq_t* q, const uint8_t* op_types, const uint32_t* op_sizes,
                   const uint64_t* in_off, uint64_t n_ops, const uint32_t* in_keys,
                   const uint32_t* in_vals, uint32_t* out_keys, uint32_t* out_vals,
                   uint32_t* op_count, uint64_t* lin_ticket, void* stream);

/* Test extension: copy the quiescent heap to HOST buffers.  node_keys / node_vals:
 * (slots)*K entries, slot 0 = pBuffer, slot 1 = root, slot i >= 2 = node i; meta: 4
 * uint32 per slot {lock, state (0 EMPTY, 1 AVAIL, 2 TARGET, 3 MARKED), min, max};
 * hdr: {heapSize, |root|, |pBuffer|, sticky error}.  Synchronizes the device. */
int bgpq_dump(bgpq_t* q, uint32_t* node_keys, uint32_t* node_vals, uint32_t* meta, uint64_t* hdr);
uint64_t bgpq_slots(bgpq_t* q); /* number of node slots (= max node index + 1) */

/* Device counters accumulated over the handle's lifetime (for the byte model), written to
 * out[0..n): see BGPQ_STAT_* in DESIGN.md.  Synchronizes the device. */
int bgpq_stats(bgpq_t* q, uint64_t* out, int n);

/* Grid control: ctas = 0 -> all co-resident CTAs (default), 1 -> serialized. */
int bgpq_set_grid(bgpq_t* q, int ctas);
int bgpq_grid(bgpq_t* q);

/* Number of kernels this library has launched in the process (for bench gpu_launches). */
uint64_t bgpq_launch_count(void);

/* Device view of a heap for application kernels that call the device API
 * (include/bgpq_dev.cuh): plain device pointers of the arena owned by the handle (valid until
 * bgpq_destroy), the node capacity, K, the creation flags, the device and its SM count.  No
 * library call may run on the heap while such a kernel does. */
typedef struct {
  void* keys;     /* uint32 node keys, slot i at keys + i*K (0 = pBuffer, 1 = root) */
  void* vals;     /* uint32 node values, same layout, or NULL for a keys-only heap   */
  void* meta;     /* 16-B node records {lock, state, min, max}, one per slot          */
  void* hdr;      /* header words                                                     */
  uint32_t cap;   /* largest node index                                               */
  uint32_t K;
  uint32_t flags;
  int device;
  int sm_count;
  int ctas;       /* CTAs requested with bgpq_set_grid (0: all co-resident) — app kernels honour it */
} bgpq_view_t;
int bgpq_view(bgpq_t* q, bgpq_view_t* out);

/* Test / profiling extensions (not part of the minimal ABI).
 * bgpq_set_debug: process-wide switches read at each call (0 = product behaviour):
 *   8   accumulate thread-0 cycle timers in the header (read with bgpq_timers);
 *   16  run deletemin-only calls on the per-node-lock engine instead of the top CTA;
 *   64  register-window merge path instead of the warp-cooperative one on the top CTA;
 *   128 light top-CTA timers (plan / phase A / phase B);
 *   256 deletemin calls skip the cluster engine (top CTA / lock engine only);
 *   1024 cluster-engine role timers and walker first-level timers;
 *   32768 schedule forcing for tests: every INSERT on the per-node-lock engine holds its
 *         target node (state TARGET) 20 us before the placement (Alg.1 l.8-13), so concurrent
 *         DELETEMINs take the TARGET -> MARKED steal (Alg.2 l.7-9) and the one-AVAIL-
 *         child path of the heapify (Alg.3 l.5-8).
 * bgpq_timers: copies the 32 uint64 cycle counters of the handle to out32 (host);
 * synchronizes the device. */
int bgpq_set_debug(uint32_t bits);
int bgpq_timers(bgpq_t* q, uint64_t* out32);

/* Test extension: run one device primitive of the hot path on n_cases independent cases
 * (one CTA each; all pointers DEVICE, stream-ordered, no synchronization).  Case c reads
 * Z = zk[c*K .. c*K+na[c]), W = wk[c*K .. c*K+nb[c]) (sorted, values zv / wv when values != 0)
 * and writes X to xk[c*2K ..] and Y to yk[c*2K ..]:
 *   variant 0: SORT_SPLIT as the lock / pipeline executions run it (bitonic split for
 *              full keys-only batches at K >= 512, register-window merge path otherwise):
 *              X = the ma smallest of Z u W, Y = the rest, both ascending;
 *   variant 1: the same split as the top CTA's 256-thread groups run it (warp-cooperative
 *              merge path; bitonic for full keys-only batches at K >= 512);
 *   variant 2: the top CTA's register-window merge path (bgpq_set_debug bit 64);
 *   variant 3: Sort(items) (Alg.1 l.2): X = the na entries of Z sorted (W, nb, ma unused).
 * Requires 0 <= na, nb <= K, ma <= na + nb (full batches na = nb = ma = K for the bitonic
 * path).  Equal keys may carry their values in any order (reading R9). */
int bgpq_test_prim(int variant, uint32_t K, int values, const uint32_t* zk, const uint32_t* zv,
                   const uint32_t* wk, const uint32_t* wv, const uint32_t* na, const uint32_t* nb,
                   const uint32_t* ma, uint32_t n_cases, uint32_t* xk, uint32_t* xv, uint32_t* yk,
                   uint32_t* yv, void* stream);

int bgpq_last_error(void);
const char* bgpq_last_error_msg(void); /* CUDA error string of the last BGPQ_ECUDA */
const char* bgpq_strerror(int code);

#ifdef __cplusplus
}
#endif

#endif /* BGPQ_H */
