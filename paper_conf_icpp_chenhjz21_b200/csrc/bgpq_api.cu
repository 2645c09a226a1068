// bgpq_api.cu — host side of the C ABI declared in include/bgpq.h.
// Owns the heap arena (node keys/values, node metadata, header), validates arguments,
// dispatches on the node capacity K (template instantiations 64..1024, keys-only or
// key+value) and launches the persistent ops kernel on the caller's stream.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "../../include/bgpq.h"
#include "bgpq_ktab.h"

using namespace bgpqd;

namespace {



thread_local int g_last_error = BGPQ_OK;
thread_local char g_last_msg[256] = "";
std::atomic<unsigned long long> g_launches{0};
unsigned g_debug = 0;  // test-only switches (bgpq_set_debug)

int fail(int code) {
  g_last_error = code;
  if (code == BGPQ_ECUDA) {
    cudaError_t e = cudaGetLastError();
    snprintf(g_last_msg, sizeof(g_last_msg), "%s", cudaGetErrorString(e));
  }
  return code;
}

}  // namespace

struct bgpq {
  int device = 0;
  u32 K = 0;
  u32 flags = 0;
  u64 capacity = 0;
  u32 cap_nodes = 0;  // largest node index
  u64 slots = 0;      // cap_nodes + 1
  u32* gk = nullptr;
  u32* gv = nullptr;
  NodeMeta* meta = nullptr;
  u32* hdr = nullptr;
  int sm_count = 0;
  int occ = 0;         // co-resident CTAs per SM for this K
  int grid_req = 0;    // 0 auto, else exact
  PipeArgs pipe{};         // insert-pipeline rings (allocated at the first pipelined insert)
  bool pipe_ok = false;
  int pipe_grid = 0;
  DtArgs dt{};             // deletemin top-CTA execution: walker task list (bgpq_dtop.cuh)
  bool dt_ok = false;
  u32* stage_k = nullptr;  // staging for the *_host calls
  u32* stage_v = nullptr;
  u64* stage_cnt = nullptr;
  u64 stage_n = 0;
  int ds_clusters = -1;    // co-resident clusters of the cluster DELETEMIN engine (-1: not queried)
  u64* ds_base = nullptr;  // device: ops of the current deletemin call done by that engine
  u32* xk = nullptr;       // mixed calls on the cluster engine: sorted INSERT batch per op pair
  u32* xv = nullptr;
  u64 x_pairs = 0;         // pairs xk / xv hold
  u32* pair_end = nullptr; // device word: pairs of the current mixed call the engine may run
  bool attr_dt = false;    // kernel attributes set / occupancy checked on q->device
  bool attr_pipe = false;
};

namespace {

// ---- per-K kernel tables (bgpq_kernels.cu, one translation unit per K) ------------------
const KTable* ktab(u32 K, bool V) {
  switch (K) {
    case 64: return V ? &ktab_64_v() : &ktab_64_k();
    case 128: return V ? &ktab_128_v() : &ktab_128_k();
    case 256: return V ? &ktab_256_v() : &ktab_256_k();
    case 512: return V ? &ktab_512_v() : &ktab_512_k();
    case 1024: return V ? &ktab_1024_v() : &ktab_1024_k();
    case 2048: return V ? &ktab_2048_v() : &ktab_2048_k();
    case 4096: return V ? &ktab_4096_v() : &ktab_4096_k();
    default: return nullptr;
  }
}
const KTable* ktab(const bgpq* q) { return ktab(q->K, (q->flags & BGPQ_FLAG_VALUES) != 0); }

cudaError_t counted(cudaError_t e) {
  if (e == cudaSuccess) g_launches.fetch_add(1);
  return e;
}

bool valid_K(u32 K) { return K >= 64 && K <= 4096 && (K & (K - 1)) == 0; }

HeapArgs heap_args(const bgpq* q) {
  HeapArgs H;
  H.gk = q->gk;
  H.gv = (q->flags & BGPQ_FLAG_VALUES) ? q->gv : nullptr;
  H.meta = q->meta;
  H.hdr = q->hdr;
  H.cap = q->cap_nodes;
  H.xk = q->xk;
  H.xv = (q->flags & BGPQ_FLAG_VALUES) ? q->xv : nullptr;
  return H;
}

int grid_for(const bgpq* q, u64 n_ops) {
  if (q->flags & BGPQ_FLAG_SERIAL) return 1;
  long long g = q->grid_req > 0 ? q->grid_req : (long long)q->sm_count * q->occ;
  if ((u64)g > n_ops) g = (long long)n_ops;
  return (int)std::max(1LL, g);
}

u32 depth_host(u32 i) {
  u32 d = 0;
  while (i > 1) { i >>= 1; ++d; }
  return d;
}

// Insert-only calls in the default execution run as a level pipeline (bgpq_pipe2.cuh).
bool pipe_mode(const bgpq* q) { return !(q->flags & (BGPQ_FLAG_SERIAL | BGPQ_FLAG_LOCKS)); }
bool has_pipe(const bgpq* q) { return ktab(q)->pipe_launch != nullptr; }

// Allocates the pipeline rings and checks that its grid (one CTA per SM: root stage, one stage
// per heap depth, sorters) is co-resident.  Returns BGPQ_OK, BGPQ_ENOMEM (allocation),
// BGPQ_ECUDA (attribute / occupancy query) or BGPQ_EINVAL (heap deeper than the grid holds
// stages for; cannot happen for capacities that fit a B200's memory).
int ensure_pipe(bgpq* q) {
  if (q->pipe_ok) return BGPQ_OK;
  const bool V = (q->flags & BGPQ_FLAG_VALUES) != 0;
  const u32 depth = depth_host(q->cap_nodes);
  int occ = 0;
  if (ktab(q)->pipe_prepare(&occ) != cudaSuccess) return fail(BGPQ_ECUDA);
  if (occ < 1) return fail(BGPQ_ECUDA);
  const int grid = q->sm_count;  // one CTA per SM, all co-resident (occ >= 1)
  if ((int)depth + 2 > grid || depth >= PIPE_MAXL) return fail(BGPQ_EINVAL);
  PipeArgs& P = q->pipe;
  const size_t kb = (size_t)q->K * sizeof(u32);
  bool ok = cudaMalloc(&P.ctl, PC_WORDS * sizeof(u32)) == cudaSuccess;
  ok = ok && cudaMalloc(&P.sbk, PIPE_NSB * kb) == cudaSuccess;
  ok = ok && cudaMalloc(&P.sready, PIPE_NSB * sizeof(u32)) == cudaSuccess;
  ok = ok && cudaMalloc(&P.rk, (size_t)PIPE_MAXL * PIPE_NL * kb) == cudaSuccess;
  ok = ok && cudaMalloc(&P.rflag, (size_t)PIPE_MAXL * PIPE_NL * sizeof(u64)) == cudaSuccess;
  if (V) {
    ok = ok && cudaMalloc(&P.sbv, PIPE_NSB * kb) == cudaSuccess;
    ok = ok && cudaMalloc(&P.rv, (size_t)PIPE_MAXL * PIPE_NL * kb) == cudaSuccess;
  }
  if (!ok) {
    cudaGetLastError();
    return fail(BGPQ_ENOMEM);
  }
  P.depth = depth;
  q->pipe_grid = grid;
  q->pipe_ok = true;
  return BGPQ_OK;
}

// Deletemin-only calls in the default execution: top CTA + walkers (bgpq_dtop.cuh).
// Debug bit 16 routes them to the per-node-lock execution instead (A/B comparisons).
bool dt_mode(const bgpq* q) { return pipe_mode(q) && !(g_debug & 16u); }
bool has_dt(const bgpq* q) { return ktab(q)->dt_launch != nullptr; }

// Walker task list: one entry per hand-off (at most one per refill node, <= cap_nodes) plus
// one ticket per walker CTA past the final count (each walker takes tickets until it sees
// the count), so cap_nodes + 2 + grid entries are ever indexed.
size_t dt_tasks(const bgpq* q) { return (size_t)q->cap_nodes + 2 + (size_t)q->sm_count; }

int ensure_dt(bgpq* q) {
  if (q->dt_ok) return BGPQ_OK;
  const bool V = (q->flags & BGPQ_FLAG_VALUES) != 0;
  int occ = 0;
  if (has_dt(q) && (ktab(q)->dt_prepare(&occ) != cudaSuccess || occ < 1)) return fail(BGPQ_ECUDA);
  DtArgs& D = q->dt;
  const size_t n = dt_tasks(q);
  bool ok = cudaMalloc(&D.task_node, n * sizeof(u32)) == cudaSuccess;
  ok = ok && cudaMalloc(&D.task_seq, n * sizeof(u32)) == cudaSuccess;
  ok = ok && cudaMalloc(&D.task_go, n * sizeof(u64)) == cudaSuccess;
  ok = ok && cudaMalloc(&D.ctl, 32 * sizeof(u32)) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    return fail(BGPQ_ENOMEM);
  }
  if (cudaMemset(D.task_seq, 0, n * sizeof(u32)) != cudaSuccess || cudaMemset(D.task_go, 0, n * sizeof(u64)) != cudaSuccess ||
      cudaMemset(D.ctl, 0, 32 * sizeof(u32)) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  D.epoch = 0;
  if (cudaMalloc(&q->ds_base, sizeof(u64)) != cudaSuccess) {
    cudaGetLastError();
    return fail(BGPQ_ENOMEM);
  }
  q->dt_ok = true;
  return BGPQ_OK;
}

// The cluster engine (bgpq_dsys.cuh) runs the steady state of a deletemin call first when the
// output is 16-B aligned for its bulk stores and enough clusters are co-resident (debug bit 256
// disables it for A/B comparisons).
bool ds_usable(bgpq* q, const CallArgs& C) {
  if (g_debug & 256u) return false;
  if (q->K < 256) return false;
  if ((reinterpret_cast<uintptr_t>(C.out_k) & 15u) || (C.out_v && (reinterpret_cast<uintptr_t>(C.out_v) & 15u)))
    return false;
  if (C.n < (u64)q->K) return false;
  if (!ktab(q)->ds_launch) return false;
  if (q->ds_clusters < 0) {
    int cl = 0;
    if (ktab(q)->ds_prepare(q->sm_count, &cl) != cudaSuccess) {
      cudaGetLastError();
      cl = 0;
    }
    q->ds_clusters = cl;
  }
  return q->ds_clusters >= 8;  // the role cluster + >= 7 clusters of walkers
}

// Mixed calls whose op stream starts with (INSERT(K), DELETEMIN(K)) pairs (the utilisation
// workload) run those pairs on the cluster engine (bgpq_dsys.cuh: ds_r0_mixed) and the
// rest on the per-node-lock engine; debug bit 256 disables it like for deletemin calls.
bool dsm_usable(bgpq* q, const CallArgs& C) {
  if (!ktab(q)->ms_launch || C.n_ops < 2) return false;
  CallArgs C1 = C;
  C1.n = q->K;  // ds_usable's size test is about deletemin calls
  return ds_usable(q, C1);
}

int ensure_mixed(bgpq* q, u64 pairs) {
  if (!q->pair_end && cudaMalloc(&q->pair_end, sizeof(u32)) != cudaSuccess) {
    cudaGetLastError();
    return fail(BGPQ_ENOMEM);
  }
  if (q->x_pairs >= pairs) return BGPQ_OK;
  cudaFree(q->xk);
  cudaFree(q->xv);
  q->xk = q->xv = nullptr;
  q->x_pairs = 0;
  const size_t bytes = pairs * (size_t)q->K * sizeof(u32);
  bool ok = cudaMalloc(&q->xk, bytes) == cudaSuccess;
  if (ok && (q->flags & BGPQ_FLAG_VALUES)) ok = cudaMalloc(&q->xv, bytes) == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    return fail(BGPQ_ENOMEM);
  }
  q->x_pairs = pairs;
  return BGPQ_OK;
}

int dt_epoch(bgpq* q, cudaStream_t s) {
  DtArgs& D = q->dt;
  D.epoch += 1;
  if (D.epoch == 0) {  // wrapped: clear the stale epochs
    D.epoch = 1;
    if (cudaMemsetAsync(D.task_seq, 0, dt_tasks(q) * sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
    if (cudaMemsetAsync(D.task_go, 0, dt_tasks(q) * sizeof(u64), s) != cudaSuccess) return fail(BGPQ_ECUDA);
  }
  if (cudaMemsetAsync(D.ctl, 0, 2 * sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
  return BGPQ_OK;
}

int run_call(bgpq* q, const CallArgs& C, cudaStream_t s) {
  const bool V = (q->flags & BGPQ_FLAG_VALUES) != 0;
  if (C.mode == MODE_DELETEMIN && dt_mode(q)) {
    if (int rc = ensure_dt(q)) return rc;
    DtArgs D = q->dt;
    D.op_base = nullptr;
    if (ds_usable(q, C)) {  // steady state on the cluster engine, the rest on the top CTA
      if (int rc = dt_epoch(q, s)) return rc;
      D = q->dt;
      D.op_base = q->ds_base;
      if (counted(ktab(q)->ds_launch(q->ds_clusters * DS_CL, heap_args(q), C, D, s)) != cudaSuccess)
        return fail(BGPQ_ECUDA);
    }
    if (!has_dt(q)) {  // K >= 2048: the rest of the call on the per-node-lock engine
      CallArgs C2 = C;
      C2.op_base = D.op_base;
      if (cudaMemsetAsync(q->hdr + H_CALL, 0, 2 * sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
      if (counted(ktab(q)->locks_launch(grid_for(q, C.n_ops), heap_args(q), C2, s)) != cudaSuccess)
        return fail(BGPQ_ECUDA);
      return BGPQ_OK;
    }
    if (int rc = dt_epoch(q, s)) return rc;
    const u64* base = D.op_base;
    D = q->dt;
    D.op_base = const_cast<u64*>(base);
    if (counted(ktab(q)->dt_launch(q->sm_count, heap_args(q), C, D, s)) != cudaSuccess) return fail(BGPQ_ECUDA);
    return BGPQ_OK;
  }
  if (C.mode == MODE_INSERT && pipe_mode(q) && has_pipe(q)) {
    if (int rc = ensure_pipe(q)) return rc;
    const PipeArgs& P = q->pipe;
    bool ok = cudaMemsetAsync(P.ctl, 0, PC_WORDS * sizeof(u32), s) == cudaSuccess;
    ok = ok && cudaMemsetAsync(P.sready, 0, PIPE_NSB * sizeof(u32), s) == cudaSuccess;
    ok = ok && cudaMemsetAsync(P.rflag, 0, (size_t)PIPE_MAXL * PIPE_NL * sizeof(u64), s) == cudaSuccess;
    if (!ok) return fail(BGPQ_ECUDA);
    if (counted(ktab(q)->pipe_launch(q->pipe_grid, heap_args(q), P, C, s)) != cudaSuccess) return fail(BGPQ_ECUDA);
    return BGPQ_OK;
  }
  if (C.mode == MODE_MIXED && dt_mode(q) && dsm_usable(q, C)) {
    // leading op pairs: Sort(items) of every pair's INSERT, then the cluster engine; the
    // per-node-lock engine continues at the first op the engine did not run (H_FETCH)
    if (int rc = ensure_dt(q)) return rc;
    if (int rc = ensure_mixed(q, C.n_ops / 2)) return rc;
    if (cudaMemsetAsync(q->pair_end, 0xFF, sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
    CallArgs Cm = C;
    Cm.pair_end = q->pair_end;
    if (counted(ktab(q)->ms_launch(q->sm_count * 4, heap_args(q), Cm, s)) != cudaSuccess) return fail(BGPQ_ECUDA);
    if (int rc = dt_epoch(q, s)) return rc;
    DtArgs D = q->dt;
    D.op_base = q->ds_base;
    if (cudaMemsetAsync(q->hdr + H_CALL, 0, 2 * sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
    if (counted(ktab(q)->ds_launch(q->ds_clusters * DS_CL, heap_args(q), Cm, D, s)) != cudaSuccess)
      return fail(BGPQ_ECUDA);
    if (counted(ktab(q)->locks_launch(grid_for(q, C.n_ops), heap_args(q), C, s)) != cudaSuccess)
      return fail(BGPQ_ECUDA);
    return BGPQ_OK;
  }
  // reset the per-call ticket and fetch counter (header words H_CALL, H_FETCH)
  if (cudaMemsetAsync(q->hdr + H_CALL, 0, 2 * sizeof(u32), s) != cudaSuccess) return fail(BGPQ_ECUDA);
  if (counted(ktab(q)->locks_launch(grid_for(q, C.n_ops), heap_args(q), C, s)) != cudaSuccess) return fail(BGPQ_ECUDA);
  return BGPQ_OK;
}

}  // namespace

extern "C" {

bgpq_t* bgpq_create_ex(uint64_t capacity, uint32_t K, uint32_t flags) {
  g_last_error = BGPQ_OK;
  if (!valid_K(K) || capacity == 0 || (flags & ~7u)) {
    fail(BGPQ_EINVAL);
    return nullptr;
  }
  bgpq* q = new bgpq();
  q->K = K;
  q->flags = flags;
  q->capacity = capacity;
  const u64 nodes = (capacity + K - 1) / K + 1;
  if (nodes + 1 > 0xFFFFFFF0ull) {
    delete q;
    fail(BGPQ_EINVAL);
    return nullptr;
  }
  q->cap_nodes = (u32)std::max<u64>(2, nodes);
  q->slots = (u64)q->cap_nodes + 1;
  if (cudaGetDevice(&q->device) != cudaSuccess ||
      cudaDeviceGetAttribute(&q->sm_count, cudaDevAttrMultiProcessorCount, q->device) != cudaSuccess) {
    delete q;
    fail(BGPQ_ECUDA);
    return nullptr;
  }
  const bool V = (flags & BGPQ_FLAG_VALUES) != 0;
  if (!ktab(K, V)->locks_prepare || ktab(K, V)->locks_prepare(&q->occ) != cudaSuccess || q->occ < 1) {
    if (!ktab(K, V)->locks_prepare) {  // (K, values) combination that no execution fits
      delete q;
      fail(BGPQ_EINVAL);
      return nullptr;
    }
    delete q;
    fail(BGPQ_ECUDA);
    return nullptr;
  }
  const size_t nbytes = q->slots * (size_t)K * sizeof(u32);
  bool ok = cudaMalloc(&q->gk, nbytes) == cudaSuccess;
  if (ok && V) ok = cudaMalloc(&q->gv, nbytes) == cudaSuccess;
  if (ok) ok = cudaMalloc(&q->meta, q->slots * sizeof(NodeMeta)) == cudaSuccess;
  if (ok) ok = cudaMalloc(&q->hdr, HEADER_WORDS * sizeof(u32)) == cudaSuccess;
  if (ok) ok = cudaMemset(q->meta, 0, q->slots * sizeof(NodeMeta)) == cudaSuccess;
  if (ok) ok = cudaMemset(q->hdr, 0, HEADER_WORDS * sizeof(u32)) == cudaSuccess;
  if (ok) ok = cudaDeviceSynchronize() == cudaSuccess;
  if (!ok) {
    cudaGetLastError();
    bgpq_destroy(q);
    fail(BGPQ_ENOMEM);
    return nullptr;
  }
  return q;
}

bgpq_t* bgpq_create(uint64_t capacity, uint32_t K) { return bgpq_create_ex(capacity, K, BGPQ_FLAG_VALUES); }

void bgpq_destroy(bgpq_t* q) {
  if (!q) return;
  cudaDeviceSynchronize();
  cudaFree(q->gk);
  cudaFree(q->gv);
  cudaFree(q->meta);
  cudaFree(q->hdr);
  cudaFree(q->stage_k);
  cudaFree(q->stage_v);
  cudaFree(q->stage_cnt);
  cudaFree(q->dt.task_node);
  cudaFree(q->dt.task_seq);
  cudaFree(q->dt.task_go);
  cudaFree(q->ds_base);
  cudaFree(q->xk);
  cudaFree(q->xv);
  cudaFree(q->pair_end);
  cudaFree(q->dt.ctl);
  PipeArgs& P = q->pipe;
  u32* pbufs[] = {P.ctl, P.sbk, P.sbv, P.sready, P.rk, P.rv};
  for (u32* b : pbufs) cudaFree(b);
  cudaFree(P.rflag);
  delete q;
}

int bgpq_insert(bgpq_t* q, const uint32_t* keys, const uint32_t* vals, uint64_t n, void* stream) {
  if (!q) return fail(BGPQ_EINVAL);
  if (n == 0) return BGPQ_OK;
  if (!keys) return fail(BGPQ_EINVAL);
  CallArgs C;
  memset(&C, 0, sizeof(C));
  C.mode = MODE_INSERT;
  C.n = n;
  C.n_ops = (n + q->K - 1) / q->K;
  C.in_k = keys;
  C.in_v = (q->flags & BGPQ_FLAG_VALUES) ? vals : nullptr;
  C.debug = g_debug;
  C.prog = nullptr;
  return run_call(q, C, (cudaStream_t)stream);
}

int bgpq_deletemin(bgpq_t* q, uint32_t* out_keys, uint32_t* out_vals, uint64_t n, uint64_t* d_count,
                   void* stream) {
  if (!q) return fail(BGPQ_EINVAL);
  if (n == 0) return BGPQ_OK;
  if (!out_keys) return fail(BGPQ_EINVAL);
  CallArgs C;
  memset(&C, 0, sizeof(C));
  C.mode = MODE_DELETEMIN;
  C.n = n;
  C.n_ops = (n + q->K - 1) / q->K;
  C.out_k = out_keys;
  C.out_v = (q->flags & BGPQ_FLAG_VALUES) ? out_vals : nullptr;
  C.d_count = reinterpret_cast<ull*>(d_count);
  C.debug = g_debug;
  C.prog = nullptr;
  return run_call(q, C, (cudaStream_t)stream);
}

int bgpq_run_mixed(bgpq_t* q, const uint8_t* op_types, const uint32_t* op_sizes, const uint64_t* in_off,
                   uint64_t n_ops, const uint32_t* in_keys, const uint32_t* in_vals, uint32_t* out_keys,
                   uint32_t* out_vals, uint32_t* op_count, uint64_t* lin_ticket, void* stream) {
  if (!q) return fail(BGPQ_EINVAL);
  if (n_ops == 0) return BGPQ_OK;
  if (!op_types || !op_sizes || !in_off || !in_keys || !out_keys || !op_count) return fail(BGPQ_EINVAL);
  CallArgs C;
  memset(&C, 0, sizeof(C));
  C.mode = MODE_MIXED;
  C.n_ops = n_ops;
  C.op_types = op_types;
  C.op_sizes = op_sizes;
  C.in_off = reinterpret_cast<const u64*>(in_off);
  C.in_k = in_keys;
  C.in_v = (q->flags & BGPQ_FLAG_VALUES) ? in_vals : nullptr;
  C.out_k = out_keys;
  C.out_v = (q->flags & BGPQ_FLAG_VALUES) ? out_vals : nullptr;
  C.op_count = op_count;
  C.lin_ticket = reinterpret_cast<ull*>(lin_ticket);
  C.debug = g_debug;
  C.prog = nullptr;
  return run_call(q, C, (cudaStream_t)stream);
}

int bgpq_size(bgpq_t* q, uint64_t* out_size, void* stream) {
  if (!q || !out_size) return fail(BGPQ_EINVAL);
  u32 h[4];
  cudaStream_t s = (cudaStream_t)stream;
  if (cudaMemcpyAsync(h, q->hdr, sizeof(h), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  *out_size = h[H_HS] == 0 ? 0 : (u64)h[H_RS] + h[H_PS] + (u64)(h[H_HS] - 1) * q->K;
  if (h[H_ERR]) return fail((int)h[H_ERR]);
  return BGPQ_OK;
}

static int ensure_stage(bgpq* q, u64 n) {
  if (q->stage_n >= n) return BGPQ_OK;
  cudaFree(q->stage_k);
  cudaFree(q->stage_v);
  q->stage_k = q->stage_v = nullptr;
  if (!q->stage_cnt && cudaMalloc(&q->stage_cnt, sizeof(u64)) != cudaSuccess) return fail(BGPQ_ENOMEM);
  if (cudaMalloc(&q->stage_k, n * sizeof(u32)) != cudaSuccess) return fail(BGPQ_ENOMEM);
  if ((q->flags & BGPQ_FLAG_VALUES) && cudaMalloc(&q->stage_v, n * sizeof(u32)) != cudaSuccess)
    return fail(BGPQ_ENOMEM);
  q->stage_n = n;
  return BGPQ_OK;
}

int bgpq_insert_host(bgpq_t* q, const uint32_t* keys_host, const uint32_t* vals_host, uint64_t n, void* stream) {
  if (!q || (n && !keys_host)) return fail(BGPQ_EINVAL);
  if (n == 0) return BGPQ_OK;
  int rc = ensure_stage(q, n);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  const bool V = (q->flags & BGPQ_FLAG_VALUES) && vals_host;
  if (cudaMemcpyAsync(q->stage_k, keys_host, n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) return fail(BGPQ_ECUDA);
  if (V && cudaMemcpyAsync(q->stage_v, vals_host, n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  rc = bgpq_insert(q, q->stage_k, V ? q->stage_v : nullptr, n, stream);
  if (rc) return rc;
  if (cudaStreamSynchronize(s) != cudaSuccess) return fail(BGPQ_ECUDA);
  return BGPQ_OK;
}

int bgpq_deletemin_host(bgpq_t* q, uint32_t* out_keys_host, uint32_t* out_vals_host, uint64_t n,
                        uint64_t* out_count_host, void* stream) {
  if (!q || (n && !out_keys_host)) return fail(BGPQ_EINVAL);
  if (n == 0) {
    if (out_count_host) *out_count_host = 0;
    return BGPQ_OK;
  }
  int rc = ensure_stage(q, n);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  const bool V = (q->flags & BGPQ_FLAG_VALUES) && out_vals_host;
  if (cudaMemsetAsync(q->stage_cnt, 0, sizeof(u64), s) != cudaSuccess) return fail(BGPQ_ECUDA);
  rc = bgpq_deletemin(q, q->stage_k, V ? q->stage_v : nullptr, n, q->stage_cnt, stream);
  if (rc) return rc;
  u64 cnt = 0;
  if (cudaMemcpyAsync(&cnt, q->stage_cnt, sizeof(u64), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  if (cnt && cudaMemcpyAsync(out_keys_host, q->stage_k, cnt * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  if (cnt && V && cudaMemcpyAsync(out_vals_host, q->stage_v, cnt * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  if (cudaStreamSynchronize(s) != cudaSuccess) return fail(BGPQ_ECUDA);
  if (out_count_host) *out_count_host = cnt;
  return BGPQ_OK;
}

uint64_t bgpq_slots(bgpq_t* q) { return q ? q->slots : 0; }

int bgpq_dump(bgpq_t* q, uint32_t* node_keys, uint32_t* node_vals, uint32_t* meta, uint64_t* hdr) {
  if (!q) return fail(BGPQ_EINVAL);
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(BGPQ_ECUDA);
  const size_t nbytes = q->slots * (size_t)q->K * sizeof(u32);
  if (node_keys && cudaMemcpy(node_keys, q->gk, nbytes, cudaMemcpyDeviceToHost) != cudaSuccess) return fail(BGPQ_ECUDA);
  if (node_vals && q->gv && cudaMemcpy(node_vals, q->gv, nbytes, cudaMemcpyDeviceToHost) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  if (meta && cudaMemcpy(meta, q->meta, q->slots * sizeof(NodeMeta), cudaMemcpyDeviceToHost) != cudaSuccess)
    return fail(BGPQ_ECUDA);
  if (hdr) {
    u32 h[4];
    if (cudaMemcpy(h, q->hdr, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess) return fail(BGPQ_ECUDA);
    for (int i = 0; i < 4; ++i) hdr[i] = h[i];
  }
  return BGPQ_OK;
}

int bgpq_stats(bgpq_t* q, uint64_t* out, int n) {
  if (!q || !out || n < 0) return fail(BGPQ_EINVAL);
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(BGPQ_ECUDA);
  ull st[NSTAT];
  if (cudaMemcpy(st, q->hdr + H_STAT, sizeof(st), cudaMemcpyDeviceToHost) != cudaSuccess) return fail(BGPQ_ECUDA);
  for (int i = 0; i < n && i < NSTAT; ++i) out[i] = st[i];
  return BGPQ_OK;
}

int bgpq_timers(bgpq_t* q, uint64_t* out32) {
  if (!q || !out32) return fail(BGPQ_EINVAL);
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(BGPQ_ECUDA);
  if (cudaMemcpy(out32, q->hdr + H_TIME, 32 * sizeof(u64), cudaMemcpyDeviceToHost) != cudaSuccess) return fail(BGPQ_ECUDA);
  return BGPQ_OK;
}

int bgpq_set_grid(bgpq_t* q, int ctas) {
  if (!q || ctas < 0) return fail(BGPQ_EINVAL);
  if (ctas > q->sm_count * q->occ) return fail(BGPQ_EINVAL);  // must stay co-resident
  q->grid_req = ctas;
  return BGPQ_OK;
}

int bgpq_grid(bgpq_t* q) { return q ? grid_for(q, ~0ull) : 0; }

int bgpq_view(bgpq_t* q, bgpq_view_t* out) {
  if (!q || !out) return fail(BGPQ_EINVAL);
  out->keys = q->gk;
  out->vals = (q->flags & BGPQ_FLAG_VALUES) ? q->gv : nullptr;
  out->meta = q->meta;
  out->hdr = q->hdr;
  out->cap = q->cap_nodes;
  out->K = q->K;
  out->flags = q->flags;
  out->device = q->device;
  out->sm_count = q->sm_count;
  out->ctas = q->grid_req;
  return BGPQ_OK;
}

int bgpq_set_debug(uint32_t bits) {
  g_debug = bits;
  return BGPQ_OK;
}

uint64_t bgpq_launch_count(void) { return g_launches.load(); }

int bgpq_last_error(void) { return g_last_error; }
const char* bgpq_last_error_msg(void) { return g_last_msg; }

const char* bgpq_strerror(int code) {
  switch (code) {
    case BGPQ_OK: return "ok";
    case BGPQ_EINVAL: return "invalid argument";
    case BGPQ_ENOMEM: return "device allocation failed";
    case BGPQ_EFULL: return "capacity exceeded (sticky; the overflowing batch was dropped)";
    case BGPQ_ECUDA: return "CUDA error";
    default: return "unknown error";
  }
}

}  // extern "C"
