// bgpq_ktab.h — per-(K, values) kernel tables.  Each table is defined in its own
// translation unit (bgpq_kernels.cu compiled with -DBGPQ_K=<K> -DBGPQ_V=<0|1>) so the
// template instantiations of the three executions compile in parallel; bgpq_api.cu picks a
// table from the handle's K and flags.  Host-internal: not part of the C ABI.
#pragma once
#include <cuda_runtime.h>

#include "bgpq_dtop.cuh"
#include "bgpq_dsys.cuh"
#include "bgpq_pipe2.cuh"

namespace bgpqd {

constexpr int NT = 512;  // compute threads per CTA (the paper's block size)

// Entries are nullptr where an execution does not fit the shared memory at (K, V).
struct KTable {
  // per-node-lock execution (bgpq_locks.cuh): prepare sets the smem attribute and returns
  // co-resident CTAs per SM in *occ
  cudaError_t (*locks_prepare)(int* occ);
  cudaError_t (*locks_launch)(int grid, const HeapArgs& H, const CallArgs& C, cudaStream_t s);
  // deletemin calls: top CTA + walkers (bgpq_dtop.cuh)
  cudaError_t (*dt_prepare)(int* occ);
  cudaError_t (*dt_launch)(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s);
  // deletemin calls, steady state: 3-CTA cluster + walkers (bgpq_dsys.cuh); prepare returns
  // the number of co-resident clusters in *clusters (0 if the engine cannot run)
  cudaError_t (*ds_prepare)(int sm_count, int* clusters);
  cudaError_t (*ds_launch)(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s);
  // mixed calls on the cluster engine: Sort(items) of the call's leading (INSERT(K),
  // DELETEMIN(K)) pairs into H.xk and the pair count into *C.pair_end (bgpq_dsys.cuh); the
  // pairs then run on ds_launch with C.mode = MODE_MIXED
  cudaError_t (*ms_launch)(int grid, const HeapArgs& H, const CallArgs& C, cudaStream_t s);
  // insert calls: level pipeline (bgpq_pipe2.cuh)
  cudaError_t (*pipe_prepare)(int* occ);
  cudaError_t (*pipe_launch)(int grid, const HeapArgs& H, const PipeArgs& P, const CallArgs& C, cudaStream_t s);
};

}  // namespace bgpqd

#define BGPQ_KTAB_DECL(KK)                   \
  const bgpqd::KTable& ktab_##KK##_k();      \
  const bgpqd::KTable& ktab_##KK##_v();
BGPQ_KTAB_DECL(64)
BGPQ_KTAB_DECL(128)
BGPQ_KTAB_DECL(256)
BGPQ_KTAB_DECL(512)
BGPQ_KTAB_DECL(1024)
BGPQ_KTAB_DECL(2048)
BGPQ_KTAB_DECL(4096)
#undef BGPQ_KTAB_DECL
