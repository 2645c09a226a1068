// bgpq_kernels.cu — the kernel table of one (K, values) instantiation (bgpq_ktab.h).
// Compiled once per K in {64, ..., 4096} and V in {0, 1} with -DBGPQ_K / -DBGPQ_V.  An
// execution whose shared-memory footprint exceeds the 227 KB per CTA at this (K, V) is left
// out of the table (nullptr); the host then uses another execution for that call.
#include "bgpq_ktab.h"

#ifndef BGPQ_K
#error "compile with -DBGPQ_K=<64..4096> -DBGPQ_V=<0|1>"
#endif

namespace {

using namespace bgpqd;
constexpr int K = BGPQ_K;
constexpr bool V = BGPQ_V != 0;
constexpr size_t SMEM_MAX = 232448;  // 227 KB opt-in shared memory per CTA (sm_100)

constexpr bool kLocks = locks_smem_bytes<K, V>() <= SMEM_MAX;
constexpr bool kDt = K <= 1024 && dt_smem_bytes<K, V>() <= SMEM_MAX;
constexpr bool kDs = K >= 256 && ds_smem_bytes<K, V>() <= SMEM_MAX;
constexpr bool kPipe = pipe2_smem_bytes<K, V>() <= SMEM_MAX;

cudaError_t locks_prepare(int* occ) {
  if constexpr (kLocks) {
    auto kern = bgpq_locks_kernel<K, V, NT>;
    const size_t smem = locks_smem_bytes<K, V>();
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, NT + 32, smem);
  }
  return cudaErrorInvalidValue;
}
cudaError_t locks_launch(int grid, const HeapArgs& H, const CallArgs& C, cudaStream_t s) {
  if constexpr (kLocks) {
    bgpq_locks_kernel<K, V, NT><<<grid, NT + 32, locks_smem_bytes<K, V>(), s>>>(H, C);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}
cudaError_t dt_prepare(int* occ) {
  if constexpr (kDt) {
    auto kern = bgpq_dtop_kernel<K, V>;
    const size_t smem = dt_smem_bytes<K, V>();
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, DT_BLOCK, smem);
  }
  return cudaErrorInvalidValue;
}
cudaError_t dt_launch(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s) {
  if constexpr (kDt) {
    bgpq_dtop_kernel<K, V><<<grid, DT_BLOCK, dt_smem_bytes<K, V>(), s>>>(H, C, D);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}
cudaError_t ds_prepare(int sm_count, int* clusters) {
  *clusters = 0;
  if constexpr (kDs) {
    auto kern = bgpq_dsys_kernel<K, V>;
    const size_t smem = ds_smem_bytes<K, V>();
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((sm_count / DS_CL) * DS_CL);
    cfg.blockDim = dim3(DS_BLOCK);
    cfg.dynamicSmemBytes = smem;
    return cudaOccupancyMaxActiveClusters(clusters, kern, &cfg);
  }
  return cudaSuccess;
}
cudaError_t ds_launch(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s) {
  if constexpr (kDs) {
    bgpq_dsys_kernel<K, V><<<grid, DS_BLOCK, ds_smem_bytes<K, V>(), s>>>(H, C, D);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}
cudaError_t ms_launch(int grid, const HeapArgs& H, const CallArgs& C, cudaStream_t s) {
  if constexpr (kDs) {
    static_assert(!kDs || msort_smem_bytes<K, V>() <= 48 * 1024, "msort fits the default smem");
    bgpq_msort_kernel<K, V, NT><<<grid, NT, msort_smem_bytes<K, V>(), s>>>(H, C);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}
cudaError_t pipe_prepare(int* occ) {
  if constexpr (kPipe) {
    auto kern = bgpq_ins_pipe2_kernel<K, V, NT>;
    const size_t smem = pipe2_smem_bytes<K, V>();
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, NT + 64, smem);
  }
  return cudaErrorInvalidValue;
}
cudaError_t pipe_launch(int grid, const HeapArgs& H, const PipeArgs& P, const CallArgs& C, cudaStream_t s) {
  if constexpr (kPipe) {
    bgpq_ins_pipe2_kernel<K, V, NT><<<grid, NT + 64, pipe2_smem_bytes<K, V>(), s>>>(H, P, C);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}

const KTable kTable = {kLocks ? locks_prepare : nullptr, kLocks ? locks_launch : nullptr,
                       kDt ? dt_prepare : nullptr,       kDt ? dt_launch : nullptr,
                       kDs ? ds_prepare : nullptr,       kDs ? ds_launch : nullptr,
                       kDs ? ms_launch : nullptr,
                       kPipe ? pipe_prepare : nullptr,   kPipe ? pipe_launch : nullptr};

}  // namespace

#define BGPQ_CAT2(a, b, c) a##b##c
#define BGPQ_CAT(a, b, c) BGPQ_CAT2(a, b, c)
#if BGPQ_V
const bgpqd::KTable& BGPQ_CAT(ktab_, BGPQ_K, _v)() { return kTable; }
#else
const bgpqd::KTable& BGPQ_CAT(ktab_, BGPQ_K, _k)() { return kTable; }
#endif
