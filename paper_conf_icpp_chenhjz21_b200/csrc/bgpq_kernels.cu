// bgpq_kernels.cu — the kernel table of one (K, values) instantiation (bgpq_ktab.h).
// Compiled once per K in {64, 128, 256, 512, 1024} and V in {0, 1} with -DBGPQ_K / -DBGPQ_V.
#include "bgpq_ktab.h"

#ifndef BGPQ_K
#error "compile with -DBGPQ_K=<64|128|256|512|1024> -DBGPQ_V=<0|1>"
#endif

namespace {

using namespace bgpqd;
constexpr int K = BGPQ_K;
constexpr bool V = BGPQ_V != 0;

cudaError_t locks_prepare(int* occ) {
  auto kern = bgpq_locks_kernel<K, V, NT>;
  const size_t smem = locks_smem_bytes<K, V>();
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, NT + 32, smem);
}
cudaError_t locks_launch(int grid, const HeapArgs& H, const CallArgs& C, cudaStream_t s) {
  bgpq_locks_kernel<K, V, NT><<<grid, NT + 32, locks_smem_bytes<K, V>(), s>>>(H, C);
  return cudaGetLastError();
}
cudaError_t dt_prepare(int* occ) {
  auto kern = bgpq_dtop_kernel<K, V>;
  const size_t smem = dt_smem_bytes<K, V>();
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, DT_BLOCK, smem);
}
cudaError_t dt_launch(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s) {
  bgpq_dtop_kernel<K, V><<<grid, DT_BLOCK, dt_smem_bytes<K, V>(), s>>>(H, C, D);
  return cudaGetLastError();
}
cudaError_t ds_prepare(int sm_count, int* clusters) {
  *clusters = 0;
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
cudaError_t ds_launch(int grid, const HeapArgs& H, const CallArgs& C, const DtArgs& D, cudaStream_t s) {
  bgpq_dsys_kernel<K, V><<<grid, DS_BLOCK, ds_smem_bytes<K, V>(), s>>>(H, C, D);
  return cudaGetLastError();
}
cudaError_t pipe_prepare(int* occ) {
  auto kern = bgpq_ins_pipe2_kernel<K, V, NT>;
  const size_t smem = pipe2_smem_bytes<K, V>();
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(occ, kern, NT + 64, smem);
}
cudaError_t pipe_launch(int grid, const HeapArgs& H, const PipeArgs& P, const CallArgs& C, cudaStream_t s) {
  bgpq_ins_pipe2_kernel<K, V, NT><<<grid, NT + 64, pipe2_smem_bytes<K, V>(), s>>>(H, P, C);
  return cudaGetLastError();
}

const KTable kTable = {locks_prepare, locks_launch, dt_prepare, dt_launch, ds_prepare, ds_launch, pipe_prepare,
                       pipe_launch};

}  // namespace

#define BGPQ_CAT2(a, b, c) a##b##c
#define BGPQ_CAT(a, b, c) BGPQ_CAT2(a, b, c)
#if BGPQ_V
const bgpqd::KTable& BGPQ_CAT(ktab_, BGPQ_K, _v)() { return kTable; }
#else
const bgpqd::KTable& BGPQ_CAT(ktab_, BGPQ_K, _k)() { return kTable; }
#endif
