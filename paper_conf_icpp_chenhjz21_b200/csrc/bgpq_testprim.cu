// bgpq_testprim.cu — test-only entry point that runs the exact device primitives of the hot
// path on caller-provided tiles, so tests can compare each one with the oracle's SORT_SPLIT
// and Sort (Alg.1 l.2) over a grid of (Na, Nb, Ma) shapes.  Declared in
// include/bgpq.h (bgpq_test_prim); not used by any product call.
#include <cuda_runtime.h>

#include "../../include/bgpq.h"
#include "bgpq_dtop.cuh"

using namespace bgpqd;

namespace {

constexpr int TP_NT = 512;

// one CTA per case; tiles staged in shared memory exactly as the executions stage them
template <int K, bool V>
__global__ void __launch_bounds__(TP_NT, 1)
    bgpq_testprim_kernel(int variant, const u32* zk, const u32* zv, const u32* wk, const u32* wv,
                         const u32* na_, const u32* nb_, const u32* ma_, u32* xk, u32* xv, u32* yk, u32* yv) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  u32* sz = reinterpret_cast<u32*>(smem_raw);  // Z: 2K (cta_sort scratch needs 2 tiles of K)
  u32* sw = sz + 2 * K;                        // W: K
  u32* sx = sw + K;                            // X: 2K
  u32* sy = sx + 2 * K;                        // Y: 2K
  u32* vz = sy + 2 * K;
  u32* vw = vz + 2 * K;
  u32* vx = vw + K;
  u32* vy = vx + 2 * K;
  const int c = blockIdx.x;
  const int na = (int)na_[c], nb = (int)nb_[c], ma = (int)ma_[c];
  for (int i = threadIdx.x; i < 2 * K; i += TP_NT) {
    sz[i] = (i < na) ? zk[(size_t)c * K + i] : KEY_MAX;
    if (V) vz[i] = (i < na) ? zv[(size_t)c * K + i] : 0u;
    sx[i] = sy[i] = 0xDEADBEEFu;
    if (i < K) {
      sw[i] = (i < nb) ? wk[(size_t)c * K + i] : KEY_MAX;
      if (V) vw[i] = (i < nb) ? wv[(size_t)c * K + i] : 0u;
    }
  }
  __syncthreads();
  const u32* rk = sx;  // where X / Y end up
  const u32* rv = vx;
  const u32* qk = sy;
  const u32* qv = vy;
  if (variant == 0) {  // the locks / pipeline SORT_SPLIT (bitonic for full keys-only K >= 512)
    sort_split<K, TP_NT, V>(sz, vz, na, sw, vw, nb, ma, sx, vx, sy, vy);
  } else if (variant == 1 || variant == 2) {  // the top CTA's group split (DT_GT threads)
    if constexpr (K <= 1024) {
      if (threadIdx.x < DT_GT)
        grp_split<K, V>((int)threadIdx.x, sz, vz, na, sw, vw, nb, ma, sx, vx, sy, vy, variant == 2);
    }
  } else if (variant == 3) {  // Sort(items) of the first na entries of Z (result in X)
    if (threadIdx.x < TP_NT) {
      const bool scratch = cta_sort<K, TP_NT, V>(sz, vz, na, sx, vx);
      if (!scratch) { rk = sz; rv = vz; }
    }
  }
  __syncthreads();
  const int nx = variant == 3 ? na : ma;
  const int ny = variant == 3 ? 0 : na + nb - ma;
  for (int i = threadIdx.x; i < nx; i += TP_NT) {
    xk[(size_t)c * 2 * K + i] = rk[i];
    if (V) xv[(size_t)c * 2 * K + i] = rv[i];
  }
  for (int i = threadIdx.x; i < ny; i += TP_NT) {
    yk[(size_t)c * 2 * K + i] = qk[i];
    if (V) yv[(size_t)c * 2 * K + i] = qv[i];
  }
}

template <int K, bool V>
int run(int variant, const u32* zk, const u32* zv, const u32* wk, const u32* wv, const u32* na, const u32* nb,
        const u32* ma, u32 n_cases, u32* xk, u32* xv, u32* yk, u32* yv, cudaStream_t s) {
  const size_t smem = (size_t)7 * K * 4 * (V ? 2 : 1);
  auto kern = bgpq_testprim_kernel<K, V>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return BGPQ_ECUDA;
  kern<<<n_cases, TP_NT, smem, s>>>(variant, zk, zv, wk, wv, na, nb, ma, xk, xv, yk, yv);
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

}  // namespace

extern "C" int bgpq_test_prim(int variant, uint32_t K, int values, const uint32_t* zk, const uint32_t* zv,
                              const uint32_t* wk, const uint32_t* wv, const uint32_t* na, const uint32_t* nb,
                              const uint32_t* ma, uint32_t n_cases, uint32_t* xk, uint32_t* xv, uint32_t* yk,
                              uint32_t* yv, void* stream) {
  if (variant < 0 || variant > 3 || n_cases == 0 || !zk || !wk || !na || !nb || !ma || !xk || !yk) return BGPQ_EINVAL;
  if (values && (!zv || !wv || !xv || !yv)) return BGPQ_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
#define TP_CASE(KK)                                                                                      \
  case KK:                                                                                               \
    return values ? run<KK, true>(variant, zk, zv, wk, wv, na, nb, ma, n_cases, xk, xv, yk, yv, s)        \
                  : run<KK, false>(variant, zk, zv, wk, wv, na, nb, ma, n_cases, xk, xv, yk, yv, s);
  switch (K) {
    TP_CASE(64)
    TP_CASE(128)
    TP_CASE(256)
    TP_CASE(512)
    TP_CASE(1024)
    case 2048:
      if (variant == 1 || variant == 2) return BGPQ_EINVAL;  // the top CTA runs K <= 1024 only
      return values ? run<2048, true>(variant, zk, zv, wk, wv, na, nb, ma, n_cases, xk, xv, yk, yv, s)
                    : run<2048, false>(variant, zk, zv, wk, wv, na, nb, ma, n_cases, xk, xv, yk, yv, s);
    case 4096:
      if (variant == 1 || variant == 2 || values) return BGPQ_EINVAL;  // keys only at K = 4096
      return run<4096, false>(variant, zk, zv, wk, wv, na, nb, ma, n_cases, xk, xv, yk, yv, s);
    default:
      return BGPQ_EINVAL;
  }
#undef TP_CASE
}
