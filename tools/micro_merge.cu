// tools/micro_merge.cu — correctness + latency of the SORT_SPLIT merge variants on one CTA.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o micro_merge micro_merge.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_icpp_chenhjz21_b200/csrc/bgpq_prim.cuh"
using namespace bgpqd;

constexpr int K = 1024;

// MODE 0: cta_rank_merge (NT threads); 1: cta_path_merge; 2: cta_merge_win<NTM>
template <int NT, int NTM, int MODE, bool V>
__global__ void k_merge(const u32* in, const int* sizes, u32* out, long long* cyc, int reps) {
  __shared__ __align__(16) u32 z[K], w[K], x[K], y[K], zv[K], wv[K], xv[K], yv[K];
  const int na = sizes[0], nb = sizes[1], ma = sizes[2];
  for (int i = threadIdx.x; i < K; i += NT) {
    z[i] = in[i]; w[i] = in[K + i]; zv[i] = i; wv[i] = 0x10000u + i;
  }
  __syncthreads();
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    if constexpr (MODE == 0) cta_rank_merge<K, NT, V>(z, zv, na, w, wv, nb, ma, x, xv, y, yv);
    else if constexpr (MODE == 1) cta_path_merge<K, NT, V>(z, zv, na, w, wv, nb, ma, x, xv, y, yv);
    else if constexpr (MODE == 2) cta_merge_win<K, NTM, V>(z, zv, na, w, wv, nb, ma, x, xv, y, yv);
    else if constexpr (MODE == 3) cta_merge_warp<K, NTM, V>(z, zv, na, w, wv, nb, ma, x, xv, y, yv);
    else if constexpr (MODE == 7) bitonic_split_full<K, NTM, V>(threadIdx.x, 1, z, zv, w, wv, x, xv, y, yv);
    else if constexpr (MODE == 4) { if (threadIdx.x == 0) x[r & 1023] = r; }
    else if constexpr (MODE == 5) { const int c = warp_corank(z, na, w, nb, (threadIdx.x >> 5) * 128); if ((threadIdx.x & 31) == 0) x[threadIdx.x >> 5] = c; }
    else if constexpr (MODE == 6) {
      const int d = threadIdx.x * 4; int lo = max(0, d - nb), hi = min(d, na);
#pragma unroll
      for (int it = 0; it < 11; ++it) { const int len = hi - lo; const int mid = lo + (len >> 1); const bool act = len > 0;
        const u32 a = z[act ? mid : 0]; const u32 b = w[act ? d - 1 - mid : 0]; const bool right = act && (a <= b);
        lo = right ? mid + 1 : lo; hi = (act && !right) ? mid : hi; }
      x[threadIdx.x] = lo;
    }
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[0] = (t1 - t0) / reps;
  for (int i = threadIdx.x; i < K; i += NT) {
    out[i] = x[i]; out[K + i] = y[i]; out[2 * K + i] = xv[i]; out[3 * K + i] = yv[i];
  }
}

static unsigned long long rng = 88172645463325252ull;
static u32 nxt() { rng ^= rng << 13; rng ^= rng >> 7; rng ^= rng << 17; return (u32)(rng >> 16); }

template <int NT, int NTM, int MODE, bool V>
bool run(const char* name, u32* d_in, int* d_sz, u32* d_out, long long* d_cyc, bool timing) {
  bool ok = true;
  std::vector<u32> z(K), w(K), out(4 * K);
  for (int tcase = 0; tcase < (timing ? 1 : 300); ++tcase) {
    int na = timing ? K : (int)(nxt() % (K + 1));
    int nb = timing ? K : (int)(nxt() % (K + 1));
    if (!timing && tcase % 7 == 0) na = K;
    if (!timing && tcase % 5 == 0) nb = K;
    int ma = timing ? K : (int)(nxt() % (na + nb + 1));
    if (MODE == 7) { na = nb = ma = K; }
    if (!timing && tcase % 3 == 0) ma = std::min(K, na + nb);
    if (ma > K || na + nb - ma > K) { ma = std::min(K, na + nb); if (na + nb - ma > K) continue; }
    const u32 mod = (tcase % 4 == 0) ? 16u : 0xFFFFFFFFu;
    for (int i = 0; i < K; ++i) { z[i] = nxt() % mod; w[i] = nxt() % mod; }
    if (tcase % 11 == 0) for (int i = 0; i < K; ++i) z[i] = 0xFFFFFFFFu;
    std::sort(z.begin(), z.begin() + na);
    std::sort(w.begin(), w.begin() + nb);
    std::vector<u32> in(2 * K);
    for (int i = 0; i < K; ++i) { in[i] = z[i]; in[K + i] = w[i]; }
    int sz[3] = {na, nb, ma};
    cudaMemcpy(d_in, in.data(), 8 * K, cudaMemcpyHostToDevice);
    cudaMemcpy(d_sz, sz, 12, cudaMemcpyHostToDevice);
    k_merge<NT, NTM, MODE, V><<<1, NT>>>(d_in, d_sz, d_out, d_cyc, timing ? 200 : 1);
    cudaMemcpy(out.data(), d_out, 16 * K, cudaMemcpyDeviceToHost);
    // reference: stable merge (Z first on ties), split at ma
    std::vector<u32> mk, mv;
    int i = 0, j = 0;
    while (i < na || j < nb) {
      if (j >= nb || (i < na && z[i] <= w[j])) { mk.push_back(z[i]); mv.push_back(i); ++i; }
      else { mk.push_back(w[j]); mv.push_back(0x10000u + j); ++j; }
    }
    for (int p = 0; p < na + nb; ++p) {
      const u32 gk = p < ma ? out[p] : out[K + p - ma];
      const u32 gv = p < ma ? out[2 * K + p] : out[3 * K + p - ma];
      if (gk != mk[p]) { ok = false; break; }
      if (V) {  // value must pair with its key
        const u32 src = (gv >= 0x10000u) ? w[gv - 0x10000u] : z[gv];
        if (src != gk) { ok = false; break; }
        if (MODE != 0 && gv != mv[p]) { ok = false; break; }  // stable variants: exact
      }
    }
    if (!ok) { printf("%s: MISMATCH na=%d nb=%d ma=%d\n", name, na, nb, ma); break; }
  }
  if (timing) {
    long long c;
    cudaMemcpy(&c, d_cyc, 8, cudaMemcpyDeviceToHost);
    printf("%-34s 2x%d: %lld cycles\n", name, K, c);
  } else {
    printf("%-34s correctness %s\n", name, ok ? "ok" : "FAILED");
  }
  return ok;
}

int main() {
  u32 *d_in, *d_out; int* d_sz; long long* d_cyc;
  cudaMalloc(&d_in, 8 * K); cudaMalloc(&d_out, 16 * K); cudaMalloc(&d_sz, 16); cudaMalloc(&d_cyc, 8);
  bool ok = true;
  for (int timing = 1; timing < 2; ++timing) {
    run<512, 16, 4, false>("EMPTY loop (syncthreads only)", d_in, d_sz, d_out, d_cyc, true);
    run<512, 16, 5, false>("warp_corank only NW=16", d_in, d_sz, d_out, d_cyc, true);
    run<512, 16, 6, false>("path search only NT=512", d_in, d_sz, d_out, d_cyc, true);
  }
  for (int timing = 0; timing < 2; ++timing) {
    ok &= run<512, 512, 0, false>("rank_merge NT=512 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 1, false>("path_merge NT=512 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 2, false>("merge_win NTM=512 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 256, 2, false>("merge_win NTM=256 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 128, 2, false>("merge_win NTM=128 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<1024, 1024, 2, false>("merge_win NTM=1024 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 7, false>("bitonic_full NT=512 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<256, 256, 7, false>("bitonic_full NT=256 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<128, 128, 7, false>("bitonic_full NT=128 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 7, true>("bitonic_full NT=512 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<256, 256, 7, true>("bitonic_full NT=256 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 4, 3, false>("merge_warp NW=4 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 8, 3, false>("merge_warp NW=8 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 16, 3, false>("merge_warp NW=16 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<1024, 32, 3, false>("merge_warp NW=32 keys", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 8, 3, true>("merge_warp NW=8 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 16, 3, true>("merge_warp NW=16 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 0, true>("rank_merge NT=512 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 512, 2, true>("merge_win NTM=512 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 256, 2, true>("merge_win NTM=256 key+val", d_in, d_sz, d_out, d_cyc, timing);
    ok &= run<512, 128, 2, true>("merge_win NTM=128 key+val", d_in, d_sz, d_out, d_cyc, timing);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s, all correct: %s\n", cudaGetErrorString(e), ok ? "yes" : "NO");
  return ok ? 0 : 1;
}
