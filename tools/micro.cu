// tools/micro.cu — latency microbenchmarks of the BGPQ device primitives on B200
// (clock64 inside the kernel).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro micro.cu
#include <cstdio>
#include <cuda_runtime.h>
#include "../paper_conf_icpp_chenhjz21_b200/csrc/bgpq_prim.cuh"
using namespace bgpqd;

template <int NT, int K, int MODE>
__global__ void k_merge(const u32* in, long long* out, int reps) {
  __shared__ u32 z[K], w[K], x[K], y[K];
  for (int i = threadIdx.x; i < K; i += NT) { z[i] = in[2 * i]; w[i] = in[2 * i + 1]; }
  __syncthreads();
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    if (MODE == 0) cta_merge_split<NT, false>(z, nullptr, K, w, nullptr, K, K, x, nullptr, y, nullptr);
    else if (MODE == 1) cta_rank_merge<K, NT, false>(z, nullptr, K, w, nullptr, K, K, x, nullptr, y, nullptr);
    else cta_path_merge<K, NT, false>(z, nullptr, K, w, nullptr, K, K, x, nullptr, y, nullptr);
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / reps;
  if (threadIdx.x == 0) { long long h = 0; for (int i = 0; i < K; ++i) h = h * 31 + x[i] * 7 + y[i]; out[1] = h; }
}

template <int NT, int K>
__global__ void k_sort(const u32* in, long long* out, int reps) {
  __shared__ u32 a[K], t[K];
  long long tot = 0;
  for (int r = 0; r < reps; ++r) {
    for (int i = threadIdx.x; i < K; i += NT) a[i] = in[i + r];
    __syncthreads();
    long long t0 = clock64();
    cta_sort<K, NT, false>(a, nullptr, K, t, nullptr);
    long long t1 = clock64();
    tot += t1 - t0;
  }
  if (threadIdx.x == 0) out[0] = tot / reps;
  if (threadIdx.x == 0) out[1] = a[3] + t[3];
}

__global__ void k_tma(const u32* g, long long* out, int reps, size_t stride_words) {
  __shared__ __align__(128) u32 buf[2048];
  __shared__ u64 bar;
  if (threadIdx.x == 0) mbar_init(&bar, 1);
  __syncthreads();
  u32 phase = 0;
  long long tot = 0;
  for (int r = 0; r < reps; ++r) {
    __syncthreads();
    long long t0 = clock64();
    if (threadIdx.x == 0) {
      mbar_arrive_expect_tx(&bar, 4096);
      bulk_g2s(buf, g + (size_t)r * stride_words, 4096, &bar);
    }
    mbar_wait(&bar, phase);
    phase ^= 1;
    long long t1 = clock64();
    tot += t1 - t0;
  }
  if (threadIdx.x == 0) { out[0] = tot / reps; out[1] = buf[17]; }
}

// two CTAs ping-pong a lock: CTA b waits for turn==b, then hands the turn over
__global__ void k_pingpong(u32* lockw, u32* turn, long long* out, int reps, int fence) {
  if (threadIdx.x != 0) return;
  const u32 me = blockIdx.x;
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    lock_acquire(lockw);
    while (ld_relaxed(turn) != me) { lock_release(lockw); __nanosleep(20); lock_acquire(lockw); }
    st_relaxed(turn, 1 - me);
    if (fence) __threadfence();
    st_release(lockw, 0u);
  }
  long long t1 = clock64();
  out[me] = (t1 - t0) / reps;
}
// release/acquire flag ping-pong (no CAS): lower bound of an inter-SM hand-off
__global__ void k_flag(u32* flag, long long* out, int reps) {
  if (threadIdx.x != 0) return;
  const u32 me = blockIdx.x;
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    const u32 want = 2 * r + me;
    while (ld_acquire(flag) != want) {}
    st_release(flag, want + 1);
  }
  long long t1 = clock64();
  out[me] = (t1 - t0) / reps;
}
__global__ void k_fence(long long* out, u32* g, int reps) {
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) { g[threadIdx.x] = r; __threadfence(); }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / reps;
}
__global__ void k_cas(u32* g, long long* out, int reps) {
  if (threadIdx.x) return;
  long long t0 = clock64();
  u32 acc = 0;
  for (int r = 0; r < reps; ++r) acc += cas_acquire(g, acc, acc + 1);
  long long t1 = clock64();
  out[0] = (t1 - t0) / reps; out[1] = acc;
}

int main() {
  const int K = 1024;
  u32* d; long long* o; long long h[4];
  size_t big = (size_t)1 << 28;  // 1 GiB of words
  cudaMalloc(&d, big * 4); cudaMalloc(&o, 64);
  u32* hin = new u32[4 * K];
  unsigned s = 1; for (int i = 0; i < 4 * K; ++i) { s = s * 1664525u + 1013904223u; hin[i] = s; }
  // sorted z, w interleaved
  u32* zz = new u32[2 * K]; u32 a = 0, b = 0;
  for (int i = 0; i < K; ++i) { a += hin[i] >> 22; b += hin[K + i] >> 22; zz[2 * i] = a; zz[2 * i + 1] = b; }
  cudaMemcpy(d, zz, 8 * K, cudaMemcpyHostToDevice);
#define MB(NT_, M_) k_merge<NT_, K, M_><<<1, NT_>>>(d, o, 100); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost); \
  printf("hash %lld  ", h[1]); printf("%s 2x%d NT=%d: %lld cycles\n", M_ == 2 ? "path_merge_v2" : M_ ? "rank_merge" : "merge_path", K, NT_, h[0]);
  MB(512, 0) MB(512, 1) MB(1024, 1) MB(512, 2) MB(1024, 2) MB(256, 2)
  cudaMemcpy(d, hin, 16 * K, cudaMemcpyHostToDevice);
  k_sort<512, K><<<1, 512>>>(d, o, 50); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("cta_sort %d NT=512: %lld cycles\n", K, h[0]);
  cudaMemset(d, 0, big * 4);
  k_tma<<<1, 128>>>(d, o, 200, 1 << 20); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("TMA 4KB load, cold (HBM, 4MB stride): %lld cycles\n", h[0]);
  k_tma<<<1, 128>>>(d, o, 200, 1024); k_tma<<<1, 128>>>(d, o, 200, 1024); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("TMA 4KB load, warm (L2): %lld cycles\n", h[0]);
  cudaMemset(d, 0, 64);
  k_pingpong<<<2, 32>>>(d, d + 32, o, 2000, 1); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("lock ping-pong (CAS acquire + fence + release) per round: %lld / %lld cycles\n", h[0], h[1]);
  cudaMemset(d, 0, 64);
  k_pingpong<<<2, 32>>>(d, d + 32, o, 2000, 0); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("lock ping-pong (no threadfence) per round: %lld / %lld cycles\n", h[0], h[1]);
  cudaMemset(d, 0, 64);
  k_flag<<<2, 32>>>(d, o, 5000); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("flag ping-pong (ld.acquire / st.release) per round trip: %lld cycles\n", h[0]);
  k_fence<<<1, 512>>>(o, d, 1000); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("store + __threadfence: %lld cycles\n", h[0]);
  cudaMemset(d, 0, 64);
  k_cas<<<1, 32>>>(d, o, 1000); cudaMemcpy(h, o, 16, cudaMemcpyDeviceToHost);
  printf("uncontended atom.cas.acquire: %lld cycles\n", h[0]);
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
