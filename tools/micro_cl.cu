// tools/micro_cl.cu — per-operation cost of the cluster-engine primitives on B200 (thread 0 of
// CTA 0 of a 2-CTA cluster; clock64).  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_cl tools/micro_cl.cu
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned int u32;
typedef unsigned long long u64;

__device__ __forceinline__ u32 sa(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ u32 mapa(const void* p, u32 r) {
  u32 a; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(sa(p)), "r"(r)); return a;
}
constexpr int NT = 512;
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NT, 1) kmicro(long long* out, int reps) {
  __shared__ __align__(128) u32 buf[2][1024];
  __shared__ __align__(16) u64 words[64];
  __shared__ u64 bar;
  __shared__ u32 flag;
  u32 rank; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  if (threadIdx.x == 0) { asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar))); flag = 0; }
  for (int i = threadIdx.x; i < 64; i += NT) words[i] = 0;
  for (int i = threadIdx.x; i < 1024; i += NT) buf[0][i] = buf[1][i] = i;
  __syncthreads();
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  long long t[24] = {0};
  if (rank == 0 && threadIdx.x == 0) {
    const u32 rw = mapa(&words[0], 1);
    long long a, b;
    // 0: 4 relaxed cluster u64 stores (remote)
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 64 + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 128 + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 192 + 8 * (r & 7)), "l"((u64)r) : "memory");
    }
    b = clock64(); t[0] = (b - a) / reps;
    // 1: 4 weak remote u64 stores
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(rw + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(rw + 64 + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(rw + 128 + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(rw + 192 + 8 * (r & 7)), "l"((u64)r) : "memory");
    }
    b = clock64(); t[1] = (b - a) / reps;
    // 2: one v2.u64 weak remote store
    a = clock64();
    for (int r = 0; r < reps; ++r)
      asm volatile("st.shared::cluster.v2.u64 [%0], {%1, %2};" ::"r"(rw + 16 * (r & 3)), "l"((u64)r), "l"((u64)r) : "memory");
    b = clock64(); t[2] = (b - a) / reps;
    // 3: 4 volatile local u64 loads
    u64 acc = 0;
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      const volatile u64* v = words + (r & 7);
      acc += v[0] + v[8] + v[16] + v[24];
    }
    b = clock64(); t[3] = (b - a) / reps;
    // 4: fence.proxy.async.shared::cta
    a = clock64();
    for (int r = 0; r < reps; ++r) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    b = clock64(); t[4] = (b - a) / reps;
    // 5: mbarrier test_wait
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      u32 ok;
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n}"
                   : "=r"(ok) : "r"(sa(&bar)), "r"(1u) : "memory");
      acc += ok;
    }
    b = clock64(); t[5] = (b - a) / reps;
    // 6: bulk s2cl 4 KB issue (+commit), then wait_group.read per iteration
    const u32 rb = mapa(&buf[1][0], 1), rbar = mapa(&bar, 1);
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(rb), "r"(sa(&buf[0][0])), "r"(4096u), "r"(rbar) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    }
    b = clock64(); t[6] = (b - a) / reps;
    // 7: bulk s2cl issue only (wait at the end)
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(rb), "r"(sa(&buf[0][0])), "r"(4096u), "r"(rbar) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    b = clock64(); t[7] = (b - a) / reps;
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    // 8: st.release.cta + ld.acquire.cta local
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      u32 v;
      asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(sa(&flag)), "r"((u32)r) : "memory");
      asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(sa(&flag)) : "memory");
      acc += v;
    }
    b = clock64(); t[8] = (b - a) / reps;
    // 9: mapa
    a = clock64();
    for (int r = 0; r < reps; ++r) acc += mapa(&words[r & 7], 1);
    b = clock64(); t[9] = (b - a) / reps;
    // 10: st.release.gpu global
    a = clock64();
    for (int r = 0; r < reps; ++r)
      asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(out + 40), "r"((u32)r) : "memory");
    b = clock64(); t[10] = (b - a) / reps;
    // 11: fence.proxy.async (generic)
    a = clock64();
    for (int r = 0; r < reps; ++r) asm volatile("fence.proxy.async;" ::: "memory");
    b = clock64(); t[11] = (b - a) / reps;
    // 12: __threadfence
    a = clock64();
    for (int r = 0; r < reps; ++r) __threadfence();
    b = clock64(); t[12] = (b - a) / reps;
    // 13: 4 remote relaxed stores followed by a local smem store + fence.proxy.async.shared::cta
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 64 + 8 * (r & 7)), "l"((u64)r) : "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    b = clock64(); t[13] = (b - a) / reps;
    // 14: remote store then a local volatile load loop (store-queue interaction)
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 8 * (r & 7)), "l"((u64)r) : "memory");
      const volatile u64* v = words + (r & 7);
      acc += v[0];
    }
    b = clock64(); t[14] = (b - a) / reps;
    // 15: ld.relaxed.cluster local u64 x4
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      u64 x0;
      for (int q = 0; q < 4; ++q) {
        asm volatile("ld.relaxed.cluster.shared::cta.u64 %0, [%1];" : "=l"(x0) : "r"(sa(&words[8 * q + (r & 7)])) : "memory");
        acc += x0;
      }
    }
    b = clock64(); t[15] = (b - a) / reps;
    // 16: atomicCAS global round trip
    a = clock64();
    for (int r = 0; r < reps; ++r) acc += atomicCAS((u32*)(out + 41), 0u, 0u);
    b = clock64(); t[16] = (b - a) / reps;
    // 17: ld.acquire.gpu global
    a = clock64();
    for (int r = 0; r < reps; ++r) { u32 v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(out + 42) : "memory"); acc += v; }
    b = clock64(); t[17] = (b - a) / reps;
    for (int q = 0; q < 18; ++q) out[q] = t[q];
    out[30] = acc;
  }
  // 18: named barrier, all 512 threads (CTA 0)
  if (rank == 0) {
    __syncthreads();
    long long a = clock64();
    for (int r = 0; r < reps; ++r) asm volatile("bar.sync 1, 512;" ::: "memory");
    long long b = clock64();
    if (threadIdx.x == 0) out[18] = (b - a) / reps;
    // 19: named barrier after thread 0 did 4 remote stores
    const u32 rw = mapa(&words[0], 1);
    __syncthreads();
    a = clock64();
    for (int r = 0; r < reps; ++r) {
      if (threadIdx.x == 0) {
        asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw), "l"((u64)r) : "memory");
        asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 8), "l"((u64)r) : "memory");
        asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 16), "l"((u64)r) : "memory");
        asm volatile("st.relaxed.cluster.shared::cluster.u64 [%0], %1;" ::"r"(rw + 24), "l"((u64)r) : "memory");
      }
      asm volatile("bar.sync 1, 512;" ::: "memory");
    }
    b = clock64();
    if (threadIdx.x == 0) out[19] = (b - a) / reps;
  }
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

int main() {
  long long* d; cudaMalloc(&d, 64 * sizeof(long long)); cudaMemset(d, 0, 64 * sizeof(long long));
  kmicro<<<2, NT>>>(d, 1000);
  kmicro<<<2, NT>>>(d, 1000);
  long long h[64];
  cudaError_t e = cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
  const char* nm[] = {"4x st.relaxed.cluster u64 remote", "4x st weak u64 remote", "1x st.v2.u64 remote",
                      "4x volatile ld u64 local", "fence.proxy.async.shared::cta", "mbarrier test_wait",
                      "bulk s2cl 4KB + wait_group.read", "bulk s2cl 4KB issue", "st.release.cta+ld.acquire.cta",
                      "mapa", "st.release.gpu global", "fence.proxy.async (generic)", "__threadfence",
                      "2 remote st + fence.proxy.async.shared::cta", "remote st + local volatile ld",
                      "4x ld.relaxed.cluster local", "atomicCAS global", "ld.acquire.gpu global",
                      "bar.sync 512 (all)", "4 remote st + bar.sync 512"};
  for (int q = 0; q < 20; ++q) printf("%-48s %6lld cyc\n", nm[q], h[q]);
  return 0;
}
