// bgpq_prim.cuh — sm_100a device primitives for the BGPQ hot path.
//
//  * PTX wrappers: acquire/release node locks (atom.cas.acquire.gpu / st.release.gpu),
//    relaxed/acquire loads, mbarrier + cp.async.bulk (TMA bulk) global->shared staging,
//    proxy fences.
//  * warp_sort64: in-register bitonic sort of 64-entry runs with __shfl_xor_sync
//    ("Sort(items)", Alg.1 l.2 = P:203; bitonic sort [22]).
//  * cta_merge_split: merge-path [11] partitioned merge of two sorted smem tiles,
//    split at Ma — the SORT_SPLIT of P:196-198.
//  * cta_sort: warp_sort64 runs followed by merge-path passes in smem.
#pragma once
#include <cstdint>
#include <type_traits>

namespace bgpqd {

typedef uint32_t u32;
typedef uint64_t u64;
typedef unsigned long long ull;
typedef uint16_t u16;
typedef uint8_t u8;

constexpr u32 KEY_MAX = 0xFFFFFFFFu;

// ----------------------------------------------------------------------------------------
// PTX wrappers
// ----------------------------------------------------------------------------------------
__device__ __forceinline__ u32 smem_addr(const void* p) {
  return static_cast<u32>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ u32 ld_relaxed(const u32* p) {
  u32 v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u32 ld_acquire(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u64 ld_acquire_u64(const u64* p) {
  u64 v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(u32* p, u32 v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_u64(u64* p, u64 v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release_u64(u64* p, u64 v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release(u32* p, u32 v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ u32 cas_acquire(u32* p, u32 cmp, u32 val) {
  u32 old;
  asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], %2, %3;"
               : "=r"(old) : "l"(p), "r"(cmp), "r"(val) : "memory");
  return old;
}
// generic <-> async proxy ordering (global and shared) — required between an acquire of a
// node lock and the cp.async.bulk that reads the node, and before re-filling a smem tile
// that generic-proxy code has touched.
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async;" ::: "memory");
}

// Node lock (D4): test-and-test-and-set with an acquire CAS; one elected thread spins
// with __nanosleep backoff so the CAS traffic does not starve the holder's accesses.
__device__ __forceinline__ u32 lock_acquire(u32* lk) {
  if (cas_acquire(lk, 0u, 1u) == 0u) return 0;  // uncontended: one round trip
  u32 spins = 1, ns = 16;
  __nanosleep(ns);
  for (;;) {
    if (ld_relaxed(lk) == 0u && cas_acquire(lk, 0u, 1u) == 0u) return spins;
    ++spins;
    __nanosleep(ns);
    ns = ns < 128 ? ns * 2 : 128;
  }
}
// Release: the caller has made all of the CTA's writes to the protected data happen-before
// this thread with a CTA barrier (bar.sync is morally strong and orders them before this
// thread's later accesses); the gpu-scope release store is cumulative and publishes them.
__device__ __forceinline__ void lock_release(u32* lk) { st_release(lk, 0u); }

// The cached {state, min, max} of a node's 16-B metadata record, in one load (several of
// these issue back to back; a separate relaxed load per word would serialise on their uses).
__device__ __forceinline__ void meta_load(const void* rec, u32& st, u32& mn, u32& mx) {
  u32 lk;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(lk), "=r"(st), "=r"(mn), "=r"(mx) : "l"(rec) : "memory");
}

// mbarrier + TMA bulk copy (global -> shared), completion by transaction bytes.
__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(u64* bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* bar, u32 phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_addr(bar)),
      "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, u32 bytes, u64* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar)) : "memory");
}

// TMA bulk copy shared -> global (bulk_group completion; the issuing thread waits with
// cp.async.bulk.wait_group[.read])
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, u32 bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_addr(src)),
               "r"(bytes) : "memory");
}

// CTA barrier over the NT compute threads only (named barrier 1): the server CTA runs an
// extra helper warp that must not take part in the compute barriers.
template <int NT>
__device__ __forceinline__ void cta_bar() { asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory"); }

// ----------------------------------------------------------------------------------------
// Sort(items) — Alg.1 l.2, bitonic sort [22].
// warp_sort64: one warp sorts 64 entries held two per lane (index e = lane + 32*s).
// Comparison key = (key << 1) | is_pad so padding entries sort after real entries with
// the same key; compare-exchange partners at distance j < 32 are fetched with
// __shfl_xor_sync, the j = 32 partner is the lane's other register.
// ----------------------------------------------------------------------------------------
template <bool V>
__device__ __forceinline__ void warp_sort64(u64& c0, u64& c1, u32& v0, u32& v1) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int k = 2; k <= 64; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      if (j == 32) {
        // e0 = lane < 32 <= e1 = lane + 32, ascending iff ((e & k) == 0); k == 64 here
        const bool asc = true;
        const bool sw = asc ? (c1 < c0) : (c0 < c1);
        if (sw) {
          u64 t = c0; c0 = c1; c1 = t;
          if (V) { u32 tv = v0; v0 = v1; v1 = tv; }
        }
      } else {
        const u64 p0 = __shfl_xor_sync(0xffffffffu, c0, j);
        const u64 p1 = __shfl_xor_sync(0xffffffffu, c1, j);
        u32 q0 = 0, q1 = 0;
        if (V) {
          q0 = __shfl_xor_sync(0xffffffffu, v0, j);
          q1 = __shfl_xor_sync(0xffffffffu, v1, j);
        }
        const int e0 = lane, e1 = lane + 32;
        const bool lower = (lane & j) == 0;
        const bool min0 = (lower == ((e0 & k) == 0));
        const bool min1 = (lower == ((e1 & k) == 0));
        const bool t0 = min0 ? (p0 < c0) : (p0 > c0);
        const bool t1 = min1 ? (p1 < c1) : (p1 > c1);
        if (t0) { c0 = p0; if (V) v0 = q0; }
        if (t1) { c1 = p1; if (V) v1 = q1; }
      }
    }
  }
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT by merge path [11].
// Z[0:na] and W[0:nb] are sorted smem tiles; the merged sequence (stable, Z before W on
// equal keys) is written with its first `ma` entries to X and the rest to Y.
// Each of the NT threads takes a contiguous range of output diagonals, finds its co-rank
// by binary search on the diagonal and merges sequentially.  X/Y must not alias Z/W.
// The caller synchronizes before and after.
// ----------------------------------------------------------------------------------------
template <int NT, bool V>
__device__ __forceinline__ void cta_merge_split(const u32* __restrict__ zk, const u32* __restrict__ zv,
                                                int na, const u32* __restrict__ wk,
                                                const u32* __restrict__ wv, int nb, int ma,
                                                u32* __restrict__ xk, u32* __restrict__ xv,
                                                u32* __restrict__ yk, u32* __restrict__ yv) {
  const int N = na + nb;
  const int per = (N + NT - 1) / NT;
  const int d = threadIdx.x * per;
  if (d >= N) return;
  const int dend = min(d + per, N);
  int lo = max(0, d - nb), hi = min(d, na);
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (zk[mid] <= wk[d - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  int i = lo, j = d - lo;
  for (int o = d; o < dend; ++o) {
    const bool takez = (j >= nb) || (i < na && zk[i] <= wk[j]);
    u32 k, v = 0;
    if (takez) { k = zk[i]; if (V) v = zv[i]; ++i; }
    else { k = wk[j]; if (V) v = wv[j]; ++j; }
    if (o < ma) { xk[o] = k; if (V) xv[o] = v; }
    else { yk[o - ma] = k; if (V) yv[o - ma] = v; }
  }
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT by co-ranking every element (the final positions of a stable merge [11]):
//   z[i] goes to i + #{w < z[i]},  w[j] goes to j + #{z <= w[j]}   (Z first on equal keys)
// Each rank is a branchless fixed-trip binary search (no divergence); a thread handles up to
// ceil(KMAX/NT) entries of each input so the independent searches overlap (ILP).  Output
// position p < ma goes to X[p], else Y[p - ma].  X/Y must not alias Z/W.
// ----------------------------------------------------------------------------------------
__device__ __forceinline__ int lower_count(const u32* __restrict__ a, int n, u32 key, int top) {
  // number of a[0:n) strictly below key; top = highest power of two <= max n (compile-time-ish)
  int pos = 0;
#pragma unroll
  for (int step = top; step > 0; step >>= 1) {
    const int q = pos + step;
    if (q <= n && a[q - 1] < key) pos = q;
  }
  return pos;
}
__device__ __forceinline__ int upper_count(const u32* __restrict__ a, int n, u32 key, int top) {
  int pos = 0;  // number of a[0:n) <= key
#pragma unroll
  for (int step = top; step > 0; step >>= 1) {
    const int q = pos + step;
    if (q <= n && a[q - 1] <= key) pos = q;
  }
  return pos;
}
template <int KMAX, int NT, bool V>
__device__ __forceinline__ void cta_rank_merge(const u32* __restrict__ zk, const u32* __restrict__ zv,
                                               int na, const u32* __restrict__ wk,
                                               const u32* __restrict__ wv, int nb, int ma,
                                               u32* __restrict__ xk, u32* __restrict__ xv,
                                               u32* __restrict__ yk, u32* __restrict__ yv) {
  constexpr int E = (KMAX + NT - 1) / NT;
  u32 kz[E], kw[E];
  int pz[E], pw[E];
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int i = threadIdx.x + e * NT;
    kz[e] = i < na ? zk[i] : 0u;
    kw[e] = i < nb ? wk[i] : 0u;
  }
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int i = threadIdx.x + e * NT;
    pz[e] = i + lower_count(wk, nb, kz[e], KMAX);
    pw[e] = i + upper_count(zk, na, kw[e], KMAX);
  }
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int i = threadIdx.x + e * NT;
    if (i < na) {
      const int p = pz[e];
      const u32 v = V ? zv[i] : 0u;
      if (p < ma) { xk[p] = kz[e]; if (V) xv[p] = v; }
      else { yk[p - ma] = kz[e]; if (V) yv[p - ma] = v; }
    }
    if (i < nb) {
      const int p = pw[e];
      const u32 v = V ? wv[i] : 0u;
      if (p < ma) { xk[p] = kw[e]; if (V) xv[p] = v; }
      else { yk[p - ma] = kw[e]; if (V) yv[p - ma] = v; }
    }
  }
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT by merge path [11] with register windows (the hot-path merge).
// Thread t produces the VT = ceil(2*KMAX/NT) consecutive outputs [t*VT, t*VT+VT) of the
// stable merge (Z before W on equal keys): one fixed-trip branchless co-rank search on its
// start diagonal, a serial merge of VT entries in registers, then vector stores (128-bit
// when VT = 4).  Values are gathered after the key merge from the recorded source index.
// Output position p < ma goes to X[p], else Y[p - ma].  X/Y must not alias Z/W.
// ----------------------------------------------------------------------------------------
template <int N>
struct Log2Ceil { static constexpr int v = (N <= 1) ? 0 : 1 + Log2Ceil<(N + 1) / 2>::v; };
template <>
struct Log2Ceil<1> { static constexpr int v = 0; };

template <int KMAX, int NT, bool V>
__device__ __forceinline__ void cta_path_merge(const u32* __restrict__ zk, const u32* __restrict__ zv,
                                               int na, const u32* __restrict__ wk,
                                               const u32* __restrict__ wv, int nb, int ma,
                                               u32* __restrict__ xk, u32* __restrict__ xv,
                                               u32* __restrict__ yk, u32* __restrict__ yv) {
  constexpr int VT = (2 * KMAX + NT - 1) / NT;
  constexpr int LOG = Log2Ceil<KMAX + 1>::v;
  const int N = na + nb;
  const int d = threadIdx.x * VT;
  if (d >= N) return;
  int lo = max(0, d - nb), hi = min(d, na);
#pragma unroll
  for (int it = 0; it < LOG; ++it) {
    const int len = hi - lo;
    const int mid = lo + (len >> 1);
    const bool act = len > 0;
    const u32 a = zk[act ? mid : 0];
    const u32 b = wk[act ? d - 1 - mid : 0];
    const bool right = act && (a <= b);
    lo = right ? mid + 1 : lo;
    hi = (act && !right) ? mid : hi;
  }
  int i = lo, j = d - lo;
  u32 a = (i < na) ? zk[i] : 0u;
  u32 b = (j < nb) ? wk[j] : 0u;
  u32 ko[VT];
  int src[VT];
#pragma unroll
  for (int k = 0; k < VT; ++k) {
    const bool takez = (j >= nb) || (i < na && a <= b);
    ko[k] = takez ? a : b;
    src[k] = takez ? i : (KMAX + j);
    if (takez) { ++i; a = (i < na) ? zk[i] : 0u; }
    else { ++j; b = (j < nb) ? wk[j] : 0u; }
  }
  u32 vo[VT];
  if (V) {
#pragma unroll
    for (int k = 0; k < VT; ++k) vo[k] = src[k] < KMAX ? zv[src[k]] : wv[src[k] - KMAX];
  }
  if (VT == 4 && d + 4 <= N && ((d + 4 <= ma) || (d >= ma && ((ma & 3) == 0)))) {
    u32* dk = (d + 4 <= ma) ? xk + d : yk + (d - ma);
    *reinterpret_cast<uint4*>(dk) = make_uint4(ko[0], ko[1 % VT], ko[2 % VT], ko[3 % VT]);
    if (V) {
      u32* dv = (d + 4 <= ma) ? xv + d : yv + (d - ma);
      *reinterpret_cast<uint4*>(dv) = make_uint4(vo[0], vo[1 % VT], vo[2 % VT], vo[3 % VT]);
    }
  } else {
#pragma unroll
    for (int k = 0; k < VT; ++k) {
      const int o = d + k;
      if (o < N) {
        if (o < ma) { xk[o] = ko[k]; if (V) xv[o] = vo[k]; }
        else { yk[o - ma] = ko[k]; if (V) yv[o - ma] = vo[k]; }
      }
    }
  }
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT by merge path [11] with a register window (the hot-path merge, v3).
// Threads 0..NTM-1 each produce VT = 2*KMAX/NTM consecutive outputs [d, d+VT) of the merge.
// After the branchless co-rank search on diagonal d (i from Z, j = d - i from W), the VT
// outputs are exactly the VT smallest of Z[i, i+VT) u W[j, j+VT): both windows are loaded
// with independent LDS, C[k] = min(A[k], B[VT-1-k]) selects them as a bitonic sequence
// (Batcher's half-cleaner) and log2(VT) compare-exchange stages sort it — no dependent
// shared-memory chain after the search.  With values the comparison key is the stable
// composite (key, Z before W, index), so equal keys never migrate between threads and the
// (key, value) pairs stay a permutation; keys-only compares 32-bit keys.
// Output position p < ma goes to X[p], else Y[p - ma].  X/Y must not alias Z/W.
// ----------------------------------------------------------------------------------------
template <int VT, typename T>
__device__ __forceinline__ void bitonic_sort_regs(T (&c)[VT]) {
#pragma unroll
  for (int s = VT / 2; s > 0; s >>= 1) {
#pragma unroll
    for (int k = 0; k < VT; ++k) {
      if ((k & s) == 0) {
        const T a = c[k], b = c[k + s];
        c[k] = a < b ? a : b;
        c[k + s] = a < b ? b : a;
      }
    }
  }
}

// grp_merge_win: the same merge executed by a group of NTM threads, t = index in the group
template <int KMAX, int NTM, bool V>
__device__ __forceinline__ void grp_merge_win(const int t, const u32* __restrict__ zk, const u32* __restrict__ zv,
                                              int na, const u32* __restrict__ wk,
                                              const u32* __restrict__ wv, int nb, int ma,
                                              u32* __restrict__ xk, u32* __restrict__ xv,
                                              u32* __restrict__ yk, u32* __restrict__ yv) {
  constexpr int VT = (2 * KMAX) / NTM;
  static_assert(VT >= 2 && (VT & (VT - 1)) == 0 && VT * NTM == 2 * KMAX, "VT must be a power of two");
  constexpr int LOG = Log2Ceil<KMAX + 1>::v;
  if (t >= NTM) return;
  const int N = na + nb;
  const int d = t * VT;
  if (d >= N) return;
  int lo = max(0, d - nb), hi = min(d, na);
#pragma unroll
  for (int it = 0; it < LOG; ++it) {
    const int len = hi - lo;
    const int mid = lo + (len >> 1);
    const bool act = len > 0;
    const u32 a = zk[act ? mid : 0];
    const u32 b = wk[act ? d - 1 - mid : 0];
    const bool right = act && (a <= b);
    lo = right ? mid + 1 : lo;
    hi = (act && !right) ? mid : hi;
  }
  const int i = lo, j = d - lo;
  if (!V) {
    u32 A[VT], C[VT];
#pragma unroll
    for (int k = 0; k < VT; ++k) A[k] = (i + k < na) ? zk[i + k] : KEY_MAX;
#pragma unroll
    for (int k = 0; k < VT; ++k) {
      const int jj = j + VT - 1 - k;
      const u32 b = (jj < nb) ? wk[jj] : KEY_MAX;
      C[k] = A[k] < b ? A[k] : b;
    }
    bitonic_sort_regs<VT>(C);
    if (VT >= 4 && d + VT <= N && (d + VT <= ma || (d >= ma && ((ma & 3) == 0)))) {
      u32* dk = (d + VT <= ma) ? xk + d : yk + (d - ma);
#pragma unroll
      for (int k = 0; k < VT; k += 4)
        *reinterpret_cast<uint4*>(dk + k) = make_uint4(C[k], C[(k + 1) % VT], C[(k + 2) % VT], C[(k + 3) % VT]);
    } else {
#pragma unroll
      for (int k = 0; k < VT; ++k) {
        const int o = d + k;
        if (o < N) {
          if (o < ma) xk[o] = C[k];
          else yk[o - ma] = C[k];
        }
      }
    }
  } else {
    u64 A[VT], C[VT];
#pragma unroll
    for (int k = 0; k < VT; ++k)
      A[k] = (i + k < na) ? (((u64)zk[i + k] << 32) | (u32)(i + k)) : ~0ull;
#pragma unroll
    for (int k = 0; k < VT; ++k) {
      const int jj = j + VT - 1 - k;
      const u64 b = (jj < nb) ? (((u64)wk[jj] << 32) | 0x80000000u | (u32)jj) : ~0ull;
      C[k] = A[k] < b ? A[k] : b;
    }
    bitonic_sort_regs<VT>(C);
    u32 ko[VT], vo[VT];
#pragma unroll
    for (int k = 0; k < VT; ++k) {
      const u32 lw = (u32)C[k];
      const u32 idx = lw & 0x7FFFFFFFu;
      ko[k] = (u32)(C[k] >> 32);
      vo[k] = (d + k < N) ? ((lw & 0x80000000u) ? wv[idx] : zv[idx]) : 0u;
    }
    if (VT >= 4 && d + VT <= N && (d + VT <= ma || (d >= ma && ((ma & 3) == 0)))) {
      u32* dk = (d + VT <= ma) ? xk + d : yk + (d - ma);
      u32* dv = (d + VT <= ma) ? xv + d : yv + (d - ma);
#pragma unroll
      for (int k = 0; k < VT; k += 4) {
        *reinterpret_cast<uint4*>(dk + k) = make_uint4(ko[k], ko[(k + 1) % VT], ko[(k + 2) % VT], ko[(k + 3) % VT]);
        *reinterpret_cast<uint4*>(dv + k) = make_uint4(vo[k], vo[(k + 1) % VT], vo[(k + 2) % VT], vo[(k + 3) % VT]);
      }
    } else {
#pragma unroll
      for (int k = 0; k < VT; ++k) {
        const int o = d + k;
        if (o < N) {
          if (o < ma) { xk[o] = ko[k]; xv[o] = vo[k]; }
          else { yk[o - ma] = ko[k]; yv[o - ma] = vo[k]; }
        }
      }
    }
  }
}

template <int KMAX, int NTM, bool V>
__device__ __forceinline__ void cta_merge_win(const u32* __restrict__ zk, const u32* __restrict__ zv,
                                              int na, const u32* __restrict__ wk,
                                              const u32* __restrict__ wv, int nb, int ma,
                                              u32* __restrict__ xk, u32* __restrict__ xv,
                                              u32* __restrict__ yk, u32* __restrict__ yv) {
  grp_merge_win<KMAX, NTM, V>((int)threadIdx.x, zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT by warp-cooperative merge path (v4, the hot-path merge).
// Warp w of the first NW warps produces the OW = 2*KMAX/NW consecutive outputs [D0, D0+OW)
// of the stable merge, E = OW/32 per lane, element e = lane + 32*k in register k:
//  1. co-rank of D0 by a two-round 32-ary search with __ballot_sync (probe stride odd so
//     the 32 probes fall in distinct banks) instead of log2(K) dependent probes per thread;
//  2. the OW outputs are the OW smallest of Z[i0, i0+OW) u W[j0, j0+OW): lane l loads
//     A[k] = Z[i0+e] and, in reversed order, B[k] = W[j0+OW-1-e]; C = min(A, B) is bitonic
//     (Batcher's half-cleaner) and holds exactly them;
//  3. C is sorted by a bitonic network: strides >= 32 inside the lane's registers, strides
//     < 32 with __shfl_xor_sync; then coalesced, conflict-free stores (lane-strided).
// With values the comparison key is the stable composite (key, Z before W, index) and the
// value is gathered from its source index; keys-only compares the 32-bit keys.
// Output position p < ma goes to X[p], else Y[p - ma].  X/Y must not alias Z/W.
// ----------------------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ T shfl_xor_t(T v, int m) {
  if constexpr (sizeof(T) == 8) {
    const u32 lo = __shfl_xor_sync(0xffffffffu, (u32)v, m);
    const u32 hi = __shfl_xor_sync(0xffffffffu, (u32)(v >> 32), m);
    return ((u64)hi << 32) | lo;
  } else {
    return __shfl_xor_sync(0xffffffffu, v, m);
  }
}

// co-rank of diagonal D (number of Z entries among the first D outputs; Z first on ties)
__device__ __forceinline__ int warp_corank(const u32* __restrict__ zk, int na, const u32* __restrict__ wk,
                                           int nb, int D) {
  const int lane = threadIdx.x & 31;
  int lo = max(0, D - nb), hi = min(D, na);
  while (hi - lo > 0) {  // at most two rounds for ranges <= 1056
    const int n = hi - lo;
    int s = (n + 31) >> 5;
    if (s > 1 && !(s & 1)) ++s;  // odd stride: distinct banks
    const int m = lo + s * (lane + 1) - 1;
    const bool valid = m < hi;
    bool q = false;
    if (valid) q = zk[m] <= wk[D - 1 - m];
    const u32 bal = __ballot_sync(0xffffffffu, valid && q);
    const int L = __popc(bal);  // Q is monotone: the first L probes are true
    lo = lo + s * L;
    hi = min(hi, lo + s - 1);
    if (s == 1) hi = lo;
  }
  return lo;
}

template <int KMAX, int NW, bool V>
__device__ __forceinline__ void grp_merge_warp(const int warp, const u32* __restrict__ zk, const u32* __restrict__ zv,
                                               int na, const u32* __restrict__ wk,
                                               const u32* __restrict__ wv, int nb, int ma,
                                               u32* __restrict__ xk, u32* __restrict__ xv,
                                               u32* __restrict__ yk, u32* __restrict__ yv) {
  constexpr int OW = (2 * KMAX) / NW;
  constexpr int E = OW / 32;
  static_assert(E >= 1 && (E & (E - 1)) == 0 && OW * NW == 2 * KMAX, "E must be a power of two");
  using T = typename std::conditional<V, u64, u32>::type;
  const int lane = threadIdx.x & 31;
  if (warp >= NW) return;
  const int N = na + nb;
  const int D0 = warp * OW;
  if (D0 >= N) return;
  const int i0 = warp_corank(zk, na, wk, nb, D0);
  const int j0 = D0 - i0;
  T C[E];
#pragma unroll
  for (int k = 0; k < E; ++k) {
    const int ia = i0 + lane + 32 * k;
    const int jb = j0 + OW - 1 - (lane + 32 * k);
    T a, b;
    if constexpr (V) {
      a = ia < na ? (((u64)zk[ia] << 32) | (u32)ia) : ~0ull;
      b = jb < nb ? (((u64)wk[jb] << 32) | 0x80000000u | (u32)jb) : ~0ull;
    } else {
      a = ia < na ? zk[ia] : KEY_MAX;
      b = jb < nb ? wk[jb] : KEY_MAX;
    }
    C[k] = a < b ? a : b;
  }
  // bitonic sort (ascending) of the OW-entry bitonic sequence
#pragma unroll
  for (int s = OW / 2; s >= 32; s >>= 1) {
    const int r = s / 32;
#pragma unroll
    for (int k = 0; k < E; ++k) {
      if ((k & r) == 0) {
        const T a = C[k], b = C[k + r];
        C[k] = a < b ? a : b;
        C[k + r] = a < b ? b : a;
      }
    }
  }
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    const bool upper = (lane & s) != 0;
#pragma unroll
    for (int k = 0; k < E; ++k) {
      const T p = shfl_xor_t(C[k], s);
      C[k] = upper ? (C[k] > p ? C[k] : p) : (C[k] < p ? C[k] : p);
    }
  }
#pragma unroll
  for (int k = 0; k < E; ++k) {
    const int o = D0 + lane + 32 * k;
    if (o < N) {
      u32 key, val = 0;
      if constexpr (V) {
        key = (u32)(C[k] >> 32);
        const u32 lw = (u32)C[k];
        const u32 idx = lw & 0x7FFFFFFFu;
        val = (lw & 0x80000000u) ? wv[idx] : zv[idx];
      } else {
        key = C[k];
      }
      if (o < ma) { xk[o] = key; if (V) xv[o] = val; }
      else { yk[o - ma] = key; if (V) yv[o - ma] = val; }
    }
  }
}

template <int KMAX, int NW, bool V>
__device__ __forceinline__ void cta_merge_warp(const u32* __restrict__ zk, const u32* __restrict__ zv,
                                               int na, const u32* __restrict__ wk,
                                               const u32* __restrict__ wv, int nb, int ma,
                                               u32* __restrict__ xk, u32* __restrict__ xv,
                                               u32* __restrict__ yk, u32* __restrict__ yv) {
  grp_merge_warp<KMAX, NW, V>((int)(threadIdx.x >> 5), zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
}

// ----------------------------------------------------------------------------------------
// SORT_SPLIT of two full sorted K-batches (Na = Nb = Ma = K, the common case of P:196) without
// co-rank searches (v5): X = K smallest, Y = K largest.  min / max of Z[p] and W[K-1-p]
// (Batcher's half-cleaner on Z ++ reverse(W)) put exactly the K smallest into L and the rest
// into U, each a bitonic sequence; each half is then sorted by a bitonic merge — strides below
// E = 2K/NT inside a thread's registers, strides up to 31 threads with __shfl_xor_sync, larger
// ones through the output tile in shared memory.  Threads 0..NT/2-1 build X, the rest Y; thread
// u of a half owns positions [u*E, u*E+E).  With values the comparison key is the stable
// composite (key, Z before W, index), so the result equals the stable merge's order; keys only
// compares the 32-bit keys.  bar_id / NT: the named barrier of the NT participating threads.
// ----------------------------------------------------------------------------------------
template <int K, int NT, bool V>
__device__ __forceinline__ void bitonic_split_full(const int t, const int bar_id, const u32* __restrict__ zk,
                                                   const u32* __restrict__ zv, const u32* __restrict__ wk,
                                                   const u32* __restrict__ wv, u32* __restrict__ xk,
                                                   u32* __restrict__ xv, u32* __restrict__ yk, u32* __restrict__ yv) {
  constexpr int HT = NT / 2;   // threads per half
  constexpr int E = K / HT;    // elements per thread
  static_assert(E >= 1 && (E & (E - 1)) == 0 && E * HT == K, "K must be a multiple of NT/2 (power of two)");
  using T = typename std::conditional<V, u64, u32>::type;
  const int half = t / HT, u = t % HT;
  u32* ok = half ? yk : xk;
  u32* ov = half ? yv : xv;
  T c[E];
  // 1. half-cleaner, strided layout: c[e] holds position p = e*HT + u of the half
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int p = e * HT + u, q = K - 1 - p;
    T a, b;
    if constexpr (V) {
      a = ((u64)zk[p] << 32) | (u32)p;
      b = ((u64)wk[q] << 32) | 0x80000000u | (u32)q;
    } else {
      a = zk[p];
      b = wk[q];
    }
    c[e] = half ? (a < b ? b : a) : (a < b ? a : b);
  }
  // 2. bitonic merge strides j >= HT: register index bits (strided layout)
#pragma unroll
  for (int jr = E / 2; jr >= 1; jr >>= 1) {
#pragma unroll
    for (int e = 0; e < E; ++e) {
      if ((e & jr) == 0) {
        const T a = c[e], b = c[e + jr];
        c[e] = a < b ? a : b;
        c[e + jr] = a < b ? b : a;
      }
    }
  }
  // 3. transpose through the output tile to the blocked layout: c[e] = position u*E + e
#pragma unroll
  for (int e = 0; e < E; ++e) {
    ok[e * HT + u] = V ? (u32)(c[e] >> 32) : (u32)c[e];
    if constexpr (V) ov[e * HT + u] = (u32)c[e];
  }
  asm volatile("bar.sync %0, %1;" ::"r"(bar_id), "n"(NT) : "memory");
#pragma unroll
  for (int e = 0; e < E; ++e) {
    if constexpr (V) c[e] = ((u64)ok[u * E + e] << 32) | ov[u * E + e];
    else c[e] = ok[u * E + e];
  }
  asm volatile("bar.sync %0, %1;" ::"r"(bar_id), "n"(NT) : "memory");
  // 4. strides HT/2 .. E: across threads (distance j/E), then < E inside the thread
#pragma unroll
  for (int j = HT / 2; j >= 1; j >>= 1) {
    if (j >= E) {
      const int d = j / E;
      const bool upper = (u & d) != 0;
      if (d < 32) {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          T pv;
          if constexpr (V) {
            const u32 lo = __shfl_xor_sync(0xffffffffu, (u32)c[e], d);
            const u32 hi = __shfl_xor_sync(0xffffffffu, (u32)(c[e] >> 32), d);
            pv = ((u64)hi << 32) | lo;
          } else {
            pv = __shfl_xor_sync(0xffffffffu, c[e], d);
          }
          c[e] = upper ? (c[e] > pv ? c[e] : pv) : (c[e] < pv ? c[e] : pv);
        }
      } else {  // across warps: exchange through the tile
        const int p0 = u * E, pp0 = (u ^ d) * E;
#pragma unroll
        for (int e = 0; e < E; ++e) {
          ok[p0 + e] = V ? (u32)(c[e] >> 32) : (u32)c[e];
          if constexpr (V) ov[p0 + e] = (u32)c[e];
        }
        asm volatile("bar.sync %0, %1;" ::"r"(bar_id), "n"(NT) : "memory");
        T pv[E];
#pragma unroll
        for (int e = 0; e < E; ++e) {
          if constexpr (V) pv[e] = ((u64)ok[pp0 + e] << 32) | ov[pp0 + e];
          else pv[e] = ok[pp0 + e];
        }
        asm volatile("bar.sync %0, %1;" ::"r"(bar_id), "n"(NT) : "memory");
#pragma unroll
        for (int e = 0; e < E; ++e) c[e] = upper ? (c[e] > pv[e] ? c[e] : pv[e]) : (c[e] < pv[e] ? c[e] : pv[e]);
      }
    }
  }
#pragma unroll
  for (int jr = E / 2; jr >= 1; jr >>= 1) {
#pragma unroll
    for (int e = 0; e < E; ++e) {
      if ((e & jr) == 0) {
        const T a = c[e], b = c[e + jr];
        c[e] = a < b ? a : b;
        c[e + jr] = a < b ? b : a;
      }
    }
  }
  // 5. write back, blocked (values gathered from the source index)
  const int p0 = u * E;
  if constexpr (V) {
    u32 kk[E], vv[E];
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const u32 lw = (u32)c[e];
      const u32 idx = lw & 0x7FFFFFFFu;
      kk[e] = (u32)(c[e] >> 32);
      vv[e] = (lw & 0x80000000u) ? wv[idx] : zv[idx];
    }
#pragma unroll
    for (int e = 0; e < E; ++e) { ok[p0 + e] = kk[e]; ov[p0 + e] = vv[e]; }
  } else {
    if constexpr (E % 4 == 0) {
#pragma unroll
      for (int e = 0; e < E; e += 4)
        *reinterpret_cast<uint4*>(ok + p0 + e) = make_uint4(c[e], c[e + 1], c[e + 2], c[e + 3]);
    } else {
#pragma unroll
      for (int e = 0; e < E; ++e) ok[p0 + e] = c[e];
    }
  }
}

// The SORT_SPLIT used on the hot path: register-window merge path with VT = 4 outputs per
// thread (threads 0 .. 2K/4-1 of the NT compute threads take part).  Measured on B200
// (tools/micro_merge.cu, K = 1024, NT = 512): 1540 cycles keys-only / 2110 key+value, vs
// 2110 / 2190 for the co-ranking merge.
// Keys-only splits of two full K-batches use the search-free bitonic split (920 vs 1540 cycles
// at K = 1024, micro_merge.txt) on the first min(512, K) threads with named barrier 5; the
// caller's CTA barrier after the split joins the rest.  Only at K >= 512: below it the
// bitonic network's per-stage named barriers cost more than the merge path saves (C3 sweep,
// profiles/r1/final2_sweep_c3.jsonl vs c3_gate.jsonl: K = 128 / 256 inserts 10-12 % faster without it).
constexpr int BAR_BITONIC = 5;
constexpr int BITONIC_MIN_K = 512;
template <int K, int NT, bool V>
__device__ __forceinline__ void sort_split(const u32* zk, const u32* zv, int na, const u32* wk, const u32* wv,
                                           int nb, int ma, u32* xk, u32* xv, u32* yk, u32* yv) {
#ifndef BGPQ_NO_BITONIC
  if constexpr (!V) {
    constexpr int NB = (K < 512 ? K : 512) <= NT ? (K < 512 ? K : 512) : 0;
    if constexpr (NB >= 64 && K >= BITONIC_MIN_K) {
      if (na == K && nb == K && ma == K) {
        if ((int)threadIdx.x < NB)
          bitonic_split_full<K, NB, false>((int)threadIdx.x, BAR_BITONIC, zk, zv, wk, wv, xk, xv, yk, yv);
        return;
      }
    }
  }
#endif
  constexpr int NTM = (2 * K / 4 <= NT) ? 2 * K / 4 : NT;
  cta_merge_win<K, NTM, V>(zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
}

// sort_split run by a group of NT threads whose index in the group is t (the group need not
// start at thread 0; the bitonic path synchronises on named barrier BAR_BITONIC of NB threads)
template <int K, int NT, bool V>
__device__ __forceinline__ void sort_split_t(const int t, const u32* zk, const u32* zv, int na, const u32* wk,
                                             const u32* wv, int nb, int ma, u32* xk, u32* xv, u32* yk, u32* yv) {
#ifndef BGPQ_NO_BITONIC
  if constexpr (!V) {
    constexpr int NB = (K < 512 ? K : 512) <= NT ? (K < 512 ? K : 512) : 0;
    if constexpr (NB >= 64 && K >= BITONIC_MIN_K) {
      if (na == K && nb == K && ma == K) {
        if (t < NB) bitonic_split_full<K, NB, false>(t, BAR_BITONIC, zk, zv, wk, wv, xk, xv, yk, yv);
        return;
      }
    }
  }
#endif
  constexpr int NTM = (2 * K / 4 <= NT) ? 2 * K / 4 : NT;
  grp_merge_win<K, NTM, V>(t, zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
}

// One pass of a bottom-up merge sort: merge sorted runs [2q*run, (2q+1)*run) and
// [(2q+1)*run, (2q+2)*run) of src (n entries, n a multiple of 2*run) into dst, by co-ranking.
template <int KMAX, int NT, bool V>
__device__ __forceinline__ void cta_rank_merge_pass(const u32* __restrict__ sk, const u32* __restrict__ sv,
                                                    u32* __restrict__ dk, u32* __restrict__ dv, int n,
                                                    int run) {
  constexpr int E = (KMAX + NT - 1) / NT;
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const int i = threadIdx.x + e * NT;
    if (i < n) {
      const u32 key = sk[i];
      const int q = i / run;             // my run
      const int base = (q & ~1) * run;   // start of the pair
      const int off = i - q * run;       // index within my run
      int p;
      if ((q & 1) == 0) p = base + off + lower_count(sk + base + run, run, key, KMAX / 2);
      else p = base + off + upper_count(sk + base, run, key, KMAX / 2);
      dk[p] = key;
      if (V) dv[p] = sv[i];
    }
  }
}

// Merge consecutive sorted runs of length `run` pairwise (src -> dst), n entries total,
// n a multiple of 2*run.  Stable (earlier run first on ties).
template <int NT, bool V>
__device__ __forceinline__ void cta_merge_pass(const u32* __restrict__ sk, const u32* __restrict__ sv,
                                               u32* __restrict__ dk, u32* __restrict__ dv, int n,
                                               int run) {
  const int per = (n + NT - 1) / NT;  // divides 2*run for the sizes used (powers of two)
  const int d0 = threadIdx.x * per;
  if (d0 >= n) return;
  const int pair = d0 / (2 * run);
  const int base = pair * 2 * run;
  const u32* zk = sk + base;
  const u32* wk = zk + run;
  const u32* zv = V ? sv + base : nullptr;
  const u32* wv = V ? zv + run : nullptr;
  const int d = d0 - base;
  int lo = max(0, d - run), hi = min(d, run);
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (zk[mid] <= wk[d - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  int i = lo, j = d - lo;
  const int dend = min(d + per, 2 * run);
  for (int o = d; o < dend; ++o) {
    const bool takez = (j >= run) || (i < run && zk[i] <= wk[j]);
    if (takez) { dk[base + o] = zk[i]; if (V) dv[base + o] = zv[i]; ++i; }
    else { dk[base + o] = wk[j]; if (V) dv[base + o] = wv[j]; ++j; }
  }
}

// Sort the first `s` entries of (k, v) (smem, capacity K >= 64, power of two).  Entries
// [s, P) with P = max(64, next_pow2(s)) are treated as padding (sort after real entries).
// Uses (t_k, t_v) as scratch; returns true if the sorted result ended up in the scratch.
template <int K, int NT, bool V>
__device__ __forceinline__ bool cta_sort(u32* k, u32* v, int s, u32* tk, u32* tv) {
  int P = 64;
  while (P < s) P <<= 1;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int r = warp; r * 64 < P; r += NT / 32) {
    const int e0 = r * 64 + lane, e1 = e0 + 32;
    u64 c0 = ((u64)k[e0] << 1) | (u64)(e0 >= s);
    u64 c1 = ((u64)k[e1] << 1) | (u64)(e1 >= s);
    u32 v0 = 0, v1 = 0;
    if (V) { v0 = v[e0]; v1 = v[e1]; }
    warp_sort64<V>(c0, c1, v0, v1);
    k[e0] = (u32)(c0 >> 1);
    k[e1] = (u32)(c1 >> 1);
    if (V) { v[e0] = v0; v[e1] = v1; }
  }
  cta_bar<NT>();
  bool in_scratch = false;
  for (int run = 64; run < P; run <<= 1) {
    if (!in_scratch) cta_rank_merge_pass<K, NT, V>(k, v, tk, tv, P, run);
    else cta_rank_merge_pass<K, NT, V>(tk, tv, k, v, P, run);
    in_scratch = !in_scratch;
    cta_bar<NT>();
  }
  return in_scratch;
}

}  // namespace bgpqd
