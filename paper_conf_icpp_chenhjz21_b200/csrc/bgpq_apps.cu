// bgpq_apps.cu — the paper's two applications on BGPQ (§6.5), as
// persistent kernels whose CTAs each loop: DELETEMIN a full batch (the device API of
// include/bgpq_dev.cuh, "a thread block always retrieves a full node"), expand the popped
// search nodes in parallel (one thread per node), prune against the global incumbent, INSERT
// the surviving children in batches of <= K.  C ABI in include/bgpq_apps.h.
//
// Termination (reading R19 / DESIGN.md R25): `pending` counts search nodes that are in the
// heap or being expanded.  A CTA adds its children's count before inserting them and removes
// its popped count after; a CTA whose DELETEMIN comes back empty stops when pending == 0 (no
// node anywhere: the search is complete) or when its round budget is spent (multi-GPU rounds,
// the heap keeps the rest).
//
// Knapsack (reading R23): items in profit/weight-descending order with prefix sums
// Wp, Pp; a node (level l, weight W, profit P) has the Dantzig bound ub = P + g(l, W) with
// g(l, W) = greedy fill of items l.. into C - W plus the floored fraction of the first item
// that does not fit.  Queue entry: key = 0xFFFFFFFF - ub (min-heap = best bound first), value
// = (l << 22) | W; P is recovered as ub - g(l, W).  Incumbent = best node profit seen; a node
// is pruned when ub <= incumbent.
//
// A* (reading R24): grid cells row-major, 8 moves, orthogonal cost 1 / diagonal 2,
// h = Manhattan distance to the target, key = (f << 15) | min(h >> 1, 0x7FFF) (f = g + h, ties
// to the smaller h), value = cell index.  g[] holds the best known cost per cell (atomicMin);
// a popped entry whose g exceeds g[cell] is stale; incumbent = best cost to the target found;
// entries with f >= incumbent are pruned.
#include <cuda_runtime.h>

#include <cstring>

#include "../../include/bgpq.h"
#include "../../include/bgpq_apps.h"
#include "../../include/bgpq_dev.cuh"

using namespace bgpqd;

namespace {

constexpr int ANT = 512;  // compute threads per CTA (as the library's executions)

enum : int { ST_INC = 0, ST_PENDING = 1, ST_EXPANDED = 2, ST_INSERTED = 3, ST_POPS = 4, ST_ERR = 5,
             ST_PRUNED = 6, ST_EMPTY_POPS = 7 };

__device__ __forceinline__ ull ld_acq64(const ull* p) {
  ull v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Block-wide exclusive scan of per-thread counts (compute threads only, ANT threads).
__device__ __forceinline__ u32 block_excl_scan(u32 x, u32* warp_tot, u32* total, int tid) {
  const int lane = tid & 31, w = tid >> 5;
  u32 incl = x;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const u32 y = __shfl_up_sync(0xffffffffu, incl, d);
    if (lane >= d) incl += y;
  }
  if (lane == 31) warp_tot[w] = incl;
  cta_bar<ANT>();
  if (w == 0) {
    u32 t = lane < ANT / 32 ? warp_tot[lane] : 0u;
    u32 ti = t;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const u32 y = __shfl_up_sync(0xffffffffu, ti, d);
      if (lane >= d) ti += y;
    }
    if (lane < ANT / 32) warp_tot[lane] = ti - t;
    if (lane == ANT / 32 - 1) *total = ti;
  }
  cta_bar<ANT>();
  return warp_tot[w] + incl - x;
}

// =========================================================================================
// Knapsack
// =========================================================================================
struct KsArgs {
  u32 n;
  u64 C;
  const u32* w;
  const u32* p;
  const u64* Wp;
  const u64* Pp;
};

__device__ __forceinline__ u64 ks_g(const KsArgs& A, u32 l, u64 W) {
  // largest j in [l, n] with Wp[j] - Wp[l] <= C - W (Wp increasing)
  const u64 room = A.C - W;
  const u64 base = A.Wp[l];
  u32 lo = l, hi = A.n;
  while (lo < hi) {
    const u32 mid = (lo + hi + 1) >> 1;
    if (A.Wp[mid] - base <= room) lo = mid;
    else hi = mid - 1;
  }
  const u32 j = lo;
  u64 g = A.Pp[j] - A.Pp[l];
  if (j < A.n) g += (room - (A.Wp[j] - base)) * (u64)A.p[j] / (u64)A.w[j];
  return g;
}

constexpr u32 KS_WBITS = 22;

template <int K>
struct KsSmem {
  u32 popk[K], popv[K];
  u32 chk[2 * K], chv[2 * K];
  u32 warp_tot[32];
  u32 total;
  u32 done;
};

template <int K>
__global__ void __launch_bounds__(ANT + 32, 1)
    bgpq_ks_kernel(bgpq_dev::HeapView hv, KsArgs A, ull* state, u32 budget) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  using Q = bgpq_dev::Queue<K, true, ANT>;
  Q q;
  q.init(hv, smem_raw);
  if (q.is_lock_warp()) {
    q.run_lock_warp();
    return;
  }
  KsSmem<K>& S = *reinterpret_cast<KsSmem<K>*>(smem_raw + Q::smem_bytes());
  const int tid = threadIdx.x;
  ull expanded = 0, inserted = 0, pops = 0, pruned = 0, empty = 0;
  u32 backoff = 128;
  for (u32 it = 0; it < budget; ++it) {
    const u32 c = q.size_hint() ? q.deletemin(S.popk, S.popv, K) : 0u;
    if (c == 0) {  // nothing in the heap: done if nothing is in flight either (uniform decision)
      ++empty;
      if (tid == 0) S.done = ld_acq64(state + ST_PENDING) == 0;
      cta_bar<ANT>();
      const bool done = S.done;
      cta_bar<ANT>();
      if (done) break;
      __nanosleep(backoff);
      backoff = backoff < 8192 ? backoff * 2 : 8192;
      continue;
    }
    backoff = 128;
    ++pops;
    const ull inc = ld_acq64(state + ST_INC);
    // expand: thread t handles popped node t (K <= ANT * 2: two rounds at K = 1024)
    u32 nch_total = 0;
    for (int base = 0; base < (int)c; base += ANT) {
      const int t = base + tid;
      u32 ck[2], cv[2], nc = 0;
      if (t < (int)c) {
        const u64 ub = (u64)(0xFFFFFFFFu - S.popk[t]);
        const u32 v = S.popv[t];
        const u32 l = v >> KS_WBITS;
        const u64 W = v & ((1u << KS_WBITS) - 1u);
        if (ub <= inc) {
          ++pruned;
        } else if (l < A.n) {
          ++expanded;
          const u64 P = ub - ks_g(A, l, W);
          u64 best = 0;
          // include item l, then exclude it (Alg.: branch on item l)
          for (int b = 0; b < 2; ++b) {
            const u64 W2 = b == 0 ? W + A.w[l] : W;
            if (W2 > A.C) continue;
            const u64 P2 = b == 0 ? P + A.p[l] : P;
            const u64 ub2 = P2 + ks_g(A, l + 1, W2);
            best = P2 > best ? P2 : best;
            if (ub2 > inc && ub2 > P2) {  // ub2 == P2: the node itself is the best completion
              ck[nc] = 0xFFFFFFFFu - (u32)ub2;
              cv[nc] = ((l + 1) << KS_WBITS) | (u32)W2;
              ++nc;
            }
          }
          if (best > inc) atomicMax(reinterpret_cast<ull*>(state + ST_INC), (ull)best);
        }
      }
      const u32 off = block_excl_scan(nc, S.warp_tot, &S.total, tid);
      for (u32 e = 0; e < nc; ++e) {
        S.chk[nch_total + off + e] = ck[e];
        S.chv[nch_total + off + e] = cv[e];
      }
      nch_total += S.total;
      cta_bar<ANT>();
    }
    if (tid == 0 && nch_total) atomicAdd(state + ST_PENDING, (ull)nch_total);
    for (u32 o = 0; o < nch_total; o += K) {
      const u32 m = nch_total - o < (u32)K ? nch_total - o : (u32)K;
      q.insert(S.chk + o, S.chv + o, m);
    }
    inserted += nch_total;
    q.sync();
    if (tid == 0) {
      __threadfence();
      atomicAdd(state + ST_PENDING, (ull)(0ull - (ull)c));
    }
  }
  // counters (per-thread partial sums for expanded / pruned, thread 0 for the rest)
  if (expanded) atomicAdd(state + ST_EXPANDED, expanded);
  if (pruned) atomicAdd(state + ST_PRUNED, pruned);
  if (tid == 0) {
    atomicAdd(state + ST_INSERTED, inserted);
    atomicAdd(state + ST_POPS, pops);
    atomicAdd(state + ST_EMPTY_POPS, empty);
  }
  q.finish();
}

// Item preparation (one CTA of 1024 threads): ratio order by a bitonic sort on the
// cross-multiplied comparison p_a * w_b > p_b * w_a (ties: original index), then prefix sums.
__global__ void __launch_bounds__(1024, 1)
    bgpq_ks_prepare_kernel(u32 n, const u32* w_in, const u32* p_in, u32* w, u32* p, u64* Wp, u64* Pp) {
  __shared__ u32 idx[1024];
  __shared__ u64 sw[1025], sp[1025];
  const int t = threadIdx.x;
  idx[t] = t < (int)n ? (u32)t : 0xFFFFFFFFu;
  __syncthreads();
  auto before = [&](u32 a, u32 b) -> bool {  // a strictly before b
    if (a == 0xFFFFFFFFu) return false;
    if (b == 0xFFFFFFFFu) return true;
    const u64 x = (u64)p_in[a] * w_in[b], y = (u64)p_in[b] * w_in[a];
    return x > y || (x == y && a < b);
  };
  for (int k = 2; k <= 1024; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      const int pr = t ^ j;
      if (pr > t) {
        const u32 a = idx[t], b = idx[pr];
        const bool asc = (t & k) == 0;
        if (asc ? before(b, a) : before(a, b)) { idx[t] = b; idx[pr] = a; }
      }
      __syncthreads();
    }
  }
  if (t < (int)n) {
    w[t] = w_in[idx[t]];
    p[t] = p_in[idx[t]];
    sw[t + 1] = w[t];
    sp[t + 1] = p[t];
  }
  if (t == 0) { sw[0] = 0; sp[0] = 0; }
  __syncthreads();
  if (t == 0) {  // n <= 1023 entries: a serial prefix sum is cheaper than a scan here
    for (u32 i = 1; i <= n; ++i) { sw[i] += sw[i - 1]; sp[i] += sp[i - 1]; }
  }
  __syncthreads();
  if (t <= (int)n) { Wp[t] = sw[t]; Pp[t] = sp[t]; }
}

// seed: the root node (level 0, W = 0, P = 0) with its bound, pending = 1 (one thread)
__global__ void bgpq_ks_root_kernel(KsArgs A, u32* key, u32* val) {
  const u64 ub = ks_g(A, 0, 0);
  key[0] = 0xFFFFFFFFu - (u32)ub;
  val[0] = 0;
}

// =========================================================================================
// A*
// =========================================================================================
struct AsArgs {
  u32 N, M;
  const uint8_t* grid;
  u32* g;  // best known cost per cell (0xFFFFFFFF = none)
  u32 tr, tc;
};

__device__ __forceinline__ u32 manh(u32 r, u32 c, u32 tr, u32 tc) {
  return (r > tr ? r - tr : tr - r) + (c > tc ? c - tc : tc - c);
}
__device__ __forceinline__ u32 as_key(u32 f, u32 h) {
  const u32 hh = (h >> 1) < 0x7FFFu ? (h >> 1) : 0x7FFFu;
  return (f << 15) | hh;
}

template <int K>
struct AsSmem {
  u32 popk[K], popv[K];
  u32 chk[8 * K], chv[8 * K];
  u32 warp_tot[32];
  u32 total;
  u32 done;
};

template <int K>
__global__ void __launch_bounds__(ANT + 32, 1)
    bgpq_astar_kernel(bgpq_dev::HeapView hv, AsArgs A, ull* state, u32 budget) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  using Q = bgpq_dev::Queue<K, true, ANT>;
  Q q;
  q.init(hv, smem_raw);
  if (q.is_lock_warp()) {
    q.run_lock_warp();
    return;
  }
  AsSmem<K>& S = *reinterpret_cast<AsSmem<K>*>(smem_raw + Q::smem_bytes());
  const int tid = threadIdx.x;
  const int DR[8] = {-1, 1, 0, 0, -1, -1, 1, 1};
  const int DC[8] = {0, 0, -1, 1, -1, 1, -1, 1};
  const u64 tcell = (u64)A.tr * A.M + A.tc;
  ull expanded = 0, inserted = 0, pops = 0, pruned = 0, empty = 0;
  u32 backoff = 128;
  for (u32 it = 0; it < budget; ++it) {
    const u32 c = q.size_hint() ? q.deletemin(S.popk, S.popv, K) : 0u;
    if (c == 0) {  // nothing in the heap: done if nothing is in flight either (uniform decision)
      ++empty;
      if (tid == 0) S.done = ld_acq64(state + ST_PENDING) == 0;
      cta_bar<ANT>();
      const bool done = S.done;
      cta_bar<ANT>();
      if (done) break;
      __nanosleep(backoff);
      backoff = backoff < 8192 ? backoff * 2 : 8192;
      continue;
    }
    backoff = 128;
    ++pops;
    u32 nch_total = 0;
    for (int base = 0; base < (int)c; base += ANT) {
      const int t = base + tid;
      u32 ck[8], cv[8], nc = 0;
      if (t < (int)c) {
        const u32 inc = (u32)ld_acq64(state + ST_INC);
        const u32 f = S.popk[t] >> 15;
        const u32 cell = S.popv[t];
        const u32 r = cell / A.M, cc = cell % A.M;
        const u32 h = manh(r, cc, A.tr, A.tc);
        const u32 gp = f - h;
        if (f >= inc) {
          ++pruned;
        } else if (atomicMin(A.g + cell, gp) < gp) {
          ++pruned;  // stale: a shorter path to this cell is known
        } else if ((u64)cell == tcell) {  // start == target
          atomicMin(reinterpret_cast<ull*>(state + ST_INC), (ull)gp);
        } else {
          ++expanded;
          u32 best = 0xFFFFFFFFu;
#pragma unroll
          for (int d = 0; d < 8; ++d) {
            const long long nr = (long long)r + DR[d], ncc = (long long)cc + DC[d];
            if (nr < 0 || ncc < 0 || nr >= A.N || ncc >= A.M) continue;
            const u64 nb = (u64)nr * A.M + (u64)ncc;
            if (A.grid[nb]) continue;
            const u32 g2 = gp + (d < 4 ? 1u : 2u);
            const u32 h2 = manh((u32)nr, (u32)ncc, A.tr, A.tc);
            if (g2 + h2 >= inc) continue;
            if (nb == tcell) {  // a path to the target: candidate incumbent, not expanded
              best = g2 < best ? g2 : best;
              atomicMin(A.g + nb, g2);
              continue;
            }
            if (atomicMin(A.g + nb, g2) <= g2) continue;  // not an improvement
            ck[nc] = as_key(g2 + h2, h2);
            cv[nc] = (u32)nb;
            ++nc;
          }
          if (best != 0xFFFFFFFFu) atomicMin(reinterpret_cast<ull*>(state + ST_INC), (ull)best);
        }
      }
      const u32 off = block_excl_scan(nc, S.warp_tot, &S.total, tid);
      for (u32 e = 0; e < nc; ++e) {
        S.chk[nch_total + off + e] = ck[e];
        S.chv[nch_total + off + e] = cv[e];
      }
      nch_total += S.total;
      cta_bar<ANT>();
    }
    if (tid == 0 && nch_total) atomicAdd(state + ST_PENDING, (ull)nch_total);
    for (u32 o = 0; o < nch_total; o += K) {
      const u32 m = nch_total - o < (u32)K ? nch_total - o : (u32)K;
      q.insert(S.chk + o, S.chv + o, m);
    }
    inserted += nch_total;
    q.sync();
    if (tid == 0) {
      __threadfence();
      atomicAdd(state + ST_PENDING, (ull)(0ull - (ull)c));
    }
  }
  if (expanded) atomicAdd(state + ST_EXPANDED, expanded);
  if (pruned) atomicAdd(state + ST_PRUNED, pruned);
  if (tid == 0) {
    atomicAdd(state + ST_INSERTED, inserted);
    atomicAdd(state + ST_POPS, pops);
    atomicAdd(state + ST_EMPTY_POPS, empty);
  }
  q.finish();
}

__global__ void bgpq_astar_fill_kernel(u32* g, u64 n) {
  for (u64 i = blockIdx.x * (u64)blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) g[i] = 0xFFFFFFFFu;
}
__global__ void bgpq_astar_start_kernel(AsArgs A, u32 sr, u32 sc, u32* key, u32* val) {
  const u32 h = manh(sr, sc, A.tr, A.tc);
  key[0] = as_key(h, h);
  val[0] = sr * A.M + sc;
  A.g[(u64)sr * A.M + sc] = 0;
}

// ---- launch helpers ----------------------------------------------------------------------
template <typename Smem, typename Kern>
int launch_app(bgpq_t* q, Kern kern, size_t q_smem, cudaStream_t s, int* grid_out) {
  bgpq_view_t v;
  if (bgpq_view(q, &v) != BGPQ_OK) return BGPQ_EINVAL;
  const size_t smem = q_smem + sizeof(Smem);
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return BGPQ_ECUDA;
  int occ = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, ANT + 32, smem) != cudaSuccess || occ < 1)
    return BGPQ_ECUDA;
  *grid_out = v.sm_count * occ;
  if (v.ctas > 0 && v.ctas < *grid_out) *grid_out = v.ctas;  // bgpq_set_grid
  return BGPQ_OK;
}

bgpq_dev::HeapView heap_view(bgpq_t* q, u32* K_out, u32* flags_out) {
  bgpq_view_t v;
  bgpq_view(q, &v);
  bgpq_dev::HeapView h;
  h.keys = static_cast<u32*>(v.keys);
  h.vals = static_cast<u32*>(v.vals);
  h.meta = static_cast<NodeMeta*>(v.meta);
  h.hdr = static_cast<u32*>(v.hdr);
  h.cap = v.cap;
  *K_out = v.K;
  *flags_out = v.flags;
  return h;
}

}  // namespace

extern "C" {

int bgpq_ks_prepare(uint32_t n, const uint32_t* w, const uint32_t* p, uint64_t C, bgpq_ks_t* out, void* stream) {
  if (!out || !w || !p || n == 0 || n > 1023 || C >= (1ull << KS_WBITS)) return BGPQ_EINVAL;
  if (!out->w || !out->p || !out->Wp || !out->Pp) return BGPQ_EINVAL;
  out->n = n;
  out->C = C;
  bgpq_ks_prepare_kernel<<<1, 1024, 0, (cudaStream_t)stream>>>(n, w, p, out->w, out->p, out->Wp, out->Pp);
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

int bgpq_ks_root(const bgpq_ks_t* ks, uint32_t* key, uint32_t* val, void* stream) {
  if (!ks || !key || !val) return BGPQ_EINVAL;
  KsArgs A{ks->n, ks->C, ks->w, ks->p, ks->Wp, ks->Pp};
  bgpq_ks_root_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(A, key, val);
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

int bgpq_ks_run(bgpq_t* q, const bgpq_ks_t* ks, uint64_t* state, uint32_t budget, void* stream) {
  if (!q || !ks || !state || budget == 0) return BGPQ_EINVAL;
  u32 K, flags;
  const bgpq_dev::HeapView hv = heap_view(q, &K, &flags);
  if (!(flags & BGPQ_FLAG_VALUES)) return BGPQ_EINVAL;
  KsArgs A{ks->n, ks->C, ks->w, ks->p, ks->Wp, ks->Pp};
  cudaStream_t s = (cudaStream_t)stream;
  int grid = 0, rc = BGPQ_EINVAL;
  if (K == 64) {
    auto kern = bgpq_ks_kernel<64>;
    rc = launch_app<KsSmem<64>>(q, kern, bgpq_dev::Queue<64, true, ANT>::smem_bytes(), s, &grid);
    if (rc == BGPQ_OK)
      kern<<<grid, ANT + 32, bgpq_dev::Queue<64, true, ANT>::smem_bytes() + sizeof(KsSmem<64>), s>>>(
          hv, A, reinterpret_cast<ull*>(state), budget);
  } else if (K == 1024) {
    auto kern = bgpq_ks_kernel<1024>;
    rc = launch_app<KsSmem<1024>>(q, kern, bgpq_dev::Queue<1024, true, ANT>::smem_bytes(), s, &grid);
    if (rc == BGPQ_OK)
      kern<<<grid, ANT + 32, bgpq_dev::Queue<1024, true, ANT>::smem_bytes() + sizeof(KsSmem<1024>), s>>>(
          hv, A, reinterpret_cast<ull*>(state), budget);
  }
  if (rc != BGPQ_OK) return rc;
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

int bgpq_astar_init(const bgpq_astar_t* as, uint32_t sr, uint32_t sc, uint32_t* key, uint32_t* val, void* stream) {
  if (!as || !as->g || !as->grid || !key || !val || sr >= as->N || sc >= as->M) return BGPQ_EINVAL;
  if ((u64)as->N * as->M >= 0xFFFFFFFFull) return BGPQ_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  bgpq_astar_fill_kernel<<<1184, 256, 0, s>>>(as->g, (u64)as->N * as->M);
  AsArgs A{as->N, as->M, as->grid, as->g, as->tr, as->tc};
  bgpq_astar_start_kernel<<<1, 1, 0, s>>>(A, sr, sc, key, val);
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

int bgpq_astar_run(bgpq_t* q, const bgpq_astar_t* as, uint64_t* state, uint32_t budget, void* stream) {
  if (!q || !as || !state || budget == 0) return BGPQ_EINVAL;
  u32 K, flags;
  const bgpq_dev::HeapView hv = heap_view(q, &K, &flags);
  if (!(flags & BGPQ_FLAG_VALUES)) return BGPQ_EINVAL;
  if (as->N + as->M >= (1u << 16)) return BGPQ_EINVAL;  // f < 2^17 in the key
  AsArgs A{as->N, as->M, as->grid, as->g, as->tr, as->tc};
  cudaStream_t s = (cudaStream_t)stream;
  int grid = 0, rc = BGPQ_EINVAL;
  if (K == 64) {
    auto kern = bgpq_astar_kernel<64>;
    rc = launch_app<AsSmem<64>>(q, kern, bgpq_dev::Queue<64, true, ANT>::smem_bytes(), s, &grid);
    if (rc == BGPQ_OK)
      kern<<<grid, ANT + 32, bgpq_dev::Queue<64, true, ANT>::smem_bytes() + sizeof(AsSmem<64>), s>>>(
          hv, A, reinterpret_cast<ull*>(state), budget);
  } else if (K == 1024) {
    auto kern = bgpq_astar_kernel<1024>;
    rc = launch_app<AsSmem<1024>>(q, kern, bgpq_dev::Queue<1024, true, ANT>::smem_bytes(), s, &grid);
    if (rc == BGPQ_OK)
      kern<<<grid, ANT + 32, bgpq_dev::Queue<1024, true, ANT>::smem_bytes() + sizeof(AsSmem<1024>), s>>>(
          hv, A, reinterpret_cast<ull*>(state), budget);
  }
  if (rc != BGPQ_OK) return rc;
  return cudaGetLastError() == cudaSuccess ? BGPQ_OK : BGPQ_ECUDA;
}

}  // extern "C"
