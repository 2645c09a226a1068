// bgpq_pipe.cuh — INSERT calls as a level pipeline (B200 design of Alg.1 for insert-only
// calls): the design, the ring layout and the sorter CTAs; the stages themselves are in
// bgpq_pipe2.cuh.
//
// Why: consecutive BGPQ_INSERTs target consecutive nodes (tar = heapSize + 1, Alg.1 l.4), so
// their INSERT_HEAPIFY paths (Alg.1 l.30-34) share every node down to the last few levels,
// and the hand-over-hand locks make each shared node pass from CTA to CTA through L2
// (~1-2k cycles per hand-off on B200) once per insert.  Here each level of the heap is owned
// by one CTA for the whole call: it keeps the level's current path node in shared memory,
// applies every insert that passes through it, in operation order, and forwards the carried
// items to the next level's CTA through a ring in global memory.  Every node therefore sees
// exactly the sequence of SORT_SPLITs of the sequential execution of Alg.1 in call order:
// the resulting layout equals the sequential model (tests/test_gpu_parity.py checks it), and
// the call is linearizable with linearization order = call order (nothing else runs during a
// call).  Roles (blockIdx.x):
//   0          root stage: PARTIAL_INSERT (Alg.1 l.15-29) with root, pBuffer and heapSize
//              on chip; forms the K-batch, assigns tar = ++heapSize and sends (tar, items) to
//              level 1;
//   1 .. D     level stage l: for (tar, items) with depth(tar) = l stores items at tar
//              (Alg.1 l.9-10); else (node, items) <- SORT_SPLIT(node, items) on the ancestor
//              of tar at depth l (l.33, with the cached-min/max no-op and swap cases) and
//              forwards items to level l + 1;
//   D+1 ..     sorters: Sort(items) of Alg.1 l.2 for batch j into a ring read by the root.
#pragma once
#include "bgpq_locks.cuh"

namespace bgpqd {

constexpr u32 PIPE_NSB = 256;  // sorted-batch ring slots
constexpr u32 PIPE_NL = 16;    // slots per level ring
constexpr u32 PIPE_MAXL = 32;  // level rings
enum : int { PC_SORT = 0, PC_ROOTCONS = 32, PC_LCONS = 64, PC_WORDS = 64 + 32 * PIPE_MAXL };

struct PipeArgs {
  u32* ctl;    // PC_WORDS control words (reset per call); consumer counters one per 128 B
  u32* sbk;    // PIPE_NSB * K sorted batches
  u32* sbv;
  u32* sready; // PIPE_NSB: j + 1 when batch j is sorted
  u32* rk;     // PIPE_MAXL * PIPE_NL * K level rings
  u32* rv;
  u64* rflag;  // PIPE_MAXL * PIPE_NL: (tar | end << 31) << 32 | message index + 1, one
               // release store per message (bgpq_pipe2.cuh)
  u32 depth;   // deepest level with a stage (= depth of the largest node index)
};

template <int K, bool V, int NT>
struct Pipe {
  static constexpr u32 NB = K * 4u;
  HeapArgs H;
  PipeArgs P;
  CallArgs C;
  u32* sk;
  u32* sv;
  LCtl* ctl;  // reuses the control block layout (barriers, broadcast words, counters)
  u32 ph0, ph1;

  __device__ __forceinline__ u32* BK(int s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(int s) const { return V ? sv + s * K : nullptr; }
  __device__ __forceinline__ u32 op_size(u64 j) const {
    const u64 rem = C.n - j * (u64)K;
    return (u32)(rem < (u64)K ? rem : (u64)K);
  }
  __device__ __forceinline__ void merge(int z, int na, int w, int nb, int ma, int x, int y) {
    cta_bar<NT>();
    sort_split<K, NT, V>(BK(z), BV(z), na, BK(w), BV(w), nb, ma, BK(x), BV(x), BK(y), BV(y));
    cta_bar<NT>();
  }
  // TMA stage-in of K entries (keys [+ values]) on ctl->bar, all compute threads wait
  __device__ __forceinline__ void load(int s, const u32* gk, const u32* gv) {
    cta_bar<NT>();
    if (threadIdx.x == 0) {
      fence_proxy_async();
      mbar_arrive_expect_tx(&ctl->bar, V ? 2u * NB : NB);
      bulk_g2s(BK(s), gk, NB, &ctl->bar);
      if (V) bulk_g2s(BV(s), gv, NB, &ctl->bar);
    }
    mbar_wait(&ctl->bar, ph0);
    ph0 ^= 1u;
  }
  __device__ __forceinline__ void store(u32* gk, u32* gv, int s) {
    cta_bar<NT>();
    uint4* dk = reinterpret_cast<uint4*>(gk);
    const uint4* srck = reinterpret_cast<const uint4*>(BK(s));
    for (int i = threadIdx.x; i < K / 4; i += NT) dk[i] = srck[i];
    if (V) {
      uint4* dv = reinterpret_cast<uint4*>(gv);
      const uint4* srcv = reinterpret_cast<const uint4*>(BV(s));
      for (int i = threadIdx.x; i < K / 4; i += NT) dv[i] = srcv[i];
    }
    cta_bar<NT>();
  }
  __device__ __forceinline__ void copy(int dst, int src, int n) {
    cta_bar<NT>();
    for (int i = threadIdx.x; i < n; i += NT) {
      BK(dst)[i] = BK(src)[i];
      if (V) BV(dst)[i] = BV(src)[i];
    }
    cta_bar<NT>();
  }
  __device__ __forceinline__ u32* ringk(u32 l, u32 slot) const { return P.rk + ((size_t)l * PIPE_NL + slot) * K; }
  __device__ __forceinline__ u32* ringv(u32 l, u32 slot) const {
    return V ? P.rv + ((size_t)l * PIPE_NL + slot) * K : nullptr;
  }
  __device__ __forceinline__ u32* cons(u32 l) const { return P.ctl + PC_LCONS + 32 * l; }

  // ======================================================================================
  // sorters: Sort(items) (Alg.1 l.2) of batch j into the ring slot j % PIPE_NSB
  // ======================================================================================
  __device__ void sorter() {
    const int tid = threadIdx.x;
    for (;;) {
      if (tid == 0) ctl->op = atomicAdd(P.ctl + PC_SORT, 1u);
      cta_bar<NT>();
      const u64 j = ctl->op;
      cta_bar<NT>();
      if (j >= C.n_ops) break;
      const u32 size = op_size(j);
      const u32 slot = (u32)(j % PIPE_NSB);
      const u32* ik = C.in_k + j * (u64)K;
      const u32* iv = C.in_v ? C.in_v + j * (u64)K : nullptr;
      for (int i = tid; i < K; i += NT) {
        BK(0)[i] = i < (int)size ? ik[i] : KEY_MAX;
        if (V) BV(0)[i] = (i < (int)size && iv) ? iv[i] : 0u;
      }
      cta_bar<NT>();
      const int res = cta_sort<K, NT, V>(BK(0), BV(0), (int)size, BK(1), BV(1)) ? 1 : 0;
      if (tid == 0 && j >= PIPE_NSB) {  // the root stage has consumed the slot's previous batch
        while (ld_acquire(P.ctl + PC_ROOTCONS) < (u32)(j + 1 - PIPE_NSB)) __nanosleep(128);
      }
      store(P.sbk + (size_t)slot * K, V ? P.sbv + (size_t)slot * K : nullptr, res);
      if (tid == 0) st_release(P.sready + slot, (u32)(j + 1));
    }
  }
};

}  // namespace bgpqd
