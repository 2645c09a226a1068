// bgpq_pipe.cuh — INSERT calls as a level pipeline (B200 design of Alg.1 for insert-only
// calls).
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
constexpr u32 PIPE_NL = 8;     // slots per level ring
constexpr u32 PIPE_MAXL = 32;  // level rings
enum : int { PC_SORT = 0, PC_ROOTCONS = 32, PC_LCONS = 64, PC_WORDS = 64 + 32 * PIPE_MAXL };

struct PipeArgs {
  u32* ctl;    // PC_WORDS control words (reset per call); consumer counters one per 128 B
  u32* sbk;    // PIPE_NSB * K sorted batches
  u32* sbv;
  u32* sready; // PIPE_NSB: j + 1 when batch j is sorted
  u32* rk;     // PIPE_MAXL * PIPE_NL * K level rings
  u32* rv;
  u32* rhdr;   // PIPE_MAXL * PIPE_NL * 4: {tar, end}
  u32* rflag;  // PIPE_MAXL * PIPE_NL: message index + 1
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

  // send message m (tar, items in slot s; end = 1: no items) to the ring of level l
  __device__ __forceinline__ void send(u32 l, u32 m, u32 tar, int s, u32 end, u32& cons_cache) {
    const u32 slot = m % PIPE_NL;
    if (threadIdx.x == 0 && m >= PIPE_NL) {  // flow control: the slot's previous message consumed
      while (cons_cache < m + 1 - PIPE_NL) {
        cons_cache = ld_acquire(cons(l));
        if (cons_cache < m + 1 - PIPE_NL) __nanosleep(64);
      }
    }
    if (!end) store(ringk(l, slot), ringv(l, slot), s);
    else cta_bar<NT>();
    if (threadIdx.x == 0) {
      u32* h = P.rhdr + ((size_t)l * PIPE_NL + slot) * 4;
      st_relaxed(h + 0, tar);
      st_relaxed(h + 1, end);
      st_release(P.rflag + (size_t)l * PIPE_NL + slot, m + 1);
    }
  }

  // ======================================================================================
  // root stage: PARTIAL_INSERT (Alg.1 l.15-29) for every batch, in call order
  // ======================================================================================
  __device__ void root_stage() {
    const int tid = threadIdx.x;
    // slots: 0 root, 1 pBuffer, 2 items, 3..5 scratch
    int R = 0, PB = 1, I = 2, A = 3, B = 4, T = 5;
    if (tid == 0) {
      ctl->b[0] = ld_relaxed(H.hdr + H_HS);
      ctl->b[1] = ld_relaxed(H.hdr + H_RS);
      ctl->b[2] = ld_relaxed(H.hdr + H_PS);
    }
    cta_bar<NT>();
    u32 hs = ctl->b[0], rs = ctl->b[1], ps = ctl->b[2];
    if (rs > 0) load(R, H.gk + (size_t)1 * K, V ? H.gv + (size_t)1 * K : nullptr);
    if (ps > 0) load(PB, H.gk, V ? H.gv : nullptr);
    u32 sent = 0, cons_cache = 0;
    ull nheap = 0;
    for (u64 j = 0; j < C.n_ops; ++j) {
      const u32 size = op_size(j);
      const u32 slot = (u32)(j % PIPE_NSB);
      if (tid == 0) {
        while (ld_acquire(P.sready + slot) != (u32)(j + 1)) __nanosleep(32);
      }
      load(I, P.sbk + (size_t)slot * K, V ? P.sbv + (size_t)slot * K : nullptr);
      if (tid == 0) st_relaxed(P.ctl + PC_ROOTCONS, (u32)(j + 1));  // the sorter may reuse it
      u32 imin = BK(I)[0];
      if (hs == 0) {  // l.16-19
        const int t = R; R = I; I = t;
        rs = size; hs = 1;
        continue;
      }
      if (rs > 0 && BK(R)[rs - 1] > imin) {  // l.20: root keeps its |root| smallest
        merge(R, rs, I, size, rs, A, B);
        int t = R; R = A; A = t;
        t = I; I = B; B = t;
      }
      if (ps + size < (u32)K) {  // l.21-24: append to the (sorted, R1) buffer
        if (ps > 0) {
          merge(PB, ps, I, size, ps + size, A, B);
          const int t = PB; PB = A; A = t;
        } else {
          const int t = PB; PB = I; I = t;
        }
        ps += size;
        continue;
      }
      const u32 nps = ps + size - K;
      if (ps > 0) {  // l.26-28: the K smallest of items u pBuffer form the batch
        merge(I, size, PB, ps, K, A, B);
        int t = I; I = A; A = t;
        t = PB; PB = B; B = t;
      }
      ps = nps;
      const u32 tar = hs + 1;  // l.4
      if (tar > H.cap) {       // R15: sticky capacity error, the batch is dropped
        if (tid == 0) st_relaxed(H.hdr + H_ERR, (u32)(-3));
        continue;
      }
      hs = tar;
      ++nheap;
      send(1, sent++, tar, I, 0, cons_cache);
    }
    send(1, sent++, 0, 0, 1, cons_cache);
    // write the on-chip state back to the arena (R, PB) and the header
    if (rs > 0) store(H.gk + (size_t)1 * K, V ? H.gv + (size_t)1 * K : nullptr, R);
    if (ps > 0) store(H.gk, V ? H.gv : nullptr, PB);
    cta_bar<NT>();
    if (tid == 0) {
      if (rs > 0) {
        st_relaxed(&H.meta[1].kmin, BK(R)[0]);
        st_relaxed(&H.meta[1].kmax, BK(R)[rs - 1]);
      }
      st_relaxed(&H.meta[1].state, hs ? ST_AVAIL : ST_EMPTY);
      if (ps > 0) {
        st_relaxed(&H.meta[0].kmin, BK(PB)[0]);
        st_relaxed(&H.meta[0].kmax, BK(PB)[ps - 1]);
      }
      st_relaxed(H.hdr + H_HS, hs);
      st_relaxed(H.hdr + H_RS, rs);
      st_relaxed(H.hdr + H_PS, ps);
      ull lin;
      asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(lin) : "l"(H.hdr + H_LIN) : "memory");
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(lin + C.n_ops) : "memory");
      ctl->st[S_INS_OPS] += C.n_ops;
      ctl->st[S_INS_HEAPIFY] += nheap;
    }
    (void)T;
  }

  // ======================================================================================
  // level stage l: INSERT_HEAPIFY steps at depth l (Alg.1 l.30-34) and placements (l.9-10)
  // ======================================================================================
  __device__ void level_stage(u32 l) {
    const int tid = threadIdx.x;
    int N = 0, I = 1, A = 2, B = 3;  // node, items, scratch
    u32 cur = 0, dirty = 0, sent = 0, cons_cache = 0;
    ull lv = 0, nnoop = 0, nswap = 0, nmerge = 0;
    for (u32 m = 0;; ++m) {
      const u32 slot = m % PIPE_NL;
      if (tid == 0) {
        const u32* f = P.rflag + (size_t)l * PIPE_NL + slot;
        while (ld_acquire(f) != m + 1) __nanosleep(32);
        const u32* h = P.rhdr + ((size_t)l * PIPE_NL + slot) * 4;
        ctl->b[0] = ld_relaxed(h + 0);
        ctl->b[1] = ld_relaxed(h + 1);
      }
      cta_bar<NT>();
      const u32 tar = ctl->b[0], end = ctl->b[1];
      if (end) break;
      load(I, ringk(l, slot), ringv(l, slot));
      if (tid == 0) st_relaxed(cons(l), m + 1);
      const u32 dt = depth_of(tar);
      if (dt == l) {  // l.9-10: Heap[tar] <- items
        store(H.gk + (size_t)tar * K, V ? H.gv + (size_t)tar * K : nullptr, I);
        if (tid == 0) {
          st_relaxed(&H.meta[tar].kmin, BK(I)[0]);
          st_relaxed(&H.meta[tar].kmax, BK(I)[K - 1]);
          st_relaxed(&H.meta[tar].state, ST_AVAIL);
        }
        continue;
      }
      const u32 a = tar >> (dt - l);  // the node of depth l on the root -> tar path
      if (a != cur) {
        if (dirty) {
          store(H.gk + (size_t)cur * K, V ? H.gv + (size_t)cur * K : nullptr, N);
          if (tid == 0) {
            st_relaxed(&H.meta[cur].kmin, BK(N)[0]);
            st_relaxed(&H.meta[cur].kmax, BK(N)[K - 1]);
          }
        }
        load(N, H.gk + (size_t)a * K, V ? H.gv + (size_t)a * K : nullptr);
        cur = a;
        dirty = 0;
      }
      // l.33: (Heap[cur], items) <- SORT_SPLIT(Heap[cur], items)
      const u32 cmin = BK(N)[0], cmax = BK(N)[K - 1], imin = BK(I)[0], imax = BK(I)[K - 1];
      ++lv;
      if (cmax <= imin) {
        ++nnoop;
      } else if (imax <= cmin) {
        const int t = N; N = I; I = t;
        dirty = 1;
        ++nswap;
      } else {
        merge(N, K, I, K, K, A, B);
        int t = N; N = A; A = t;
        t = I; I = B; B = t;
        dirty = 1;
        ++nmerge;
      }
      send(l + 1, sent++, tar, I, 0, cons_cache);
    }
    if (l < P.depth) send(l + 1, sent++, 0, 0, 1, cons_cache);
    if (dirty) {
      store(H.gk + (size_t)cur * K, V ? H.gv + (size_t)cur * K : nullptr, N);
      if (tid == 0) {
        st_relaxed(&H.meta[cur].kmin, BK(N)[0]);
        st_relaxed(&H.meta[cur].kmax, BK(N)[K - 1]);
      }
    }
    if (tid == 0) {
      ctl->st[S_INS_LEVELS] += lv;
      ctl->st[S_INS_NOOP] += nnoop;
      ctl->st[S_INS_SWAP] += nswap;
      ctl->st[S_INS_MERGE] += nmerge;
    }
  }

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
