// bgpq_server.cuh — the B200 execution of BGPQ: a root-server CTA plus worker CTAs.
//
// Why: on B200 an inter-SM lock hand-off through L2 costs ~840 cycles
// one way and a 4 KB node stage-in 370-960 cycles, while every DELETEMIN must hand the
// root and the level-1 nodes from one operation to the next (Alg.3 l.11-15: the next
// operation needs the level-1 result).  The paper's per-node locks on the top levels
// therefore serialize the whole queue on L2 round trips.  Here the root, the pBuffer and
// the top T levels (nodes 1 .. 2^(T+1)-1) live in the shared memory of ONE persistent
// "server" CTA which executes every operation's root section and its top-level heapify
// steps in order (flat combining: the operations are combined by one thread block, P:136,
// and it holds the "root lock" for good).  Below level T the paper's protocol runs
// unchanged on worker CTAs: hand-over-hand per-node locks top-down, the TARGET/MARKED
// hand-off, nodes staged with TMA bulk copies.
//
//   server CTA (blockIdx 0):  warps 0-15 = main (SORT_SPLITs in smem, ops in index order)
//                             warp 16    = helper (takes the refill node of the NEXT
//                                          DELETEMIN under its lock, reloads top nodes
//                                          returned by workers)
//   worker CTAs:              pre-sort INSERT batches (Alg.1 l.2, before the root);
//                             INS_BODY tasks: INSERT_HEAPIFY below level T (Alg.1 l.30-34)
//                             DEL_BODY tasks: DELETEMIN_HEAPIFY from a level-T node (Alg.3)
//
// Ordering at the boundary: the depth-(T+1) "gate" nodes use ticket locks whose tickets are
// issued by the server in operation order, so body walks enter the lower heap in the same
// order as the root sections (the hand-over-hand property of P:172 across the boundary).
// A level-T node handed to a DEL_BODY task is "lent": the server does not touch it until
// the worker returns its new content (Alg.3 l.12-14: UNLOCK(cur) after SORT_SPLIT(cur, y)).
// Linearization point of operation j = its root section on the server; the order is
// the operation index order of the call.
#pragma once
#include "bgpq_ops.cuh"

namespace bgpqd {

// top depth T: root + pBuffer + nodes of depth 1..T + 9 scratch/staging slots in smem
template <int K, bool V>
constexpr int srv_depth() {
  constexpr int w = V ? 8 : 4;
  constexpr long budget = 216 * 1024;  // of the 227 KB a CTA may use; the rest is control
  int T = 1;
  while (T < 9 && (long)((1 << (T + 2)) + 9) * K * w <= budget) ++T;
  return T;
}

enum : u32 { TASK_INS = 1, TASK_DEL = 2 };
// cycle counters (header words H_TIME..): server thread 0 and worker thread 0 sums
enum : int {
  TM_SRV_TOTAL = 0, TM_SRV_BATCH_WAIT, TM_SRV_TAR_WAIT, TM_SRV_HOME_WAIT, TM_SRV_TASK_WAIT,
  TM_SRV_MERGE, TM_SRV_INS, TM_SRV_DEL, TM_SRV_MERGES_N,
  TM_W_SORT = 16, TM_W_INS, TM_W_DEL, TM_W_IDLE, TM_W_INS_N, TM_W_DEL_N, TM_W_SORT_N, TM_W_LOCKWAIT,
  TM_N = 32
};
constexpr u32 NTASK = 8192;  // task ring
constexpr u32 NSB = 1024;    // sorted-batch ring

// per-call control words (reset by the host before each call)
// (each word on its own 128-B line: the workers poll some of them)
enum : int {
  C_TASK_HEAD = 0, C_TASK_TAIL = 32, C_SORT_NEXT = 64, C_CONSUMED = 96, C_DONE = 128, C_MAIL = 160,
  C_WORDS = 192
};

struct SrvArgs {
  u32* ctl;        // C_WORDS
  u32* task;       // NTASK * 8 descriptor words
  u32* task_pub;   // NTASK: task index + 1 when published
  u32* payk;       // NTASK * K (INS_BODY batches)
  u32* payv;
  u32* sbk;        // NSB * K sorted insert batches
  u32* sbv;
  u32* sready;     // NSB: op index + 1 when sorted
  u32* serving;    // gate ticket "now serving" counters
  u32* ret;        // per top node: lend sequence returned by the worker
  u32* mailk;      // K: MARKED delivery mailbox ("Heap[root] <- items", Alg.1 l.12)
  u32* mailv;
};

template <int K, bool V, int NT>
struct SrvShape {
  static constexpr int T = srv_depth<K, V>();
  static constexpr int NTOP = 1 << (T + 1);  // node indices 0..NTOP-1 are on-chip (0 = pBuffer)
  static constexpr int GATE0 = NTOP;         // depth T+1 "gate" nodes: GATE0 .. 2*NTOP-1
  static constexpr int NSCR = 6;
  static constexpr int S_TAR = NTOP + NSCR;  // helper's refill staging slot
  static constexpr int S_B0 = S_TAR + 1;     // two insert-batch staging slots
  static constexpr int NSLOTS = S_B0 + 2;
  static constexpr size_t ctl_bytes = ((1024 + 32 * NTOP) + 127) / 128 * 128;
  static constexpr size_t smem = ctl_bytes + (size_t)NSLOTS * K * 4 * (V ? 2 : 1);
};

struct SrvSmem {
  u64 bar_main;
  u64 bar_b[2];
  u64 bar_help;
  u32 b[32];               // main broadcast
  volatile u32 tar_req, tar_done, tar_node, tar_ticket, tar_marked;
  volatile u32 stop;
  volatile u32 nfree;
  u32 freel[16];
  u32 mail_expect;
  volatile u32 pf_node;   // node whose take is requested from the helper (prefetch)
};

__device__ __forceinline__ void main_sync() { cta_bar<512>(); }

__device__ __forceinline__ u32 ld_acquire_cta_shared(const volatile u32* p) {
  u32 v;
  asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_addr((const void*)p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_cta_shared(volatile u32* p, u32 v) {
  asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(smem_addr((const void*)p)), "r"(v) : "memory");
}

// ========================================================================================
// Server CTA
// ========================================================================================
template <int K, bool V, int NT>
struct Server {
  using S = SrvShape<K, V, NT>;
  static constexpr int T = S::T, NTOP = S::NTOP, GATE0 = S::GATE0;
  HeapArgs H;
  SrvArgs A;
  CallArgs C;
  SrvSmem* sm;
  u16* slot_of;   // [NTOP]
  u32* tmin;      // [NTOP]
  u32* tmax;      // [NTOP]
  volatile u32* tlent;  // [NTOP] 0 or 1 (set by main, cleared by the helper)
  volatile u32* texp;  // [NTOP] expected return sequence of a lent node
  u32* tnext;     // [NTOP] gate ticket dispenser (gate g = GATE0 + i)
  u8* tav;        // [NTOP] AVAIL flag of on-chip nodes
  u32* sk;
  u32* sv;
  u32 phase_main, phase_b[2];
  // thread-0 state
  u32 hs, rs, ps;
  u32 tail;  // next task index (only the server publishes tasks)
  ull lin;
  ull st[NSTAT];
  ull tm[TM_N];

  __device__ __forceinline__ u32* BK(int s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(int s) const { return V ? sv + s * K : nullptr; }
  __device__ __forceinline__ bool is_gate(u32 n) const { return n >= (u32)GATE0 && n < 2u * GATE0; }

  ull tmark;
  __device__ __forceinline__ void sec(int id) {  // thread 0: cycles since the previous mark -> tm[id]
    if (threadIdx.x == 0) { const ull t = clock64(); tm[id] += t - tmark; tmark = t; }
  }

  __device__ __forceinline__ int alloc() {  // thread 0
    const u32 n = sm->nfree;
    sm->nfree = n - 1;
    return (int)sm->freel[n - 1];
  }
  __device__ __forceinline__ void release_slot(int s) {  // thread 0
    const u32 n = sm->nfree;
    sm->freel[n] = (u32)s;
    sm->nfree = n + 1;
  }

  // ---- synchronous bulk load by main (global -> smem slot)
  __device__ __forceinline__ void load_sync(int s, const u32* gk, const u32* gv) {
    main_sync();
    if (threadIdx.x == 0) {
      fence_proxy_async();
      const u32 bytes = K * 4u;
      mbar_arrive_expect_tx(&sm->bar_main, V ? 2u * bytes : bytes);
      bulk_g2s(BK(s), gk, bytes, &sm->bar_main);
      if (V) bulk_g2s(BV(s), gv, bytes, &sm->bar_main);
    }
    mbar_wait(&sm->bar_main, phase_main);
    phase_main ^= 1u;
  }
  __device__ __forceinline__ void store_global(u32* gk, u32* gv, int s) {
    main_sync();
    uint4* dk = reinterpret_cast<uint4*>(gk);
    const uint4* srck = reinterpret_cast<const uint4*>(BK(s));
    for (int i = threadIdx.x; i < K / 4; i += NT) dk[i] = srck[i];
    if (V) {
      uint4* dv = reinterpret_cast<uint4*>(gv);
      const uint4* srcv = reinterpret_cast<const uint4*>(BV(s));
      for (int i = threadIdx.x; i < K / 4; i += NT) dv[i] = srcv[i];
    }
    main_sync();
  }
  __device__ __forceinline__ void copy_slot(int dst, int src, int off, int n) {
    main_sync();
    for (int i = threadIdx.x; i < n; i += NT) {
      BK(dst)[i] = BK(src)[i + off];
      if (V) BV(dst)[i] = BV(src)[i + off];
    }
    main_sync();
  }
  __device__ __forceinline__ void merge(int z, int na, int w, int nb, int ma, int x, int y) {
    main_sync();
    const ull t0 = clock64();
    sort_split<K, NT, V>(BK(z), BV(z), na, BK(w), BV(w), nb, ma, BK(x), BV(x), BK(y), BV(y));
    main_sync();
    if (threadIdx.x == 0) { tm[TM_SRV_MERGE] += clock64() - t0; tm[TM_SRV_MERGES_N]++; }
  }
  __device__ __forceinline__ void emit(u32* ok, u32* ov, u32 pos, int s, int off, int n) {
    for (int i = threadIdx.x; i < n; i += NT) {
      ok[pos + i] = BK(s)[off + i];
      if (V && ov) ov[pos + i] = BV(s)[off + i];
    }
  }
  // wait until an on-chip node is not lent to a worker (thread 0)
  __device__ __forceinline__ void wait_home(u32 n) {
    if (n >= (u32)NTOP) return;
    if (!ld_acquire_cta_shared(tlent + n)) return;
    const ull t0 = clock64();
    u32 ns = 32;
    while (ld_acquire_cta_shared(tlent + n)) { __nanosleep(ns); ns = ns < 512 ? ns * 2 : 512; }
    tm[TM_SRV_HOME_WAIT] += clock64() - t0;
  }

  // ---- task publication (thread 0, after main_sync so payload stores are ordered)
  __device__ __forceinline__ u32 task_begin() {
    const u32 t = tail;
    if (t >= NTASK) {  // ring slot reuse: the task NTASK earlier must have been claimed+copied
      const ull t0 = clock64();
      if (C.prog) C.prog[1] = 4;
      while (ld_acquire(A.task_pub + (t % NTASK)) != 0xFFFFFFFFu - (t - NTASK)) __nanosleep(64);
      tm[TM_SRV_TASK_WAIT] += clock64() - t0;
    }
    return t;
  }
  __device__ __forceinline__ void task_publish(u32 t, u32 type, u32 a0, u32 a1, u32 a2, u32 a3) {
    u32* d = A.task + (size_t)(t % NTASK) * 8;
    st_relaxed(d + 0, type);
    st_relaxed(d + 1, a0);
    st_relaxed(d + 2, a1);
    st_relaxed(d + 3, a2);
    st_relaxed(d + 4, a3);
    st_release(A.task_pub + (t % NTASK), t + 1);
    st_release(A.ctl + C_TASK_TAIL, t + 1);
    tail = t + 1;
  }

  // ---- op descriptors
  __device__ __forceinline__ bool op_is_insert(u64 j) const {
    return C.mode == MODE_INSERT || (C.mode == MODE_MIXED && C.op_types[j] == 0);
  }
  __device__ __forceinline__ u32 op_size(u64 j) const {
    if (C.mode == MODE_MIXED) return C.op_sizes[j];
    const u64 rem = C.n - j * (u64)K;
    return (u32)(rem < (u64)K ? rem : (u64)K);
  }

  // ---- async prefetch of the sorted batch of op j into staging slot S_B0 + (j & 1)
  __device__ __forceinline__ bool try_prefetch_batch(u64 j, u64* issued) {  // thread 0
    if (j >= C.n_ops || *issued > j) return true;
    if (!op_is_insert(j)) { *issued = j + 1; return true; }
    if (ld_acquire(A.sready + (j % NSB)) != (u32)(j + 1)) return false;
    const int b = (int)(j & 1);
    fence_proxy_async();
    const u32 bytes = K * 4u;
    mbar_arrive_expect_tx(&sm->bar_b[b], V ? 2u * bytes : bytes);
    bulk_g2s(BK(S::S_B0 + b), A.sbk + (size_t)(j % NSB) * K, bytes, &sm->bar_b[b]);
    if (V) bulk_g2s(BV(S::S_B0 + b), A.sbv + (size_t)(j % NSB) * K, bytes, &sm->bar_b[b]);
    *issued = j + 1;
    return true;
  }

  // request the helper to take node `tar` (the refill source of the NEXT deletemin)
  __device__ __forceinline__ void request_tar(u32 tar) {  // thread 0
    u32 ticket = 0;
    if (is_gate(tar)) ticket = tnext[tar - GATE0]++;
    sm->tar_node = tar;
    sm->tar_ticket = ticket;
    __threadfence_block();
    sm->tar_req = sm->tar_req + 1;
  }

  // ======================================================================================
  // INSERT (Alg.1) — root section + top levels on chip; continuation as an INS_BODY task
  // ======================================================================================
  __device__ void do_insert(u64 j, u32 size, u64* issued) {
    const int tid = threadIdx.x;
    const int b = (int)(j & 1);
    // the sorted batch (Alg.1 l.2 done by a worker before the root section)
    if (tid == 0) {
      const ull t0 = clock64();
      if (C.prog) C.prog[1] = 1;
      while (!try_prefetch_batch(j, issued)) __nanosleep(64);
      if (C.prog) C.prog[1] = 2;
      tm[TM_SRV_BATCH_WAIT] += clock64() - t0;
      if (*issued < j + 2) try_prefetch_batch(j + 1, issued);
      st[S_INS_OPS]++;
    }
    main_sync();
    {
      const ull t0 = clock64();
      if (tid == 0 && C.prog) C.prog[2] = (u32)(*issued);
      mbar_wait(&sm->bar_b[b], phase_b[b]);
      if (tid == 0 && C.prog) C.prog[1] = 3;
      if (tid == 0) tm[TM_SRV_BATCH_WAIT] += clock64() - t0;
    }
    phase_b[b] ^= 1u;
    if (tid == 0) {
      sm->b[0] = alloc();
      sm->b[1] = hs;
      sm->b[2] = rs;
      sm->b[3] = ps;
    }
    main_sync();
    int it = (int)sm->b[0];
    const u32 hs0 = sm->b[1], rs0 = sm->b[2], ps0 = sm->b[3];
    copy_slot(it, S::S_B0 + b, 0, K);
    if (tid == 0) {  // staging slot b is free again: prefetch op j+2 if it is an insert
      st_relaxed(A.ctl + C_CONSUMED, (u32)(j + 1));
      if (*issued == j + 2) try_prefetch_batch(j + 2, issued);
    }
    u32 imin = BK(it)[0], imax = BK(it)[size - 1];
    if (hs0 == 0) {  // l.16-19
      if (tid == 0) {
        release_slot(slot_of[1]);
        slot_of[1] = (u16)it;
        tmin[1] = imin; tmax[1] = imax;
        rs = size; hs = 1;
      }
      main_sync();
      return;
    }
    // l.20: root keeps the |root| smallest
    if (rs0 > 0 && !(tmax[1] <= imin)) {
      if (tid == 0) { sm->b[0] = alloc(); sm->b[1] = alloc(); }
      main_sync();
      const int a = (int)sm->b[0], c = (int)sm->b[1];
      merge(slot_of[1], rs0, it, size, rs0, a, c);
      if (tid == 0) {
        release_slot(slot_of[1]);
        release_slot(it);
        slot_of[1] = (u16)a;
        tmin[1] = BK(a)[0];
        tmax[1] = BK(a)[rs0 - 1];
      }
      it = c;
      imin = BK(it)[0];
      imax = BK(it)[size - 1];
    }
    if (ps0 + size < (u32)K) {  // l.21-24: append (pBuffer kept sorted)
      if (ps0 > 0) {
        if (tid == 0) { sm->b[0] = alloc(); sm->b[1] = alloc(); }
        main_sync();
        const int a = (int)sm->b[0], c = (int)sm->b[1];
        merge(slot_of[0], ps0, it, size, ps0 + size, a, c);
        if (tid == 0) {
          release_slot(slot_of[0]); release_slot(it); release_slot(c);
          slot_of[0] = (u16)a;
        }
      } else if (tid == 0) {
        release_slot(slot_of[0]);
        slot_of[0] = (u16)it;
      }
      if (tid == 0) ps = ps0 + size;
      main_sync();
      return;
    }
    // l.26-28: the K smallest of items ∪ pBuffer form the batch, the rest stays
    const u32 nps = ps0 + size - K;
    if (ps0 > 0) {
      if (tid == 0) { sm->b[0] = alloc(); sm->b[1] = alloc(); }
      main_sync();
      const int a = (int)sm->b[0], c = (int)sm->b[1];
      merge(it, size, slot_of[0], ps0, K, a, c);
      if (tid == 0) {
        release_slot(slot_of[0]); release_slot(it);
        slot_of[0] = (u16)c;
      }
      it = a;
      imin = BK(it)[0];
      imax = BK(it)[K - 1];
    }
    // l.4: heapSize <- heapSize + 1; tar <- heapSize
    const u32 tar = hs0 + 1;
    if (tar > H.cap) {  // R15
      if (tid == 0) { ps = nps; st_relaxed(H.hdr + H_ERR, (u32)(-3)); release_slot(it); }
      main_sync();
      return;
    }
    if (tid == 0) {
      ps = nps; hs = tar;
      st[S_INS_HEAPIFY]++;
    }
    // l.7, l.30-34: the on-chip part of INSERT_HEAPIFY
    const u32 dt = depth_of(tar);
    const u32 last_onchip = dt <= (u32)T ? dt - 1 : (u32)T;  // deepest on-chip path node depth
    for (u32 d = 1; d <= last_onchip; ++d) {
      const u32 c = tar >> (dt - d);
      main_sync();
      if (tid == 0) {
        wait_home(c);
        const u32 cmin = tmin[c], cmax = tmax[c];
        const u32 dec = (cmax <= imin) ? 0u : (imax <= cmin) ? 1u : 2u;
        st[S_INS_LEVELS]++;
        st[dec == 0 ? S_INS_NOOP : dec == 1 ? S_INS_SWAP : S_INS_MERGE]++;
        u32 a = 0, e = 0;
        if (dec == 1) {  // node <- items, items <- node
          const u32 old = slot_of[c];
          slot_of[c] = (u16)it;
          tmin[c] = imin; tmax[c] = imax;
          a = old;
        } else if (dec == 2) {
          a = alloc(); e = alloc();
        }
        sm->b[0] = dec; sm->b[1] = a; sm->b[2] = e; sm->b[3] = slot_of[c];
      }
      main_sync();
      const u32 dec = sm->b[0];
      if (dec == 1) {
        it = (int)sm->b[1];
        imin = BK(it)[0];
        imax = BK(it)[K - 1];
      } else if (dec == 2) {
        const int a = (int)sm->b[1], e = (int)sm->b[2], cs = (int)sm->b[3];
        merge(cs, K, it, K, K, a, e);
        if (tid == 0) {
          release_slot(cs); release_slot(it);
          slot_of[c] = (u16)a;
          tmin[c] = BK(a)[0]; tmax[c] = BK(a)[K - 1];
        }
        it = e;
        imin = BK(it)[0];
        imax = BK(it)[K - 1];
      }
    }
    if (dt <= (u32)T) {  // l.9-10: target on chip
      if (tid == 0) {
        release_slot(slot_of[tar]);  // every on-chip node keeps a slot; tar's was empty
        slot_of[tar] = (u16)it;
        tav[tar] = 1;
        tmin[tar] = imin; tmax[tar] = imax;
      }
      main_sync();
      return;
    }
    // continuation below level T: INS_BODY task (gate g = ancestor of tar at depth T+1)
    const u32 g = tar >> (dt - (u32)(T + 1));
    u32 t = 0;
    main_sync();
    if (tid == 0) {
      t = task_begin();
      sm->b[0] = t;
    }
    main_sync();
    t = sm->b[0];
    store_global(A.payk + (size_t)(t % NTASK) * K, V ? A.payv + (size_t)(t % NTASK) * K : nullptr, it);
    if (tid == 0) {
      release_slot(it);
      st_relaxed(&H.meta[tar].state, ST_TARGET);  // l.5-6 (only its own insert writes tar, R-notes)
      const u32 ticket = tnext[g - GATE0]++;
      task_publish(t, TASK_INS, g, tar, ticket, 0);
      maybe_prefetch_tar(j + 1);  // after TARGET is visible and g's ticket is issued
    }
  }

  // ======================================================================================
  // DELETEMIN (Alg.2 + Alg.3) — on-chip part; the walk below level T is a DEL_BODY task
  // ======================================================================================
  __device__ void do_deletemin(u64 j, u32 size, u32* ok, u32* ov, u32* count_out) {
    // (the refill node of op j+1 is requested as soon as |root| and heapSize are final)
    const int tid = threadIdx.x;
    if (tid == 0) tmark = clock64();
    if (tid == 0) {
      st[S_DEL_OPS]++;
      sm->b[0] = hs; sm->b[1] = rs; sm->b[2] = ps;
    }
    main_sync();
    const u32 hs0 = sm->b[0], rs0 = sm->b[1], ps0 = sm->b[2];
    u32 nout = 0;
    sec(9);
    if (hs0 == 0) {  // l.16-17
      if (tid == 0) *count_out = 0;
      return;
    }
    if (size < rs0) {  // l.18-20: EXTRACT_ROOT
      const int rsl = slot_of[1];
      emit(ok, ov, 0, rsl, 0, size);
      if (tid == 0) sm->b[3] = alloc();
      main_sync();
      const int a = (int)sm->b[3];
      copy_slot(a, rsl, size, rs0 - size);
      if (tid == 0) {
        release_slot(rsl);
        slot_of[1] = (u16)a;
        rs = rs0 - size;
        tmin[1] = BK(a)[0];
        *count_out = size;
        maybe_prefetch_tar(j + 1);
      }
      return;
    }
    emit(ok, ov, 0, slot_of[1], 0, rs0);  // l.22
    nout = rs0;
    main_sync();  // the root slot is read by every thread before thread 0 may swap it
    sec(10);
    if (hs0 == 1) {  // l.23-29: refill from the buffer
      const u32 take = min(rs0 + ps0, size) - rs0;
      const int pb = slot_of[0];
      emit(ok, ov, nout, pb, 0, take);
      if (tid == 0) sm->b[3] = alloc();
      main_sync();
      const int a = (int)sm->b[3];
      copy_slot(a, pb, take, ps0 - take);
      if (tid == 0) {
        release_slot(slot_of[1]);
        slot_of[1] = (u16)a;
        rs = ps0 - take;
        ps = 0;
        if (rs) { tmin[1] = BK(a)[0]; tmax[1] = BK(a)[rs - 1]; }
        *count_out = nout + take;
        maybe_prefetch_tar(j + 1);
      }
      return;
    }
    const u32 remained = size - rs0;
    const u32 tar = hs0;  // l.5
    // ---- l.6-12: refill the root with node tar
    if (tid == 0) {
      st[S_DEL_REFILL]++;
      hs = hs0 - 1;
      if (tar < (u32)NTOP) {  // on chip: the root takes tar's slot (l.11)
        wait_home(tar);
        const u16 t = slot_of[1]; slot_of[1] = slot_of[tar]; slot_of[tar] = t;
        tav[tar] = 0;
        sm->b[3] = 0;
      } else {  // taken by the helper under tar's lock (normally prefetched)
        if (sm->pf_node != tar) request_tar(tar);
        const ull t0 = clock64();
        while (ld_acquire_cta_shared(&sm->tar_done) != sm->tar_req) __nanosleep(32);
        tm[TM_SRV_TAR_WAIT] += clock64() - t0;
        if (sm->tar_marked) st[S_MARKED]++;
        sm->b[3] = 1;
      }
      sm->pf_node = 0xFFFFFFFFu;
    }
    main_sync();
    if (sm->b[3]) copy_slot(slot_of[1], S::S_TAR, 0, K);
    if (tid == 0) { tmin[1] = BK(slot_of[1])[0]; tmax[1] = BK(slot_of[1])[K - 1]; }
    sec(11);
    // l.13: (root, pBuffer) <- SORT_SPLIT(root, K, pBuffer, |pB|, K)
    if (ps0 > 0) {
      if (tid == 0) {
        const int pb = slot_of[0];
        sm->b[0] = (BK(slot_of[1])[K - 1] <= BK(pb)[0]) ? 0u : 1u;
        if (sm->b[0]) { sm->b[1] = alloc(); sm->b[2] = alloc(); }
      }
      main_sync();
      if (sm->b[0]) {
        const int a = (int)sm->b[1], c = (int)sm->b[2];
        merge(slot_of[1], K, slot_of[0], ps0, K, a, c);
        if (tid == 0) {
          release_slot(slot_of[1]); release_slot(slot_of[0]);
          slot_of[1] = (u16)a; slot_of[0] = (u16)c;
          tmin[1] = BK(a)[0]; tmax[1] = BK(a)[K - 1];
        }
      }
    }
    sec(12);
    // ---- l.14: DELETEMIN_HEAPIFY on chip (cur at depth < T: children on chip)
    u32 cur = 1;
    bool stopped = false;
    for (;;) {
      main_sync();  // thread 0's slot-table updates are visible; previous broadcast consumed
      const u32 dcur = depth_of(cur);
      if (dcur >= (u32)T) break;  // children are gate nodes: lend cur to a DEL_BODY task
      const u32 l = 2u * cur, r = l + 1u;
      if (tid == 0) {
        wait_home(l);
        wait_home(r);
        const u32 al = tav[l], ar = tav[r];
        const u64 minc = min(al ? (u64)tmin[l] : (u64)1 << 32, ar ? (u64)tmin[r] : (u64)1 << 32);
        const u32 stop = (u64)tmax[cur] <= minc;  // l.4
        u32 x = 0, y = 0, lr = 0, a = 0, c = 0;
        if (!stop) {
          st[S_DEL_LEVELS]++;
          if (al && ar) {
            if (tmax[l] > tmax[r]) { x = l; y = r; } else { x = r; y = l; }  // l.9 (R6)
            lr = (tmax[l] <= tmin[r] || (tmax[r] <= tmin[l] && x == l)) ? 1u : 2u;
            if (lr == 2) { a = alloc(); c = alloc(); }
            st[lr == 1 ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
          } else {
            y = al ? l : r; x = al ? r : l; lr = 0;
            st[S_DEL_LR_SKIP]++;
          }
        }
        sm->b[0] = stop; sm->b[1] = x; sm->b[2] = y; sm->b[3] = lr; sm->b[4] = a; sm->b[5] = c;
        sm->b[6] = slot_of[l]; sm->b[7] = slot_of[r];
      }
      main_sync();
      sec(13);
      const u32 stop = sm->b[0], x = sm->b[1], y = sm->b[2], lr = sm->b[3];
      if (stop) { stopped = true; break; }
      if (lr == 2) {  // l.10: (Heap[y], Heap[x]) <- SORT_SPLIT(Heap[l], Heap[r])
        const int a = (int)sm->b[4], c = (int)sm->b[5];
        merge((int)sm->b[6], K, (int)sm->b[7], K, K, a, c);
        if (tid == 0) {
          release_slot(slot_of[l]); release_slot(slot_of[r]);
          slot_of[y] = (u16)a; slot_of[x] = (u16)c;
          tmin[y] = BK(a)[0]; tmax[y] = BK(a)[K - 1];
          tmin[x] = BK(c)[0]; tmax[x] = BK(c)[K - 1];
        }
      }
      // l.12: (Heap[cur], Heap[y]) <- SORT_SPLIT(Heap[cur], Heap[y])
      main_sync();
      sec(14);
      if (tid == 0) {
        const u32 swp = tmax[y] <= tmin[cur];
        if (swp) {
          const u16 t = slot_of[cur]; slot_of[cur] = slot_of[y]; slot_of[y] = t;
          u32 q = tmin[cur]; tmin[cur] = tmin[y]; tmin[y] = q;
          q = tmax[cur]; tmax[cur] = tmax[y]; tmax[y] = q;
          st[S_DEL_CY_SWAP]++;
        } else {
          sm->b[1] = alloc(); sm->b[2] = alloc();
        }
        sm->b[0] = swp; sm->b[3] = slot_of[cur]; sm->b[4] = slot_of[y];
      }
      main_sync();
      if (!sm->b[0]) {
        const int a = (int)sm->b[1], c = (int)sm->b[2];
        merge((int)sm->b[3], K, (int)sm->b[4], K, K, a, c);
        if (tid == 0) {
          release_slot(slot_of[cur]); release_slot(slot_of[y]);
          slot_of[cur] = (u16)a; slot_of[y] = (u16)c;
          tmin[cur] = BK(a)[0]; tmax[cur] = BK(a)[K - 1];
          tmin[y] = BK(c)[0]; tmax[y] = BK(c)[K - 1];
        }
      }
      sec(15);
      if (cur == 1) {  // l.13: EXTRACT_ROOT(items, remainedSize)
        main_sync();
        const int rsl = slot_of[1];
        emit(ok, ov, nout, rsl, 0, remained);
        nout += remained;
        if (tid == 0) sm->b[5] = alloc();
        main_sync();
        const int a = (int)sm->b[5];
        copy_slot(a, rsl, remained, K - remained);
        if (tid == 0) {
          release_slot(rsl);
          slot_of[1] = (u16)a;
          rs = K - remained;
          if (rs) { tmin[1] = BK(a)[0]; tmax[1] = BK(a)[rs - 1]; }
          maybe_prefetch_tar(j + 1);
        }
      }
      sec(16);
      cur = y;  // l.15
    }
    sec(17);
    if (stopped) {
      if (cur == 1) {  // l.5-6
        main_sync();
        const int rsl = slot_of[1];
        emit(ok, ov, nout, rsl, 0, remained);
        nout += remained;
        if (tid == 0) sm->b[5] = alloc();
        main_sync();
        const int a = (int)sm->b[5];
        copy_slot(a, rsl, remained, K - remained);
        if (tid == 0) {
          release_slot(rsl);
          slot_of[1] = (u16)a;
          rs = K - remained;
          if (rs) { tmin[1] = BK(a)[0]; tmax[1] = BK(a)[rs - 1]; }
          maybe_prefetch_tar(j + 1);
        }
      }
    } else {
      // lend cur (depth T) to a DEL_BODY task: its content goes to its global slot
      store_global(H.gk + (size_t)cur * K, V ? H.gv + (size_t)cur * K : nullptr, slot_of[cur]);
      if (tid == 0) {
        const u32 l = 2u * cur, r = l + 1u;
        const u32 tl = (l <= H.cap) ? tnext[l - GATE0]++ : 0u;
        const u32 tr = (r <= H.cap) ? tnext[r - GATE0]++ : 0u;
        const u32 seq = texp[cur] + 1u;
        texp[cur] = seq;
        st_release_cta_shared(tlent + cur, 1u);  // texp before the lend flag (helper pairs them)
        const u32 t = task_begin();
        task_publish(t, TASK_DEL, cur, tl, tr, seq);
        if (C.debug & 2u) wait_home(cur);
      }
    }
    sec(18);
    if (tid == 0) *count_out = nout;
    main_sync();
  }

  // ---- prefetch the refill node of the next op if it is a refilling DELETEMIN (thread 0)
  __device__ __forceinline__ void maybe_prefetch_tar(u64 jn) {
    if (C.debug & 1u) return;
    if (jn >= C.n_ops || op_is_insert(jn)) return;
    if (hs < 2 || hs < (u32)NTOP) return;      // no refill, or the node is on chip
    if (op_size(jn) < rs) return;              // served from the root (Alg.2 l.18)
    if (sm->pf_node == hs) return;
    request_tar(hs);
    sm->pf_node = hs;
  }

  // debug (C.debug & 4): check the on-chip invariants after every operation (all main
  // threads); the first violation is recorded in header words 60..63 {op+1, node, kind, hs}
  __device__ void debug_check(u64 j) {
    main_sync();
    __shared__ u32 bad;
    if (threadIdx.x == 0) bad = 0;
    main_sync();
    const u32 nn = min((u32)NTOP - 1, hs);
    for (u32 i = 1; i <= nn; ++i) {
      if (i >= 2 && (!tav[i] || tlent[i])) continue;
      const u32 len = (i == 1) ? rs : (u32)K;
      const u32* d = BK(slot_of[i]);
      for (u32 e = threadIdx.x + 1; e < len; e += NT)
        if (d[e - 1] > d[e]) atomicCAS(&bad, 0u, (i << 8) | 1u);
      if (threadIdx.x == 0 && i >= 2) {
        const u32 p = i / 2;
        const bool pok = (p == 1) ? (rs == 0 || BK(slot_of[1])[rs - 1] <= d[0]) : (tlent[p] || BK(slot_of[p])[K - 1] <= d[0]);
        if (!pok) atomicCAS(&bad, 0u, (i << 8) | 2u);
        if (tmin[i] != d[0] || tmax[i] != d[K - 1]) atomicCAS(&bad, 0u, (i << 8) | 3u);
      }
    }
    if (threadIdx.x == 0 && ps && rs && BK(slot_of[0])[0] < BK(slot_of[1])[rs - 1]) atomicCAS(&bad, 0u, 4u);
    main_sync();
    if (threadIdx.x == 0 && bad && ld_relaxed(H.hdr + 60) == 0) {
      st_relaxed(H.hdr + 61, bad >> 8);
      st_relaxed(H.hdr + 62, bad & 255u);
      st_relaxed(H.hdr + 63, hs);
      st_relaxed(H.hdr + 60, (u32)(j + 1));
    }
    main_sync();
  }

  __device__ void run() {
    const int tid = threadIdx.x;
    // ---- load the on-chip state (root, pBuffer, top nodes) from the heap arena
    if (tid == 0) {
      hs = ld_relaxed(H.hdr + H_HS);
      rs = ld_relaxed(H.hdr + H_RS);
      ps = ld_relaxed(H.hdr + H_PS);
      ull v;
      asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(H.hdr + H_LIN) : "memory");
      lin = v;
      for (int i = 0; i < NSTAT; ++i) st[i] = 0;
      for (int i = 0; i < TM_N; ++i) tm[i] = 0;
      tm[31] = clock64();
      tail = 0;
      tmark = 0;
      sm->pf_node = 0xFFFFFFFFu;
    }
    for (int i = tid; i < NTOP; i += NT) {
      slot_of[i] = (u16)i;
      tlent[i] = 0;
      texp[i] = 0;
      tnext[i] = 0;
      const bool ex = (u32)i <= H.cap;
      const u32 sti = (i >= 2 && ex) ? ld_relaxed(&H.meta[i].state) : 0u;
      tav[i] = (i >= 2 && ex && sti == ST_AVAIL) ? 1 : 0;
      tmin[i] = ex ? ld_relaxed(&H.meta[i].kmin) : 0u;
      tmax[i] = ex ? ld_relaxed(&H.meta[i].kmax) : 0u;
    }
    const u32 nload = min((u32)NTOP, H.cap + 1);
    for (u32 i = 0; i < nload; ++i) load_sync((int)i, H.gk + (size_t)i * K, V ? H.gv + (size_t)i * K : nullptr);
    main_sync();
    // ---- the operations, in index order
    u64 issued = 0;
    if (tid == 0) try_prefetch_batch(0, &issued);
    for (u64 j = 0; j < C.n_ops; ++j) {
      const u32 size = op_size(j);
      if (tid == 0 && C.mode == MODE_MIXED && C.lin_ticket) C.lin_ticket[j] = lin;
      const ull top0 = clock64();
      if (tid == 0 && C.prog) { C.prog[0] = (u32)j; C.prog[1] = 0; }
      if (op_is_insert(j)) {
        do_insert(j, size, &issued);
        if (tid == 0) tm[TM_SRV_INS] += clock64() - top0;
      } else {
        u32* ok = C.out_k;
        u32* ov = C.out_v;
        if (C.mode == MODE_MIXED || C.mode == MODE_DELETEMIN) {
          ok += j * (u64)K;
          if (ov) ov += j * (u64)K;
        }
        u32 cnt = 0;
        do_deletemin(j, size, ok, ov, &sm->b[20]);
        main_sync();
        cnt = sm->b[20];
        if (tid == 0) {
          tm[TM_SRV_DEL] += clock64() - top0;
          st[S_KEYS_OUT] += cnt;
          if (C.mode == MODE_MIXED) C.op_count[j] = cnt;
          if (C.d_count && cnt) atomicAdd(C.d_count, (ull)cnt);
          maybe_prefetch_tar(j + 1);
        }
      }
      if (C.debug & 4u) debug_check(j);
      if (tid == 0) {
        ++lin;
        st_relaxed(A.ctl + C_CONSUMED, (u32)(j + 1));
        if (*(&issued) <= j + 1) try_prefetch_batch(j + 1, &issued);
        maybe_prefetch_tar(j + 1);
      }
      main_sync();
    }
    // ---- end of call: wait for lent nodes, write the on-chip state back, stop helper
    if (tid == 0 && C.prog) C.prog[1] = 10;
    if (tid == 0) {
      for (int i = 2; i < NTOP; ++i) wait_home((u32)i);
      st_release(A.ctl + C_DONE, 1u);
      if (ps) { tmin[0] = BK(slot_of[0])[0]; tmax[0] = BK(slot_of[0])[ps - 1]; }
    }
    main_sync();
    for (int i = 0; i < NTOP && (u32)i <= H.cap; ++i) {
      store_global(H.gk + (size_t)i * K, V ? H.gv + (size_t)i * K : nullptr, slot_of[i]);
    }
    main_sync();
    for (int i = tid; i < NTOP; i += NT) {
      if ((u32)i > H.cap) continue;
      if (i >= 2) st_relaxed(&H.meta[i].state, tav[i] ? ST_AVAIL : ST_EMPTY);
      st_relaxed(&H.meta[i].kmin, tmin[i]);
      st_relaxed(&H.meta[i].kmax, tmax[i]);
    }
    if (tid == 0) {
      st_relaxed(&H.meta[1].state, hs ? ST_AVAIL : ST_EMPTY);
      st_relaxed(H.hdr + H_HS, hs);
      st_relaxed(H.hdr + H_RS, rs);
      st_relaxed(H.hdr + H_PS, ps);
      asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(lin) : "memory");
      ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
      for (int i = 0; i < NSTAT; ++i) if (st[i]) atomicAdd(stat + i, st[i]);
      tm[TM_SRV_TOTAL] = clock64() - tm[31];
      tm[31] = 0;
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      for (int i = 0; i < 9; ++i) if (tm[i]) atomicAdd(tms + i, tm[i]);
      for (int i = 9; i <= 18; ++i) if (tm[i]) atomicAdd(tms + (i < 16 ? i : i + 8), tm[i]);
      sm->stop = 1;
      if (C.prog) C.prog[1] = 11;
    }
  }
};

// ========================================================================================
// Helper warp of the server CTA: refill-node prefetch and reload of returned top nodes
// ========================================================================================
template <int K, bool V, int NT>
__device__ void helper_loop(Server<K, V, NT>& s) {
  using S = SrvShape<K, V, NT>;
  if ((threadIdx.x & 31) != 0) return;
  u32 phase = 0;
  u32 done = 0;
  u32 mail_seen = ld_relaxed(s.A.ctl + C_MAIL);
  const u32 bytes = K * 4u;
  for (;;) {
    bool idle = true;
    // (1) refill node of the next DELETEMIN (Alg.2 l.6-12, taken under its lock)
    if (s.sm->tar_req != done) {
      const u32 req = ld_acquire_cta_shared(&s.sm->tar_req);
      idle = false;
      const u32 n = s.sm->tar_node, ticket = s.sm->tar_ticket;
      const bool gate = s.is_gate(n);
      if (gate) {
        u32 ns = 32;
        while (ld_acquire(s.A.serving + (n - S::GATE0)) != ticket) { __nanosleep(ns); ns = ns < 256 ? 2 * ns : 256; }
      } else {
        lock_acquire(&s.H.meta[n].lock);
      }
      fence_proxy_async();
      const u32 state = ld_relaxed(&s.H.meta[n].state);
      u32 marked = 0;
      if (state == ST_TARGET) {  // l.7-9: steal the keys of the insert in flight
        st_relaxed(&s.H.meta[n].state, ST_MARKED);
        if (gate) st_release(s.A.serving + (n - S::GATE0), ticket + 1);
        else lock_release(&s.H.meta[n].lock);
        while (ld_acquire(s.A.ctl + C_MAIL) == mail_seen) __nanosleep(64);
        mail_seen++;
        fence_proxy_async();
        mbar_arrive_expect_tx(&s.sm->bar_help, V ? 2 * bytes : bytes);
        bulk_g2s(s.BK(S::S_TAR), s.A.mailk, bytes, &s.sm->bar_help);
        if (V) bulk_g2s(s.BV(S::S_TAR), s.A.mailv, bytes, &s.sm->bar_help);
        mbar_wait(&s.sm->bar_help, phase);
        phase ^= 1u;
        marked = 1;
      } else {  // l.11: Heap[root] <- Heap[tar]; Heap[tar].state <- EMPTY
        mbar_arrive_expect_tx(&s.sm->bar_help, V ? 2 * bytes : bytes);
        bulk_g2s(s.BK(S::S_TAR), s.H.gk + (size_t)n * K, bytes, &s.sm->bar_help);
        if (V) bulk_g2s(s.BV(S::S_TAR), s.H.gv + (size_t)n * K, bytes, &s.sm->bar_help);
        mbar_wait(&s.sm->bar_help, phase);
        phase ^= 1u;
        st_relaxed(&s.H.meta[n].state, ST_EMPTY);
        if (gate) st_release(s.A.serving + (n - S::GATE0), ticket + 1);
        else lock_release(&s.H.meta[n].lock);
      }
      s.sm->tar_marked = marked;
      done = req;
      st_release_cta_shared(&s.sm->tar_done, done);
    }
    // (2) reload on-chip nodes returned by DEL_BODY workers
    for (int i = (1 << S::T); i < S::NTOP; ++i) {
      if (!s.tlent[i]) continue;  // plain scan; acquire only on a hit
      if (!ld_acquire_cta_shared(s.tlent + i)) continue;
      if (ld_acquire(s.A.ret + i) != s.texp[i]) continue;
      idle = false;
      fence_proxy_async();
      const int sl = s.slot_of[i];
      mbar_arrive_expect_tx(&s.sm->bar_help, V ? 2 * bytes : bytes);
      bulk_g2s(s.BK(sl), s.H.gk + (size_t)i * K, bytes, &s.sm->bar_help);
      if (V) bulk_g2s(s.BV(sl), s.H.gv + (size_t)i * K, bytes, &s.sm->bar_help);
      mbar_wait(&s.sm->bar_help, phase);
      phase ^= 1u;
      s.tmin[i] = ld_relaxed(&s.H.meta[i].kmin);
      s.tmax[i] = ld_relaxed(&s.H.meta[i].kmax);
      s.tav[i] = ld_relaxed(&s.H.meta[i].state) == ST_AVAIL;
      st_release_cta_shared(s.tlent + i, 0u);
    }
    if (s.sm->stop) break;
    if (idle) __nanosleep(64);
  }
}

// ========================================================================================
// Worker CTAs: batch sorting and the body walks (paper protocol below level T)
// ========================================================================================
template <int K, bool V, int NT>
struct Worker {
  using S = SrvShape<K, V, NT>;
  static constexpr int T = S::T, GATE0 = S::GATE0;
  HeapArgs H;
  SrvArgs A;
  CallArgs C;
  Op<K, V, NT> op;  // smem slots / load / store / merge helpers (6 slots)
  ull tm[8];

  __device__ __forceinline__ bool is_gate(u32 n) const { return n >= (u32)GATE0 && n < 2u * GATE0; }
  __device__ __forceinline__ void acquire(u32 n, u32 ticket) {  // thread 0
    if (is_gate(n)) {
      u32 ns = 32;
      while (ld_acquire(A.serving + (n - GATE0)) != ticket) { __nanosleep(ns); ns = ns < 256 ? 2 * ns : 256; }
    } else {
      lock_acquire(&H.meta[n].lock);
    }
    fence_proxy_async();
  }
  __device__ __forceinline__ void release(u32 n, u32 ticket) {  // thread 0
    if (is_gate(n)) st_release(A.serving + (n - GATE0), ticket + 1);
    else lock_release(&H.meta[n].lock);
  }

  // ---- sort job: Alg.1 l.2 for op j (before its root section)
  __device__ void sort_job(u64 j) {
    const int tid = threadIdx.x;
    const u32 size = (C.mode == MODE_MIXED) ? C.op_sizes[j] : (u32)min((u64)K, C.n - j * (u64)K);
    const u64 off = (C.mode == MODE_MIXED) ? C.in_off[j] : j * (u64)K;
    const u32* ik = C.in_k + off;
    const u32* iv = C.in_v ? C.in_v + off : nullptr;
    int it = 0, tmp = 1;
    cta_bar<NT>();
    for (int i = tid; i < K; i += NT) {
      op.BK(it)[i] = i < (int)size ? ik[i] : KEY_MAX;
      if (V) op.BV(it)[i] = (i < (int)size && iv) ? iv[i] : 0u;
    }
    cta_bar<NT>();
    if (cta_sort<K, NT, V>(op.BK(it), op.BV(it), (int)size, op.BK(tmp), op.BV(tmp))) it = tmp;
    const u32 s = (u32)(j % NSB);
    uint4* dk = reinterpret_cast<uint4*>(A.sbk + (size_t)s * K);
    const uint4* sk4 = reinterpret_cast<const uint4*>(op.BK(it));
    for (int i = tid; i < K / 4; i += NT) dk[i] = sk4[i];
    if (V) {
      uint4* dv = reinterpret_cast<uint4*>(A.sbv + (size_t)s * K);
      const uint4* sv4 = reinterpret_cast<const uint4*>(op.BV(it));
      for (int i = tid; i < K / 4; i += NT) dv[i] = sv4[i];
    }
    cta_bar<NT>();
    if (tid == 0) st_release(A.sready + s, (u32)(j + 1));
  }

  // ---- INS_BODY: INSERT_HEAPIFY from gate node g (held via its ticket) to tar
  __device__ void ins_body(u32 task) {
    const int tid = threadIdx.x;
    const u32* d = A.task + (size_t)(task % NTASK) * 8;
    const u32 g = ld_relaxed(d + 1), tar = ld_relaxed(d + 2), ticket = ld_relaxed(d + 3);
    int it = 0, sc = 1, a = 2, b = 3;
    cta_bar<NT>();
    if (tid == 0) {
      fence_proxy_async();
      const u32 bytes = K * 4u;
      mbar_arrive_expect_tx(&op.ctl->bar, V ? 2u * bytes : bytes);
      bulk_g2s(op.BK(it), A.payk + (size_t)(task % NTASK) * K, bytes, &op.ctl->bar);
      if (V) bulk_g2s(op.BV(it), A.payv + (size_t)(task % NTASK) * K, bytes, &op.ctl->bar);
    }
    mbar_wait(&op.ctl->bar, op.phase);
    op.phase ^= 1u;
    cta_bar<NT>();
    if (tid == 0) {  // payload copied: the ring slot may be reused
      __threadfence();
      st_release(A.task_pub + (task % NTASK), 0xFFFFFFFFu - task);
      if (C.prog) C.prog[17 + 2 * blockIdx.x] = 1;
      acquire(g, ticket);  // LOCK(g): gate tickets keep the server's order
      if (C.prog) C.prog[17 + 2 * blockIdx.x] = 2;
    }
    cta_bar<NT>();
    u32 imin = op.BK(it)[0], imax = op.BK(it)[K - 1];
    u32 held = g, held_ticket = ticket;
    u32 c = g;
    bool first = true;
    for (;;) {
      cta_bar<NT>();
      if (tid == 0) {
        u32 brk = (c == tar) || (ld_relaxed(&H.meta[tar].state) == ST_MARKED);  // l.31
        u32 dec = 0, cmin = 0, cmax = 0;
        if (!brk) {
          if (!first) {  // l.32: LOCK(cur); UNLOCK(PARENT(cur))
            if (C.prog) C.prog[17 + 2 * blockIdx.x] = 0x100000 | c;
            acquire(c, 0);
            release(held, held_ticket);
          }
          cmin = ld_relaxed(&H.meta[c].kmin);
          cmax = ld_relaxed(&H.meta[c].kmax);
          dec = (cmax <= imin) ? 0u : (imax <= cmin) ? 1u : 2u;
          op.st[S_INS_LEVELS]++;
          op.st[dec == 0 ? S_INS_NOOP : dec == 1 ? S_INS_SWAP : S_INS_MERGE]++;
        }
        op.ctl->b[0] = brk; op.ctl->b[1] = dec; op.ctl->b[2] = cmin; op.ctl->b[3] = cmax;
      }
      cta_bar<NT>();
      const u32 brk = op.ctl->b[0], dec = op.ctl->b[1];
      if (brk) break;
      if (!first) { held = c; held_ticket = 0; }  // we now hold c (its parent was released)
      first = false;
      if (dec == 1) {
        const u32 cmin = op.ctl->b[2], cmax = op.ctl->b[3];
        op.load(sc, c);
        op.store(c, it);
        if (tid == 0) op.set_minmax(c, imin, imax);
        const int t = it; it = sc; sc = t;
        imin = cmin; imax = cmax;
      } else if (dec == 2) {
        op.load(sc, c);
        op.merge_split(sc, K, it, K, K, a, b);
        op.store(c, a);
        if (tid == 0) op.set_minmax(c, op.BK(a)[0], op.BK(a)[K - 1]);
        const int t = it; it = b; b = t;
        imin = op.BK(it)[0];
        imax = op.BK(it)[K - 1];
      }
      c = next_on_path(c, tar);
    }
    // l.8: LOCK(tar); UNLOCK(PARENT(cur))
    cta_bar<NT>();
    if (tid == 0) {
      if (tar != held) {
        if (C.prog) C.prog[17 + 2 * blockIdx.x] = 0x200000 | tar;
        acquire(tar, 0);  // tar lies below the gate node: an ordinary node lock
        release(held, held_ticket);
      } else {
        fence_proxy_async();  // tar == g, already held through its ticket
      }
      op.ctl->b[0] = ld_relaxed(&H.meta[tar].state);
    }
    cta_bar<NT>();
    const u32 tar_ticket = (tar == held) ? held_ticket : 0u;
    if (tid == 0 && C.prog) C.prog[17 + 2 * blockIdx.x] = 0x300000 | op.ctl->b[0];
    if (op.ctl->b[0] == ST_TARGET) {  // l.9-10
      op.store(tar, it);
      if (tid == 0) {
        op.set_minmax(tar, imin, imax);
        st_relaxed(&H.meta[tar].state, ST_AVAIL);
        release(tar, tar_ticket);
      }
    } else {  // l.11-13: a DELETEMIN waits for these keys (MARKED): deliver to the root
      cta_bar<NT>();
      uint4* dk = reinterpret_cast<uint4*>(A.mailk);
      const uint4* sk4 = reinterpret_cast<const uint4*>(op.BK(it));
      for (int i = tid; i < K / 4; i += NT) dk[i] = sk4[i];
      if (V) {
        uint4* dv = reinterpret_cast<uint4*>(A.mailv);
        const uint4* sv4 = reinterpret_cast<const uint4*>(op.BV(it));
        for (int i = tid; i < K / 4; i += NT) dv[i] = sv4[i];
      }
      cta_bar<NT>();
      if (tid == 0) {
        op.st[S_MARKED]++;
        st_relaxed(&H.meta[tar].state, ST_EMPTY);
        __threadfence();
        atomicAdd(A.ctl + C_MAIL, 1u);
        release(tar, tar_ticket);
      }
    }
  }

  // ---- DEL_BODY: DELETEMIN_HEAPIFY starting at the lent level-T node y
  __device__ void del_body(u32 task) {
    const int tid = threadIdx.x;
    const u32* d = A.task + (size_t)(task % NTASK) * 8;
    const u32 y0 = ld_relaxed(d + 1), tl0 = ld_relaxed(d + 2), tr0 = ld_relaxed(d + 3), seq = ld_relaxed(d + 4);
    if (tid == 0) st_release(A.task_pub + (task % NTASK), 0xFFFFFFFFu - task);
    int R = 0;
    op.load(R, y0);  // the sinking keys the server left in y's global slot
    u32 cur = y0, cur_ticket = 0;
    for (;;) {
      const u32 l = 2u * cur, r = 2u * cur + 1u;
      int o[NSLOT - 1];
      for (int q = 1, f = 0; q < NSLOT; ++q) o[f++] = (R + q) % NSLOT;
      cta_bar<NT>();
      if (tid == 0) {
        const u32 le = l <= H.cap, re = r <= H.cap;
        const bool first = (cur == y0);
        if (le) acquire(l, first ? tl0 : 0u);  // l.3: LOCK(l); LOCK(r)
        if (re) acquire(r, first ? tr0 : 0u);
        const u32 al = le && ld_relaxed(&H.meta[l].state) == ST_AVAIL;
        const u32 ar = re && ld_relaxed(&H.meta[r].state) == ST_AVAIL;
        const u32 lmin = al ? ld_relaxed(&H.meta[l].kmin) : 0u, lmax = al ? ld_relaxed(&H.meta[l].kmax) : 0u;
        const u32 rmin = ar ? ld_relaxed(&H.meta[r].kmin) : 0u, rmax = ar ? ld_relaxed(&H.meta[r].kmax) : 0u;
        const u64 minc = min(al ? (u64)lmin : (u64)1 << 32, ar ? (u64)rmin : (u64)1 << 32);
        const u32 stop = (u64)op.BK(R)[K - 1] <= minc;
        u32 x = 0, y = 0, lr = 0;
        if (!stop) {
          if (al && ar) {
            if (lmax > rmax) { x = l; y = r; } else { x = r; y = l; }
            lr = (lmax <= rmin) ? 1u : ((rmax <= lmin && x == l) ? 1u : 2u);
            op.st[lr == 1 ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
          } else {
            y = al ? l : r; x = al ? r : l; lr = 0;
            op.st[S_DEL_LR_SKIP]++;
          }
          op.st[S_DEL_LEVELS]++;
        }
        op.ctl->b[0] = stop; op.ctl->b[1] = x; op.ctl->b[2] = y; op.ctl->b[3] = lr;
        op.ctl->b[4] = le; op.ctl->b[5] = re;
      }
      cta_bar<NT>();
      const u32 stop = op.ctl->b[0], x = op.ctl->b[1], y = op.ctl->b[2], lr = op.ctl->b[3];
      const u32 le = op.ctl->b[4], re = op.ctl->b[5];
      const bool first = (cur == y0);
      const u32 tx = first ? (x == l ? tl0 : tr0) : 0u;
      const u32 ty = first ? (y == l ? tl0 : tr0) : 0u;
      if (stop) {  // l.4-8: write cur back and release
        op.store(cur, R);
        if (tid == 0) {
          op.set_minmax(cur, op.BK(R)[0], op.BK(R)[K - 1]);
          if (first) {
            st_relaxed(&H.meta[cur].state, ST_AVAIL);
            st_release(A.ret + cur, seq);  // return the lent node to the server
          } else {
            release(cur, cur_ticket);
          }
          if (le) release(l, first ? tl0 : 0u);
          if (re) release(r, first ? tr0 : 0u);
        }
        break;
      }
      int Y;
      if (lr == 2) {  // l.10-11
        op.load2(o[0], l, o[1], r);
        op.merge_split(o[0], K, o[1], K, K, o[2], o[3]);
        op.store(x, o[3]);
        if (tid == 0) {
          op.set_minmax(x, op.BK(o[3])[0], op.BK(o[3])[K - 1]);
          release(x, tx);
        }
        Y = o[2];
      } else {
        op.load(o[2], y);
        if (tid == 0) {
          if (lr == 1 || (x == l ? le : re)) release(x, tx);
        }
        Y = o[2];
      }
      // l.12
      int C2, Y2;
      if (op.BK(Y)[K - 1] <= op.BK(R)[0]) {
        C2 = Y; Y2 = R;
        if (tid == 0) op.st[S_DEL_CY_SWAP]++;
      } else {
        op.merge_split(R, K, Y, K, K, o[0], o[1]);
        C2 = o[0]; Y2 = o[1];
      }
      op.store(cur, C2);
      if (tid == 0) {  // l.14: UNLOCK(cur)
        op.set_minmax(cur, op.BK(C2)[0], op.BK(C2)[K - 1]);
        if (first) {
          st_relaxed(&H.meta[cur].state, ST_AVAIL);
          st_release(A.ret + cur, seq);
        } else {
          release(cur, cur_ticket);
        }
      }
      cur = y;  // l.15
      cur_ticket = ty;
      R = Y2;
    }
  }

  __device__ void run() {
    const int tid = threadIdx.x;
    for (int i = 0; i < 8; ++i) tm[i] = 0;
    for (;;) {
      if (tid == 0) {
        u32 kind = 0, arg = 0;
        u32 ns = 32;
        const ull ti = clock64();
        for (;;) {
          // body tasks first (they unblock the server)
          const u32 tail = ld_acquire(A.ctl + C_TASK_TAIL);
          u32 head = ld_relaxed(A.ctl + C_TASK_HEAD);
          bool got = false;
          while (head < tail) {
            const u32 prev = atomicCAS(A.ctl + C_TASK_HEAD, head, head + 1);
            if (prev == head) { got = true; break; }
            head = prev;
          }
          if (got) {
            if (C.prog) C.prog[17 + 2 * blockIdx.x] = 0xD0000000u | head;
            while (ld_acquire(A.task_pub + (head % NTASK)) != head + 1) {}
            kind = ld_relaxed(A.task + (size_t)(head % NTASK) * 8);
            arg = head;
            break;
          }
          // sort jobs (bounded by the ring)
          if (C.mode != MODE_DELETEMIN) {
            u32 sn = ld_relaxed(A.ctl + C_SORT_NEXT);
            const u32 cons = ld_relaxed(A.ctl + C_CONSUMED);
            bool gots = false;
            while ((u64)sn < C.n_ops && sn < cons + NSB) {
              const u32 prev = atomicCAS(A.ctl + C_SORT_NEXT, sn, sn + 1);
              if (prev == sn) { gots = true; break; }
              sn = prev;
            }
            if (gots) {
              if (C.mode == MODE_MIXED && C.op_types[sn] != 0) continue;
              kind = 3; arg = sn;
              break;
            }
          }
          if (C.prog) {
            C.prog[17 + 2 * blockIdx.x] = 0xE0000000u | ((ld_relaxed(A.ctl + C_TASK_HEAD) & 0x3FFF) << 14) |
                                          (ld_relaxed(A.ctl + C_TASK_TAIL) & 0x3FFF);
            C.prog[16 + 2 * blockIdx.x] = 0xEE000000u | (ld_relaxed(A.ctl + C_DONE) << 16) |
                                          (ld_relaxed(A.ctl + C_SORT_NEXT) & 0xFFFF);
          }
          if (ld_acquire(A.ctl + C_DONE) && ld_relaxed(A.ctl + C_TASK_HEAD) >= ld_acquire(A.ctl + C_TASK_TAIL)) {
            kind = 0xFFFFFFFFu;
            break;
          }
          __nanosleep(ns);
          ns = ns < 1024 ? ns * 2 : 1024;
        }
        op.ctl->b[8] = kind; op.ctl->b[9] = arg;
        tm[3] += clock64() - ti;
      }
      cta_bar<NT>();
      const u32 kind = op.ctl->b[8], arg = op.ctl->b[9];
      cta_bar<NT>();
      if (kind == 0xFFFFFFFFu) break;
      const ull tw = clock64();
      if (tid == 0 && C.prog) { C.prog[16 + 2 * blockIdx.x] = (kind << 24) | (arg & 0xFFFFFF); C.prog[17 + 2 * blockIdx.x] = 0; }
      if (kind == 3) { sort_job(arg); if (tid == 0) { tm[0] += clock64() - tw; tm[6]++; } }
      else if (kind == TASK_INS) { ins_body(arg); if (tid == 0) { tm[1] += clock64() - tw; tm[4]++; } }
      else if (kind == TASK_DEL) { del_body(arg); if (tid == 0) { tm[2] += clock64() - tw; tm[5]++; } }
    }
    if (tid == 0) {
      ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
      for (int i = 0; i < NSTAT; ++i) if (op.st[i]) atomicAdd(stat + i, op.st[i]);
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME) + 16;
      for (int i = 0; i < 8; ++i) if (tm[i]) atomicAdd(tms + i, tm[i]);
    }
  }
};

template <int K, bool V, int NT>
__global__ void __launch_bounds__(NT + 32, 1) bgpq_srv_kernel(HeapArgs H, CallArgs C, SrvArgs A) {
  using S = SrvShape<K, V, NT>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  if (blockIdx.x == 0) {
    SrvSmem* sm = reinterpret_cast<SrvSmem*>(smem_raw);
    unsigned char* p = smem_raw + 1024;
    Server<K, V, NT> s;
    s.H = H; s.A = A; s.C = C; s.sm = sm;
    s.slot_of = reinterpret_cast<u16*>(p); p += 2 * S::NTOP;
    p = reinterpret_cast<unsigned char*>((reinterpret_cast<size_t>(p) + 15) & ~(size_t)15);
    s.tmin = reinterpret_cast<u32*>(p); p += 4 * S::NTOP;
    s.tmax = reinterpret_cast<u32*>(p); p += 4 * S::NTOP;
    s.tlent = reinterpret_cast<volatile u32*>(p); p += 4 * S::NTOP;
    s.texp = reinterpret_cast<volatile u32*>(p); p += 4 * S::NTOP;
    s.tnext = reinterpret_cast<u32*>(p); p += 4 * S::NTOP;
    s.tav = reinterpret_cast<u8*>(p); p += S::NTOP;
    s.sk = reinterpret_cast<u32*>(smem_raw + S::ctl_bytes);
    s.sv = s.sk + S::NSLOTS * K;
    s.phase_main = 0; s.phase_b[0] = 0; s.phase_b[1] = 0;
    if (threadIdx.x == 0) {
      mbar_init(&sm->bar_main, 1);
      mbar_init(&sm->bar_b[0], 1);
      mbar_init(&sm->bar_b[1], 1);
      mbar_init(&sm->bar_help, 1);
      sm->tar_req = 0; sm->tar_done = 0; sm->tar_marked = 0; sm->stop = 0; sm->pf_node = 0xFFFFFFFFu;
      sm->nfree = S::NSCR;
      for (int i = 0; i < S::NSCR; ++i) sm->freel[i] = S::NTOP + i;
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x < NT) s.run();
    else helper_loop<K, V, NT>(s);
  } else {
    if (threadIdx.x >= NT) return;
    Worker<K, V, NT> w;
    w.H = H; w.A = A; w.C = C;
    Ctl* ctl = reinterpret_cast<Ctl*>(smem_raw);
    w.op.H = H;
    w.op.ctl = ctl;
    w.op.sk = reinterpret_cast<u32*>(smem_raw + 256);
    w.op.sv = w.op.sk + NSLOT * K;
    w.op.phase = 0;
    for (int i = 0; i < NSTAT; ++i) w.op.st[i] = 0;
    if (threadIdx.x == 0) {
      mbar_init(&ctl->bar, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    cta_bar<NT>();
    w.run();
  }
}

}  // namespace bgpqd
