// bgpq_dtop.cuh — DELETEMIN calls with the top of the heap on chip (B200 design of Alg.2+3
// for deletemin-only calls; the default execution of bgpq_deletemin).
//
// Why.  Every BGPQ_DELETEMIN must wait for the previous one's level-1 step (Alg.3 l.11-15):
// with the root passed between CTAs through L2 the chain costs ~16k cycles per operation on
// B200.  Two facts of Alg.3 remove most of that chain:
//   (1) the l/r split of one operation at depth d (Alg.3 l.10, (y, x) <- SORT_SPLIT(l, r))
//       reads only the children of its cur, which that operation has not modified yet, and
//       the path (x/y choice, l.9) needs only the children's cached max keys — so all l/r
//       splits of one operation along its path are independent and can run concurrently;
//       only the cheap (cur, y) splits (l.12; a pure swap in >98% of top-level steps) chain;
//   (2) consecutive operations leave the root on opposite sides: a sequential model of
//       Alg.2+3 at C2 shape gives P(op i+1 visits op i's depth-2 node) = 3%, depth-3 0.3%.
// Execution (blockIdx.x == 0, the "top CTA": 3 groups of 256 threads + a helper warp):
//   the root, the pBuffer and the nodes of depths 1-2 (indices 1..7) live in shared memory
//   for the whole call.  Slot i (one per operation) runs concurrently
//     G0: (y1, x1) <- SORT_SPLIT(Heap[2], Heap[3])            op i, depth 0 (l.10)
//     G1: (y2, x2) <- SORT_SPLIT(children of y1)              op i, depth 1
//     G2: (y3, x3) <- SORT_SPLIT(children of y2(i-1))         op i-1, depth 2 (lagged one slot)
//   then thread 0 applies op i-1's depth-2 step and op i's root section (PARTIAL_DELETEMIN,
//   Alg.2 l.15-31) and depth-0/1 steps (the (cur, y) splits, stop tests l.4) in that order,
//   which is the sequential order of Alg.2+3.  If op i's depth-1 children include op i-1's
//   depth-2 node (y1(i) == y1(i-1)) G1's split is deferred until after op i-1's step.
//   Split results land in fresh slots, so a walk that stops early (l.4) just drops them.
//   The depth-3 children of the lagged step are LOCKed and staged by the helper warp
//   one slot ahead; x3 is written back and UNLOCKed (l.11) and y3 — still locked, holding
//   the carried keys — is handed to a worker CTA (blockIdx.x >= 1), which continues Alg.3
//   from l.2 with the paper's hand-over-hand locks (OpL's lock-ahead agents).
//   The helper warp also takes the refill node of the next operation (Alg.2 l.6-12: LOCK,
//   copy, state <- EMPTY, UNLOCK) one slot ahead while heapSize >= 64 (the node is then
//   at depth >= 6, far below anything the top CTA or the lagged step touches).
// Linearizability: operations are applied in call order and each root section sees the
// effects of all earlier ones; the walks below depth 3 are the paper's concurrent walks.
// The early refill take is the interleaving in which op i+1 takes its node right after op
// i's root section; the node is deep, so its keys are not among the K smallest.
#pragma once
#include "bgpq_locks.cuh"

namespace bgpqd {

constexpr int DT_GT = 256;              // threads per merge group
constexpr int DT_NG = 3;                // merge groups
constexpr int DT_NTC = DT_GT * DT_NG;   // compute threads of the top CTA (= worker NT)
constexpr int DT_BLOCK = DT_NTC + 96;   // + control warp, helper warps A, B (top) / lock warp (walkers)
constexpr int DT_BAR_READY = 6, DT_BAR_DONE = 7;  // named barriers: control warp <-> the 3 groups
constexpr int DT_NSLOT = 28;            // smem node slots of the top CTA
constexpr int DT_RQ = 16;               // helper request ring
constexpr u32 DT_BIG = 64;              // pipelined mode needs heapSize >= DT_BIG
constexpr u32 DT_NONE = 0xFFFFFFFFu;

struct DtArgs {
  u32* task_node;  // [cap_nodes + 2 + grid]: node handed to a walker (locked, content in HBM)
  u32* task_seq;   // [cap_nodes + 2 + grid]: call epoch once task_node is valid (release)
  u64* task_go;    // [cap_nodes + 2 + grid]: (epoch << 32) | node whose HBM copy holds the
                   // carried keys, or | 0xFFFFFFFF: cancelled (published early, walk stopped above)
  u32* ctl;        // [0] walker ticket, [1] final task count + 1 (release), reset per call
  u64* op_base;    // nullable: ops of this call already executed by the cluster engine
                   // (bgpq_dsys.cuh); this launch executes the rest
  u32 epoch;       // per launch, >= 1
};

enum : u32 { RQ_STAGE = 1, RQ_REFILL = 2, RQ_WB = 3, RQ_END = 4, RQ_WB2 = 5 };
enum : u32 { J_NONE = 0, J_MERGE = 1, J_STORE = 2, J_OUT = 3, J_SHIFT = 4 };

struct DtJob {
  u32 type, a, b, c, d, e, f, g;  // MERGE: z na w nb ma x y | STORE: node slot n | OUT: slot off n pos_lo pos_hi | SHIFT: dst src off n
};

// thread-0 state of the top CTA (see dt_top)
struct DtS {
  u32 fm;  // free slot mask
  u32 defer, ndq;        // control-warp driver: helper requests queued until the groups run
  u32 dq[6][10];
  u32 eseq;              // early-split sequence number
  u32 est_lo, est_hi;    // output slots of the early depth-2 split of the staged children (G2, phase B)
  u32 lag_early, lag_lo, lag_hi;  // the pending lag step's split was done early into lag_lo / lag_hi
  u32 pout, pout_old;  // slots read by the output bulk copies of this / the previous slot
  u32 wbs, pa0, pb0, pq0, pa1, pb1, pq1;  // write-back sequence, slots pending the helper's read
  u32 hs;
  u32 rs;
  u32 ps;
  u32 sph;
  u32 rph;
  u32 sbi;
  u32 rbi;
  u32 lag_cur;
  u32 lag_bi;
  u32 lag_par;
  u32 lag_s0;
  u32 lag_s1;
  u32 pre_tar;
  u32 pre_slot;
  u32 pre_bi;
  u32 pre_par;
  u32 est_y2;
  u32 est_bi;
  u32 est_par;
  u32 est_s0;
  u32 est_s1;
  u32 fl;
  u32 size;
  u32 path;
  u32 R;
  u32 remained;
  u32 rs_old;
  u32 y1;
  u32 y2;
  u32 car1;
  u32 m1lo;
  u32 m1hi;
  u32 mfa;
  u32 mfb;
  u32 tsl;
  u32 lx;
  u32 ly;
  u32 lX;
  u32 lcar;
  u32 lcar3;
  u32 lcf;
  u32 take_sv;
  u32 stage;
  u32 lag;
  u32 pre;
  u32 est;
  u32 walk;
  u32 walk2;
  u32 m1v;
  u32 conflict;
  u64 i;
  u64 nout;
  u64 tmark;
  __device__ __forceinline__ void init() {
    hs = 0; rs = 0; ps = 0; sph = 0; rph = 0; sbi = 0; rbi = 0; lag_cur = 0; lag_bi = 0; lag_par = 0; lag_s0 = 0; lag_s1 = 0; pre_tar = 0; pre_slot = 0; pre_bi = 0; pre_par = 0; est_y2 = 0; est_bi = 0; est_par = 0; est_s0 = 0; est_s1 = 0; fl = 0; size = 0; path = 0; R = 0; remained = 0; rs_old = 0; y1 = 0; y2 = 0; car1 = 0; m1lo = 0; m1hi = 0; mfa = 0; mfb = 0; tsl = 0; lx = 0; ly = 0; lX = 0; lcar = 0; lcar3 = 0; lcf = 0; take_sv = 0; stage = 0; lag = 0; pre = 0; est = 0; walk = 0; walk2 = 0; m1v = 0; conflict = 0; i = 0; nout = 0; tmark = 0;
    pout = pout_old = DT_NONE;
    defer = 0; ndq = 0;
    est_lo = est_hi = lag_lo = lag_hi = DT_NONE; lag_early = 0;
    wbs = pq0 = pq1 = 0; pa0 = pb0 = pa1 = pb1 = DT_NONE;
    car1 = m1lo = m1hi = mfa = mfb = tsl = lX = lcar = lcar3 = lcf = R = DT_NONE;
  }
};

struct DtCtl {
  u64 sbar[2];   // STAGE completions (helper TMA)
  u64 rbar[2];   // REFILL completions (helper TMA)
  u64 lbar;      // loads issued by thread 0 (call start)
  u32 rq_head[2];  // thread 0 -> helper A (ring 0: STAGE, REFILL) / helper B (ring 1: WB, WB2)
  u32 rq_done[2];  // helper progress
  u32 rq[2][DT_RQ][10];
  u64 qbar[2][DT_RQ];  // entry h of ring r is published by an arrive on qbar[r][h % DT_RQ]
  u32 wb_rd;     // helper: sequence number of the last RQ_WB2 whose smem slots were read
  u32 stg_st[2][2], stg_min[2][2], stg_max[2][2];
  u32 tasks;     // tasks published (helper)
  u32 freemask;
  u32 ns[8];     // slot of on-chip node i (1..7); ns[0] = pBuffer slot (DT_NONE if none)
  // plan of the current slot (written by thread 0 before phase A)
  u32 p_flags;   // F_* below; DT_NONE = call finished
  u32 p_out_slot, p_out_n, p_iop_lo, p_iop_hi;
  u32 p_m[3][4]; // group g: split slots z, w -> lo, hi
  u32 p_sbi, p_spar, p_rwait, p_rbi, p_rpar;
  u32 ctl_done;  // control warp: the slot's decisions are complete
  u32 g2_done;   // G2: sequence number of the last early split finished
  u32 p_e[7];    // early depth-2 split for G2 in phase B: staged s0, s1 -> lo, hi; sbar index, parity
  u32 more;      // another job round follows
  u32 njobs;
  DtJob job[12];
  ull st[NSTAT];
  DtS s;
  ull ts[12];    // debug: thread-0 cycles per phase-B stage
  ull tm[12];    // debug timers (C.debug & 8): plan, phase A, G2 stage wait, refill wait, phase B, slots, conflicts, helper lock wait
};
enum : u32 { F_NEW = 1, F_LAG = 2, F_M0 = 4, F_M1 = 8, F_LAGDONE = 16, F_EARLY = 32, F_JOBS = 64 };
constexpr size_t DTCTL_BYTES = (sizeof(DtCtl) + 127) / 128 * 128;

static_assert(DTCTL_BYTES + (size_t)DT_NSLOT * 1024 * 4 * 2 <= 232448, "top CTA exceeds 227 KB of shared memory at K=1024 w=8");
template <int K, bool V>
constexpr size_t dt_smem_bytes() {
  const size_t top = DTCTL_BYTES + (size_t)DT_NSLOT * K * 4 * (V ? 2 : 1);
  const size_t wrk = LCTL_BYTES + (size_t)LSLOT * K * 4 * (V ? 2 : 1);
  return top > wrk ? top : wrk;
}

__device__ __forceinline__ void grp_bar(int g) {
  asm volatile("bar.sync %0, %1;" ::"r"(2 + g), "n"(DT_GT) : "memory");
}

// SORT_SPLIT by a group of DT_GT threads (t = index in the group): warp-cooperative
// merge path (one ballot co-rank per warp, conflict-free window loads) by default; the
// per-thread register-window merge path with test switch win (BGPQ_DEBUG bit 64)
template <int K, bool V>
__device__ __forceinline__ void grp_split(int t, const u32* zk, const u32* zv, int na, const u32* wk, const u32* wv,
                                          int nb, int ma, u32* xk, u32* xv, u32* yk, u32* yv, bool win = false) {
#ifndef BGPQ_NO_BITONIC
  if constexpr (!V && K >= BITONIC_MIN_K) {  // keys only, full batches: bitonic split (bgpq_prim.cuh)
    constexpr int NB = K < DT_GT ? K : DT_GT;
    if (!win && na == K && nb == K && ma == K) {
      // named barrier 8 + group: its own id (grp_bar uses 2 + g with all DT_GT threads)
      if (t < NB) bitonic_split_full<K, NB, false>(t, 8 + (int)(threadIdx.x / DT_GT), zk, zv, wk, wv, xk, xv, yk, yv);
      return;
    }
  }
#endif
  if (!win) {
    constexpr int NW = (2 * K / 32 < DT_GT / 32) ? 2 * K / 32 : DT_GT / 32;
    grp_merge_warp<K, NW, V>(t >> 5, zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
  } else {
    constexpr int NTM = (2 * K / 4 <= DT_GT) ? 2 * K / 4 : DT_GT;
    if (t < NTM) grp_merge_win<K, NTM, V>(t, zk, zv, na, wk, wv, nb, ma, xk, xv, yk, yv);
  }
}

// =========================================================================================
// The top CTA
// =========================================================================================
template <int K, bool V>
struct DTop {
  static constexpr u32 NB = K * 4u;
  HeapArgs H;
  CallArgs C;
  DtArgs D;
  DtCtl* c;
  u32* sk;
  u32* sv;

  __device__ __forceinline__ u32* BK(u32 s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(u32 s) const { return V ? sv + s * K : nullptr; }
  __device__ __forceinline__ u32* lk(u32 n) const { return &H.meta[n].lock; }
  __device__ __forceinline__ u32* stp(u32 n) const { return &H.meta[n].state; }

  // ---- thread 0: slot allocation
  __device__ __forceinline__ u32 alloc(DtS& S) {
    const u32 m = S.fm;
    if (m == 0) __trap();  // slot budget exceeded: a bug, never silent corruption
    const u32 s = __ffs(m) - 1;
    S.fm = m & ~(1u << s);
    return s;
  }
  __device__ __forceinline__ void release_slot(DtS& S, u32 s) {
    if (s != DT_NONE) S.fm |= 1u << s;
  }
  __device__ __forceinline__ u32 kmax(u32 s) const { return BK(s)[K - 1]; }
  __device__ __forceinline__ u32 kmin(u32 s) const { return BK(s)[0]; }

  // ---- thread 0: helper requests (FIFO, processed in order by the helper warp)
  __device__ __forceinline__ void enqueue(u32 type, u32 a0 = 0, u32 a1 = 0, u32 a2 = 0, u32 a3 = 0, u32 a4 = 0,
                                          u32 a5 = 0, u32 a6 = 0, u32 a7 = 0, u32 a8 = 0) {
    const ull tq = (C.debug & 8u) ? clock64() : 0;
    const u32 r = (type == RQ_STAGE || type == RQ_REFILL) ? 0u : 1u;
    const u32 h = c->rq_head[r];
    if (h - *reinterpret_cast<volatile u32*>(&c->rq_done[r]) >= (u32)DT_RQ) {
      while (h - *reinterpret_cast<volatile u32*>(&c->rq_done[r]) >= (u32)DT_RQ) __nanosleep(32);
      (void)ld_acq_cta(&c->rq_done[r]);
    }
    u32* e = c->rq[r][h % DT_RQ];
    e[0] = type; e[1] = a0; e[2] = a1; e[3] = a2; e[4] = a3; e[5] = a4;
    e[6] = a5; e[7] = a6; e[8] = a7; e[9] = a8;
    c->rq_head[r] = h + 1u;  // (thread 0's own counter)
    // publish: mbarrier arrive (release, CTA scope); the helper's try_wait acquires
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&c->qbar[r][h % DT_RQ])) : "memory");
    if (C.debug & 8u) c->ts[9] += clock64() - tq;
  }
  // ---- a helper request now, or (control-warp driver) after the groups were released
  __device__ __forceinline__ void req(DtS& S, u32 type, u32 a0 = 0, u32 a1 = 0, u32 a2 = 0, u32 a3 = 0, u32 a4 = 0,
                                      u32 a5 = 0, u32 a6 = 0, u32 a7 = 0, u32 a8 = 0) {
    if (!S.defer) { enqueue(type, a0, a1, a2, a3, a4, a5, a6, a7, a8); return; }
    u32* e = S.dq[S.ndq++];
    e[0] = type; e[1] = a0; e[2] = a1; e[3] = a2; e[4] = a3; e[5] = a4; e[6] = a5; e[7] = a6; e[8] = a7; e[9] = a8;
  }
  __device__ __forceinline__ void flush(DtS& S) {
    const u32 n = S.ndq;
    for (u32 q = 0; q < n; ++q) {
      const u32* e = S.dq[q];
      enqueue(e[0], e[1], e[2], e[3], e[4], e[5], e[6], e[7], e[8], e[9]);
    }
    S.ndq = 0;
  }

  // ---- thread 0: hand the write-back of a lag step to the helper (RQ_WB2): node x <- slot X
  // (X = DT_NONE: only UNLOCK x), node y <- slot Y, then UNLOCK x and publish y to a walker
  // (pub) or UNLOCK it.  The slots stay allocated until the helper has read them (wb_rd).
  __device__ __forceinline__ void writeback(DtS& S, u32 x, u32 X, u32 y, u32 Y, bool pub) {
    const u32 seq = ++S.wbs;
    enqueue(RQ_WB2, x, X, y, Y, (pub ? 1u : 0u) | (seq << 1), X != DT_NONE ? kmin(X) : 0u,
            X != DT_NONE ? kmax(X) : 0u, kmin(Y), kmax(Y));
    // free slots of older write-backs whose bulk reads are done; keep two generations
    if (S.pq1 != 0) {
      while ((int)(*reinterpret_cast<volatile u32*>(&c->wb_rd) - S.pq1) < 0) __nanosleep(32);
      release_slot(S, S.pa1); release_slot(S, S.pb1);
    }
    S.pa1 = S.pa0; S.pb1 = S.pb0; S.pq1 = S.pq0;
    S.pa0 = X; S.pb0 = Y; S.pq0 = seq;
  }

  // ---- thread 0: collective jobs for the next barrier round
  __device__ __forceinline__ void job(u32 type, u32 a = 0, u32 b = 0, u32 cc = 0, u32 d = 0, u32 e = 0, u32 f = 0,
                                      u32 g = 0) {
    DtJob& j = c->job[c->njobs++];
    j.type = type; j.a = a; j.b = b; j.c = cc; j.d = d; j.e = e; j.f = f; j.g = g;
  }

  // ---- all compute threads: execute the posted jobs (independent of each other)
  __device__ __forceinline__ void run_jobs() {
    const int tid = threadIdx.x;
    const u32 nj = c->njobs;
    for (u32 q = 0; q < nj; ++q) {
      const DtJob j = c->job[q];
      if (j.type == J_MERGE) {
        constexpr int NTM = (2 * K / 4 <= DT_NTC) ? 2 * K / 4 : 512;
        if (tid < NTM)
          grp_merge_win<K, NTM, V>(tid, BK(j.a), BV(j.a), (int)j.b, BK(j.c), BV(j.c), (int)j.d, (int)j.e, BK(j.f),
                                   BV(j.f), BK(j.g), BV(j.g));
      } else if (j.type == J_STORE) {  // node j.a <- slot j.b (K entries, 128-bit stores)
        uint4* dk = reinterpret_cast<uint4*>(H.gk + (size_t)j.a * K);
        const uint4* s4 = reinterpret_cast<const uint4*>(BK(j.b));
        for (int i = tid; i < K / 4; i += DT_NTC) dk[i] = s4[i];
        if (V) {
          uint4* dv = reinterpret_cast<uint4*>(H.gv + (size_t)j.a * K);
          const uint4* v4 = reinterpret_cast<const uint4*>(BV(j.b));
          for (int i = tid; i < K / 4; i += DT_NTC) dv[i] = v4[i];
        }
      } else if (j.type == J_OUT) {  // out[pos .. pos+n) <- slot j.a [off, off+n)
        const u64 pos = ((u64)j.e << 32) | j.d;
        const u32* sk2 = BK(j.a) + j.b;
        for (u32 i = tid; i < j.c; i += DT_NTC) C.out_k[pos + i] = sk2[i];
        if (V && C.out_v) {
          const u32* sv2 = BV(j.a) + j.b;
          for (u32 i = tid; i < j.c; i += DT_NTC) C.out_v[pos + i] = sv2[i];
        }
      } else if (j.type == J_SHIFT) {  // slot a [0, n) <- slot b [off, off+n)
        for (u32 i = tid; i < j.d; i += DT_NTC) {
          BK(j.a)[i] = BK(j.b)[j.c + i];
          if (V) BV(j.a)[i] = BV(j.b)[j.c + i];
        }
      }
    }
  }
};

// ---- the helper warp (lane 0): locks, staging, write-back publication
template <int K, bool V>
__device__ __forceinline__ void dt_helper(DTop<K, V>& T, const u32 hr) {
  DtCtl* c = T.c;
  const HeapArgs& H = T.H;
  const u32 NB = K * 4u;
  u32 seen = 0;
  for (;;) {
    {
      u64* qb = &c->qbar[hr][seen % DT_RQ];
      const u32 par = (seen / DT_RQ) & 1u;
      while (!mbar_test(qb, par)) __nanosleep(20);
    }
    {
      const u32* e = c->rq[hr][seen % DT_RQ];
      const u32 type = e[0];
      if (T.C.prog) { T.C.prog[2 + 5 * hr] = seen; T.C.prog[3 + 5 * hr] = (type << 24) | (e[1] & 0xFFFFFFu); }
      if (type == RQ_STAGE && e[5] == DT_NONE) {  // ring-0 end marker
        st_rel_cta(&c->rq_done[hr], seen + 1u);
        return;
      }
      if (type == RQ_STAGE) {  // LOCK(l); LOCK(r) (Alg.3 l.3) and stage the AVAIL ones
        const u32 n[2] = {e[1], e[2]};
        const u32 s[2] = {e[3], e[4]};
        const u32 bi = e[5];
        u32 bytes = 0;
        u32 stv[2];
        {  // both CASes in flight at once; holding only r while l is busy is not allowed (l before r)
          const ull tw = (T.C.debug & 8u) ? clock64() : 0;
          const u32 ra = cas_acquire(T.lk(n[0]), 0u, 1u);
          const u32 rb = n[1] ? cas_acquire(T.lk(n[1]), 0u, 1u) : 0u;
          if (ra != 0u) {
            if (n[1] && rb == 0u) lock_release(T.lk(n[1]));
            lock_acquire(T.lk(n[0]));
            if (n[1]) lock_acquire(T.lk(n[1]));
          } else if (rb != 0u) {
            lock_acquire(T.lk(n[1]));
          }
          if (T.C.debug & 8u) c->tm[7] += clock64() - tw;
        }
        for (int q = 0; q < 2; ++q) {
          stv[q] = ST_EMPTY;
          u32 mn = 0, mx = 0;
          if (n[q]) {
            stv[q] = ld_relaxed(T.stp(n[q]));
            mn = ld_relaxed(&H.meta[n[q]].kmin);
            mx = ld_relaxed(&H.meta[n[q]].kmax);
            if (stv[q] == ST_AVAIL) bytes += V ? 2u * NB : NB;
          }
          c->stg_st[bi][q] = stv[q]; c->stg_min[bi][q] = mn; c->stg_max[bi][q] = mx;
        }
        fence_proxy_async();
        mbar_arrive_expect_tx(&c->sbar[bi], bytes);
        for (int q = 0; q < 2; ++q) {
          if (stv[q] != ST_AVAIL) continue;
          bulk_g2s(T.BK(s[q]), H.gk + (size_t)n[q] * K, NB, &c->sbar[bi]);
          if (V) bulk_g2s(T.BV(s[q]), H.gv + (size_t)n[q] * K, NB, &c->sbar[bi]);
        }
      } else if (type == RQ_REFILL) {  // Alg.2 l.6-12: LOCK(tar); copy; state <- EMPTY; UNLOCK
        const u32 tar = e[1], s = e[2], bi = e[3];
        lock_acquire(T.lk(tar));
        fence_proxy_async();
        mbar_arrive_expect_tx(&c->rbar[bi], V ? 2u * NB : NB);
        bulk_g2s(T.BK(s), H.gk + (size_t)tar * K, NB, &c->rbar[bi]);
        if (V) bulk_g2s(T.BV(s), H.gv + (size_t)tar * K, NB, &c->rbar[bi]);
        // in a deletemin-only call nothing writes an EMPTY node, so the lock can go at once
        st_relaxed(T.stp(tar), ST_EMPTY);
        lock_release(T.lk(tar));
        if (tar - 1u >= DT_BIG) {  // the refill node after this one: warm it in L2
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gk + (size_t)(tar - 1u) * K), "r"(NB)
                       : "memory");
          if (V)
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gv + (size_t)(tar - 1u) * K), "r"(NB)
                         : "memory");
        }
      } else if (type == RQ_WB) {  // UNLOCK written nodes (l.11 / l.7) and hand y3 to a walker
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        if (e[1]) st_relaxed(T.lk(e[1]), 0u);
        if (e[2]) st_relaxed(T.lk(e[2]), 0u);
        if (e[3]) {
          const u32 t = c->tasks++;
          st_relaxed(T.D.task_node + t, e[3]);
          st_relaxed_u64(T.D.task_go + t, ((u64)T.D.epoch << 32) | e[3]);
          st_release(T.D.task_seq + t, T.D.epoch);
        }
      } else if (type == RQ_WB2) {  // Alg.3 l.10-15 write-backs of the lag step, then UNLOCK / hand over
        const u32 x = e[1], X = e[2], y = e[3], Y = e[4], fl2 = e[5];
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (X != DT_NONE) {
          bulk_s2g(H.gk + (size_t)x * K, T.BK(X), NB);
          if (V) bulk_s2g(H.gv + (size_t)x * K, T.BV(X), NB);
        }
        bulk_s2g(H.gk + (size_t)y * K, T.BK(Y), NB);
        if (V) bulk_s2g(H.gv + (size_t)y * K, T.BV(Y), NB);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        st_rel_cta(&c->wb_rd, fl2 >> 1);  // thread 0 may reuse the slots
        if (X != DT_NONE) { st_relaxed(&H.meta[x].kmin, e[6]); st_relaxed(&H.meta[x].kmax, e[7]); }
        st_relaxed(&H.meta[y].kmin, e[8]); st_relaxed(&H.meta[y].kmax, e[9]);
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        asm volatile("fence.proxy.async.global;" ::: "memory");
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        if (x) st_relaxed(T.lk(x), 0u);
        if (fl2 & 1u) {
          const u32 t = c->tasks++;
          st_relaxed(T.D.task_node + t, y);
          st_relaxed_u64(T.D.task_go + t, ((u64)T.D.epoch << 32) | y);
          st_release(T.D.task_seq + t, T.D.epoch);
        } else {
          st_relaxed(T.lk(y), 0u);
        }
      } else if (type == RQ_END) {
        if (hr == 1) st_release(T.D.ctl + 1, c->tasks + 1u);
        st_rel_cta(&c->rq_done[hr], seen + 1u);
        return;
      }
      ++seen;
      st_rel_cta(&c->rq_done[hr], seen);
    }
  }
}

// The top CTA's compute threads.  Thread 0 owns the heap state (heapSize, |root|,
// |pBuffer|, the on-chip slot table) and makes every decision; all compute threads execute
// the splits of phase A and the collective jobs thread 0 posts in phase B.
// Phase B fast path (thread 0): the common pipelined slot — op i-1's depth-2 step and op i's
// REFILL root section and depth-0/1 steps with both children AVAIL, no stop (l.4), every
// (cur, y) split a swap (l.12), empty pBuffer or no pBuffer merge, no extraction and no
// deferred split.  All tests are evaluated from independent shared-memory loads first; if
// any fails nothing has been modified and the general state machine runs instead.
template <int K, bool V>
__device__ __forceinline__ bool dt_fast(DTop<K, V>& T, DtS& S) {
  DtCtl* c = T.c;
  const HeapArgs& H = T.H;
  // ---- the state this path reads, into registers (independent shared-memory loads)
  const u32 fl = S.fl, path = S.path, conflict = S.conflict, m1v = S.m1v, size = S.size, rs0 = S.rs;
  const u32 hs0 = S.hs, y1 = S.y1, R = S.R, lo1 = S.m1lo, hi1 = S.m1hi, ps = S.ps;
  const u64 i = S.i;
  if (!(fl & F_NEW) || path != 3u || conflict || !(fl & F_M0) || !m1v || size != (u32)K ||
      (rs0 != (u32)K && rs0 != 0u))
    return false;
  const bool lag = (fl & F_LAG) != 0;
  const bool lt = (T.C.debug & 128u) != 0;
  ull tq = lt ? clock64() : 0;
#define DT_MARK(k) if (lt) { const ull t_ = clock64(); c->ts[k] += t_ - tq; tq = t_; }
  const u32 hs = hs0 - 1u;  // after the refill
  const u32 x1 = y1 ^ 1u, cl = 2u * y1, cr = cl + 1u;
  if (cr > hs) return false;
  // |root| = 0 (R4: a drained heap keeps heapSize = 1): the whole refilled root is the output
  // (EXTRACT_ROOT(items, remainedSize = K), Alg.3), emitted by one TMA bulk store
  const bool emit_root = rs0 == 0u;
  const u64 opos = i * (u64)K;
  if (emit_root && (((reinterpret_cast<uintptr_t>(T.C.out_k + opos) & 15u) != 0) ||
                    (V && T.C.out_v && (reinterpret_cast<uintptr_t>(T.C.out_v + opos) & 15u) != 0)))
    return false;
  const u32 nl = c->ns[cl], nr = c->ns[cr], n2 = c->ns[2], n3 = c->ns[3], oroot = c->ns[1];
  const u32 lo0 = c->p_m[0][2], hi0 = c->p_m[0][3];
  const u32 Rmax = T.kmax(R), Rmin = T.kmin(R);
  const u32 min2 = T.kmin(n2), min3 = T.kmin(n3), max2 = T.kmax(n2);
  const u32 lo0max = T.kmax(lo0), lo1max = T.kmax(lo1);
  const u32 minl = T.kmin(nl), minr = T.kmin(nr), maxl = T.kmax(nl), maxr = T.kmax(nr);
  const u32 pbmin = ps ? T.kmin(c->ns[0]) : KEY_MAX;
  u32 lcur = 0, lcar = DT_NONE, lo2 = DT_NONE, hi2 = DT_NONE, st0 = 0, st1 = 0, mn0 = 0, mn1 = 0, mx0 = 0, mx1 = 0;
  u32 lcarmax = 0, lcarmin = 0, lo2max = 0, lag_s0 = 0, lag_s1 = 0;
  if (lag) {
    const u32 bi = S.lag_bi;
    lcur = S.lag_cur; lag_s0 = S.lag_s0; lag_s1 = S.lag_s1;
    lcar = c->ns[lcur];
    lo2 = c->p_m[2][2]; hi2 = c->p_m[2][3];
    st0 = c->stg_st[bi][0]; st1 = c->stg_st[bi][1];
    mn0 = c->stg_min[bi][0]; mn1 = c->stg_min[bi][1];
    mx0 = c->stg_max[bi][0]; mx1 = c->stg_max[bi][1];
    lcarmax = T.kmax(lcar); lcarmin = T.kmin(lcar); lo2max = T.kmax(lo2);
  }
  // ---- tests
  if (ps && Rmax > pbmin) return false;                        // l.13 would merge
  if (Rmax <= min(min2, min3)) return false;                    // l.4 stop at the root
  if (lo0max > Rmin) return false;                              // l.12 not a swap at the root
  if (Rmax <= min(minl, minr)) return false;                    // l.4 stop at y1 (carry = R)
  if (lo1max > Rmin) return false;                              // l.12 not a swap at y1
  if (lag) {
    if (st0 != ST_AVAIL || st1 != ST_AVAIL) return false;
    if (lcarmax <= min(mn0, mn1)) return false;                 // l.4 stop at y2(i-1)
    if (lo2max > lcarmin) return false;                         // l.12 not a swap at y2(i-1)
  }
  DT_MARK(0)
  u32 fm = S.fm;
  u32 d_lv = 2, d_merge = 0, d_nomove = 0;
  // ---- commit: op i-1's depth-2 step (l.9-12), write-back + hand-over by helper B
  if (lag) {
    const u32 c0 = 2u * lcur, c1 = c0 + 1u;
    const u32 x3 = mx0 > mx1 ? c0 : c1, y3 = mx0 > mx1 ? c1 : c0;  // l.9 (R6)
    ++d_lv;
    if (mx0 <= mn1) ++d_nomove; else ++d_merge;
    c->ns[lcur] = lo2;
    fm |= (1u << lag_s0) | (1u << lag_s1);
    const u32 seq = S.wbs + 1u;
    S.wbs = seq;
    T.req(S, RQ_WB2, x3, hi2, y3, lcar, ((2u * y3 <= hs0) ? 1u : 0u) | (seq << 1), T.kmin(hi2), T.kmax(hi2),
          lcarmin, lcarmax);
    // slots of the write-back two generations ago: free once helper B has read them
    const u32 pq1 = S.pq1;
    if (pq1 != 0) {
      while ((int)(*reinterpret_cast<volatile u32*>(&c->wb_rd) - pq1) < 0) __nanosleep(32);
      fm |= (1u << S.pa1) | (1u << S.pb1);
    }
    S.pa1 = S.pa0; S.pb1 = S.pb0; S.pq1 = S.pq0;
    S.pa0 = hi2; S.pb0 = lcar; S.pq0 = seq;
    S.lag = 0;
  }
  DT_MARK(1)
  // ---- commit: op i (Alg.2 refill path, Alg.3 at the root and at y1)
  if (max2 <= min3) ++d_nomove; else ++d_merge;
  if (maxl <= minr) ++d_nomove; else ++d_merge;
  S.pout = oroot;  // old root: read by phase A's output copy, freed after its bulk read
  fm |= (1u << n2) | (1u << n3) | (1u << nl) | (1u << nr);
  c->ns[1] = lo0;
  c->ns[x1] = hi0;
  if (emit_root) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    bulk_s2g(T.C.out_k + opos, T.BK(lo0), (u32)K * 4u);
    if (V && T.C.out_v) bulk_s2g(T.C.out_v + opos, T.BV(lo0), (u32)K * 4u);
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    c->ns[1] = DT_NONE;
    S.pout = lo0;  // freed once the bulk copy has read it (next plan)
    S.rs = 0;
  } else {
    S.rs = (u32)K;
  }
  const u32 x2 = maxl > maxr ? cl : cr, y2 = maxl > maxr ? cr : cl;
  c->ns[y1] = lo1;
  c->ns[x2] = hi1;
  c->ns[y2] = R;
  S.m1v = 0;
  S.nout += (u32)K;
  S.hs = hs;
  // op i's depth-2 step goes to the next slot
  u32 est = S.est;
  const u32 est_y2 = S.est_y2;
  if (est && !(2u * y2 <= hs && est_y2 == y2)) {  // (not expected: the prediction is exact)
    T.enqueue(RQ_WB, 2u * est_y2, 2u * est_y2 + 1u <= H.cap ? 2u * est_y2 + 1u : 0u, 0u);
    mbar_wait(&c->sbar[S.est_bi], S.est_par);
    if (S.est_lo != DT_NONE)
      while (*reinterpret_cast<volatile u32*>(&c->g2_done) != S.eseq) __nanosleep(32);  // G2's early split
    fm |= (1u << S.est_s0) | (1u << S.est_s1);
    if (S.est_lo != DT_NONE) fm |= (1u << S.est_lo) | (1u << S.est_hi);
    est = 0;
  }
  S.lag_early = 0;
  if (2u * y2 <= hs) {
    S.lag = 1; S.lag_cur = y2;
    if (est) {
      S.lag_bi = S.est_bi; S.lag_par = S.est_par; S.lag_s0 = S.est_s0; S.lag_s1 = S.est_s1;
      S.lag_early = S.est_lo != DT_NONE; S.lag_lo = S.est_lo; S.lag_hi = S.est_hi;
      est = 0;
    } else {
      const u32 c0 = 2u * y2, c1 = c0 + 1u;
      if (fm == 0) __trap();
      const u32 sa = __ffs(fm) - 1; fm &= ~(1u << sa);
      if (fm == 0) __trap();
      const u32 sb = __ffs(fm) - 1; fm &= ~(1u << sb);
      const u32 sbi = S.sbi, sph = S.sph;
      S.lag_s0 = sa; S.lag_s1 = sb;
      S.lag_bi = sbi; S.lag_par = (sph >> sbi) & 1u;
      T.req(S, RQ_STAGE, c0, c1 <= H.cap ? c1 : 0u, sa, sb, sbi);
      S.sph = sph ^ (1u << sbi); S.sbi = sbi ^ 1u;
    }
  }
  S.est = est;
  S.fm = fm;
  S.i = i + 1;
  S.stage = 99;
  // device counters (byte model)
  ull* st = c->st;
  st[S_DEL_OPS] += 1;
  st[S_DEL_REFILL] += 1;
  st[S_DEL_LEVELS] += d_lv;
  st[S_DEL_LR_MERGE] += d_merge;
  st[S_DEL_LR_NOMOVE] += d_nomove;
  st[S_DEL_CY_SWAP] += d_lv;
  DT_MARK(2)
  return true;
}

// Plan of the next slot (thread 0): which operation runs, its refill source, the splits the
// three groups run in phase A, and the helper requests that can be issued ahead (refill node
// of op i+1, depth-3 children of op i).  The state it touches is loaded into registers once
// and written back once (shared-memory round trips serialise single-thread code).
template <int K, bool V>
__device__ __forceinline__ void dt_plan(DTop<K, V>& T, DtS& S, const u64 n_ops, const bool timing) {
  DtCtl* c = T.c;
  const HeapArgs& H = T.H;
  const CallArgs& C = T.C;
  const bool lt = (C.debug & 128u) != 0;
  ull tq = lt ? clock64() : 0;
  const ull twg = timing ? clock64() : 0;
  // output copies (one bulk group per slot, issued by this thread): all but the newest have
  // read their source slot, which is freed now; the newest one's slot is freed next slot
  asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
  if (timing) c->ts[10] += clock64() - twg;
  u32 fm = S.fm;
  if (S.pout_old != DT_NONE) fm |= 1u << S.pout_old;
  S.pout_old = S.pout;
  S.pout = DT_NONE;
  auto alloc = [&]() -> u32 {
    if (fm == 0) __trap();  // slot budget exceeded: a bug, never silent corruption
    const u32 q = __ffs(fm) - 1;
    fm &= ~(1u << q);
    return q;
  };
  const u64 i = S.i;
  const u32 hs = S.hs, rs = S.rs, lag = S.lag, lag_cur = S.lag_cur;
  u32 pre = S.pre;
  const u32 pre_tar = S.pre_tar;
  u32 rbi = S.rbi, rph = S.rph, sbi = S.sbi, sph = S.sph;
  if (C.prog) { C.prog[0] = (u32)i; C.prog[1] = 1; C.prog[4] = hs; C.prog[5] = lag ? (0x80000000u | lag_cur) : 0u; C.prog[6] = pre ? pre_tar : 0u; }
  u32 fl = 0;
  bool new_op = i < n_ops;
  const bool pipelined = pre && pre_tar == hs;
  if (new_op && lag && !pipelined) new_op = false;  // small heap: finish op i-1 first
  if (!new_op && !lag) {
    c->p_flags = DT_NONE;
    S.fm = fm;
    return;
  }
  if (lag) {
    fl |= F_LAG;
    c->p_m[2][0] = S.lag_s0; c->p_m[2][1] = S.lag_s1;
    if (S.lag_early) {  // G2 already split the staged children during the last phase B
      fl |= F_LAGDONE;
      c->p_m[2][2] = S.lag_lo; c->p_m[2][3] = S.lag_hi;
    } else {
      c->p_m[2][2] = alloc(); c->p_m[2][3] = alloc();
    }
    c->p_sbi = S.lag_bi; c->p_spar = S.lag_par;
  }
  u32 rwait = 0, conflict = 0, m1v = 0, y1 = 0;
  if (new_op) {
    fl |= F_NEW;
    const u64 rem = C.n - i * (u64)K;
    const u32 size = (u32)(rem < (u64)K ? rem : (u64)K);
    const u32 path = hs == 0 ? 0u : size < rs ? 1u : hs == 1 ? 2u : 3u;  // EMPTY EXTRACT PBUF REFILL
    S.size = size; S.path = path; S.rs_old = rs;
    c->p_out_slot = c->ns[1];
    c->p_out_n = path == 1 ? size : (path >= 2 ? rs : 0u);
    c->p_iop_lo = (u32)i; c->p_iop_hi = (u32)(i >> 32);
    if (path == 3) {
      const u32 hn = hs - 1u;
      u32 R;
      if (pipelined) {  // Alg.2 l.6-12 done ahead by the helper
        R = S.pre_slot;
        rwait = 1; c->p_rbi = S.pre_bi; c->p_rpar = S.pre_par;
        pre = 0;
      } else if (hs <= 7u) {  // the last node is on chip
        R = c->ns[hs];
        c->ns[hs] = DT_NONE;
      } else {  // synchronous take by the helper
        R = alloc();
        T.req(S, RQ_REFILL, hs, R, rbi);
        rwait = 1; c->p_rbi = rbi; c->p_rpar = (rph >> rbi) & 1u;
        rph ^= 1u << rbi; rbi ^= 1u;
      }
      S.R = R;
      // op i's path and its speculative l/r splits (l.9-10 on cached max keys)
      const bool a2 = 2u <= hn, a3 = 3u <= hn;
      const u32 n2 = c->ns[2], n3 = c->ns[3];
      if (a2 && a3) {
        fl |= F_M0;
        c->p_m[0][0] = n2; c->p_m[0][1] = n3;
        c->p_m[0][2] = alloc(); c->p_m[0][3] = alloc();
        y1 = T.kmax(n2) > T.kmax(n3) ? 3u : 2u;  // R6: tie -> x = r, y = l
      } else if (a2) {
        y1 = 2u;
      }
      DT_MARK(3)
      // (the STAGE for op i's depth-3 children goes first: G2 needs it this slot; the refill
      // node of op i+1 is needed one slot later)
      if (y1) {
        const u32 cl = 2u * y1, cr = cl + 1u;
        const bool al = cl <= hn, ar = cr <= hn;
        const u32 ncl = c->ns[cl], ncr = c->ns[cr];
        conflict = lag && (lag_cur == cl || lag_cur == cr);
        if (al && ar && !conflict) {
          fl |= F_M1;
          m1v = 1;
          const u32 lo = alloc(), hi = alloc();
          S.m1lo = lo; S.m1hi = hi;
          c->p_m[1][0] = ncl; c->p_m[1][1] = ncr;
          c->p_m[1][2] = lo; c->p_m[1][3] = hi;
        }
        if (pipelined && !conflict && (al || ar)) {  // lock + stage op i's depth-3 children now
          const u32 p2 = (al && ar) ? (T.kmax(ncl) > T.kmax(ncr) ? cr : cl) : (al ? cl : cr);
          const u32 c0 = 2u * p2, c1 = c0 + 1u;
          if (c0 <= hn) {
            const bool early = !(C.debug & 256u) && !S.defer;  // (control-warp driver: split in phase A)
            const u32 e0 = alloc(), e1 = alloc();
            const u32 elo = early ? alloc() : DT_NONE, ehi = early ? alloc() : DT_NONE;
            S.est = 1; S.est_y2 = p2; S.est_s0 = e0; S.est_s1 = e1; S.est_lo = elo; S.est_hi = ehi;
            S.est_bi = sbi; S.est_par = (sph >> sbi) & 1u;
            if (early) fl |= F_EARLY;
            const u32 q = S.eseq + 1u;
            S.eseq = q;
            c->p_e[0] = e0; c->p_e[1] = e1; c->p_e[2] = elo; c->p_e[3] = ehi; c->p_e[4] = sbi; c->p_e[5] = S.est_par;
            c->p_e[6] = q;
            T.req(S, RQ_STAGE, c0, c1 <= H.cap ? c1 : 0u, e0, e1, sbi);
            sph ^= 1u << sbi; sbi ^= 1u;
          }
        }
      }
      // take the refill node of op i+1 ahead (deep node, full-K op)
      if (i + 1 < n_ops && C.n - (i + 1) * (u64)K >= (u64)K && hn >= DT_BIG) {
        const u32 ps_ = alloc();
        pre = 1; S.pre_tar = hn; S.pre_slot = ps_;
        S.pre_bi = rbi; S.pre_par = (rph >> rbi) & 1u;
        T.req(S, RQ_REFILL, hn, ps_, rbi);
        rph ^= 1u << rbi; rbi ^= 1u;
      }
      
      DT_MARK(5)
    }
  }
  c->p_rwait = rwait;
  c->p_flags = fl;
  S.fl = fl; S.m1v = m1v; S.conflict = conflict; S.walk = 0; S.walk2 = 0; S.y1 = y1;
  S.pre = pre; S.rbi = rbi; S.rph = rph; S.sbi = sbi; S.sph = sph;
  S.fm = fm;
  DT_MARK(6)
}

// Phase B general path (thread 0): Alg.2/Alg.3 as a state machine; returns when it posted a
// collective job list (merges, copies) for the compute threads or finished the slot.
template <int K, bool V>
__device__ __forceinline__ bool dt_slow(DTop<K, V>& T, DtS& S, const bool timing) {
  DtCtl* c = T.c;
  const HeapArgs& H = T.H;
  bool done = false;
        while (c->njobs == 0 && !done) {
          const u32 st_in = S.stage;
          const ull tsw = timing ? clock64() : 0;
          switch (S.stage) {
            case 0: {  // ---- op i-1's depth-2 step (Alg.3 at cur = y2(i-1)), part 1
              S.stage = 2;
              if (!(S.fl & F_LAG)) break;
              const u32 bi = S.lag_bi, cur = S.lag_cur, c0 = 2u * cur, c1 = c0 + 1u;
              S.lcar = c->ns[cur];
              const bool a0 = c->stg_st[bi][0] == ST_AVAIL, a1 = c->stg_st[bi][1] == ST_AVAIL;
              const u64 inf = (u64)1 << 32;
              const u64 minc = min(a0 ? (u64)c->stg_min[bi][0] : inf, a1 ? (u64)c->stg_min[bi][1] : inf);
              const u32 lo = c->p_m[2][2], hi = c->p_m[2][3];
              if ((u64)T.kmax(S.lcar) <= minc) {  // l.4: stop, l.7: UNLOCK(l), UNLOCK(r)
                T.enqueue(RQ_WB, c0, c1 <= H.cap ? c1 : 0u, 0u);
                T.release_slot(S, lo); T.release_slot(S, hi);
                T.release_slot(S, S.lag_s0); T.release_slot(S, S.lag_s1);
                S.lag = false;
                break;
              }
              c->st[S_DEL_LEVELS]++;
              u32 Y;
              S.lX = DT_NONE;
              if (a0 && a1) {  // l.9-10
                const u32 mx0 = c->stg_max[bi][0], mx1 = c->stg_max[bi][1];
                if (mx0 > mx1) { S.lx = c0; S.ly = c1; } else { S.lx = c1; S.ly = c0; }
                c->st[(mx0 <= c->stg_min[bi][1]) ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
                Y = lo; S.lX = hi;
                T.release_slot(S, S.lag_s0); T.release_slot(S, S.lag_s1);
              } else {  // exactly one AVAIL child (R5): y = it, no l/r split
                S.ly = a0 ? c0 : c1;
                S.lx = a0 ? c1 : c0;
                if (S.lx > H.cap) S.lx = 0;
                Y = a0 ? S.lag_s0 : S.lag_s1;
                T.release_slot(S, a0 ? S.lag_s1 : S.lag_s0);
                T.release_slot(S, lo); T.release_slot(S, hi);
                c->st[S_DEL_LR_SKIP]++;
              }
              if (T.kmax(Y) <= T.kmin(S.lcar)) {  // l.12 as a swap
                S.lcf = Y; S.lcar3 = S.lcar;
                c->st[S_DEL_CY_SWAP]++;
              } else {
                S.lcf = T.alloc(S); S.lcar3 = T.alloc(S);
                T.job(J_MERGE, S.lcar, K, Y, K, K, S.lcf, S.lcar3);
                S.mfa = S.lcar; S.mfb = Y;
              }
              S.stage = 1;
              break;
            }
            case 1: {  // ---- part 2: write-backs are posted with the last round of the slot
              T.release_slot(S, S.mfa); T.release_slot(S, S.mfb);
              S.mfa = S.mfb = DT_NONE;
              c->ns[S.lag_cur] = S.lcf;
              // x3 (l.10) and y3 with its carried keys (l.12) go back to HBM; a walker continues at y3
              T.writeback(S, S.lx, S.lX, S.ly, S.lcar3, 2u * S.ly <= S.hs);
              S.lag = false;
              S.stage = 2;
              break;
            }
            case 2: {  // ---- deferred depth-1 split (y1(i) == y1(i-1)), on the updated nodes
              S.stage = 3;
              if (!(S.fl & F_NEW) || S.path != 3 || !S.conflict) break;
              const u32 cl = 2u * S.y1, cr = cl + 1u, hn = S.hs - 1u;
              if (cl <= hn && cr <= hn) {
                S.m1v = true;
                S.m1lo = T.alloc(S); S.m1hi = T.alloc(S);
                T.job(J_MERGE, c->ns[cl], K, c->ns[cr], K, K, S.m1lo, S.m1hi);
              }
              break;
            }
            case 3: {  // ---- op i's root section (Alg.2 PARTIAL_DELETEMIN)
              if (!(S.fl & F_NEW)) { S.stage = 9; break; }
              c->st[S_DEL_OPS]++;
              const u64 pos = S.i * (u64)K;
              if (S.path == 0) {  // l.16-17
                S.stage = 9;
              } else if (S.path == 1) {  // l.18-20: EXTRACT_ROOT(items, size)
                S.tsl = T.alloc(S);
                T.job(J_SHIFT, S.tsl, c->ns[1], S.size, S.rs - S.size);
                S.nout += S.size;
                S.stage = 30;
              } else if (S.path == 2) {  // l.23-29: root <- sorted pBuffer (R1), heapSize stays 1
                const u32 take = min(S.rs + S.ps, S.size) - S.rs;
                S.nout += S.rs + take;
                S.tsl = DT_NONE;
                if (S.ps > 0) {
                  S.tsl = T.alloc(S);
                  if (take) T.job(J_OUT, c->ns[0], 0, take, (u32)(pos + S.rs), (u32)((pos + S.rs) >> 32));
                  T.job(J_SHIFT, S.tsl, c->ns[0], take, S.ps - take);
                }
                S.take_sv = take;
                S.stage = 31;
              } else {  // l.4-13: refill from the last node, then the pBuffer split
                c->st[S_DEL_REFILL]++;
                S.remained = S.size - S.rs;
                S.nout += S.size;
                S.hs -= 1u;
                asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                T.release_slot(S, c->ns[1]);  // the old root, output in phase A
                c->ns[1] = DT_NONE;
                S.mfa = S.mfb = DT_NONE;
                if (S.ps > 0 && T.kmax(S.R) > T.kmin(c->ns[0])) {
                  const u32 a = T.alloc(S), b = T.alloc(S);
                  T.job(J_MERGE, S.R, K, c->ns[0], S.ps, K, a, b);
                  S.mfa = S.R; S.mfb = c->ns[0];
                  S.R = a; c->ns[0] = b;
                }
                S.stage = 4;
              }
              break;
            }
            case 30: {
              asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // phase A output read it
              T.release_slot(S, c->ns[1]);
              c->ns[1] = S.tsl;
              S.rs -= S.size;
              S.stage = 9;
              break;
            }
            case 31: {
              const u32 take = S.take_sv;
              asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // phase A output read it
              T.release_slot(S, c->ns[1]);
              T.release_slot(S, c->ns[0]);
              c->ns[0] = DT_NONE;
              S.rs = S.ps - take;
              S.ps = 0;
              c->ns[1] = S.tsl;
              if (S.rs == 0) { T.release_slot(S, S.tsl); c->ns[1] = DT_NONE; }
              S.stage = 9;
              break;
            }
            case 4: {  // ---- Alg.3 at cur = root (children 2, 3 on chip)
              T.release_slot(S, S.mfa); T.release_slot(S, S.mfb);
              S.mfa = S.mfb = DT_NONE;
              const bool a2 = 2u <= S.hs, a3 = 3u <= S.hs;
              const u64 inf = (u64)1 << 32;
              const u64 minc = min(a2 ? (u64)T.kmin(c->ns[2]) : inf, a3 ? (u64)T.kmin(c->ns[3]) : inf);
              S.stage = 5;
              if ((u64)T.kmax(S.R) <= minc) {  // l.4
                c->ns[1] = S.R;
                if (S.fl & F_M0) { T.release_slot(S, c->p_m[0][2]); T.release_slot(S, c->p_m[0][3]); }
                break;
              }
              c->st[S_DEL_LEVELS]++;
              u32 Y;
              if (a2 && a3) {
                const u32 x1 = S.y1 ^ 1u;
                c->st[(T.kmax(c->ns[2]) <= T.kmin(c->ns[3])) ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
                T.release_slot(S, c->ns[2]); T.release_slot(S, c->ns[3]);
                c->ns[x1] = c->p_m[0][3];
                c->ns[S.y1] = DT_NONE;
                Y = c->p_m[0][2];
              } else {
                c->st[S_DEL_LR_SKIP]++;
                Y = c->ns[S.y1];
              }
              if (T.kmax(Y) <= T.kmin(S.R)) {  // l.12 as a swap
                c->ns[1] = Y; S.car1 = S.R;
                c->st[S_DEL_CY_SWAP]++;
              } else {
                const u32 a = T.alloc(S), b = T.alloc(S);
                T.job(J_MERGE, S.R, K, Y, K, K, a, b);
                c->ns[1] = a; S.car1 = b;
                S.mfa = S.R; S.mfb = Y;
              }
              S.walk = true;
              break;
            }
            case 5: {  // ---- EXTRACT_ROOT(items, remainedSize) (Alg.3 with cur == root)
              T.release_slot(S, S.mfa); T.release_slot(S, S.mfb);
              S.mfa = S.mfb = DT_NONE;
              S.tsl = DT_NONE;
              if (S.remained) {
                const u64 pos = S.i * (u64)K + S.rs_old;
                S.tsl = T.alloc(S);
                T.job(J_OUT, c->ns[1], 0, S.remained, (u32)pos, (u32)(pos >> 32));
                T.job(J_SHIFT, S.tsl, c->ns[1], S.remained, K - S.remained);
              }
              S.stage = 6;
              break;
            }
            case 6: {  // ---- Alg.3 at cur = y1 (children at depth 2, on chip)
              if (S.tsl != DT_NONE) { T.release_slot(S, c->ns[1]); c->ns[1] = S.tsl; S.tsl = DT_NONE; }
              S.rs = K - S.remained;
              if (S.rs == 0) { T.release_slot(S, c->ns[1]); c->ns[1] = DT_NONE; }
              S.stage = 7;
              if (!S.walk) {
                if (S.m1v) { T.release_slot(S, S.m1lo); T.release_slot(S, S.m1hi); S.m1v = false; }
                break;
              }
              const u32 cl = 2u * S.y1, cr = cl + 1u;
              const bool al = cl <= S.hs, ar = cr <= S.hs;
              const u64 inf = (u64)1 << 32;
              const u64 minc = min(al ? (u64)T.kmin(c->ns[cl]) : inf, ar ? (u64)T.kmin(c->ns[cr]) : inf);
              if ((u64)T.kmax(S.car1) <= minc) {  // l.4
                c->ns[S.y1] = S.car1;
                if (S.m1v) { T.release_slot(S, S.m1lo); T.release_slot(S, S.m1hi); S.m1v = false; }
                break;
              }
              c->st[S_DEL_LEVELS]++;
              u32 Y;
              if (al && ar) {
                const u32 mxl = T.kmax(c->ns[cl]), mxr = T.kmax(c->ns[cr]);
                const u32 x2 = mxl > mxr ? cl : cr;
                S.y2 = mxl > mxr ? cr : cl;
                c->st[(mxl <= T.kmin(c->ns[cr])) ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
                T.release_slot(S, c->ns[cl]); T.release_slot(S, c->ns[cr]);
                c->ns[x2] = S.m1hi;
                c->ns[S.y2] = DT_NONE;
                Y = S.m1lo;
                S.m1v = false;
              } else {
                c->st[S_DEL_LR_SKIP]++;
                S.y2 = al ? cl : cr;
                Y = c->ns[S.y2];
              }
              if (T.kmax(Y) <= T.kmin(S.car1)) {  // l.12 as a swap
                c->ns[S.y1] = Y; c->ns[S.y2] = S.car1;
                c->st[S_DEL_CY_SWAP]++;
              } else {
                const u32 a = T.alloc(S), b = T.alloc(S);
                T.job(J_MERGE, S.car1, K, Y, K, K, a, b);
                c->ns[S.y1] = a; c->ns[S.y2] = b;
                S.mfa = S.car1; S.mfb = Y;
              }
              S.walk2 = 2u * S.y2 <= S.hs;
              break;
            }
            case 7: {  // ---- op i's depth-2 step goes to the next slot
              T.release_slot(S, S.mfa); T.release_slot(S, S.mfb);
              S.mfa = S.mfb = DT_NONE;
              S.stage = 8;  // (op i-1's write-back request precedes any new STAGE in the FIFO)
              break;
            }
            case 8: {
              S.lag_early = 0;
              if (S.walk2) {
                S.lag = true; S.lag_cur = S.y2;
                const u32 c0 = 2u * S.y2, c1 = c0 + 1u;
                if (S.est && S.est_y2 == S.y2) {
                  S.lag_bi = S.est_bi; S.lag_par = S.est_par; S.lag_s0 = S.est_s0; S.lag_s1 = S.est_s1;
                  S.lag_early = S.est_lo != DT_NONE; S.lag_lo = S.est_lo; S.lag_hi = S.est_hi;
                  S.est = false;
                } else {
                  S.lag_s0 = T.alloc(S); S.lag_s1 = T.alloc(S);
                  S.lag_bi = S.sbi; S.lag_par = (S.sph >> S.sbi) & 1u;
                  T.enqueue(RQ_STAGE, c0, c1 <= H.cap ? c1 : 0u, S.lag_s0, S.lag_s1, S.sbi);
                  S.sph ^= 1u << S.sbi; S.sbi ^= 1u;
                }
              }
              S.stage = 9;
              break;
            }
            default: {  // 9: end of the slot; the lag step's write-backs ride on this round
              if (S.est) {  // the walk stopped above depth 2: UNLOCK the staged children
                T.enqueue(RQ_WB, 2u * S.est_y2, 2u * S.est_y2 + 1u <= H.cap ? 2u * S.est_y2 + 1u : 0u, 0u);
                mbar_wait(&c->sbar[S.est_bi], S.est_par);  // the staging TMA must land before reuse
                if (S.est_lo != DT_NONE)
                  while (*reinterpret_cast<volatile u32*>(&c->g2_done) != S.eseq) __nanosleep(32);  // and G2's split
                T.release_slot(S, S.est_s0); T.release_slot(S, S.est_s1);
                T.release_slot(S, S.est_lo); T.release_slot(S, S.est_hi);
                S.est = false;
              }
              if (S.fl & F_NEW) ++S.i;
              done = true;
              break;
            }
          }
          if (timing) c->ts[st_in >= 30 ? 8 : (st_in > 8 ? 8 : st_in)] += clock64() - tsw;
        }
  return done;
}

template <int K, bool V>
__device__ __forceinline__ void dt_top(DTop<K, V>& T) {
  DtCtl* c = T.c;
  const HeapArgs& H = T.H;
  const CallArgs& C = T.C;
  const int tid = threadIdx.x;
  const int g = tid / DT_GT, gt = tid % DT_GT;
  const u64 n_ops = C.n_ops;
  constexpr u32 NBY = K * 4u;
  // ---- thread-0 state lives in shared memory (DtS): the helper warp's gpu-scope acquires
  // invalidate L1, so registers spilled to local memory would cost an L2 round trip each
  DtS& SS = c->s;
  if (tid == 0) { SS.init(); SS.fm = (1u << DT_NSLOT) - 1u; }
  // ---- call start: stage the on-chip part (pBuffer, root, nodes 2..7)
  if (tid == 0) {
    DtS* __restrict__ const Sp = &SS;
    DtS& S = *Sp;
    S.hs = ld_relaxed(H.hdr + H_HS);
    S.rs = ld_relaxed(H.hdr + H_RS);
    S.ps = ld_relaxed(H.hdr + H_PS);
    u32 bytes = 0;
    for (u32 q = 0; q < 8; ++q) {
      const bool have = q == 0 ? S.ps > 0 : (q == 1 ? (S.hs >= 1 && S.rs > 0) : q <= S.hs);
      c->ns[q] = have ? T.alloc(S) : DT_NONE;
      if (have) bytes += V ? 2u * NBY : NBY;
    }
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->lbar, bytes);
    for (u32 q = 0; q < 8; ++q) {
      if (c->ns[q] == DT_NONE) continue;
      bulk_g2s(T.BK(c->ns[q]), H.gk + (size_t)q * K, NBY, &c->lbar);
      if (V) bulk_g2s(T.BV(c->ns[q]), H.gv + (size_t)q * K, NBY, &c->lbar);
    }
    (void)0;
  }
  mbar_wait(&c->lbar, 0);
  cta_bar<DT_NTC>();

  const bool timing = (C.debug & 8u) != 0;
  const bool ltime = timing || (C.debug & 128u) != 0;  // light timing: plan / phase A / phase B only
  const bool mwin = (C.debug & 64u) != 0;
  // the first plan; every later one is made by thread 0 at the end of the previous slot's
  // phase B, so a common slot has two CTA barriers (after phase A, after phase B)
  if (tid == 0 && ltime) SS.tmark = clock64();
  if (tid == 0) dt_plan<K, V>(T, SS, n_ops, timing);
  cta_bar<DT_NTC>();
  for (;;) {
    const u32 pf = c->p_flags;
    if (pf == DT_NONE) break;
    // plan words used after phase A: read now (thread 0 rewrites them during phase B)
    const u32 w_sbi = c->p_sbi, w_spar = c->p_spar, w_rwait = c->p_rwait, w_rbi = c->p_rbi, w_rpar = c->p_rpar;
    if (tid == 0 && C.prog) C.prog[1] = 2;
    if (tid == 0 && ltime) { const ull t = clock64(); c->tm[0] += t - SS.tmark; SS.tmark = t; c->tm[5]++; if (SS.conflict) c->tm[6]++; }

    // =========================== phase A: concurrent work ===========================
    const ull tg0 = (timing && gt == 0) ? clock64() : 0;
    if (g == 0) {
      if (pf & F_NEW) {  // Alg.2 l.18-22: the old root keys are the first output of op i
        const u32 n = c->p_out_n;
        const u64 pos0 = (((u64)c->p_iop_hi << 32) | c->p_iop_lo) * (u64)K;
        const bool bulk = (n & 3u) == 0 && ((reinterpret_cast<uintptr_t>(C.out_k + pos0) & 15u) == 0) &&
                          (!V || !C.out_v || (reinterpret_cast<uintptr_t>(C.out_v + pos0) & 15u) == 0);
        if (n && bulk) {  // one TMA bulk store (async proxy); its smem read is awaited before the slot is reused
          if (gt == 0) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            bulk_s2g(C.out_k + pos0, T.BK(c->p_out_slot), n * 4u);
            if (V && C.out_v) bulk_s2g(C.out_v + pos0, T.BV(c->p_out_slot), n * 4u);
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
        } else if (n) {
          const u64 pos = (((u64)c->p_iop_hi << 32) | c->p_iop_lo) * (u64)K;
          const u32* s = T.BK(c->p_out_slot);
          if ((n & 3u) == 0) {
            uint4* d4 = reinterpret_cast<uint4*>(C.out_k + pos);
            for (u32 q = gt; q < n / 4; q += DT_GT) d4[q] = reinterpret_cast<const uint4*>(s)[q];
          } else {
            for (u32 q = gt; q < n; q += DT_GT) C.out_k[pos + q] = s[q];
          }
          if (V && C.out_v) {
            const u32* v = T.BV(c->p_out_slot);
            for (u32 q = gt; q < n; q += DT_GT) C.out_v[pos + q] = v[q];
          }
        }
      }
      if (pf & F_M0) {
        const u32* m = c->p_m[0];
        grp_split<K, V>(gt, T.BK(m[0]), T.BV(m[0]), K, T.BK(m[1]), T.BV(m[1]), K, K, T.BK(m[2]), T.BV(m[2]),
                        T.BK(m[3]), T.BV(m[3]), mwin);
      }
    } else if (g == 1) {
      if (pf & F_M1) {
        const u32* m = c->p_m[1];
        grp_split<K, V>(gt, T.BK(m[0]), T.BV(m[0]), K, T.BK(m[1]), T.BV(m[1]), K, K, T.BK(m[2]), T.BV(m[2]),
                        T.BK(m[3]), T.BV(m[3]), mwin);
      }
    } else {
      if ((pf & F_LAG) && !(pf & F_LAGDONE)) {
        const u32 bi = c->p_sbi;
        const ull tw = (timing && gt == 0) ? clock64() : 0;
        mbar_wait(&c->sbar[bi], c->p_spar);
        if (timing && gt == 0) c->tm[2] += clock64() - tw;
        if (c->stg_st[bi][0] == ST_AVAIL && c->stg_st[bi][1] == ST_AVAIL) {
          const u32* m = c->p_m[2];
          grp_split<K, V>(gt, T.BK(m[0]), T.BV(m[0]), K, T.BK(m[1]), T.BV(m[1]), K, K, T.BK(m[2]), T.BV(m[2]),
                          T.BK(m[3]), T.BV(m[3]), mwin);
        }
      }
    }
    if (timing && gt == 0) c->tm[8 + g] += clock64() - tg0;
    // G2's early split of op i's staged depth-3 children (runs during phase B); its plan words
    // are read before the barrier, after which thread 0 may plan the next slot
    u32 e0 = 0, e1 = 0, elo = 0, ehi = 0, ebi = 0, epar = 0, eq = 0;
    if (g == 2 && (pf & F_EARLY)) {
      e0 = c->p_e[0]; e1 = c->p_e[1]; elo = c->p_e[2]; ehi = c->p_e[3]; ebi = c->p_e[4]; epar = c->p_e[5]; eq = c->p_e[6];
    }
    cta_bar<DT_NTC>();
    if (tid == 0 && ltime) { const ull t = clock64(); c->tm[1] += t - SS.tmark; SS.tmark = t; }
    // every thread observes the TMA data phase B may read
    const ull tw7 = (tid == 0 && ltime) ? clock64() : 0;
    if (pf & F_LAG) mbar_wait(&c->sbar[w_sbi], w_spar);
    if (w_rwait) mbar_wait(&c->rbar[w_rbi], w_rpar);
    if (tid == 0 && ltime) c->ts[7] += clock64() - tw7;
    if (g == 2 && (pf & F_EARLY)) {
      mbar_wait(&c->sbar[ebi], epar);
      if (c->stg_st[ebi][0] == ST_AVAIL && c->stg_st[ebi][1] == ST_AVAIL)
        grp_split<K, V>(gt, T.BK(e0), T.BV(e0), K, T.BK(e1), T.BV(e1), K, K, T.BK(elo), T.BV(elo), T.BK(ehi),
                        T.BV(ehi), mwin);
      grp_bar(2);
      if (gt == 0) st_rel_cta(&c->g2_done, eq);
    }
    if (tid == 0 && timing) { const ull t = clock64(); c->tm[3] += t - SS.tmark; SS.tmark = t; }

    // =========================== phase B: decisions + job rounds ===========================
    if (tid == 0) SS.stage = 0;
    for (;;) {
      if (tid == 0) {
        DtS* __restrict__ const Sp = &SS;
        DtS& S = *Sp;
        c->njobs = 0;
        bool done = false;
        if (S.stage == 0) done = dt_fast<K, V>(T, S);  // the common slot, straight-line
        if (!done) done = dt_slow<K, V>(T, S, timing);
        if (done) {  // the slot is complete: plan the next one now
          if (ltime) { const ull t = clock64(); c->tm[4] += t - SS.tmark; SS.tmark = t; }
          dt_plan<K, V>(T, SS, n_ops, timing);
        }
        c->more = done ? 0u : 1u;
        if (C.prog) C.prog[1] = 100 + S.stage;
        (void)0;
      }
      if (tid == 0 && timing) c->tm[11]++;
      const ull trd = (tid == 0 && timing) ? clock64() : 0;
      cta_bar<DT_NTC>();
      T.run_jobs();
      const u32 more = c->more;
      if (!more) break;  // no job list follows: thread 0 writes none before the next phase A
      cta_bar<DT_NTC>();
      if (tid == 0 && timing) c->ts[11] += clock64() - trd;
    }
  }

  // =========================== call end: write the on-chip part back ===========================
  if (tid == 0) {
    DtS* __restrict__ const Sp = &SS;
    DtS& S = *Sp;
    c->njobs = 0;
    for (u32 q = 0; q < 8; ++q) {
      const u32 s = c->ns[q];
      if (q >= 1) st_relaxed(T.stp(q), q <= S.hs ? ST_AVAIL : ST_EMPTY);
      if (s == DT_NONE) continue;
      const u32 cnt = q == 0 ? S.ps : (q == 1 ? S.rs : K);
      if (q > S.hs || cnt == 0) continue;
      st_relaxed(&H.meta[q].kmin, T.BK(s)[0]);
      st_relaxed(&H.meta[q].kmax, T.BK(s)[cnt - 1]);
      T.job(J_STORE, q, s);
    }
    (void)0;
  }
  cta_bar<DT_NTC>();
  T.run_jobs();
  cta_bar<DT_NTC>();
  if (tid == 0) {
    DtS* __restrict__ const Sp = &SS;
    DtS& S = *Sp;
    st_relaxed(H.hdr + H_HS, S.hs);
    st_relaxed(H.hdr + H_RS, S.rs);
    st_relaxed(H.hdr + H_PS, S.ps);
    ull lin;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(lin) : "l"(H.hdr + H_LIN) : "memory");
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(lin + n_ops) : "memory");
    c->st[S_KEYS_OUT] += S.nout;
    if (C.d_count && S.nout) atomicAdd(C.d_count, (ull)S.nout);
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    T.enqueue(RQ_END);                     // ring 1 (helper B publishes the final task count)
    T.enqueue(RQ_STAGE, 0u, 0u, 0u, 0u, DT_NONE);  // ring 0 end marker
    while (ld_acq_cta(&c->rq_done[0]) != c->rq_head[0] || ld_acq_cta(&c->rq_done[1]) != c->rq_head[1]) {}
    ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
    for (int q = 0; q < NSTAT; ++q)
      if (c->st[q]) atomicAdd(stat + q, c->st[q]);
    if (ltime) {
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      for (int q = 0; q < 12; ++q) { atomicAdd(tms + 16 + q, c->tm[q]); atomicAdd(tms + q, c->ts[q]); }
    }
    (void)0;
  }
}

// =========================================================================================
// Walkers: Alg.3 from l.2 at a depth-3 node handed over by the top CTA (locked, carried
// keys stored in the node), with OpL's lock-ahead agents (bgpq_locks.cuh).
// =========================================================================================
template <int K, bool V, int NT>
__device__ void dt_walk(OpL<K, V, NT>& op, u32 cur, const u64* go, u32 epoch, ull* wtm = nullptr) {
  ull t_go = 0;
  bool first = true;
  const int tid = threadIdx.x;
  LCtl* ctl = op.ctl;
  if (tid == 0) {
    const u32 l = 2u * cur, r = l + 1u;
    const u32 n0 = l <= op.H.cap ? l : 0u, n1 = r <= op.H.cap ? r : 0u;
    const int s0 = op.alloc(), s1 = op.alloc();
    op.post_p(n0, n1, s0, s1, 0u);  // LOCK + stage the children while the hand-over completes
    ctl->b[8] = (u32)s0; ctl->b[9] = (u32)s1;
    ctl->b[10] = (u32)op.alloc();
    // the task may have been published before its carried keys were final: wait for them
    u64 g;
    u32 ns = 32;
    for (;;) {
      asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(g) : "l"(go) : "memory");
      if ((u32)(g >> 32) == epoch) break;
      __nanosleep(ns);
      ns = ns < 256 ? ns * 2 : 256;
    }
    ctl->b[11] = (u32)g;
    if (wtm) t_go = clock64();
  }
  cta_bar<NT>();
  int R = (int)ctl->b[10];
  int SL = (int)ctl->b[8], SRr = (int)ctl->b[9];
  const u32 src = ctl->b[11];
  if (src == 0xFFFFFFFFu) {  // cancelled: the walk stopped above this node — release the children
    op.wait_p(LT_DEL_PWAIT);
    if (tid == 0) {
      const u32 l = 2u * cur, r = l + 1u;
      if (l <= op.H.cap) lock_release(op.lk(l));
      if (r <= op.H.cap) lock_release(op.lk(r));
      op.free_slot(SL); op.free_slot(SRr); op.free_slot(R);
    }
    cta_bar<NT>();
    return;
  }
  op.load(R, src);  // the carried keys (in cur's HBM copy, or in the refill node they came from)
  for (;;) {
    const u32 l = 2u * cur, r = l + 1u;
    op.wait_p(LT_DEL_PWAIT);  // l.3: LOCK(l); LOCK(r), children staged
    if (tid == 0) {
      const u32 le = l <= op.H.cap, re = r <= op.H.cap;
      const u32 al = le && ctl->p_st[0] == ST_AVAIL;
      const u32 ar = re && ctl->p_st[1] == ST_AVAIL;
      const u32 lmin = ctl->p_min[0], lmax = ctl->p_max[0], rmin = ctl->p_min[1], rmax = ctl->p_max[1];
      const u64 minc = min(al ? (u64)lmin : (u64)1 << 32, ar ? (u64)rmin : (u64)1 << 32);
      const u32 maxcur = op.BK(R)[K - 1];
      const u32 stop = (u64)maxcur <= minc;  // l.4
      u32 x = 0, y = 0, lr = 0;
      if (!stop) {
        if (al && ar) {
          if (lmax > rmax) { x = l; y = r; } else { x = r; y = l; }  // l.9 (R6)
          lr = (lmax <= rmin) ? 1u : ((rmax <= lmin && x == l) ? 1u : 2u);
          op.st[lr == 1 ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
        } else {
          y = al ? l : r;
          x = al ? r : l;
          lr = 0;
          op.st[S_DEL_LR_SKIP]++;
        }
        op.st[S_DEL_LEVELS]++;
        const u32 yl = 2u * y, yr = yl + 1u;
        const u32 n0 = yl <= op.H.cap ? yl : 0u, n1 = yr <= op.H.cap ? yr : 0u;
        int s0 = -1, s1 = -1;
        if (n0 || n1) {
          s0 = op.alloc(); s1 = op.alloc();
          op.post_p(n0, n1, s0, s1, 0u);
        }
        ctl->b[8] = (u32)s0; ctl->b[9] = (u32)s1;
        ctl->b[13] = (n0 || n1) ? 1u : 0u;
        if (lr == 2) { ctl->b[10] = op.alloc(); ctl->b[11] = op.alloc(); }
      }
      ctl->b[0] = stop; ctl->b[1] = x; ctl->b[2] = y; ctl->b[3] = lr;
      ctl->b[4] = le; ctl->b[5] = re;
    }
    cta_bar<NT>();
    const u32 stop = ctl->b[0], x = ctl->b[1], y = ctl->b[2], lr = ctl->b[3];
    const u32 le = ctl->b[4], re = ctl->b[5];
    if (stop) {  // l.4-8: cur keeps its keys
      op.store(cur, R);
      if (tid == 0) {
        if (le) lock_release(op.lk(l));
        if (re) lock_release(op.lk(r));
        op.free_slot(SL); op.free_slot(SRr);
        op.set_minmax(cur, op.BK(R)[0], op.BK(R)[K - 1]);
        op.free_slot(R);
        op.release_locks(cur);
      }
      break;
    }
    const int nSL = (int)ctl->b[8], nSRr = (int)ctl->b[9];
    const u32 more = ctl->b[13];
    int Y;
    if (lr == 2) {  // l.10
      const int a = (int)ctl->b[10], b = (int)ctl->b[11];
      op.merge_split(SL, K, SRr, K, K, a, b);
      op.store(x, b);
      if (tid == 0) {
        op.set_minmax(x, op.BK(b)[0], op.BK(b)[K - 1]);
        ctl->b[16] = x;
        op.free_slot(b); op.free_slot(SL); op.free_slot(SRr);
      }
      Y = a;
    } else {
      Y = (y == l) ? SL : SRr;
      if (tid == 0) {
        ctl->b[16] = (x == l ? le : re) ? x : 0u;
        op.free_slot(y == l ? SRr : SL);
      }
    }
    // l.12
    int C2, Y2;
    if (op.BK(Y)[K - 1] <= op.BK(R)[0]) {
      C2 = Y; Y2 = R;
      if (tid == 0) op.st[S_DEL_CY_SWAP]++;
    } else {
      cta_bar<NT>();
      if (tid == 0) { ctl->b[14] = op.alloc(); ctl->b[15] = op.alloc(); }
      cta_bar<NT>();
      const int a = (int)ctl->b[14], b = (int)ctl->b[15];
      op.merge_split(R, K, Y, K, K, a, b);
      if (tid == 0) { op.free_slot(R); op.free_slot(Y); }
      C2 = a; Y2 = b;
    }
    op.store(cur, C2);
    if (tid == 0) {
      op.set_minmax(cur, op.BK(C2)[0], op.BK(C2)[K - 1]);
      op.free_slot(C2);
      op.release_locks(cur, ctl->b[16]);  // l.14 (and l.11)
      if (wtm && first) { wtm[0] += clock64() - t_go; wtm[1] += 1; first = false; }
    }
    cur = y;  // l.15
    R = Y2;
    if (!more) {
      cta_bar<NT>();
      op.store(cur, R);
      if (tid == 0) {
        op.set_minmax(cur, op.BK(R)[0], op.BK(R)[K - 1]);
        op.free_slot(R);
        lock_release(op.lk(cur));
      }
      break;
    }
    SL = nSL;
    SRr = nSRr;
  }
}

// Walker CTAs: take tasks (a depth-3 node handed over locked + the node holding its carried
// keys) by ticket and run Alg.3 from l.2 below it (dt_walk), until the final count is published.
template <int K, bool V, int NT>
__device__ __forceinline__ void dt_walkers(const HeapArgs& H, const CallArgs& C, const DtArgs& D,
                                           unsigned char* smem_raw) {
  LCtl* ctl = reinterpret_cast<LCtl*>(smem_raw);
  OpL<K, V, NT> op;
  op.H = H;
  op.ctl = ctl;
  op.sk = reinterpret_cast<u32*>(smem_raw + LCTL_BYTES);
  op.sv = op.sk + LSLOT * K;
  op.mphase = 0; op.pph = 0; op.tphase = 0; op.pb = 0;
  op.st = ctl->st;
  op.tm = ctl->tm;
  op.timing = false;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NSTAT; ++i) ctl->st[i] = 0;
    ctl->tm[28] = 0; ctl->tm[29] = 0;
    mbar_init(&ctl->bar, 1);
    mbar_init(&ctl->pbar[0], 1);
    mbar_init(&ctl->pbar[1], 1);
    mbar_init(&ctl->tbar, 1);
    ctl->freemask = (1u << LSLOT) - 1u;
    ctl->p_req = 0; ctl->t_req = 0; ctl->t_done = 0; ctl->stop = 0; ctl->t_marked = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x >= NT) {
    if (threadIdx.x < NT + 32) lock_warp<K, V, NT>(op);
    return;
  }
  for (;;) {
    if (threadIdx.x == 0) {
      const u32 t = atomicAdd(D.ctl, 1u);
      u32 node = 0, ns = 32, k = 0;
      for (;;) {
        if (ld_acquire(D.task_seq + t) == D.epoch) {
          node = ld_relaxed(D.task_node + t);
          break;
        }
        if ((++k & 7u) == 0) {
          const u32 fin = ld_acquire(D.ctl + 1);
          if (fin && t + 1u >= fin) break;
        }
        __nanosleep(ns);
        ns = ns < 512 ? ns * 2 : 512;
      }
      ctl->b[0] = node;
      ctl->b[1] = t;
    }
    cta_bar<NT>();
    const u32 node = ctl->b[0], tk = ctl->b[1];
    cta_bar<NT>();
    if (threadIdx.x == 0 && C.prog && blockIdx.x < 500) C.prog[16 + 2 * blockIdx.x] = node;
    if (!node) break;
    dt_walk<K, V, NT>(op, node, D.task_go + tk, D.epoch, (C.debug & 1024u) ? &ctl->tm[28] : nullptr);
  }
  if (threadIdx.x == 0) {
    st_rel_cta(&ctl->stop, 1u);
    ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
    for (int i = 0; i < NSTAT; ++i)
      if (op.st[i]) atomicAdd(stat + i, op.st[i]);
    if (C.debug & 1024u) {  // walker first-level hold time (go -> release of the start node)
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      atomicAdd(tms + 30, ctl->tm[28]);
      atomicAdd(tms + 31, ctl->tm[29]);
    }
  }
}

template <int K, bool V>
__global__ void __launch_bounds__(DT_BLOCK, 1) bgpq_dtop_kernel(HeapArgs H, CallArgs C, DtArgs D) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  if (D.op_base) {  // the cluster engine executed the first ops of the call: continue after them
    const u64 b = *reinterpret_cast<volatile const u64*>(D.op_base);
    C.n -= b * (u64)K;
    C.n_ops -= b;
    C.out_k += b * (u64)K;
    if (C.out_v) C.out_v += b * (u64)K;
  }
  if (blockIdx.x == 0) {
    DtCtl* c = reinterpret_cast<DtCtl*>(smem_raw);
    DTop<K, V> T;
    T.H = H; T.C = C; T.D = D; T.c = c;
    T.sk = reinterpret_cast<u32*>(smem_raw + DTCTL_BYTES);
    T.sv = T.sk + DT_NSLOT * K;
    if (threadIdx.x == 0) {
      for (int q = 0; q < NSTAT; ++q) c->st[q] = 0;
      for (int q = 0; q < 12; ++q) { c->tm[q] = 0; c->ts[q] = 0; }
      mbar_init(&c->sbar[0], 1); mbar_init(&c->sbar[1], 1);
      mbar_init(&c->rbar[0], 1); mbar_init(&c->rbar[1], 1);
      mbar_init(&c->lbar, 1);
      c->rq_head[0] = c->rq_head[1] = 0; c->rq_done[0] = c->rq_done[1] = 0; c->tasks = 0; c->g2_done = 0;
      for (int q = 0; q < 2 * (int)DT_RQ; ++q) mbar_init(&c->qbar[q / DT_RQ][q % DT_RQ], 1); c->njobs = 0; c->wb_rd = 0;
      c->freemask = (1u << DT_NSLOT) - 1u;
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x >= DT_NTC + 32) {
      if (threadIdx.x == DT_NTC + 32) dt_helper<K, V>(T, 0u);
      if (threadIdx.x == DT_NTC + 64) dt_helper<K, V>(T, 1u);
      return;
    }
    if (threadIdx.x >= DT_NTC) return;  // control warp: idle
    dt_top<K, V>(T);
    return;
  }
  dt_walkers<K, V, DT_NTC>(H, C, D, smem_raw);
}

}  // namespace bgpqd
