// bgpq_dsys.cuh — DELETEMIN calls on a 3-CTA thread-block cluster (B200 design of Alg.2+3 for
// the steady state of deletemin-only calls; the first stage of bgpq_deletemin).
//
// Why.  Alg.3 chains consecutive DELETEMINs: op i+1's depth-0 SORT_SPLIT (l.10) reads the node
// op i's depth-1 step produced (l.11-15).  On one SM the three SORT_SPLITs of a slot (depth 0
// and 1 of op i, the lagged depth 2) share the issue and shared-memory bandwidth (~3.3k cycles
// together, ~0.9-1.5k alone) and one thread's decisions serialise around them (bgpq_dtop.cuh:
// ~9k cycles per op).  Here every on-chip depth has its own SM: a cluster of three CTAs, a
// systolic array over the top of the heap, connected by distributed shared memory (DSMEM):
//   R0 (cluster rank 0): root, nodes 2-3.  Root section of Alg.2 (output of the root, refill
//       from the last node — taken ahead by R0's helper warp, R20), depth-0 step of Alg.3.
//   R1 (rank 1): nodes 4-7.  Depth-1 step (SORT_SPLIT of y1's children, l.10; (y1, y2) split,
//       l.12); the new y1 is pushed into R0's shared memory by a DSMEM bulk copy.
//   R2 (rank 2): nodes 8-15.  Depth-2 step, pushes y2 to R1; hands y3 (LOCKed) with the
//       carried keys to a walker CTA (blockIdx >= 3: dt_walk, Alg.3 from l.2 with the paper's
//       hand-over-hand locks) and, through its helper warp, re-loads y3 once the walker has
//       released it (the node is "lent" meanwhile).
// Every level runs op i's step only after the level above sent op i's path node y_d (message
// "a", sent as soon as it is known from the children's cached max keys, l.9 — before the
// level's own SORT_SPLIT) and commits it after message "b" (the carried keys' descriptor and
// whether the walk continues, l.4).  Each level applies the ops in call order, so every node
// sees exactly the sequence of steps of the sequential execution of Alg.2+3 in call order,
// except for the early refill take (R20): linearizable with linearization order = call order.
// Carried keys (the refill node's keys as they sink, l.12 swaps in >99% of top-level steps)
// travel by reference: a global node index whose HBM copy holds them (the refill node, EMPTY
// after the take and never written during the call) — materialised only when a (cur, y)
// SORT_SPLIT really merges (then into the HBM copy of the on-chip node y_d, dead while on chip).
//
// Scope: full-K DELETEMINs while heapSize >= DS_HMIN, |root| = K, empty pBuffer (the state of
// a drain after insert calls of whole batches).  The rest of the call (partial batches, small
// heaps, non-empty buffers) is executed by bgpq_dtop_kernel, launched right after on the same
// stream, which reads how many ops this kernel did (DtArgs::op_base).
#pragma once
#include "bgpq_dtop.cuh"

namespace bgpqd {

constexpr int DS_NT = 512;             // split threads per role CTA (= walker compute threads)
constexpr int DS_NC = DS_NT + 32;      // role CTAs: control warp 0 (thread 0 decides) + split warps 1-16
constexpr int DS_BLOCK = DS_NC + 64;   // + 2 helper warps (roles) / lock warp + idle warps (walkers)
constexpr int DS_CL = 5;               // cluster size: steps of depths 0 .. DS_CL-1 in the cluster
constexpr int DS_NSLOT = 24;           // node slots per role CTA
constexpr u32 DS_MAXOWN = 1u << (DS_CL - 1);  // nodes the deepest owning level holds (depth DS_CL-1)
constexpr u32 DS_RING = 16;            // inbox entries
constexpr u32 DS_CREDIT = 4;           // credits are returned every DS_CREDIT entries
constexpr u32 DS_RF = 8;               // refill takes run at most this many ops ahead (R20)
constexpr u32 DS_HMIN = 1024;          // heapSize floor of the engine (depth >= 10 > DS_RF)
constexpr u32 DS_NONE = 0xFFFFFFFFu;
constexpr u32 DS_PULL = 0x40000000u;   // carried-keys source: a slot in a role's shared memory
constexpr u32 DSM_HMIN = 64;           // mixed calls: heapSize floor (nodes 1..63 AVAIL: the levels
                                       // and the stager's children are never EMPTY)

enum : u32 { MK_A = 1, MK_ASTOP = 2, MK_B = 3, MK_BSTOP = 4 };
// MK_A flag: every level above that swaps its (cur, y) split (l.12) passes the refill keys R
// on unchanged (src, [cmin, cmax] of the message), and the walk does not stop above given
// that.  A level whose own step then provably swaps commits it without message b (early
// commit, see ds_level).
constexpr u32 MA_EARLY = 1;


struct __align__(16) DsMsg {
  u32 op, kind, y, slot, src, cmin, cmax, pad;
};

// per role CTA control block (same layout in every CTA of the cluster: DSMEM addresses are
// obtained with mapa from local addresses)
struct DsCtl {
  u64 inbar[DS_RING];    // inbox entry barriers: armed (expect_tx) by this CTA, completed by the
                         // sender's bulk copy of the message (async proxy: no sender-side fence)
  u64 slotbar[DS_NSLOT]; // push completion per slot: armed by this CTA when it designates the slot
  DsMsg stage[DS_RING];  // outgoing messages (source of the bulk copies)
  u64 ainbar[DS_RING];   // second inbox (path messages "a" for the stager's staging helper)
  DsMsg ainbox[DS_RING];
  DsMsg astage[DS_RING];
  u32 aconsumed;
  u64 lbar;              // local TMA loads
  u64 hbar;              // helper's TMA loads
  u64 sbar[4];           // stager: staging completion of the op in staging ring entry k % 4
  DsMsg inbox[DS_RING];
  u32 consumed;          // inbox entries consumed (written remotely by the receiver into the SENDER,
                         // every DS_CREDIT entries)
  u32 b[16];             // thread-0 broadcasts
  // R0 helper: refill takes
  u32 rf_seq;            // takes published
  u32 rf_min[DS_RF], rf_max[DS_RF];
  u32 rf_used;           // ops whose take thread 0 consumed
  u32 pfs[4];            // mixed calls: R0's prefetch ring of sorted INSERT batches (slots)
  u32 pfreed;            // slots holding carried keys a lower level has pulled (remote red.or)
  // stager: helper A (LOCK + stage children) and helper B (tasks, write-backs, UNLOCKs) rings
  u32 sq_done;           // staging records published (helper A -> thread 0), one per op
  u32 sq_ret;            // ops whose staging slots thread 0 returned
  u32 stg_y[16], stg_up[16], stg_min[16][2], stg_max[16][2];
  u32 wq_head, wq_done, wq[16 * 5];
  u32 wb_free;           // slots helper B finished reading (atomicOr; thread 0 collects)
  u32 tasks;             // walker tasks published
  u32 quit;
  // thread-0 node table (shared memory, not local arrays: cluster-scope acquires invalidate
  // L1, so local memory would cost an L2 round trip per access)
  u32 ns[DS_MAXOWN], mn[DS_MAXOWN], mx[DS_MAXOWN], pend[DS_MAXOWN];
  ull st[NSTAT];
  ull tm[8];  // debug timers (bgpq_set_debug bit 1024): total, wait-above, wait-children, split, wait-b, sends
  ull tm2[16];  // debug 2097152: R1's per-segment timers (tools/ds_seg.py)
};
constexpr size_t DSCTL_BYTES = (sizeof(DsCtl) + 127) / 128 * 128;

template <int K, bool V>
constexpr size_t ds_smem_bytes() {
  const size_t role = DSCTL_BYTES + (size_t)DS_NSLOT * K * 4 * (V ? 2 : 1);
  const size_t wrk = LCTL_BYTES + (size_t)LSLOT * K * 4 * (V ? 2 : 1);
  return role > wrk ? role : wrk;
}

// ---- cluster / DSMEM PTX -----------------------------------------------------------------
__device__ __forceinline__ u32 cl_rank() {
  u32 r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ u32 cl_map(const void* p, u32 rank) {  // local smem -> cluster address in `rank`
  u32 a;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(smem_addr(p)), "r"(rank));
  return a;
}
__device__ __forceinline__ void cl_st(u32 addr, u32 v) {
  asm volatile("st.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ void cl_st_release(u32 addr, u32 v) {
  asm volatile("st.release.cluster.shared::cluster.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}
__device__ __forceinline__ u32 ld_acq_cluster(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.cluster.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_addr(p)) : "memory");
  return v;
}
__device__ __forceinline__ void cl_arrive(u32 bar_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar_addr) : "memory");
}
__device__ __forceinline__ void cl_arrive_tx(u32 bar_addr, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cluster.shared::cluster.b64 _, [%0], %1;" ::"r"(bar_addr),
               "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(u64* bar, u32 phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAITC_%=;\n}" ::"r"(smem_addr(bar)),
      "r"(phase) : "memory");
}
// bulk copy of `bytes` from this CTA's smem to a cluster address, completing tx on a
// (remote) mbarrier
__device__ __forceinline__ void bulk_s2cl(u32 dst, const void* src, u32 bytes, u32 bar) {
  asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "r"(smem_addr(src)), "r"(bytes), "r"(bar) : "memory");
}
// 16-B asynchronous store into another CTA's shared memory that completes its bytes on that
// CTA's mbarrier (st.async, sm_90+): the message transport of the cluster engine
__device__ __forceinline__ void st_async_v4(u32 addr, u32 a, u32 b, u32 c, u32 d, u32 bar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];"
               ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d), "r"(bar) : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// =========================================================================================
// One role CTA of the cluster
// =========================================================================================
template <int K, bool V>
struct DsRole {
  static constexpr u32 NB = K * 4u;
  static constexpr u32 SLOTB = V ? 2u * NB : NB;
  HeapArgs H;
  CallArgs C;
  DtArgs D;
  DsCtl* c;
  u32* sk;
  u32* sv;
  u32 rank;
  // thread-0 state (registers)
  u32 fm;                 // free slot mask
  u32 sbph;               // slot barrier parities (bit s)
  u32 in_seq;             // inbox entries consumed
  u32 out_seq;            // messages sent to the level below
  u32 out_seq2;           // path messages sent to the stager's second inbox
  u32 lph;                // lbar parity
  bool timing;
  // thread 0's per-op counters in registers (a shared-memory u64 read-modify-write per counter
  // per op sat on the decision chain); flushed into c->st by flush_counts at the role's end
  u32 n_lev = 0, n_nomove = 0, n_swap = 0, n_ilev = 0, n_inoop = 0, n_iswap = 0;
  __device__ __forceinline__ void flush_counts() {
    c->st[S_DEL_LEVELS] += n_lev;
    c->st[S_DEL_LR_NOMOVE] += n_nomove;
    c->st[S_DEL_LR_MERGE] += n_lev - n_nomove;
    c->st[S_DEL_CY_SWAP] += n_swap;
    c->st[S_INS_LEVELS] += n_ilev;
    c->st[S_INS_NOOP] += n_inoop;
    c->st[S_INS_SWAP] += n_iswap;
    c->st[S_INS_MERGE] += n_ilev - n_inoop - n_iswap;
  }
  __device__ __forceinline__ ull tnow() const { return timing ? clock64() : 0ull; }
  bool seg = false;  // debug 2097152: segment timers of R1
  ull tseg = 0;
  __device__ __forceinline__ void segmark(int k) {
    if (seg) { const ull t = clock64(); c->tm2[k] += t - tseg; tseg = t; }
  }
  __device__ __forceinline__ void tacc(int k, ull t0) { if (timing) c->tm[k] += clock64() - t0; }

  __device__ __forceinline__ u32* BK(u32 s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(u32 s) const { return V ? sv + s * K : nullptr; }
  // ---- carried keys that live only in a role's shared memory (a (cur, y) SORT_SPLIT merged
  // them on chip): message b names them as PULL | owner rank << 8 | slot; the level that needs
  // their content copies them over DSMEM (pull_copy) and returns the slot (pull_free).
  __device__ __forceinline__ u32 pull_ref(u32 s) const { return DS_PULL | (rank << 8) | s; }
  // thread 0, before the message b that carries a pull reference: the compute threads' writes
  // of the slot (ordered before thread 0 by the CTA barrier) are released at cluster scope
  __device__ __forceinline__ void pull_publish() const { asm volatile("fence.acq_rel.cluster;" ::: "memory"); }
  // all DS_NT compute threads (the caller's thread 0 ran fence.acq_rel.cluster after the
  // message and a CTA barrier followed): slot `dst` <- the referenced slot of its owner
  __device__ __forceinline__ void pull_copy(u32 ref, u32 dst) const {
    const u32 owner = (ref >> 8) & 0xFFu, src = ref & 0xFFu;
    const u32 rk = cl_map(BK(src), owner);
    for (int q = threadIdx.x; q < K / 4; q += DS_NC) {
      uint4 v;
      asm volatile("ld.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];"
                   : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(rk + 16u * q) : "memory");
      reinterpret_cast<uint4*>(BK(dst))[q] = v;
    }
    if (V) {
      const u32 rv = cl_map(BV(src), owner);
      for (int q = threadIdx.x; q < K / 4; q += DS_NC) {
        uint4 v;
        asm volatile("ld.shared::cluster.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(rv + 16u * q) : "memory");
        reinterpret_cast<uint4*>(BV(dst))[q] = v;
      }
    }
  }
  // thread 0, after the CTA barrier that ended pull_copy: the owner may reuse the slot
  __device__ __forceinline__ void pull_free(u32 ref) const {
    const u32 owner = (ref >> 8) & 0xFFu, src = ref & 0xFFu;
    asm volatile("red.relaxed.cluster.shared::cluster.or.b32 [%0], %1;" ::"r"(cl_map(&c->pfreed, owner)),
                 "r"(1u << src) : "memory");
  }
  __device__ __forceinline__ void collect_pulled() { fm |= atomicExch(&c->pfreed, 0u); }
  __device__ __forceinline__ u32 alloc() {
    while (fm == 0) {  // slots lent to lower levels for pulls come back through pfreed
      const u32 fr = atomicExch(&c->pfreed, 0u);
      fm |= fr;
    }
    const u32 s = __ffs(fm) - 1;
    fm &= ~(1u << s);
    return s;
  }
  __device__ __forceinline__ void release(u32 s) {
    if (s != DS_NONE) fm |= 1u << s;
  }
  // ---- inbox (thread 0).  A message is a 32-B bulk copy from the sender's staging ring into
  // this CTA's inbox entry, completing the entry's barrier (armed here with expect_tx); so the
  // sender needs no cluster-scope release and the receiver waits at CTA scope.
  __device__ __forceinline__ void arm_inbox(u32 e) {
    mbar_arrive_expect_tx(&c->inbar[e], (u32)sizeof(DsMsg));
  }
  __device__ __forceinline__ DsMsg recv() {
    const u32 e = in_seq % DS_RING;
    mbar_wait(&c->inbar[e], (in_seq / DS_RING) & 1u);
    DsMsg m;
    volatile DsMsg* pm = &c->inbox[e];
    m.op = pm->op; m.kind = pm->kind; m.y = pm->y; m.slot = pm->slot;
    m.src = pm->src; m.cmin = pm->cmin; m.cmax = pm->cmax; m.pad = pm->pad;
    ++in_seq;
    arm_inbox(e);  // for the message DS_RING entries later
    if (in_seq % DS_CREDIT == 0) {  // credit back to the sender (its staging entries are free too)
      const ull t0 = tnow();
      asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(cl_map(&c->consumed, rank - 1)),
                   "r"(in_seq) : "memory");
      tacc(6, t0);
    }
    return m;
  }
  // ---- send to the level below (thread 0)
  __device__ __forceinline__ void send(u32 op, u32 kind, u32 y = 0, u32 slot = 0, u32 src = 0, u32 cmin = 0,
                                       u32 cmax = 0, u32 flags = 0) {
    const ull t0 = tnow();
    while (out_seq - *reinterpret_cast<volatile u32*>(&c->consumed) >= DS_RING - DS_CREDIT) {}
    const u32 e = out_seq % DS_RING;
    const u32 dst = rank + 1;
    // two 16-B remote async stores, each completing its bytes on the receiver's armed inbox
    // barrier (no staging copy, no proxy fence, no bulk group)
    const u32 ia = cl_map(&c->inbox[e], dst), ib = cl_map(&c->inbar[e], dst);
    st_async_v4(ia, op, kind, y, slot, ib);
    st_async_v4(ia + 16u, src, cmin, cmax, flags, ib);
    ++out_seq;
    tacc(5, t0);
  }
  // ---- path messages to the stager go to its second inbox (read by its staging helper)
  __device__ __forceinline__ void send_a2(u32 op, u32 kind, u32 y, u32 slot) {
    const ull t0 = tnow();
    while (out_seq2 - *reinterpret_cast<volatile u32*>(&c->aconsumed) >= DS_RING - DS_CREDIT) {}
    const u32 e = out_seq2 % DS_RING;
    const u32 dst = rank + 1;
    const u32 ia = cl_map(&c->ainbox[e], dst), ib = cl_map(&c->ainbar[e], dst);
    st_async_v4(ia, op, kind, y, slot, ib);
    st_async_v4(ia + 16u, 0u, 0u, 0u, 0u, ib);
    ++out_seq2;
    tacc(5, t0);
  }
  __device__ __forceinline__ void send_path(u32 op, u32 kind, u32 y = 0, u32 slot = 0, u32 src = 0, u32 cmin = 0,
                                            u32 cmax = 0, u32 flags = 0) {
    if (rank + 2 == (u32)DS_CL) send_a2(op, kind, y, slot);
    else send(op, kind, y, slot, src, cmin, cmax, flags);
  }
  // ---- slots the level below pushes into: armed when designated, disarmed if no push comes
  __device__ __forceinline__ void arm_slot(u32 s) { mbar_arrive_expect_tx(&c->slotbar[s], SLOTB); }
  __device__ __forceinline__ void disarm_slot(u32 s) {
    asm volatile("mbarrier.complete_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(&c->slotbar[s])),
                 "r"(SLOTB) : "memory");
    wait_pushed(s);
  }
  // ---- push slot s (K entries) into slot `ds` of the level above, which armed it (thread 0;
  // the caller made the slot's generic writes visible with a CTA barrier)
  __device__ __forceinline__ void push_up(u32 s, u32 ds) {
    const ull t0 = tnow();
    const u32 up = rank - 1;
    const u32 bar = cl_map(&c->slotbar[ds], up);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    bulk_s2cl(cl_map(BK(ds), up), BK(s), NB, bar);
    if (V) bulk_s2cl(cl_map(BV(ds), up), BV(s), NB, bar);
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    tacc(7, t0);
  }
  __device__ __forceinline__ void wait_pushed(u32 s) {  // a push into local slot s has landed
    mbar_wait(&c->slotbar[s], (sbph >> s) & 1u);
    sbph ^= 1u << s;
  }
  // synchronous TMA load of HBM node n into slot s (thread 0)
  __device__ __forceinline__ void load_node(u32 s, u32 n) {
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->lbar, SLOTB);
    bulk_g2s(BK(s), src_keys<K>(H, n), NB, &c->lbar);
    if (V) bulk_g2s(BV(s), src_vals<K>(H, n), NB, &c->lbar);
    mbar_wait(&c->lbar, lph);
    lph ^= 1u;
  }
  // write slot s to HBM node n (thread 0, TMA bulk store, waits for completion)
  __device__ __forceinline__ void store_node(u32 n, u32 s) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    bulk_s2g(H.gk + (size_t)n * K, BK(s), NB);
    if (V) bulk_s2g(H.gv + (size_t)n * K, BV(s), NB);
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
};

// All NT compute threads: SORT_SPLIT of two full K-batches, X = K smallest, Y = rest.
// LEAD = false where the caller's own CTA barrier directly precedes the call (only broadcast
// words were read since): the leading barrier would be a second one back to back.
// The split runs on warps 1-16 while thread 0 (warp 0) runs `during` — the role's bookkeeping
// that the split does not need (its path message to the level below, slot arming, ...).
template <int K, bool V, bool LEAD = true, typename F>
__device__ __forceinline__ void ds_split_h(DsRole<K, V>& R, u32 z, u32 w, u32 x, u32 y, F&& during) {
  if (LEAD) cta_bar<DS_NC>();
  if (threadIdx.x >= 32)
    sort_split_t<K, DS_NT, V>((int)threadIdx.x - 32, R.BK(z), R.BV(z), K, R.BK(w), R.BV(w), K, K, R.BK(x), R.BV(x),
                              R.BK(y), R.BV(y));
  else if (threadIdx.x == 0)
    during();
  cta_bar<DS_NC>();
}
template <int K, bool V, bool LEAD = true>
__device__ __forceinline__ void ds_split(DsRole<K, V>& R, u32 z, u32 w, u32 x, u32 y) {
  ds_split_h<K, V, LEAD>(R, z, w, x, y, [] {});
}

// Number of full-K ops the engine executes (identical in every role CTA): the call's full
// batches, while heapSize stays >= DS_HMIN, if |root| is K or 0 and the pBuffer is empty.
// (|root| = 0 is the state a drained heap keeps, reading R4: then every DELETEMIN refills the
// root and extracts all K keys of it after the heapify, Alg.2 l.4-14 + l.5-6 of Alg.3.)
__device__ __forceinline__ u64 ds_ops(const HeapArgs& H, const CallArgs& C, int K) {
  const u32 hs = ld_relaxed(H.hdr + H_HS), rs = ld_relaxed(H.hdr + H_RS), ps = ld_relaxed(H.hdr + H_PS);
  if (C.mode == MODE_MIXED) {  // op pairs (INSERT(K), DELETEMIN(K)) from the call's start
    if ((rs != (u32)K && rs != 0) || ps != 0 || hs < DSM_HMIN || hs + 1u > H.cap) return 0;
    const u64 np = C.n_ops / 2, pe = ld_relaxed(C.pair_end);
    return np < pe ? np : pe;
  }
  if ((rs != (u32)K && rs != 0) || ps != 0 || hs < DS_HMIN + 2) return 0;
  const u64 full = C.n / (u64)K;
  const u64 room = hs - DS_HMIN;
  return full < room ? full : room;
}

// -----------------------------------------------------------------------------------------
// R0: root section + depth 0
// -----------------------------------------------------------------------------------------
template <int K, bool V>
__device__ void ds_r0(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  const int tid = threadIdx.x;
  u32 hs = ld_relaxed(H.hdr + H_HS);
  // |root| = K: op i outputs the root (Alg.2 l.22) and refills it; |root| = 0 (R4): op i
  // refills the empty root and extracts all K keys after the heapify (l.14 + Alg.3 l.5-6),
  // so it outputs the root's new content and leaves it empty
  const bool rz = ld_relaxed(H.hdr + H_RS) == 0;
  // on-chip nodes: 1 (root), 2, 3
  u32* ns = c->ns;
  u32* mn = c->mn;
  u32* mx = c->mx;
  u32* pend = c->pend;
  if (tid == 0) {
    ns[1] = DS_NONE;
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      ns[q] = R.alloc();
      pend[q] = 0;
      mn[q] = ld_relaxed(&H.meta[q].kmin);
      mx[q] = ld_relaxed(&H.meta[q].kmax);
    }
    pend[1] = 0;
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->lbar, (rz ? 2u : 3u) * DsRole<K, V>::SLOTB);
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      bulk_g2s(R.BK(ns[q]), H.gk + (size_t)q * K, DsRole<K, V>::NB, &c->lbar);
      if (V) bulk_g2s(R.BV(ns[q]), H.gv + (size_t)q * K, DsRole<K, V>::NB, &c->lbar);
    }
    mbar_wait(&c->lbar, R.lph);
    R.lph ^= 1u;
  }
  cta_bar<DS_NC>();
  u32 out_old = DS_NONE;  // slot whose output store may still be reading it
  // op i's K output keys from slot s (TMA bulk store; the slot is freed once it was read)
  auto output = [&](u64 i, u32 s) {
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // the previous output's read
    R.release(out_old);
    const u64 pos = i * (u64)K;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    bulk_s2g(R.C.out_k + pos, R.BK(s), DsRole<K, V>::NB);
    if (V && R.C.out_v) bulk_s2g(R.C.out_v + pos, R.BV(s), DsRole<K, V>::NB);
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    out_old = s;
  };
  const ull t_start = R.tnow();
  for (u64 i = 0; i < m; ++i) {
    if (tid == 0) {
      R.collect_pulled();
      // refill of op i (Alg.2 l.5-12), taken ahead by the helper: node hs, now EMPTY
      const u32 t = hs;
      const ull t1 = R.tnow();
      while (ld_acq_cta(&c->rf_seq) <= (u32)i) {}
      R.tacc(1, t1);
      const u32 rmin = c->rf_min[i % DS_RF], rmax = c->rf_max[i % DS_RF];
      st_rel_cta(&c->rf_used, (u32)i + 1u);
      hs -= 1;
      // a pending y1 push of op i-1 must have landed before depth 0 reads it
      const ull t2 = R.tnow();
      for (u32 q = 2; q <= 3; ++q)
        if (pend[q]) {
          R.wait_pushed(ns[q]);
          pend[q] = 0;
          mn[q] = R.BK(ns[q])[0];
          mx[q] = R.BK(ns[q])[K - 1];
        }
      R.tacc(2, t2);
      if (!rz) output(i, ns[1]);  // Alg.2 l.22: the root's K keys are op i's output
      // Alg.3 at the root: cur = root holding the refill keys
      const u32 minc = mn[2] < mn[3] ? mn[2] : mn[3];
      if (rmax <= minc) {  // l.4: stop at the root — root <- the refill keys
        const u32 s = R.alloc();
        R.load_node(s, t);
        if (rz) output(i, s);
        else { ns[1] = s; mn[1] = rmin; mx[1] = rmax; }
        R.send((u32)i, MK_ASTOP);
        c->b[0] = 1;
      } else {
        const u32 x = mx[2] > mx[3] ? 2u : 3u, y = 5u - x;  // l.9 (R6: tie -> x = r)
        const u32 sy = R.alloc();  // y1's new content arrives here from R1
        R.arm_slot(sy);
        R.send((u32)i, MK_A, y, sy, t, rmin, rmax, MA_EARLY);
        const u32 A = R.alloc(), B = R.alloc();
        c->b[0] = 0; c->b[1] = ns[2]; c->b[2] = ns[3]; c->b[3] = A; c->b[4] = B;
        c->b[5] = x; c->b[6] = y; c->b[7] = sy; c->b[8] = t; c->b[9] = rmin; c->b[10] = rmax;
        ++R.n_lev;
        R.n_nomove += (mx[2] <= mn[3] || mx[3] <= mn[2]) ? 1u : 0u;
      }
    }
    cta_bar<DS_NC>();
    if (c->b[0]) continue;
    const u32 s2 = c->b[1], s3 = c->b[2], A = c->b[3], B = c->b[4];
    const ull t3 = R.tnow();
    ds_split<K, V, false>(R, s2, s3, A, B);  // l.10: (Heap[y], Heap[x]) <- SORT_SPLIT(l, r)
    if (tid == 0) R.tacc(3, t3);
    if (tid == 0) {
      const u32 x = c->b[5], y = c->b[6], sy = c->b[7], t = c->b[8], rmin = c->b[9], rmax = c->b[10];
      R.release(s2); R.release(s3);
      const u32 ymax = R.BK(A)[K - 1];
      if (ymax <= rmin) {  // l.12 is a swap: root <- Y, the refill keys sink on (by reference)
        ++R.n_swap;
        R.send((u32)i, MK_B, 0, 0, t, rmin, rmax);
        if (rz) output(i, A);  // Alg.3 l.5-6 / l.13: the root's new keys are extracted
        else { ns[1] = A; mn[1] = R.BK(A)[0]; mx[1] = ymax; }
        c->b[15] = 0;
      } else {  // l.12 merges: (root, C1) <- SORT_SPLIT(refill, Y); C1 into y1's dead HBM copy
        const u32 r = R.alloc(), lo = R.alloc(), hi = R.alloc();
        R.load_node(r, t);
        c->b[11] = r; c->b[12] = lo; c->b[13] = hi;
        c->b[15] = 1;
      }
      ns[x] = B; mn[x] = R.BK(B)[0]; mx[x] = R.BK(B)[K - 1];
      ns[y] = sy; pend[y] = 1;
    }
    cta_bar<DS_NC>();
    if (c->b[15]) {  // rare: a real (cur, y) merge at the root
      const u32 r = c->b[11], lo = c->b[12], hi = c->b[13];
      ds_split<K, V, false>(R, r, A, lo, hi);
      if (tid == 0) {
        // C1 stays in slot hi; the level that needs its content pulls it (DS_PULL)
        R.pull_publish();
        R.send((u32)i, MK_B, 0, 0, R.pull_ref(hi), R.BK(hi)[0], R.BK(hi)[K - 1]);
        if (rz) output(i, lo);
        else { ns[1] = lo; mn[1] = R.BK(lo)[0]; mx[1] = R.BK(lo)[K - 1]; }
        R.release(r); R.release(A);
      }
      cta_bar<DS_NC>();
    }
  }
  // ---- end: wait for the last pushes, write the on-chip nodes back, update the header
  if (tid == 0) {
    R.tacc(0, t_start);
    for (u32 q = 2; q <= 3; ++q)
      if (pend[q]) { R.wait_pushed(ns[q]); pend[q] = 0; mn[q] = R.BK(ns[q])[0]; mx[q] = R.BK(ns[q])[K - 1]; }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      R.store_node(q, ns[q]);
      st_relaxed(&H.meta[q].kmin, mn[q]);
      st_relaxed(&H.meta[q].kmax, mx[q]);
    }
    st_relaxed(H.hdr + H_HS, hs);
    ull lin;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(lin) : "l"(H.hdr + H_LIN) : "memory");
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(lin + m) : "memory");
    c->st[S_KEYS_OUT] += m * (u64)K;
    c->st[S_DEL_OPS] += m;
    c->st[S_DEL_REFILL] += m;
    R.flush_counts();
    if (R.C.d_count && m) atomicAdd(R.C.d_count, (ull)(m * (u64)K));
    *reinterpret_cast<volatile u64*>(R.D.op_base) = m;
  }
}

// -----------------------------------------------------------------------------------------
// R0 of a mixed call: op pairs (INSERT(K), DELETEMIN(K)) in call order (the utilisation
// workload).  Pair i's INSERT takes the target tar = heapSize + 1 (Alg.1 l.4-6), runs
// its root section (l.20; the pBuffer is empty and the batch full, so l.26-28 leave both as
// they are) and its first INSERT_HEAPIFY step at NEXT(root, tar) (l.33), a node R0 holds on
// chip.  The DELETEMIN that follows takes tar as its refill node (Alg.2 l.5): tar is TARGET,
// so the DELETEMIN marks it MARKED (l.7-9), the INSERT breaks out at its next check (Alg.1
// l.31) and puts its items into the root (l.11-13): the refill keys are the INSERT's
// items after its depth-1 step, heapSize is back at its old value and tar EMPTY again.  That
// is the interleaving in which the DELETEMIN's root section starts as soon as the INSERT
// released the root — R0 executes it without touching tar (reading R26).  The
// DELETEMIN then continues exactly as in ds_r0 (depth-0 step; levels below unchanged).
// The items arrive sorted (Alg.1 l.2) from bgpq_msort_kernel in H.xk + i*K; they sink by
// reference (XREF | i) while unchanged, otherwise R0 stores them back there first.
// -----------------------------------------------------------------------------------------
template <int K, bool V>
__device__ void ds_r0_mixed(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  const CallArgs& C = R.C;
  const int tid = threadIdx.x;
  constexpr u32 PF = 3;  // sorted INSERT batches loaded ahead (ring of 4: c->pfs / c->sbar)
  constexpr u32 NB = DsRole<K, V>::NB;
  const u32 hs = ld_relaxed(H.hdr + H_HS);
  const bool rz = ld_relaxed(H.hdr + H_RS) == 0;  // R4: a drained root stays empty
  const u32 d1 = next_on_path(1u, hs + 1u);         // NEXT(root, tar) of every pair (2 or 3)
  u32* ns = c->ns;
  u32* mn = c->mn;
  u32* mx = c->mx;
  u32* pend = c->pend;
  ull lin0 = 0;
  u32 pfph = 0;                      // sbar parities (thread 0)
  u32 it = 0, imin = 0, imax = 0;    // thread 0: the INSERT's items (slot, min, max)
  u32 dirty = 0;                     // thread 0: items differ from H.xk + i*K
  if (tid == 0) {
    ns[1] = DS_NONE;
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      ns[q] = R.alloc();
      pend[q] = 0;
      mn[q] = ld_relaxed(&H.meta[q].kmin);
      mx[q] = ld_relaxed(&H.meta[q].kmax);
    }
    pend[1] = 0;
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->lbar, (rz ? 2u : 3u) * DsRole<K, V>::SLOTB);
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      bulk_g2s(R.BK(ns[q]), H.gk + (size_t)q * K, NB, &c->lbar);
      if (V) bulk_g2s(R.BV(ns[q]), H.gv + (size_t)q * K, NB, &c->lbar);
    }
    mbar_wait(&c->lbar, R.lph);
    R.lph ^= 1u;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(lin0) : "l"(H.hdr + H_LIN) : "memory");
  }
  cta_bar<DS_NC>();
  u32 out_old = DS_NONE;
  auto output = [&](u64 j, u32 s) {  // op j's K output keys from slot s (TMA bulk store)
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
    R.release(out_old);
    const u64 pos = j * (u64)K;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    bulk_s2g(C.out_k + pos, R.BK(s), NB);
    if (V && C.out_v) bulk_s2g(C.out_v + pos, R.BV(s), NB);
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    out_old = s;
  };
  auto prefetch = [&](u64 k) {  // pair k's sorted items into a fresh slot
    const u32 s = R.alloc();
    c->pfs[k % 4] = s;
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->sbar[k % 4], DsRole<K, V>::SLOTB);
    bulk_g2s(R.BK(s), H.xk + (size_t)k * K, NB, &c->sbar[k % 4]);
    if (V) bulk_g2s(R.BV(s), H.xv + (size_t)k * K, NB, &c->sbar[k % 4]);
  };
  if (tid == 0)
    for (u64 k = 0; k < PF && k < m; ++k) prefetch(k);
  const ull t_start = R.tnow();
  for (u64 i = 0; i < m; ++i) {
    const u64 jd = 2 * i + 1;  // the DELETEMIN's op index (the INSERT is 2i)
    // ---- INSERT, Alg.1 l.20: (root, items) <- SORT_SPLIT(root, |root|, items, K, |root|)
    if (tid == 0) {
      R.collect_pulled();
      if (i + PF < m) prefetch(i + PF);
      const ull t1 = R.tnow();
      mbar_wait(&c->sbar[i % 4], (pfph >> (i % 4)) & 1u);
      pfph ^= 1u << (i % 4);
      R.tacc(1, t1);
      it = c->pfs[i % 4];
      imin = R.BK(it)[0];
      imax = R.BK(it)[K - 1];
      const ull t2 = R.tnow();
      if (pend[d1]) {  // the INSERT's depth-1 node: op i-1's push into it must have landed
        R.wait_pushed(ns[d1]);
        pend[d1] = 0;
        mn[d1] = R.BK(ns[d1])[0];
        mx[d1] = R.BK(ns[d1])[K - 1];
      }
      R.tacc(2, t2);

      const u32 ra = rz ? 0u : (mx[1] <= imin) ? 0u : (imax <= mn[1]) ? 1u : 2u;
      if (ra == 1) {  // the batch lies entirely below the root: swap the contents
        const u32 t = ns[1]; ns[1] = it; it = t;
        const u32 a = mn[1], b = mx[1]; mn[1] = imin; mx[1] = imax; imin = a; imax = b;
      }
      dirty = ra != 0;
      c->b[0] = ra;
      if (ra == 2) { c->b[1] = ns[1]; c->b[2] = it; c->b[3] = R.alloc(); c->b[4] = R.alloc(); }
    }
    cta_bar<DS_NC>();
    if (c->b[0] == 2) {
      ds_split<K, V, false>(R, c->b[1], c->b[2], c->b[3], c->b[4]);
      if (tid == 0) {
        R.release(ns[1]); R.release(it);
        ns[1] = c->b[3]; it = c->b[4];
        mn[1] = R.BK(ns[1])[0]; mx[1] = R.BK(ns[1])[K - 1];
        imin = R.BK(it)[0]; imax = R.BK(it)[K - 1];
      }
    }
    // ---- INSERT, l.33 at cur = NEXT(root, tar): (Heap[cur], items) <- SORT_SPLIT(Heap[cur], items)
    if (tid == 0) {
      const u32 da = (mx[d1] <= imin) ? 0u : (imax <= mn[d1]) ? 1u : 2u;
      ++R.n_ilev;
      R.n_inoop += da == 0 ? 1u : 0u;
      R.n_iswap += da == 1 ? 1u : 0u;
      if (da == 1) {
        const u32 t = ns[d1]; ns[d1] = it; it = t;
        const u32 a = mn[d1], b = mx[d1]; mn[d1] = imin; mx[d1] = imax; imin = a; imax = b;
      }
      dirty |= da != 0;
      c->b[0] = da;
      if (da == 2) { c->b[1] = ns[d1]; c->b[2] = it; c->b[3] = R.alloc(); c->b[4] = R.alloc(); }
    }
    cta_bar<DS_NC>();
    // thread 0's work for the DELETEMIN that the INSERT's depth-1 split does not need: the other
    // depth-1 node's push (op i-1's y1) and the op tickets — overlapped with that split
    const u32 o1 = 5u - d1;
    auto pre_del = [&] {
      if (pend[o1]) {
        const ull t2 = R.tnow();
        R.wait_pushed(ns[o1]);
        pend[o1] = 0;
        mn[o1] = R.BK(ns[o1])[0];
        mx[o1] = R.BK(ns[o1])[K - 1];
        R.tacc(2, t2);
      }
      if (C.lin_ticket) {
        st_relaxed_u64(reinterpret_cast<u64*>(C.lin_ticket) + 2 * i, lin0 + 2 * i);
        st_relaxed_u64(reinterpret_cast<u64*>(C.lin_ticket) + jd, lin0 + jd);
      }
      st_relaxed(C.op_count + jd, (u32)K);
    };
    if (c->b[0] == 2) {
      ds_split_h<K, V, false>(R, c->b[1], c->b[2], c->b[3], c->b[4], pre_del);
      if (tid == 0) {
        R.release(ns[d1]); R.release(it);
        ns[d1] = c->b[3]; it = c->b[4];
        mn[d1] = R.BK(ns[d1])[0]; mx[d1] = R.BK(ns[d1])[K - 1];
        imin = R.BK(it)[0]; imax = R.BK(it)[K - 1];
      }
    } else if (tid == 0) {
      pre_del();
    }
    // ---- DELETEMIN: the root's keys are its output (Alg.2 l.22), the refill keys are the
    // INSERT's items (the MARKED hand-off, l.7-12), then Alg.3 at the root as in ds_r0
    if (tid == 0) {

      if (!rz) output(jd, ns[1]);
      const u32 minc = mn[2] < mn[3] ? mn[2] : mn[3];
      if (imax <= minc) {  // l.4: stop at the root — root <- the refill keys
        if (rz) output(jd, it);
        else { ns[1] = it; mn[1] = imin; mx[1] = imax; }
        R.send((u32)i, MK_ASTOP);
        c->b[0] = 1;
      } else {
        const u32 x = mx[2] > mx[3] ? 2u : 3u, y = 5u - x;  // l.9 (R6: tie -> x = r)
        const u32 sy = R.alloc();
        R.arm_slot(sy);
        // early commit below (MA_EARLY) only while the items are still the HBM copy H.xk + i*K
        R.send((u32)i, MK_A, y, sy, XREF | (u32)i, imin, imax, dirty ? 0u : MA_EARLY);
        const u32 A = R.alloc(), B = R.alloc();
        c->b[0] = 0; c->b[1] = ns[2]; c->b[2] = ns[3]; c->b[3] = A; c->b[4] = B;
        c->b[5] = x; c->b[6] = y; c->b[7] = sy;
        ++R.n_lev;
        R.n_nomove += (mx[2] <= mn[3] || mx[3] <= mn[2]) ? 1u : 0u;
      }
    }
    cta_bar<DS_NC>();
    if (c->b[0]) continue;
    const u32 s2 = c->b[1], s3 = c->b[2], A = c->b[3], B = c->b[4];
    const ull t3 = R.tnow();
    ds_split<K, V, false>(R, s2, s3, A, B);  // l.10
    if (tid == 0) R.tacc(3, t3);
    if (tid == 0) {
      const u32 x = c->b[5], y = c->b[6], sy = c->b[7];
      R.release(s2); R.release(s3);
      const u32 ymax = R.BK(A)[K - 1];
      if (ymax <= imin) {  // l.12 is a swap: root <- Y, the refill keys sink on (by reference)
        ++R.n_swap;
        if (dirty) {  // the items changed on chip: a lower level pulls them from slot it
          R.pull_publish();
          R.send((u32)i, MK_B, 0, 0, R.pull_ref(it), imin, imax);
        } else {      // still the sorted batch H.xk + i*K
          R.send((u32)i, MK_B, 0, 0, XREF | (u32)i, imin, imax);
          R.release(it);
        }
        if (rz) output(jd, A);
        else { ns[1] = A; mn[1] = R.BK(A)[0]; mx[1] = ymax; }
        c->b[15] = 0;
      } else {  // l.12 merges: (root, C1) <- SORT_SPLIT(refill, Y); C1 into y1's dead HBM copy
        c->b[11] = it; c->b[12] = R.alloc(); c->b[13] = R.alloc();
        c->b[15] = 1;
      }
      ns[x] = B; mn[x] = R.BK(B)[0]; mx[x] = R.BK(B)[K - 1];
      ns[y] = sy; pend[y] = 1;
    }
    cta_bar<DS_NC>();
    if (c->b[15]) {
      const u32 r = c->b[11], lo = c->b[12], hi = c->b[13];
      ds_split<K, V, false>(R, r, A, lo, hi);
      if (tid == 0) {
        R.pull_publish();  // C1 stays in slot hi until a lower level pulled it
        R.send((u32)i, MK_B, 0, 0, R.pull_ref(hi), R.BK(hi)[0], R.BK(hi)[K - 1]);
        if (rz) output(jd, lo);
        else { ns[1] = lo; mn[1] = R.BK(lo)[0]; mx[1] = R.BK(lo)[K - 1]; }
        R.release(r); R.release(A);
      }
      cta_bar<DS_NC>();
    }
  }
  // ---- end: the on-chip nodes back to HBM; heapSize is unchanged by every pair
  if (tid == 0) {
    R.tacc(0, t_start);
    for (u32 q = 2; q <= 3; ++q)
      if (pend[q]) { R.wait_pushed(ns[q]); pend[q] = 0; mn[q] = R.BK(ns[q])[0]; mx[q] = R.BK(ns[q])[K - 1]; }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    for (u32 q = rz ? 2 : 1; q <= 3; ++q) {
      R.store_node(q, ns[q]);
      st_relaxed(&H.meta[q].kmin, mn[q]);
      st_relaxed(&H.meta[q].kmax, mx[q]);
    }
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(lin0 + 2 * m) : "memory");
    st_relaxed(H.hdr + H_FETCH, (u32)(2 * m));  // the lock engine continues at op 2m
    c->st[S_KEYS_OUT] += m * (u64)K;
    c->st[S_INS_OPS] += m;
    c->st[S_INS_HEAPIFY] += m;
    c->st[S_DEL_OPS] += m;
    c->st[S_DEL_REFILL] += m;
    c->st[S_MARKED] += m;
    R.flush_counts();
    *reinterpret_cast<volatile u64*>(R.D.op_base) = m;
  }
}

// R0's helper (lane 0): the refill takes (Alg.2 l.6-12) up to DS_RF ops ahead (R20).
template <int K, bool V>
__device__ void ds_r0_helper(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  const u32 hs0 = ld_relaxed(H.hdr + H_HS);
  for (u64 j = 0; j < m; ++j) {
    while ((u32)j >= ld_acq_cta(&c->rf_used) + DS_RF) __nanosleep(32);
    const u32 t = hs0 - (u32)j;
    lock_acquire(&H.meta[t].lock);  // l.6: LOCK(tar)
    const u32 mnv = ld_relaxed(&H.meta[t].kmin), mxv = ld_relaxed(&H.meta[t].kmax);
    st_relaxed(&H.meta[t].state, ST_EMPTY);  // l.11: its keys move to the root, tar <- EMPTY
    lock_release(&H.meta[t].lock);           // l.12: UNLOCK(tar)
    // the keys sink by reference (the HBM copy of t): warm them in L2 for the walker that
    // will load them below the cluster's levels
    if (!(R.C.debug & 2048u))
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gk + (size_t)t * K), "r"(DsRole<K, V>::NB)
                 : "memory");
    if (V && !(R.C.debug & 2048u))
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gv + (size_t)t * K), "r"(DsRole<K, V>::NB)
                   : "memory");
    c->rf_min[j % DS_RF] = mnv;
    c->rf_max[j % DS_RF] = mxv;
    st_rel_cta(&c->rf_seq, (u32)j + 1u);
  }
}

// -----------------------------------------------------------------------------------------
// R1 .. R(DS_CL-2): the depth-d step (d = rank), owning the nodes of depth d+1
// -----------------------------------------------------------------------------------------
template <int K, bool V>
__device__ void ds_level(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  const int tid = threadIdx.x;
  const u32 d = R.rank;              // this CTA's step depth
  const u32 base = 1u << (d + 1);    // first owned node
  const u32 cnt = base;              // owned nodes: base .. 2*base-1
  u32* ns = c->ns;
  u32* mn = c->mn;
  u32* mx = c->mx;
  u32* pend = c->pend;
  if (tid == 0) {
    fence_proxy_async();
    mbar_arrive_expect_tx(&c->lbar, cnt * DsRole<K, V>::SLOTB);
    for (u32 j = 0; j < cnt; ++j) {
      const u32 n = base + j;
      ns[j] = R.alloc();
      pend[j] = 0;
      mn[j] = ld_relaxed(&H.meta[n].kmin);
      mx[j] = ld_relaxed(&H.meta[n].kmax);
      bulk_g2s(R.BK(ns[j]), H.gk + (size_t)n * K, DsRole<K, V>::NB, &c->lbar);
      if (V) bulk_g2s(R.BV(ns[j]), H.gv + (size_t)n * K, DsRole<K, V>::NB, &c->lbar);
    }
    mbar_wait(&c->lbar, R.lph);
    R.lph ^= 1u;
  }
  cta_bar<DS_NC>();
  u32 push_old = DS_NONE;  // slot whose push may still be reading it
  u32 a_src = 0, a_cmin = 0, a_cmax = 0, early = 0, a_flags = 0;  // thread 0: the path message's refill-key info
  const ull t_start = R.tnow();
  if (tid == 0) R.tseg = clock64();
  for (u64 i = 0; i < m; ++i) {
    if (tid == 0) {
      R.collect_pulled();
      const ull t1 = R.tnow();
      R.segmark(15);
      const DsMsg a = R.recv();
      R.segmark(0);
      R.tacc(1, t1);
      c->b[0] = 0;
      if (a.kind == MK_ASTOP) {  // the walk stopped above: nothing at this depth
        R.send_path((u32)i, MK_ASTOP);
        c->b[0] = 1;
      } else {
        const u32 l = 2u * a.y, r = l + 1u, jl = l - base, jr = r - base;
        const ull t2 = R.tnow();
        for (u32 q = 0; q < 2; ++q) {  // both children current (their pushes landed)
          const u32 j = q ? jr : jl;
          if (pend[j]) {
            R.wait_pushed(ns[j]);
            pend[j] = 0;
            mn[j] = R.BK(ns[j])[0];
            mx[j] = R.BK(ns[j])[K - 1];
          }
        }
        R.tacc(2, t2);
        R.segmark(1);
        const u32 x = mx[jl] > mx[jr] ? l : r, y = l + r - x;  // l.9 (R6)
        const u32 minc = mn[jl] < mn[jr] ? mn[jl] : mn[jr];
        // early commit (MA_EARLY): the carried keys are R = [a.cmin, a.cmax] at a.src if every
        // level above swapped; with R the walk does not stop here (l.4) iff a.cmax > minc
        a_src = a.src; a_cmin = a.cmin; a_cmax = a.cmax;
        early = !(R.C.debug & 1048576u) && (a.pad & MA_EARLY) && a.cmax > minc;  // debug 1048576: off
        const u32 A = R.alloc(), B = R.alloc();
        c->b[1] = ns[jl]; c->b[2] = ns[jr]; c->b[3] = A; c->b[4] = B; c->b[5] = x; c->b[6] = y;
        c->b[9] = a.slot;
        a_flags = early ? MA_EARLY : 0u;
        c->b[10] = (mx[jl] <= mn[jr] || mx[jr] <= mn[jl]) ? 1u : 0u;
        c->b[13] = minc;
        R.segmark(2);
      }
    }
    cta_bar<DS_NC>();
    if (tid == 0) R.segmark(3);
    if (c->b[0]) continue;
    const u32 sl = c->b[1], sr = c->b[2], A = c->b[3], B = c->b[4];
    const ull t3 = R.tnow();
    ds_split_h<K, V, false>(R, sl, sr, A, B, [&] {  // l.10 (speculative until message b)
      // during the split: y's slot for the level below's push, and the path message to it
      const u32 sy = R.alloc();
      R.arm_slot(sy);
      R.send_path((u32)i, MK_A, c->b[6], sy, a_src, a_cmin, a_cmax, a_flags);
      c->b[7] = sy;
    });
    if (tid == 0) {
      R.segmark(4);
      R.tacc(3, t3);
      const u32 x = c->b[5], y = c->b[6], sy = c->b[7], up = c->b[9];
      const u32 minc = c->b[13];
      c->b[14] = 0;
      if (early && R.BK(A)[K - 1] <= a_cmin) {
        // Early commit.  max(Y_d) <= min(R) implies max(Y_k) <= min(R) at every level k above
        // (max(Y_k) <= max(y_k+1) <= min(children of y_k+1) <= max(Y_k+1), heap order), so every
        // (cur, y) split above was a swap passing R on unchanged, and so is this one: cur <- Y
        // is final now (pushed up before the level above's message b arrives), R sinks on.
        // The push goes first: the level above is waiting for it.
        R.segmark(5);
        R.push_up(A, up);
        R.segmark(6);
        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // all but this push read
        R.release(push_old);
        ++R.n_lev;
        R.n_nomove += c->b[10];
        ++R.n_swap;
        const u32 jx = x - base, jy = y - base;
        R.release(sl); R.release(sr);
        ns[jx] = B; mn[jx] = R.BK(B)[0]; mx[jx] = R.BK(B)[K - 1];
        ns[jy] = sy; pend[jy] = 1;
        push_old = A;
        R.send((u32)i, MK_B, 0, 0, a_src, a_cmin, a_cmax);
        R.segmark(7);
        const ull t4 = R.tnow();
        const DsMsg b = R.recv();  // the level above's message b, consumed in order
        R.segmark(8);
        R.tacc(4, t4);
        if (b.kind != MK_B || b.src != a_src) __trap();  // contradicts the argument above
      } else {
      const ull t4 = R.tnow();
      const DsMsg b = R.recv();  // the carried keys of cur (l.12) from the level above
      R.tacc(4, t4);
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // the previous push's read
      R.release(push_old);
      push_old = DS_NONE;
      if (b.kind == MK_BSTOP) {  // the walk stopped above after all: drop the speculative split
        R.release(A); R.release(B);
        R.disarm_slot(sy);
        R.release(sy);
        R.send((u32)i, MK_BSTOP);
      } else if (b.cmax <= minc) {  // l.4: stop at cur — cur keeps the carried keys
        const u32 s = R.alloc();
        if (b.src & DS_PULL) {  // on chip above: pulled by all threads below, then pushed up
          asm volatile("fence.acq_rel.cluster;" ::: "memory");
          c->b[14] = 2; c->b[4] = s; c->b[9] = up; c->b[15] = b.src;
        } else {
          R.load_node(s, b.src);
          R.push_up(s, up);
          push_old = s;
        }
        R.release(A); R.release(B);
        R.disarm_slot(sy);
        R.release(sy);
        R.send((u32)i, MK_BSTOP);
      } else {
        ++R.n_lev;
        R.n_nomove += c->b[10];
        const u32 ymax = R.BK(A)[K - 1];
        const u32 jx = x - base, jy = y - base;
        R.release(sl); R.release(sr);
        ns[jx] = B; mn[jx] = R.BK(B)[0]; mx[jx] = R.BK(B)[K - 1];
        ns[jy] = sy; pend[jy] = 1;
        if (ymax <= b.cmin) {  // l.12 swap: cur <- Y (pushed up), the carried keys sink on
          ++R.n_swap;
          R.push_up(A, up);
          push_old = A;
          R.send((u32)i, MK_B, 0, 0, b.src, b.cmin, b.cmax);
        } else {  // l.12 merges: (cur, C) <- SORT_SPLIT(carried, Y); C stays on chip (DS_PULL)
          const u32 cs = R.alloc(), lo = R.alloc(), hi = R.alloc();
          if (b.src & DS_PULL) asm volatile("fence.acq_rel.cluster;" ::: "memory");
          else R.load_node(cs, b.src);
          c->b[14] = 1; c->b[4] = cs; c->b[5] = lo; c->b[6] = hi; c->b[7] = y; c->b[9] = up; c->b[12] = A;
          c->b[15] = b.src;
        }
      }
      }
    }
    cta_bar<DS_NC>();
    if (tid == 0) R.segmark(9);
    if (c->b[14] == 2) {  // stop at cur with carried keys on chip above: pull, push up
      const u32 s2 = c->b[4], up = c->b[9], ref = c->b[15];
      R.pull_copy(ref, s2);
      cta_bar<DS_NC>();
      if (tid == 0) {
        R.pull_free(ref);
        R.push_up(s2, up);
        push_old = s2;
      }
    } else if (c->b[14]) {  // a real (cur, y) merge at this depth
      const u32 cs = c->b[4], lo = c->b[5], hi = c->b[6], Y = c->b[12], ref = c->b[15];
      if (ref & DS_PULL) R.pull_copy(ref, cs);
      ds_split<K, V>(R, cs, Y, lo, hi);  // (begins with a CTA barrier)
      if (tid == 0) {
        if (ref & DS_PULL) R.pull_free(ref);
        const u32 up = c->b[9];
        R.push_up(lo, up);
        push_old = lo;
        R.release(cs); R.release(Y);
        R.pull_publish();  // the new carried keys stay in slot hi until a lower level pulled them
        R.send((u32)i, MK_B, 0, 0, R.pull_ref(hi), R.BK(hi)[0], R.BK(hi)[K - 1]);
      }
      cta_bar<DS_NC>();
    }
  }
  // ---- end: pending pushes landed, write the owned nodes back
  if (tid == 0) {
    R.tacc(0, t_start);
    R.flush_counts();
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    for (u32 j = 0; j < cnt; ++j) {
      const u32 n = base + j;
      if (pend[j]) {
        R.wait_pushed(ns[j]);
        pend[j] = 0;
        mn[j] = R.BK(ns[j])[0];
        mx[j] = R.BK(ns[j])[K - 1];
      }
      R.store_node(n, ns[j]);
      st_relaxed(&H.meta[n].kmin, mn[j]);
      st_relaxed(&H.meta[n].kmax, mx[j]);
    }
  }
}

// -----------------------------------------------------------------------------------------
// R(DS_CL-1), the stager: the depth-(DS_CL-1) step on children staged from HBM (LOCKed by its
// helper warp A as soon as the level above names the path node), write-back of x and
// UNLOCK by helper warp B, hand-over of y (still LOCKed) with the carried keys to a walker
// (published early so the walker LOCKs and stages y's children meanwhile).  Owns no nodes:
// the new content of its cur is pushed into the level above.
// -----------------------------------------------------------------------------------------
enum : u32 { WQ_PUBLISH = 1, WQ_COMMIT = 2, WQ_CANCEL = 3, WQ_WB = 4, WQ_UNLOCK = 5, WQ_END = 6 };

template <int K, bool V>
__device__ __forceinline__ void sq_req(DsRole<K, V>& R, u32* head, const u32* done, u32* ring, u32 a0, u32 a1,
                                       u32 a2, u32 a3, u32 a4) {
  const u32 h = *head;
  while (h - ld_acq_cta(done) >= 16u) {}
  u32* e = ring + (h % 16) * 5;
  e[0] = a0; e[1] = a1; e[2] = a2; e[3] = a3; e[4] = a4;
  st_rel_cta(head, h + 1u);
}

template <int K, bool V>
__device__ void ds_stager(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const int tid = threadIdx.x;
  u32 sbp = 0;  // parities of sbar[0..3]
  u32 push_old = DS_NONE;
  const ull t_start = R.tnow();
  for (u64 i = 0; i < m; ++i) {
    if (tid == 0) {
      const ull t2 = R.tnow();
      while (ld_acq_cta(&c->sq_done) <= (u32)i) {}  // op i's children LOCKed and staged (helper A)
      R.tacc(2, t2);
      c->b[0] = 0;
      const u32 e = (u32)i % 16;
      const u32 y4 = c->stg_y[e];
      if (y4 == 0) {  // the walk stopped above
        c->b[0] = 1;
        st_rel_cta(&c->sq_ret, (u32)i + 1u);
      } else {
        const u32 l = 2u * y4, r = l + 1u;
        const u32 sl = DS_NSLOT - 8 + 2 * (u32)(i % 4), sr = sl + 1;
        mbar_wait(&c->sbar[i % 4], sbp >> (i % 4) & 1u);  // the staged data
        sbp ^= 1u << (i % 4);
        const u32 lmin = c->stg_min[e][0], lmax = c->stg_max[e][0], rmin = c->stg_min[e][1], rmax = c->stg_max[e][1];
        const u32 x = lmax > rmax ? l : r, y = l + r - x;  // l.9 (R6)
        sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_PUBLISH, y, 0, 0, 0);
        const u32 A = R.alloc(), B = R.alloc();
        c->b[1] = sl; c->b[2] = sr; c->b[3] = A; c->b[4] = B; c->b[5] = x; c->b[6] = y; c->b[9] = c->stg_up[e];
        c->b[10] = (lmax <= rmin || rmax <= lmin) ? 1u : 0u;
        c->b[13] = lmin < rmin ? lmin : rmin;
        c->b[11] = l; c->b[12] = r;
      }
    }
    cta_bar<DS_NC>();
    if (c->b[0]) continue;
    const u32 sl = c->b[1], sr = c->b[2], A = c->b[3], B = c->b[4];
    const ull t3 = R.tnow();
    ds_split<K, V, false>(R, sl, sr, A, B);
    if (tid == 0) {
      R.tacc(3, t3);
      const u32 x = c->b[5], y = c->b[6], up = c->b[9], minc = c->b[13], l = c->b[11], r = c->b[12];
      const ull t4 = R.tnow();
      const DsMsg b = R.recv();
      R.tacc(4, t4);
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      R.release(push_old);
      push_old = DS_NONE;
      c->b[14] = 0;
      if (b.kind == MK_BSTOP || b.cmax <= minc) {  // stopped above / at cur: nothing changes below
        if (b.kind != MK_BSTOP) {                  // cur keeps the carried keys
          const u32 s = R.alloc();
          if (b.src & DS_PULL) {
            asm volatile("fence.acq_rel.cluster;" ::: "memory");
            c->b[14] = 2; c->b[4] = s; c->b[9] = up; c->b[15] = b.src;
          } else {
            R.load_node(s, b.src);
            R.push_up(s, up);
            push_old = s;
          }
        }
        sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_CANCEL, y, l, r, 0);
        R.release(A); R.release(B);
        st_rel_cta(&c->sq_ret, (u32)i + 1u);
      } else {
        ++R.n_lev;
        R.n_nomove += c->b[10];
        st_rel_cta(&c->sq_ret, (u32)i + 1u);  // the staged children were only split inputs
        // x <- X: HBM write-back, then UNLOCK(x) (helper B, l.11); it frees slot B
        sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_WB, x, B, R.BK(B)[0], R.BK(B)[K - 1]);
        const u32 ymax = R.BK(A)[K - 1];
        if (ymax <= b.cmin) {  // l.12 swap: cur <- Y, the carried keys go on to y's walker
          ++R.n_swap;
          R.push_up(A, up);
          push_old = A;
          if (b.src & DS_PULL) {  // on chip above: pull them and store them in y's HBM copy
            asm volatile("fence.acq_rel.cluster;" ::: "memory");
            c->b[14] = 3; c->b[4] = R.alloc(); c->b[7] = y; c->b[15] = b.src;
          } else {
            sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_COMMIT, y, b.src, 0, 0);
          }
        } else {
          const u32 cs = R.alloc(), lo = R.alloc(), hi = R.alloc();
          if (b.src & DS_PULL) asm volatile("fence.acq_rel.cluster;" ::: "memory");
          else R.load_node(cs, b.src);
          c->b[14] = 1; c->b[4] = cs; c->b[5] = lo; c->b[6] = hi; c->b[7] = y; c->b[9] = up; c->b[12] = A;
          c->b[15] = b.src;
        }
      }
    }
    cta_bar<DS_NC>();
    if (c->b[14] == 2 || c->b[14] == 3) {  // carried keys on chip above: pull them
      const u32 s2 = c->b[4], ref = c->b[15], mode = c->b[14];
      R.pull_copy(ref, s2);
      cta_bar<DS_NC>();
      if (tid == 0) {
        R.pull_free(ref);
        if (mode == 2) {  // stop at cur: cur <- the carried keys
          R.push_up(s2, c->b[9]);
          push_old = s2;
        } else {  // swap: the walker below y reads them from y's HBM copy (y is LOCKed by us)
          const u32 y = c->b[7];
          R.store_node(y, s2);
          __threadfence();
          R.release(s2);
          sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_COMMIT, y, y, 0, 0);
        }
      }
      cta_bar<DS_NC>();
    } else if (c->b[14]) {  // a real (cur, y) merge
      const u32 cs = c->b[4], lo = c->b[5], hi = c->b[6], Y = c->b[12], ref = c->b[15];
      if (ref & DS_PULL) R.pull_copy(ref, cs);
      ds_split<K, V>(R, cs, Y, lo, hi);
      if (tid == 0) {
        if (ref & DS_PULL) R.pull_free(ref);
        const u32 y = c->b[7], up = c->b[9];
        R.store_node(y, hi);  // the carried keys in y's HBM copy (y is LOCKed by us)
        __threadfence();
        R.push_up(lo, up);
        push_old = lo;
        R.release(cs); R.release(Y); R.release(hi);
        sq_req<K, V>(R, &c->wq_head, &c->wq_done, c->wq, WQ_COMMIT, y, y, 0, 0);
      }
      cta_bar<DS_NC>();
    }
    if (tid == 0) {  // slots the write-back helper finished with
      const u32 fr = atomicExch(&c->wb_free, 0u);
      R.fm |= fr;
    }
  }
  if (tid == 0) {
    R.tacc(0, t_start);
    R.flush_counts();
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

// stager helper A (lane 0 of warp DS_NT/32): reads the path messages "a" from the second inbox
// as they arrive (up to 4 ops ahead of thread 0), LOCKs and stages the two children of each
// path node (in op order) into its own slot ring, and publishes one record per op.
template <int K, bool V>
__device__ void ds_stage_helper(DsRole<K, V>& R, const u64 m) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  for (u32 k = 0; k < (u32)m; ++k) {
    const u32 e = k % DS_RING;
    mbar_wait(&c->ainbar[e], (k / DS_RING) & 1u);
    const u32 kind = c->ainbox[e].kind, y = c->ainbox[e].y, up = c->ainbox[e].slot;
    mbar_arrive_expect_tx(&c->ainbar[e], (u32)sizeof(DsMsg));  // re-arm
    if ((k + 1) % DS_CREDIT == 0)
      asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(cl_map(&c->aconsumed, R.rank - 1)),
                   "r"(k + 1) : "memory");
    const u32 q = k % 16;
    while (k >= ld_acq_cta(&c->sq_ret) + 4u) {}  // op k - 4 done: its record and staging slots are free
    if (kind == MK_ASTOP) {
      c->stg_y[q] = 0;
    } else {
      const u32 n0 = 2u * y, n1 = n0 + 1u;
      const u32 s0 = DS_NSLOT - 8 + 2 * (k % 4), s1 = s0 + 1;
      const ull tl = R.tnow();
      lock_acquire(&H.meta[n0].lock);  // l.3: LOCK(l); LOCK(r)
      lock_acquire(&H.meta[n1].lock);
      R.tacc(1, tl);  // timers: the stager's "wait-above" column = helper A's LOCK time
      fence_proxy_async();
      u64* bar = &c->sbar[k % 4];  // thread 0 waits for the data; this helper moves on
      mbar_arrive_expect_tx(bar, 2u * DsRole<K, V>::SLOTB);
      bulk_g2s(R.BK(s0), H.gk + (size_t)n0 * K, DsRole<K, V>::NB, bar);
      bulk_g2s(R.BK(s1), H.gk + (size_t)n1 * K, DsRole<K, V>::NB, bar);
      if (V) {
        bulk_g2s(R.BV(s0), H.gv + (size_t)n0 * K, DsRole<K, V>::NB, bar);
        bulk_g2s(R.BV(s1), H.gv + (size_t)n1 * K, DsRole<K, V>::NB, bar);
      }
      u32 st0, st1, mn0, mx0, mn1, mx1;
      meta_load(&H.meta[n0], st0, mn0, mx0);
      meta_load(&H.meta[n1], st1, mn1, mx1);
      c->stg_min[q][0] = mn0; c->stg_max[q][0] = mx0;
      c->stg_min[q][1] = mn1; c->stg_max[q][1] = mx1;
      c->stg_y[q] = y;
      c->stg_up[q] = up;
    }
    st_rel_cta(&c->sq_done, k + 1u);
  }
}

// stager helper B (lane 0 of warp DS_NT/32 + 1): walker tasks, write-backs, UNLOCKs
template <int K, bool V>
__device__ void ds_wb_helper(DsRole<K, V>& R) {
  DsCtl* c = R.c;
  const HeapArgs& H = R.H;
  u32 seen = 0, tasks = 0, go_next = 0;
  for (;;) {
    const u32 head = ld_acq_cta(&c->wq_head);
    if (seen == head) {
      if (ld_acq_cta(&c->quit)) break;
      continue;
    }
    const u32* e = c->wq + (seen % 16) * 5;
    const u32 kind = e[0];
    if (kind == WQ_PUBLISH) {  // y is LOCKed (staged by helper A): task visible, carried keys later
      st_relaxed(R.D.task_node + tasks, e[1]);
      st_release(R.D.task_seq + tasks, R.D.epoch);
      ++tasks;
    } else if (kind == WQ_COMMIT || kind == WQ_CANCEL) {
      // a merged carried set was stored to HBM by thread 0 (wait_group + __threadfence) before
      // its request, which this thread acquired
      const u32 t = go_next++;
      st_release_u64(R.D.task_go + t, ((u64)R.D.epoch << 32) | (kind == WQ_COMMIT ? e[2] : 0xFFFFFFFFu));
      if (kind == WQ_CANCEL) {  // y and its sibling stay as they were: UNLOCK both
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        st_relaxed(&H.meta[e[2]].lock, 0u);
        st_relaxed(&H.meta[e[3]].lock, 0u);
      }
    } else if (kind == WQ_WB) {  // Alg.3 l.10-11: x <- X, UNLOCK(x)
      const ull tw = R.tnow();
      const u32 x = e[1], B = e[2];
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      bulk_s2g(H.gk + (size_t)x * K, R.BK(B), DsRole<K, V>::NB);
      if (V) bulk_s2g(H.gv + (size_t)x * K, R.BV(B), DsRole<K, V>::NB);
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
      st_relaxed(&H.meta[x].kmin, e[3]);
      st_relaxed(&H.meta[x].kmax, e[4]);
      asm volatile("fence.proxy.async.global;" ::: "memory");
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
      st_relaxed(&H.meta[x].lock, 0u);
      atomicOr(&c->wb_free, 1u << B);
      R.tacc(5, tw);  // timers: the stager's "sends" column = helper B's write-back time
    }
    ++seen;
    st_rel_cta(&c->wq_done, seen);
  }
  st_release(R.D.ctl + 1, tasks + 1u);  // walkers: the final task count
}

template <int K, bool V>
__global__ void __cluster_dims__(DS_CL, 1, 1) __launch_bounds__(DS_BLOCK, 1)
    bgpq_dsys_kernel(HeapArgs H, CallArgs C, DtArgs D) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const u64 m = ds_ops(H, C, K);
  if (blockIdx.x < DS_CL) {
    DsCtl* c = reinterpret_cast<DsCtl*>(smem_raw);
    DsRole<K, V> R;
    R.H = H; R.C = C; R.D = D; R.c = c;
    R.sk = reinterpret_cast<u32*>(smem_raw + DSCTL_BYTES);
    R.sv = R.sk + DS_NSLOT * K;
    R.rank = cl_rank();
    // the stager keeps its last 8 slots for staging (helper A's ring)
    R.fm = (R.rank == DS_CL - 1) ? ((1u << (DS_NSLOT - 8)) - 1u) : ((1u << DS_NSLOT) - 1u);
    R.sbph = 0; R.in_seq = 0; R.out_seq = 0; R.out_seq2 = 0; R.lph = 0;
    R.timing = (C.debug & 1024u) != 0;
    R.seg = (C.debug & 2097152u) != 0 && cl_rank() == 1;
    if (threadIdx.x == 0) {
      for (u32 e = 0; e < DS_RING; ++e) mbar_init(&c->inbar[e], 1);
      for (u32 e = 0; e < DS_RING; ++e) R.arm_inbox(e);
      for (u32 s = 0; s < DS_NSLOT; ++s) mbar_init(&c->slotbar[s], 1);
      mbar_init(&c->lbar, 1);
      mbar_init(&c->hbar, 1);
      for (int q = 0; q < 4; ++q) mbar_init(&c->sbar[q], 1);
      c->consumed = 0; c->rf_seq = 0; c->rf_used = 0; c->tasks = 0; c->quit = 0; c->pfreed = 0;
      c->sq_done = 0; c->sq_ret = 0; c->wq_head = 0; c->wq_done = 0; c->wb_free = 0; c->aconsumed = 0;
      for (u32 e = 0; e < DS_RING; ++e) {
        mbar_init(&c->ainbar[e], 1);
        mbar_arrive_expect_tx(&c->ainbar[e], (u32)sizeof(DsMsg));
      }
      for (int q = 0; q < NSTAT; ++q) c->st[q] = 0;
      for (int q = 0; q < 8; ++q) c->tm[q] = 0;
      for (int q = 0; q < 16; ++q) c->tm2[q] = 0;
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    cluster_sync_all();  // every barrier of the cluster initialised before any remote copy
    const bool stager = R.rank == DS_CL - 1;
    if (threadIdx.x >= DS_NC) {
      if (threadIdx.x == DS_NC) {
        if (R.rank == 0) { if (C.mode != MODE_MIXED) ds_r0_helper<K, V>(R, m); }
        else if (stager) ds_stage_helper<K, V>(R, m);
      } else if (threadIdx.x == DS_NC + 32 && stager) {
        ds_wb_helper<K, V>(R);
      }
    } else {
      if (m) {
        if (R.rank == 0) {
          if (C.mode == MODE_MIXED) ds_r0_mixed<K, V>(R, m);
          else ds_r0<K, V>(R, m);
        }
        else if (stager) ds_stager<K, V>(R, m);
        else ds_level<K, V>(R, m);
      } else if (threadIdx.x == 0 && R.rank == 0) {
        *reinterpret_cast<volatile u64*>(D.op_base) = 0;
      }
      cta_bar<DS_NC>();
      if (threadIdx.x == 0) st_rel_cta(&c->quit, 1u);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
      for (int q = 0; q < NSTAT; ++q)
        if (c->st[q]) atomicAdd(stat + q, c->st[q]);
      if (R.timing) {
        ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
        for (int q = 0; q < 6; ++q) atomicAdd(tms + 6 * R.rank + q, c->tm[q]);
      }
      if (R.seg) {
        ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
        for (int q = 0; q < 16; ++q) atomicAdd(tms + q, c->tm2[q]);
      }
    }
    cluster_sync_all();  // no CTA leaves while a peer may still access its shared memory
    return;
  }
  dt_walkers<K, V, DS_NT>(H, C, D, smem_raw);
}

// Mixed calls on the cluster engine, step 1: Alg.1 l.2 (Sort(items), done before the root is
// locked) for every op pair (INSERT(K), DELETEMIN(K)) at the call's start, into H.xk + p*K, and
// the first op pair of another shape (atomicMin into *C.pair_end, preset to all-ones).  Pairs
// after that one are left unsorted (the per-node-lock engine executes them).
template <int K, bool V, int NT>
__global__ void __launch_bounds__(NT, 1) bgpq_msort_kernel(HeapArgs H, CallArgs C) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  u32* ak = reinterpret_cast<u32*>(smem_raw);
  u32* tk = ak + K;
  u32* av = V ? tk + K : nullptr;
  u32* tv = V ? av + K : nullptr;
  u32* pe = const_cast<u32*>(C.pair_end);
  const u64 np = C.n_ops / 2;
  __shared__ u32 go;
  for (u64 p = blockIdx.x; p < np; p += gridDim.x) {
    const u64 j = 2 * p;
    if (threadIdx.x == 0) {  // one thread decides: the CTA leaves the loop as a whole
      go = 0;
      if (p < *reinterpret_cast<volatile const u32*>(pe)) {
        if (C.op_types[j] == 0 && C.op_types[j + 1] == 1 && C.op_sizes[j] == (u32)K && C.op_sizes[j + 1] == (u32)K)
          go = 1;
        else
          atomicMin(pe, (u32)p);
      }
    }
    cta_bar<NT>();
    if (!go) break;
    const u32* ik = C.in_k + C.in_off[j];
    const u32* iv = C.in_v ? C.in_v + C.in_off[j] : nullptr;
    for (int e = threadIdx.x; e < K; e += NT) {
      ak[e] = ik[e];
      if (V) av[e] = iv ? iv[e] : 0u;
    }
    cta_bar<NT>();
    const bool swapped = cta_sort<K, NT, V>(ak, av, K, tk, tv);
    cta_bar<NT>();
    const uint4* sk = reinterpret_cast<const uint4*>(swapped ? tk : ak);
    uint4* dk = reinterpret_cast<uint4*>(H.xk + p * (u64)K);
    for (int e = threadIdx.x; e < K / 4; e += NT) dk[e] = sk[e];
    if (V) {
      const uint4* sv = reinterpret_cast<const uint4*>(swapped ? tv : av);
      uint4* dv = reinterpret_cast<uint4*>(H.xv + p * (u64)K);
      for (int e = threadIdx.x; e < K / 4; e += NT) dv[e] = sv[e];
    }
    cta_bar<NT>();
  }
}
template <int K, bool V>
constexpr size_t msort_smem_bytes() { return (size_t)2 * K * 4 * (V ? 2 : 1); }

}  // namespace bgpqd
