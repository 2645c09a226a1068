// bgpq_locks.cuh — the paper's per-node-lock execution of BGPQ (one operation per CTA,
// locks taken top-down hand over hand, TARGET/MARKED hand-off), restructured for B200's
// latencies: every CTA runs NT compute threads plus one "lock warp" whose lanes act as two
// agents that take node locks and stage node data while the compute threads merge.
//
// Why: one inter-SM lock hand-off through L2 costs ~800-1500 cycles and a 4 KB node stage-in
// ~400-1000 cycles on B200, the same order as a 2K-entry SORT_SPLIT (~1500 cycles, see
// tools/micro_merge.cu).  The serial chain of DELETEMINs (each needs the previous one's
// level-1 result, Alg.3 l.11-15) therefore pays lock + load latency at every level.  Here:
//   agent P (lane 0): LOCK(l); LOCK(r) + TMA stage-in of the children of the node the walk
//            will visit next ("lock-ahead"): issued as soon as y is chosen at the current
//            level (Alg.3 l.9 needs only the cached max keys), so the next level's locks and
//            data arrive while the current level's SORT_SPLITs run.  Locks are still
//            acquired top-down (depth order), so the deadlock-freedom argument of P:172 holds.
//            INSERT walks use it for NEXT(cur, tar) (Alg.1 l.32-34).
//   agent T (lane 1): the refill of DELETEMIN (Alg.2 l.6-12): LOCK(tar), TARGET -> MARKED
//            hand-off or Heap[root] <- Heap[tar], UNLOCK(tar) — concurrently with LOCK of the
//            root's children by agent P.  The root lock is released only after T is done, so
//            the take still happens inside the root critical section.
// Correspondence with the paper: insert() = Alg.1, deletemin() = Alg.2 + Alg.3 (readings
// R1-R15).  Same heap arena and metadata as bgpq_ops.cuh.
#pragma once
#include "bgpq_ops.cuh"

namespace bgpqd {

constexpr int LSLOT = 10;  // smem node slots
#ifndef BGPQ_T_MARK
#define BGPQ_T_MARK 1
#endif
#ifndef BGPQ_JOINT_RELEASE
#define BGPQ_JOINT_RELEASE 1
#endif
#ifndef BGPQ_PREFETCH
#define BGPQ_PREFETCH 1
#endif
#ifndef BGPQ_HDR_BATCH
#define BGPQ_HDR_BATCH 1
#endif

struct LCtl {
  u64 bar;      // compute-thread TMA loads
  u64 pbar[2];  // agent P completions (alternating)
  u64 tbar;     // agent T completion
  u32 op;
  u32 freemask;  // free slot bitmask (thread 0)
  u32 b[24];     // thread-0 broadcasts
  // agent P mailbox
  u32 p_req;
  u32 p_n[2], p_s[2], p_bi, p_force;
  u32 p_st[2], p_min[2], p_max[2];
  // agent T mailbox
  u32 t_req;
  u32 t_kind;  // 0: take the refill node (Alg.2 l.6-12); 1: mark tar TARGET (Alg.1 l.5-6)
  u32 t_node, t_slot, t_rootload, t_rootpar;
  u32 t_marked;
  u32 t_done;
  u32 stop;
  ull st[NSTAT];  // thread 0's device counters (shared memory: gpu-scope acquires and fences
  ull tm[32];     // invalidate L1, so local-memory counters would cost an L2 round trip)
};
constexpr size_t LCTL_BYTES = (sizeof(LCtl) + 127) / 128 * 128;  // node slots start here

__device__ __forceinline__ u32 ld_acq_cta(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_addr(p)) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel_cta(u32* p, u32 v) {
  asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(smem_addr(p)), "r"(v) : "memory");
}
__device__ __forceinline__ u32 mbar_test(u64* bar, u32 phase) {
  u32 ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok) : "r"(smem_addr(bar)), "r"(phase) : "memory");
  return ok;
}

// phase timers (thread 0, cycles; enabled by CallArgs.debug & 8, accumulated in H_TIME)
enum : int {
  LT_DEL_TOTAL = 0, LT_DEL_ROOTACQ, LT_DEL_ROOTHOLD, LT_DEL_ROOTLOAD, LT_DEL_TWAIT, LT_DEL_PWAIT,
  LT_DEL_MERGE, LT_DEL_STORE, LT_DEL_LEVELS, LT_INS_TOTAL, LT_INS_SORT, LT_INS_ROOTACQ,
  LT_INS_ROOTHOLD, LT_INS_PWAIT, LT_INS_MERGE, LT_INS_STORE, LT_INS_TARWAIT, LT_P_LOCKWAIT,
  LT_T_LOCKWAIT, LT_T_TOTAL, LT_R1, LT_R2, LT_R3, LT_R4, LT_R5, LT_R6, LT_R7, LT_N
};

template <int K, bool V, int NT>
struct OpL {
  static constexpr u32 NBYTES = K * 4u;
  HeapArgs H;
  bool timing;
  // schedule forcing (test only, bgpq_set_debug bit 32768): an INSERT holds its target node in
  // state TARGET this many ns before the placement (Alg.1 l.8-13), so concurrent DELETEMINs
  // meet the in-flight insert: the refill steals it (TARGET -> MARKED, Alg.2 l.7-9) and
  // heapify walks see exactly one AVAIL child (R5)
  u32 delay_ns = 0;
  ull* tm;  // -> ctl->tm
  int tmerge = LT_DEL_MERGE, tstore = LT_DEL_STORE;  // timer ids of the current op type
  __device__ __forceinline__ ull now() const { return timing ? clock64() : 0ull; }
  __device__ __forceinline__ void acc(int id, ull t0) { if (timing && threadIdx.x == 0) tm[id] += clock64() - t0; }
  ull tmark;  // root-hold section marks (thread 0)
  __device__ __forceinline__ void mark(int id) {
    if (timing && threadIdx.x == 0) { const ull t = clock64(); tm[id] += t - tmark; tmark = t; }
  }
  u32* sk;
  u32* sv;
  LCtl* ctl;
  u32 mphase;      // ctl->bar phase (all compute threads)
  u32 pph;         // pbar[0] / pbar[1] phases in bits 0 / 1 (registers, not a local array)
  u32 tphase;      // tbar phase (all compute threads)
  u32 pb;          // next pbar index
  ull* st;         // -> ctl->st (thread 0's counters)

  __device__ __forceinline__ u32* BK(int s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(int s) const { return V ? sv + s * K : nullptr; }
  __device__ __forceinline__ u32 hget(int w) const { return ld_relaxed(H.hdr + w); }
  __device__ __forceinline__ void hset(int w, u32 v) const { st_relaxed(H.hdr + w, v); }
  __device__ __forceinline__ u32* lk(u32 node) const { return &H.meta[node].lock; }
  __device__ __forceinline__ u32* stp(u32 node) const { return &H.meta[node].state; }
  __device__ __forceinline__ void set_minmax(u32 node, u32 mn, u32 mx) const {
    st_relaxed(&H.meta[node].kmin, mn);
    st_relaxed(&H.meta[node].kmax, mx);
  }
  // ---- slot allocation (thread 0 only)
  __device__ __forceinline__ int alloc() {
    const u32 m = ctl->freemask;
    const int s = __ffs(m) - 1;
    ctl->freemask = m & ~(1u << s);
    return s;
  }
  __device__ __forceinline__ void free_slot(int s) { ctl->freemask |= (1u << s); }

  // ---- synchronous TMA stage-in by the compute threads
  __device__ __forceinline__ void load(int s, u32 node) {
    cta_bar<NT>();
    if (threadIdx.x == 0) {
      fence_proxy_async();
      mbar_arrive_expect_tx(&ctl->bar, V ? 2u * NBYTES : NBYTES);
      bulk_g2s(BK(s), src_keys<K>(H, node), NBYTES, &ctl->bar);
      if (V) bulk_g2s(BV(s), src_vals<K>(H, node), NBYTES, &ctl->bar);
    }
    mbar_wait(&ctl->bar, mphase);
    mphase ^= 1u;
  }
  // coalesced 128-bit write-back; ends with a barrier so thread 0 may publish it
  __device__ __forceinline__ void store(u32 node, int s) {
    cta_bar<NT>();
    const ull t0 = now();
    uint4* dk = reinterpret_cast<uint4*>(H.gk + (size_t)node * K);
    const uint4* srck = reinterpret_cast<const uint4*>(BK(s));
    for (int i = threadIdx.x; i < K / 4; i += NT) dk[i] = srck[i];
    if (V) {
      uint4* dv = reinterpret_cast<uint4*>(H.gv + (size_t)node * K);
      const uint4* srcv = reinterpret_cast<const uint4*>(BV(s));
      for (int i = threadIdx.x; i < K / 4; i += NT) dv[i] = srcv[i];
    }
    cta_bar<NT>();
    acc(tstore, t0);
  }
  __device__ __forceinline__ void merge_split(int z, int na, int w, int nb, int ma, int x, int y) {
    cta_bar<NT>();
    const ull t0 = now();
    sort_split<K, NT, V>(BK(z), BV(z), na, BK(w), BV(w), nb, ma, BK(x), BV(x), BK(y), BV(y));
    cta_bar<NT>();
    acc(tmerge, t0);
  }
  __device__ __forceinline__ void shift(int dst, int src, int off, int n) {
    cta_bar<NT>();
    for (int i = threadIdx.x; i < n; i += NT) {
      BK(dst)[i] = BK(src)[i + off];
      if (V) BV(dst)[i] = BV(src)[i + off];
    }
    cta_bar<NT>();
  }
  __device__ __forceinline__ void emit(u32* ok, u32* ov, u32 pos, int s, int off, int n) {
    for (int i = threadIdx.x; i < n; i += NT) {
      ok[pos + i] = BK(s)[off + i];
      if (V && ov) ov[pos + i] = BV(s)[off + i];
    }
  }
  // One round trip for the words the root lock protects: {heapSize, |root|, |pBuffer|, err},
  // the per-call ticket, the 64-bit linearization ticket, min(pBuffer) and max(root).
  struct Hdr { u32 hs, rs, ps, call, pbmin, rootmax; ull lin; };
  __device__ __forceinline__ Hdr hdr_load() const {
    Hdr h;
#if !BGPQ_HDR_BATCH
    h.lin = lin_get(); h.call = hget(H_CALL); h.hs = hget(H_HS); h.rs = hget(H_RS); h.ps = hget(H_PS);
    h.pbmin = ld_relaxed(&H.meta[0].kmin); h.rootmax = ld_relaxed(&H.meta[1].kmax);
    return h;
#endif
    u32 err;
    asm volatile(
        "ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%7];\n\t"
        "ld.relaxed.gpu.global.u32 %4, [%8];\n\t"
        "ld.relaxed.gpu.global.u64 %5, [%9];\n\t"
        "ld.relaxed.gpu.global.u32 %6, [%10];"
        : "=r"(h.hs), "=r"(h.rs), "=r"(h.ps), "=r"(err), "=r"(h.call), "=l"(h.lin), "=r"(h.pbmin)
        : "l"(H.hdr), "l"(H.hdr + H_CALL), "l"(H.hdr + H_LIN), "l"(&H.meta[0].kmin)
        : "memory");
    h.rootmax = ld_relaxed(&H.meta[1].kmax);
    return h;
  }
  // release several node locks behind one gpu-scope fence (the caller's CTA barrier has
  // ordered every thread's node writes before this thread)
  __device__ __forceinline__ void release_locks(u32 a, u32 b = 0) const {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    if (a) st_relaxed(lk(a), 0u);
    if (b) st_relaxed(lk(b), 0u);
  }
  __device__ __forceinline__ void prefetch_l2(u32 node) const {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gk + (size_t)node * K), "r"(NBYTES) : "memory");
    if (V) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(H.gv + (size_t)node * K), "r"(NBYTES) : "memory");
  }
  __device__ __forceinline__ ull lin_get() const {
    ull v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(H.hdr + H_LIN) : "memory");
    return v;
  }
  __device__ __forceinline__ void lin_set(ull v) const {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(H.hdr + H_LIN), "l"(v) : "memory");
  }

  // ---- agent requests (thread 0).  P: lock n0, n1 (0 = none) top-down and stage them into
  // slots s0, s1 (if AVAIL, or always when force); completion on pbar[pb].
  __device__ __forceinline__ void post_p(u32 n0, u32 n1, int s0, int s1, u32 force) {
    ctl->p_n[0] = n0; ctl->p_n[1] = n1; ctl->p_s[0] = (u32)s0; ctl->p_s[1] = (u32)s1;
    ctl->p_bi = pb; ctl->p_force = force;
    st_rel_cta(&ctl->p_req, ctl->p_req + 1u);
  }
  // compute threads: wait for the P request issued on pbar[pb]; advances pb
  __device__ __forceinline__ void wait_p(int id) {
    const ull t0 = now();
    mbar_wait(&ctl->pbar[pb], (pph >> pb) & 1u);
    acc(id, t0);
    pph ^= 1u << pb;
    pb ^= 1u;
  }
  __device__ __forceinline__ void post_mark(u32 tar) {
    ctl->t_kind = 1u; ctl->t_node = tar;
    st_rel_cta(&ctl->t_req, ctl->t_req + 1u);
  }
  __device__ __forceinline__ void wait_t_done() const {
    while (ld_acq_cta(&ctl->t_done) != ctl->t_req) {}
  }
  __device__ __forceinline__ void post_t(u32 tar, int slot, u32 rootload) {
    ctl->t_kind = 0u;
    ctl->t_node = tar; ctl->t_slot = (u32)slot; ctl->t_rootload = rootload; ctl->t_rootpar = mphase;
    st_rel_cta(&ctl->t_req, ctl->t_req + 1u);
  }

  // =====================================================================================
  // BGPQ_INSERT (Alg.1).  Keys ik[0:size), values iv (nullable), 1 <= size <= K.
  // =====================================================================================
  __device__ __forceinline__ void insert(const u32* ik, const u32* iv, u32 size, ull* lin_out) {
    const int tid = threadIdx.x;
    tmerge = LT_INS_MERGE; tstore = LT_INS_STORE;
    const ull t_ins = now();
    tmark = t_ins;
    cta_bar<NT>();
    if (tid == 0) {
      ctl->b[0] = alloc();
      ctl->b[1] = alloc();
    }
    cta_bar<NT>();
    int it = (int)ctl->b[0], tmp = (int)ctl->b[1];
    for (int i = tid; i < K; i += NT) {
      BK(it)[i] = i < (int)size ? ik[i] : KEY_MAX;
      if (V) BV(it)[i] = (i < (int)size && iv) ? iv[i] : 0u;
    }
    cta_bar<NT>();
    // l.2: items[1:size] <- Sort(items[1:size])   (before the root is locked)
    if (cta_sort<K, NT, V>(BK(it), BV(it), (int)size, BK(tmp), BV(tmp))) { int t = it; it = tmp; tmp = t; }
    acc(LT_INS_SORT, t_ins);
    // l.3: LOCK(root)
    ull t_root = 0;
    if (tid == 0) {
      free_slot(tmp);
      st[S_INS_OPS]++;
      const ull ta = now();
      st[S_ROOT_SPINS] += lock_acquire(lk(1));
      acc(LT_INS_ROOTACQ, ta);
      t_root = now();
      fence_proxy_async();
      const Hdr h = hdr_load();
      lin_set(h.lin + 1);
      if (lin_out) *lin_out = h.lin;
      ctl->b[0] = h.hs;
      ctl->b[1] = h.rs;
      ctl->b[2] = h.ps;
      ctl->b[3] = h.rootmax;
    }
    cta_bar<NT>();
    const u32 hs = ctl->b[0], rs = ctl->b[1], ps = ctl->b[2], rootmax = ctl->b[3];
    u32 imin = BK(it)[0], imax = BK(it)[size - 1];
    // ---- PARTIAL_INSERT (l.15-29)
    if (hs == 0) {  // l.16-19: the heap is empty
      store(1, it);
      if (tid == 0) {
        free_slot(it);
        set_minmax(1, imin, imax);
        st_relaxed(stp(1), ST_AVAIL);
        hset(H_RS, size);
        hset(H_HS, 1);
        lock_release(lk(1));
      }
      return;
    }
    // l.20: (root, items) <- SORT_SPLIT(root, |root|, items, size, |root|)
    if (rs > 0 && !(rootmax <= imin)) {
      if (tid == 0) { ctl->b[4] = alloc(); ctl->b[5] = alloc(); ctl->b[6] = alloc(); }
      cta_bar<NT>();
      const int rsl = (int)ctl->b[4], a = (int)ctl->b[5], b = (int)ctl->b[6];
      load(rsl, 1);
      merge_split(rsl, rs, it, size, rs, a, b);
      store(1, a);
      if (tid == 0) {
        set_minmax(1, BK(a)[0], BK(a)[rs - 1]);
        free_slot(rsl); free_slot(a); free_slot(it);
      }
      it = b;
      imin = BK(it)[0];
      imax = BK(it)[size - 1];
    }
    if (ps + size < (u32)K) {  // l.21-24: append to the buffer (kept sorted, R1/R2)
      int res = it;
      if (ps > 0) {
        cta_bar<NT>();
        if (tid == 0) { ctl->b[4] = alloc(); ctl->b[5] = alloc(); ctl->b[6] = alloc(); }
        cta_bar<NT>();
        const int p = (int)ctl->b[4], a = (int)ctl->b[5], b = (int)ctl->b[6];
        load(p, 0);
        merge_split(p, ps, it, size, ps + size, a, b);
        if (tid == 0) { free_slot(p); free_slot(b); free_slot(it); }
        res = a;
      }
      store(0, res);
      if (tid == 0) {
        free_slot(res);
        set_minmax(0, BK(res)[0], BK(res)[ps + size - 1]);
        hset(H_PS, ps + size);
        lock_release(lk(1));
      }
      return;
    }
    // l.26-28: (items[1:K], pBuffer) <- SORT_SPLIT(items, size, pBuffer, |pB|, K)
    const u32 nps = ps + size - K;
    if (ps > 0) {
      cta_bar<NT>();
      if (tid == 0) { ctl->b[4] = alloc(); ctl->b[5] = alloc(); ctl->b[6] = alloc(); }
      cta_bar<NT>();
      const int p = (int)ctl->b[4], a = (int)ctl->b[5], b = (int)ctl->b[6];
      load(p, 0);
      merge_split(it, size, p, ps, K, a, b);
      if (nps > 0) store(0, b);
      if (tid == 0) {
        if (nps > 0) set_minmax(0, BK(b)[0], BK(b)[nps - 1]);
        free_slot(p); free_slot(b); free_slot(it);
      }
      it = a;
      imin = BK(it)[0];
      imax = BK(it)[K - 1];
    }
    // l.4: heapSize <- heapSize + 1; tar <- heapSize
    const u32 tar = hs + 1;
    if (tar > H.cap) {  // R15: sticky capacity error, the batch is dropped
      cta_bar<NT>();
      if (tid == 0) {
        free_slot(it);
        hset(H_PS, nps);
        hset(H_ERR, (u32)(-3));
        lock_release(lk(1));
      }
      return;
    }
    u32 c = next_on_path(1, tar);
    cta_bar<NT>();
    if (tid == 0) {
      st[S_INS_HEAPIFY]++;
      hset(H_PS, nps);
      hset(H_HS, tar);
      // l.5-6: LOCK(tar); Heap[tar].state <- TARGET; UNLOCK(tar) — by agent T; the root is
      // not released before it is done
#if BGPQ_T_MARK
      post_mark(tar);
#else
      lock_acquire(lk(tar));
      st_relaxed(stp(tar), ST_TARGET);
      lock_release(lk(tar));
#endif
      if (c != tar) {  // lock-ahead of the first path node (still holding the root)
        const int s = alloc();
        ctl->b[7] = (u32)s;
        post_p(c, 0, s, 0, 1u);
      }
    }
    cta_bar<NT>();
    // ---- l.7, l.30-34: INSERT_HEAPIFY(NEXT(root, tar), tar, items), hand over hand
    u32 held = 1;
    int sc = (int)ctl->b[7];
    while (c != tar) {
      wait_p(LT_INS_PWAIT);  // cur is locked (by agent P) and staged in slot sc
      const u32 nx = next_on_path(c, tar);
      if (tid == 0) {
        const u32 brk = ld_relaxed(stp(tar)) == ST_MARKED;  // l.31
        u32 dec = 0;
        const u32 cmin = ctl->p_min[0], cmax = ctl->p_max[0];
        if (brk) {
          lock_release(lk(c));  // as if the loop had exited before LOCK(cur)
          free_slot(sc);
        } else {
          if (held == 1) wait_t_done();
          lock_release(lk(held));  // l.32: UNLOCK(PARENT(cur)) — cur is held
          if (held == 1) acc(LT_INS_ROOTHOLD, t_root);
          dec = (cmax <= imin) ? 0u : (imax <= cmin) ? 1u : 2u;  // l.33 fast paths
          st[S_INS_LEVELS]++;
          st[dec == 0 ? S_INS_NOOP : dec == 1 ? S_INS_SWAP : S_INS_MERGE]++;
          if (nx != tar) {  // lock-ahead: NEXT(cur, tar) while this level merges
            const int s = alloc();
            ctl->b[7] = (u32)s;
            post_p(nx, 0, s, 0, 1u);
          }
          if (dec == 2) { ctl->b[4] = alloc(); ctl->b[5] = alloc(); }
        }
        ctl->b[0] = brk; ctl->b[1] = dec; ctl->b[2] = cmin; ctl->b[3] = cmax;
      }
      cta_bar<NT>();
      const u32 brk = ctl->b[0], dec = ctl->b[1];
      if (brk) break;
      const int nsc = (int)ctl->b[7];
      if (dec == 1) {  // node <- items, items <- node
        const u32 cmin = ctl->b[2], cmax = ctl->b[3];
        store(c, it);
        if (tid == 0) set_minmax(c, imin, imax);
        const int t = it; it = sc; sc = t;
        imin = cmin; imax = cmax;
        if (tid == 0) free_slot(sc);
      } else if (dec == 2) {  // (Heap[cur], items) <- SORT_SPLIT(Heap[cur], items)
        const int a = (int)ctl->b[4], b = (int)ctl->b[5];
        merge_split(sc, K, it, K, K, a, b);
        store(c, a);
        if (tid == 0) {
          set_minmax(c, BK(a)[0], BK(a)[K - 1]);
          free_slot(a); free_slot(sc); free_slot(it);
        }
        it = b;  // items <- the K largest
        imin = BK(it)[0];
        imax = BK(it)[K - 1];
      } else if (tid == 0) {
        free_slot(sc);
      }
      held = c;
      c = nx;  // l.34
      sc = nsc;
    }
    // ---- l.8: LOCK(tar); UNLOCK(PARENT(cur)); l.9-14
    cta_bar<NT>();
    if (tid == 0) {
      for (u32 w = 0; w < delay_ns; w += 1000) __nanosleep(1000);  // test-only schedule forcing
      const ull tt = now();
      if (held == 1) wait_t_done();  // agent T's LOCK(tar) of l.5-6 must be over first
      lock_acquire(lk(tar));
      acc(LT_INS_TARWAIT, tt);
      fence_proxy_async();
      lock_release(lk(held));
      ctl->b[0] = ld_relaxed(stp(tar));
    }
    cta_bar<NT>();
    if (ctl->b[0] == ST_TARGET) {  // l.9-10
      store(tar, it);
      if (tid == 0) {
        free_slot(it);
        set_minmax(tar, imin, imax);
        st_relaxed(stp(tar), ST_AVAIL);
        lock_release(lk(tar));
      }
    } else {  // l.11-13: a DELETEMIN waits at the root (MARKED): fill the root
      store(1, it);
      if (tid == 0) {
        free_slot(it);
        st[S_MARKED]++;
        set_minmax(1, imin, imax);
        hset(H_RS, K);
        st_release(stp(1), ST_AVAIL);
        st_relaxed(stp(tar), ST_EMPTY);
        lock_release(lk(tar));
      }
    }
    acc(LT_INS_TOTAL, t_ins);
  }

  // =====================================================================================
  // BGPQ_DELETEMIN (Alg.2 + Alg.3).  call_n > 0: deletemin-call mode (size and output slot
  // from the per-call ticket); else `size` and `ok/ov` are given.  Returns #keys written.
  // =====================================================================================
  __device__ __forceinline__ u32 deletemin(u32* ok, u32* ov, u32 size, u64 call_n, ull* lin_out) {
    const int tid = threadIdx.x;
    enum : u32 { P_EMPTY = 0, P_EXTRACT = 1, P_PBUF = 2, P_REFILL = 3 };
    tmerge = LT_DEL_MERGE; tstore = LT_DEL_STORE;
    const ull t_del = now();
    ull t_root = 0;
    cta_bar<NT>();
    if (tid == 0) {
      // l.2: LOCK(root)
      st[S_DEL_OPS]++;
      st[S_ROOT_SPINS] += lock_acquire(lk(1));
      acc(LT_DEL_ROOTACQ, t_del);
      t_root = now();
      fence_proxy_async();
      const Hdr h = hdr_load();
      lin_set(h.lin + 1);
      if (lin_out) *lin_out = h.lin;
      u32 cno = 0;
      if (call_n) {
        cno = h.call;
        hset(H_CALL, cno + 1);
        const u64 rem = call_n - (u64)cno * K;
        size = (u32)(rem < (u64)K ? rem : (u64)K);
      }
      const u32 hs = h.hs, rs = h.rs, ps = h.ps;
      const u32 pbmin = h.pbmin;
      const u32 path = hs == 0 ? P_EMPTY : size < rs ? P_EXTRACT : hs == 1 ? P_PBUF : P_REFILL;
      int sr = -1, stt = -1;
      if (rs > 0 && path != P_EMPTY) {  // stage the root (its keys are output first)
        sr = alloc();
        fence_proxy_async();
        mbar_arrive_expect_tx(&ctl->bar, V ? 2u * NBYTES : NBYTES);
        bulk_g2s(BK(sr), H.gk + (size_t)1 * K, NBYTES, &ctl->bar);
        if (V) bulk_g2s(BV(sr), H.gv + (size_t)1 * K, NBYTES, &ctl->bar);
      }
      u32 c0 = 0, c1 = 0;
      if (path == P_REFILL) {
        const u32 tar = hs;  // l.5
        st[S_DEL_REFILL]++;
        st_relaxed(stp(1), ST_EMPTY);  // l.31
        hset(H_HS, hs - 1);
        if (BGPQ_PREFETCH && hs - 1 >= 2) prefetch_l2(hs - 1);  // the next DELETEMIN's refill node
        stt = alloc();
        post_t(tar, stt, rs > 0 ? 1u : 0u);  // l.6-12 by agent T
        if (tar >= 4) {  // LOCK(l); LOCK(r) of the root concurrently (agent P)
          c0 = 2u <= H.cap ? 2u : 0u;
          c1 = 3u <= H.cap ? 3u : 0u;
          const int s0 = alloc(), s1 = alloc();
          ctl->b[8] = (u32)s0; ctl->b[9] = (u32)s1;
          post_p(c0, c1, s0, s1, 0u);
        }
      }
      ctl->b[0] = hs; ctl->b[1] = rs; ctl->b[2] = ps; ctl->b[3] = pbmin;
      ctl->b[4] = cno; ctl->b[5] = size; ctl->b[6] = path;
      ctl->b[10] = (u32)sr; ctl->b[11] = (u32)stt;
      tmark = t_root;
    }
    cta_bar<NT>();
    mark(LT_R1);
    const u32 hs = ctl->b[0], rs = ctl->b[1], ps = ctl->b[2], pbmin = ctl->b[3];
    const u32 path = ctl->b[6];
    size = ctl->b[5];
    if (call_n) {
      const u64 cno = ctl->b[4];
      ok += cno * (u64)K;
      if (ov) ov += cno * (u64)K;
    }
    if (path == P_EMPTY) {  // l.16-17
      if (tid == 0) lock_release(lk(1));
      return 0;
    }
    const int SR = (int)ctl->b[10];
    if (rs > 0) {
      const ull t0 = now();
      mbar_wait(&ctl->bar, mphase);
      mphase ^= 1u;
      acc(LT_DEL_ROOTLOAD, t0);
    }
    if (path == P_EXTRACT) {  // l.18-20: EXTRACT_ROOT(items, size)
      emit(ok, ov, 0, SR, 0, size);
      if (tid == 0) ctl->b[12] = alloc();
      cta_bar<NT>();
      const int t = (int)ctl->b[12];
      shift(t, SR, size, rs - size);
      store(1, t);
      if (tid == 0) {
        hset(H_RS, rs - size);
        set_minmax(1, BK(t)[0], BK(t)[rs - size - 1]);
        free_slot(t); free_slot(SR);
        lock_release(lk(1));
      }
      return size;
    }
    // l.22: items[1:|root|] <- Heap[root][1:|root|]; |root| <- 0
    if (rs > 0) emit(ok, ov, 0, SR, 0, rs);
    u32 nout = rs;
    if (path == P_PBUF) {  // l.23-29: refill the root from the (sorted, R1) buffer
      const u32 take = min(rs + ps, size) - rs;
      cta_bar<NT>();
      if (tid == 0) { ctl->b[12] = alloc(); ctl->b[13] = alloc(); }
      cta_bar<NT>();
      const int a = (int)ctl->b[12], b = (int)ctl->b[13];
      if (ps > 0) {
        load(a, 0);
        emit(ok, ov, nout, a, 0, take);
        shift(b, a, take, ps - take);
        store(1, b);
      }
      cta_bar<NT>();
      if (tid == 0) {
        hset(H_RS, ps - take);
        hset(H_PS, 0);
        if (ps > take) set_minmax(1, BK(b)[0], BK(b)[ps - take - 1]);
        free_slot(a); free_slot(b);
        if (SR >= 0) free_slot(SR);
        lock_release(lk(1));
      }
      return nout + take;
    }
    // ---- refill path (l.4-13)
    const u32 remained = size - rs;  // l.4 (R8)
    const u32 tar = hs;
    const ull t_tw = now();
    mbar_wait(&ctl->tbar, tphase);  // agent T staged the refill keys (tar's, or a MARKED insert's)
    tphase ^= 1u;
    acc(LT_DEL_TWAIT, t_tw);
    mark(LT_R2);
    int R = (int)ctl->b[11];
    cta_bar<NT>();
    if (tid == 0) {
      if (SR >= 0) free_slot(SR);
      if (ctl->t_marked) st[S_MARKED]++;
      if (tar < 4) {  // tiny heap: the children may be tar itself — lock them after the take
        while (ld_acq_cta(&ctl->t_done) != ctl->t_req) {}
        const u32 c0 = 2u <= H.cap ? 2u : 0u, c1 = 3u <= H.cap ? 3u : 0u;
        const int s0 = alloc(), s1 = alloc();
        ctl->b[8] = (u32)s0; ctl->b[9] = (u32)s1;
        post_p(c0, c1, s0, s1, 0u);
      }
    }
    // l.13: (Heap[root][1:K], pBuffer) <- SORT_SPLIT(Heap[root], K, pBuffer, |pB|, K)
    if (ps > 0 && !(BK(R)[K - 1] <= pbmin)) {
      cta_bar<NT>();
      if (tid == 0) { ctl->b[12] = alloc(); ctl->b[13] = alloc(); ctl->b[14] = alloc(); }
      cta_bar<NT>();
      const int p = (int)ctl->b[12], a = (int)ctl->b[13], b = (int)ctl->b[14];
      load(p, 0);
      merge_split(R, K, p, ps, K, a, b);
      store(0, b);
      if (tid == 0) {
        set_minmax(0, BK(b)[0], BK(b)[ps - 1]);
        free_slot(p); free_slot(b); free_slot(R);
      }
      R = a;
    }
    // ---- l.14: DELETEMIN_HEAPIFY(root, items, remainedSize)  (Alg.3)
    u32 cur = 1;
    cta_bar<NT>();
    int SL = (int)ctl->b[8], SRr = (int)ctl->b[9];
    for (;;) {
      const u32 l = 2u * cur, r = 2u * cur + 1u;  // l.2 (R7)
      wait_p(LT_DEL_PWAIT);  // l.3: LOCK(l); LOCK(r) — done by agent P, children staged
      if (cur == 1) mark(LT_R3);
      if (tid == 0) {
        const u32 le = l <= H.cap, re = r <= H.cap;
        const u32 al = le && ctl->p_st[0] == ST_AVAIL;  // R5
        const u32 ar = re && ctl->p_st[1] == ST_AVAIL;
        const u32 lmin = ctl->p_min[0], lmax = ctl->p_max[0], rmin = ctl->p_min[1], rmax = ctl->p_max[1];
        const u64 minc = min(al ? (u64)lmin : (u64)1 << 32, ar ? (u64)rmin : (u64)1 << 32);
        const u32 maxcur = BK(R)[K - 1];
        const u32 stop = (u64)maxcur <= minc;  // l.4
        u32 x = 0, y = 0, lr = 0;
        if (!stop) {
          if (al && ar) {
            if (lmax > rmax) { x = l; y = r; } else { x = r; y = l; }  // l.9 (R6)
            lr = (lmax <= rmin) ? 1u : ((rmax <= lmin && x == l) ? 1u : 2u);  // 1: no data moves
            st[lr == 1 ? S_DEL_LR_NOMOVE : S_DEL_LR_MERGE]++;
          } else {
            y = al ? l : r;  // R5: exactly one AVAIL child
            x = al ? r : l;
            lr = 0;
            st[S_DEL_LR_SKIP]++;
          }
          st[S_DEL_LEVELS]++;
          // lock-ahead: LOCK the children of y (the next level's l, r) while this level merges
          const u32 yl = 2u * y, yr = 2u * y + 1u;
          const u32 n0 = yl <= H.cap ? yl : 0u, n1 = yr <= H.cap ? yr : 0u;
          int s0 = -1, s1 = -1;
          if (n0 || n1) {
            s0 = alloc(); s1 = alloc();
            post_p(n0, n1, s0, s1, 0u);
          }
          ctl->b[8] = (u32)s0; ctl->b[9] = (u32)s1;
          ctl->b[13] = (n0 || n1) ? 1u : 0u;
          if (lr == 2) { ctl->b[10] = alloc(); ctl->b[11] = alloc(); }
        }
        ctl->b[0] = stop; ctl->b[1] = x; ctl->b[2] = y; ctl->b[3] = lr;
        ctl->b[4] = le; ctl->b[5] = re;
      }
      cta_bar<NT>();
      const u32 stop = ctl->b[0], x = ctl->b[1], y = ctl->b[2], lr = ctl->b[3];
      const u32 le = ctl->b[4], re = ctl->b[5];
      if (stop) {  // l.4-8
        if (tid == 0) {
          if (le) lock_release(lk(l));  // l.7: UNLOCK(l); UNLOCK(r) (unchanged)
          if (re) lock_release(lk(r));
          free_slot(SL); free_slot(SRr);
        }
        if (cur == 1) {
          emit(ok, ov, nout, R, 0, remained);  // l.5-6: EXTRACT_ROOT(items, remainedSize)
          nout += remained;
          if (tid == 0) ctl->b[12] = alloc();
          cta_bar<NT>();
          const int t = (int)ctl->b[12];
          shift(t, R, remained, K - remained);
          store(1, t);
          if (tid == 0) {
            hset(H_RS, K - remained);
            if (remained < (u32)K) set_minmax(1, BK(t)[0], BK(t)[K - remained - 1]);
            free_slot(t);
          }
        } else {
          store(cur, R);
          if (tid == 0) set_minmax(cur, BK(R)[0], BK(R)[K - 1]);
        }
        if (tid == 0) {
          free_slot(R);
          if (cur == 1) while (ld_acq_cta(&ctl->t_done) != ctl->t_req) {}
          lock_release(lk(cur));  // l.7: UNLOCK(cur)
          if (cur == 1) acc(LT_DEL_ROOTHOLD, t_root);
        }
        break;
      }
      const int nSL = (int)ctl->b[8], nSRr = (int)ctl->b[9];
      const u32 more = ctl->b[13];
      int Y;
      if (lr == 2) {  // l.10: (Heap[y], Heap[x]) <- SORT_SPLIT(Heap[l], Heap[r])
        const int a = (int)ctl->b[10], b = (int)ctl->b[11];
        merge_split(SL, K, SRr, K, K, a, b);
        if (cur == 1) mark(LT_R4);
        store(x, b);
        if (tid == 0) {
          set_minmax(x, BK(b)[0], BK(b)[K - 1]);
          ctl->b[16] = x;  // l.11: UNLOCK(x) — released with cur below (one fence)
          if (!BGPQ_JOINT_RELEASE) { lock_release(lk(x)); ctl->b[16] = 0; }
          free_slot(b); free_slot(SL); free_slot(SRr);
        }
        if (cur == 1) mark(LT_R5);
        Y = a;
      } else {  // no data moves between l and r (or only y is AVAIL)
        Y = (y == l) ? SL : SRr;
        if (tid == 0) {
          ctl->b[16] = (x == l ? le : re) ? x : 0u;
          if (!BGPQ_JOINT_RELEASE && ctl->b[16]) { lock_release(lk(x)); ctl->b[16] = 0; }
          free_slot(y == l ? SRr : SL);
        }
      }
      // l.12: (Heap[cur], Heap[y]) <- SORT_SPLIT(Heap[cur], Heap[y])
      int C2, Y2;
      if (BK(Y)[K - 1] <= BK(R)[0]) {  // y entirely below cur: swap contents
        C2 = Y; Y2 = R;
        if (tid == 0) st[S_DEL_CY_SWAP]++;
      } else {
        cta_bar<NT>();
        if (tid == 0) { ctl->b[14] = alloc(); ctl->b[15] = alloc(); }
        cta_bar<NT>();
        const int a = (int)ctl->b[14], b = (int)ctl->b[15];
        merge_split(R, K, Y, K, K, a, b);
        if (tid == 0) { free_slot(R); free_slot(Y); }
        C2 = a; Y2 = b;
      }
      if (cur == 1) {  // l.13: EXTRACT_ROOT(items, remainedSize)
        emit(ok, ov, nout, C2, 0, remained);
        nout += remained;
        int src = C2;
        if (remained > 0) {
          if (tid == 0) ctl->b[12] = alloc();
          cta_bar<NT>();
          src = (int)ctl->b[12];
          shift(src, C2, remained, K - remained);
        }
        store(1, src);
        mark(LT_R6);
        if (tid == 0) {
          hset(H_RS, K - remained);
          if (remained < (u32)K) set_minmax(1, BK(src)[0], BK(src)[K - remained - 1]);
          if (src != C2) free_slot(src);
        }
      } else {
        store(cur, C2);
        if (tid == 0) set_minmax(cur, BK(C2)[0], BK(C2)[K - 1]);
      }
      if (tid == 0) {
        free_slot(C2);
        if (cur == 1) while (ld_acq_cta(&ctl->t_done) != ctl->t_req) {}  // the take is done
        release_locks(cur, ctl->b[16]);  // l.14: UNLOCK(cur) (and l.11's UNLOCK(x))
        if (cur == 1) { acc(LT_DEL_ROOTHOLD, t_root); mark(LT_R7); }
        if (timing && tid == 0) tm[LT_DEL_LEVELS]++;
      }
      cur = y;  // l.15
      R = Y2;
      if (!more) {  // y has no children within capacity: the next level stops at once
        cta_bar<NT>();
        store(cur, R);
        if (tid == 0) {
          set_minmax(cur, BK(R)[0], BK(R)[K - 1]);
          free_slot(R);
          lock_release(lk(cur));
        }
        break;
      }
      SL = nSL;
      SRr = nSRr;
    }
    acc(LT_DEL_TOTAL, t_del);
    return nout;
  }
};

// ---- the lock warp: lane 0 = agent P, lane 1 = agent T
template <int K, bool V, int NT>
__device__ __forceinline__ void lock_warp(OpL<K, V, NT>& op) {
  LCtl* c = op.ctl;
  const int lane = threadIdx.x & 31;
  const u32 NB = K * 4u;
  if (lane == 0) {  // agent P
    u32 seen = 0;
    for (;;) {
      u32 r;
      while ((r = ld_acq_cta(&c->p_req)) == seen) {
        if (ld_acq_cta(&c->stop)) return;
        __nanosleep(20);
      }
      seen = r;
      const u32 bi = c->p_bi, force = c->p_force;
      u32 bytes = 0;
      u32 stv[2], mn[2], mx[2];
      for (int q = 0; q < 2; ++q) {
        const u32 n = c->p_n[q];
        stv[q] = ST_EMPTY; mn[q] = 0; mx[q] = 0;
        if (!n) continue;
        const ull t0 = op.timing ? clock64() : 0;
        lock_acquire(op.lk(n));
        if (op.timing) op.tm[LT_P_LOCKWAIT] += clock64() - t0;
        meta_load(&op.H.meta[n], stv[q], mn[q], mx[q]);
        if (force || stv[q] == ST_AVAIL) bytes += V ? 2u * NB : NB;
      }
      for (int q = 0; q < 2; ++q) { c->p_st[q] = stv[q]; c->p_min[q] = mn[q]; c->p_max[q] = mx[q]; }
      fence_proxy_async();
      mbar_arrive_expect_tx(&c->pbar[bi], bytes);
      for (int q = 0; q < 2; ++q) {
        const u32 n = c->p_n[q];
        if (!n || !(force || stv[q] == ST_AVAIL)) continue;
        const int s = (int)c->p_s[q];
        bulk_g2s(op.BK(s), op.H.gk + (size_t)n * K, NB, &c->pbar[bi]);
        if (V) bulk_g2s(op.BV(s), op.H.gv + (size_t)n * K, NB, &c->pbar[bi]);
      }
    }
  } else if (lane == 1) {  // agent T
    u32 seen = 0, tph = 0;
    for (;;) {
      u32 r;
      while ((r = ld_acq_cta(&c->t_req)) == seen) {
        if (ld_acq_cta(&c->stop)) return;
        __nanosleep(20);
      }
      seen = r;
      const u32 n = c->t_node;
      const int s = (int)c->t_slot;
      if (c->t_kind == 1u) {  // Alg.1 l.5-6
        lock_acquire(op.lk(n));
        st_relaxed(op.stp(n), ST_TARGET);
        lock_release(op.lk(n));
        st_rel_cta(&c->t_done, seen);
        continue;
      }
      const ull t0 = op.timing ? clock64() : 0;
      lock_acquire(op.lk(n));  // l.6: LOCK(tar)
      if (op.timing) op.tm[LT_T_LOCKWAIT] += clock64() - t0;
      fence_proxy_async();
      const u32 stn = ld_relaxed(op.stp(n));
      if (stn == ST_TARGET) {  // l.7-9: steal the keys of the insert in flight
        // the old root keys must be staged before the MARKED insert may overwrite them
        if (c->t_rootload) mbar_wait(&c->bar, c->t_rootpar);
        st_relaxed(op.stp(n), ST_MARKED);
        lock_release(op.lk(n));
        u32 ns = 32;
        while (ld_acquire(op.stp(1)) != ST_AVAIL) {
          __nanosleep(ns);
          ns = ns < 256 ? ns * 2 : 256;
        }
        fence_proxy_async();
        c->t_marked = 1;
        mbar_arrive_expect_tx(&c->tbar, V ? 2u * NB : NB);
        bulk_g2s(op.BK(s), op.H.gk + (size_t)1 * K, NB, &c->tbar);
        if (V) bulk_g2s(op.BV(s), op.H.gv + (size_t)1 * K, NB, &c->tbar);
        mbar_wait(&c->tbar, tph);
      } else {  // l.11: Heap[root] <- Heap[tar]; Heap[tar].state <- EMPTY
        c->t_marked = 0;
        mbar_arrive_expect_tx(&c->tbar, V ? 2u * NB : NB);
        bulk_g2s(op.BK(s), op.H.gk + (size_t)n * K, NB, &c->tbar);
        if (V) bulk_g2s(op.BV(s), op.H.gv + (size_t)n * K, NB, &c->tbar);
        mbar_wait(&c->tbar, tph);
        st_relaxed(op.stp(n), ST_EMPTY);
        lock_release(op.lk(n));
        st_relaxed(op.stp(1), ST_AVAIL);  // l.12
      }
      tph ^= 1u;
      if (op.timing) op.tm[LT_T_TOTAL] += clock64() - t0;
      st_rel_cta(&c->t_done, seen);
    }
  }
}

template <int K, bool V, int NT>
__global__ void __launch_bounds__(NT + 32, 1) bgpq_locks_kernel(HeapArgs H, CallArgs C) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  if (C.op_base) {  // the cluster engine executed the first ops of this deletemin call
    const u64 b = *reinterpret_cast<volatile const u64*>(C.op_base);
    C.n -= b * (u64)K;
    C.n_ops -= b;
    C.out_k += b * (u64)K;
    if (C.out_v) C.out_v += b * (u64)K;
  }
  LCtl* ctl = reinterpret_cast<LCtl*>(smem_raw);
  OpL<K, V, NT> op;
  op.H = H;
  op.ctl = ctl;
  op.sk = reinterpret_cast<u32*>(smem_raw + LCTL_BYTES);
  op.sv = op.sk + LSLOT * K;
  op.mphase = 0; op.pph = 0; op.tphase = 0; op.pb = 0;
  op.st = ctl->st;
  op.tm = ctl->tm;
  op.timing = (C.debug & 8u) != 0;
  op.delay_ns = (C.debug & 32768u) ? 20000u : 0u;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NSTAT; ++i) ctl->st[i] = 0;
    for (int i = 0; i < 32; ++i) ctl->tm[i] = 0;
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
    lock_warp<K, V, NT>(op);
    if (op.timing) {
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      for (int i = LT_P_LOCKWAIT; i < LT_R1; ++i)
        if (op.tm[i]) atomicAdd(tms + i, op.tm[i]);
    }
    return;
  }
  for (;;) {
    if (threadIdx.x == 0) ctl->op = atomicAdd(H.hdr + H_FETCH, 1u);
    cta_bar<NT>();
    const u64 j = ctl->op;
    cta_bar<NT>();
    if (j >= C.n_ops) break;
    // one call site per operation type (both are force-inlined: no local-memory copy of op)
    bool ins;
    const u32* ik = nullptr;
    const u32* iv = nullptr;
    u32* ok = C.out_k;
    u32* ov = C.out_v;
    u32 size = 0;
    u64 call_n = 0;
    ull* lt = nullptr;
    if (C.mode == MODE_INSERT) {
      ins = true;
      const u64 off = j * (u64)K;
      const u64 rem = C.n - off;
      size = (u32)(rem < (u64)K ? rem : (u64)K);
      ik = C.in_k + off;
      iv = C.in_v ? C.in_v + off : nullptr;
    } else if (C.mode == MODE_DELETEMIN) {
      ins = false;
      call_n = C.n;
    } else {
      ins = C.op_types[j] == 0;
      size = C.op_sizes[j];
      lt = C.lin_ticket ? C.lin_ticket + j : nullptr;
      if (size == 0u || size > (u32)K) {  // op sizes must be in 1..K: sticky EINVAL, op skipped
        if (threadIdx.x == 0) {
          atomicCAS(H.hdr + H_ERR, 0u, (u32)-1);
          if (!ins) C.op_count[j] = 0;
        }
        continue;
      }
      if (ins) {
        const u64 off = C.in_off[j];
        ik = C.in_k + off;
        iv = C.in_v ? C.in_v + off : nullptr;
      } else {
        ok = C.out_k + j * (u64)K;
        ov = C.out_v ? C.out_v + j * (u64)K : nullptr;
      }
    }
    if (ins) {
      op.insert(ik, iv, size, lt);
    } else {
      const u32 cnt = op.deletemin(ok, ov, size, call_n, lt);
      if (threadIdx.x == 0) {
        op.st[S_KEYS_OUT] += cnt;
        if (C.mode == MODE_MIXED) C.op_count[j] = cnt;
        else if (C.d_count && cnt) atomicAdd(C.d_count, (ull)cnt);
      }
    }
  }
  if (threadIdx.x == 0) {
    st_rel_cta(&ctl->stop, 1u);
    ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
    for (int i = 0; i < NSTAT; ++i)
      if (op.st[i]) atomicAdd(stat + i, op.st[i]);
    if (op.timing) {
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      for (int i = 0; i < LT_N; ++i)
        if (i < LT_P_LOCKWAIT || i >= LT_R1)
        if (op.tm[i]) atomicAdd(tms + i, op.tm[i]);
    }
  }
}

template <int K, bool V>
constexpr size_t locks_smem_bytes() {
  return LCTL_BYTES + (size_t)LSLOT * K * 4 * (V ? 2 : 1);
}

}  // namespace bgpqd
