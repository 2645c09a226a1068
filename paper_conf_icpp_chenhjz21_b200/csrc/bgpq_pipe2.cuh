// bgpq_pipe2.cuh — INSERT calls as a level pipeline with decoupled data movement (the default
// execution of bgpq_insert; bgpq_pipe.cuh is the synchronous version it replaces).
//
// Same protocol as bgpq_pipe.cuh (one CTA per heap level applies every INSERT_HEAPIFY step of
// its depth in call order, Alg.1 l.30-34; the root stage runs PARTIAL_INSERT, l.15-29; sorter
// CTAs run Sort(items), l.2), so the heap after a call equals the sequential Alg.1 model node
// for node.  What changes is who moves the data.  In the synchronous version every message
// cost a flag poll, a TMA load of the items (and of the path node when it changes), the merge,
// 4 KB of stores and a gpu-scope release, one after the other.  Here each pipeline CTA has
//   H1 (helper warp 1): polls the next message's flag, TMA-loads its items — and the node of
//      depth l on its root -> tar path when that node changes — into free smem slots, and
//      marks the ring slot consumed (runs up to PIN messages ahead);
//   H2 (helper warp 2): executes sends (TMA bulk store of the carried items into the next
//      level's ring slot, completion, proxy fence, release of the flag, with flow control)
//      and node write-backs (bulk store + cached min/max + state for placements, Alg.1 l.9-10);
// so the compute threads only take decisions and run SORT_SPLITs.  Path nodes of depth l are
// non-decreasing in the message order while tar stays at one depth (tar = heapSize + 1
// grows); two hazards remain: a node placed by this stage and needed as a path node later in
// the same call (H1 waits for H2's completion of the placements), and the restart of the
// path at the leftmost node of depth l when tar enters the next depth — that node was this
// stage's path node before, so H1 waits until every earlier message was processed and its
// write-back retired (a round-1 H1 could prefetch the stale HBM copy while the compute still
// held the dirty one: keys lost on small reused heaps, seen at K = 4096).
#pragma once
#include "bgpq_pipe.cuh"

namespace bgpqd {

constexpr u32 P2_PIN = 4;     // in-ring entries (H1 -> compute)
constexpr u32 P2_RQ = 16;     // H2 request ring
constexpr u32 P2_H2D = 8;     // H2 requests in flight (bulk groups), retired as one batch
// smem node slots per stage: 24, fewer for the largest nodes (the stage needs >= 12: root,
// pBuffer, the in-ring entries' item and node slots, the sends in flight)
template <int K, bool V>
__host__ __device__ constexpr int p2_nsl() {
  return (size_t)24 * K * 4 * (V ? 2 : 1) <= 200704 ? 24 : 12;
}
constexpr u32 P2_NONE = 0xFFFFFFFFu;
enum : u32 { P2_WB = 1, P2_SEND = 2, P2_END = 3, P2_STOP = 4 };

struct P2Ctl {
  u64 ibar[P2_PIN];
  u32 pool;                 // free slot bitmask (atomic: H1 allocates, compute / H2 free)
  u32 icons;                // compute: in-ring entries consumed
  u32 ent[P2_PIN][4];       // tar, end, item slot, node slot
  u32 rq_head, rq_done;
  u32 rq[P2_RQ][4];
  u32 place_done;           // H2: placements completed
  u32 mdone;                // compute: messages fully processed (their H2 requests issued)
  u32 fq[P2_H2D][7];        // H2: in-flight requests (type, a, b, c, smem source, min, max)
  u32 b[8];                 // thread-0 broadcasts
};
constexpr size_t P2CTL_BYTES = (sizeof(P2Ctl) + 127) / 128 * 128;

template <int K, bool V>
constexpr size_t pipe2_smem_bytes() {
  return LCTL_BYTES + P2CTL_BYTES + (size_t)p2_nsl<K, V>() * K * 4 * (V ? 2 : 1);
}

__device__ __forceinline__ u32 vld(const u32* p) { return *reinterpret_cast<const volatile u32*>(p); }
// back-off of the pipeline's hot polls (flags, flow control, ring room): a short sleep keeps the
// single-thread pollers from taking issue slots from the compute warps of their SM (measured:
// C2 insert 148 ms with 32 ns vs 160 ms with no sleep)
#ifndef BGPQ_P2_SLEEP
#define BGPQ_P2_SLEEP 32
#endif
__device__ __forceinline__ void p2_pause() {
  if (BGPQ_P2_SLEEP) __nanosleep(BGPQ_P2_SLEEP);
}

template <int K, bool V, int NT>
struct Pipe2 {
  static constexpr u32 NB = K * 4u;
  HeapArgs H;
  PipeArgs P;
  CallArgs C;
  u32* sk;
  u32* sv;
  LCtl* ctl;
  P2Ctl* pc;

  __device__ __forceinline__ u32* BK(u32 s) const { return sk + s * K; }
  __device__ __forceinline__ u32* BV(u32 s) const { return V ? sv + s * K : nullptr; }
  __device__ __forceinline__ u32 op_size(u64 j) const {
    const u64 rem = C.n - j * (u64)K;
    return (u32)(rem < (u64)K ? rem : (u64)K);
  }
  __device__ __forceinline__ u32* ringk(u32 l, u32 slot) const { return P.rk + ((size_t)l * PIPE_NL + slot) * K; }
  __device__ __forceinline__ u32* ringv(u32 l, u32 slot) const {
    return V ? P.rv + ((size_t)l * PIPE_NL + slot) * K : nullptr;
  }
  __device__ __forceinline__ u32* cons(u32 l) const { return P.ctl + PC_LCONS + 32 * l; }

  // ---- slot pool (any thread)
  __device__ __forceinline__ u32 alloc() {
    for (;;) {
      const u32 m = vld(&pc->pool);
      if (m) {
        const u32 s = __ffs(m) - 1;
        if (atomicAnd(&pc->pool, ~(1u << s)) & (1u << s)) return s;
      } else {
        __nanosleep(32);
      }
    }
  }
  __device__ __forceinline__ void release(u32 s) {
    if (s != P2_NONE) atomicOr(&pc->pool, 1u << s);
  }
  // ---- thread 0 -> H2
  ull th2 = 0;  // debug 128|16384: cycles thread 0 waited for room in H2's request ring
  __device__ __forceinline__ void h2(u32 type, u32 a = 0, u32 b = 0, u32 c = 0) {
    const u32 h = pc->rq_head;
    if (h - vld(&pc->rq_done) >= P2_RQ) {
      const ull t0 = (C.debug & 16384u) ? clock64() : 0ull;
      while (h - vld(&pc->rq_done) >= P2_RQ) p2_pause();
      if (C.debug & 16384u) th2 += clock64() - t0;
    }
    u32* e = pc->rq[h % P2_RQ];
    e[0] = type; e[1] = a; e[2] = b; e[3] = c;
    st_rel_cta(&pc->rq_head, h + 1u);
  }
  // SORT_SPLIT by all compute threads into two fresh slots; the inputs are released
  __device__ __forceinline__ void merge2(u32 z, u32 na, u32 w, u32 nb, u32 ma, u32& x, u32& y) {
    if (threadIdx.x == 0) { ctl->b[20] = alloc(); ctl->b[21] = alloc(); }
    cta_bar<NT>();
    const ull ts = (threadIdx.x == 0 && (C.debug & 131072u)) ? clock64() : 0ull;
    x = ctl->b[20]; y = ctl->b[21];
    sort_split<K, NT, V>(BK(z), BV(z), (int)na, BK(w), BV(w), (int)nb, (int)ma, BK(x), BV(x), BK(y), BV(y));
    cta_bar<NT>();
    if (threadIdx.x == 0 && (C.debug & 131072u)) twait += clock64() - ts;  // debug 131072: split only
    if (threadIdx.x == 0) { release(z); release(w); }
  }
  // compute threads: wait for in-ring entry m, read it, hand the entry back to H1
  ull twait = 0;  // debug 128: cycles thread 0 waited for the next message (per stage)
  __device__ __forceinline__ void take(u32 m, u32& tar, u32& end, u32& is, u32& ns) {
    const u32 e = m % P2_PIN;
    const ull t0 = (threadIdx.x == 0 && (C.debug & 128u)) ? clock64() : 0ull;
    mbar_wait(&pc->ibar[e], (m / P2_PIN) & 1u);
    if (threadIdx.x == 0 && (C.debug & 128u) && !(C.debug & 65536u)) twait += clock64() - t0;
    tar = pc->ent[e][0]; end = pc->ent[e][1]; is = pc->ent[e][2]; ns = pc->ent[e][3];
    cta_bar<NT>();
    if (threadIdx.x == 0) {
      st_rel_cta(&pc->icons, m + 1u);
      // the entry's ring slot may be reused by the sender at once (relaxed: its TMA load into
      // shared memory completed before the wait above returned)
      st_relaxed(mycons, m + 1u);
    }
  }
  u32* mycons;  // this stage's consumption counter read by its sender (P.ctl word)

  // ======================================================================================
  // H1 of a level stage l (l >= 1): prefetch messages m = 0, 1, ... from ring l
  // ======================================================================================
  __device__ void h1_level(u32 l) {
    u32 last_a = 0, nplace = 0;
    for (u32 m = 0;; ++m) {
      const u32 e = m % P2_PIN;
      while (m - vld(&pc->icons) >= P2_PIN) p2_pause();
      (void)ld_acq_cta(&pc->icons);
      const u32 slot = m % PIPE_NL;
      const u64* f = P.rflag + (size_t)l * PIPE_NL + slot;
      u64 w;  // one acquire load: the message index and its header {tar, end}
      while ((u32)(w = ld_acquire_u64(f)) != m + 1) p2_pause();
      const u32 tar = (u32)(w >> 32) & 0x7FFFFFFFu, end = (u32)(w >> 63);
      pc->ent[e][0] = tar; pc->ent[e][1] = end; pc->ent[e][2] = P2_NONE; pc->ent[e][3] = P2_NONE;
      if (end) {
        st_release(cons(l), m + 1);
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(&pc->ibar[e])) : "memory");
        return;
      }
      const u32 dt = depth_of(tar);
      u32 bytes = V ? 2u * NB : NB;
      const u32 is = alloc();
      u32 ns = P2_NONE, a = 0;
      if (dt > l) {
        a = tar >> (dt - l);
        if (a != last_a) {
          if (a < last_a) {
            // tar entered the next depth: the path at depth l restarts at the leftmost node,
            // which this stage held (and may have written back) earlier in the call — load it
            // only after every earlier message was processed and its write-back retired
            while (ld_acq_cta(&pc->mdone) < m) __nanosleep(32);
            const u32 h = ld_acq_cta(&pc->rq_head);
            while ((int)(ld_acq_cta(&pc->rq_done) - h) < 0) __nanosleep(32);
          }
          last_a = a;
          ns = alloc();
          bytes += V ? 2u * NB : NB;
          // every placement at depth l precedes the first path node of depth l in a call
          // (tar grows): a node placed in this call must be written before it is loaded
          while ((int)(ld_acq_cta(&pc->place_done) - nplace) < 0) __nanosleep(32);
        }
      } else {
        ++nplace;
      }
      pc->ent[e][2] = is; pc->ent[e][3] = ns;
      fence_proxy_async();
      mbar_arrive_expect_tx(&pc->ibar[e], bytes);
      bulk_g2s(BK(is), ringk(l, slot), NB, &pc->ibar[e]);
      if (V) bulk_g2s(BV(is), ringv(l, slot), NB, &pc->ibar[e]);
      if (ns != P2_NONE) {
        bulk_g2s(BK(ns), H.gk + (size_t)a * K, NB, &pc->ibar[e]);
        if (V) bulk_g2s(BV(ns), H.gv + (size_t)a * K, NB, &pc->ibar[e]);
      }
    }
  }

  // H1 of the root stage: prefetch sorted batches j = 0, 1, ...
  __device__ void h1_root() {
    const bool tm = (C.debug & 128u) != 0;
    ull w_icons = 0, w_ready = 0, w_alloc = 0;
    for (u32 j = 0; j < (u32)C.n_ops; ++j) {
      const u32 e = j % P2_PIN;
      ull t0 = tm ? clock64() : 0;
      while (j - vld(&pc->icons) >= P2_PIN) p2_pause();
      (void)ld_acq_cta(&pc->icons);
      if (tm) { const ull t = clock64(); w_icons += t - t0; t0 = t; }
      const u32 slot = j % PIPE_NSB;
      while (ld_acquire(P.sready + slot) != j + 1) p2_pause();
      if (tm) { const ull t = clock64(); w_ready += t - t0; t0 = t; }
      const u32 is = alloc();
      if (tm) { const ull t = clock64(); w_alloc += t - t0; t0 = t; }
      pc->ent[e][0] = op_size(j); pc->ent[e][1] = 0; pc->ent[e][2] = is; pc->ent[e][3] = P2_NONE;
      fence_proxy_async();
      mbar_arrive_expect_tx(&pc->ibar[e], V ? 2u * NB : NB);
      bulk_g2s(BK(is), P.sbk + (size_t)slot * K, NB, &pc->ibar[e]);
      if (V) bulk_g2s(BV(is), P.sbv + (size_t)slot * K, NB, &pc->ibar[e]);
    }
    if (tm) {
      ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
      atomicAdd(tms + 29, w_icons); atomicAdd(tms + 30, w_ready); atomicAdd(tms + 31, w_alloc);
    }
  }

  // ======================================================================================
  // H2: sends and write-backs, in request order
  // ======================================================================================
  __device__ void h2_loop() {
    // Requests are issued in order and completed in order with up to P2_H2D bulk groups in
    // flight (one commit group per request): a send's flag (release) and a write-back's
    // metadata are published only after cp.async.bulk.wait_group has retired that request's
    // own group, so every message's data is globally visible before its flag.
    constexpr u32 D = P2_H2D;
    u32 seen = 0, nplaced = 0, inflight = 0, head_i = 0;
    u32 cache_l = P2_NONE, cache_c = 0;
    const bool tm = (C.debug & 262144u) != 0;  // debug: H2 flow-control / wait_group / publish cycles
    ull w_fc = 0, w_wg = 0, w_pub = 0;
    auto retire = [&](u32 keep) {  // more than `keep` requests in flight: complete all of them
      if (inflight <= keep) return;
      const ull t0 = tm ? clock64() : 0ull;
      // the source slots come back as soon as the copies have read them (a node write-back's
      // HBM write takes far longer to complete than its shared-memory read)
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      for (u32 q = 0; q < inflight; ++q) {
        u32* f = pc->fq[(head_i + q) % D];
        if (f[4] != P2_NONE) { release(f[4]); f[4] = P2_NONE; }
      }
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
      const ull t1 = tm ? clock64() : 0ull;
      if (tm) w_wg += t1 - t0;
      // one proxy fence and one release fence publish the whole batch: every request's bulk
      // data is complete and ordered before the relaxed flag / metadata stores below
      asm volatile("fence.proxy.async.global;" ::: "memory");
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
      while (inflight) {
        const u32* f = pc->fq[head_i % D];
        const u32 type = f[0], a = f[1], b = f[2], c = f[3];
        if (type == P2_WB) {
          st_relaxed(&H.meta[a].kmin, f[5]);
          st_relaxed(&H.meta[a].kmax, f[6]);
          if (c) {
            st_relaxed(&H.meta[a].state, ST_AVAIL);
            st_rel_cta(&pc->place_done, ++nplaced);
          }
        } else {  // SEND / END: the flag word with the header
          const u32 l = a >> 8, m = b, rs = m % PIPE_NL;
          const u64 hdr = type == P2_SEND ? (u64)(c & 0x7FFFFFFFu) : (u64)1u << 31;
          st_relaxed_u64(P.rflag + (size_t)l * PIPE_NL + rs, (hdr << 32) | (u64)(m + 1));
        }
        ++head_i;
        --inflight;
        ++seen;
      }
      st_rel_cta(&pc->rq_done, seen);
      if (tm) w_pub += clock64() - t1;
    };
    auto report = [&]() {
      const u32 b = blockIdx.x - ((C.debug & 524288u) ? 8u : 0u);  // debug 524288: stages 8..23
      if (tm && b < 16) {
        ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
        atomicAdd(tms + b, w_fc + (w_wg << 32));   // low: flow control, high: wait_group (cycles >> 0)
        atomicAdd(tms + 16 + b, w_pub);
      }
    };
    u32 issued = 0;
    for (;;) {
      while (vld(&pc->rq_head) == issued) {
        if (inflight) retire(0);
        else p2_pause();
      }
      (void)ld_acq_cta(&pc->rq_head);
      const u32* e = pc->rq[issued % P2_RQ];
      const u32 type = e[0], a = e[1], b = e[2], c = e[3];
      if (type == P2_STOP) {
        retire(0);
        ++issued;
        ++seen;
        st_rel_cta(&pc->rq_done, seen);
        report();
        return;
      }
      retire((C.debug & 4096u) ? 0u : D - 1);  // room for one more group (debug 4096: one at a time)
      u32* f = pc->fq[(head_i + inflight) % D];
      f[0] = type; f[1] = a; f[2] = b; f[3] = c; f[4] = P2_NONE;
      if (type == P2_WB) {  // node a <- slot b (K entries); c = 1: placement (state AVAIL)
        f[5] = BK(b)[0]; f[6] = BK(b)[K - 1]; f[4] = b;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        bulk_s2g(H.gk + (size_t)a * K, BK(b), NB);
        if (V) bulk_s2g(H.gv + (size_t)a * K, BV(b), NB);
      } else {  // P2_SEND (a = level << 8 | slot, b = message, c = tar) / P2_END
        const u32 l = a >> 8, m = b;
        const u32 rs = m % PIPE_NL;
        const ull tf = tm ? clock64() : 0ull;
        if (m >= PIPE_NL) {  // flow control: the receiver consumed the slot's previous message
          if (cache_l != l) { cache_l = l; cache_c = 0; }
          while (cache_c < m + 1 - PIPE_NL) {
            cache_c = ld_acquire(cons(l));
            if (cache_c < m + 1 - PIPE_NL) p2_pause();
          }
        }
        if (tm) w_fc += clock64() - tf;
        if (type == P2_SEND) {
          const u32 s = a & 0xFFu;
          f[4] = s;
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          bulk_s2g(ringk(l, rs), BK(s), NB);
          if (V) bulk_s2g(ringv(l, rs), BV(s), NB);
        }
      }
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");  // (empty for END: retires in order)
      ++inflight;
      ++issued;
    }
  }
  __device__ __forceinline__ void send(u32 l, u32 m, u32 tar, u32 s) { h2(P2_SEND, (l << 8) | s, m, tar); }
  __device__ __forceinline__ void send_end(u32 l, u32 m) { h2(P2_END, l << 8, m, 0); }
  __device__ __forceinline__ void h2_drain() {
    if (threadIdx.x == 0) {
      h2(P2_STOP);
      while (vld(&pc->rq_done) != pc->rq_head) __nanosleep(32);
    }
    cta_bar<NT>();
  }

  // ======================================================================================
  // compute threads of the root stage: PARTIAL_INSERT (Alg.1 l.15-29) in call order
  // ======================================================================================
  __device__ void root_stage() {
    const int tid = threadIdx.x;
    if (tid == 0) {
      ctl->b[0] = ld_relaxed(H.hdr + H_HS);
      ctl->b[1] = ld_relaxed(H.hdr + H_RS);
      ctl->b[2] = ld_relaxed(H.hdr + H_PS);
      ctl->b[3] = alloc();  // root
      ctl->b[4] = alloc();  // pBuffer
    }
    cta_bar<NT>();
    u32 hs = ctl->b[0], rs = ctl->b[1], ps = ctl->b[2];
    u32 R = ctl->b[3], PB = ctl->b[4];
    {  // stage the root and the pBuffer
      u32 bytes = 0;
      if (rs > 0) bytes += V ? 2u * NB : NB;
      if (ps > 0) bytes += V ? 2u * NB : NB;
      if (tid == 0) {
        fence_proxy_async();
        mbar_arrive_expect_tx(&ctl->bar, bytes);
        if (rs > 0) { bulk_g2s(BK(R), H.gk + (size_t)K, NB, &ctl->bar); if (V) bulk_g2s(BV(R), H.gv + (size_t)K, NB, &ctl->bar); }
        if (ps > 0) { bulk_g2s(BK(PB), H.gk, NB, &ctl->bar); if (V) bulk_g2s(BV(PB), H.gv, NB, &ctl->bar); }
      }
      mbar_wait(&ctl->bar, 0);
    }
    u32 sent = 0;
    ull nheap = 0;
    for (u32 j = 0; j < (u32)C.n_ops; ++j) {
      u32 size, end_, I, ns_;
      take(j, size, end_, I, ns_);
      const u32 imin = BK(I)[0];
      if (hs == 0) {  // l.16-19
        if (tid == 0) release(R);
        R = I;
        rs = size; hs = 1;
        continue;
      }
      if (rs > 0 && BK(R)[rs - 1] > imin) {  // l.20: the root keeps its |root| smallest
        u32 a, b;
        merge2(R, rs, I, size, rs, a, b);
        R = a; I = b;
      }
      if (ps + size < (u32)K) {  // l.21-24: append to the (sorted, R1) buffer
        if (ps > 0) {
          u32 a, b;
          merge2(PB, ps, I, size, ps + size, a, b);
          if (tid == 0) release(b);
          PB = a;
        } else {
          if (tid == 0) release(PB);
          PB = I;
        }
        ps += size;
        continue;
      }
      const u32 nps = ps + size - K;
      if (ps > 0) {  // l.26-28: the K smallest of items u pBuffer form the batch
        u32 a, b;
        merge2(I, size, PB, ps, K, a, b);
        I = a; PB = b;
      }
      ps = nps;
      const u32 tar = hs + 1;  // l.4
      if (tar > H.cap) {       // R15: sticky capacity error, the batch is dropped
        if (tid == 0) { st_relaxed(H.hdr + H_ERR, (u32)(-3)); release(I); }
        continue;
      }
      hs = tar;
      ++nheap;
      if (tid == 0) send(1, sent, tar, I);
      ++sent;
    }
    if (tid == 0) send_end(1, sent);
    ++sent;
    h2_drain();
    // the on-chip root and pBuffer back to the arena, and the header
    if (rs > 0) {
      for (int i = tid; i < K / 4; i += NT) {
        reinterpret_cast<uint4*>(H.gk + (size_t)K)[i] = reinterpret_cast<const uint4*>(BK(R))[i];
        if (V) reinterpret_cast<uint4*>(H.gv + (size_t)K)[i] = reinterpret_cast<const uint4*>(BV(R))[i];
      }
    }
    if (ps > 0) {
      for (int i = tid; i < K / 4; i += NT) {
        reinterpret_cast<uint4*>(H.gk)[i] = reinterpret_cast<const uint4*>(BK(PB))[i];
        if (V) reinterpret_cast<uint4*>(H.gv)[i] = reinterpret_cast<const uint4*>(BV(PB))[i];
      }
    }
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
  }

  // ======================================================================================
  // compute threads of level stage l: INSERT_HEAPIFY steps at depth l (Alg.1 l.30-34) and
  // placements at depth l (l.9-10)
  // ======================================================================================
  __device__ void level_stage(u32 l) {
    const int tid = threadIdx.x;
    u32 N = P2_NONE, cur = 0, dirty = 0, sent = 0;
    ull lv = 0, nnoop = 0, nswap = 0, nmerge = 0;
    // two spare slots receive a merge's outputs and its inputs become the next spares: tracked
    // identically by every compute thread, so a merge needs no slot-pool atomics and no
    // barrier before the split (the inputs were last read before the previous split's barrier;
    // neither input is ever referenced by a pending H2 request)
    if (tid == 0) { ctl->b[22] = alloc(); ctl->b[23] = alloc(); }
    cta_bar<NT>();
    u32 sp0 = ctl->b[22], sp1 = ctl->b[23];
    for (u32 m = 0;; ++m) {
      u32 tar, end, I, ns;
      take(m, tar, end, I, ns);
      if (end) break;
      const u32 dt = depth_of(tar);
      if (dt == l) {  // l.9-10: Heap[tar] <- items (state AVAIL)
        if (tid == 0) { h2(P2_WB, tar, I, 1u); st_rel_cta(&pc->mdone, m + 1u); }
        continue;
      }
      if (ns != P2_NONE) {  // the path node of depth l changed: write the old one back
        if (tid == 0) {
          if (dirty) h2(P2_WB, cur, N, 0u);
          else release(N);
        }
        N = ns;
        cur = tar >> (dt - l);
        dirty = 0;
      }
      // l.33: (Heap[cur], items) <- SORT_SPLIT(Heap[cur], items), O(1) no-op / swap cases
      const u32 cmin = BK(N)[0], cmax = BK(N)[K - 1], imin = BK(I)[0], imax = BK(I)[K - 1];
      ++lv;
      if (cmax <= imin) {
        ++nnoop;
      } else if (imax <= cmin) {
        const u32 t = N; N = I; I = t;
        dirty = 1;
        ++nswap;
      } else {
        const ull tq = (tid == 0 && (C.debug & 65536u)) ? clock64() : 0ull;
        sort_split<K, NT, V>(BK(N), BV(N), K, BK(I), BV(I), K, K, BK(sp0), BV(sp0), BK(sp1), BV(sp1));
        cta_bar<NT>();
        if (tid == 0 && (C.debug & 65536u)) twait += clock64() - tq;  // debug 65536: merge time instead
        const u32 a = sp0, b = sp1;
        sp0 = N; sp1 = I;
        N = a; I = b;
        dirty = 1;
        ++nmerge;
      }
      if (tid == 0) { send(l + 1, sent, tar, I); st_rel_cta(&pc->mdone, m + 1u); }
      ++sent;
    }
    if (tid == 0) {
      if (l < P.depth) send_end(l + 1, sent);
      if (dirty) h2(P2_WB, cur, N, 0u);
      else release(N);
      release(sp0);
      release(sp1);
    }
    h2_drain();
    if (tid == 0) {
      ctl->st[S_INS_LEVELS] += lv;
      ctl->st[S_INS_NOOP] += nnoop;
      ctl->st[S_INS_SWAP] += nswap;
      ctl->st[S_INS_MERGE] += nmerge;
    }
  }
};

template <int K, bool V, int NT>
__global__ void __launch_bounds__(NT + 64, 1) bgpq_ins_pipe2_kernel(HeapArgs H, PipeArgs P, CallArgs C) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  LCtl* ctl = reinterpret_cast<LCtl*>(smem_raw);
  P2Ctl* pc = reinterpret_cast<P2Ctl*>(smem_raw + LCTL_BYTES);
  const u32 b = blockIdx.x;
  if (b > P.depth) {  // sorters: the synchronous version's code, compute threads only
    if (threadIdx.x >= NT) return;
    Pipe<K, V, NT> p;
    p.H = H; p.P = P; p.C = C; p.ctl = ctl;
    p.sk = reinterpret_cast<u32*>(smem_raw + LCTL_BYTES + P2CTL_BYTES);
    p.sv = p.sk + p2_nsl<K, V>() * K;
    p.ph0 = 0; p.ph1 = 0;
    if (threadIdx.x == 0) {
      mbar_init(&ctl->bar, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    cta_bar<NT>();
    p.sorter();
    return;
  }
  Pipe2<K, V, NT> p;
  p.H = H; p.P = P; p.C = C; p.ctl = ctl; p.pc = pc;
  p.sk = reinterpret_cast<u32*>(smem_raw + LCTL_BYTES + P2CTL_BYTES);
  p.sv = p.sk + p2_nsl<K, V>() * K;
  if (threadIdx.x == 0) {
    mbar_init(&ctl->bar, 1);
    for (u32 i = 0; i < P2_PIN; ++i) mbar_init(&pc->ibar[i], 1);
    for (int i = 0; i < NSTAT; ++i) ctl->st[i] = 0;
    pc->pool = (1u << p2_nsl<K, V>()) - 1u;
    pc->icons = 0; pc->rq_head = 0; pc->rq_done = 0; pc->place_done = 0; pc->mdone = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x >= NT) {
    if (threadIdx.x == NT) { if (b == 0) p.h1_root(); else p.h1_level(b); }
    if (threadIdx.x == NT + 32) p.h2_loop();
    return;
  }
  p.mycons = b == 0 ? P.ctl + PC_ROOTCONS : p.cons(b);
  const ull t0 = clock64();
  if (b == 0) p.root_stage();
  else p.level_stage(b);
  const u32 bt = b - ((C.debug & 524288u) ? 8u : 0u);  // debug 524288: stages 8..23
  if (threadIdx.x == 0 && (C.debug & 128u) && !(C.debug & 262144u) && bt < 16) {
    ull* tms = reinterpret_cast<ull*>(H.hdr + H_TIME);
    atomicAdd(tms + bt, p.twait);
    atomicAdd(tms + 16 + bt, (C.debug & 16384u) ? p.th2 : clock64() - t0);
  }
  if (threadIdx.x == 0) {
    ull* stat = reinterpret_cast<ull*>(H.hdr + H_STAT);
    for (int i = 0; i < NSTAT; ++i)
      if (ctl->st[i]) atomicAdd(stat + i, ctl->st[i]);
  }
}

}  // namespace bgpqd
