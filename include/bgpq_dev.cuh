/* include/bgpq_dev.cuh — device API of the BGPQ library (last bullet): one
 * BGPQ_INSERT or BGPQ_DELETEMIN executed cooperatively by the compute threads of one CTA
 * inside an application kernel, on a heap created with bgpq_create_ex (include/bgpq.h) and
 * exported with bgpq_view().  This is how the paper's applications use the queue (P:477-481:
 * "A thread block in BGPQ always retrieves a full node from the priority queue"; P:166-174:
 * many thread blocks operate on the heap concurrently, task parallelism across nodes and data
 * parallelism inside a node).
 *
 * The operations are the per-node-lock execution of Alg.1 (INSERT) and Alg.2+3 (DELETEMIN)
 * (bgpq_locks.cuh, OpL), linearizable at the root section: any number of CTAs of any
 * number of kernels on one stream may call them concurrently on the same heap, as long as no
 * library call (bgpq_insert / bgpq_deletemin / ...) runs on that heap at the same time.
 *
 * Launch contract of a kernel that uses a Queue<K, V, NT>:
 *   - blockDim.x == NT + 32: threads [0, NT) are the compute threads that call insert /
 *     deletemin / sync; warp NT/32 is the queue's lock warp (Queue::run_lock_warp);
 *   - dynamic shared memory >= Queue::smem_bytes(), the queue's part starting at the pointer
 *     given to init() (128-B aligned); the application may use the rest;
 *   - all CTAs of the grid co-resident (the locks are spin locks), one CTA per SM at most
 *     occupancy as cudaOccupancyMaxActiveBlocksPerMultiprocessor reports;
 *   - K and V (values stored) must match the heap's K and BGPQ_FLAG_VALUES.
 * Pointers given to insert / deletemin are generic: global or shared memory.
 */
#pragma once

#include "../paper_conf_icpp_chenhjz21_b200/csrc/bgpq_locks.cuh"

namespace bgpq_dev {

using bgpqd::u32;
using bgpqd::u64;
using bgpqd::ull;

// Device pointers of one heap (bgpq_view_t of include/bgpq.h, cast).
struct HeapView {
  u32* keys;                // node keys, slot i at keys + i*K (0 = pBuffer, 1 = root)
  u32* vals;                // node values (nullptr for a keys-only heap)
  bgpqd::NodeMeta* meta;    // per-node lock / state / cached min-max
  u32* hdr;                 // header words (heapSize, |root|, |pBuffer|, sticky error, ...)
  u32 cap;                  // largest node index
};

template <int K, bool V, int NT = 512>
struct Queue {
  bgpqd::OpL<K, V, NT> op;

  __host__ __device__ static constexpr size_t smem_bytes() {
    return bgpqd::LCTL_BYTES + (size_t)bgpqd::LSLOT * K * 4 * (V ? 2 : 1);
  }
  __host__ __device__ static constexpr int block_threads() { return NT + 32; }

  // All threads of the CTA; ends with __syncthreads().
  __device__ __forceinline__ void init(const HeapView& h, unsigned char* smem) {
    bgpqd::HeapArgs H;
    H.gk = h.keys;
    H.gv = V ? h.vals : nullptr;
    H.meta = h.meta;
    H.hdr = h.hdr;
    H.cap = h.cap;
    H.xk = nullptr;  // carried-keys sources are heap nodes here (no cluster-engine scratch)
    H.xv = nullptr;
    bgpqd::LCtl* ctl = reinterpret_cast<bgpqd::LCtl*>(smem);
    op.H = H;
    op.ctl = ctl;
    op.sk = reinterpret_cast<u32*>(smem + bgpqd::LCTL_BYTES);
    op.sv = op.sk + bgpqd::LSLOT * K;
    op.mphase = 0; op.pph = 0; op.tphase = 0; op.pb = 0;
    op.st = ctl->st;
    op.tm = ctl->tm;
    op.timing = false;
    if (threadIdx.x == 0) {
      for (int i = 0; i < bgpqd::NSTAT; ++i) ctl->st[i] = 0;
      bgpqd::mbar_init(&ctl->bar, 1);
      bgpqd::mbar_init(&ctl->pbar[0], 1);
      bgpqd::mbar_init(&ctl->pbar[1], 1);
      bgpqd::mbar_init(&ctl->tbar, 1);
      ctl->freemask = (1u << bgpqd::LSLOT) - 1u;
      ctl->p_req = 0; ctl->t_req = 0; ctl->t_done = 0; ctl->stop = 0; ctl->t_marked = 0;
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
  }
  __device__ __forceinline__ bool is_lock_warp() const { return threadIdx.x >= NT; }
  // The lock warp's loop (agents P and T); returns after finish().
  __device__ __forceinline__ void run_lock_warp() { bgpqd::lock_warp<K, V, NT>(op); }
  // Barrier over the NT compute threads (named barrier 1).
  __device__ __forceinline__ void sync() const { bgpqd::cta_bar<NT>(); }

  // BGPQ_INSERT of n in 1..K entries (Alg.1).  Compute threads only.
  __device__ __forceinline__ void insert(const u32* k, const u32* v, u32 n) {
    op.insert(k, V ? v : nullptr, n, nullptr);
  }
  // BGPQ_DELETEMIN of up to n in 1..K entries (Alg.2+3): the min(n, size) smallest keys,
  // ascending, to ok / ov.  Returns the count (identical in every compute thread).
  __device__ __forceinline__ u32 deletemin(u32* ok, u32* ov, u32 n) {
    const u32 c = op.deletemin(ok, V ? ov : nullptr, n, 0, nullptr);
    sync();
    if (threadIdx.x == 0) op.ctl->b[23] = c;
    sync();
    const u32 r = op.ctl->b[23];
    sync();
    if (threadIdx.x == 0) op.st[bgpqd::S_KEYS_OUT] += r;
    return r;
  }
  // Approximate number of keys in the heap from the header words, read without the root
  // lock (a hint: exact at quiescence).  Identical in every compute thread.  Lets a CTA that
  // would only find an empty heap back off instead of taking the root lock away from
  // the CTAs that are inserting.
  __device__ __forceinline__ u64 size_hint() {
    sync();
    if (threadIdx.x == 0) {
      const u32 hs = bgpqd::ld_relaxed(op.H.hdr + bgpqd::H_HS);
      const u32 rs = bgpqd::ld_relaxed(op.H.hdr + bgpqd::H_RS);
      const u32 ps = bgpqd::ld_relaxed(op.H.hdr + bgpqd::H_PS);
      const u64 n = hs == 0 ? 0ull : (u64)rs + ps + (u64)(hs - 1) * K;
      op.ctl->b[22] = n > 0xFFFFFFFFull ? 0xFFFFFFFFu : (u32)n;
    }
    sync();
    const u64 r = op.ctl->b[22];
    sync();
    return r;
  }
  // Compute threads: stop the lock warp and add this CTA's device counters to the heap's.
  __device__ __forceinline__ void finish() {
    sync();
    if (threadIdx.x == 0) {
      bgpqd::st_rel_cta(&op.ctl->stop, 1u);
      ull* stat = reinterpret_cast<ull*>(op.H.hdr + bgpqd::H_STAT);
      for (int i = 0; i < bgpqd::NSTAT; ++i)
        if (op.st[i]) atomicAdd(stat + i, op.st[i]);
    }
  }
};

}  // namespace bgpq_dev
