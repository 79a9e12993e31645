/*
 * tq_device.cuh -- device-side, warp-collective operations of the retry-free,
 * arbitrary-n queue (Troendle, Ta & Jang, ICPP 2019; PAPER.md cited P:<line>)
 * for sm_100a.
 *
 * Calling convention: every function named tq_warp_* is warp-collective and
 * must be called by all 32 lanes of a warp together (convergent, mask
 * 0xffffffff); lanes that do not take part pass hungry = false / n = 0.  Lane 0
 * is the proxy: "We arbitrarily chose the first thread in each wavefront as
 * the proxy thread" (§4.1); on sm_100a a warp is 32 lanes.
 *
 * Slot protocol (see tq.h): slot[t & mask] = {item:32 | seq:32}.
 *   empty for ticket t  : seq == (u32)t        (the paper's dna sentinel)
 *   item for ticket t   : seq == (u32)(t + 1)
 *   after the take      : seq := (u32)(t + C)   (empty for ticket t + C)
 * A writer that does not find "empty for t" has hit the queue-full exception
 * and aborts (no retry; Listing 3 line 25).
 *
 * Memory ordering: slot polls and the writer's full check use ld.relaxed.gpu
 * (served by L2, never a stale L1 line); publication is ordered after the
 * producer's prior writes by a gpu-scope fence; a consumer that finds data
 * issues a gpu-scope fence before reading the task's state.
 */
#ifndef TQ_DEVICE_CUH_
#define TQ_DEVICE_CUH_

#include <stdint.h>
#include "tq.h"

#define TQ_FULL_MASK 0xffffffffu
#define TQ_STATUS_COPIES 32 /* replicas of the status word, 128 B apart */
#define TQ_STATUS_STRIDE 32 /* in uint32 words */
#define TQ_NO_TICKET 0xffffffffffffffffull

/* ---------------------------------------------------------------- */
/* Memory-model helpers (PTX ISA memory consistency model, sm_70+)   */
/* ---------------------------------------------------------------- */
__device__ __forceinline__ unsigned long long tq_ld_relaxed(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned int tq_ld_relaxed_u32(const unsigned int *p)
{
    unsigned int v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long tq_ld_acquire(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
/* fire-and-forget add with release semantics (completion counter) */
__device__ __forceinline__ void tq_red_add_release(unsigned long long *p, unsigned long long v)
{
    asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void tq_red_add_relaxed(unsigned long long *p, unsigned long long v)
{
    asm volatile("red.relaxed.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
/* Release fence (sm_100a SASS: MEMBAR.ALL.GPU; unlike fence.acq_rel it does
 * not also invalidate L1).  An acquire is cheaper as a load: ld.acquire.gpu
 * is LDG.STRONG.GPU + CCTL.IVALL, with no membar. */
__device__ __forceinline__ void tq_fence_release()
{
    asm volatile("fence.release.gpu;" ::: "memory");
}
__device__ __forceinline__ void tq_st_relaxed(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void tq_st_relaxed_u32(unsigned int *p, unsigned int v)
{
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void tq_fence_gpu()
{
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
/* atomic fetch-add with acquire-release semantics (termination counter) */
__device__ __forceinline__ unsigned long long tq_atom_add_acqrel(unsigned long long *p,
                                                                 unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
/* relaxed fetch-add: the AFA of the paper (§3.2) */
__device__ __forceinline__ unsigned long long tq_atom_add(unsigned long long *p, unsigned long long v)
{
    unsigned long long old;
    asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old) : "l"(p), "l"(v) : "memory");
    return old;
}
__device__ __forceinline__ unsigned long long tq_atom_cas(unsigned long long *p,
                                                          unsigned long long cmp,
                                                          unsigned long long val)
{
    unsigned long long old;
    asm volatile("atom.relaxed.gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old) : "l"(p), "l"(cmp), "l"(val) : "memory");
    return old;
}
__device__ __forceinline__ unsigned int tq_lane()
{
    unsigned int l;
    asm("mov.u32 %0, %%laneid;" : "=r"(l));
    return l;
}
__device__ __forceinline__ unsigned int tq_lanemask_lt()
{
    unsigned int m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}
__device__ __forceinline__ unsigned long long tq_shfl64(unsigned long long v, int src)
{
    unsigned lo = __shfl_sync(TQ_FULL_MASK, (unsigned)v, src);
    unsigned hi = __shfl_sync(TQ_FULL_MASK, (unsigned)(v >> 32), src);
    return ((unsigned long long)hi << 32) | lo;
}
__device__ __forceinline__ unsigned long long tq_globaltimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

/* ---------------------------------------------------------------- */
/* Status word (WorkRemains / abort; Alg 1 line 1)             */
/* ---------------------------------------------------------------- */
__device__ __forceinline__ unsigned int tq_status_read(const tq_device_view &q, unsigned int warp_gid)
{
    return tq_ld_relaxed_u32(q.status + (warp_gid % TQ_STATUS_COPIES) * TQ_STATUS_STRIDE);
}
/* single-thread: write every replica */
__device__ __forceinline__ void tq_status_set_thread(const tq_device_view &q, unsigned int s)
{
    for (int i = 0; i < TQ_STATUS_COPIES; ++i)
        atomicMax(q.status + i * TQ_STATUS_STRIDE, s);
}
/* warp-collective: lane i writes replica i */
__device__ __forceinline__ void tq_warp_status_set(const tq_device_view &q, unsigned int s)
{
    atomicMax(q.status + tq_lane() * TQ_STATUS_STRIDE, s);
}

/* ---------------------------------------------------------------- */
/* Listing 1: dequeue reservation by the proxy lane.      */
/* Hungry lanes are counted with a ballot (the paper's local          */
/* atomic_inc on lQueueSlotsNeeded) and ranked in lane order;  */
/* lane 0 performs the single atomic_add(Front, n) only if n > 0      */
/* (P:238).  Returns the lane's ticket, TQ_NO_TICKET if not hungry.   */
/* *atomics is incremented on lane 0 when an atomic was issued.       */
/* ---------------------------------------------------------------- */
__device__ __forceinline__ unsigned long long tq_warp_dequeue_n(const tq_device_view &q, bool hungry,
                                                                unsigned int *atomics = nullptr)
{
    const unsigned m = __ballot_sync(TQ_FULL_MASK, hungry);
    if (m == 0) return TQ_NO_TICKET;
    unsigned long long base = 0;
    if (tq_lane() == 0) {
        base = tq_atom_add(q.front, (unsigned long long)__popc(m));
        if (atomics) ++*atomics;
    }
    base = tq_shfl64(base, 0);
    return hungry ? base + __popc(m & tq_lanemask_lt()) : TQ_NO_TICKET;
}

/* ---------------------------------------------------------------- */
/* Listing 2: data-arrival check of one ticket.  A plain  */
/* (non-atomic) load of the lane's unique slot; if the item has       */
/* arrived the lane takes it and puts the slot back to dna for the    */
/* next lap ("picks up its work token from its slot and replaces it   */
/* with the sentinel").  Non-blocking; per lane.               */
/* ---------------------------------------------------------------- */
/* The arrival check alone (Listing 2 lines 3-5), an acquire load: true if
 * the item for `ticket` has arrived, and then everything the producer wrote
 * before publishing it is visible.  The caller takes it by storing
 * seq = ticket + C to the slot (the reset half of tq_take). */
__device__ __forceinline__ bool tq_poll(const tq_device_view &q, unsigned long long ticket,
                                        unsigned int *item)
{
    if (ticket == TQ_NO_TICKET) return false;
    const unsigned long long v = tq_ld_acquire(q.slots + (ticket & q.mask));
    if ((unsigned int)v != (unsigned int)(ticket + 1)) return false;
    *item = (unsigned int)(v >> 32);
    return true;
}

__device__ __forceinline__ bool tq_take(const tq_device_view &q, unsigned long long ticket,
                                        unsigned int *item)
{
    if (ticket == TQ_NO_TICKET) return false;
    unsigned long long *s = q.slots + (ticket & q.mask);
    const unsigned long long v = tq_ld_acquire(s);
    if ((unsigned int)v != (unsigned int)(ticket + 1)) return false;
    *item = (unsigned int)(v >> 32);
    tq_st_relaxed(s, (unsigned long long)(unsigned int)(ticket + q.mask + 1));
    return true;
}

/* tq_take with a relaxed arrival check (ld.relaxed.gpu: served by L2, no
 * L1 invalidation per poll).  For items that carry their whole payload: a
 * hit makes the item visible, but NOT other data the producer wrote before
 * publishing it -- use tq_take when the item names such data. */
__device__ __forceinline__ bool tq_take_relaxed(const tq_device_view &q, unsigned long long ticket,
                                                unsigned int *item)
{
    if (ticket == TQ_NO_TICKET) return false;
    unsigned long long *s = q.slots + (ticket & q.mask);
    const unsigned long long v = tq_ld_relaxed(s);
    if ((unsigned int)v != (unsigned int)(ticket + 1)) return false;
    *item = (unsigned int)(v >> 32);
    tq_st_relaxed(s, (unsigned long long)(unsigned int)(ticket + q.mask + 1));
    return true;
}

/* ---------------------------------------------------------------- */
/* Listing 3: enqueue.                                    */
/* tq_warp_reserve_rear: lane 0 reserves `n_warp` tickets at Rear     */
/* with one AFA (only if n_warp > 0); returns the base on all  */
/* lanes.                                                             */
/* tq_publish: per lane, write one item to its reserved ticket after  */
/* checking the slot still holds the dna sentinel for that ticket;    */
/* otherwise raise the queue-full abort (P:268 line 25).  The caller  */
/* must have issued tq_fence_release() after producing the task state the */
/* item refers to.                                                    */
/* ---------------------------------------------------------------- */
__device__ __forceinline__ unsigned long long tq_warp_reserve_rear(const tq_device_view &q,
                                                                   unsigned int n_warp,
                                                                   unsigned int *atomics = nullptr)
{
    unsigned long long base = 0;
    if (n_warp == 0) return 0;
    if (tq_lane() == 0) {
        base = tq_atom_add(q.rear, (unsigned long long)n_warp);
        if (atomics) ++*atomics;
    }
    return tq_shfl64(base, 0);
}

__device__ __forceinline__ bool tq_publish(const tq_device_view &q, unsigned long long ticket,
                                           unsigned int item)
{
    unsigned long long *s = q.slots + (ticket & q.mask);
    const unsigned long long v = tq_ld_relaxed(s);
    if ((unsigned int)v != (unsigned int)ticket) {
        tq_status_set_thread(q, TQ_ABORTED_FULL);
        return false;
    }
    tq_st_relaxed(s, ((unsigned long long)item << 32) | (unsigned int)(ticket + 1));
    return true;
}

/* Warp-collective enqueue of n_mine items per lane from a per-lane array
 * (n_mine <= 32 typical).  One AFA for the whole warp (arbitrary-n);
 * lane i writes its items at base + exclusive_prefix(n) + j.  Returns the
 * lane's first ticket, or TQ_NO_TICKET if the queue was full. */
template <int MAXN>
__device__ __forceinline__ unsigned long long tq_warp_enqueue_n(const tq_device_view &q,
                                                                unsigned int n_mine,
                                                                const unsigned int (&items)[MAXN],
                                                                unsigned int *atomics = nullptr)
{
    const unsigned lane = tq_lane();
    unsigned incl = n_mine;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned t = __shfl_up_sync(TQ_FULL_MASK, incl, o);
        if (lane >= (unsigned)o) incl += t;
    }
    const unsigned total = __shfl_sync(TQ_FULL_MASK, incl, 31);
    const unsigned long long base = tq_warp_reserve_rear(q, total, atomics);
    tq_fence_release();
    const unsigned long long mine = base + (incl - n_mine);
    bool ok = true;
#pragma unroll
    for (int j = 0; j < MAXN; ++j)
        if ((unsigned)j < n_mine) ok &= tq_publish(q, mine + j, items[j]);
    return ok ? mine : TQ_NO_TICKET;
}

#endif /* TQ_DEVICE_CUH_ */
