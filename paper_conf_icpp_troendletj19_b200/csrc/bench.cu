// bench.cu -- queue micro-benchmark (BASELINE.json configs[1]):
// every warp repeatedly enqueues `batch` unique items, reserves `batch`
// dequeue tickets, waits for its items to arrive and consumes them, for the
// RF/AN queue (Listings 1-3) and the comparison queues
// (per-thread AFA, CAS-retry BASE, AN).  The retry ratio of
// Fig 5 is atomics_issued / items.
#include "internal.cuh"
#ifdef TQ_DEBUG_PIPE
#include <cstdio>
#endif

namespace tqk {

enum BenchOut {
    BO_ENQ = 0, BO_DEQ, BO_ATOM, BO_FAIL, BO_EMPTY, BO_SUM_ENQ, BO_SUM_DEQ, BO_XOR_ENQ, BO_XOR_DEQ,
    BO_SINK, BO_COUNT_
};

// Twin of inputs/items.py:item_of (a bijection on 32-bit integers).
__device__ __forceinline__ uint32_t item_of(uint32_t seed32, unsigned long long g)
{
    uint32_t x = (uint32_t)g ^ seed32;
    x *= 0x9E3779B1u;
    x ^= x >> 16;
    x *= 0x85EBCA6Bu;
    x ^= x >> 13;
    return x;
}

// Twin of inputs/graphs.py:_mix64 (splitmix64 finaliser), item fingerprints.
__device__ __forceinline__ unsigned long long mix64(unsigned long long x)
{
    x ^= x >> 30;
    x *= 0xBF58476D1CE4E5B9ull;
    x ^= x >> 27;
    x *= 0x94D049BB133111EBull;
    x ^= x >> 31;
    return x;
}

__device__ __forceinline__ bool bench_publish(const tq_device_view &q, unsigned long long t, uint32_t item)
{
    return tq_publish(q, t, item);
}

// Bounded, randomised exponential back-off after a failed CAS
// (tq_bench_cfg.cas_backoff_ns; 0 = retry at once, the naive form), the same
// two forms as the BFS comparators (bfs.cu): per-thread BASE lanes sit out a
// random number of ~32 ns retry rounds (lanes of a warp fail together and a
// sleep would stall the warp as a unit); the AN proxy's warp sleeps a random
// time in [window/2, window].  The window doubles from 32 ns up to bo_max.
__device__ __forceinline__ unsigned b_rand()
{
    unsigned r;
    asm volatile("mov.u32 %0, %%globaltimer_lo;" : "=r"(r));
    r ^= (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u;
    r ^= r >> 15;
    r *= 0x2C1B3C6Du;
    r ^= r >> 12;
    return r;
}
struct BLaneBackoff {
    unsigned win = 0, skip = 0;
};
__device__ __forceinline__ bool b_backoff_wait(BLaneBackoff &b)
{
    if (!b.skip) return false;
    --b.skip;
    __nanosleep(32);
    return true;
}
__device__ __forceinline__ void b_backoff_fail(BLaneBackoff &b, unsigned bo_max)
{
    if (!bo_max) return;
    const unsigned maxw = bo_max / 32 > 1 ? bo_max / 32 : 1;
    b.win = b.win ? min(2 * b.win, maxw) : 1;
    b.skip = b_rand() % (b.win + 1);
}
__device__ __forceinline__ void b_backoff(unsigned *bo, unsigned bo_max)
{
    if (!bo_max) return;
    *bo = *bo ? min(*bo * 2, bo_max) : min(32u, bo_max);
    const unsigned r = __shfl_sync(TQ_FULL_MASK, b_rand(), 0);  // one draw per warp
    __nanosleep(*bo / 2 + r % (*bo / 2 + 1));
}

// BASE enqueue / dequeue with the ticket returned (for the logs)
__device__ __forceinline__ bool b_cas_enqueue(const tq_device_view &q, uint32_t item,
                                              unsigned long long *t_out, unsigned *atom, unsigned *fail,
                                              unsigned bo_max)
{
    BLaneBackoff bo;
    for (unsigned tries = 0; tries < (1u << 24); ++tries) {
        if (b_backoff_wait(bo)) continue;
        const unsigned long long pos = tq_ld_relaxed(q.rear);
        unsigned long long *s = q.slots + (pos & q.mask);
        const unsigned long long v = tq_ld_relaxed(s);
        const int dif = (int)((unsigned)v - (unsigned)pos);
        if (dif == 0) {
            ++*atom;
            if (tq_atom_cas(q.rear, pos, pos + 1) == pos) {
                tq_st_relaxed(s, ((unsigned long long)item << 32) | (unsigned)(pos + 1));
                *t_out = pos;
                return true;
            }
            ++*fail;
            b_backoff_fail(bo, bo_max);
        } else if (dif < 0) {
            tq_status_set_thread(q, TQ_ABORTED_FULL);
            return false;
        }
    }
    tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
    return false;
}

__device__ __forceinline__ int b_cas_dequeue(const tq_device_view &q, uint32_t *item,
                                             unsigned long long *t_out, unsigned *atom, unsigned *fail,
                                             unsigned bo_max)
{
    BLaneBackoff bo;
    for (unsigned tries = 0; tries < (1u << 12); ++tries) {
        if (b_backoff_wait(bo)) continue;
        const unsigned long long pos = tq_ld_relaxed(q.front);
        unsigned long long *s = q.slots + (pos & q.mask);
        const unsigned long long v = tq_ld_relaxed(s);
        const int dif = (int)((unsigned)v - (unsigned)(pos + 1));
        if (dif == 0) {
            ++*atom;
            if (tq_atom_cas(q.front, pos, pos + 1) == pos) {
                *item = (uint32_t)(v >> 32);
                tq_st_relaxed(s, (unsigned long long)(unsigned)(pos + q.mask + 1));
                *t_out = pos;
                return 1;
            }
            ++*fail;
            b_backoff_fail(bo, bo_max);
        } else if (dif < 0) {
            return 0;
        }
    }
    return 0;
}

// polled every 1024 empty spins: watchdog + abort propagation
__device__ __noinline__ bool should_stop(const tq_device_view &q, unsigned warp, unsigned long long deadline)
{
    if (tq_globaltimer() > deadline) tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
    return tq_status_read(q, warp) != TQ_RUNNING;
}

template <int VARIANT>
__global__ void __launch_bounds__(256) bench_kernel(const BenchParams p)
{
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long warp_gid = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const tq_device_view q = p.q;
    const unsigned long long cap = q.mask + 1;
    const bool active = (int)lane < p.batch;
    unsigned n_enq = 0, n_deq = 0, atom = 0, fail = 0, empty = 0;
    unsigned long long s_enq = 0, s_deq = 0, x_enq = 0, x_deq = 0, sink = 0;
    const unsigned long long deadline = tq_globaltimer() + p.timeout_ns;
    bool stop = false;
    // RF_AN_CTA: the proxy group is the whole CTA (double-buffered bases)
    __shared__ unsigned long long cta_base[2][2];
    const unsigned wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;

    // (the CTA variant leaves the loop only through its block-wide vote)
    for (int it = 0; it < p.iters && (VARIANT == TQ_VARIANT_RF_AN_CTA || !stop); ++it) {
        const unsigned long long g = (warp_gid * (unsigned long long)p.iters + it) * p.batch + lane;
        const uint32_t item = item_of(p.seed32, g);

        if constexpr (VARIANT == TQ_VARIANT_RF_AN_CTA) {
            // One thread reserves the enqueue tickets and the dequeue tickets
            // of all warps of the block (arbitrary-n with a CTA-wide proxy
            // group, "a proxy thread in each thread group"); warp w owns
            // [base + w*b, base + (w+1)*b) of each.
            unsigned long long *cb = cta_base[it & 1];
            if (threadIdx.x == 0) {
                const unsigned long long n = (unsigned long long)nwb * p.batch;
                cb[0] = tq_atom_add(q.rear, n);
                cb[1] = tq_atom_add(q.front, n);
                atom += 2;
            }
            if (__syncthreads_or(stop)) break;
            const unsigned long long et = cb[0] + (unsigned long long)wib * p.batch + lane;
            const unsigned long long dt = cb[1] + (unsigned long long)wib * p.batch + lane;
            bool eok = true;
            if (active) {
                eok = bench_publish(q, et, item);
                if (eok) {
                    ++n_enq;
                    const unsigned long long f = mix64(item);
                    s_enq += f;
                    x_enq ^= f;
                    if (p.enq_log) p.enq_log[et] = item;
                }
            }
            if (active && eok) {
                uint32_t got_item = 0;
                unsigned spins = 0;
                bool have = false;
                while (!have) {
                    have = p.relaxed_poll ? tq_take_relaxed(q, dt, &got_item) : tq_take(q, dt, &got_item);
                    if (!have && (++spins & 1023) == 0 && should_stop(q, (unsigned)warp_gid, deadline)) {
                        stop = true;
                        break;
                    }
                    if (!have) ++empty;
                }
                if (have) {
                    ++n_deq;
                    const unsigned long long f = mix64(got_item);
                    s_deq += f;
                    x_deq ^= f;
                    if (p.deq_log) p.deq_log[dt] = got_item;
                    uint32_t x = got_item;
                    for (int w = 0; w < p.work_iters; ++w) x = x * 1664525u + 1013904223u;
                    sink += x;
                }
            } else if (active) {
                stop = true;
            }
            continue;
        } else if constexpr (VARIANT == TQ_VARIANT_ATOMIC_CEILING) {
            if (lane == 0) {
                sink += tq_atom_add(q.rear, (unsigned long long)p.batch);
                ++atom;
            }
            if (active) {
                ++n_enq;
                ++n_deq;
            }
            continue;
        } else {
            // ------------------------------ enqueue ------------------------------
            unsigned long long et = 0;
            bool eok = true;
            if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
                const unsigned long long base = tq_warp_reserve_rear(q, (unsigned)p.batch, &atom);
                et = base + lane;
                if (active) eok = bench_publish(q, et, item);
            } else if constexpr (VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
                if (active) {
                    et = tq_atom_add(per_lane_addr(q.rear), 1ull);
                    ++atom;
                    eok = bench_publish(q, et, item);
                }
            } else if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
                if (active) eok = b_cas_enqueue(q, item, &et, &atom, &fail, p.cas_backoff_ns);
            } else {  // AN: proxy CAS loop reserving `batch` slots
                unsigned long long base = 0;
                unsigned spins = 0, bo = 0;
                for (;;) {
                    if ((++spins & 1023) == 0 && should_stop(q, (unsigned)warp_gid, deadline)) {
                        eok = false;
                        break;
                    }
                    unsigned long long pos = 0;
                    if (lane == 0) pos = tq_ld_relaxed(q.rear);
                    pos = tq_shfl64(pos, 0);
                    int dif = 0;
                    if (active) dif = (int)((unsigned)tq_ld_relaxed(q.slots + ((pos + lane) & q.mask)) -
                                            (unsigned)(pos + lane));
                    if (__any_sync(TQ_FULL_MASK, dif > 0)) continue;
                    if (__any_sync(TQ_FULL_MASK, dif < 0)) {
                        if (lane == 0) tq_status_set_thread(q, TQ_ABORTED_FULL);
                        eok = false;
                        break;
                    }
                    unsigned long long old = 0;
                    if (lane == 0) {
                        ++atom;
                        old = tq_atom_cas(q.rear, pos, pos + (unsigned)p.batch);
                        if (old != pos) ++fail;
                    }
                    old = tq_shfl64(old, 0);
                    if (old == pos) {
                        base = pos;
                        break;
                    }
                    b_backoff(&bo, p.cas_backoff_ns);
                }
                et = base + lane;
                if (active && eok) tq_st_relaxed(q.slots + (et & q.mask),
                                                 ((unsigned long long)item << 32) | (unsigned)(et + 1));
            }
            if (active && eok) {
                ++n_enq;
                const unsigned long long f = mix64(item);
                s_enq += f;
                x_enq ^= f;
                if (p.enq_log) p.enq_log[et] = item;
            }
            if (__any_sync(TQ_FULL_MASK, active && !eok)) break;

            // ------------------------------ dequeue ------------------------------
            uint32_t got_item = 0;
            unsigned long long dt = 0;
            bool have = !active;  // inactive lanes need nothing
            if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
                if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
                    dt = tq_warp_dequeue_n(q, active, &atom);
                } else if (active) {
                    dt = tq_atom_add(per_lane_addr(q.front), 1ull);
                    ++atom;
                }
                unsigned spins = 0;
                while (!have) {
                    have = p.relaxed_poll ? tq_take_relaxed(q, dt, &got_item) : tq_take(q, dt, &got_item);
                    if (!have) {
                        ++empty;
                        if ((++spins & 1023) == 0 &&
                            should_stop(q, (unsigned)warp_gid, deadline)) {
                            stop = true;
                            break;
                        }
                    }
                }
            } else if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
                unsigned spins = 0;
                while (!have) {
                    have = b_cas_dequeue(q, &got_item, &dt, &atom, &fail, p.cas_backoff_ns);
                    if (!have) {
                        ++empty;
                        if ((++spins & 1023) == 0 &&
                            should_stop(q, (unsigned)warp_gid, deadline)) {
                            stop = true;
                            break;
                        }
                    }
                }
            } else {  // AN: the proxy reserves up to n ready slots per CAS
                unsigned spins = 0, bo = 0;
                for (;;) {
                    const bool need = !have;
                    const unsigned m = __ballot_sync(TQ_FULL_MASK, need);
                    if (m == 0) break;
                    if ((++spins & 1023) == 0 && should_stop(q, (unsigned)warp_gid, deadline)) {
                        stop = true;
                        break;
                    }
                    const unsigned n = __popc(m);
                    unsigned long long pos = 0;
                    if (lane == 0) pos = tq_ld_relaxed(q.front);
                    pos = tq_shfl64(pos, 0);
                    int dif = -1;
                    if (lane < n) dif = (int)((unsigned)tq_ld_relaxed(q.slots + ((pos + lane) & q.mask)) -
                                              (unsigned)(pos + lane + 1));
                    const unsigned rm = __ballot_sync(TQ_FULL_MASK, lane < n && dif == 0);
                    const unsigned k = rm == TQ_FULL_MASK ? 32u : (unsigned)(__ffs(~rm) - 1);
                    if (k == 0) {
                        if (!__any_sync(TQ_FULL_MASK, lane < n && dif > 0) && lane == 0) ++empty;
                        continue;
                    }
                    unsigned long long old = 0;
                    if (lane == 0) {
                        ++atom;
                        old = tq_atom_cas(q.front, pos, pos + k);
                        if (old != pos) ++fail;
                    }
                    old = tq_shfl64(old, 0);
                    if (old != pos) {
                        b_backoff(&bo, p.cas_backoff_ns);
                        continue;
                    }
                    const unsigned rank = __popc(m & tq_lanemask_lt());
                    if (need && rank < k) {
                        dt = pos + rank;
                        unsigned long long *s = q.slots + (dt & q.mask);
                        got_item = (uint32_t)(tq_ld_relaxed(s) >> 32);
                        tq_st_relaxed(s, (unsigned long long)(unsigned)(dt + cap));
                        have = true;
                    }
                }
                stop = __any_sync(TQ_FULL_MASK, stop);
            }
            if (active && have) {
                ++n_deq;
                const unsigned long long f = mix64(got_item);
                s_deq += f;
                x_deq ^= f;
                if (p.deq_log) p.deq_log[dt] = got_item;
                uint32_t x = got_item;
                for (int w = 0; w < p.work_iters; ++w) x = x * 1664525u + 1013904223u;
                sink += x;
            }
            stop = __any_sync(TQ_FULL_MASK, stop);
        }
    }

    // reduce and publish
    unsigned long long v[BO_COUNT_] = {n_enq, n_deq, atom, fail, empty, s_enq, s_deq, 0, 0, sink};
#pragma unroll
    for (int k = 0; k < BO_COUNT_; ++k) {
        if (k == BO_XOR_ENQ || k == BO_XOR_DEQ) continue;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_xor_sync(TQ_FULL_MASK, v[k], o);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        x_enq ^= __shfl_xor_sync(TQ_FULL_MASK, x_enq, o);
        x_deq ^= __shfl_xor_sync(TQ_FULL_MASK, x_deq, o);
    }
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < BO_COUNT_; ++k) {
            if (k == BO_XOR_ENQ || k == BO_XOR_DEQ) continue;
            if (v[k]) atomicAdd(p.out + k, v[k]);
        }
        atomicXor(p.out + BO_XOR_ENQ, x_enq);
        atomicXor(p.out + BO_XOR_DEQ, x_deq);
    }
}

// ---------------------------------------------------------------------------
// Pipelined variant (tq_bench_cfg.depth = 2): the group's proxy reserves the
// Rear and Front tickets of iteration k+1 at the start of iteration k, so the
// two atomics' latency overlaps the poll of iteration k, and the items of
// iteration k+1 are published right after it; a dequeue then finds its item
// already published one iteration earlier instead of waiting for another
// group's producer to catch up.  Each warp still enqueues and dequeues b items
// per iteration (<= 2b in flight).  Proxy group: GROUP 1 = CTA (thread 0,
// bases through shared memory), 2 = thread-block cluster (CTA rank 0 thread 0,
// bases written into every CTA's shared memory over DSMEM, one barrier.cluster
// per iteration).  Not offered for single-warp groups: a group publishes
// iteration k+1's items only after its poll of k, so a slow group delays its
// consumers, and with 5920 independent warps the lag compounds until a
// consumer holds a ticket a whole ring lap behind Rear (queue full at C = 2^20
// with 0.4M items in flight, measured); CTA groups average it out.
//
// Deadlock freedom (all groups reserve the same gsz tickets on both counters
// together, so ranges align): in a state where every group is blocked polling,
// each group g has published all its Rear ranges but its last, and polls its
// second-to-last Front range.  The globally last Rear range is unpublished but
// no group polls the globally last Front range (it is some group's last), so
// at most G-1 unpublished ranges can hold the G polled ranges: some group is
// not blocked, and it publishes its last range before it polls again.
// ---------------------------------------------------------------------------
__device__ __forceinline__ unsigned cluster_ctarank()
{
    unsigned r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ unsigned cluster_nctarank()
{
    unsigned r;
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
    return r;
}
// store a u64 into CTA `rank`'s copy of the shared variable at `p`
__device__ __forceinline__ void st_dsmem_u64(void *p, unsigned rank, unsigned long long v)
{
    const unsigned a = (unsigned)__cvta_generic_to_shared(p);
    unsigned ra;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank));
    asm volatile("st.shared::cluster.u64 [%0], %1;" ::"r"(ra), "l"(v) : "memory");
}
__device__ __forceinline__ void cluster_barrier()
{
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int GROUP>
__global__ void __launch_bounds__(256) bench_pipe_kernel(const BenchParams p)
{
    const unsigned lane = threadIdx.x & 31;
    const unsigned long long warp_gid = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const tq_device_view q = p.q;
    const bool active = (int)lane < p.batch;
    const unsigned wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
    unsigned n_enq = 0, n_deq = 0, atom = 0, empty = 0;
    unsigned long long s_enq = 0, s_deq = 0, x_enq = 0, x_deq = 0, sink = 0;
    const unsigned long long deadline = tq_globaltimer() + p.timeout_ns;
    bool stop = false;

    unsigned crank = 0, csize = 1;
    if constexpr (GROUP == 2) {
        crank = cluster_ctarank();
        csize = cluster_nctarank();
    }
    // tickets per group per iteration and this lane's offset inside them
    const unsigned long long gsz = (unsigned long long)nwb * csize * p.batch;
    const unsigned long long off = ((unsigned long long)crank * nwb + wib) * p.batch + lane;
    const bool leader = threadIdx.x == 0 && crank == 0;
    // [parity][0 rear base, 1 front base, 2 stop]
    __shared__ unsigned long long sb[2][3];

    // Returns the group's (rear, front) bases reserved by the leader as
    // (ra, fa); false if the group must stop.  One synchronisation.
    auto distribute = [&](int par, unsigned long long ra, unsigned long long fa, unsigned long long lstop,
                          unsigned long long *rb, unsigned long long *fb) -> bool {
        if constexpr (GROUP == 1) {
            if (leader) {
                sb[par][0] = ra;
                sb[par][1] = fa;
            }
            const bool st = __syncthreads_or(stop);
            *rb = sb[par][0];
            *fb = sb[par][1];
            return !st;
        } else {
            if (leader) {
                for (unsigned r = 0; r < csize; ++r) {
                    st_dsmem_u64(&sb[par][0], r, ra);
                    st_dsmem_u64(&sb[par][1], r, fa);
                    st_dsmem_u64(&sb[par][2], r, lstop);
                }
            }
            cluster_barrier();
            *rb = sb[par][0];
            *fb = sb[par][1];
            return sb[par][2] == 0;
        }
    };
    auto item_at = [&](int it) -> uint32_t {
        return item_of(p.seed32, (warp_gid * (unsigned long long)p.iters + it) * p.batch + lane);
    };
    auto publish = [&](int it, unsigned long long rb) {
        if (!active) return;
        const unsigned long long et = rb + off;
        const uint32_t item = item_at(it);
        if (bench_publish(q, et, item)) {
            ++n_enq;
            const unsigned long long f = mix64(item);
            s_enq += f;
            x_enq ^= f;
            if (p.enq_log) p.enq_log[et] = item;
        } else {
#ifdef TQ_DEBUG_PIPE
            printf("full: warp %llu it %d ticket %llu slot %llx front %llu rear %llu\n", warp_gid, it, et,
                   tq_ld_relaxed(q.slots + (et & q.mask)), tq_ld_relaxed(q.front), tq_ld_relaxed(q.rear));
#endif
            stop = true;
        }
    };

    // prologue: reserve and publish iteration 0
    unsigned long long ra = 0, fa = 0, rb = 0, fb = 0;
    if (leader) {
        ra = tq_atom_add(q.rear, gsz);
        fa = tq_atom_add(q.front, gsz);
        atom += 2;
    }
    bool go = distribute(0, ra, fa, 0ull, &rb, &fb);
    if (go) publish(0, rb);
    unsigned long long dt = fb + off;

    for (int it = 0; go && it < p.iters; ++it) {
        const bool more = it + 1 < p.iters;
        unsigned long long lstop = 0;
        if (more && leader) {  // iteration it+1's tickets, in flight during the poll
            ra = tq_atom_add(q.rear, gsz);
            fa = tq_atom_add(q.front, gsz);
            atom += 2;
            if constexpr (GROUP == 2) lstop = tq_status_read(q, (unsigned)warp_gid) != TQ_RUNNING;
        }
        if (active && !stop) {
            uint32_t got_item = 0;
            unsigned spins = 0;
            bool have = false;
            while (!have) {
                have = p.relaxed_poll ? tq_take_relaxed(q, dt, &got_item) : tq_take(q, dt, &got_item);
                if (!have) {
                    ++empty;
                    if ((++spins & 1023) == 0 && should_stop(q, (unsigned)warp_gid, deadline)) {
                        stop = true;
                        break;
                    }
                }
            }
            if (have) {
                ++n_deq;
                const unsigned long long f = mix64(got_item);
                s_deq += f;
                x_deq ^= f;
                if (p.deq_log) p.deq_log[dt] = got_item;
                uint32_t x = got_item;
                for (int w = 0; w < p.work_iters; ++w) x = x * 1664525u + 1013904223u;
                sink += x;
            }
        }
        if (!more) break;
        go = distribute((it + 1) & 1, ra, fa, lstop, &rb, &fb);
        if (go) publish(it + 1, rb);
        dt = fb + off;
    }

    unsigned long long v[BO_COUNT_] = {n_enq, n_deq, atom, 0, empty, s_enq, s_deq, 0, 0, sink};
#pragma unroll
    for (int k = 0; k < BO_COUNT_; ++k) {
        if (k == BO_XOR_ENQ || k == BO_XOR_DEQ) continue;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v[k] += __shfl_xor_sync(TQ_FULL_MASK, v[k], o);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        x_enq ^= __shfl_xor_sync(TQ_FULL_MASK, x_enq, o);
        x_deq ^= __shfl_xor_sync(TQ_FULL_MASK, x_deq, o);
    }
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < BO_COUNT_; ++k) {
            if (k == BO_XOR_ENQ || k == BO_XOR_DEQ) continue;
            if (v[k]) atomicAdd(p.out + k, v[k]);
        }
        atomicXor(p.out + BO_XOR_ENQ, x_enq);
        atomicXor(p.out + BO_XOR_DEQ, x_deq);
    }
}

template <int V>
static cudaError_t launch_b(const BenchParams &p, int blocks, int block, cudaStream_t s)
{
    bench_kernel<V><<<blocks, block, 0, s>>>(p);
    return cudaGetLastError();
}

// group: 1 CTA, 2 cluster of `cluster` CTAs (blocks % cluster == 0)
cudaError_t launch_bench_pipe(int group, int cluster, const BenchParams &p, int blocks, int block,
                              cudaStream_t s)
{
    if (group == 1) {
        bench_pipe_kernel<1><<<blocks, block, 0, s>>>(p);
    } else {
        if (cluster < 1 || blocks % cluster) return cudaErrorInvalidValue;
        if (cluster > 8) {
            cudaError_t e = cudaFuncSetAttribute(bench_pipe_kernel<2>,
                                                 cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            if (e != cudaSuccess) return e;
        }
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(blocks);
        cfg.blockDim = dim3(block);
        cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = cluster;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        return cudaLaunchKernelEx(&cfg, bench_pipe_kernel<2>, p);
    }
    return cudaGetLastError();
}

cudaError_t bench_pipe_occupancy(int block, int *blocks_per_sm)
{
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_pipe_kernel<1>, block, 0);
}

// co-resident clusters of `cluster` CTAs of `block` threads on this device
cudaError_t bench_max_clusters(int cluster, int block, int *clusters)
{
    if (cluster > 8) {
        cudaError_t e =
            cudaFuncSetAttribute(bench_pipe_kernel<2>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(cluster * 148);
    cfg.blockDim = dim3(block);
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cluster;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaOccupancyMaxActiveClusters(clusters, bench_pipe_kernel<2>, &cfg);
}

cudaError_t launch_bench(int variant, const BenchParams &p, int blocks, int block, cudaStream_t s)
{
    switch (variant) {
    case TQ_VARIANT_RF_AN: return launch_b<TQ_VARIANT_RF_AN>(p, blocks, block, s);
    case TQ_VARIANT_PER_THREAD_AFA: return launch_b<TQ_VARIANT_PER_THREAD_AFA>(p, blocks, block, s);
    case TQ_VARIANT_CAS_RETRY: return launch_b<TQ_VARIANT_CAS_RETRY>(p, blocks, block, s);
    case TQ_VARIANT_AN: return launch_b<TQ_VARIANT_AN>(p, blocks, block, s);
    case TQ_VARIANT_ATOMIC_CEILING: return launch_b<TQ_VARIANT_ATOMIC_CEILING>(p, blocks, block, s);
    case TQ_VARIANT_RF_AN_CTA: return launch_b<TQ_VARIANT_RF_AN_CTA>(p, blocks, block, s);
    default: return cudaErrorInvalidValue;
    }
}

// ---------------------------------------------------------------------------
// Random-probe ceiling (tq_probe_ceiling): the expansion's mirror-probe access
// pattern alone -- a coalesced 4-byte index stream and one random byte probe
// per index through L2, 4 in flight per lane, the BFS kernel's block shape.
// ---------------------------------------------------------------------------
__global__ void probe_fill_kernel(uint32_t *idx, unsigned long long n, unsigned long long range,
                                  unsigned long long seed)
{
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        unsigned long long x = (i + 1) * 0x9E3779B97F4A7C15ull ^ seed;  // splitmix64 finaliser
        x ^= x >> 31;
        x *= 0xBF58476D1CE4E5B9ull;
        x ^= x >> 29;
        idx[i] = (uint32_t)(x % range);
    }
}

__global__ void __launch_bounds__(256) probe_ceiling_kernel(const uint32_t *idx, unsigned long long n,
                                                            const uint8_t *tab, unsigned long long *sink)
{
    const unsigned long long tid = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (unsigned long long i = tid; i < n; i += 4 * stride) {
        uint32_t u[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) u[j] = (i + j * stride < n) ? __ldg(idx + i + j * stride) : 0u;
        unsigned m[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) asm volatile("ld.global.cg.u8 %0, [%1];" : "=r"(m[j]) : "l"(tab + u[j]));
#pragma unroll
        for (int j = 0; j < 4; ++j) acc += m[j];
    }
    if (acc == 0xdeadbeefu) *sink = acc;  // keeps the probes live
}

cudaError_t probe_ceiling(unsigned long long table_bytes, unsigned long long probes, int blocks_per_sm,
                          cudaStream_t s, double *g_per_s)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    uint32_t *idx = nullptr;
    uint8_t *tab = nullptr;
    unsigned long long *sink = nullptr;
    cudaEvent_t a = nullptr, b = nullptr;
    cudaError_t e = cudaMalloc(&idx, probes * 4);
    if (e == cudaSuccess) e = cudaMalloc(&tab, table_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&sink, 8);
    if (e == cudaSuccess) e = cudaMemsetAsync(tab, 1, table_bytes, s);
    if (e == cudaSuccess) e = cudaEventCreate(&a);
    if (e == cudaSuccess) e = cudaEventCreate(&b);
    if (e == cudaSuccess) {
        probe_fill_kernel<<<sms * 8, 256, 0, s>>>(idx, probes, table_bytes, 12345ull);
        probe_ceiling_kernel<<<sms * blocks_per_sm, 256, 0, s>>>(idx, probes, tab, sink);  // warm-up
        cudaEventRecord(a, s);
        probe_ceiling_kernel<<<sms * blocks_per_sm, 256, 0, s>>>(idx, probes, tab, sink);
        cudaEventRecord(b, s);
        e = cudaEventSynchronize(b);
        if (e == cudaSuccess) e = cudaGetLastError();
        float ms = 0;
        if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, a, b);
        if (e == cudaSuccess) *g_per_s = (double)probes / (ms * 1e-3) / 1e9;
    }
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    cudaFree(idx);
    cudaFree(tab);
    cudaFree(sink);
    return e;
}

cudaError_t bench_occupancy(int variant, int block, int *blocks_per_sm)
{
    switch (variant) {
    case TQ_VARIANT_RF_AN:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_RF_AN>, block, 0);
    case TQ_VARIANT_PER_THREAD_AFA:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_PER_THREAD_AFA>, block, 0);
    case TQ_VARIANT_CAS_RETRY:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_CAS_RETRY>, block, 0);
    case TQ_VARIANT_AN:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_AN>, block, 0);
    case TQ_VARIANT_ATOMIC_CEILING:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_ATOMIC_CEILING>, block, 0);
    case TQ_VARIANT_RF_AN_CTA:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, bench_kernel<TQ_VARIANT_RF_AN_CTA>, block, 0);
    default: return cudaErrorInvalidValue;
    }
}

}  // namespace tqk
