// bfs.cu -- persistent-thread top-down BFS driven by the retry-free,
// arbitrary-n queue (Troendle, Ta & Jang, ICPP 2019; PAPER.md cited P:<line>),
// hand-written for sm_100a.
//
// One persistent grid (SMs x occupancy, P:63/P:83/P:346) runs Algorithm 1
// (P:85-102):
//
//   while WorkRemains():                 status word, a8 / DESIGN.md R6
//     if GetWorkToken():                 Listing 1 (dequeue) + Listing 2 (poll)
//       DoWorkUnit()                     expansion of <= `chunk` edges / token
//       ScheduleNewlyDiscovered...()     Listing 3 (enqueue)
//
// B200 re-design:
//   * tokens are taken per lane (each lane owns one ticket), but the
//     expansion of all arrived tokens is warp-cooperative: a warp-wide prefix
//     sum over the lanes' edge counts maps 32 consecutive CSR entries to the
//     32 lanes, so `col` reads are coalesced whatever the degree mix;
//   * vertices with more than `chunk` edges are split into chunk tokens put
//     back in the same queue (P:153 sub-task refactoring), so hubs spread
//     over many warps;
//   * levels stay exact without level barriers by label correcting on the
//     packed W = (level << 32 | parent) with 64-bit atomicMin; the minimum
//     also yields the smallest-id parent (R4, R5);
//   * discovered tokens are staged in shared memory per warp and published
//     with one AFA on Rear per flush (arbitrary-n) and coalesced 8-byte
//     slot stores.
#include <cub/device/device_scan.cuh>

#include "internal.cuh"

namespace tqk {

constexpr int kBlock = 256;          // threads per block (8 warps)
constexpr int kWarps = kBlock / 32;
constexpr int kStageCap = 512;       // staged tokens per warp (2 KiB smem)
constexpr int kU = 4;                // 32-edge rounds in flight per lane
// bound on CAS retries of one operation; reaching it can only mean a broken
// queue state (the loops are lock-free), which is reported as a timeout
constexpr unsigned kMaxEnqRetries = 1u << 24;
// a dequeue that keeps losing simply reports "empty" and retries next cycle
constexpr unsigned kMaxDeqRetries = 1u << 12;

__device__ __forceinline__ unsigned long long ld_cg_u64(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int32_t ld_nc_i32(const int32_t *p)
{
    int32_t v;
    asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int64_t ld_nc_i64(const int64_t *p)
{
    int64_t v;
    asm("ld.global.nc.s64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

// number of lanes whose inclusive prefix `incl` is <= g (owner lane of g)
__device__ __forceinline__ int owner_of(int incl, int g)
{
    int o = 0;
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
        const int c = __shfl_sync(TQ_FULL_MASK, incl, o + s - 1);
        if (c <= g) o += s;
    }
    return o;
}

__device__ __forceinline__ int warp_incl_scan(int x, unsigned lane)
{
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(TQ_FULL_MASK, x, o);
        if (lane >= (unsigned)o) x += t;
    }
    return x;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T x)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(TQ_FULL_MASK, x, o);
    return x;
}

// ---------------------------------------------------------------------------
// CAS-based comparison queues (BASE and AN)
// ---------------------------------------------------------------------------

// BASE dequeue of one item by one lane: a classic bounded CAS queue (per-slot
// sequence numbers); retries on CAS failure, returns false on empty.
__device__ __forceinline__ bool cas_dequeue_one(const tq_device_view &q, uint32_t *item,
                                                unsigned *atom, unsigned *fail)
{
    for (unsigned tries = 0; tries < kMaxDeqRetries; ++tries) {
        const unsigned long long pos = tq_ld_relaxed(q.front);
        unsigned long long *s = q.slots + (pos & q.mask);
        const unsigned long long v = tq_ld_relaxed(s);
        const int dif = (int)((unsigned)v - (unsigned)(pos + 1));
        if (dif == 0) {
            ++*atom;
            if (tq_atom_cas(q.front, pos, pos + 1) == pos) {
                *item = (uint32_t)(v >> 32);
                tq_st_relaxed(s, (unsigned long long)(unsigned)(pos + q.mask + 1));
                return true;
            }
            ++*fail;
        } else if (dif < 0) {
            return false;  // queue empty: the exception BASE retries on
        }
    }
    return false;
}

// BASE enqueue of one item by one lane; queue-full aborts (no retry).
__device__ __forceinline__ bool cas_enqueue_one(const tq_device_view &q, uint32_t item,
                                                unsigned *atom, unsigned *fail)
{
    for (unsigned tries = 0; tries < kMaxEnqRetries; ++tries) {
        const unsigned long long pos = tq_ld_relaxed(q.rear);
        unsigned long long *s = q.slots + (pos & q.mask);
        const unsigned long long v = tq_ld_relaxed(s);
        const int dif = (int)((unsigned)v - (unsigned)pos);
        if (dif == 0) {
            ++*atom;
            if (tq_atom_cas(q.rear, pos, pos + 1) == pos) {
                tq_st_relaxed(s, ((unsigned long long)item << 32) | (unsigned)(pos + 1));
                return true;
            }
            ++*fail;
        } else if (dif < 0) {
            tq_status_set_thread(q, TQ_ABORTED_FULL);
            return false;
        }
    }
    tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
    return false;
}

// AN dequeue: the proxy reserves up to n ready slots with one CAS (retrying on
// failure); lanes check the n candidate slots in parallel.  Returns the
// item count k taken for the warp; hungry lane of rank r < k gets ticket base+r.
__device__ __forceinline__ unsigned an_dequeue(const tq_device_view &q, unsigned n,
                                               unsigned long long *base_out, unsigned *atom,
                                               unsigned *fail)
{
    const unsigned lane = tq_lane();
    unsigned tries = 0;
    for (;;) {
        unsigned long long pos = 0;
        if (lane == 0) pos = tq_ld_relaxed(q.front);
        pos = tq_shfl64(pos, 0);
        bool ready = false;
        int dif = 0;
        if (lane < n) {
            const unsigned long long v = tq_ld_relaxed(q.slots + ((pos + lane) & q.mask));
            dif = (int)((unsigned)v - (unsigned)(pos + lane + 1));
            ready = dif == 0;
        }
        const unsigned rm = __ballot_sync(TQ_FULL_MASK, ready);
        const unsigned k = rm == TQ_FULL_MASK ? 32u : (unsigned)(__ffs(~rm) - 1);  // leading ready slots
        const unsigned stale = __ballot_sync(TQ_FULL_MASK, lane < n && dif > 0);
        if (k == 0) {
            if ((stale & 1u) && ++tries < kMaxDeqRetries) continue;  // Front moved on: retry
            return 0;                                             // empty
        }
        unsigned long long old = 0;
        if (lane == 0) {
            ++*atom;
            old = tq_atom_cas(q.front, pos, pos + k);
            if (old != pos) ++*fail;
        }
        old = tq_shfl64(old, 0);
        if (old == pos) {
            *base_out = pos;
            return k;
        }
        if (++tries >= kMaxDeqRetries) return 0;
    }
}

// AN enqueue: the proxy reserves n slots with one CAS after the warp checked
// they are all empty; retries on CAS failure; aborts on queue-full.
__device__ __forceinline__ bool an_reserve_rear(const tq_device_view &q, unsigned n,
                                                unsigned long long *base_out, unsigned *atom,
                                                unsigned *fail)
{
    const unsigned lane = tq_lane();
    for (unsigned tries = 0;; ++tries) {
        if (tries >= kMaxEnqRetries) {
            if (lane == 0) tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
            return false;
        }
        unsigned long long pos = 0;
        if (lane == 0) pos = tq_ld_relaxed(q.rear);
        pos = tq_shfl64(pos, 0);
        bool full = false, stale = false;
        for (unsigned i = lane; i < n; i += 32) {
            const unsigned long long v = tq_ld_relaxed(q.slots + ((pos + i) & q.mask));
            const int dif = (int)((unsigned)v - (unsigned)(pos + i));
            full |= dif < 0;
            stale |= dif > 0;
        }
        if (__any_sync(TQ_FULL_MASK, stale)) continue;
        if (__any_sync(TQ_FULL_MASK, full)) {
            if (lane == 0) tq_status_set_thread(q, TQ_ABORTED_FULL);
            return false;
        }
        unsigned long long old = 0;
        if (lane == 0) {
            ++*atom;
            old = tq_atom_cas(q.rear, pos, pos + n);
            if (old != pos) ++*fail;
        }
        old = tq_shfl64(old, 0);
        if (old == pos) {
            *base_out = pos;
            return true;
        }
    }
}

// ---------------------------------------------------------------------------
// Enqueue of a warp's staged tokens (Listing 3).  `items` in shared memory,
// `cnt` warp-uniform.  Coalesced: lane i writes tickets base+i, base+i+32, ...
// ---------------------------------------------------------------------------
template <int VARIANT>
__device__ __forceinline__ void enqueue_staged(const tq_device_view &q, const uint32_t *items,
                                               unsigned cnt, unsigned lane, unsigned *qatom,
                                               unsigned *casfail)
{
    if (cnt == 0) return;
    if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_AN) {
        unsigned long long base;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            base = tq_warp_reserve_rear(q, cnt, qatom);
        } else {
            if (!an_reserve_rear(q, cnt, &base, qatom, casfail)) return;
        }
        tq_fence_gpu();  // release: W updates before the tokens that name them
        for (unsigned i0 = 0; i0 < cnt; i0 += 32 * 4) {
            unsigned long long sv[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const unsigned i = i0 + 32 * k + lane;
                sv[k] = i < cnt ? tq_ld_relaxed(q.slots + ((base + i) & q.mask)) : 0ull;
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const unsigned i = i0 + 32 * k + lane;
                if (i < cnt) {
                    const unsigned long long t = base + i;
                    if ((unsigned)sv[k] != (unsigned)t) {  // P:268 line 25
                        tq_status_set_thread(q, TQ_ABORTED_FULL);
                    } else {
                        tq_st_relaxed(q.slots + (t & q.mask),
                                      ((unsigned long long)items[i] << 32) | (unsigned)(t + 1));
                    }
                }
            }
        }
    } else if constexpr (VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
        // every lane reserves its own share with its own atomic
        const unsigned mine = lane < cnt ? (cnt - lane + 31) / 32 : 0;
        unsigned long long base = 0;
        if (mine) {
            base = tq_atom_add(q.rear, mine);
            ++*qatom;
        }
        tq_fence_gpu();
        for (unsigned k = 0; k < mine; ++k) tq_publish(q, base + k, items[lane + 32 * k]);
    } else {  // CAS_RETRY: one CAS-reserved slot per item, per lane
        tq_fence_gpu();
        for (unsigned i = lane; i < cnt; i += 32)
            if (!cas_enqueue_one(q, items[i], qatom, casfail)) break;
    }
}

// chunk tokens of one hub: CHUNK_FLAG | (first + k), k < n (warp-uniform args)
template <int VARIANT>
__device__ __forceinline__ void enqueue_chunks(const tq_device_view &q, uint32_t first, unsigned n,
                                               unsigned lane, unsigned *qatom, unsigned *casfail)
{
    if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
        for (unsigned i = lane; i < n; i += 32)
            if (!cas_enqueue_one(q, CHUNK_FLAG | (first + i), qatom, casfail)) break;
        return;
    } else {
        unsigned long long base;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            base = tq_warp_reserve_rear(q, n, qatom);
        } else if constexpr (VARIANT == TQ_VARIANT_AN) {
            if (!an_reserve_rear(q, n, &base, qatom, casfail)) return;
        } else {  // PER_THREAD_AFA: each lane reserves its own share
            const unsigned mine = lane < n ? (n - lane + 31) / 32 : 0;
            base = 0;
            if (mine) {
                base = tq_atom_add(q.rear, mine);
                ++*qatom;
            }
            for (unsigned k = 0; k < mine; ++k)
                tq_publish(q, base + k, CHUNK_FLAG | (first + lane + 32 * k));
            return;
        }
        for (unsigned i = lane; i < n; i += 32) tq_publish(q, base + i, CHUNK_FLAG | (first + i));
    }
}

// ---------------------------------------------------------------------------
// The persistent kernel
// ---------------------------------------------------------------------------
template <int VARIANT>
__global__ void __launch_bounds__(kBlock) bfs_persistent_kernel(const BfsParams p)
{
    __shared__ uint32_t stage_all[kWarps][kStageCap];
    const unsigned lane = threadIdx.x & 31;
    const unsigned warp_gid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint32_t *stage = stage_all[threadIdx.x >> 5];
    const tq_device_view q = p.q;
    const unsigned long long cap = q.mask + 1;
    const int chunk = p.chunk;

    unsigned long long ticket = TQ_NO_TICKET;  // the lane's DequeueThreadSlotIndex
    unsigned st_tasks = 0, st_chunks = 0, st_min = 0, st_reenq = 0, st_qatom = 0, st_fail = 0,
             st_empty = 0;
    unsigned long long st_edges = 0;
    unsigned backoff = 0, idle = 0;
    const unsigned long long deadline = tq_globaltimer() + p.timeout_ns;

    for (;;) {
        // ---- Algorithm 1 line 1: WorkRemains() ----
        if (tq_status_read(q, warp_gid) != TQ_RUNNING) break;

        // ---- Listing 1 + Listing 2: GetWorkToken() ----
        bool got = false;
        uint32_t item = 0;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            const bool hungry = ticket == TQ_NO_TICKET;
            const unsigned long long t = tq_warp_dequeue_n(q, hungry, &st_qatom);
            if (hungry) ticket = t;
            got = tq_take(q, ticket, &item);
            if (got) ticket = TQ_NO_TICKET;
        } else if constexpr (VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
            if (ticket == TQ_NO_TICKET) {
                ticket = tq_atom_add(q.front, 1ull);
                ++st_qatom;
            }
            got = tq_take(q, ticket, &item);
            if (got) ticket = TQ_NO_TICKET;
        } else if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
            got = cas_dequeue_one(q, &item, &st_qatom, &st_fail);
        } else {  // AN: every lane is hungry each cycle (no held tickets)
            unsigned long long base = 0;
            const unsigned k = an_dequeue(q, 32, &base, &st_qatom, &st_fail);
            if (lane < k) {
                unsigned long long *s = q.slots + ((base + lane) & q.mask);
                const unsigned long long v = tq_ld_relaxed(s);
                item = (uint32_t)(v >> 32);
                tq_st_relaxed(s, (unsigned long long)(unsigned)(base + lane + cap));
                got = true;
            }
        }
        const unsigned gm = __ballot_sync(TQ_FULL_MASK, got);
        if (gm == 0) {
            if (lane == 0) ++st_empty;
            if (p.backoff_ns > 0) {
                backoff = backoff ? min(backoff * 2, (unsigned)p.backoff_ns) : 32u;
                __nanosleep(backoff);
            }
            if ((++idle & 63) == 0 && tq_globaltimer() > deadline) {
                if (lane == 0) tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
            }
            continue;
        }
        backoff = 0;
        tq_fence_gpu();  // acquire: the producer's W update is visible now

        // ---- enumeration prolog (Listing 2 lines 6-22) ----
        int32_t v = 0;
        long long lo = 0, hi = 0;
        unsigned nch = 0;
        uint32_t chb = 0;
        unsigned long long offer = 0;
        if (got) {
            ++st_tasks;
            if (item & CHUNK_FLAG) {
                ++st_chunks;
                const int2 c = p.chunk_tab[item & ~CHUNK_FLAG];
                v = c.x;
                const long long re = ld_nc_i64(p.row_ptr + v + 1);
                lo = ld_nc_i64(p.row_ptr + v) + (long long)c.y * chunk;
                hi = min(lo + (long long)chunk, re);
            } else {
                v = (int32_t)item;
                lo = ld_nc_i64(p.row_ptr + v);
                hi = ld_nc_i64(p.row_ptr + v + 1);
                if (hi - lo > chunk) {  // hub: schedule its sub-tasks instead
                    nch = (unsigned)((hi - lo + chunk - 1) / chunk);
                    chb = (uint32_t)p.hub_base[v];
                    hi = lo;
                }
            }
            // current cost of the node (Listing 2 line 21), read fresh
            const unsigned L = (unsigned)(tq_ld_relaxed(p.W + v) >> 32);
            offer = ((unsigned long long)(L + 1) << 32) | (unsigned)v;
        }

        // ---- DoWorkUnit(): warp-cooperative expansion ----
        const int deg = (int)(hi - lo);
        const int incl = warp_incl_scan(deg, lane);
        const int total = __shfl_sync(TQ_FULL_MASK, incl, 31);
        const long long ebase = lo - (incl - deg);
        unsigned cnt = 0;
        for (int b = 0; b < total; b += 32 * kU) {
            int32_t u[kU];
            unsigned long long off[kU];
            bool val[kU];
#pragma unroll
            for (int j = 0; j < kU; ++j) {
                const int g = b + j * 32 + (int)lane;
                val[j] = g < total;
                const int gg = val[j] ? g : total - 1;
                const int o = owner_of(incl, gg);
                const long long eb = (long long)tq_shfl64((unsigned long long)ebase, o);
                off[j] = tq_shfl64(offer, o);
                u[j] = val[j] ? ld_nc_i32(p.col + eb + gg) : 0;
            }
            unsigned long long w[kU];
#pragma unroll
            for (int j = 0; j < kU; ++j) w[j] = val[j] ? ld_cg_u64(p.W + u[j]) : 0ull;
            bool nt[kU];
#pragma unroll
            for (int j = 0; j < kU; ++j) {
                nt[j] = false;
                if (val[j]) {
                    ++st_edges;
                    if (off[j] < w[j]) {  // stale-tolerant prefilter (R4)
                        const unsigned long long old = atomicMin(p.W + u[j], off[j]);
                        ++st_min;
                        if ((old >> 32) > (off[j] >> 32)) {  // level strictly lowered
                            nt[j] = true;
                            if ((old >> 32) != 0xffffffffull) ++st_reenq;
                        }
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < kU; ++j) {
                const unsigned m = __ballot_sync(TQ_FULL_MASK, nt[j]);
                if (nt[j]) stage[cnt + __popc(m & tq_lanemask_lt())] = (uint32_t)u[j];
                cnt += __popc(m);
            }
            if (cnt > kStageCap - 32 * kU) {
                __syncwarp();
                enqueue_staged<VARIANT>(q, stage, cnt, lane, &st_qatom, &st_fail);
                __syncwarp();
                cnt = 0;
            }
        }

        // ---- ScheduleNewlyDiscoveredWorkTokens(): Listing 3 ----
        __syncwarp();
        enqueue_staged<VARIANT>(q, stage, cnt, lane, &st_qatom, &st_fail);
        __syncwarp();
        unsigned hubm = __ballot_sync(TQ_FULL_MASK, nch > 0);
        while (hubm) {
            const int h = __ffs(hubm) - 1;
            hubm &= hubm - 1;
            const unsigned n = __shfl_sync(TQ_FULL_MASK, nch, h);
            const uint32_t first = __shfl_sync(TQ_FULL_MASK, chb, h);
            enqueue_chunks<VARIANT>(q, first, n, lane, &st_qatom, &st_fail);
        }

        // ---- completion accounting for WorkRemains() (R6) ----
        bool fin = false;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_AN) {
            // lane 0 issued every Rear reservation of this warp, so its
            // acq_rel add on Done is ordered after them
            if (lane == 0) {
                const unsigned nf = __popc(gm);
                const unsigned long long old = tq_atom_add_acqrel(q.done, nf);
                ++st_qatom;
                fin = old + nf == tq_ld_relaxed(q.rear);
            }
        } else {
            __syncwarp();
            tq_fence_gpu();
            if (got) {
                const unsigned long long old = tq_atom_add_acqrel(q.done, 1ull);
                ++st_qatom;
                fin = old + 1 == tq_ld_relaxed(q.rear);
            }
        }
        if (__any_sync(TQ_FULL_MASK, fin)) tq_warp_status_set(q, TQ_FINISHED);
    }

    // ---- statistics (one atomic per counter per warp) ----
    const unsigned long long s[8] = {st_tasks, st_chunks, st_edges, st_min,
                                     st_reenq, st_qatom,  st_fail,  st_empty};
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const unsigned long long x = warp_sum(s[k]);
        if (lane == 0 && x) atomicAdd(p.stats + k, x);
    }
}

// ---------------------------------------------------------------------------
// a2: state + queue init for one run.  W[:] = unreached, W[root] = (0, root);
// the root is published at ticket t0 (Front = Done = t0, Rear = t0 + 1).
// ---------------------------------------------------------------------------
__global__ void bfs_init_kernel(const BfsParams p, int32_t root, unsigned long long t0)
{
    const int64_t n = p.n_vertices;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
        p.W[i] = (i == root) ? (unsigned long long)(uint32_t)root : ~0ull;
    if (blockIdx.x == 0) {
        if (threadIdx.x < TQ_STATUS_COPIES) p.q.status[threadIdx.x * TQ_STATUS_STRIDE] = TQ_RUNNING;
        if (threadIdx.x < kStatCount) p.stats[threadIdx.x] = 0;
        if (threadIdx.x == 0) {
            p.q.slots[t0 & p.q.mask] =
                ((unsigned long long)(uint32_t)root << 32) | (unsigned)(t0 + 1);
            *p.q.front = t0;
            *p.q.rear = t0 + 1;
            *p.q.done = t0;
        }
    }
}

// ---------------------------------------------------------------------------
// a9: unpack W -> level, parent (-1 unreached) and the TEPS statistics.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) bfs_unpack_kernel(const BfsParams p, int32_t *level,
                                                          int32_t *parent)
{
    const int64_t n = p.n_vertices;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    unsigned long long reached = 0, degsum = 0;
    unsigned maxl = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const unsigned long long w = p.W[i];
        const unsigned l = (unsigned)(w >> 32);
        const bool r = l != 0xffffffffu;
        if (level) level[i] = r ? (int32_t)l : -1;
        if (parent) parent[i] = r ? (int32_t)(uint32_t)w : -1;
        if (r) {
            ++reached;
            degsum += (unsigned long long)(ld_nc_i64(p.row_ptr + i + 1) - ld_nc_i64(p.row_ptr + i));
            maxl = max(maxl, l);
        }
    }
    reached = warp_sum(reached);
    degsum = warp_sum(degsum);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) maxl = max(maxl, __shfl_xor_sync(TQ_FULL_MASK, maxl, o));
    __shared__ unsigned long long sh_r[8], sh_d[8];
    __shared__ unsigned sh_m[8];
    const int w = threadIdx.x >> 5;
    if ((threadIdx.x & 31) == 0) {
        sh_r[w] = reached;
        sh_d[w] = degsum;
        sh_m[w] = maxl;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int k = 1; k < (int)(blockDim.x >> 5); ++k) {
            reached += sh_r[k];
            degsum += sh_d[k];
            maxl = max(maxl, sh_m[k]);
        }
        if (reached) {
            atomicAdd(p.stats + ST_REACHED, reached);
            atomicAdd(p.stats + ST_DEG_SUM, degsum);
            atomicMax(p.stats + ST_MAX_LEVEL, (unsigned long long)maxl);
        }
    }
}

// ---------------------------------------------------------------------------
// Plan build: chunk table for vertices with more than `chunk` edges.
// ---------------------------------------------------------------------------
__global__ void count_chunks_kernel(const int64_t *row_ptr, int64_t n, int chunk, int32_t *nch)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const int64_t d = row_ptr[v + 1] - row_ptr[v];
        nch[v] = d > chunk ? (int32_t)((d + chunk - 1) / chunk) : 0;
    }
}

__global__ void fill_chunks_kernel(const int64_t *row_ptr, int64_t n, int chunk,
                                   const int32_t *hub_base, int2 *tab)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const int64_t d = row_ptr[v + 1] - row_ptr[v];
        if (d > chunk) {
            const int32_t k_n = (int32_t)((d + chunk - 1) / chunk);
            const int32_t b = hub_base[v];
            for (int32_t k = 0; k < k_n; ++k) tab[b + k] = make_int2((int)v, k);
        }
    }
}

__global__ void queue_reset_kernel(tq_device_view q)
{
    const unsigned long long cap = q.mask + 1;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < cap;
         i += stride)
        q.slots[i] = (unsigned)i;  // empty for ticket i (lap 0)
    if (blockIdx.x == 0) {
        if (threadIdx.x < TQ_STATUS_COPIES) q.status[threadIdx.x * TQ_STATUS_STRIDE] = TQ_RUNNING;
        if (threadIdx.x == 0) {
            *q.front = 0;
            *q.rear = 0;
            *q.done = 0;
        }
    }
}

// ---------------------------------------------------------------------------
// Launchers
// ---------------------------------------------------------------------------
static int grid_for(int64_t n, int block)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t want = (n + block - 1) / block;
    const int64_t cap = (int64_t)sms * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

cudaError_t launch_bfs_init(const BfsParams &p, int32_t root, unsigned long long t0, cudaStream_t s)
{
    bfs_init_kernel<<<grid_for(p.n_vertices, 256), 256, 0, s>>>(p, root, t0);
    return cudaGetLastError();
}

cudaError_t launch_bfs_unpack(const BfsParams &p, int32_t *level, int32_t *parent, cudaStream_t s)
{
    bfs_unpack_kernel<<<grid_for(p.n_vertices, 256), 256, 0, s>>>(p, level, parent);
    return cudaGetLastError();
}

cudaError_t launch_queue_reset(const tq_device_view &q, cudaStream_t s)
{
    queue_reset_kernel<<<grid_for((int64_t)(q.mask + 1), 256), 256, 0, s>>>(q);
    return cudaGetLastError();
}

template <int V>
static cudaError_t launch_v(const BfsParams &p, int blocks, int block, cudaStream_t s)
{
    if (block != kBlock) return cudaErrorInvalidValue;
    bfs_persistent_kernel<V><<<blocks, kBlock, 0, s>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_bfs_persistent(int variant, const BfsParams &p, int blocks, int block,
                                  cudaStream_t s)
{
    switch (variant) {
    case TQ_VARIANT_RF_AN: return launch_v<TQ_VARIANT_RF_AN>(p, blocks, block, s);
    case TQ_VARIANT_PER_THREAD_AFA: return launch_v<TQ_VARIANT_PER_THREAD_AFA>(p, blocks, block, s);
    case TQ_VARIANT_CAS_RETRY: return launch_v<TQ_VARIANT_CAS_RETRY>(p, blocks, block, s);
    case TQ_VARIANT_AN: return launch_v<TQ_VARIANT_AN>(p, blocks, block, s);
    default: return cudaErrorInvalidValue;
    }
}

cudaError_t bfs_occupancy(int variant, int block, int *blocks_per_sm)
{
    if (block != kBlock) return cudaErrorInvalidValue;
    switch (variant) {
    case TQ_VARIANT_RF_AN:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            blocks_per_sm, bfs_persistent_kernel<TQ_VARIANT_RF_AN>, kBlock, 0);
    case TQ_VARIANT_PER_THREAD_AFA:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            blocks_per_sm, bfs_persistent_kernel<TQ_VARIANT_PER_THREAD_AFA>, kBlock, 0);
    case TQ_VARIANT_CAS_RETRY:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            blocks_per_sm, bfs_persistent_kernel<TQ_VARIANT_CAS_RETRY>, kBlock, 0);
    case TQ_VARIANT_AN:
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
            blocks_per_sm, bfs_persistent_kernel<TQ_VARIANT_AN>, kBlock, 0);
    default: return cudaErrorInvalidValue;
    }
}

cudaError_t build_chunk_table(const int64_t *row_ptr, int64_t n, int chunk, int32_t *hub_base,
                              int2 **chunk_tab_out, int64_t *n_chunks_out, cudaStream_t s)
{
    *chunk_tab_out = nullptr;
    *n_chunks_out = 0;
    int32_t *nch = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    cudaError_t e = cudaMalloc(&nch, (size_t)n * sizeof(int32_t));
    if (e != cudaSuccess) return e;
    count_chunks_kernel<<<grid_for(n, 256), 256, 0, s>>>(row_ptr, n, chunk, nch);
    e = cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, nch, hub_base, (int)n, s);
    if (e == cudaSuccess) e = cudaMalloc(&tmp, tmp_bytes);
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, nch, hub_base, (int)n, s);
    int32_t last_base = 0, last_n = 0;
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(&last_base, hub_base + n - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(&last_n, nch + n - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    const int64_t total = (int64_t)last_base + last_n;
    if (e == cudaSuccess && total > 0) {
        int2 *tab = nullptr;
        e = cudaMalloc(&tab, (size_t)total * sizeof(int2));
        if (e == cudaSuccess) {
            fill_chunks_kernel<<<grid_for(n, 256), 256, 0, s>>>(row_ptr, n, chunk, hub_base, tab);
            e = cudaGetLastError();
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e == cudaSuccess) {
                *chunk_tab_out = tab;
                *n_chunks_out = total;
            } else {
                cudaFree(tab);
            }
        }
    }
    cudaFree(tmp);
    cudaFree(nch);
    return e;
}

}  // namespace tqk
