// bfs_small.cu -- the persistent-thread BFS of bfs.cu for graphs that fit in
// one SM's shared memory (BASELINE.json configs[0], R-MAT scale 10):
// Algorithm 1 with the retry-free / arbitrary-n queue (P:155,
// Listings 1-3) held in shared memory, run by ONE 1024-thread
// block that also loads the graph and unpacks the result, so a run is a
// single launch.
//
// Why: a 1K-vertex BFS is a chain of ~6 level hops
// with ~3K edges each.  In global memory every hop is a release fence, an L2
// atomic, a slot store and an L2 poll (~4 us); here the whole state -- CSR,
// packed W, expanded-level markers, the ring of slots and its Front / Rear /
// Done tickets -- sits in shared memory, so a hop is a few hundred cycles and
// the run is bounded by the launch and the first read of the graph.
//
// The queue protocol is the one of include/tq_device.cuh, moved to the CTA
// scope: a 32-bit ticket t owns slot t mod C, whose 64-bit word holds
// {item:32 | seq:32}; seq == t means "empty for t", seq == t + 1 "item for t
// has arrived" (P:163 data-not-arrived flag); one proxy atomicAdd on Front /
// Rear per warp operation reserves any number of tickets (P:167-171,
// P:258); a reservation past the first lap checks its slot and aborts on a
// queue-full exception (Listing 3 line 25).  Tickets restart at
// 0 every launch (the ring is initialised by the kernel).
#include <atomic>

#include "internal.cuh"

namespace tqk {

namespace {

constexpr int kSB = 1024;          // threads of the single block
constexpr int kSW = kSB / 32;      // warps
constexpr int kSU = 4;             // 32-entry slices per expansion round
constexpr unsigned kSat = 254;     // expanded-level marker: 255 = never
constexpr int kSChunk = 128;       // hub sub-task size (one expansion round)
constexpr unsigned kChunk = 0x80000000u;

__device__ __forceinline__ unsigned long long lds_u64_volatile(const unsigned long long *p)
{
    return *reinterpret_cast<const volatile unsigned long long *>(p);
}
__device__ __forceinline__ void sts_u64_volatile(unsigned long long *p, unsigned long long v)
{
    *reinterpret_cast<volatile unsigned long long *>(p) = v;
}
__device__ __forceinline__ unsigned lds_u32_volatile(const unsigned *p)
{
    return *reinterpret_cast<const volatile unsigned *>(p);
}
__device__ __forceinline__ unsigned mix32_s(unsigned x)
{
    x ^= x >> 16;
    x *= 0x7feb352du;
    x ^= x >> 15;
    x *= 0x846ca68bu;
    x ^= x >> 16;
    return x;
}

// CTA-scope acquire-release fence (fence.acq_rel.cta; __threadfence_block
// is the sequentially consistent fence.sc.cta)
__device__ __forceinline__ void fence_cta() { asm volatile("fence.acq_rel.cta;" ::: "memory"); }

// Listing 3 lines 23-27 for ticket t: past the first lap the slot must hold
// "empty for t", else the queue is full: abort, no retry
__device__ __forceinline__ void publish(unsigned long long *slots, unsigned mask, unsigned cap, unsigned t,
                                        unsigned item, unsigned *status)
{
    unsigned long long *s = slots + (t & mask);
    if (t >= cap && (unsigned)lds_u64_volatile(s) != t)
        atomicCAS(status, TQ_RUNNING, TQ_ABORTED_FULL);
    else
        sts_u64_volatile(s, ((unsigned long long)item << 32) | (t + 1u));
}

struct SmallCtl {
    unsigned front, rear, done, status;
};

}  // namespace

size_t small_smem_bytes(int64_t n, int64_t nnz, uint64_t cap)
{
    const size_t rp = ((size_t)(n + 1) * 4 + 15) / 16 * 16;
    const size_t col = ((size_t)nnz * 4 + 15) / 16 * 16;
    const size_t w = ((size_t)n * 4 + 15) / 16 * 16;
    const size_t x8 = ((size_t)n + 15) / 16 * 16;
    return rp + col + w + x8 + (size_t)cap * 8;
}

__global__ void __launch_bounds__(kSB, 1)
    bfs_small_kernel(const BfsParams p, int32_t root, int32_t *level_out, int32_t *parent_out)
{
    extern __shared__ __align__(16) unsigned char sm[];
    const int n = (int)p.n_vertices;
    const int nnz = (int)p.nnz;
    const unsigned cap = p.small_cap;  // power of two
    const unsigned mask = cap - 1;
    unsigned *rp = reinterpret_cast<unsigned *>(sm);
    int32_t *col = reinterpret_cast<int32_t *>(sm + ((size_t)(n + 1) * 4 + 15) / 16 * 16);
    // W: packed (level << 16) | parent, 0xFFFFFFFF = unreached (n <= 2^16:
    // levels < n and ids fit 16 bits), so atomicMin is one native 32-bit
    // shared-memory atomic; the minimum is the min-id parent (R5)
    unsigned *W = reinterpret_cast<unsigned *>(reinterpret_cast<unsigned char *>(col) + ((size_t)nnz * 4 + 15) / 16 * 16);
    uint8_t *x8 = reinterpret_cast<uint8_t *>(W) + ((size_t)n * 4 + 15) / 16 * 16;
    unsigned long long *slots = reinterpret_cast<unsigned long long *>(x8 + ((size_t)n + 15) / 16 * 16);
    __shared__ SmallCtl ctl;
    __shared__ unsigned long long wst[kSW][kStatCount];
    __shared__ unsigned long long red_r[kSW], red_d[kSW];
    __shared__ unsigned red_m[kSW];
    __shared__ uint2 trec_all[kSW][32];

    const unsigned tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;

    // ---- load the graph, initialise W / markers / the ring (a2) ----
    // row_ptr as 32-bit offsets (nnz < 2^32 whenever the graph fits)
    for (int i = tid; i <= n; i += kSB) rp[i] = (unsigned)p.row_ptr[i];
    {
        const int n4 = ((uintptr_t)p.col & 15) == 0 ? nnz / 4 : 0;
        const int4 *c4 = reinterpret_cast<const int4 *>(p.col);
        for (int i = tid; i < n4; i += kSB) reinterpret_cast<int4 *>(col)[i] = __ldg(c4 + i);
        for (int i = 4 * n4 + tid; i < nnz; i += kSB) col[i] = __ldg(p.col + i);
    }
    for (int i = tid; i < n; i += kSB) {
        W[i] = i == root ? (unsigned)root : ~0u;
        x8[i] = 0xFF;
    }
    for (unsigned i = tid; i < cap; i += kSB) slots[i] = (unsigned long long)i;  // empty for ticket i
    if (tid < kStatCount * kSW) (&wst[0][0])[tid] = 0;
    if (tid == 0) {
        slots[0] = ((unsigned long long)(uint32_t)root << 32) | 1u;  // root at ticket 0
        ctl.front = 0;
        ctl.rear = 1;
        ctl.done = 0;
        ctl.status = TQ_RUNNING;
    }
    __syncthreads();

    unsigned long long *S = wst[wid];
    uint2 *trec = trec_all[wid];
    const bool min_id = p.parent_rule == TQ_PARENT_MIN_ID;
    const unsigned long long deadline = tq_globaltimer() + p.timeout_ns;
    const unsigned tl = p.ticket_lanes;  // lanes holding a ticket
    unsigned tk = 0;
    bool have = false;
    unsigned idle = 0, busy = 0, backoff = 0;

    for (;;) {
        // ---- Listing 1: the proxy reserves tickets for the hungry lanes ----
        const unsigned hungry = __ballot_sync(TQ_FULL_MASK, !have) & tl;
        if (hungry) {
            unsigned base = 0;
            if (lane == 0) base = atomicAdd(&ctl.front, (unsigned)__popc(hungry));
            base = __shfl_sync(TQ_FULL_MASK, base, 0);
            if ((hungry >> lane) & 1u) {
                tk = base + __popc(hungry & tq_lanemask_lt());
                have = true;
            }
            if (lane == 0) ++S[ST_QUEUE_ATOMICS];
        }
        // ---- Listing 2: arrival check of the held ticket ----
        const unsigned long long sv = have ? lds_u64_volatile(slots + (tk & mask)) : 0ull;
        const bool got = have && (unsigned)sv == tk + 1u;
        const unsigned gm = __ballot_sync(TQ_FULL_MASK, got);
        if (gm == 0) {
            // ---- idle: WorkRemains() ----
            if (lane == 0) ++S[ST_EMPTY_POLLS];
            if (lds_u32_volatile(&ctl.status) != TQ_RUNNING) break;
            if (p.backoff_ns > 0) {  // idle back-off, short: a hop here is ~100s of ns
                backoff = backoff ? min(2 * backoff, (unsigned)p.backoff_ns) : 32u;
                __nanosleep(backoff);
            }
            if ((++idle & 3) == 0) {
                bool fin = false;
                if (lane == 0) {
                    // Done before Rear (R6)
                    const unsigned d = lds_u32_volatile(&ctl.done);
                    fence_cta();
                    fin = d == lds_u32_volatile(&ctl.rear);
                    if (!fin && tq_globaltimer() > deadline) atomicCAS(&ctl.status, TQ_RUNNING, TQ_ABORTED_TIMEOUT);
                }
                if (__shfl_sync(TQ_FULL_MASK, fin, 0)) {
                    if (lane == 0) atomicCAS(&ctl.status, TQ_RUNNING, TQ_FINISHED);
                    break;
                }
            }
            continue;
        }
        idle = 0;
        backoff = 0;
        // the watchdog is honoured by busy warps too
        if ((++busy & 1023) == 0) {
            if (lds_u32_volatile(&ctl.status) != TQ_RUNNING) break;
            if (lane == 0 && tq_globaltimer() > deadline) atomicCAS(&ctl.status, TQ_RUNNING, TQ_ABORTED_TIMEOUT);
        }
        fence_cta();  // acquire: the producers' W updates before their tokens
        uint32_t item = 0;
        if (got) {
            item = (uint32_t)(sv >> 32);
            sts_u64_volatile(slots + (tk & mask), (unsigned long long)(tk + cap));  // dna for the next lap
            have = false;
        }
        // ---- enumeration prolog: level, expanded-level marker, hub chunks ----
        // item: a vertex v (< 2^16), or kChunk | k << 16 | v: entries
        // [k * kSChunk, (k + 1) * kSChunk) of hub v's row (P:153 sub-tasks)
        int lo = 0, hi = 0;
        unsigned offer = 0, nch = 0;
        bool skipped = false;
        if (got) {
            const unsigned v = item & 0xFFFFu;
            if (p.delay_ns && (mix32_s(v ^ p.delay_seed) & 7u) == 0) __nanosleep(p.delay_ns);
            const unsigned L = W[v] >> 16;
            lo = (int)rp[v];
            hi = (int)rp[v + 1];
            offer = ((L + 1) << 16) | v;
            if (item & kChunk) {
                lo += (int)((item >> 16) & 0x7FFFu) * kSChunk;
                hi = min(hi, lo + kSChunk);
            } else {
                const unsigned xprev = x8[v];
                if (xprev < kSat && xprev <= L) {
                    skipped = true;
                    hi = lo;
                } else {
                    x8[v] = (uint8_t)(L < kSat ? L : kSat);
                    if (hi - lo > kSChunk) {  // hub: its chunks go back to the queue
                        nch = (unsigned)(hi - lo + kSChunk - 1) / kSChunk;
                        hi = lo;
                    }
                }
            }
        }
        // Listing 3 for the chunk tokens of this cycle's hubs (one AFA per hub)
        for (unsigned hubm = __ballot_sync(TQ_FULL_MASK, nch > 0); hubm; hubm &= hubm - 1) {
            const int h = __ffs(hubm) - 1;
            const unsigned nh = __shfl_sync(TQ_FULL_MASK, nch, h);
            const unsigned vh = __shfl_sync(TQ_FULL_MASK, item & 0xFFFFu, h);
            unsigned base = 0;
            if (lane == 0) {
                fence_cta();  // release (the hub's level was read above)
                base = atomicAdd(&ctl.rear, nh);
                ++S[ST_QUEUE_ATOMICS];
            }
            base = __shfl_sync(TQ_FULL_MASK, base, 0);
            for (unsigned k = lane; k < nh; k += 32) publish(slots, mask, cap, base + k, kChunk | (k << 16) | vh, &ctl.status);
        }
        const int deg = hi - lo;
        int incl = deg;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(TQ_FULL_MASK, incl, o);
            if (lane >= (unsigned)o) incl += t;
        }
        const int total = __shfl_sync(TQ_FULL_MASK, incl, 31);
        const int tstart = incl - deg;
        const unsigned skm = __ballot_sync(TQ_FULL_MASK, skipped);
        const unsigned chm = __ballot_sync(TQ_FULL_MASK, got && (item & kChunk));
        // the warp's non-empty tokens in lane order: {first CSR entry minus
        // the token's start in the concatenation, offer}; the token of entry
        // g is the one with the largest start <= g (a running count of token
        // starts per 32-entry slice, as in bfs.cu)
        const unsigned ne = __ballot_sync(TQ_FULL_MASK, deg > 0);
        if (deg > 0) trec[__popc(ne & tq_lanemask_lt())] = make_uint2((unsigned)(lo - tstart), offer);
        __syncwarp();
        if (lane == 0) {
            S[ST_TASKS] += __popc(gm);
            S[ST_CHUNK_TASKS] += __popc(chm);
            S[ST_SKIPPED] += __popc(skm);
            S[ST_EDGES] += (unsigned)total;
            S[ST_BUSY_CYCLES] += 1;
            S[ST_ROUNDS] += (unsigned)((total + 32 * kSU - 1) / (32 * kSU));
        }
        // ---- DoWorkUnit(): warp-cooperative expansion from shared memory ----
        const unsigned lemask = TQ_FULL_MASK >> (31u - lane);
        for (int b = 0; b < total; b += 32 * kSU) {
            int cb = __popc(__ballot_sync(TQ_FULL_MASK, deg > 0 && tstart < b));
            int u[kSU];
            unsigned off[kSU], w[kSU];
            bool val[kSU];
#pragma unroll
            for (int j = 0; j < kSU; ++j) {
                const int sj = b + j * 32;
                const int g = sj + (int)lane;
                val[j] = g < total;
                const unsigned rel = (unsigned)(tstart - sj);
                const unsigned bs = __reduce_or_sync(TQ_FULL_MASK, (deg > 0 && rel < 32u) ? (1u << rel) : 0u);
                const int r = cb + __popc(bs & lemask) - 1;
                cb += __popc(bs);
                const uint2 t = trec[r < 0 ? 0 : r];
                u[j] = val[j] ? col[(int)t.x + g] : 0;
                off[j] = t.y;
            }
#pragma unroll
            for (int j = 0; j < kSU; ++j) w[j] = val[j] ? W[u[j]] : 0u;
            bool nt[kSU];
            unsigned nmin = 0, nre = 0;
#pragma unroll
            for (int j = 0; j < kSU; ++j) {
                // the packed word is exact here: one compare serves both
                // parent rules (min-id also improves on level ties)
                const bool cand = val[j] && (min_id ? off[j] < w[j] : (off[j] >> 16) < (w[j] >> 16));
                const unsigned old = cand ? atomicMin(W + u[j], off[j]) : 0u;
                nt[j] = cand && (old >> 16) > (off[j] >> 16);  // level strictly lowered
                nre += nt[j] && old != 0xffffffffu;            // a re-discovery
                nmin += cand;
            }
            // ---- ScheduleNewlyDiscoveredWorkTokens(): Listing 3, per round ----
            unsigned ntm[kSU], tot = 0;
#pragma unroll
            for (int j = 0; j < kSU; ++j) {
                ntm[j] = __ballot_sync(TQ_FULL_MASK, nt[j]);
                tot += __popc(ntm[j]);
            }
            if (tot) {
                unsigned base = 0;
                if (lane == 0) {
                    fence_cta();  // release: W updates before the tokens naming them
                    base = atomicAdd(&ctl.rear, tot);  // the proxy's AFA
                }
                base = __shfl_sync(TQ_FULL_MASK, base, 0);
                unsigned k = base;
#pragma unroll
                for (int j = 0; j < kSU; ++j) {
                    if (nt[j]) publish(slots, mask, cap, k + __popc(ntm[j] & tq_lanemask_lt()), (unsigned)u[j], &ctl.status);
                    k += __popc(ntm[j]);
                }
            }
            nmin = __reduce_add_sync(TQ_FULL_MASK, nmin);
            nre = __reduce_add_sync(TQ_FULL_MASK, nre);
            if (lane == 0) {
                S[ST_MIN_ATOMICS] += nmin;
                S[ST_REENQUEUES] += nre;
                S[ST_QUEUE_ATOMICS] += tot ? 1 : 0;
            }
        }
        // ---- completion accounting (R6): after this warp's Rear AFAs ----
        __syncwarp();
        if (lane == 0) {
            fence_cta();
            atomicAdd(&ctl.done, (unsigned)__popc(gm));
            ++S[ST_QUEUE_ATOMICS];
        }
    }

    // ---- a9: unpack + statistics ----
    __syncthreads();
    unsigned long long reached = 0, degsum = 0;
    unsigned maxl = 0;
    for (int i = tid; i < n; i += kSB) {
        const unsigned w = W[i];
        const unsigned l = w >> 16;
        const bool r = w != 0xffffffffu;
        if (level_out) level_out[i] = r ? (int32_t)l : -1;
        if (parent_out) parent_out[i] = r ? (int32_t)(w & 0xFFFFu) : -1;
        if (r) {
            ++reached;
            degsum += rp[i + 1] - rp[i];
            maxl = max(maxl, l);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        reached += __shfl_xor_sync(TQ_FULL_MASK, reached, o);
        degsum += __shfl_xor_sync(TQ_FULL_MASK, degsum, o);
        maxl = max(maxl, __shfl_xor_sync(TQ_FULL_MASK, maxl, o));
    }
    if (lane == 0) {
        red_r[wid] = reached;
        red_d[wid] = degsum;
        red_m[wid] = maxl;
    }
    __syncthreads();
    if (tid < kStatCount) {
        unsigned long long s = 0;
        for (int w = 0; w < kSW; ++w) s += wst[w][tid];
        if (tid == ST_SMEM_TICKETS) s = ctl.rear;
        if (tid == ST_REACHED || tid == ST_DEG_SUM || tid == ST_MAX_LEVEL) {
            s = 0;
            for (int w = 0; w < kSW; ++w)
                s = tid == ST_MAX_LEVEL ? max(s, (unsigned long long)red_m[w])
                                        : s + (tid == ST_REACHED ? red_r[w] : red_d[w]);
        }
        p.stats[tid] = s;
    }
    if (tid < TQ_STATUS_COPIES) p.q.status[tid * TQ_STATUS_STRIDE] = ctl.status;
}

cudaError_t launch_bfs_small(const BfsParams &p, int32_t root, int32_t *level, int32_t *parent, cudaStream_t s)
{
    const size_t smem = small_smem_bytes(p.n_vertices, p.nnz, p.small_cap);
    if (smem > 48 * 1024) {
        // opt in to more than 48 KB of dynamic shared memory, once per device
        // and size (a function attribute; the kernel is otherwise launched
        // with no host-side work beyond the launch)
        static std::atomic<size_t> configured[256];
        int dev = 0;
        cudaError_t e = cudaGetDevice(&dev);
        if (e != cudaSuccess) return e;
        if (configured[dev & 255].load() < smem) {
            e = cudaFuncSetAttribute(bfs_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            if (e != cudaSuccess) return e;
            configured[dev & 255].store(smem);
        }
    }
    bfs_small_kernel<<<1, kSB, smem, s>>>(p, root, level, parent);
    return cudaGetLastError();
}

size_t small_smem_limit(int dev)
{
    int v = 0;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) return 0;
    // minus the kernel's static shared memory (control words, per-warp
    // counters and token tables)
    cudaFuncAttributes fa{};
    if (cudaFuncGetAttributes(&fa, bfs_small_kernel) != cudaSuccess) return 0;
    return (size_t)v > fa.sharedSizeBytes ? (size_t)v - fa.sharedSizeBytes : 0;
}

}  // namespace tqk
