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
// Staged tokens per warp (2-3 KiB smem). A larger stage publishes children in
// bigger, later batches: fewer label-correcting re-scans, less work visible to
// idle warps. Measured (results/ab_occupancy_r01.md, stage sweeps): 768 is best
// for byte-mirror graphs (<= 2^25 vertices; kron24 3.87 -> 3.62 ms); 640 for
// nibble-mirror ones (round 2: kron26 over the bench's 64 roots 14.61 -> 14.43
// ms together with no idle back-off, results/level_tokens_r02.log).
// SSSP keeps 512, the setting it was tuned and validated with (its run-to-run
// spread, 18.6-25.4 ms per s24 source at either size, hides any difference).
template <int MIR, int TASK> __host__ __device__ constexpr int stage_cap()
{
    return TASK == kTaskBFS ? (MIR == 8 ? 768 : 640) : 512;
}
constexpr int kU = 4;                // 32-edge rounds in flight per lane
// Resident blocks per SM requested from ptxas (40 warps/SM; <= 48 registers).
// The expansion is bound by the L2 request rate of its random mirror probes
// (DESIGN.md section 6), so occupancy matters through latency hiding and
// spills; interleaved A/B on B200 (results/ab_occupancy_r01.md): 5 blocks
// beat 6 by 1-3% on Kronecker and 8% on the grid, 4 and 8 blocks are slower.
constexpr int kMinBlocks = 5;
constexpr unsigned kLvlSat = 254;    // byte: 0..253 exact, 254 = ">= 254", 255 = unreached / none
// Level mirror (R8), MIR bits per vertex:
//   MIR = 8: one byte per vertex: 0..253 exact-or-stale-high, 254 = ">= 254",
//            255 = unreached; updated with a plain store.
//   MIR = 4: one nibble per vertex, eight per 32-bit word (u in word u >> 3,
//            bits 4 * (u & 7)): 0..13, 14 = ">= 14", 15 = unreached; updated
//            with a CAS loop.  Half the bytes, so it stays L2-resident where a
//            byte mirror does not (scale 26: 34 MB vs 67 MB); the plan picks it
//            when the byte mirror would exceed 32 MB.
template <int MIR> struct Mirror;
template <> struct Mirror<8> { static constexpr unsigned kSat = 254; };
template <> struct Mirror<4> { static constexpr unsigned kSat = 14; };
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
// L2 eviction policies (createpolicy, sm_80+): the col stream is read once
// per expansion and must not evict the L2-resident byte mirror.
__device__ __forceinline__ unsigned long long l2_policy_evict_first()
{
    unsigned long long pol;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ unsigned long long l2_policy_evict_last()
{
    unsigned long long pol;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ int32_t ld_nc_i32(const int32_t *p, unsigned long long pol)
{
    int32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int64_t ld_nc_i64(const int64_t *p)
{
    int64_t v;
    asm("ld.global.nc.s64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ unsigned ld_cg_u32(const unsigned *p, unsigned long long pol)
{
    unsigned v;
    asm volatile("ld.global.cg.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ unsigned ld_cg_u8(const uint8_t *p, unsigned long long pol)
{
    unsigned v;
    asm volatile("ld.global.cg.L2::cache_hint.u8 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
// The byte mirror's probe through L1 (a weak load): stale-high values are all
// the prefilter needs (R8), and with levels in the tokens (R22) no acquire
// poll invalidates the L1, so the relabelled plan's top hubs (the first 2^14
// ids, relabel.cu) stay cached there.  kron24: -0.4% over the bench's batches, up to
// -3.5% in per-root A/Bs (results/level_tokens_r02.log).
__device__ __forceinline__ unsigned ld_l1_u8(const uint8_t *p, unsigned long long pol)
{
    unsigned v;
    asm("ld.global.L2::cache_hint.u8 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ unsigned mix32(unsigned x)
{
    x ^= x >> 16;
    x *= 0x7feb352du;
    x ^= x >> 15;
    x *= 0x846ca68bu;
    x ^= x >> 16;
    return x;
}
__device__ __forceinline__ unsigned ld_relaxed_u8(const uint8_t *p)
{
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u8 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_u8(uint8_t *p, unsigned v)
{
    asm volatile("st.global.u8 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_relaxed_i32(const int32_t *p)
{
    int v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_i32(int32_t *p, int v)
{
    asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
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

__device__ __forceinline__ unsigned backoff_rand()
{
    unsigned r;
    asm volatile("mov.u32 %0, %%globaltimer_lo;" : "=r"(r));
    r ^= (blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B9u;
    r ^= r >> 15;
    r *= 0x2C1B3C6Du;
    r ^= r >> 12;
    return r;
}

// Bounded, randomised exponential back-off after a failed CAS
// (bfs_opts.cas_backoff_ns; 0 = retry at once, the naive form).
//
// Per-thread form (BASE): the 32 lanes of a warp fail together in lock-step
// (one CAS of the 32 wins), and a sleep would stall the warp as a unit, so a
// lane instead sits out a random number of ~32 ns retry rounds in a window
// that doubles per failure up to bo_max ns: only lanes whose wait expired
// issue the next CAS.
struct LaneBackoff {
    unsigned win = 0, skip = 0;
};
__device__ __forceinline__ bool backoff_wait(LaneBackoff &b)
{
    if (!b.skip) return false;
    --b.skip;
    __nanosleep(32);
    return true;
}
__device__ __forceinline__ void backoff_fail(LaneBackoff &b, unsigned bo_max)
{
    if (!bo_max) return;
    const unsigned maxw = bo_max / 32 > 1 ? bo_max / 32 : 1;
    b.win = b.win ? min(2 * b.win, maxw) : 1;
    b.skip = backoff_rand() % (b.win + 1);
}
// Warp form (AN, the proxy's CAS): the warp sleeps a random time in
// [window/2, window], the window doubling from 32 ns up to bo_max ns.
__device__ __forceinline__ void cas_backoff(unsigned *bo, unsigned bo_max)
{
    if (!bo_max) return;
    *bo = *bo ? min(*bo * 2, bo_max) : min(32u, bo_max);
    const unsigned r = __shfl_sync(TQ_FULL_MASK, backoff_rand(), 0);  // one draw per warp
    __nanosleep(*bo / 2 + r % (*bo / 2 + 1));
}

// BASE dequeue of one item by one lane: a classic bounded CAS queue (per-slot
// sequence numbers); retries on CAS failure, returns false on empty.
__device__ __forceinline__ bool cas_dequeue_one(const tq_device_view &q, uint32_t *item,
                                                unsigned *atom, unsigned *fail, unsigned bo_max)
{
    LaneBackoff bo;
    for (unsigned tries = 0; tries < kMaxDeqRetries; ++tries) {
        if (backoff_wait(bo)) continue;
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
            backoff_fail(bo, bo_max);
        } else if (dif < 0) {
            return false;  // queue empty: the exception BASE retries on
        }
    }
    return false;
}

// BASE enqueue of one item by one lane; queue-full aborts (no retry).
__device__ __forceinline__ bool cas_enqueue_one(const tq_device_view &q, uint32_t item,
                                                unsigned *atom, unsigned *fail, unsigned bo_max)
{
    LaneBackoff bo;
    for (unsigned tries = 0; tries < kMaxEnqRetries; ++tries) {
        if (backoff_wait(bo)) continue;
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
            backoff_fail(bo, bo_max);
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
                                               unsigned *fail, unsigned bo_max)
{
    const unsigned lane = tq_lane();
    unsigned tries = 0, bo = 0;
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
        cas_backoff(&bo, bo_max);
        if (++tries >= kMaxDeqRetries) return 0;
    }
}

// AN enqueue: the proxy reserves n slots with one CAS after the warp checked
// they are all empty; retries on CAS failure; aborts on queue-full.
__device__ __forceinline__ bool an_reserve_rear(const tq_device_view &q, unsigned n,
                                                unsigned long long *base_out, unsigned *atom,
                                                unsigned *fail, unsigned bo_max)
{
    const unsigned lane = tq_lane();
    unsigned bo = 0;
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
        cas_backoff(&bo, bo_max);
    }
}

// ---------------------------------------------------------------------------
// Enqueue of a warp's staged tokens (Listing 3).  `items` in shared memory,
// `cnt` warp-uniform.  Coalesced: lane i writes tickets base+i, base+i+32, ...
// ---------------------------------------------------------------------------
//
// lap_end: every slot of a ticket below lap_end is known to hold "empty for
// t" -- at run start all slots of [t0, t0 + C) do (R18) -- so
// Listing 3's queue-full check (P:268 line 25) cannot fail there and its slot
// read is skipped; tickets at or past lap_end are checked.
template <int VARIANT>
__device__ __forceinline__ void enqueue_staged(const tq_device_view &q, const uint32_t *items,
                                               unsigned cnt, unsigned lane, unsigned *qatom,
                                               unsigned *casfail, unsigned long long lap_end, unsigned bo_max,
                                               bool need_fence = true)
{
    if (cnt == 0) return;
    if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_AN) {
        unsigned long long base;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            // the proxy's AFA is issued, then the release fence, and
            // only then is the reserved base read: the fence's drain of this
            // warp's earlier stores overlaps the atomic's round trip
            unsigned long long b0 = 0;
            if (lane == 0) {
                b0 = tq_atom_add(q.rear, (unsigned long long)cnt);
                ++*qatom;
            }
            // release: the W updates (and this warp's Rear reservation) are
            // ordered before the tokens that name them -- needed only when a
            // token does not carry its level (R22)
            if (need_fence) tq_fence_release();
            base = tq_shfl64(b0, 0);
        } else {
            if (!an_reserve_rear(q, cnt, &base, qatom, casfail, bo_max)) return;
            tq_fence_release();  // as above
        }
        if (VARIANT == TQ_VARIANT_RF_AN && base + cnt <= lap_end) {  // warp-uniform
            for (unsigned i = lane; i < cnt; i += 32) {
                const unsigned long long t = base + i;
                tq_st_relaxed(q.slots + (t & q.mask), ((unsigned long long)items[i] << 32) | (unsigned)(t + 1));
            }
            return;
        }
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
            base = tq_atom_add(per_lane_addr(q.rear), mine);
            ++*qatom;
        }
        tq_fence_release();
        for (unsigned k = 0; k < mine; ++k) tq_publish(q, base + k, items[lane + 32 * k]);
    } else {  // CAS_RETRY: one CAS-reserved slot per item, per lane
        tq_fence_release();
        for (unsigned i = lane; i < cnt; i += 32)
            if (!cas_enqueue_one(q, items[i], qatom, casfail, bo_max)) break;
    }
}

// LIT (R22): does any of the cnt staged vertex tokens lack its
// level (all-ones level field)?  Then the flush needs the release fence.
__device__ __forceinline__ bool staged_unknown(const uint32_t *items, unsigned cnt, unsigned lane, unsigned vb)
{
    const unsigned lu = 0x7FFFFFFFu >> vb;
    bool u = false;
    for (unsigned i = lane; i < cnt; i += 32) u |= (items[i] >> vb) == lu;
    return __any_sync(TQ_FULL_MASK, u);
}

// chunk tokens of one hub: CHUNK_FLAG | (first + k), k < n (warp-uniform args)
template <int VARIANT>
__device__ __forceinline__ void enqueue_chunks(const tq_device_view &q, uint32_t first, unsigned n,
                                               unsigned lane, unsigned *qatom, unsigned *casfail,
                                               unsigned long long lap_end, unsigned bo_max,
                                               uint32_t lvbits = 0, bool need_fence = true)
{
    if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
        for (unsigned i = lane; i < n; i += 32)
            if (!cas_enqueue_one(q, CHUNK_FLAG | (first + i), qatom, casfail, bo_max)) break;
        return;
    } else {
        unsigned long long base;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            unsigned long long b0 = 0;  // AFA, then the fence, then its result (as in enqueue_staged)
            if (lane == 0) {
                b0 = tq_atom_add(q.rear, (unsigned long long)n);
                ++*qatom;
            }
            // release: a chunk token names the hub's W entry (its level) --
            // needed only when the token does not carry the level (R22)
            if (need_fence) tq_fence_release();
            base = tq_shfl64(b0, 0);
        } else if constexpr (VARIANT == TQ_VARIANT_AN) {
            if (!an_reserve_rear(q, n, &base, qatom, casfail, bo_max)) return;
            tq_fence_release();  // as above
        } else {  // PER_THREAD_AFA: each lane reserves its own share
            const unsigned mine = lane < n ? (n - lane + 31) / 32 : 0;
            base = 0;
            if (mine) {
                base = tq_atom_add(per_lane_addr(q.rear), mine);
                ++*qatom;
            }
            for (unsigned k = 0; k < mine; ++k)
                tq_publish(q, base + k, CHUNK_FLAG | (first + lane + 32 * k));
            return;
        }
        if (VARIANT == TQ_VARIANT_RF_AN && base + n <= lap_end) {  // first lap: no full check
            for (unsigned i = lane; i < n; i += 32)
                tq_st_relaxed(q.slots + ((base + i) & q.mask),
                              ((unsigned long long)(CHUNK_FLAG | lvbits | (first + i)) << 32) | (unsigned)(base + i + 1));
            return;
        }
        for (unsigned i = lane; i < n; i += 32) tq_publish(q, base + i, CHUNK_FLAG | lvbits | (first + i));
    }
}

// ---------------------------------------------------------------------------
// The persistent kernel
// ---------------------------------------------------------------------------
template <int VARIANT, int TASK = kTaskBFS, int KU = kU, int MINB = kMinBlocks, int MIR = 8, bool LITT = false>
__global__ void __launch_bounds__(kBlock, MINB) bfs_persistent_kernel(const BfsParams p)
{
    constexpr unsigned kMirSat = Mirror<MIR>::kSat;
    constexpr int kStageCap = stage_cap<MIR, TASK>();
    __shared__ uint32_t stage_all[kWarps][kStageCap];
    const unsigned lane = threadIdx.x & 31;
    const unsigned warp_gid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    uint32_t *stage = stage_all[threadIdx.x >> 5];
    // owner lanes of one round's atomicMin candidates (ids go to the stage tail)
    __shared__ uint8_t cown_all[kWarps][32 * KU];
    uint8_t *cown = cown_all[threadIdx.x >> 5];
    // nibble mirror: their probed mirror words (the CAS's expected value)
    __shared__ unsigned cw_all[MIR == 4 ? kWarps : 1][MIR == 4 ? 32 * KU : 1];
    unsigned *cw = cw_all[MIR == 4 ? (threadIdx.x >> 5) : 0];
    // BFS: the warp's non-empty tokens of the current cycle (edge -> token map)
    __shared__ uint4 trec_all[TASK == kTaskBFS ? kWarps : 1][32];
    uint4 *trec = trec_all[TASK == kTaskBFS ? (threadIdx.x >> 5) : 0];
    const tq_device_view q = p.q;
    const unsigned long long cap = q.mask + 1;
    const int chunk = p.chunk;

    // The lane's DequeueThreadSlotIndex.  Only the low 32 bits of the 64-bit
    // ticket are kept: with C <= 2^31 they fix both the slot (t & mask) and
    // the sequence tag (u32)(t + 1) the slot protocol compares.
    unsigned tk = 0;
    bool have = false;
    const unsigned cap32 = (unsigned)cap;
    // statistics: per-warp counters in shared memory, updated by lane 0 with
    // warp-aggregated counts (keeps them out of the hot loop's registers)
    __shared__ unsigned long long wst_all[kWarps][kStatCount];
    __shared__ unsigned long long wdeadline[kWarps];
    unsigned long long *S = wst_all[threadIdx.x >> 5];
    if (lane < kStatCount) S[lane] = 0;
    if (lane == 0) wdeadline[threadIdx.x >> 5] = tq_globaltimer() + p.timeout_ns;
    __syncwarp();
    unsigned st_qatom = 0, st_fail = 0;
    const bool min_id = p.parent_rule == TQ_PARENT_MIN_ID;
    unsigned backoff = 0, idle = 0, busy = 0;
    // Level in the token (R22; RF/AN BFS): a vertex token is
    // [0 | level : 31 - vb | id : vb], a chunk token [1 | level : 31 - cb | id : cb]
    // (vb, cb = p.tok_vbits, p.tok_cbits); an all-ones level field means
    // "not carried" (the level did not fit).  A consumer of a token that
    // carries its level needs nothing its producer wrote besides the slot
    // word, so such tokens are published without a release fence and
    // polled without acquire semantics (no L1 invalidation per poll).
    // (an instantiation of its own: a plan whose levels outgrew the field
    // runs the kernel without it, unchanged)
    constexpr bool LIT = LITT && VARIANT == TQ_VARIANT_RF_AN && TASK == kTaskBFS;
    // LIT: tasks finished, added to Done when the warp goes idle (lane 0; in
    // shared memory, out of the hot loop's registers)
    __shared__ unsigned pend_done_all[kWarps];
    unsigned &pend_done = pend_done_all[threadIdx.x >> 5];
    if (lane == 0) pend_done = 0;

    // Listing 1, split in two halves: the proxy's
    // atomic_add(Front, n) for the lanes that became hungry is issued right
    // after their take and its result is consumed one cycle later, so the
    // atomic's latency hides behind the expansion.
    unsigned pend_base = 0;  // lane 0: (low half of the) base of the in-flight reservation
    unsigned pend_mask = 0;  // warp-uniform: lanes waiting for it
    // Chunk queue: a second RF/AN queue holding
    // only chunk tokens; lane 0 of every warp holds one ticket in it and
    // polls it before its main-queue ticket, so a hub's chunks are expanded
    // by consecutive warps right after the hub is dequeued.
    const bool hubq = VARIANT == TQ_VARIANT_RF_AN && p.hub_queue;
    const tq_device_view q1 = p.q1;
    // lanes holding a chunk-queue ticket (warp-uniform mask, e.g. lanes 0,8,16,24)
    const unsigned q1_lanes = hubq ? p.q1_lanes : 0u;
    const bool q1_lane = (q1_lanes >> lane) & 1u;
    unsigned tk1 = 0, pend1_base = 0, pend1_mask = 0;
    bool have1 = false;
    if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
        // lanes that hold main-queue tickets (all 32, or the first few on small
        // graphs, so that a level's consecutive tokens spread over more warps):
        // the start-up reservation covers popc(ticket_lanes) tickets and the
        // consume below ranks only the lanes in the mask (a lane outside it
        // never becomes hungry)
        pend_mask = TQ_FULL_MASK;
        pend1_mask = q1_lanes;
        if (lane == 0) {
            pend_base = (unsigned)tq_atom_add(q.front, (unsigned long long)__popc(p.ticket_lanes));
            ++st_qatom;
            if (hubq) {
                pend1_base = (unsigned)tq_atom_add(q1.front, (unsigned long long)__popc(q1_lanes));
                ++st_qatom;
            }
        }
    }

    for (;;) {
        // ---- Listing 1 + Listing 2: GetWorkToken() ----
        bool got = false, got1 = false;
        uint32_t item = 0;
        if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
            if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
                if (pend_mask) {  // Listing 1 lines 16-19
                    pend_mask &= p.ticket_lanes;
                    const unsigned base = __shfl_sync(TQ_FULL_MASK, pend_base, 0);
                    if (pend_mask >> lane & 1u) {
                        tk = base + __popc(pend_mask & tq_lanemask_lt());
                        have = true;
                    }
                    pend_mask = 0;
                }
                if (pend1_mask) {
                    const unsigned base = __shfl_sync(TQ_FULL_MASK, pend1_base, 0);
                    if (pend1_mask >> lane & 1u) {
                        tk1 = base + __popc(pend1_mask & tq_lanemask_lt());
                        have1 = true;
                    }
                    pend1_mask = 0;
                }
            } else if (!have) {
                tk = (unsigned)tq_atom_add(per_lane_addr(q.front), 1ull);
                have = true;
                ++st_qatom;
            }
            // Listing 2 lines 3-5: non-atomic arrival checks; a chunk-queue
            // lane issues both polls back to back and prefers the chunk
            // (acquire loads: a hit makes the producer's W update visible,
            // with no fence; ld.acquire.gpu is LDG.STRONG.GPU + CCTL.IVALL)
            // (LIT: relaxed; the rare token without its level takes a fence below)
            const unsigned long long sv0 =
                have ? (LIT ? tq_ld_relaxed(q.slots + (tk & q.mask)) : tq_ld_acquire(q.slots + (tk & q.mask))) : 0ull;
            const unsigned long long sv1 =
                (q1_lane && have1) ? (LIT ? tq_ld_relaxed(q1.slots + (tk1 & q1.mask))
                                          : tq_ld_acquire(q1.slots + (tk1 & q1.mask)))
                                   : 0ull;
            got1 = q1_lane && have1 && (unsigned)sv1 == tk1 + 1u;
            got = !got1 && have && (unsigned)sv0 == tk + 1u;
            item = (uint32_t)((got1 ? sv1 : sv0) >> 32);
        } else if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY) {
            got = cas_dequeue_one(q, &item, &st_qatom, &st_fail, p.cas_backoff_ns);
        } else {  // AN: every lane is hungry each cycle (no held tickets)
            unsigned long long base = 0;
            const unsigned k = an_dequeue(q, 32, &base, &st_qatom, &st_fail, p.cas_backoff_ns);
            if (lane < k) {
                unsigned long long *s = q.slots + ((base + lane) & q.mask);
                const unsigned long long v = tq_ld_relaxed(s);
                item = (uint32_t)(v >> 32);
                tq_st_relaxed(s, (unsigned long long)(unsigned)(base + lane + cap));
                got = true;
            }
        }
        const bool got0 = got;  // token from the main queue
        got = got || got1;
        const unsigned gm = __ballot_sync(TQ_FULL_MASK, got);
        if (gm == 0) {
            // ---- idle work cycle: Algorithm 1 line 1, WorkRemains() ----
            if (lane == 0) ++S[ST_EMPTY_POLLS];
            if constexpr (LIT) {
                // Done += the tasks this warp finished (R6), released
                // after every Rear reservation of theirs (all issued by lane 0)
                if (lane == 0 && pend_done) {
                    tq_fence_release();
                    tq_red_add_relaxed(q.done, (unsigned long long)pend_done);
                    pend_done = 0;
                }
            }
            ++idle;
            if ((idle & 3) == 0 && tq_status_read(q, warp_gid) != TQ_RUNNING) break;
            // termination test: 1 warp in 8, every 4 idle cycles, so idle
            // warps do not crowd the Rear / Done lines busy warps update
            if ((idle & 3) == 0 && (warp_gid & 7) == 0) {
                bool fin = false;
                if (lane == 0) {
                    // Done is read before Rear (R6): done(t1) ==
                    // rear(t2), t1 < t2, implies nothing is queued or in flight
                    const unsigned long long d = tq_ld_acquire(q.done);
                    fin = d == tq_ld_relaxed(q.rear) + (hubq ? tq_ld_relaxed(q1.rear) : 0ull);
                    if (!fin && tq_globaltimer() > wdeadline[threadIdx.x >> 5])
                        tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
                }
                if (__any_sync(TQ_FULL_MASK, fin)) {
                    tq_warp_status_set(q, TQ_FINISHED);
                    break;
                }
            }
            if (p.backoff_ns > 0) {
                backoff = backoff ? min(backoff * 2, (unsigned)p.backoff_ns) : 32u;
                __nanosleep(backoff);
            }
            continue;
        }
        backoff = 0;
        idle = 0;
        if (((++busy) & 63) == 0) {
            if (tq_status_read(q, warp_gid) != TQ_RUNNING) break;
            // the watchdog is honoured by busy warps too: a livelock that keeps
            // every warp busy never reaches the idle-path check
            if ((busy & 1023) == 0 && lane == 0 && tq_globaltimer() > wdeadline[threadIdx.x >> 5])
                tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
        }
        if constexpr (VARIANT == TQ_VARIANT_CAS_RETRY || VARIANT == TQ_VARIANT_AN)
            tq_fence_gpu();  // acquire for the comparators' relaxed dequeues
        // LIT: the token's level field; a token without one was published
        // after a release fence, and its consumer acquires before reading W
        bool unk = false;
        unsigned Lt = 0;
        if constexpr (LIT) {
            if (got) {
                const unsigned b = (item & CHUNK_FLAG) ? p.tok_cbits : p.tok_vbits;
                Lt = (item & ~CHUNK_FLAG) >> b;
                unk = Lt == (0x7FFFFFFFu >> b);
                // its producer fenced before publishing it: an acquire re-read
                // of the (still full) slot synchronises with that release
                if (unk) {
                    if (got1)
                        tq_ld_acquire(q1.slots + (tk1 & q1.mask));
                    else
                        tq_ld_acquire(q.slots + (tk & q.mask));
                }
            }
        }
        if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_PER_THREAD_AFA) {
            if (got0) {  // put the slot back to dna for the next lap
                tq_st_relaxed(q.slots + (tk & q.mask), (unsigned long long)(tk + cap32));
                have = false;
            }
        }
        if constexpr (VARIANT == TQ_VARIANT_RF_AN) {
            // first half of the next dequeue (Listing 1 lines 12-14)
            pend_mask = __ballot_sync(TQ_FULL_MASK, got0);
            pend1_mask = __ballot_sync(TQ_FULL_MASK, got1);
            if (got1) {
                tq_st_relaxed(q1.slots + (tk1 & q1.mask), (unsigned long long)(tk1 + (unsigned)(q1.mask + 1)));
                have1 = false;
            }
            if (lane == 0) {
                if (pend_mask) {
                    pend_base = (unsigned)tq_atom_add(q.front, (unsigned long long)__popc(pend_mask));
                    ++st_qatom;
                }
                if (pend1_mask) {
                    pend1_base = (unsigned)tq_atom_add(q1.front, (unsigned long long)__popc(pend1_mask));
                    ++st_qatom;
                }
            }
        }

        // ---- enumeration prolog (Listing 2 lines 6-22) ----
        int32_t v = 0;
        long long lo = 0, hi = 0;
        unsigned nch = 0;
        uint32_t chb = 0;
        unsigned long long offer = 0;
        bool skipped = false;
        if (got) {
            if (item & CHUNK_FLAG) {
                const int2 c = p.chunk_tab[LIT ? (item & ((1u << p.tok_cbits) - 1u)) : (item & ~CHUNK_FLAG)];
                v = c.x;
                const long long re = ld_nc_i64(p.row_ptr + v + 1);
                lo = ld_nc_i64(p.row_ptr + v) + (long long)c.y * chunk;
                hi = min(lo + (long long)chunk, re);
            } else {
                v = (int32_t)(LIT ? (item & ((1u << p.tok_vbits) - 1u)) : item);
                lo = ld_nc_i64(p.row_ptr + v);
                hi = ld_nc_i64(p.row_ptr + v + 1);
                if (hi - lo > chunk) {  // hub: schedule its sub-tasks instead
                    nch = (unsigned)((hi - lo + chunk - 1) >> p.log2_chunk);
                    chb = (uint32_t)p.hub_base[v];
                    hi = lo;
                }
            }
            // test-only schedule perturbation (bfs_opts.debug_delay_ns)
            unsigned dly = 8;
            if (p.delay_ns) {
                dly = (unsigned)(mix32((unsigned)v ^ p.delay_seed) & 7u);
                if (dly == 0) __nanosleep(p.delay_ns);
            }
            // the parent id W records: on a relabelled plan with min-id
            // parents, v's original id (the minimum must be the one of the
            // original numbering); else v itself (the unpack translates)
            const unsigned pid = (TASK == kTaskBFS && p.pid_orig) ? (unsigned)__ldg(p.new2old + v) : (unsigned)v;
            // current cost of the node (Listing 2 line 21), read fresh
            // (LIT: the token's level, or a lower one W already holds: any
            // value read is a level v has held, so the relaxed read is safe)
            unsigned L = (unsigned)(tq_ld_relaxed(p.W + v) >> 32);
            if constexpr (LIT) {
                if (!unk) L = min(L, Lt);
            }
            if (dly == 1) __nanosleep(p.delay_ns);
            if constexpr (TASK == kTaskSSSP) {
                // the edge weight is added per edge in the expansion
                offer = ((unsigned long long)L << 32) | (unsigned)v;
                if (!(item & CHUNK_FLAG)) {  // expanded-distance marker (R7 for SSSP)
                    const unsigned xprev = (unsigned)ld_relaxed_i32((const int32_t *)p.xd + v);
                    if (xprev <= L) {
                        skipped = true;
                        hi = lo;
                        nch = 0;
                    } else {
                        st_relaxed_i32((int32_t *)p.xd + v, (int)L);
                    }
                }
            } else {
            offer = ((unsigned long long)(L + 1) << 32) | pid;
            if (!(item & CHUNK_FLAG)) {
                // expanded-level marker (R7): a vertex already
                // expanded at a level <= L has offered <= L+1 to every
                // neighbour, so this token has nothing left to do.  Same
                // width as the mirror, saturating like it ("expanded at >=
                // sat" never skips).  The nibble form rewrites the byte it
                // read: a concurrent update of the pair vertex can be undone,
                // which only restores an older (higher) marker -- a weaker
                // skip, never a wrong one (a vertex's expansion levels only
                // fall).
                if constexpr (MIR == 8) {
                    const unsigned xprev = ld_relaxed_u8(p.x8 + v);
                    if (xprev < kLvlSat && xprev <= L) {
                        skipped = true;
                        hi = lo;
                        nch = 0;
                    } else {
                        // (a saturated marker never skips: not stored)
                        if (L < kLvlSat) st_u8(p.x8 + v, L);
                    }
                } else {
                    const unsigned xb = ld_relaxed_u8(p.x8 + ((unsigned)v >> 1));
                    const unsigned sh = ((unsigned)v & 1u) << 2;
                    const unsigned xprev = (xb >> sh) & 0xFu;
                    if (xprev < kMirSat && xprev <= L) {
                        skipped = true;
                        hi = lo;
                        nch = 0;
                    } else if (L < kMirSat) {
                        st_u8(p.x8 + ((unsigned)v >> 1), (xb & ~(0xFu << sh)) | (L << sh));
                    }
                }
            }
            }
        }

        // ---- DoWorkUnit(): warp-cooperative expansion ----
        const int deg = (int)(hi - lo);
        const int incl = warp_incl_scan(deg, lane);
        const int total = __shfl_sync(TQ_FULL_MASK, incl, 31);
        const long long ebase = lo - (incl - deg);
        {
            const unsigned chm = __ballot_sync(TQ_FULL_MASK, got && (item & CHUNK_FLAG));
            const unsigned skm = __ballot_sync(TQ_FULL_MASK, skipped);
            if (lane == 0) {
                S[ST_TASKS] += __popc(gm);
                S[ST_CHUNK_TASKS] += __popc(chm);
                S[ST_SKIPPED] += __popc(skm);
                S[ST_EDGES] += (unsigned)total;
                S[ST_BUSY_CYCLES] += 1;
                S[ST_ROUNDS] += (unsigned)((total + 32 * KU - 1) / (32 * KU));
            }
        }
        unsigned cnt = 0;
        const unsigned long long pol_stream = l2_policy_evict_first();
        const unsigned long long pol_keep = l2_policy_evict_last();
        // Edge -> token map: lane l takes concatenated edges b + 32j + l.
        // SSSP finds its token by a 5-step shuffle binary search over the
        // lanes' inclusive prefix sums; BFS by the rank map below (round 2:
        // kron24 -1.9%, results/ab_round2_r02.md section 10).
        const unsigned offer_hi = (unsigned)(offer >> 32);  // BFS: the offered level L + 1
        // BFS edge -> token map without the shuffle search: the warp's
        // non-empty tokens, in lane order, as {ebase, offered level, lane}
        // records in shared memory; the token of entry g is the one with the
        // largest start <= g, found from a bitmask of the token starts inside
        // each 32-entry slice (one redux.or) plus a running count.
        const int tstart = incl - deg;
        if constexpr (TASK == kTaskBFS) {
            const unsigned ne = __ballot_sync(TQ_FULL_MASK, deg > 0);
            if (deg > 0)
                trec[__popc(ne & tq_lanemask_lt())] =
                    make_uint4((unsigned)ebase, (unsigned)((unsigned long long)ebase >> 32), offer_hi, lane);
            __syncwarp();
        }
        for (int b = 0; b < total; b += 32 * KU) {
            int32_t u[KU];
            unsigned long long off[KU];  // SSSP: per-edge offer (dist + w, v)
            unsigned lv1[KU];            // BFS: offered level of each edge's token
            unsigned ownp = 0;           // BFS: owner lane of edge j in byte j
            bool val[KU];
            if constexpr (TASK == kTaskBFS) {
                // tokens that start before this round
                int cb = __popc(__ballot_sync(TQ_FULL_MASK, deg > 0 && tstart < b));
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    const int sj = b + j * 32;
                    const int g = sj + (int)lane;
                    val[j] = g < total;
                    const unsigned rel = (unsigned)(tstart - sj);
                    const unsigned bs = __reduce_or_sync(TQ_FULL_MASK, (deg > 0 && rel < 32u) ? (1u << rel) : 0u);
                    const int r = cb + __popc(bs & (TQ_FULL_MASK >> (31u - lane))) - 1;
                    cb += __popc(bs);
                    const uint4 t = trec[r < 0 ? 0 : r];
                    const long long eb = (long long)(((unsigned long long)t.y << 32) | t.x);
                    u[j] = val[j] ? ld_nc_i32(p.col + eb + g, pol_stream) : 0;
                    lv1[j] = t.z;
                    ownp |= t.w << (8 * j);
                }
            } else
#pragma unroll
            for (int j = 0; j < KU; ++j) {
                const int g = b + j * 32 + (int)lane;
                val[j] = g < total;
                const int gg = val[j] ? g : total - 1;
                const int o = owner_of(incl, gg);
                const long long eb = (long long)tq_shfl64((unsigned long long)ebase, o);
                u[j] = val[j] ? ld_nc_i32(p.col + eb + gg, pol_stream) : 0;
                if constexpr (TASK == kTaskSSSP) {
                    off[j] = tq_shfl64(offer, o);
                    const unsigned wt = val[j] ? (unsigned)ld_nc_i32(p.wgt + eb + gg, pol_stream) : 0u;
                    const unsigned long long d = (off[j] >> 32) + wt;  // dist(v) + w(v -> u)
                    val[j] = val[j] && d < 0xffffffffull;
                    off[j] = (d << 32) | (off[j] & 0xffffffffull);
                } else {
                    lv1[j] = __shfl_sync(TQ_FULL_MASK, offer_hi, o);
                    ownp |= (unsigned)o << (8 * j);
                }
            }
            bool cand[KU];
            unsigned b8[KU];  // BFS: the probed mirror byte / word
            if constexpr (TASK == kTaskSSSP) {
                // prefilter: the packed word itself (dist, parent) -- stale
                // values are never below the true word, so skipping offers
                // that do not beat it drops no improvement
                unsigned long long w[KU];
#pragma unroll
                for (int j = 0; j < KU; ++j) w[j] = val[j] ? ld_cg_u64(p.W + u[j]) : 0ull;
#pragma unroll
                for (int j = 0; j < KU; ++j) cand[j] = val[j] && off[j] < w[j];
            } else {
                // prefilter 1: the level mirror (L2-resident; stale values are
                // never below the true level, R8)
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    // offers at a level >= the mirror's saturation cannot be
                    // filtered: skip the probe (saves a dependent round trip on
                    // deep graphs, e.g. the grid's 8,191 levels), go to atomicMin
                    const bool deep = lv1[j] >= kMirSat;
                    if constexpr (MIR == 8)
                        b8[j] = (val[j] && !deep) ? (LIT ? ld_l1_u8((const uint8_t *)p.mir + u[j], pol_keep)
                                                          : ld_cg_u8((const uint8_t *)p.mir + u[j], pol_keep))
                                                  : 0xFFu;
                    else
                        b8[j] = (val[j] && !deep) ? ld_cg_u32(p.mir + ((unsigned)u[j] >> 3), pol_keep) : ~0u;
                }
                bool tie[KU];
                bool any_tie = false;
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    const unsigned m8 = MIR == 8 ? b8[j] : (b8[j] >> (((unsigned)u[j] & 7u) << 2)) & 0xFu;
                    const bool known = m8 < kMirSat;  // exact-or-stale-high level
                    tie[j] = val[j] && min_id && known && m8 == lv1[j];
                    cand[j] = val[j] && !(known && m8 <= lv1[j]);
                    any_tie |= tie[j];
                }
                // prefilter 2 (min-id parents only): the packed word, only for
                // offers that tie on level and may still win on parent id
                if (min_id && __any_sync(TQ_FULL_MASK, any_tie)) {
                    unsigned long long w[KU];
#pragma unroll
                    for (int j = 0; j < KU; ++j) w[j] = tie[j] ? ld_cg_u64(p.W + u[j]) : 0ull;
#pragma unroll
                    for (int j = 0; j < KU; ++j) {
                        const unsigned long long oj = tq_shfl64(offer, (ownp >> (8 * j)) & 31u);
                        cand[j] = cand[j] || (tie[j] && oj < w[j]);
                    }
                }
            }
            if constexpr (TASK == kTaskBFS) {
                // Candidates (a few percent of the edges) are compacted into
                // the free tail of the staging buffer -- vertex ids at
                // stage[cnt..), owner lanes in cown[] -- and their atomicMins
                // issued as dense warp instructions, so the round trips of a
                // round's atomics overlap instead of running one per j (the
                // mirror stores between them are ordered).  The vertices whose
                // level fell are then compacted in place, to stage[cnt..).
                unsigned ncand = 0;
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    const unsigned m = __ballot_sync(TQ_FULL_MASK, cand[j]);
                    if (cand[j]) {
                        const unsigned k = ncand + __popc(m & tq_lanemask_lt());
                        stage[cnt + k] = (uint32_t)u[j];
                        cown[k] = (uint8_t)(ownp >> (8 * j));
                        if constexpr (MIR == 4) cw[k] = b8[j];
                    }
                    ncand += __popc(m);
                }
                if (ncand) {
                    __syncwarp();
                    unsigned n_reenq = 0, wr = cnt;
                    for (unsigned i0 = 0; i0 < ncand; i0 += 32) {
                        const unsigned i = i0 + lane;
                        const bool c = i < ncand;
                        const uint32_t cv = c ? stage[cnt + i] : 0u;
                        const unsigned long long co = tq_shfl64(offer, c ? cown[i] : 0u);
                        const unsigned cb = (MIR == 4 && c) ? cw[i] : ~0u;
                        __syncwarp();  // all reads of this slice before the in-place writes
                        const unsigned L1 = (unsigned)(co >> 32);
                        const unsigned oldhi = c ? (unsigned)(atomicMin(p.W + cv, co) >> 32) : 0u;
                        const bool nt = c && oldhi > L1;  // level strictly lowered: (re)discovered
                        // Lower v's mirror entry.  It only ever receives levels
                        // v has held (installed by a successful atomicMin, so
                        // >= the final level): the mirror stays stale-high,
                        // the only property the prefilter needs.  Byte: a
                        // plain store.  Nibble: one fire-and-forget CAS from
                        // the word probed this round (no wait; if another of
                        // the word's 8 vertices changed meanwhile it fails and
                        // v's nibble stays high), and a failed candidate whose
                        // probe read a nibble above v's current level repairs
                        // it the same way, so a missed lowering costs one
                        // extra atomicMin, not one per later probe.
                        if constexpr (MIR == 8) {
                            // (a saturated entry filters nothing -- offers at
                            // or past saturation skip the probe -- so it is not
                            // stored: on deep graphs the flush's release fence
                            // then has no store of this round to wait for)
                            if (nt && L1 < kMirSat) st_u8((uint8_t *)p.mir + cv, L1);
                        } else {
                            const unsigned nv = nt ? L1 : oldhi;  // v's level now
                            const unsigned sh = (cv & 7u) << 2;
                            if (c && nv < kMirSat && nv < ((cb >> sh) & 0xFu))
                                atomicCAS(p.mir + (cv >> 3), cb, (cb & ~(0xFu << sh)) | (nv << sh));
                        }
                        n_reenq += __popc(__ballot_sync(TQ_FULL_MASK, nt && oldhi != 0xffffffffu));
                        const unsigned m = __ballot_sync(TQ_FULL_MASK, nt);
                        if (nt) {
                            uint32_t tok = cv;
                            if constexpr (LIT) {  // the token carries its level (R22)
                                const unsigned lu = 0x7FFFFFFFu >> p.tok_vbits;
                                tok |= min(L1, lu) << p.tok_vbits;
                            }
                            stage[wr + __popc(m & tq_lanemask_lt())] = tok;
                        }
                        wr += __popc(m);
                        __syncwarp();
                    }
                    cnt = wr;
                    if (lane == 0) {
                        S[ST_MIN_ATOMICS] += ncand;
                        S[ST_REENQUEUES] += n_reenq;
                    }
                }
            } else {
                bool nt[KU];
                unsigned n_min = 0, n_reenq = 0;
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    nt[j] = false;
                    bool re = false;
                    if (cand[j]) {
                        const unsigned long long old = atomicMin(p.W + u[j], off[j]);
                        const unsigned L1 = (unsigned)(off[j] >> 32);
                        if ((old >> 32) > L1) {  // level strictly lowered: (re)discovered
                            nt[j] = true;
                            re = (old >> 32) != 0xffffffffull;
                        }
                    }
                    n_min += __popc(__ballot_sync(TQ_FULL_MASK, cand[j]));
                    n_reenq += __popc(__ballot_sync(TQ_FULL_MASK, re));
                }
                if (lane == 0) {
                    S[ST_MIN_ATOMICS] += n_min;
                    S[ST_REENQUEUES] += n_reenq;
                }
#pragma unroll
                for (int j = 0; j < KU; ++j) {
                    const unsigned m = __ballot_sync(TQ_FULL_MASK, nt[j]);
                    if (nt[j]) stage[cnt + __popc(m & tq_lanemask_lt())] = (uint32_t)u[j];
                    cnt += __popc(m);
                }
            }
            if (cnt > kStageCap - 32 * KU) {
                __syncwarp();
                enqueue_staged<VARIANT>(q, stage, cnt, lane, &st_qatom, &st_fail, p.q_lap_end, p.cas_backoff_ns,
                                        !LIT || staged_unknown(stage, cnt, lane, p.tok_vbits));
                __syncwarp();
                cnt = 0;
            }
        }

        // ---- ScheduleNewlyDiscoveredWorkTokens(): Listing 3 ----
        __syncwarp();
        enqueue_staged<VARIANT>(q, stage, cnt, lane, &st_qatom, &st_fail, p.q_lap_end, p.cas_backoff_ns,
                                !LIT || staged_unknown(stage, cnt, lane, p.tok_vbits));
        __syncwarp();
        unsigned hubm = __ballot_sync(TQ_FULL_MASK, nch > 0);
        while (hubm) {
            const int h = __ffs(hubm) - 1;
            hubm &= hubm - 1;
            const unsigned n = __shfl_sync(TQ_FULL_MASK, nch, h);
            const uint32_t first = __shfl_sync(TQ_FULL_MASK, chb, h);
            uint32_t lvbits = 0;
            bool fence = true;
            if constexpr (LIT) {  // the chunk tokens carry the hub's level
                const unsigned Lh = __shfl_sync(TQ_FULL_MASK, (unsigned)(offer >> 32) - 1u, h);
                const unsigned lu = 0x7FFFFFFFu >> p.tok_cbits;
                lvbits = min(Lh, lu) << p.tok_cbits;
                fence = Lh >= lu;
            }
            enqueue_chunks<VARIANT>(hubq ? q1 : q, first, n, lane, &st_qatom, &st_fail,
                                    hubq ? p.q1_lap_end : p.q_lap_end, p.cas_backoff_ns, lvbits, fence);
        }

        // ---- completion accounting for WorkRemains() (R6) ----
        // Done += tasks finished, with release semantics and no round trip:
        // it is ordered after this warp's Rear reservations; idle warps
        // compare Done with Rear.
        if constexpr (VARIANT == TQ_VARIANT_RF_AN || VARIANT == TQ_VARIANT_AN) {
            // lane 0 issued every Rear reservation of this warp, and the
            // release fence that follows each reservation (staged tokens and
            // chunk tokens alike) already ordered it before this increment.
            if (lane == 0) {
                if constexpr (LIT) {
                    pend_done += __popc(gm);  // added when the warp goes idle
                } else {
                    tq_red_add_relaxed(q.done, (unsigned long long)__popc(gm));
                    ++st_qatom;
                }
            }
        } else {
            __syncwarp();
            tq_fence_release();
            if (got) {
                tq_red_add_relaxed(q.done, 1ull);
                ++st_qatom;
            }
        }
    }

    // ---- statistics (one atomic per counter per warp) ----
    {
        const unsigned long long qa = warp_sum((unsigned long long)st_qatom);
        const unsigned long long cf = warp_sum((unsigned long long)st_fail);
        if (lane == 0) {
            S[ST_QUEUE_ATOMICS] += qa;
            S[ST_CAS_FAILURES] += cf;
        }
        __syncwarp();
        if (lane < ST_REACHED && S[lane]) atomicAdd(p.stats + lane, S[lane]);
    }
}

// ---------------------------------------------------------------------------
// a2: state + queue init for one run.  W[:] = unreached, W[root] = (0, root);
// the root is published at ticket t0 (Front = Done = t0, Rear = t0 + 1).
// ---------------------------------------------------------------------------
// Fill nbytes of a 16-byte-aligned buffer with 0xFF, byte `sb` ANDed with
// `smask` (the root's mirror entry), 16 bytes per store.
__device__ __forceinline__ void fill_ff(uint8_t *buf, int64_t nbytes, int64_t sb, unsigned smask,
                                        int64_t tid, int64_t stride)
{
    const int64_t n16 = nbytes / 16;
    for (int64_t c = tid; c < n16; c += stride) {
        uint4 v = make_uint4(~0u, ~0u, ~0u, ~0u);
        if (sb >= 16 * c && sb < 16 * c + 16) {
            unsigned *w = &v.x;
            const int b = (int)(sb - 16 * c);
            w[b >> 2] &= ~((~smask & 0xFFu) << (8 * (b & 3)));
        }
        reinterpret_cast<uint4 *>(buf)[c] = v;
    }
    for (int64_t b = 16 * n16 + tid; b < nbytes; b += stride) buf[b] = (uint8_t)(b == sb ? (0xFFu & smask) : 0xFFu);
}

__global__ void bfs_init_kernel(const BfsParams p, int32_t root, unsigned long long t0,
                                unsigned long long t1)
{
    const int64_t n = p.n_vertices;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    // the root's position (its new id on a relabelled plan) and the parent
    // id W records for it (the original id when W holds original ids)
    const int32_t rn = p.old2new ? __ldg(p.old2new + root) : root;
    const uint32_t rpid = p.pid_orig ? (uint32_t)root : (uint32_t)rn;
    // W: 4 entries (32 bytes) per store pair; plan buffers are pool
    // allocations (256-byte aligned)
    const int64_t n4 = n / 4;
    for (int64_t k = tid; k < n4; k += stride) {
        ulonglong2 a = make_ulonglong2(~0ull, ~0ull), b = a;
        const int64_t i = 4 * k;
        if (rn >= i && rn < i + 4) {
            unsigned long long *e = rn < i + 2 ? &a.x : &b.x;
            e[(rn - i) & 1] = (unsigned long long)rpid;
        }
        reinterpret_cast<ulonglong2 *>(p.W + i)[0] = a;
        reinterpret_cast<ulonglong2 *>(p.W + i)[1] = b;
    }
    for (int64_t i = 4 * n4 + tid; i < n; i += stride)
        p.W[i] = (i == rn) ? (unsigned long long)rpid : ~0ull;
    if (p.mir) {  // level mirror: bytes (root's = 0) or nibbles (15 = unreached, root's = 0)
        if (p.mirror_bits == 8)
            fill_ff((uint8_t *)p.mir, n, rn, 0x00u, tid, stride);
        else
            fill_ff((uint8_t *)p.mir, (n + 7) / 8 * 4, rn >> 1, ~(0xFu << ((rn & 1) << 2)), tid, stride);
    }
    if (p.x8) fill_ff(p.x8, p.mirror_bits == 8 ? n : (n + 1) / 2, -1, 0xFFu, tid, stride);  // markers
    if (p.xd) fill_ff(reinterpret_cast<uint8_t *>(p.xd), 4 * n, -1, 0xFFu, tid, stride);
    if (blockIdx.x == 0) {
        if (threadIdx.x < TQ_STATUS_COPIES) p.q.status[threadIdx.x * TQ_STATUS_STRIDE] = TQ_RUNNING;
        if (threadIdx.x < kStatCount) p.stats[threadIdx.x] = 0;
        if (threadIdx.x == 0) {
            p.q.slots[t0 & p.q.mask] =
                ((unsigned long long)(uint32_t)rn << 32) | (unsigned)(t0 + 1);
            *p.q.front = t0;
            *p.q.rear = t0 + 1;
            // Done counts tasks of both queues: termination is
            // done == rear(main) + rear(chunk queue)
            *p.q.done = t0 + (p.hub_queue ? t1 : 0ull);
            if (p.hub_queue) {
                *p.q1.front = t1;
                *p.q1.rear = t1;
            }
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
    // outputs and statistics in the original vertex order: on a relabelled
    // plan vertex o's word is W[old2new[o]] (a gather), its degree from the
    // original offsets
    const int32_t *o2n = p.old2new;
    const int64_t *rp0 = p.row_ptr0 ? p.row_ptr0 : p.row_ptr;
    // parents recorded as new ids are translated back
    const int32_t *n2o = p.pid_orig ? nullptr : p.new2old;
    // 4 vertices per thread with 16-byte accesses when every array is 16-byte
    // aligned (HBM-bound: W 8 B + row_ptr 8 B read, level + parent 8 B written
    // per vertex); the scalar loop takes the tail and unaligned outputs
    const bool vec = ((reinterpret_cast<uintptr_t>(p.W) | reinterpret_cast<uintptr_t>(rp0) |
                       reinterpret_cast<uintptr_t>(o2n) | reinterpret_cast<uintptr_t>(level) |
                       reinterpret_cast<uintptr_t>(parent)) & 15) == 0;
    int64_t done = 0;
    if (vec) {
        const int64_t n4 = n / 4;
        for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n4; k += stride) {
            const int64_t i = 4 * k;
            unsigned long long w[4];
            if (o2n) {
                const int4 m = __ldg(reinterpret_cast<const int4 *>(o2n + i));
                w[0] = p.W[m.x];
                w[1] = p.W[m.y];
                w[2] = p.W[m.z];
                w[3] = p.W[m.w];
            } else {
                const ulonglong2 w01 = *reinterpret_cast<const ulonglong2 *>(p.W + i);
                const ulonglong2 w23 = *reinterpret_cast<const ulonglong2 *>(p.W + i + 2);
                w[0] = w01.x;
                w[1] = w01.y;
                w[2] = w23.x;
                w[3] = w23.y;
            }
            int4 lv, pa;
            int *lvp = &lv.x, *pap = &pa.x;
            bool any = false;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const unsigned l = (unsigned)(w[j] >> 32);
                const bool r = l != 0xffffffffu;
                lvp[j] = r ? (int32_t)l : -1;
                pap[j] = r ? (n2o ? __ldg(n2o + (uint32_t)w[j]) : (int32_t)(uint32_t)w[j]) : -1;
                if (r) {
                    ++reached;
                    maxl = max(maxl, l);
                }
                any |= r;
            }
            if (level) *reinterpret_cast<int4 *>(level + i) = lv;
            if (parent) *reinterpret_cast<int4 *>(parent + i) = pa;
            if (any) {
                const longlong2 r01 = *reinterpret_cast<const longlong2 *>(rp0 + i);
                const longlong2 r23 = *reinterpret_cast<const longlong2 *>(rp0 + i + 2);
                const long long r4 = ld_nc_i64(rp0 + i + 4);
                const long long rp[5] = {r01.x, r01.y, r23.x, r23.y, r4};
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    if (lvp[j] >= 0) degsum += (unsigned long long)(rp[j + 1] - rp[j]);
            }
        }
        done = 4 * n4;
    }
    for (int64_t i = done + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const unsigned long long w = p.W[o2n ? o2n[i] : i];
        const unsigned l = (unsigned)(w >> 32);
        const bool r = l != 0xffffffffu;
        if (level) level[i] = r ? (int32_t)l : -1;
        if (parent) parent[i] = r ? (n2o ? __ldg(n2o + (uint32_t)w) : (int32_t)(uint32_t)w) : -1;
        if (r) {
            ++reached;
            degsum += (unsigned long long)(ld_nc_i64(rp0 + i + 1) - ld_nc_i64(rp0 + i));
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

// Slot i holds "empty" for the ticket t in [t0, t0 + C) with t mod C == i.
__global__ void queue_reset_kernel(tq_device_view q, unsigned long long t0)
{
    const unsigned long long cap = q.mask + 1;
    const unsigned long long stride = (unsigned long long)gridDim.x * blockDim.x;
    for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < cap;
         i += stride)
        q.slots[i] = (unsigned)(t0 + ((i - t0) & q.mask));
    if (blockIdx.x == 0) {
        if (threadIdx.x < TQ_STATUS_COPIES) q.status[threadIdx.x * TQ_STATUS_STRIDE] = TQ_RUNNING;
        if (threadIdx.x == 0) {
            *q.front = t0;
            *q.rear = t0;
            *q.done = t0;
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

cudaError_t launch_bfs_init(const BfsParams &p, int32_t root, unsigned long long t0,
                            unsigned long long t1, cudaStream_t s)
{
    bfs_init_kernel<<<grid_for(p.n_vertices, 256), 256, 0, s>>>(p, root, t0, t1);
    return cudaGetLastError();
}

cudaError_t launch_bfs_unpack(const BfsParams &p, int32_t *level, int32_t *parent, cudaStream_t s)
{
    bfs_unpack_kernel<<<grid_for(p.n_vertices, 256), 256, 0, s>>>(p, level, parent);
    return cudaGetLastError();
}

cudaError_t launch_queue_reset(const tq_device_view &q, unsigned long long t0, cudaStream_t s)
{
    queue_reset_kernel<<<grid_for((int64_t)(q.mask + 1), 256), 256, 0, s>>>(q, t0);
    return cudaGetLastError();
}

template <int V, int TASK = kTaskBFS, int KU = kU, int MINB = kMinBlocks, int MIR = 8, bool LITT = false>
static cudaError_t launch_v(const BfsParams &p, int blocks, int block, cudaStream_t s)
{
    if (block != kBlock) return cudaErrorInvalidValue;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(kBlock);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    if (p.l2_window_bytes) {
        // keep the level mirror (probed once per edge) resident in the
        // persisting part of L2 while the col stream and the per-task arrays
        // pass through
        attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[0].val.accessPolicyWindow.base_ptr = (void *)p.mir;
        attr[0].val.accessPolicyWindow.num_bytes = p.l2_window_bytes;
        attr[0].val.accessPolicyWindow.hitRatio = 1.0f;
        attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
    }
    return cudaLaunchKernelEx(&cfg, bfs_persistent_kernel<V, TASK, KU, MINB, MIR, LITT>, p);
}

cudaError_t launch_bfs_persistent(int variant, const BfsParams &p, int blocks, int block,
                                  cudaStream_t s)
{
    if (p.task == kTaskSSSP) {  // the generic-scheduler row runs on the RF/AN queue
        if (variant != TQ_VARIANT_RF_AN) return cudaErrorInvalidValue;
        return launch_v<TQ_VARIANT_RF_AN, kTaskSSSP>(p, blocks, block, s);
    }
    // One block per SM (small graphs, deep-graph plans): the instantiation
    // compiled for one resident block, with every register it wants instead
    // of the 48 that five blocks allow (grid 4096^2: 41.0 -> 38.7 ms,
    // results/deep_stores_r02.log)
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const bool one_per_sm = blocks <= sms;
    switch (variant) {
    case TQ_VARIANT_RF_AN:  // with / without levels in the tokens (R22)
        if (one_per_sm) {
            if (p.mirror_bits == 4)
                return p.lit ? launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, 1, 4, true>(p, blocks, block, s)
                             : launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, 1, 4>(p, blocks, block, s);
            return p.lit ? launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, 1, 8, true>(p, blocks, block, s)
                         : launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, 1, 8>(p, blocks, block, s);
        }
        if (p.mirror_bits == 4)
            return p.lit ? launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, kMinBlocks, 4, true>(p, blocks, block, s)
                         : launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, kMinBlocks, 4>(p, blocks, block, s);
        return p.lit ? launch_v<TQ_VARIANT_RF_AN, kTaskBFS, kU, kMinBlocks, 8, true>(p, blocks, block, s)
                     : launch_v<TQ_VARIANT_RF_AN>(p, blocks, block, s);
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
                              int2 **chunk_tab_out, int64_t *n_chunks_out, int32_t *pinned8, cudaStream_t s)
{
    *chunk_tab_out = nullptr;
    *n_chunks_out = 0;
    int32_t *nch = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    cudaError_t e = pool_alloc(&nch, (size_t)n * sizeof(int32_t), s);
    if (e != cudaSuccess) return e;
    count_chunks_kernel<<<grid_for(n, 256), 256, 0, s>>>(row_ptr, n, chunk, nch);
    e = cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, nch, hub_base, (int)n, s);
    if (e == cudaSuccess) e = pool_alloc(&tmp, tmp_bytes, s);
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, nch, hub_base, (int)n, s);
    // (read back through pinned memory: a pageable copy would serialise with
    // other streams' work, e.g. a BFS running while the next plan is built)
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(pinned8, hub_base + n - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(pinned8 + 1, nch + n - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    const int64_t total = e == cudaSuccess ? (int64_t)pinned8[0] + pinned8[1] : 0;
    if (e == cudaSuccess && total > 0) {
        int2 *tab = nullptr;
        e = pool_alloc(&tab, (size_t)total * sizeof(int2), s);
        if (e == cudaSuccess) {
            fill_chunks_kernel<<<grid_for(n, 256), 256, 0, s>>>(row_ptr, n, chunk, hub_base, tab);
            e = cudaGetLastError();
            if (e == cudaSuccess) e = cudaStreamSynchronize(s);
            if (e == cudaSuccess) {
                *chunk_tab_out = tab;
                *n_chunks_out = total;
            } else {
                pool_free(tab, s);
            }
        }
    }
    pool_free(tmp, s);
    pool_free(nch, s);
    return e;
}

}  // namespace tqk
