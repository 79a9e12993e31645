// internal.cuh -- declarations shared by the kernels (bfs.cu, bench.cu) and
// the C-ABI implementation (api.cu).  Not part of the public boundary.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/tq.h"
#include "../../include/tq_device.cuh"

namespace tqk {

// Token encoding: a 32-bit item is either a vertex
// id (< 2^31) or CHUNK_FLAG | chunk id.  A chunk token names up to `chunk`
// consecutive CSR entries of one high-degree vertex: the paper's refactoring
// of a task into "a fixed number of uniformly complex sub-tasks".
constexpr uint32_t CHUNK_FLAG = 0x80000000u;

// The per-thread-AFA comparator must issue one atomic per lane.  ptxas
// warp-aggregates an atom.add whose address it can prove warp-uniform
// (VOTEU.ANY + FLO + UPOPC + a single ATOMG: the paper's proxy lane, P:167,
// inserted by the compiler).  Offsetting the address by (lane & zero), with
// `zero` a device global that is always 0 but opaque to the compiler, keeps
// the comparator's atomics per lane (checked in the SASS: one ATOMG per lane).
static __device__ unsigned g_opaque_zero = 0;
__device__ __forceinline__ unsigned long long *per_lane_addr(unsigned long long *p)
{
    const unsigned zero = *(volatile const unsigned *)&g_opaque_zero;
    return p + (tq_lane() & zero);
}

// Device memory of queues and plans comes from a library-owned, stream-ordered
// pool (one per device) that keeps freed memory reserved (release threshold =
// max), so plans created and destroyed every step -- bench.py's e2e leg builds
// one from the host CSR per step -- do not pay cudaMalloc / cudaFree of
// multi-GB buffers each time.  tq_memory_trim() returns it to the driver.
cudaError_t pool_alloc_raw(void **p, size_t bytes, cudaStream_t s);
void pool_free(void *p, cudaStream_t s);
template <typename T>
inline cudaError_t pool_alloc(T **p, size_t bytes, cudaStream_t s)
{
    return pool_alloc_raw(reinterpret_cast<void **>(p), bytes, s);
}

constexpr int kStatCount = 16;

// Task run by the persistent kernel over the queue (the queue is the same).
constexpr int kTaskBFS = 0;   // top-down BFS levels (the paper's driver)
constexpr int kTaskSSSP = 1;  // label-correcting shortest paths (NEXT row 4)
enum StatIndex {
    ST_TASKS = 0,
    ST_CHUNK_TASKS,
    ST_EDGES,
    ST_MIN_ATOMICS,
    ST_REENQUEUES,
    ST_QUEUE_ATOMICS,
    ST_CAS_FAILURES,
    ST_EMPTY_POLLS,
    ST_SKIPPED,
    ST_BUSY_CYCLES,  // work cycles that processed >= 1 token
    ST_ROUNDS,       // 32 x 4-edge expansion rounds
    // filled by the unpack kernel
    ST_REACHED,
    ST_DEG_SUM,
    ST_MAX_LEVEL,
    ST_SMEM_TICKETS,  // shared-memory path: tickets issued (its Rear at the end)
    ST_COUNT_
};

struct BfsParams {
    tq_device_view q;          // main queue: vertex tokens (and chunk tokens if !hub_queue)
    tq_device_view q1;         // chunk queue (hub sub-tasks), valid if hub_queue
    int hub_queue;             // RF/AN only: chunk tokens go to q1, polled first
    unsigned q1_lanes;         // lanes of each warp that hold a q1 ticket
    const int64_t *row_ptr;
    const int32_t *col;
    unsigned long long *W;     // packed (level << 32) | parent, ~0 = unreached
    const int2 *chunk_tab;     // chunk id -> {vertex, k}
    const int32_t *hub_base;   // vertex -> first chunk id (read for hubs only)
    unsigned *mir;             // level mirror (prefilter): bytes or nibbles, see bfs.cu Mirror<>
    int mirror_bits;           // 8 (byte per vertex) or 4 (nibble; RF/AN BFS on large graphs)
    uint8_t *x8;               // level at which the vertex was expanded (saturating byte)
    unsigned *xd;              // SSSP: distance at which the vertex was expanded
    const int32_t *wgt;        // SSSP: edge weights (one per CSR entry), else null
    int task;                  // kTaskBFS / kTaskSSSP
    unsigned long long *stats; // kStatCount counters
    int64_t n_vertices;
    int chunk;                 // max edges per token (power of 2)
    int log2_chunk;
    int backoff_ns;            // max idle back-off, 0 = none
    int parent_rule;           // TQ_PARENT_ANY / TQ_PARENT_MIN_ID (include/tq.h)
    unsigned long long timeout_ns;
    size_t l2_window_bytes;    // persisting-L2 window over the level mirror (0 = none)
    unsigned delay_ns;         // test only: schedule perturbation (bfs_opts.debug_delay_ns)
    unsigned delay_seed;
    // first-lap bounds: tickets below these are known empty at run start
    // (t0 + C of each queue), so their enqueue skips the full check
    unsigned long long q_lap_end;
    unsigned long long q1_lap_end;
    unsigned cas_backoff_ns;   // CAS variants: max back-off after a failed CAS (0 = none)
    unsigned ticket_lanes;     // RF/AN: mask of the lanes that hold main-queue tickets
    int64_t nnz;               // CSR entries (the shared-memory path loads them all)
    // vertex relabelling (relabel.cu): row_ptr / col above are then the
    // relabelled CSR; tokens, W, mirror and markers use new ids, W's parent
    // field original ids; null = no relabelling
    const int32_t *new2old;
    const int32_t *old2new;
    const int64_t *row_ptr0;   // the original row offsets (unpack statistics)
    // RF/AN BFS token layout (R22): id bits of vertex / chunk tokens;
    // the bits between them and the chunk flag carry the token's level
    unsigned tok_vbits;
    unsigned tok_cbits;
    int lit;                   // levels travel in the tokens (off once a plan's levels outgrew the field)
    int pid_orig;              // W's parent field holds original ids (relabelled
                               // min-id plans: the kernel reads new2old); else
                               // the plan's own ids, translated by the unpack
    unsigned small_cap;        // shared-memory path: ring slots (power of two)
};

// bfs.cu
cudaError_t launch_bfs_init(const BfsParams &p, int32_t root, unsigned long long t0,
                            unsigned long long t1, cudaStream_t s);
cudaError_t launch_bfs_persistent(int variant, const BfsParams &p, int blocks, int block,
                                  cudaStream_t s);
cudaError_t launch_bfs_unpack(const BfsParams &p, int32_t *level, int32_t *parent, cudaStream_t s);
cudaError_t bfs_occupancy(int variant, int block, int *blocks_per_sm);
cudaError_t build_chunk_table(const int64_t *row_ptr, int64_t n, int chunk, int32_t *hub_base,
                              int2 **chunk_tab_out, int64_t *n_chunks_out, int32_t *pinned8, cudaStream_t s);
cudaError_t launch_queue_reset(const tq_device_view &q, unsigned long long t0, cudaStream_t s);

// relabel.cu: degree-descending vertex relabelling of a CSR (plan build).
// Nothing is allocated (out stays zero) unless the largest degree exceeds
// min_max_degree; the caller then owns out's four pool buffers.  pinned4:
// 4 bytes of pinned host memory (the one read-back: the largest degree).
struct RelabelOut {
    int32_t *new2old, *old2new;
    int64_t *row_ptr;
    int32_t *col;
};
cudaError_t build_relabel(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int min_max_degree,
                          int64_t hub_region, int32_t *pinned4, RelabelOut *out, cudaStream_t s);

// bfs_small.cu: the whole run (load, BFS over a shared-memory queue, unpack)
// in one 1024-thread block, for graphs whose state fits in shared memory
size_t small_smem_bytes(int64_t n, int64_t nnz, uint64_t cap);
size_t small_smem_limit(int dev);
cudaError_t launch_bfs_small(const BfsParams &p, int32_t root, int32_t *level, int32_t *parent, cudaStream_t s);

// bench.cu
struct BenchParams {
    tq_device_view q;
    int batch;
    int iters;                 // per warp
    int work_iters;
    uint32_t seed32;
    uint32_t *enq_log;
    uint32_t *deq_log;
    unsigned long long *out;   // [0..] counters (see bench.cu)
    unsigned long long timeout_ns;
    unsigned cas_backoff_ns;   // CAS variants: max back-off after a failed CAS (0 = none)
    int relaxed_poll;          // 1: relaxed arrival checks (tq_take_relaxed)
};
cudaError_t launch_bench(int variant, const BenchParams &p, int blocks, int block, cudaStream_t s);
cudaError_t bench_occupancy(int variant, int block, int *blocks_per_sm);
cudaError_t launch_bench_pipe(int group, int cluster, const BenchParams &p, int blocks, int block,
                              cudaStream_t s);
cudaError_t bench_max_clusters(int cluster, int block, int *clusters);
cudaError_t bench_pipe_occupancy(int block, int *blocks_per_sm);
cudaError_t probe_ceiling(unsigned long long table_bytes, unsigned long long probes, int blocks_per_sm,
                          cudaStream_t s, double *g_per_s);

}  // namespace tqk
