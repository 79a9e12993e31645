/*
 * tq.h -- C ABI of the B200 retry-free / arbitrary-n task queue and the
 * persistent-thread top-down BFS that drives it.
 *
 * Method: Troendle, Ta & Jang, "A Specialized Concurrent Queue for
 * Scheduling Irregular Workloads on GPUs", ICPP 2019.  Citations are to
 * /root/reference/PAPER.md lines (P:<line>) with section / listing.
 *
 * Conventions for every entry point
 *   - Plain C types only; no exception or C++ type crosses the ABI.
 *   - Every function returns a tq_status; TQ_OK (0) on success.  Outputs are
 *     undefined on any non-OK status.
 *   - `stream` arguments are cudaStream_t values passed as void* (NULL = the
 *     legacy default stream).
 *   - Device pointers are CUDA global-memory pointers on the device the object
 *     was created on.  Where an entry point says "host or device", the
 *     library inspects the pointer (cudaPointerGetAttributes) and stages host
 *     buffers through device memory itself.
 *   - Ownership: the caller owns every buffer it passes in (CSR arrays, output
 *     arrays); the library owns the queue storage, the BFS state and scratch,
 *     and frees them in the matching *_destroy.
 */
#ifndef TQ_H_
#define TQ_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    TQ_OK = 0,
    TQ_ERR_INVALID = -1,     /* bad argument (null pointer, range, size)      */
    TQ_ERR_CUDA = -2,        /* a CUDA runtime call failed                    */
    TQ_ERR_NOMEM = -3,       /* device allocation failed                      */
    TQ_ERR_QUEUE_FULL = -4,  /* queue-full exception: the kernel aborted, no
                                retry (P:71 fn2; Listing 3 line 25;
                                P:281 §4.4 "the user can retry the kernel with
                                a larger queue")                              */
    TQ_ERR_TIMEOUT = -5,     /* watchdog expired (protects against hangs)     */
    TQ_ERR_UNSUPPORTED = -6  /* variant / option not available                */
} tq_status;

/* Queue variants (§5.3).  RF_AN is the paper's queue; the others
 * are the comparison designs of the evaluation, built in-repo.              */
typedef enum {
    TQ_VARIANT_RF_AN = 0,          /* retry-free + arbitrary-n: proxy lane, one
                                      64-bit atomicAdd per warp op (P:155,
                                      P:167-171, Listings 1 and 3)           */
    TQ_VARIANT_PER_THREAD_AFA = 1, /* retry-free, no proxy: every lane issues
                                      its own atomicAdd (north-star comparator) */
    TQ_VARIANT_CAS_RETRY = 2,      /* BASE: traditional lock-free CAS queue,
                                      one slot per CAS, retries on CAS failure
                                      and on empty            */
    TQ_VARIANT_AN = 3,             /* AN: BASE + arbitrary-n (proxy CAS loop
                                      reserving n slots)             */
    TQ_VARIANT_ATOMIC_CEILING = 4, /* tq_bench only: proxy atomicAdd on Rear
                                      with no slot traffic -> R_atom          */
    TQ_VARIANT_RF_AN_CTA = 5,      /* tq_bench only: RF/AN with the CTA as the
                                      proxy group (one atomicAdd on Rear and
                                      one on Front per block per iteration;
                                      the abstract's "thread group")   */
    TQ_VARIANT_RF_AN_CLUSTER = 6   /* tq_bench only, pipelined (depth 2): RF/AN
                                      with a thread-block cluster of
                                      cfg.cluster CTAs as the proxy group
                                      (bases broadcast over DSMEM)           */
} tq_variant;

/* ------------------------------------------------------------------------ */
/* Queue object                                                              */
/* ------------------------------------------------------------------------ */

/* A bounded circular array of C = 2^k slots (§3.1, Fig 2) with
 * Front / Rear counters.  Each slot is 8 bytes
 * {item:32 (high) | seq:32 (low)}; seq replaces the data-not-arrived sentinel
 * (§4) and the bounds check of Listing 2: for ticket t the slot
 * is t mod C, seq == (uint32)t means "empty, waiting for ticket t" (dna),
 * seq == (uint32)(t+1) means "item for ticket t has arrived".  Front, Rear
 * and Done are monotonic 64-bit tickets.  Requires 2 <= C <= 2^31. */
typedef struct tq_queue tq_queue;

/* Allocate a queue of at least `capacity` slots (rounded up to a power of
 * two; capacity < 2 or > 2^31 -> TQ_ERR_INVALID) on CUDA device `device`,
 * initialised empty.  *out receives the handle. */
tq_status tq_create(uint64_t capacity, int device, tq_queue **out);

/* Free the queue.  NULL-safe. */
tq_status tq_destroy(tq_queue *q);

/* Reset to the empty state (every slot dna for lap 0, Front = Rear = Done =
 * 0, status running) on `stream`; required after a queue-full abort or a
 * timeout, which can leave slots written but untaken. */
tq_status tq_reset(tq_queue *q, void *stream);

/* Reset to the empty state with the counters at ticket t0 instead of 0:
 * Front = Rear = Done = t0, and every slot holds "empty" for the unique
 * ticket t in [t0, t0 + C) that maps to it (seq == (uint32)t).  Lets a test
 * start a queue just below a 2^32 boundary of the 32-bit sequence tags.
 * t0 < 2^63; stream-ordered like tq_reset. */
tq_status tq_reset_at(tq_queue *q, uint64_t t0, void *stream);

/* Queue status words (replicated; see tq_device.cuh). */
enum { TQ_RUNNING = 0, TQ_FINISHED = 1, TQ_ABORTED_FULL = 2, TQ_ABORTED_TIMEOUT = 3 };

/* Raw device view for user kernels that call the device-side operations in
 * include/tq_device.cuh.  All pointers are device pointers owned by the
 * queue.  `status` points at TQ_STATUS_COPIES replicas spaced 32 words
 * apart. */
typedef struct {
    unsigned long long *slots;  /* C slots                                  */
    unsigned long long *front;  /* Front ticket (dequeue reservations)      */
    unsigned long long *rear;   /* Rear ticket (enqueue reservations)       */
    unsigned long long *done;   /* completed tasks (termination detection)  */
    unsigned int *status;       /* TQ_RUNNING / FINISHED / ABORTED_*        */
    unsigned long long mask;    /* C - 1                                    */
    unsigned int log2_capacity; /* k                                        */
    unsigned int reserved_;
} tq_device_view;

tq_status tq_device_view_get(const tq_queue *q, tq_device_view *out);

/* Host-side copy of the counters (synchronous). */
typedef struct {
    uint64_t front, rear, done;
    uint32_t status;
} tq_counters;
tq_status tq_counters_get(const tq_queue *q, tq_counters *out);

/* ------------------------------------------------------------------------ */
/* Top-down persistent-thread BFS (Algorithm 1; §5.1)        */
/* ------------------------------------------------------------------------ */

/* Undirected graph as a symmetric CSR with ascending rows, no self loops or
 * duplicates (the paper's Nodes[]/Edges[], Listing 2).
 * row_ptr: int64[n_vertices + 1], col: int32[nnz]; 1 <= n_vertices < 2^31.
 * Pointers are host or device (see the entry point). */
typedef struct {
    int64_t n_vertices;
    int64_t nnz;
    const int64_t *row_ptr;
    const int32_t *col;
} tq_csr;

/* Options; a zero-initialised struct selects every default. */
typedef struct {
    uint64_t capacity;  /* queue slots; 0 = 2^ceil(log2(2V)), at least 2^16   */
    int threads;        /* persistent threads; 0 = SMs x occupancy (P:63,
                           P:83 "just enough threads to saturate"), and a
                           BFS plan whose run reached >= 1,024 levels uses
                           one block per SM for its later runs (deep graphs:
                           the too-many-threads side of the dilemma);
                           > 0 = exactly this many (rounded up to blocks)    */
    int block;          /* threads per block; 0 = 256                        */
    int chunk;          /* sub-task size: max edges per task token (P:153
                           "a fixed number of uniformly complex sub-tasks";
                           P:159 fn3).  Vertices with more edges are split
                           into chunk tokens.  0 = 512; power of 2 in
                           [32, 2^16]                                        */
    int variant;        /* tq_variant (RF_AN, PER_THREAD_AFA, CAS_RETRY, AN) */
    void *stream;       /* cudaStream_t                                      */
    double timeout_s;   /* watchdog; 0 = 60 s                                */
    int backoff_ns;     /* max idle back-off per empty work cycle; 0 = the
                           default (none for RF_AN BFS, whose polls are
                           relaxed loads; 256 otherwise), < 0 = none        */
    int device;         /* CUDA device for bfs_plan_create / host-pointer runs;
                           ignored when the CSR is device memory             */
    int parent_rule;    /* TQ_PARENT_ANY (0, default): some neighbour one level
                           up (a valid Graph500 BFS tree; schedule-dependent);
                           TQ_PARENT_MIN_ID (1): the smallest-id neighbour one
                           level up (unique, bit-exact; ~20% slower: level
                           ties must consult the packed word)               */
    int hub_queue;      /* RF_AN: chunk tokens of high-degree vertices go to a
                           second RF/AN queue that lane 0 of every warp polls
                           first (0 = default on, < 0 = off: chunks share the
                           main queue).  Ignored by the other variants.     */
    int debug_delay_ns; /* TEST ONLY (schedule perturbation, SURVEY §8(c)
                           "schedule independence"): the lane holding vertex
                           v sleeps this long before reading v's level when
                           mix(v ^ seed) % 8 == 0, and after reading it when
                           == 1, so tokens are expanded late and with stale
                           levels.  0 = off (default); at most 1,000,000     */
    uint32_t debug_delay_seed;
    int cas_backoff_ns; /* CAS_RETRY / AN only: after a failed CAS, sleep 32 ns
                           doubling up to this many ns before retrying (a
                           bounded exponential back-off); 0 = retry at once
                           (the naive form); 0..1,000,000                   */
    int mirror_bits;    /* level-mirror width (R8): 0 = auto (a nibble
                           per vertex when a byte mirror would exceed 32 MB,
                           RF_AN only; else a byte), 8 = byte, 4 = nibble
                           (RF_AN only, else TQ_ERR_UNSUPPORTED); other
                           values TQ_ERR_INVALID                            */
    int deep_grid;      /* threads == 0 only: 0 = default on (after a run of
                           >= 1,024 levels later runs use one block per SM),
                           < 0 = always the full persistent grid            */
    int ticket_lanes;   /* RF_AN: lanes per warp that hold a main-queue ticket
                           (each holds one DequeueThreadSlotIndex);
                           0 = auto: 32; 2 on graphs below 2^20 CSR entries
                           (consecutive tickets -- a level's consecutive
                           tokens -- then spread over 16x more warps); 8
                           after the plan dropped to the deep-graph grid
                           (see threads); 1..32 = exactly that many; else
                           TQ_ERR_INVALID                                    */
    int l2_persist;     /* 0 = default on: the level mirror is launched with a
                           persisting-L2 access-policy window (the device's
                           persisting limit is raised while any such plan
                           exists, shared by reference count); < 0 = off    */
    int smem_path;      /* RF_AN BFS: 0 = auto (default): a graph whose whole
                           run state -- CSR (32-bit offsets), packed W,
                           expanded-level markers and a ring of 2^ceil(log2
                           (2V)) slots (at least 64, at most `capacity` when
                           set) -- fits in one block's shared memory (<= ~227
                           KB, e.g. config 1's R-MAT scale 10) runs as ONE
                           1024-thread block with the queue in shared memory,
                           graph load and unpack included (DESIGN.md "Small
                           graphs"); < 0 = off (always the global-memory
                           persistent grid); > 0 = required (TQ_ERR_UNSUPPORTED
                           if the graph does not fit or the variant / task is
                           not RF_AN BFS).  threads / ticket_lanes / chunk /
                           hub_queue / mirror_bits do not apply to it       */
    int relabel;        /* BFS on the persistent grid: renumber the vertices by
                           descending degree inside the plan (DESIGN.md
                           "Vertex relabelling"; the top 2^17 ranks dealt over
                           their 128-byte lines) so that the hubs' mirror
                           bytes, W words and markers share sectors.  The plan
                           then owns a relabelled copy of the CSR (4 B per
                           entry + 16 B per vertex; a host-CSR plan keeps only
                           that copy and the original offsets).  Outputs,
                           roots and parent ids stay in the original
                           numbering (min-id parents too).  0 = auto (default):
                           on when some vertex has more than `chunk` edges;
                           < 0 = off; > 0 = on                              */
    int level_bits;     /* TEST ONLY: width cap of the level field that RF/AN
                           BFS tokens carry (R22) -- levels at or
                           beyond 2^level_bits - 1 then travel the fenced
                           path; 0 = every bit the ids leave (default);
                           1..30                                            */
} bfs_opts;

enum { TQ_PARENT_ANY = 0, TQ_PARENT_MIN_ID = 1 };

/* Per-run statistics (device counters, summed over warps). */
typedef struct {
    double ms;                  /* device time: init + persistent + unpack     */
    double ms_kernel;           /* persistent kernel alone                     */
    uint64_t traversed_edges;   /* undirected edges with a reached endpoint     */
    uint64_t reached;           /* vertices with level >= 0                    */
    uint64_t tasks;             /* task tokens processed (vertex + chunk)      */
    uint64_t chunk_tasks;       /* of which chunk tokens                       */
    uint64_t edges_scanned;     /* CSR entries examined                        */
    uint64_t min_atomics;       /* atomicMin issued on W (prefilter passed)    */
    uint64_t reenqueues;        /* vertices re-enqueued after a level decrease */
    uint64_t queue_atomics;     /* atomics on Front/Rear/Done (incl. failed CAS) */
    uint64_t cas_failures;      /* CAS variants only                           */
    uint64_t empty_polls;       /* work cycles that found no data              */
    uint64_t tickets;           /* tasks enqueued (Rear advance)               */
    uint64_t busy_cycles;       /* warp work cycles that processed >= 1 token  */
    uint64_t rounds;            /* 128-edge expansion rounds                   */
    uint64_t skipped_tasks;     /* vertex tokens dropped by the expanded-level
                                   marker (already expanded at <= level)      */
    int32_t max_level;
    int32_t persistent_threads;
    int32_t mirror_bits;        /* level-mirror width of the plan (8 or 4; 0 SSSP) */
    int32_t ticket_lanes;       /* lanes per warp holding main-queue tickets      */
    int32_t smem_path;          /* 1: the run used the shared-memory path         */
    int32_t relabelled;         /* 1: the plan runs on a relabelled copy (opts)   */
    int32_t level_tokens;       /* 1: the run's tokens carried their levels
                                   (R22; a plan whose levels outgrew
                                   the token's level field runs later BFS with
                                   acquire polls instead)                       */
} bfs_stats;

/* Single-source BFS.  level_out[v] = hop distance from root (-1 unreached);
 * parent_out[v] = a neighbour one level closer to the root (the smallest-id
 * one under TQ_PARENT_MIN_ID), parent_out[root] = root, -1 unreached.
 * Either output may be NULL.
 * Graph and outputs: host or device pointers (device pointers must be on the
 * current device).  Synchronous.  Returns TQ_ERR_QUEUE_FULL if the queue
 * overflowed (retry with a larger opts->capacity). */
tq_status bfs_run(const tq_csr *g, int32_t root, int32_t *level_out, int32_t *parent_out);
tq_status bfs_run_ex(const tq_csr *g, int32_t root, int32_t *level_out, int32_t *parent_out,
                     const bfs_opts *opts, bfs_stats *stats);

/* Plans: all application data "must be allocated statically before kernel
 * launch" (§3.1).  A plan holds a device copy / view of the graph, the
 * queue, the per-vertex state W and the chunk table, so that repeated runs
 * (multi-root batches) pay no allocation.  If g's pointers are host memory
 * the plan copies the graph to the device once; device pointers are used in
 * place and must outlive the plan. */
typedef struct bfs_plan bfs_plan;
tq_status bfs_plan_create(const tq_csr *g, const bfs_opts *opts, bfs_plan **out);
/* (The build -- host-CSR upload, chunk table -- runs on an internal stream
 * and is synchronous; runs use opts->stream.  A plan's vertex relabelling
 * (bfs_opts.relabel) is done by its first run, on opts->stream, before the
 * BFS: that first launch is then synchronous, and a plan built while another
 * plan's BFS runs does not relabel beside it.) */
/* level_out / parent_out: DEVICE pointers (or NULL). Stream-ordered on
 * opts->stream, but synchronous (it reads the status word back). */
tq_status bfs_plan_run(bfs_plan *p, int32_t root, int32_t *level_out, int32_t *parent_out,
                       bfs_stats *stats);
/* Asynchronous form: bfs_plan_launch enqueues the run on the plan's stream
 * and returns; bfs_plan_wait blocks until it finished and returns its status
 * (and statistics).  At most one run per plan in flight (TQ_ERR_INVALID
 * otherwise); outputs must be device pointers.  Several plans on different
 * streams run concurrently (multi-root batches). */
tq_status bfs_plan_launch(bfs_plan *p, int32_t root, int32_t *level_out, int32_t *parent_out);
tq_status bfs_plan_wait(bfs_plan *p, bfs_stats *stats);
/* A batch of roots.  Root i writes level_out + i * out_stride and
 * parent_out + i * out_stride (host or device; either may be NULL;
 * out_stride = 0 reuses one buffer, leaving the last root's result).  Host
 * outputs are copied from double-buffered device scratch on a second stream,
 * overlapped with the next root's BFS.  stats: NULL or n_roots entries.
 * Synchronous; stops at the first non-OK root and returns its status. */
tq_status bfs_plan_run_batch(bfs_plan *p, const int32_t *roots, int32_t n_roots,
                             int32_t *level_out, int32_t *parent_out, int64_t out_stride,
                             bfs_stats *stats);
tq_status bfs_plan_destroy(bfs_plan *p);
/* Restart the plan's queues at the given tickets (tq_reset_at on the main
 * queue at t_main and on the chunk queue, if the plan has one, at t_chunk);
 * later runs continue from there.  For tests of the ticket arithmetic across
 * the 2^32 wrap of the 32-bit sequence tags: a benchmark plan reaches ~5e10
 * tickets after 1,600 scale-26 runs.  Not while a run is in flight
 * (TQ_ERR_INVALID); t_main, t_chunk < 2^62. */
tq_status bfs_plan_set_tickets(bfs_plan *p, uint64_t t_main, uint64_t t_chunk);
/* Current tickets (the main queue's Rear where the next run starts, and the
 * chunk queue's), for the same tests. */
tq_status bfs_plan_get_tickets(const bfs_plan *p, uint64_t *t_main, uint64_t *t_chunk);

/* ------------------------------------------------------------------------ */
/* The queue as a generic scheduler (NEXT row 4; "it can be used for    */
/* other purposes with little change"): label-correcting single-source      */
/* shortest paths on the same persistent kernel, queues and termination.    */
/* ------------------------------------------------------------------------ */

/* weights: int32[nnz], one per CSR entry, each >= 1 (host or device, like the
 * CSR; paths must sum below 2^32 - 1).  dist_out[v] = shortest distance
 * (0xFFFFFFFF unreached); parent_out[v] = the smallest-id u with
 * dist[u] + w(u->v) == dist[v] (parent_out[src] = src, -1 unreached).  RF_AN
 * only (opts->variant must be 0); parent_rule is always min-id.  The plan
 * is destroyed with bfs_plan_destroy. */
tq_status sssp_plan_create(const tq_csr *g, const int32_t *weights, const bfs_opts *opts,
                           bfs_plan **out);
tq_status sssp_plan_run(bfs_plan *p, int32_t src, uint32_t *dist_out, int32_t *parent_out,
                        bfs_stats *stats);
tq_status sssp_run_ex(const tq_csr *g, const int32_t *weights, int32_t src, uint32_t *dist_out,
                      int32_t *parent_out, const bfs_opts *opts, bfs_stats *stats);

/* ------------------------------------------------------------------------ */
/* Queue micro-benchmark (BASELINE.json configs[1]; Fig 4 / Fig 5 analogue)  */
/* ------------------------------------------------------------------------ */

typedef struct {
    int variant;        /* tq_variant                                         */
    int warps;          /* persistent warps; 0 = SMs x occupancy              */
    int batch;          /* items per warp operation b, 1..32                 */
    uint64_t items;     /* total items N (rounded down to warps*batch*iters)  */
    uint64_t capacity;  /* queue slots                                        */
    int work_iters;     /* synthetic ALU work per consumed item               */
    uint64_t seed;      /* item ids = item_of(seed, g) (inputs/items.py)      */
    int log_mode;       /* 1: record ticket -> item logs (enq_log/deq_log)    */
    uint32_t *enq_log;  /* device uint32[items] or NULL                       */
    uint32_t *deq_log;  /* device uint32[items] or NULL                       */
    void *stream;
    double timeout_s;   /* 0 = 60 s                                           */
    int device;
    int depth;          /* 0/1: per iteration reserve Rear, publish, reserve
                           Front, poll (the paper's order).  2: pipelined --
                           the proxy reserves iteration k+1's Rear and Front
                           tickets at the start of iteration k and publishes
                           k+1's items after k's poll (<= 2b items in flight
                           per warp; RF_AN_CTA and RF_AN_CLUSTER only, else
                           TQ_ERR_UNSUPPORTED)                               */
    int cluster;        /* RF_AN_CLUSTER: CTAs per cluster (0 = 4; 1..16);
                           warps must be a multiple of 8*cluster and fit the
                           co-resident cluster count, else TQ_ERR_INVALID    */
    int cas_backoff_ns; /* CAS_RETRY / AN: bounded exponential back-off after
                           a failed CAS (32 ns doubling up to this); 0 =
                           none (the naive form); 0..1,000,000              */
    int relaxed_poll;   /* 1: the arrival check is a relaxed load and the
                           acquire is skipped (the benchmark's items carry
                           their whole payload, so nothing else must become
                           visible); 0 = acquire load per poll (tq_take)    */
} tq_bench_cfg;

typedef struct {
    double ms;
    uint64_t items;           /* items actually pushed through                */
    uint64_t enq, deq;        /* successful enqueues / dequeues               */
    uint64_t atomics;         /* global atomics on Front/Rear (incl. failed CAS) */
    uint64_t cas_failures;
    uint64_t empty_retries;   /* polls / dequeue attempts that found no data  */
    uint64_t sum_enq, sum_deq, xor_enq, xor_deq; /* fingerprints of splitmix64(item) */
    int32_t warps;
    tq_status status;
} tq_bench_result;

tq_status tq_bench(const tq_bench_cfg *cfg, tq_bench_result *res);

/* ------------------------------------------------------------------------ */
/* Misc                                                                      */
/* ------------------------------------------------------------------------ */
const char *tq_strerror(tq_status s);
/* Occupancy-derived persistent thread count for the BFS kernel of `variant`
 * with `block` threads per block on `device`. */
tq_status tq_persistent_threads(int variant, int block, int device, int *threads_out);
/* Library version string. */
const char *tq_version(void);
/* Device memory of queues and plans is drawn from a library-owned
 * stream-ordered pool per device that keeps freed memory reserved, so a plan
 * created right after another one of the same size (e.g. every step of a
 * benchmark that rebuilds it from a host CSR) reuses it without cudaMalloc /
 * cudaFree.  tq_memory_trim releases the cached, unused part of `device`'s
 * pool to the driver (memory of live queues and plans stays).  Synchronises
 * the device.  TQ_OK also when the pool was never created. */
tq_status tq_memory_trim(int device);
/* sizeof() of a public struct by name ("tq_csr", "bfs_opts", "bfs_stats",
 * "tq_device_view", "tq_counters", "tq_bench_cfg", "tq_bench_result"), 0 for
 * an unknown name: lets bindings check their struct mirrors without a GPU. */
size_t tq_struct_size(const char *name);

/* Measurement utility (the roofline of the BFS
 * expansion): the random-probe ceiling of this GPU.  Streams `probes` 4-byte
 * indices (uniform random over [0, table_bytes), generated on the device) and
 * reads one byte of a table_bytes-long table per index with ld.global.cg (L2),
 * 4 probes in flight per lane, at the BFS kernel's shape (256-thread blocks,
 * its occupancy): the access pattern of the expansion's level-mirror probes
 * (one random 32-byte sector per CSR entry).  *g_per_s = probes per second /
 * 1e9 of the second of two launches (CUDA events on `stream`).  Allocates and
 * frees its own device memory.  table_bytes in [2^12, 2^32), probes in
 * [2^20, 2^32); TQ_ERR_INVALID otherwise.  Synchronous. */
tq_status tq_probe_ceiling(int device, uint64_t table_bytes, uint64_t probes, void *stream,
                           double *g_per_s);

#ifdef __cplusplus
}
#endif
#endif /* TQ_H_ */
