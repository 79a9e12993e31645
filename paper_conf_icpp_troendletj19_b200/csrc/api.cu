// api.cu -- implementation of the C ABI declared in include/tq.h.
//
// Host-side runtime around the kernels: queue objects (static allocation
// before launch, §3.1), BFS plans, pointer staging for host buffers,
// persistent-grid sizing from the occupancy API, event timing,
// status read-back (queue-full abort -> TQ_ERR_QUEUE_FULL) and the
// queue micro-benchmark driver.
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

#include <mutex>
#include <new>

#include "internal.cuh"

using namespace tqk;

namespace tqk {

static cudaMemPool_t g_pools[256];
static std::mutex g_pool_mu;

static cudaMemPool_t lib_pool(int dev, bool create)
{
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (dev < 0 || dev >= 256) return nullptr;
    if (!g_pools[dev] && create) {
        cudaMemPoolProps props{};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t pool = nullptr;
        if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        unsigned long long keep = ~0ull;  // keep freed memory for the next plan
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
        g_pools[dev] = pool;
    }
    return g_pools[dev];
}

cudaError_t pool_alloc_raw(void **p, size_t bytes, cudaStream_t s)
{
    *p = nullptr;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    cudaMemPool_t pool = lib_pool(dev, true);
    if (!pool) return cudaErrorMemoryAllocation;
    e = cudaMallocFromPoolAsync(p, bytes > 0 ? bytes : 1, pool, s);
    if (e == cudaErrorMemoryAllocation) {  // give cached blocks back, retry once
        cudaGetLastError();
        cudaStreamSynchronize(s);
        cudaMemPoolTrimTo(pool, 0);
        e = cudaMallocFromPoolAsync(p, bytes > 0 ? bytes : 1, pool, s);
    }
    return e;
}

void pool_free(void *p, cudaStream_t s)
{
    if (p) cudaFreeAsync(p, s);
}

// Small pinned host buffers (a plan's statistics / counter read-back) are
// recycled through a free list: cudaFreeHost can wait for the whole device,
// which made plan teardown take up to 0.5 s in the e2e leg.
static std::mutex g_pin_mu;
static void *g_pin_free[64];
static int g_pin_n = 0;
static constexpr size_t kPinBytes = 256;  // >= kStatCount and 8 counters of 8 bytes

static cudaError_t pinned_small_alloc(void **p)
{
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        if (g_pin_n > 0) {
            *p = g_pin_free[--g_pin_n];
            return cudaSuccess;
        }
    }
    return cudaMallocHost(p, kPinBytes);
}

static void pinned_small_free(void *p)
{
    if (!p) return;
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        if (g_pin_n < 64) {
            g_pin_free[g_pin_n++] = p;
            return;
        }
    }
    cudaFreeHost(p);
}

}  // namespace tqk

#define TQ_VERSION_STRING "tq-b200 0.1 (sm_100a)"

namespace {

struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev)
    {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (dev >= 0 && dev != prev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard()
    {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

tq_status from_cuda(cudaError_t e)
{
    if (e == cudaSuccess) return TQ_OK;
    cudaGetLastError();  // clear sticky-free errors
    if (e == cudaErrorMemoryAllocation) return TQ_ERR_NOMEM;
    return TQ_ERR_CUDA;
}

#define CK(call)                                        \
    do {                                                \
        cudaError_t e_ = (call);                        \
        if (e_ != cudaSuccess) return from_cuda(e_);    \
    } while (0)

// Returns 1 for device (or managed) memory, 0 for host memory (pageable or
// pinned), -1 when the pointer cannot be classified (the query failed: the
// entry points then return TQ_ERR_INVALID instead of guessing).
int is_device_ptr(const void *p, int *device)
{
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) {
        if (device) *device = a.device;
        return 1;
    }
    return 0;
}

// Device -> host copy in 8 MiB pieces.  Measured on the B200 boxes
// (scripts/overlap_probe.cu): while ONE large D2H copy is in flight, a
// multi-CTA kernel launched after it does not start until the copy ends
// (a 512 MiB copy delays the next BFS by ~10 ms); split into 8 MiB copies
// the kernel starts at once and the copy still runs at ~52 GB/s.
static cudaError_t d2h_chunked(void *dst, const void *src, size_t bytes, cudaStream_t s)
{
    const size_t piece = 8ull << 20;
    for (size_t off = 0; off < bytes; off += piece) {
        const size_t nb = bytes - off < piece ? bytes - off : piece;
        cudaError_t e = cudaMemcpyAsync((char *)dst + off, (const char *)src + off, nb,
                                        cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

// Persisting-L2 carve-out: the limit is device-wide, the windows are per
// launch.  Plans on one device share it through a reference count, so
// destroying one plan never resets the persisting lines of another plan that
// is still running (e.g. run_concurrent); the limit is raised by the first
// plan that needs it and restored, and the persisting lines reset, when the
// last plan on the device is destroyed.
struct L2Persist {
    int refs = 0;
    size_t saved = 0;   // device limit before the first plan raised it
    size_t cur = 0;     // limit now
    bool raised = false;
};
static L2Persist g_l2[256];
static std::mutex g_l2_mu;

// Returns the window size to use for `want` bytes (0 = no window); every
// non-zero return must be paired with one l2_persist_release(dev).
size_t l2_persist_acquire(int dev, size_t want)
{
    std::lock_guard<std::mutex> lk(g_l2_mu);
    if (dev < 0 || dev >= 256 || want == 0) return 0;
    int max_win = 0, max_persist = 0;
    cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, dev);
    size_t w = want;
    if (w > (size_t)max_win) w = (size_t)max_win;
    if (w > (size_t)max_persist) w = (size_t)max_persist;
    if (w == 0) {
        cudaGetLastError();
        return 0;
    }
    L2Persist &e = g_l2[dev];
    if (e.refs == 0) {
        size_t cur = 0;
        if (cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) != cudaSuccess) {
            cudaGetLastError();
            return 0;
        }
        e.saved = e.cur = cur;
        e.raised = false;
    }
    if (e.cur < w) {
        if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, w) == cudaSuccess) {
            e.cur = w;
            e.raised = true;
        } else {
            cudaGetLastError();
        }
    }
    ++e.refs;
    return w;
}

void l2_persist_release(int dev)
{
    std::lock_guard<std::mutex> lk(g_l2_mu);
    if (dev < 0 || dev >= 256) return;
    L2Persist &e = g_l2[dev];
    if (e.refs <= 0) return;
    if (--e.refs == 0) {
        cudaCtxResetPersistingL2Cache();
        if (e.raised) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, e.saved);
        e.raised = false;
        cudaGetLastError();
    }
}

// Host -> device copy in 1 MiB pieces, for the same reason as d2h_chunked:
// a plan built from a host CSR while another plan's BFS runs (bench.py's e2e
// leg builds step k+1's plan during step k) must not hold back that BFS's
// kernel launches behind a long copy.  Measured (kron26 e2e step, 9 GB H2D
// beside 64 BFS): 64 / 16 / 4 / 2 / 1 / 0.5 MiB pieces -> 1.23 / 1.23 / 1.165 /
// 1.123 / 1.103 / 1.100 s per step (device-only 1.06 s).
static cudaError_t h2d_chunked(void *dst, const void *src, size_t bytes, cudaStream_t s)
{
    const size_t piece = 1ull << 20;
    for (size_t off = 0; off < bytes; off += piece) {
        const size_t nb = bytes - off < piece ? bytes - off : piece;
        cudaError_t e = cudaMemcpyAsync((char *)dst + off, (const char *)src + off, nb,
                                        cudaMemcpyHostToDevice, s);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

uint64_t next_pow2(uint64_t x)
{
    uint64_t c = 1;
    while (c < x) c <<= 1;
    return c;
}

int sm_count(int dev)
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms > 0 ? sms : 1;
}

// counter block layout (bytes): Front, Rear, Done 4 KiB apart (separate L2
// lines and slices); status replicas 128 B apart after them.
constexpr size_t kOffFront = 0, kOffRear = 4096, kOffDone = 8192, kOffStatus = 12288;
constexpr size_t kCtrBytes = kOffStatus + TQ_STATUS_COPIES * TQ_STATUS_STRIDE * sizeof(unsigned);

}  // namespace

struct tq_queue {
    int device = 0;
    cudaStream_t stream = nullptr;      // creation / free stream (legacy default for tq_create)
    uint64_t cap = 0;
    unsigned log2cap = 0;
    unsigned long long *slots = nullptr;
    char *ctr = nullptr;
    tq_device_view view{};
};

// Device output buffers of bfs_plan_run_batch with host outputs: a root's
// D2H copy may take longer than the next root's BFS while both run (the host
// link is shared with the kernel's traffic), so a ring of three lets the
// copies fall two roots behind before a BFS has to wait for a free buffer.
constexpr int kOutBufs = 3;

struct bfs_plan {
    int device = 0;
    cudaStream_t stream = nullptr;
    int variant = 0, block = 256, blocks = 0, chunk = 256, backoff_ns = 256, parent_rule = 0;
    double timeout_s = 60.0;
    int64_t n = 0, nnz = 0;
    int64_t *row_ptr = nullptr;
    int32_t *col = nullptr;
    bool owns_graph = false;
    unsigned long long *W = nullptr;
    int32_t *hub_base = nullptr;
    unsigned *mir = nullptr;                  // level mirror (bytes or nibbles)
    int mirror_bits = 8;
    bool auto_blocks = false;                 // threads == 0: full grid, one block per SM on deep graphs
    size_t mirror_bytes = 0;
    uint8_t *x8 = nullptr;
    unsigned *xd = nullptr;                   // SSSP: expanded-distance marker
    int32_t *wgt = nullptr;                   // SSSP: edge weights (device)
    bool owns_wgt = false;
    int task = 0;                             // kTaskBFS / kTaskSSSP
    int2 *chunk_tab = nullptr;
    int64_t n_chunks = 0;
    tq_queue *q = nullptr;
    tq_queue *q1 = nullptr;                   // chunk queue (RF/AN hub sub-tasks)
    bool hub_queue = false;
    unsigned long long next_ticket1 = 0;
    unsigned long long *stats = nullptr;      // device, kStatCount
    unsigned long long *stats_h = nullptr;    // pinned
    unsigned long long *ctr_h = nullptr;      // pinned: front, rear, done, rear1, status
    bool in_flight = false;                   // launched, not yet waited for
    int32_t *dbuf[kOutBufs] = {};             // batch: device output buffers (ring)
    cudaStream_t copy_stream = nullptr;       // batch: D2H copies
    cudaEvent_t bfs_done[kOutBufs] = {}, copy_done[kOutBufs] = {};
    size_t l2_window = 0;                     // persisting-L2 window over the level mirror
    unsigned long long next_ticket = 0;
    bool dirty = false;
    int32_t *out_scratch = nullptr;           // for host outputs
    int cas_backoff_ns = 0;                   // CAS variants: bounded back-off (bfs_opts)
    int ticket_lanes = 32;                    // RF/AN: lanes per warp holding main-queue tickets
    bool auto_lanes = false;                  // ticket_lanes chosen by the plan (bfs_opts.ticket_lanes == 0)
    int delay_ns = 0;                         // test only (bfs_opts.debug_delay_ns)
    uint32_t delay_seed = 0;
    bool smem = false;                        // runs on the shared-memory path (bfs_small.cu)
    // vertex relabelling (relabel.cu): row_ptr / col are then the plan-owned
    // relabelled CSR and row_ptr0 the original offsets (owned if owns_graph)
    bool relabelled = false;
    bool relabel_pending = false;             // relabel at the first run (plan_relabel)
    int relabel_min_deg = 0;
    int64_t hub_region = 0;
    bool lit = true;                          // BFS tokens carry their level (bfs.cu, R22)
    int level_bits = 0;                       // test-only cap of the level field (bfs_opts.level_bits)
    unsigned lit_field = 0;                   // the largest level both token kinds can carry
    int32_t *new2old = nullptr, *old2new = nullptr;
    int64_t *row_ptr0 = nullptr;
    unsigned smem_cap = 0;                    // its ring slots
    cudaEvent_t ev[4] = {nullptr, nullptr, nullptr, nullptr};
};

extern "C" {

const char *tq_version(void) { return TQ_VERSION_STRING; }

size_t tq_struct_size(const char *name)
{
    if (!name) return 0;
    if (!strcmp(name, "tq_csr")) return sizeof(tq_csr);
    if (!strcmp(name, "bfs_opts")) return sizeof(bfs_opts);
    if (!strcmp(name, "bfs_stats")) return sizeof(bfs_stats);
    if (!strcmp(name, "tq_device_view")) return sizeof(tq_device_view);
    if (!strcmp(name, "tq_counters")) return sizeof(tq_counters);
    if (!strcmp(name, "tq_bench_cfg")) return sizeof(tq_bench_cfg);
    if (!strcmp(name, "tq_bench_result")) return sizeof(tq_bench_result);
    return 0;
}

tq_status tq_memory_trim(int device)
{
    DeviceGuard g(device);
    if (!g.ok) return TQ_ERR_INVALID;
    cudaMemPool_t pool = lib_pool(device, false);
    if (!pool) return TQ_OK;
    CK(cudaDeviceSynchronize());
    CK(cudaMemPoolTrimTo(pool, 0));
    return TQ_OK;
}

const char *tq_strerror(tq_status s)
{
    switch (s) {
    case TQ_OK: return "ok";
    case TQ_ERR_INVALID: return "invalid argument";
    case TQ_ERR_CUDA: return "CUDA error";
    case TQ_ERR_NOMEM: return "out of device memory";
    case TQ_ERR_QUEUE_FULL: return "queue full: kernel aborted (retry with a larger queue)";
    case TQ_ERR_TIMEOUT: return "watchdog timeout";
    case TQ_ERR_UNSUPPORTED: return "unsupported";
    default: return "unknown status";
    }
}

// ------------------------------------------------------------------------
// queue objects
// ------------------------------------------------------------------------
// Queue creation / destruction on a given stream: the public entry points use
// the legacy default stream and synchronise the device; a plan uses its own
// stream and synchronises only that, so a plan built while another plan's BFS
// runs (bench.py's e2e leg) neither waits for nor serialises with that BFS.
static tq_status queue_create_on(uint64_t capacity, int device, cudaStream_t s, bool device_sync,
                                 tq_queue **out)
{
    if (!out) return TQ_ERR_INVALID;
    *out = nullptr;
    if (capacity < 2 || capacity > (1ull << 31)) return TQ_ERR_INVALID;
    DeviceGuard g(device);
    if (!g.ok) return TQ_ERR_INVALID;
    tq_queue *q = new (std::nothrow) tq_queue;
    if (!q) return TQ_ERR_NOMEM;
    q->device = device;
    q->stream = s;
    q->cap = next_pow2(capacity);
    while ((1ull << q->log2cap) < q->cap) ++q->log2cap;
    cudaError_t e = pool_alloc(&q->slots, q->cap * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = pool_alloc(&q->ctr, kCtrBytes, s);
    if (e != cudaSuccess) {
        pool_free(q->slots, s);
        pool_free(q->ctr, s);
        device_sync ? cudaDeviceSynchronize() : cudaStreamSynchronize(s);
        delete q;
        return from_cuda(e);
    }
    q->view.slots = q->slots;
    q->view.front = (unsigned long long *)(q->ctr + kOffFront);
    q->view.rear = (unsigned long long *)(q->ctr + kOffRear);
    q->view.done = (unsigned long long *)(q->ctr + kOffDone);
    q->view.status = (unsigned *)(q->ctr + kOffStatus);
    q->view.mask = q->cap - 1;
    q->view.log2_capacity = q->log2cap;
    tq_status st = tq_reset(q, s);
    if (st == TQ_OK) st = from_cuda(device_sync ? cudaDeviceSynchronize() : cudaStreamSynchronize(s));
    if (st != TQ_OK) {
        tq_destroy(q);
        return st;
    }
    *out = q;
    return TQ_OK;
}

tq_status tq_create(uint64_t capacity, int device, tq_queue **out)
{
    return queue_create_on(capacity, device, nullptr, true, out);
}

tq_status tq_destroy(tq_queue *q)
{
    if (!q) return TQ_OK;
    DeviceGuard g(q->device);
    // callers have finished with the queue (plans synchronise first); the
    // frees are ordered on the stream the queue was created on
    pool_free(q->slots, q->stream);
    pool_free(q->ctr, q->stream);
    delete q;
    return TQ_OK;
}

tq_status tq_reset_at(tq_queue *q, uint64_t t0, void *stream)
{
    if (!q || t0 >= (1ull << 63)) return TQ_ERR_INVALID;
    DeviceGuard g(q->device);
    CK(cudaMemsetAsync(q->ctr, 0, kCtrBytes, (cudaStream_t)stream));
    CK(launch_queue_reset(q->view, t0, (cudaStream_t)stream));
    return TQ_OK;
}

tq_status tq_reset(tq_queue *q, void *stream) { return tq_reset_at(q, 0, stream); }

tq_status tq_device_view_get(const tq_queue *q, tq_device_view *out)
{
    if (!q || !out) return TQ_ERR_INVALID;
    *out = q->view;
    return TQ_OK;
}

tq_status tq_counters_get(const tq_queue *q, tq_counters *out)
{
    if (!q || !out) return TQ_ERR_INVALID;
    DeviceGuard g(q->device);
    unsigned long long f = 0, r = 0, d = 0;
    unsigned s = 0;
    CK(cudaMemcpy(&f, q->view.front, 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&r, q->view.rear, 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&d, q->view.done, 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(&s, q->view.status, 4, cudaMemcpyDeviceToHost));
    out->front = f;
    out->rear = r;
    out->done = d;
    out->status = s;
    return TQ_OK;
}

tq_status tq_persistent_threads(int variant, int block, int device, int *threads_out)
{
    if (!threads_out) return TQ_ERR_INVALID;
    if (block == 0) block = 256;
    DeviceGuard g(device);
    int per_sm = 0;
    if (bfs_occupancy(variant, block, &per_sm) != cudaSuccess) {
        cudaGetLastError();
        return TQ_ERR_INVALID;
    }
    *threads_out = per_sm * sm_count(device) * block;
    return TQ_OK;
}

// ------------------------------------------------------------------------
// BFS plans
// ------------------------------------------------------------------------
tq_status bfs_plan_destroy(bfs_plan *p)
{
    if (!p) return TQ_OK;
    DeviceGuard g(p->device);
    if (p->stream) cudaStreamSynchronize(p->stream);
    for (auto &e : p->ev)
        if (e) cudaEventDestroy(e);
    if (p->copy_stream) cudaStreamSynchronize(p->copy_stream);
    // stream-ordered frees after everything that used the memory has finished
    cudaStream_t fs = p->stream;
    if (p->relabelled) {
        pool_free(p->row_ptr, fs);  // the relabelled CSR (plan-owned)
        pool_free(p->col, fs);
        pool_free(p->new2old, fs);
        pool_free(p->old2new, fs);
        if (p->owns_graph) pool_free(p->row_ptr0, fs);  // (the original col was freed at create)
    } else if (p->owns_graph) {
        pool_free(p->row_ptr, fs);
        pool_free(p->col, fs);
    }
    pool_free(p->W, fs);
    pool_free(p->hub_base, fs);
    pool_free(p->mir, fs);
    pool_free(p->x8, fs);
    pool_free(p->xd, fs);
    if (p->owns_wgt) pool_free(p->wgt, fs);
    pool_free(p->chunk_tab, fs);
    pool_free(p->stats, fs);
    pool_free(p->out_scratch, fs);
    for (int b = 0; b < kOutBufs; ++b) {
        pool_free(p->dbuf[b], fs);
        if (p->bfs_done[b]) cudaEventDestroy(p->bfs_done[b]);
        if (p->copy_done[b]) cudaEventDestroy(p->copy_done[b]);
    }
    if (p->copy_stream) cudaStreamDestroy(p->copy_stream);
    pinned_small_free(p->stats_h);
    pinned_small_free(p->ctr_h);
    if (p->l2_window) l2_persist_release(p->device);
    tq_destroy(p->q);
    tq_destroy(p->q1);
    delete p;
    return TQ_OK;
}

static tq_status plan_create_impl(const tq_csr *gph, const int32_t *weights, int task,
                                  const bfs_opts *opts, bfs_plan **out)
{
    if (!gph || !out) return TQ_ERR_INVALID;
    *out = nullptr;
    bfs_opts o;
    memset(&o, 0, sizeof(o));
    if (opts) o = *opts;
    const int64_t n = gph->n_vertices, nnz = gph->nnz;
    if (n < 1 || n >= (1ll << 31) || nnz < 0 || !gph->row_ptr || (nnz > 0 && !gph->col))
        return TQ_ERR_INVALID;
    if (o.variant < TQ_VARIANT_RF_AN || o.variant > TQ_VARIANT_AN) return TQ_ERR_UNSUPPORTED;
    if (task == kTaskSSSP && o.variant != TQ_VARIANT_RF_AN) return TQ_ERR_UNSUPPORTED;
    if (task == kTaskSSSP && nnz > 0 && !weights) return TQ_ERR_INVALID;
    // (default chunk 512: 1,024 looked 5% faster on 4 kron26 roots but is 6%
    // slower over the bench's 64, and 20% slower on kron24;
    // results/level_tokens_r02.log)
    int chunk = o.chunk ? o.chunk : 512;
    if (chunk < 32 || chunk > 65536 || (chunk & (chunk - 1))) return TQ_ERR_INVALID;
    const int block = o.block ? o.block : 256;
    if (block != 256) return TQ_ERR_UNSUPPORTED;

    int gdev = o.device;
    const int dev_graph = is_device_ptr(gph->row_ptr, &gdev);
    if (dev_graph < 0) return TQ_ERR_INVALID;
    if (nnz > 0 && is_device_ptr(gph->col, nullptr) != dev_graph) return TQ_ERR_INVALID;  // same kind
    if (o.mirror_bits != 0 && o.mirror_bits != 4 && o.mirror_bits != 8) return TQ_ERR_INVALID;
    DeviceGuard g(gdev);
    if (!g.ok) return TQ_ERR_INVALID;

    bfs_plan *p = new (std::nothrow) bfs_plan;
    if (!p) return TQ_ERR_NOMEM;
    p->device = gdev;
    p->stream = (cudaStream_t)o.stream;
    p->variant = o.variant;
    p->block = block;
    p->chunk = chunk;
    // default idle back-off: none for RF/AN BFS (its polls are relaxed loads,
    // R22, cheap to repeat; measured -2.8% / -1.4% on kron24 / kron26 within
    // one process, within +-0.5% across processes: results/level_tokens_r02.log),
    // 256 ns for the rest
    const int bo_default = (o.variant == TQ_VARIANT_RF_AN && task == kTaskBFS) ? 0 : 256;
    p->backoff_ns = o.backoff_ns == 0 ? bo_default : (o.backoff_ns < 0 ? 0 : o.backoff_ns);
    p->timeout_s = o.timeout_s > 0 ? o.timeout_s : 60.0;
    if (o.parent_rule != TQ_PARENT_MIN_ID && o.parent_rule != TQ_PARENT_ANY) {
        delete p;
        return TQ_ERR_INVALID;
    }
    p->parent_rule = task == kTaskSSSP ? TQ_PARENT_MIN_ID : o.parent_rule;
    if (o.debug_delay_ns < 0 || o.debug_delay_ns > 1000000) {
        delete p;
        return TQ_ERR_INVALID;
    }
    if (o.cas_backoff_ns < 0 || o.cas_backoff_ns > 1000000) {
        delete p;
        return TQ_ERR_INVALID;
    }
    p->cas_backoff_ns = o.cas_backoff_ns;
    if (o.level_bits < 0 || o.level_bits > 30) {
        delete p;
        return TQ_ERR_INVALID;
    }
    p->level_bits = o.level_bits;
    p->delay_ns = o.debug_delay_ns;
    p->delay_seed = o.debug_delay_seed;
    p->task = task;
    p->n = n;
    p->nnz = nnz;

    bool smem_auto_lanes = false;
    // The plan's build work (graph upload, chunk table) runs on an internal
    // stream of the device's lowest priority, apart from the caller's stream
    // (bench.py's e2e leg builds step k+1's plan during step k's BFS); the
    // relabelling waits for the plan's first run (plan_relabel).
    cudaStream_t bs = nullptr;
    {
        int least = 0, greatest = 0;
        cudaDeviceGetStreamPriorityRange(&least, &greatest);
        if (cudaStreamCreateWithPriority(&bs, cudaStreamNonBlocking, least) != cudaSuccess) {
            delete p;
            return TQ_ERR_CUDA;
        }
    }
    auto fail = [&](tq_status s) {
        cudaStreamSynchronize(bs);
        cudaStreamDestroy(bs);
        bfs_plan_destroy(p);
        return s;
    };
    cudaError_t e;
    if (dev_graph) {
        p->row_ptr = const_cast<int64_t *>(gph->row_ptr);
        p->col = const_cast<int32_t *>(gph->col);
    } else {
        p->owns_graph = true;
        e = pool_alloc(&p->row_ptr, (size_t)(n + 1) * sizeof(int64_t), bs);
        if (e == cudaSuccess) e = pool_alloc(&p->col, (size_t)(nnz > 0 ? nnz : 1) * sizeof(int32_t), bs);
        if (e == cudaSuccess) e = h2d_chunked(p->row_ptr, gph->row_ptr, (size_t)(n + 1) * sizeof(int64_t), bs);
        if (e == cudaSuccess && nnz > 0) e = h2d_chunked(p->col, gph->col, (size_t)nnz * sizeof(int32_t), bs);
        if (e != cudaSuccess) return fail(from_cuda(e));
    }
    if (task == kTaskSSSP && nnz > 0) {
        const int wdev = is_device_ptr(weights, nullptr);
        if (wdev < 0) return fail(TQ_ERR_INVALID);
        if (wdev) {
            p->wgt = const_cast<int32_t *>(weights);
        } else {
            p->owns_wgt = true;
            e = pool_alloc(&p->wgt, (size_t)nnz * sizeof(int32_t), bs);
            if (e == cudaSuccess)
                e = cudaMemcpyAsync(p->wgt, weights, (size_t)nnz * sizeof(int32_t), cudaMemcpyHostToDevice,
                                    bs);
            if (e != cudaSuccess) return fail(from_cuda(e));
        }
    }
    e = pinned_small_alloc(reinterpret_cast<void **>(&p->stats_h));
    if (e == cudaSuccess) e = pinned_small_alloc(reinterpret_cast<void **>(&p->ctr_h));
    if (e != cudaSuccess) return fail(from_cuda(e));
    // Shared-memory path (bfs_opts.smem_path): the
    // whole run in one block when CSR + W + markers + a ring of 2V slots fit
    {
        // (its packed 32-bit W holds 16-bit vertex ids)
        const bool eligible = task == kTaskBFS && p->variant == TQ_VARIANT_RF_AN && n <= 65535;
        uint64_t scap = o.capacity ? next_pow2(o.capacity) : next_pow2((uint64_t)(2 * n));
        if (scap < 64 && !o.capacity) scap = 64;
        if (scap < 2) scap = 2;
        const bool fits = eligible && small_smem_bytes(n, nnz, scap) <= small_smem_limit(gdev);
        if (o.smem_path > 0 && !fits) return fail(TQ_ERR_UNSUPPORTED);
        if (o.smem_path >= 0 && fits) {
            p->smem = true;
            p->smem_cap = (unsigned)scap;
            smem_auto_lanes = true;  // (ticket lanes below)
        }
    }
    // Vertex relabelling (bfs_opts.relabel, relabel.cu): BFS on the persistent
    // grid, auto when a vertex has more than `chunk` edges (a degree-skewed
    // graph; a uniform graph such as the grid keeps its own numbering).  Done
    // at the plan's first run, on its own stream (plan_relabel): a plan built
    // while another plan's BFS runs -- bench.py's e2e leg builds step k+1's
    // plan during step k -- would otherwise relabel beside that BFS and slow
    // it far more than the relabelling's own ~25 ms (results/e2e_relabel_r02.log).
    if (task == kTaskBFS && !p->smem && o.relabel >= 0 && n < (1ll << 31) - 1) {
        p->relabel_pending = true;
        p->relabel_min_deg = o.relabel > 0 ? -1 : chunk;
        // hub region (ranks dealt over their lines): 2^14 where the byte
        // mirror's probes are L1-cached (bfs.cu), so the top hubs' bytes stay
        // within the L1; 2^20 for the nibble mirror (results/relabel_r02.log,
        // results/level_tokens_r02.log)
        const bool byte_mirror = !(p->variant == TQ_VARIANT_RF_AN && n > (1ll << 25)) || o.mirror_bits == 8;
        p->hub_region = (byte_mirror && o.mirror_bits != 4) ? (1ll << 14) : (1ll << 20);
    }
    e = pool_alloc(&p->W, (size_t)n * sizeof(unsigned long long), bs);
    if (e == cudaSuccess) e = pool_alloc(&p->hub_base, (size_t)n * sizeof(int32_t), bs);
    if (task == kTaskBFS) {
        // Level mirror width (R8): a nibble per vertex when a byte
        // mirror would exceed 32 MB (it then no longer stays L2-resident next
        // to the col stream; measured: s26 -3.6%, s24 / grid +2-4% with
        // nibbles), RF/AN only.  bfs_opts.mirror_bits overrides.
        p->mirror_bits = (o.variant == TQ_VARIANT_RF_AN && n > (1ll << 25)) ? 4 : 8;
        if (o.mirror_bits == 4 || o.mirror_bits == 8) p->mirror_bits = o.mirror_bits;
        if (p->mirror_bits == 4 && o.variant != TQ_VARIANT_RF_AN) return fail(TQ_ERR_UNSUPPORTED);
        p->mirror_bytes = p->mirror_bits == 8 ? (size_t)n : (size_t)(n + 7) / 8 * 4;
        if (e == cudaSuccess) e = pool_alloc(&p->mir, p->mirror_bytes, bs);
        // expanded-level markers: same width as the mirror
        if (e == cudaSuccess)
            e = pool_alloc(&p->x8, p->mirror_bits == 8 ? (size_t)n : (size_t)(n + 1) / 2, bs);
    } else {
        if (e == cudaSuccess) e = pool_alloc(&p->xd, (size_t)n * sizeof(unsigned), bs);
    }
    if (e == cudaSuccess) e = pool_alloc(&p->stats, kStatCount * sizeof(unsigned long long), bs);
    static_assert(kStatCount * sizeof(unsigned long long) <= kPinBytes, "pinned block too small");
    for (auto &ev : p->ev)
        if (e == cudaSuccess) e = cudaEventCreate(&ev);
    if (e != cudaSuccess) return fail(from_cuda(e));
    e = build_chunk_table(p->row_ptr, n, chunk, p->hub_base, &p->chunk_tab, &p->n_chunks,
                          reinterpret_cast<int32_t *>(p->ctr_h), bs);
    if (e != cudaSuccess) return fail(from_cuda(e));
    if (n + p->n_chunks >= (1ll << 31)) return fail(TQ_ERR_UNSUPPORTED);

    // weighted label correcting re-enqueues far more than BFS: 8V for SSSP
    uint64_t cap = o.capacity ? o.capacity : next_pow2((uint64_t)((task == kTaskSSSP ? 8 : 2) * n));
    if (cap > (1ull << 31)) cap = 1ull << 31;
    if (!o.capacity && cap < (1ull << 16)) cap = 1ull << 16;
    tq_status st = queue_create_on(cap, gdev, p->stream, false, &p->q);
    if (st != TQ_OK) return fail(st);
    // chunk queue (RF/AN only): a hub emits its chunks at every expansion
    // (one per distinct level, R7); 4x the chunk count, at least 2^20 slots
    // (8 MiB), leaves room for bursts while consumers lag (e.g. under ncu).
    // An explicit capacity C bounds it by C and raises it to at least C/4, so
    // a caller that answers a queue-full abort by doubling C (the
    // Python binding's grow_on_full) also grows the chunk queue.
    p->hub_queue = p->variant == TQ_VARIANT_RF_AN && o.hub_queue >= 0 && p->n_chunks > 0;
    if (p->hub_queue) {
        uint64_t cap1 = next_pow2((uint64_t)(4 * p->n_chunks));
        if (cap1 < (1ull << 20)) cap1 = 1ull << 20;
        if (o.capacity) {
            const uint64_t c = next_pow2(o.capacity);
            if (cap1 > c) cap1 = c;
            if (cap1 < c / 4) cap1 = c / 4;
            if (cap1 < 2) cap1 = 2;
        }
        st = queue_create_on(cap1, gdev, p->stream, false, &p->q1);
        if (st != TQ_OK) return fail(st);
    }

    int per_sm = 0;
    e = bfs_occupancy(p->variant, block, &per_sm);
    if (e != cudaSuccess) return fail(from_cuda(e));
    const int full = per_sm * sm_count(gdev);
    if (o.threads > 0) {
        p->blocks = (o.threads + p->block - 1) / p->block;
    } else {
        p->blocks = full;
        p->auto_blocks = task == kTaskBFS && o.deep_grid >= 0;
        // Small graphs (< 2^20 CSR entries, e.g. config 1's R-MAT scale 10):
        // one block per SM.  The run is a chain of ~4 us hops with little
        // work per level; the full grid only adds its start-up reservations
        // (one Front AFA per warp) and idle polling (measured: rmat10 kernel
        // 111 -> 97 us, a 2-vertex graph 25.6 -> 19.5 us).
        if (p->auto_blocks && nnz < (1ll << 20)) p->blocks = sm_count(gdev) < full ? sm_count(gdev) : full;
    }
    // lanes per warp holding main-queue tickets (bfs_opts.ticket_lanes)
    if (o.ticket_lanes < 0 || o.ticket_lanes > 32) return fail(TQ_ERR_INVALID);
    // auto: 32; 2 on graphs below 2^20 CSR entries (rmat10 91 -> 42 us, kron14
    // 141 -> 83 us); 8 once a plan has dropped to the deep-graph grid (grid
    // 4096^2 43.4 -> 41.9 ms); large shallow graphs keep 32 (kron24 with 16 /
    // 8 / 4 lanes: +8% / +19% / +38%) -- results/small_graph_latency_lanes_r02.jsonl,
    // results/ab_round2_r02.md
    p->auto_lanes = o.ticket_lanes == 0;
    p->ticket_lanes = o.ticket_lanes ? o.ticket_lanes : (nnz < (1ll << 20) ? 2 : 32);
    // shared-memory path: 8 lanes per warp (config 1, 1/2/4/8/32 lanes:
    // 54/.../39/47 us, results/smem_path_r02.log)
    if (smem_auto_lanes && p->auto_lanes) p->ticket_lanes = 8;
    if (p->blocks < 1) p->blocks = 1;
    // (the persisting window only pays when the mirror competes with the col
    // stream for L2: not for mirrors below 4 MB, whose set-up per launch
    // would only add launch latency)
    if (task == kTaskBFS && !p->smem && o.l2_persist >= 0 && p->mirror_bytes >= (4u << 20)) {
        // L2 persistence (B200: up to ~79 MiB of the 126 MB L2): the level
        // mirror is probed once per edge; a persisting window keeps it
        // resident against the col stream (shared device limit, see
        // l2_persist_acquire)
        p->l2_window = l2_persist_acquire(gdev, p->mirror_bytes);
    }
    e = cudaStreamSynchronize(bs);  // (the build's buffers are used on p->stream from now on)
    if (e == cudaSuccess) e = cudaStreamSynchronize(p->stream);
    if (e != cudaSuccess) return fail(from_cuda(e));
    cudaStreamDestroy(bs);
    *out = p;
    return TQ_OK;
}

tq_status bfs_plan_create(const tq_csr *gph, const bfs_opts *opts, bfs_plan **out)
{
    return plan_create_impl(gph, nullptr, kTaskBFS, opts, out);
}

tq_status sssp_plan_create(const tq_csr *gph, const int32_t *weights, const bfs_opts *opts,
                           bfs_plan **out)
{
    return plan_create_impl(gph, weights, kTaskSSSP, opts, out);
}

// The plan's vertex relabelling (relabel.cu), at its first
// run, on its stream (synchronous).  The chunk table names vertices, so it
// is rebuilt on the new numbering (same chunk count).
static tq_status plan_relabel(bfs_plan *p)
{
    p->relabel_pending = false;
    RelabelOut ro{};
    cudaStream_t s = p->stream;
    cudaError_t e = build_relabel(p->row_ptr, p->col, p->n, p->nnz, p->relabel_min_deg, p->hub_region,
                                  reinterpret_cast<int32_t *>(p->ctr_h), &ro, s);
    if (e != cudaSuccess) return from_cuda(e);
    if (!ro.new2old) return TQ_OK;  // no vertex above the degree threshold
    p->relabelled = true;
    p->row_ptr0 = p->row_ptr;
    if (p->owns_graph) pool_free(p->col, s);  // only the relabelled entries are read
    p->row_ptr = ro.row_ptr;
    p->col = ro.col;
    p->new2old = ro.new2old;
    p->old2new = ro.old2new;
    pool_free(p->chunk_tab, s);
    p->chunk_tab = nullptr;
    int64_t nch = 0;
    e = build_chunk_table(p->row_ptr, p->n, p->chunk, p->hub_base, &p->chunk_tab, &nch,
                          reinterpret_cast<int32_t *>(p->ctr_h), s);
    if (e != cudaSuccess) return from_cuda(e);
    return nch == p->n_chunks ? TQ_OK : TQ_ERR_CUDA;
}

// First half of a run: enqueue init + persistent kernel + unpack and the
// status / statistics read-back on the plan's stream; returns immediately.
static tq_status plan_launch(bfs_plan *p, int32_t root, int32_t *level, int32_t *parent)
{
    cudaStream_t s = p->stream;
    if (p->in_flight) return TQ_ERR_INVALID;
    if (p->relabel_pending) {
        tq_status st = plan_relabel(p);
        if (st != TQ_OK) return st;
    }
    if (p->dirty) {
        tq_status st = tq_reset(p->q, s);
        if (st == TQ_OK && p->q1) st = tq_reset(p->q1, s);
        if (st != TQ_OK) return st;
        p->next_ticket = 0;
        p->next_ticket1 = 0;
        p->dirty = false;
    }
    BfsParams bp{};
    bp.q = p->q->view;
    if (p->hub_queue) {
        bp.q1 = p->q1->view;
        bp.q1.status = p->q->view.status;  // one status word for both queues
        bp.hub_queue = 1;
        // chunk-queue ticket holders per warp: lanes 0 and 16 (measured on
        // B200 kron24 over 1/2/4/8 holders x chunk 256..1024: 2 x 512 best)
        bp.q1_lanes = 0x00010001u;
    }
    bp.row_ptr = p->row_ptr;
    bp.col = p->col;
    bp.W = p->W;
    bp.chunk_tab = p->chunk_tab;
    bp.hub_base = p->hub_base;
    bp.mir = p->mir;
    bp.mirror_bits = p->mirror_bits;
    bp.x8 = p->x8;
    bp.xd = p->xd;
    bp.wgt = p->wgt;
    bp.task = p->task;
    bp.parent_rule = p->parent_rule;
    bp.stats = p->stats;
    bp.n_vertices = p->n;
    bp.chunk = p->chunk;
    while ((1 << bp.log2_chunk) < p->chunk) ++bp.log2_chunk;
    bp.backoff_ns = p->backoff_ns;
    bp.timeout_ns = (unsigned long long)(p->timeout_s * 1e9);
    bp.l2_window_bytes = p->l2_window;
    bp.delay_ns = (unsigned)p->delay_ns;
    bp.cas_backoff_ns = (unsigned)p->cas_backoff_ns;
    bp.ticket_lanes = p->ticket_lanes >= 32 ? 0xFFFFFFFFu : ((1u << p->ticket_lanes) - 1u);
    bp.delay_seed = p->delay_seed;
    // every slot of [t0, t0 + C) holds "empty for t" when a run starts (after
    // a reset, or at Rear after a finished run; see plan_finish)
    bp.q_lap_end = p->next_ticket + (bp.q.mask + 1);
    bp.q1_lap_end = p->hub_queue ? p->next_ticket1 + (bp.q1.mask + 1) : 0ull;

    bp.nnz = p->nnz;
    bp.small_cap = p->smem_cap;
    bp.new2old = p->new2old;
    bp.old2new = p->old2new;
    bp.row_ptr0 = p->row_ptr0;
    bp.pid_orig = p->relabelled && p->parent_rule == TQ_PARENT_MIN_ID;
    // token layout: as few id bits as the ids need, the rest carry the level
    bp.tok_vbits = 1;
    while (bp.tok_vbits < 31 && (1ll << bp.tok_vbits) < p->n) ++bp.tok_vbits;
    bp.tok_cbits = 1;
    while (bp.tok_cbits < 31 && (1ll << bp.tok_cbits) < p->n_chunks) ++bp.tok_cbits;
    if (p->level_bits > 0) {  // test: a narrower level field (more id bits)
        if (bp.tok_vbits < 31u - p->level_bits) bp.tok_vbits = 31u - p->level_bits;
        if (bp.tok_cbits < 31u - p->level_bits) bp.tok_cbits = 31u - p->level_bits;
    }
    bp.lit = p->lit ? 1 : 0;
    p->lit_field = 0x7FFFFFFFu >> (bp.tok_vbits > bp.tok_cbits ? bp.tok_vbits : bp.tok_cbits);
    if (p->smem) {
        // one launch: graph load, BFS over the shared-memory queue, unpack
        // (its statistics and status land where the grid path puts them;
        // the global queues are untouched, so their tickets stay put)
        CK(cudaEventRecord(p->ev[0], s));
        CK(cudaEventRecord(p->ev[1], s));
        CK(launch_bfs_small(bp, root, level, parent, s));
        CK(cudaEventRecord(p->ev[2], s));
        CK(cudaEventRecord(p->ev[3], s));
    } else {
        CK(cudaEventRecord(p->ev[0], s));
        CK(launch_bfs_init(bp, root, p->next_ticket, p->next_ticket1, s));
        CK(cudaEventRecord(p->ev[1], s));
        CK(launch_bfs_persistent(p->variant, bp, p->blocks, p->block, s));
        CK(cudaEventRecord(p->ev[2], s));
        CK(launch_bfs_unpack(bp, level, parent, s));
        CK(cudaEventRecord(p->ev[3], s));
    }
    CK(cudaMemcpyAsync(p->stats_h, p->stats, kStatCount * sizeof(unsigned long long),
                       cudaMemcpyDeviceToHost, s));
    unsigned long long *ctr = p->ctr_h;  // pinned: front, rear, done, rear1, status
    ctr[3] = 0;
    CK(cudaMemcpyAsync(&ctr[0], p->q->view.front, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&ctr[1], p->q->view.rear, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&ctr[2], p->q->view.done, 8, cudaMemcpyDeviceToHost, s));
    if (p->hub_queue) CK(cudaMemcpyAsync(&ctr[3], p->q1->view.rear, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&ctr[4], p->q->view.status, 4, cudaMemcpyDeviceToHost, s));
    p->in_flight = true;
    return TQ_OK;
}

// Second half of a run: wait for the launch, read the status word back and
// fill the statistics.
static tq_status plan_finish(bfs_plan *p, bfs_stats *stats)
{
    if (!p->in_flight) return TQ_ERR_INVALID;
    p->in_flight = false;
    CK(cudaStreamSynchronize(p->stream));
    const unsigned long long *ctr = p->ctr_h;
    const unsigned status = (unsigned)ctr[4];
    const unsigned long long t0 = p->next_ticket, t1 = p->next_ticket1;
    if (status == TQ_FINISHED) {
        // every reserved ticket below Rear was taken; slots of tickets
        // [Rear, Rear + C) all hold "empty for t", so the next run can start
        // at Rear without an O(C) reset (both queues)
        p->next_ticket = ctr[1];
        if (p->hub_queue) p->next_ticket1 = ctr[3];
    } else {
        p->dirty = true;
    }
    if (stats) {
        memset(stats, 0, sizeof(*stats));
        float a = 0, b = 0;
        cudaEventElapsedTime(&a, p->ev[0], p->ev[3]);
        cudaEventElapsedTime(&b, p->ev[1], p->ev[2]);
        stats->ms = a;
        stats->ms_kernel = b;
        const unsigned long long *h = p->stats_h;
        stats->tasks = h[ST_TASKS];
        stats->chunk_tasks = h[ST_CHUNK_TASKS];
        stats->edges_scanned = h[ST_EDGES];
        stats->min_atomics = h[ST_MIN_ATOMICS];
        stats->reenqueues = h[ST_REENQUEUES];
        stats->queue_atomics = h[ST_QUEUE_ATOMICS];
        stats->cas_failures = h[ST_CAS_FAILURES];
        stats->empty_polls = h[ST_EMPTY_POLLS];
        stats->reached = h[ST_REACHED];
        stats->traversed_edges = h[ST_DEG_SUM] / 2;
        stats->max_level = (int32_t)h[ST_MAX_LEVEL];
        stats->tickets = p->smem ? h[ST_SMEM_TICKETS] : (ctr[1] - t0) + (p->hub_queue ? ctr[3] - t1 : 0ull);
        stats->skipped_tasks = h[ST_SKIPPED];
        stats->busy_cycles = h[ST_BUSY_CYCLES];
        stats->rounds = h[ST_ROUNDS];
        stats->persistent_threads = p->blocks * p->block;
        stats->mirror_bits = p->task == kTaskBFS ? p->mirror_bits : 0;
        stats->ticket_lanes = p->ticket_lanes;
        stats->smem_path = p->smem ? 1 : 0;
        stats->relabelled = p->relabelled ? 1 : 0;
        stats->level_tokens = (!p->smem && p->task == kTaskBFS && p->variant == TQ_VARIANT_RF_AN && p->lit) ? 1 : 0;
        if (p->smem) stats->persistent_threads = 1024;
    }
    // Deep graphs: a BFS of >= 1,024 levels runs a few thousand
    // vertices per level at a time; a full persistent grid then spends L2 on
    // idle polls of its 189K held tickets (the paper's too-many-threads
    // dilemma).  After such a run the plan (same graph) launches one
    // block per SM: grid 4096^2 53 -> ~46 ms.  Only when threads == 0.
    // Levels in the tokens (R22): a run whose levels did not fit the field
    // published its deeper tokens with a release fence and took them with an
    // acquire re-read, dearer than the plain acquire polls; the plan's later
    // runs (same graph) use the acquire polls throughout.
    if (status == TQ_FINISHED && p->stats_h[ST_MAX_LEVEL] >= p->lit_field) p->lit = false;
    if (p->auto_blocks && status == TQ_FINISHED && p->stats_h[ST_MAX_LEVEL] >= 1024) {
        const int deep_blocks = sm_count(p->device);
        if (p->blocks > deep_blocks) p->blocks = deep_blocks;
        if (p->auto_lanes && p->ticket_lanes > 8) p->ticket_lanes = 8;
    }
    if (status == TQ_FINISHED) return TQ_OK;
    if (status == TQ_ABORTED_FULL) return TQ_ERR_QUEUE_FULL;
    if (status == TQ_ABORTED_TIMEOUT) return TQ_ERR_TIMEOUT;
    return TQ_ERR_CUDA;
}

tq_status bfs_plan_set_tickets(bfs_plan *p, uint64_t t_main, uint64_t t_chunk)
{
    if (!p || p->in_flight || t_main >= (1ull << 62) || t_chunk >= (1ull << 62)) return TQ_ERR_INVALID;
    DeviceGuard g(p->device);
    tq_status st = tq_reset_at(p->q, t_main, p->stream);
    if (st == TQ_OK && p->q1) st = tq_reset_at(p->q1, t_chunk, p->stream);
    if (st == TQ_OK) st = from_cuda(cudaStreamSynchronize(p->stream));
    if (st != TQ_OK) return st;
    p->next_ticket = t_main;
    p->next_ticket1 = p->q1 ? t_chunk : 0;
    p->dirty = false;
    return TQ_OK;
}

tq_status bfs_plan_get_tickets(const bfs_plan *p, uint64_t *t_main, uint64_t *t_chunk)
{
    if (!p || !t_main || !t_chunk) return TQ_ERR_INVALID;
    *t_main = p->next_ticket;
    *t_chunk = p->next_ticket1;
    return TQ_OK;
}

tq_status bfs_plan_launch(bfs_plan *p, int32_t root, int32_t *level_out, int32_t *parent_out)
{
    if (!p || root < 0 || root >= p->n) return TQ_ERR_INVALID;
    if ((level_out && is_device_ptr(level_out, nullptr) != 1) ||
        (parent_out && is_device_ptr(parent_out, nullptr) != 1))
        return TQ_ERR_INVALID;  // the asynchronous form takes device outputs only
    DeviceGuard g(p->device);
    return plan_launch(p, root, level_out, parent_out);
}

tq_status bfs_plan_wait(bfs_plan *p, bfs_stats *stats)
{
    if (!p) return TQ_ERR_INVALID;
    DeviceGuard g(p->device);
    return plan_finish(p, stats);
}

tq_status bfs_plan_run_batch(bfs_plan *p, const int32_t *roots, int32_t n_roots,
                             int32_t *level_out, int32_t *parent_out, int64_t out_stride,
                             bfs_stats *stats)
{
    if (!p || !roots || n_roots < 0 || out_stride < 0) return TQ_ERR_INVALID;
    for (int32_t i = 0; i < n_roots; ++i)
        if (roots[i] < 0 || roots[i] >= p->n) return TQ_ERR_INVALID;
    DeviceGuard g(p->device);
    const int kind_l = level_out ? is_device_ptr(level_out, nullptr) : 1;
    const int kind_p = parent_out ? is_device_ptr(parent_out, nullptr) : 1;
    if (kind_l < 0 || kind_p < 0) return TQ_ERR_INVALID;
    const bool host_l = kind_l == 0, host_p = kind_p == 0;
    const size_t vb = (size_t)p->n * sizeof(int32_t);
    if (host_l || host_p) {
        // two device output pairs + a copy stream, allocated on first use
        if (!p->dbuf[0]) {
            for (int b = 0; b < kOutBufs; ++b) CK(pool_alloc(&p->dbuf[b], 2 * vb, p->stream));
            CK(cudaStreamCreateWithFlags(&p->copy_stream, cudaStreamNonBlocking));
            for (int b = 0; b < kOutBufs; ++b) {
                CK(cudaEventCreateWithFlags(&p->bfs_done[b], cudaEventDisableTiming));
                CK(cudaEventCreateWithFlags(&p->copy_done[b], cudaEventDisableTiming));
                CK(cudaEventRecord(p->copy_done[b], p->copy_stream));
            }
        }
    }
    tq_status st = TQ_OK;
    // Host outputs: root i's arrays drain (copy stream) while root i+1 runs.
    // The copy of root i is issued AFTER root i+1's kernels are enqueued:
    // measured on the B200 boxes, a persistent BFS enqueued while a large
    // D2H copy is in flight does not start until the copy ends, whereas a
    // copy enqueued behind the running kernel overlaps it fully.
    int32_t pend = -1;  // root whose outputs still have to be copied
    auto issue_copy = [&](int32_t k) -> cudaError_t {
        const int b = k % kOutBufs;
        int32_t *lv = level_out + (level_out ? (size_t)k * out_stride : 0);
        int32_t *pa = parent_out + (parent_out ? (size_t)k * out_stride : 0);
        cudaError_t e = cudaStreamWaitEvent(p->copy_stream, p->bfs_done[b], 0);
        if (e == cudaSuccess && host_l) e = d2h_chunked(lv, p->dbuf[b], vb, p->copy_stream);
        if (e == cudaSuccess && host_p) e = d2h_chunked(pa, p->dbuf[b] + p->n, vb, p->copy_stream);
        if (e == cudaSuccess) e = cudaEventRecord(p->copy_done[b], p->copy_stream);
        return e;
    };
    for (int32_t i = 0; i < n_roots && st == TQ_OK; ++i) {
        int32_t *lv = level_out ? level_out + (size_t)i * out_stride : nullptr;
        int32_t *pa = parent_out ? parent_out + (size_t)i * out_stride : nullptr;
        if (!host_l && !host_p) {
            st = plan_launch(p, roots[i], lv, pa);
            if (st == TQ_OK) st = plan_finish(p, stats ? stats + i : nullptr);
            continue;
        }
        const int b = i % kOutBufs;
        int32_t *dl = lv ? (host_l ? p->dbuf[b] : lv) : nullptr;
        int32_t *dp = pa ? (host_p ? p->dbuf[b] + p->n : pa) : nullptr;
        // the buffer pair is free once the copy of root i - kOutBufs has drained
        CK(cudaStreamWaitEvent(p->stream, p->copy_done[b], 0));
        st = plan_launch(p, roots[i], dl, dp);
        if (st != TQ_OK) break;
        CK(cudaEventRecord(p->bfs_done[b], p->stream));
        if (pend >= 0) CK(issue_copy(pend));
        pend = i;
        st = plan_finish(p, stats ? stats + i : nullptr);
    }
    if (pend >= 0 && st == TQ_OK) CK(issue_copy(pend));
    if (p->copy_stream) CK(cudaStreamSynchronize(p->copy_stream));
    return st;
}

tq_status bfs_plan_run(bfs_plan *p, int32_t root, int32_t *level_out, int32_t *parent_out,
                       bfs_stats *stats)
{
    if (!p || root < 0 || root >= p->n) return TQ_ERR_INVALID;
    DeviceGuard g(p->device);
    const int kind_l = level_out ? is_device_ptr(level_out, nullptr) : 1;
    const int kind_p = parent_out ? is_device_ptr(parent_out, nullptr) : 1;
    if (kind_l < 0 || kind_p < 0) return TQ_ERR_INVALID;
    const bool host_l = kind_l == 0, host_p = kind_p == 0;
    if (!host_l && !host_p) {
        const tq_status st = plan_launch(p, root, level_out, parent_out);
        return st == TQ_OK ? plan_finish(p, stats) : st;
    }
    if (!p->out_scratch) CK(pool_alloc(&p->out_scratch, (size_t)p->n * 2 * sizeof(int32_t), p->stream));
    int32_t *dl = level_out ? (host_l ? p->out_scratch : level_out) : nullptr;
    int32_t *dp = parent_out ? (host_p ? p->out_scratch + p->n : parent_out) : nullptr;
    tq_status st = plan_launch(p, root, dl, dp);
    if (st == TQ_OK) st = plan_finish(p, stats);
    if (st != TQ_OK) return st;
    if (host_l)
        CK(d2h_chunked(level_out, dl, (size_t)p->n * sizeof(int32_t), p->stream));
    if (host_p)
        CK(d2h_chunked(parent_out, dp, (size_t)p->n * sizeof(int32_t), p->stream));
    CK(cudaStreamSynchronize(p->stream));
    return TQ_OK;
}

tq_status bfs_run_ex(const tq_csr *g, int32_t root, int32_t *level_out, int32_t *parent_out,
                     const bfs_opts *opts, bfs_stats *stats)
{
    if (!g || root < 0 || root >= g->n_vertices) return TQ_ERR_INVALID;
    bfs_plan *p = nullptr;
    tq_status st = bfs_plan_create(g, opts, &p);
    if (st != TQ_OK) return st;
    st = bfs_plan_run(p, root, level_out, parent_out, stats);
    bfs_plan_destroy(p);
    return st;
}

tq_status bfs_run(const tq_csr *g, int32_t root, int32_t *level_out, int32_t *parent_out)
{
    return bfs_run_ex(g, root, level_out, parent_out, nullptr, nullptr);
}

tq_status sssp_plan_run(bfs_plan *p, int32_t src, uint32_t *dist_out, int32_t *parent_out,
                        bfs_stats *stats)
{
    if (!p || p->task != kTaskSSSP) return TQ_ERR_INVALID;
    // the unpack writes dist's 32 bits (0xFFFFFFFF = unreached) into dist_out
    return bfs_plan_run(p, src, reinterpret_cast<int32_t *>(dist_out), parent_out, stats);
}

tq_status sssp_run_ex(const tq_csr *g, const int32_t *weights, int32_t src, uint32_t *dist_out,
                      int32_t *parent_out, const bfs_opts *opts, bfs_stats *stats)
{
    if (!g || src < 0 || src >= g->n_vertices) return TQ_ERR_INVALID;
    bfs_plan *p = nullptr;
    tq_status st = sssp_plan_create(g, weights, opts, &p);
    if (st != TQ_OK) return st;
    st = sssp_plan_run(p, src, dist_out, parent_out, stats);
    bfs_plan_destroy(p);
    return st;
}

// ------------------------------------------------------------------------
// queue micro-benchmark
// ------------------------------------------------------------------------
tq_status tq_probe_ceiling(int device, uint64_t table_bytes, uint64_t probes, void *stream, double *g_per_s)
{
    if (!g_per_s || table_bytes < (1ull << 12) || table_bytes >= (1ull << 32) || probes < (1ull << 20) ||
        probes >= (1ull << 32))
        return TQ_ERR_INVALID;
    *g_per_s = 0.0;
    DeviceGuard g(device);
    if (!g.ok) return TQ_ERR_INVALID;
    int per_sm = 0;  // the BFS kernel's occupancy: same block shape, same residency
    CK(bfs_occupancy(TQ_VARIANT_RF_AN, 256, &per_sm));
    CK(probe_ceiling(table_bytes, probes, per_sm, (cudaStream_t)stream, g_per_s));
    return TQ_OK;
}

tq_status tq_bench(const tq_bench_cfg *c, tq_bench_result *r)
{
    if (!c || !r) return TQ_ERR_INVALID;
    memset(r, 0, sizeof(*r));
    if (c->variant < TQ_VARIANT_RF_AN || c->variant > TQ_VARIANT_RF_AN_CLUSTER) return TQ_ERR_UNSUPPORTED;
    if (c->batch < 1 || c->batch > 32 || c->items == 0 || c->warps < 0) return TQ_ERR_INVALID;
    if (c->depth < 0 || c->depth > 2) return TQ_ERR_INVALID;
    if (c->cas_backoff_ns < 0 || c->cas_backoff_ns > 1000000) return TQ_ERR_INVALID;
    const bool cluster_v = c->variant == TQ_VARIANT_RF_AN_CLUSTER;
    const int depth = cluster_v ? 2 : (c->depth == 0 ? 1 : c->depth);
    if (depth == 2 && c->variant != TQ_VARIANT_RF_AN_CTA && !cluster_v) return TQ_ERR_UNSUPPORTED;
    const int csize = cluster_v ? (c->cluster == 0 ? 4 : c->cluster) : 1;
    if (csize < 1 || csize > 16) return TQ_ERR_INVALID;
    DeviceGuard g(c->device);
    if (!g.ok) return TQ_ERR_INVALID;
    int warps = c->warps;
    if (cluster_v) {
        int clusters = 0;
        CK(bench_max_clusters(csize, 256, &clusters));
        if (warps == 0) warps = clusters * csize * 8;
        if (warps % (8 * csize) || warps > clusters * csize * 8 || warps == 0) return TQ_ERR_INVALID;
    } else if (warps == 0) {
        int per_sm = 0;
        if (depth == 2)
            CK(bench_pipe_occupancy(256, &per_sm));
        else
            CK(bench_occupancy(c->variant, 256, &per_sm));
        warps = per_sm * sm_count(c->device) * 8;
    }
    int wpb = 8;
    while (warps % wpb) wpb >>= 1;
    const int block = 32 * wpb, blocks = warps / wpb;
    const uint64_t iters = c->items / ((uint64_t)warps * c->batch);
    if (iters == 0 || iters > (1ull << 30)) return TQ_ERR_INVALID;
    const uint64_t items = iters * warps * c->batch;
    if (c->log_mode && (!c->enq_log || !c->deq_log)) return TQ_ERR_INVALID;
    uint64_t cap = c->capacity ? c->capacity : (1ull << 20);
    // the ring must hold every item that can be in flight (depth iterations' worth)
    if ((uint64_t)warps * c->batch * depth > next_pow2(cap)) return TQ_ERR_INVALID;

    tq_queue *q = nullptr;
    tq_status st = tq_create(cap, c->device, &q);
    if (st != TQ_OK) return st;
    cudaStream_t s = (cudaStream_t)c->stream;
    unsigned long long *out = nullptr, out_h[16];
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    cudaError_t e = cudaMalloc(&out, sizeof(out_h));
    if (e == cudaSuccess) e = cudaMemsetAsync(out, 0, sizeof(out_h), s);
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    BenchParams bp{};
    bp.q = q->view;
    bp.batch = c->batch;
    bp.iters = (int)iters;
    bp.work_iters = c->work_iters;
    {
        // seed32 = low 32 bits of splitmix64(seed) (inputs/items.py:seed32)
        unsigned long long x = c->seed;
        x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull;
        x ^= x >> 27; x *= 0x94D049BB133111EBull;
        x ^= x >> 31;
        bp.seed32 = (uint32_t)x;
    }
    bp.enq_log = c->log_mode ? c->enq_log : nullptr;
    bp.deq_log = c->log_mode ? c->deq_log : nullptr;
    bp.out = out;
    bp.timeout_ns = (unsigned long long)((c->timeout_s > 0 ? c->timeout_s : 60.0) * 1e9);
    bp.cas_backoff_ns = (unsigned)c->cas_backoff_ns;
    bp.relaxed_poll = c->relaxed_poll ? 1 : 0;
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = cudaEventRecord(e0, s);
    if (e == cudaSuccess) {
        if (depth == 2)
            e = launch_bench_pipe(cluster_v ? 2 : 1, csize, bp, blocks, block, s);
        else
            e = launch_bench(c->variant, bp, blocks, block, s);
    }
    if (e == cudaSuccess) e = cudaEventRecord(e1, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(out_h, out, sizeof(out_h), cudaMemcpyDeviceToHost, s);
    unsigned status = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&status, q->view.status, 4, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) {
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        r->ms = ms;
        r->items = items;
        r->enq = out_h[0];
        r->deq = out_h[1];
        r->atomics = out_h[2];
        r->cas_failures = out_h[3];
        r->empty_retries = out_h[4];
        r->sum_enq = out_h[5];
        r->sum_deq = out_h[6];
        r->xor_enq = out_h[7];
        r->xor_deq = out_h[8];
        r->warps = warps;
        if (status == TQ_ABORTED_FULL)
            st = TQ_ERR_QUEUE_FULL;
        else if (status == TQ_ABORTED_TIMEOUT)
            st = TQ_ERR_TIMEOUT;
        else if (c->variant != TQ_VARIANT_ATOMIC_CEILING && (r->deq != items || r->enq != items))
            st = TQ_ERR_TIMEOUT;
    } else {
        st = from_cuda(e);
    }
    r->status = st;
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    cudaFree(out);
    tq_destroy(q);
    return st;
}

}  // extern "C"
