// relabel.cu -- plan-build vertex relabelling for the persistent BFS
// (bfs_opts.relabel).
//
// The expansion probes one level-mirror byte and, for candidates, one packed
// W word per CSR entry.  On a Kronecker graph half of
// all entries name the few-percent highest-degree vertices, scattered over the
// whole id range by the generator's random permutation, so their mirror bytes,
// W words, markers and row offsets each sit in their own 32-byte sector.  The
// plan therefore renumbers vertices by descending degree (stable, so equal
// degrees keep their order), which packs the hubs' per-vertex state into few
// sectors; the first kHubRegion ranks are dealt round-robin over the region's
// 128-byte lines (rank r -> (r mod lines) * 128 + r / lines) so that the very
// top hubs -- the most-probed bytes -- land in different lines and L2 slices
// instead of all in the first one.  Measured (results/relabel_r02.log): kron24
// -8.4%, kron26 -6.2% kernel time; without the dealing the hot lines make it
// 2x slower.
//
// The BFS itself runs on the relabelled CSR (tokens, W, mirror, markers and
// chunk table are indexed by new ids).  W's parent field holds new ids, which
// the unpack translates (one gather per reached vertex), except under the
// min-id rule (R5), whose minimum must be the one of the original numbering:
// there the kernel offers original ids (one new2old read per task, +3% kernel
// time).  The unpack reads W through old2new and writes the outputs in the
// original order.  No other part of the method
// changes: it is a data layout of the plan (Graph500 allows kernel-1
// relabelling), and the oracle compares the original-order outputs.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "internal.cuh"

namespace tqk {

namespace {

// ranks dealt over the region's lines: 2^20 (kron26 -6.2% vs -2.2% with 2^17,
// kron24 -8.4% vs -7.4%; results/relabel_r02.log)
constexpr int64_t kHubRegion = 1 << 20;
constexpr int64_t kBigRow = 4096;        // rows copied by a whole block

__host__ __device__ __forceinline__ int64_t rank_to_new(int64_t r, int64_t H, int64_t lines)
{
    return r < H ? (r % lines) * 128 + r / lines : r;
}

__global__ void degree_kernel(const int64_t *rp, int64_t n, int32_t *deg, int32_t *iota)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        deg[i] = (int32_t)(rp[i + 1] - rp[i]);
        iota[i] = (int32_t)i;
    }
}

// new ids from ranks; new-order degrees (int64, for the offsets scan)
__global__ void place_kernel(const int32_t *deg_sorted, const int32_t *rank2old, int64_t n, int64_t H,
                             int64_t lines, int32_t *new2old, int32_t *old2new, int64_t *deg_new)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride) {
        const int64_t i = rank_to_new(r, H, lines);
        const int32_t o = rank2old[r];
        new2old[i] = o;
        old2new[o] = (int32_t)i;
        deg_new[i] = deg_sorted[r];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) deg_new[n] = 0;
}

// rows of rank >= r0 (at most kBigRow entries): one warp per row
__global__ void copy_rows_warp(const int64_t *rp, const int32_t *col, const int64_t *rp_new,
                               const int32_t *rank2old, const int32_t *old2new, int64_t n, int64_t r0,
                               int64_t H, int64_t lines, int32_t *col_new)
{
    const unsigned lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t r = r0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); r < n; r += nw) {
        const int64_t i = rank_to_new(r, H, lines);
        const int32_t o = rank2old[r];
        const int64_t src = rp[o], d = rp[o + 1] - src, dst = rp_new[i];
        for (int64_t k = lane; k < d; k += 32) col_new[dst + k] = old2new[__ldg(col + src + k)];
    }
}

// rows of rank < r0 (more than kBigRow entries): one block per row, four
// gathers in flight per thread
__global__ void __launch_bounds__(512) copy_rows_block(const int64_t *rp, const int32_t *col, const int64_t *rp_new,
                                                       const int32_t *rank2old, const int32_t *old2new,
                                                       int64_t H, int64_t lines, int32_t *col_new)
{
    const int64_t r = blockIdx.x;
    const int64_t i = rank_to_new(r, H, lines);
    const int32_t o = rank2old[r];
    const int64_t src = rp[o], d = rp[o + 1] - src, dst = rp_new[i];
    const int64_t step = 4 * (int64_t)blockDim.x;
    int64_t k = threadIdx.x;
    for (; k + 3 * blockDim.x < d; k += step) {
        int32_t c[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) c[j] = __ldg(col + src + k + j * blockDim.x);
#pragma unroll
        for (int j = 0; j < 4; ++j) c[j] = old2new[c[j]];
#pragma unroll
        for (int j = 0; j < 4; ++j) col_new[dst + k + j * blockDim.x] = c[j];
    }
    for (; k < d; k += blockDim.x) col_new[dst + k] = old2new[__ldg(col + src + k)];
}

int grid_of(int64_t n, int block)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int64_t want = (n + block - 1) / block, cap = (int64_t)sms * 8;
    return (int)(want < 1 ? 1 : (want < cap ? want : cap));
}

}  // namespace

cudaError_t build_relabel(const int64_t *rp, const int32_t *col, int64_t n, int64_t nnz, int min_max_degree,
                          RelabelOut *out, cudaStream_t s)
{
    *out = RelabelOut{};
    int32_t *deg = nullptr, *iota = nullptr, *deg_sorted = nullptr, *rank2old = nullptr;
    int64_t *deg_new = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0, t2 = 0;
    RelabelOut o{};
    cudaError_t e = pool_alloc(&deg, (size_t)n * 4, s);
    if (e == cudaSuccess) e = pool_alloc(&iota, (size_t)n * 4, s);
    if (e == cudaSuccess) e = pool_alloc(&deg_sorted, (size_t)n * 4, s);
    if (e == cudaSuccess) e = pool_alloc(&rank2old, (size_t)n * 4, s);
    if (e == cudaSuccess) {
        degree_kernel<<<grid_of(n, 256), 256, 0, s>>>(rp, n, deg, iota);
        e = cudaGetLastError();
    }
    if (e == cudaSuccess)
        e = cub::DeviceRadixSort::SortPairsDescending(nullptr, tmp_bytes, deg, deg_sorted, iota, rank2old, (int)n, 0,
                                                      32, s);
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(nullptr, t2, deg_new, deg_new, (int)(n + 1), s);
    if (e == cudaSuccess) e = pool_alloc(&tmp, tmp_bytes > t2 ? tmp_bytes : t2, s);
    if (e == cudaSuccess)
        e = cub::DeviceRadixSort::SortPairsDescending(tmp, tmp_bytes, deg, deg_sorted, iota, rank2old, (int)n, 0, 32,
                                                      s);
    int32_t maxdeg = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&maxdeg, deg_sorted, 4, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e == cudaSuccess && maxdeg > min_max_degree) {
        // hub region: the first H ranks, dealt over H / 128 lines
        int64_t H = (n < kHubRegion ? n : kHubRegion) / 128 * 128;
        if (H < 2 * 128) H = 0;
        const int64_t lines = H ? H / 128 : 1;
        e = pool_alloc(&o.new2old, (size_t)n * 4, s);
        if (e == cudaSuccess) e = pool_alloc(&o.old2new, (size_t)n * 4, s);
        if (e == cudaSuccess) e = pool_alloc(&deg_new, (size_t)(n + 1) * 8, s);
        if (e == cudaSuccess) e = pool_alloc(&o.row_ptr, (size_t)(n + 1) * 8, s);
        if (e == cudaSuccess) e = pool_alloc(&o.col, (size_t)(nnz > 0 ? nnz : 1) * 4, s);
        if (e == cudaSuccess) {
            place_kernel<<<grid_of(n, 256), 256, 0, s>>>(deg_sorted, rank2old, n, H, lines, o.new2old, o.old2new,
                                                         deg_new);
            e = cudaGetLastError();
        }
        size_t tb = tmp_bytes > t2 ? tmp_bytes : t2;
        if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(tmp, tb, deg_new, o.row_ptr, (int)(n + 1), s);
        // rows with more than kBigRow entries are the first ranks
        int64_t nbig = 0;
        if (e == cudaSuccess) {
            // count on the host from a bounded binary search over the sorted degrees
            int64_t lo = 0, hi = n;  // first rank with degree <= kBigRow
            while (lo < hi && e == cudaSuccess) {
                const int64_t mid = (lo + hi) / 2;
                int32_t dm = 0;
                e = cudaMemcpyAsync(&dm, deg_sorted + mid, 4, cudaMemcpyDeviceToHost, s);
                if (e == cudaSuccess) e = cudaStreamSynchronize(s);
                if (dm > kBigRow) lo = mid + 1;
                else hi = mid;
            }
            nbig = lo;
        }
        if (e == cudaSuccess && nbig > 0) {
            copy_rows_block<<<(unsigned)nbig, 512, 0, s>>>(rp, col, o.row_ptr, rank2old, o.old2new, H, lines, o.col);
            e = cudaGetLastError();
        }
        if (e == cudaSuccess && nbig < n) {
            copy_rows_warp<<<grid_of((n - nbig) * 32, 256), 256, 0, s>>>(rp, col, o.row_ptr, rank2old, o.old2new, n,
                                                                        nbig, H, lines, o.col);
            e = cudaGetLastError();
        }
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        if (e == cudaSuccess) {
            *out = o;
        } else {
            pool_free(o.new2old, s);
            pool_free(o.old2new, s);
            pool_free(o.row_ptr, s);
            pool_free(o.col, s);
        }
    }
    pool_free(deg_new, s);
    pool_free(tmp, s);
    pool_free(rank2old, s);
    pool_free(deg_sorted, s);
    pool_free(iota, s);
    pool_free(deg, s);
    return e;
}

}  // namespace tqk
