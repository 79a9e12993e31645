// tqgen.cu -- seeded synthetic graph generation on the GPU (INPUT GENERATOR).
//
// Twin of inputs/graphs.py for sizes numpy cannot build quickly (Kronecker
// scale 24/26, the 4096^2 grid).  Same counter-based RNG, same integer R-MAT
// thresholds, same vertex permutation, same CSR convention (symmetric, no
// self loops, no duplicates, rows ascending), so both produce bit-identical
// CSRs for the same seed (checked by tests/test_gpu_inputs.py).  Holds none
// of the method's arithmetic; shares no code with libtq or the oracle.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t x)
{
    x ^= x >> 30;
    x *= 0xBF58476D1CE4E5B9ull;
    x ^= x >> 27;
    x *= 0x94D049BB133111EBull;
    x ^= x >> 31;
    return x;
}

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;
// int(p * 2**32) for p = .57, .76, .95 (inputs/graphs.py T_A, T_AB, T_ABC)
constexpr uint64_t kTA = 2448131358ull, kTAB = 3264175144ull, kTABC = 4080218931ull;

struct Perm {
    uint64_t m1, a1, m2, a2, mask, sh;
};

__host__ __device__ __forceinline__ uint64_t permute(uint64_t x, const Perm &p)
{
    x = (x * p.m1 + p.a1) & p.mask;
    x ^= x >> p.sh;
    x = (x * p.m2 + p.a2) & p.mask;
    x ^= x >> p.sh;
    return x;
}

__global__ void kron_keys_kernel(int scale, uint64_t m, uint64_t s_mixed, Perm perm, uint64_t *keys)
{
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += stride) {
        uint64_t src = 0, dst = 0;
        for (int l = 0; l < scale; ++l) {
            const uint64_t r = mix64(s_mixed + (i * 64ull + (uint64_t)l) * kGolden) >> 32;
            const bool qc = r >= kTAB && r < kTABC, qb = r >= kTA && r < kTAB, qd = r >= kTABC;
            if (qc || qd) src |= 1ull << l;
            if (qb || qd) dst |= 1ull << l;
        }
        src = permute(src, perm);
        dst = permute(dst, perm);
        if (src == dst) {
            keys[2 * i] = keys[2 * i + 1] = ~0ull;
        } else {
            keys[2 * i] = (src << scale) | dst;
            keys[2 * i + 1] = (dst << scale) | src;
        }
    }
}

// undirected edges (u, v) -> both directed keys u*nv+v (nv need not be 2^k)
__global__ void grid_keys_kernel(int64_t rows, int64_t cols, uint64_t *keys)
{
    const int64_t n = rows * cols;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
        const int64_t r = v / cols, c = v % cols;
        // each vertex emits its right and down edges in both directions: slots 4v..4v+3
        uint64_t k0 = ~0ull, k1 = ~0ull, k2 = ~0ull, k3 = ~0ull;
        if (c + 1 < cols) {
            k0 = (uint64_t)v * n + (v + 1);
            k1 = (uint64_t)(v + 1) * n + v;
        }
        if (r + 1 < rows) {
            k2 = (uint64_t)v * n + (v + cols);
            k3 = (uint64_t)(v + cols) * n + v;
        }
        keys[4 * v] = k0;
        keys[4 * v + 1] = k1;
        keys[4 * v + 2] = k2;
        keys[4 * v + 3] = k3;
    }
}

__global__ void tree4_keys_kernel(int64_t n, uint64_t *keys)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        if (i == 0) {
            keys[0] = keys[1] = ~0ull;
            continue;
        }
        const uint64_t p = (uint64_t)((i - 1) / 4);
        keys[2 * i] = p * (uint64_t)n + i;
        keys[2 * i + 1] = (uint64_t)i * n + p;
    }
}

// keys sorted unique, n_valid entries; row_ptr[v] = lower_bound(keys, v*nv)
__global__ void keys_to_csr_kernel(const uint64_t *keys, int64_t n_keys, int64_t nv, int64_t *row_ptr,
                                   int32_t *col)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_keys; i += stride)
        col[i] = (int32_t)(keys[i] % (uint64_t)nv);
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v <= nv; v += stride) {
        const uint64_t target = (uint64_t)v * (uint64_t)nv;
        int64_t lo = 0, hi = n_keys;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (keys[mid] < target) lo = mid + 1;
            else hi = mid;
        }
        row_ptr[v] = lo;
    }
}

// twin of inputs/graphs.py:edge_weights -- one thread per row
__global__ void edge_weights_kernel(const int64_t *row_ptr, const int32_t *col, int64_t nv,
                                    uint64_t s_mixed, uint32_t wmax, int32_t *w)
{
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nv; v += stride) {
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
            const uint64_t u = (uint64_t)col[e];
            const uint64_t lo = u < (uint64_t)v ? u : (uint64_t)v, hi = u < (uint64_t)v ? (uint64_t)v : u;
            const uint64_t h = mix64(s_mixed + ((lo << 32) | hi) * kGolden);
            w[e] = (int32_t)(h % wmax + 1);
        }
    }
}

int grid_for(int64_t n)
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t g = (n + 255) / 256;
    if (g > (int64_t)sms * 16) g = (int64_t)sms * 16;
    return (int)(g < 1 ? 1 : g);
}

}  // namespace

extern "C" {

// Permutation parameters exactly as inputs/graphs.py:perm_params.
static Perm make_perm(int scale, uint64_t seed)
{
    const uint64_t s = mix64(seed ^ 0x5EED5EEDull);
    const uint64_t mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1);
    uint64_t h[4];
    for (int k = 0; k < 4; ++k) h[k] = mix64(s + (uint64_t)k * kGolden);
    Perm p;
    p.m1 = (h[0] & mask) | 1;
    p.a1 = h[1] & mask;
    p.m2 = (h[2] & mask) | 1;
    p.a2 = h[3] & mask;
    p.mask = mask;
    p.sh = (uint64_t)(scale / 2 + 1 > 1 ? scale / 2 + 1 : 1);
    return p;
}

// keys: device uint64[2 * (edgefactor << scale)]
int tqgen_kron_keys(int scale, int edgefactor, uint64_t seed, uint64_t *keys, void *stream)
{
    if (scale < 1 || scale > 31 || edgefactor < 1 || !keys) return -1;
    const uint64_t m = (uint64_t)edgefactor << scale;
    kron_keys_kernel<<<grid_for((int64_t)m), 256, 0, (cudaStream_t)stream>>>(
        scale, m, mix64(seed), make_perm(scale, seed), keys);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// keys: device uint64[4 * rows * cols]
int tqgen_grid_keys(int64_t rows, int64_t cols, uint64_t *keys, void *stream)
{
    if (rows < 1 || cols < 1 || !keys) return -1;
    grid_keys_kernel<<<grid_for(rows * cols), 256, 0, (cudaStream_t)stream>>>(rows, cols, keys);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// weights: device int32[nnz]; same values as inputs/graphs.py:edge_weights
int tqgen_edge_weights(const int64_t *row_ptr, const int32_t *col, int64_t nv, uint64_t seed,
                       uint32_t wmax, int32_t *w, void *stream)
{
    if (!row_ptr || nv < 1 || wmax < 1 || !w) return -1;
    edge_weights_kernel<<<grid_for(nv), 256, 0, (cudaStream_t)stream>>>(
        row_ptr, col, nv, mix64(seed ^ 0x77E16475ull), wmax, w);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// keys: device uint64[2 * n]
int tqgen_tree4_keys(int64_t n, uint64_t *keys, void *stream)
{
    if (n < 1 || !keys) return -1;
    tree4_keys_kernel<<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(n, keys);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

// Sort `keys` ascending (radix sort over `end_bit` bits, plus the ~0 invalid
// marker), drop duplicates and invalid (~0) keys.  Result in `keys`, count in
// *n_out.  `alt` is caller-provided scratch of the same size.
int tqgen_sort_unique(uint64_t *keys, uint64_t *alt, int64_t n, int64_t *n_out, void *stream_)
{
    cudaStream_t stream = (cudaStream_t)stream_;
    if (!keys || !alt || n < 0 || !n_out) return -1;
    *n_out = 0;
    if (n == 0) return 0;
    cub::DoubleBuffer<uint64_t> db(keys, alt);
    size_t tmp_bytes = 0, tmp2 = 0;
    cudaError_t e = cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, db, n, 0, 64, stream);
    int64_t *d_count = nullptr;
    e = e == cudaSuccess ? cub::DeviceSelect::Unique(nullptr, tmp2, keys, alt, d_count, n, stream) : e;
    if (tmp2 > tmp_bytes) tmp_bytes = tmp2;
    tmp_bytes = (tmp_bytes + 255) & ~(size_t)255;  // d_count follows, 8-byte aligned
    void *tmp = nullptr;
    if (e == cudaSuccess) e = cudaMalloc(&tmp, tmp_bytes + 256);
    if (e == cudaSuccess) {
        d_count = (int64_t *)((char *)tmp + tmp_bytes);
        e = cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, n, 0, 64, stream);
    }
    uint64_t *sorted = db.Current();
    uint64_t *other = db.Alternate();
    if (e == cudaSuccess) e = cub::DeviceSelect::Unique(tmp, tmp2, sorted, other, d_count, n, stream);
    int64_t cnt = 0;
    if (e == cudaSuccess) e = cudaMemcpyAsync(&cnt, d_count, sizeof(cnt), cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    // drop the trailing ~0 marker (at most one after Unique)
    uint64_t last = 0;
    if (e == cudaSuccess && cnt > 0) {
        e = cudaMemcpy(&last, other + cnt - 1, sizeof(last), cudaMemcpyDeviceToHost);
        if (last == ~0ull) --cnt;
    }
    if (e == cudaSuccess && other != keys)
        e = cudaMemcpyAsync(keys, other, (size_t)cnt * sizeof(uint64_t), cudaMemcpyDeviceToDevice, stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    cudaFree(tmp);
    if (e != cudaSuccess) return -2;
    *n_out = cnt;
    return 0;
}

// keys sorted unique (u * nv + v); row_ptr int64[nv+1], col int32[n_keys]
int tqgen_keys_to_csr(const uint64_t *keys, int64_t n_keys, int64_t nv, int64_t *row_ptr,
                      int32_t *col, void *stream)
{
    if (!keys || !row_ptr || (!col && n_keys) || nv < 1) return -1;
    keys_to_csr_kernel<<<grid_for(n_keys > nv ? n_keys : nv + 1), 256, 0, (cudaStream_t)stream>>>(
        keys, n_keys, nv, row_ptr, col);
    return cudaGetLastError() == cudaSuccess ? 0 : -2;
}

}  // extern "C"
