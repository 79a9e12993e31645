// probe_ceiling.cu -- measurement tool (not product code): the random-probe
// ceiling that bounds top-down BFS expansion on B200.  Each lane streams
// 4-byte indices from a large array (like `col`) and probes a random byte of
// a table (like the level mirror) with ld.global.cg, 4 probes in flight per
// lane, at the BFS kernel's occupancy (256-thread blocks, 6 per SM).
// Prints G probes/s for table sizes 16 MB .. 512 MB.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe scripts/probe_ceiling.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_cg_u8(const uint8_t *p)
{
    unsigned v;
    asm volatile("ld.global.cg.u8 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__global__ void __launch_bounds__(256, 6) probe_kernel(const uint32_t *idx, long long n, const uint8_t *tab,
                                                       unsigned long long *sink)
{
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long stride = (long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (long long i = tid; i < n; i += 4 * stride) {
        uint32_t u[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) u[j] = (i + j * stride < n) ? __ldg(idx + i + j * stride) : 0u;
        unsigned m[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) m[j] = ld_cg_u8(tab + u[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) acc += m[j];
    }
    if (acc == 0xdeadbeef) *sink = acc;
}

__global__ void fill_idx(uint32_t *idx, long long n, uint32_t range, unsigned long long seed)
{
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        unsigned long long x = (i + 1) * 0x9E3779B97F4A7C15ull ^ seed;
        x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29;
        idx[i] = (uint32_t)(x % range);
    }
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long long n = 1ll << 29;  // 512M probes (2 GB of indices)
    uint32_t *idx;
    uint8_t *tab;
    unsigned long long *sink;
    cudaMalloc(&idx, n * 4);
    cudaMalloc(&tab, 1ull << 29);
    cudaMalloc(&sink, 8);
    cudaMemset(tab, 1, 1ull << 29);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, probe_kernel, 256, 0);
    printf("{\"sms\": %d, \"blocks_per_sm\": %d}\n", sms, occ);
    for (uint32_t mb : {16u, 67u, 128u, 512u}) {
        const uint32_t range = mb << 20;
        fill_idx<<<sms * 8, 256>>>(idx, n, range, 12345);
        probe_kernel<<<sms * occ, 256>>>(idx, n, tab, sink);  // warm-up
        cudaEventRecord(a);
        probe_kernel<<<sms * occ, 256>>>(idx, n, tab, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        printf("{\"table_mb\": %u, \"probes\": %lld, \"ms\": %.3f, \"g_probes_per_s\": %.1f, "
               "\"index_gbs\": %.0f}\n", mb, n, ms, n / (ms * 1e-3) / 1e9, n * 4.0 / (ms * 1e-3) / 1e9);
    }
    return 0;
}
