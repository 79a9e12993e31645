// probe_paths.cu -- measurement tool (not product code): random 1-byte probe
// throughput on B200 by path, to decide where the BFS level prefilter should
// live.  Indices stream coalesced (4 B each) as in the BFS col stream; each
// lane has KP probes in flight; 256-thread blocks x 6 per SM.
//   mode 0: ld.global.cg (L2), mode 1: ld.global.ca (L1-allocating),
//   mode 2: shared memory table (the first `smem` bytes, copied per block).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pp scripts/probe_paths.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE, int KP>
__global__ void __launch_bounds__(256, 6) probe_kernel(const uint32_t *idx, long long n, const uint8_t *tab,
                                                       unsigned smem_bytes, unsigned long long *sink)
{
    extern __shared__ uint8_t st[];
    if (MODE == 2) {
        for (unsigned i = threadIdx.x; i < smem_bytes / 4; i += blockDim.x)
            ((uint32_t *)st)[i] = ((const uint32_t *)tab)[i];
        __syncthreads();
    }
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long stride = (long long)gridDim.x * blockDim.x;
    unsigned acc = 0;
    for (long long i = tid; i < n; i += KP * stride) {
        uint32_t u[KP];
#pragma unroll
        for (int j = 0; j < KP; ++j) u[j] = (i + j * stride < n) ? __ldg(idx + i + j * stride) : 0u;
        unsigned m[KP];
#pragma unroll
        for (int j = 0; j < KP; ++j) {
            if (MODE == 0) asm volatile("ld.global.cg.u8 %0, [%1];" : "=r"(m[j]) : "l"(tab + u[j]));
            else if (MODE == 1) asm volatile("ld.global.ca.u8 %0, [%1];" : "=r"(m[j]) : "l"(tab + u[j]));
            else m[j] = st[u[j]];
        }
#pragma unroll
        for (int j = 0; j < KP; ++j) acc += m[j];
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

template <int MODE, int KP>
static void run(const uint32_t *idx, long long n, const uint8_t *tab, unsigned range, unsigned smem,
                unsigned long long *sink, int sms)
{
    auto k = probe_kernel<MODE, KP>;
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, 256, MODE == 2 ? smem : 0);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    k<<<sms * occ, 256, MODE == 2 ? smem : 0>>>(idx, n, tab, smem, sink);
    cudaEventRecord(a);
    k<<<sms * occ, 256, MODE == 2 ? smem : 0>>>(idx, n, tab, smem, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    printf("{\"mode\": %d, \"kp\": %d, \"table_bytes\": %u, \"blocks_per_sm\": %d, \"ms\": %.3f, "
           "\"g_probes_per_s\": %.1f, \"err\": \"%s\"}\n", MODE, KP, range, occ, ms, n / (ms * 1e-3) / 1e9,
           cudaGetErrorString(cudaGetLastError()));
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long long n = 1ll << 28;
    uint32_t *idx;
    uint8_t *tab;
    unsigned long long *sink;
    cudaMalloc(&idx, n * 4);
    cudaMalloc(&tab, 1ull << 26);
    cudaMalloc(&sink, 8);
    cudaMemset(tab, 1, 1ull << 26);
    for (uint32_t range : {4096u, 16384u, 32768u, 65536u, 1u << 20, 16u << 20}) {
        fill_idx<<<sms * 8, 256>>>(idx, n, range, 12345);
        run<0, 4>(idx, n, tab, range, 0, sink, sms);
        run<1, 4>(idx, n, tab, range, 0, sink, sms);
        run<0, 8>(idx, n, tab, range, 0, sink, sms);
        run<1, 8>(idx, n, tab, range, 0, sink, sms);
        if (range <= 32768u) {
            run<2, 4>(idx, n, tab, range, range, sink, sms);
            run<2, 8>(idx, n, tab, range, range, sink, sms);
        }
    }
    return 0;
}
