// Does a kernel on stream A start while a large D2H copy on stream B runs?
// nvcc -gencode arch=compute_100a,code=sm_100a -o build/overlap_probe scripts/overlap_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void spin(unsigned long long ns)
{
    unsigned long long t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    for (;;) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (t - t0 > ns) break;
    }
}

__global__ void zcopy(const int4 *__restrict__ s, int4 *d, size_t n)
{
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        d[i] = s[i];
}

#define CK(x)                                                                   \
    do {                                                                        \
        cudaError_t e_ = (x);                                                   \
        if (e_ != cudaSuccess) {                                                \
            printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            return 1;                                                           \
        }                                                                       \
    } while (0)

int main()
{
    float c, k1;
    const size_t bytes = 512ull << 20;
    void *d, *h, *hp;
    CK(cudaMalloc(&d, bytes));
    CK(cudaMallocHost(&h, bytes));
    hp = malloc(bytes);
    cudaStream_t a, b;
    CK(cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking));
    cudaEvent_t e[6];
    for (auto &x : e) CK(cudaEventCreate(&x));
    for (int kind = 0; kind < 4; ++kind) {
        CK(cudaDeviceSynchronize());
        // kind 0: D2H pinned; 1: H2D pinned; 2: D2D; 3: D2H pinned, kernel 1 SM
        CK(cudaEventRecord(e[0], a));
        CK(cudaStreamWaitEvent(b, e[0], 0));
        if (kind == 0 || kind == 3) CK(cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, b));
        if (kind == 1) CK(cudaMemcpyAsync(d, h, bytes, cudaMemcpyHostToDevice, b));
        if (kind == 2) CK(cudaMemcpyAsync((char *)d + bytes / 2, d, bytes / 2, cudaMemcpyDeviceToDevice, b));
        CK(cudaEventRecord(e[1], b));
        CK(cudaEventRecord(e[2], a));
        spin<<<kind == 3 ? 1 : 148 * 4, 256, 0, a>>>(2000000);
        CK(cudaEventRecord(e[3], a));
        CK(cudaDeviceSynchronize());
        float c, k0, k1;
        cudaEventElapsedTime(&c, e[0], e[1]);
        cudaEventElapsedTime(&k0, e[0], e[2]);
        cudaEventElapsedTime(&k1, e[0], e[3]);
        printf("kind %d: copy end %.2f ms, kernel-stream event %.2f ms, 2ms kernel end %.2f ms\n", kind, c, k0, k1);
    }
    // reverse order: kernel first, then copy
    CK(cudaEventRecord(e[0], a));
    spin<<<148 * 4, 256, 0, a>>>(2000000);
    CK(cudaEventRecord(e[3], a));
    CK(cudaStreamWaitEvent(b, e[0], 0));
    CK(cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, b));
    CK(cudaEventRecord(e[1], b));
    CK(cudaDeviceSynchronize());
    cudaEventElapsedTime(&c, e[0], e[1]);
    cudaEventElapsedTime(&k1, e[0], e[3]);
    printf("kernel then D2H: copy end %.2f ms, kernel end %.2f ms\n", c, k1);
    // chunked D2H (64 x 8 MB), then the kernel
    {
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e[0], a));
        CK(cudaStreamWaitEvent(b, e[0], 0));
        for (int i = 0; i < 64; ++i)
            CK(cudaMemcpyAsync((char *)h + i * (bytes / 64), (char *)d + i * (bytes / 64), bytes / 64,
                               cudaMemcpyDeviceToHost, b));
        CK(cudaEventRecord(e[1], b));
        spin<<<148 * 4, 256, 0, a>>>(2000000);
        CK(cudaEventRecord(e[3], a));
        CK(cudaDeviceSynchronize());
        cudaEventElapsedTime(&c, e[0], e[1]);
        cudaEventElapsedTime(&k1, e[0], e[3]);
        printf("chunked D2H then kernel: copy end %.2f ms, kernel end %.2f ms\n", c, k1);
    }
    // zero-copy: device stores into mapped pinned memory, alone and beside a
    // kernel holding 6 x 256 threads per SM (the persistent BFS footprint)
    {
        void *hd;
        CK(cudaHostGetDevicePointer(&hd, h, 0));
        for (int blocks : {148, 296, 592}) {
            CK(cudaDeviceSynchronize());
            CK(cudaEventRecord(e[0], b));
            zcopy<<<blocks, 256, 0, b>>>((const int4 *)d, (int4 *)hd, bytes / 16);
            CK(cudaEventRecord(e[1], b));
            CK(cudaDeviceSynchronize());
            cudaEventElapsedTime(&c, e[0], e[1]);
            printf("zero-copy %d blocks alone: %.2f ms = %.1f GB/s\n", blocks, c, bytes / c / 1e6);
        }
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e[0], a));
        spin<<<148 * 6, 256, 0, a>>>(20000000);
        CK(cudaEventRecord(e[3], a));
        CK(cudaStreamWaitEvent(b, e[0], 0));
        zcopy<<<148, 128, 0, b>>>((const int4 *)d, (int4 *)hd, bytes / 16);
        CK(cudaEventRecord(e[1], b));
        CK(cudaDeviceSynchronize());
        cudaEventElapsedTime(&c, e[0], e[1]);
        cudaEventElapsedTime(&k1, e[0], e[3]);
        printf("zero-copy 148x128 beside a 20 ms 6x256/SM kernel: copy end %.2f ms, kernel end %.2f ms\n", c, k1);
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e[0], a));
        spin<<<148 * 6, 256, 0, a>>>(20000000);
        CK(cudaEventRecord(e[3], a));
        CK(cudaStreamWaitEvent(b, e[0], 0));
        CK(cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, b));
        CK(cudaEventRecord(e[1], b));
        CK(cudaDeviceSynchronize());
        cudaEventElapsedTime(&c, e[0], e[1]);
        cudaEventElapsedTime(&k1, e[0], e[3]);
        printf("D2H memcpy beside a 20 ms 6x256/SM kernel: copy end %.2f ms, kernel end %.2f ms\n", c, k1);
    }
    // the run_batch pipeline: kernel i+1 on stream a while root i's output
    // drains on stream b; host waits for kernel i (stream a) each iteration
    unsigned long long *small_h;
    CK(cudaMallocHost(&small_h, 4096));
    for (int variant = 0; variant < 6; ++variant) {
        const int chunked = variant & 1, smallcp = variant >= 2, bigrid = variant >= 4;
        cudaEvent_t kd[2], cd[2];
        for (int i = 0; i < 2; ++i) {
            CK(cudaEventCreateWithFlags(&kd[i], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&cd[i], cudaEventDisableTiming));
            CK(cudaEventRecord(cd[i], b));
        }
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e[0], a));
        const int K = 6;
        for (int i = 0; i < K; ++i) {
            const int j = i & 1;
            CK(cudaStreamWaitEvent(a, cd[j], 0));
            if (bigrid) zcopy<<<262144, 256, 0, a>>>((const int4 *)d, (int4 *)d + (bytes / 32), bytes / 32);
            spin<<<148 * 6, 256, 0, a>>>(18000000);
            if (smallcp)
                for (int t = 0; t < 6; ++t)
                    CK(cudaMemcpyAsync(small_h + t * 16, (char *)d + t * 4096, 64, cudaMemcpyDeviceToHost, a));
            CK(cudaEventRecord(kd[j], a));
            CK(cudaStreamWaitEvent(b, kd[j], 0));
            if (chunked) {
                for (size_t off = 0; off < bytes; off += 8 << 20)
                    CK(cudaMemcpyAsync((char *)h + off, (char *)d + off, 8 << 20, cudaMemcpyDeviceToHost, b));
            } else {
                CK(cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, b));
            }
            CK(cudaEventRecord(cd[j], b));
            CK(cudaStreamSynchronize(a));
        }
        CK(cudaStreamSynchronize(b));
        CK(cudaEventRecord(e[1], a));
        CK(cudaDeviceSynchronize());
        cudaEventElapsedTime(&c, e[0], e[1]);
        printf("pipeline (18 ms kernel + 512 MiB D2H, %s, small D2H on kernel stream %d, big-grid kernel %d): %.2f ms per iteration\n",
               chunked ? "8 MiB pieces" : "one copy", smallcp, bigrid, c / K);
    }
    free(hp);
    return 0;
}
