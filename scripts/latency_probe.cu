// Dependent-access latency of the memory operations on the BFS hop chain
// (single warp, lane 0, L2-resident 1 MB table, pointer chase): plain,
// .cg, .nc, ld.relaxed.gpu, ld.acquire.gpu loads, atom.add / atom.min /
// atom.cas, and fence.release / fence.acq_rel + load.  Cycles per access.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o latency_probe latency_probe.cu
#include <cstdio>
#include <cuda_runtime.h>

enum { PLAIN, CG, NC, RELAXED, ACQUIRE, ATOM_ADD, ATOM_MIN, ATOM_CAS, REL_FENCE_LD, ACQREL_FENCE_LD, STORE_FENCE, NKIND };
static const char *names[NKIND] = {"ld (default)", "ld.cg", "ld.nc", "ld.relaxed.gpu", "ld.acquire.gpu", "atom.add.u64",
                                   "atom.min.u64", "atom.cas.b64", "fence.release + ld.relaxed", "fence.acq_rel + ld.relaxed",
                                   "st.relaxed + fence.release + ld.relaxed"};

__global__ void chase(unsigned long long *tab, int kind, int iters, unsigned long long *out)
{
    if (threadIdx.x != 0) return;
    unsigned long long i = 0, acc = 0;
    long long t0 = clock64();
    for (int k = 0; k < iters; ++k) {
        unsigned long long *p = tab + i;
        unsigned long long v;
        switch (kind) {
        case PLAIN: v = *(volatile unsigned long long *)p; break;
        case CG: asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p)); break;
        case NC: asm volatile("ld.global.nc.u64 %0, [%1];" : "=l"(v) : "l"(p)); break;
        case RELAXED: asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); break;
        case ACQUIRE: asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); break;
        case ATOM_ADD: asm volatile("atom.relaxed.gpu.global.add.u64 %0, [%1], 0;" : "=l"(v) : "l"(p) : "memory"); break;
        case ATOM_MIN: asm volatile("atom.relaxed.gpu.global.min.u64 %0, [%1], 0xffffffffffffffff;" : "=l"(v) : "l"(p) : "memory"); break;
        case ATOM_CAS: asm volatile("atom.relaxed.gpu.global.cas.b64 %0, [%1], 1, 2;" : "=l"(v) : "l"(p) : "memory"); break;
        case REL_FENCE_LD:
            asm volatile("fence.release.gpu;" ::: "memory");
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
            break;
        case ACQREL_FENCE_LD:
            asm volatile("fence.acq_rel.gpu;" ::: "memory");
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
            break;
        default:
            asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(out + 8), "l"(acc) : "memory");
            asm volatile("fence.release.gpu;" ::: "memory");
            asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
            break;
        }
        acc += v;
        i = v & 0x1ffffull;  // next index (the table holds a random cycle)
    }
    long long t1 = clock64();
    out[0] = (unsigned long long)(t1 - t0);
    out[1] = acc;
}

int main()
{
    const int n = 1 << 17;  // 1 MB of u64
    unsigned long long *h = new unsigned long long[n];
    // random single cycle over n entries, stride > a line
    unsigned *perm = new unsigned[n];
    for (int k = 0; k < n; ++k) perm[k] = k;
    unsigned long long s = 88172645463325252ull;
    for (int k = n - 1; k > 0; --k) {
        s ^= s << 13; s ^= s >> 7; s ^= s << 17;
        int j = (int)(s % (unsigned long long)(k + 1));
        unsigned t = perm[k]; perm[k] = perm[j]; perm[j] = t;
    }
    for (int k = 0; k < n; ++k) h[perm[k]] = perm[(k + 1) % n];
    unsigned long long *tab, *out;
    cudaMalloc(&tab, n * 8);
    cudaMalloc(&out, 16 * 8);
    const int iters = 4096;
    for (int kind = 0; kind < NKIND; ++kind) {
        cudaMemcpy(tab, h, n * 8, cudaMemcpyHostToDevice);
        chase<<<1, 32>>>(tab, kind, iters, out);  // warm L2
        cudaMemcpy(tab, h, n * 8, cudaMemcpyHostToDevice);
        chase<<<1, 32>>>(tab, kind, 1 << 17, out);
        chase<<<1, 32>>>(tab, kind, iters, out);
        unsigned long long o[2];
        cudaMemcpy(o, out, 16, cudaMemcpyDeviceToHost);
        printf("{\"op\": \"%s\", \"cycles_per_access\": %.1f}\n", names[kind], (double)o[0] / iters);
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) printf("error %s\n", cudaGetErrorString(e));
    return 0;
}
