// devapi_test.cu -- TEST ONLY: a user kernel compiled against the public
// device API (include/tq_device.cuh) of the retry-free, arbitrary-n queue.
//
// Every warp runs `rounds` rounds of
//   tq_warp_enqueue_n<32>: lane i enqueues nmine[i] (0..32) items with one
//                          AFA on Rear for the warp (Listing 3, P:240-273;
//                          arbitrary n),
//   tq_warp_dequeue_n:     the warp then dequeues as many tickets as it
//                          enqueued, <= 32 hungry lanes per reservation
//                          (Listing 1),
//   tq_take / tq_poll:     each ticket holder polls its slot until its item
//                          arrives (Listing 2),
// logging ticket -> item on both sides, so tests/test_gpu_devapi.py can replay
// the run through the oracle's sequential ticket model.  A warp dequeues only
// after it enqueued the same count, so Front <= Rear always and every polled
// ticket is reserved by a producer that publishes without waiting: the run
// terminates unless the queue-full abort fires (then pollers bail out).
#include <cuda_runtime.h>
#include <stdint.h>

#include "tq_device.cuh"

namespace {

__global__ void devapi_kernel(tq_device_view q, int rounds, const unsigned *nmine, unsigned long long t0,
                              unsigned *enq_log, unsigned *deq_log, unsigned long long log_len, int use_poll,
                              unsigned long long timeout_ns, unsigned long long *out)
{
    const unsigned lane = tq_lane();
    const unsigned warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    unsigned atomics = 0;
    const unsigned long long deadline = tq_globaltimer() + timeout_ns;
    bool bail = false;
    for (int r = 0; r < rounds && !bail; ++r) {
        const unsigned idx = (warp * (unsigned)rounds + (unsigned)r) * 32u + lane;
        const unsigned n = nmine[idx];
        unsigned items[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) items[j] = idx * 32u + (unsigned)j;  // unique ids
        const unsigned long long first = tq_warp_enqueue_n<32>(q, n, items, &atomics);
        if (first != TQ_NO_TICKET) {
            for (unsigned j = 0; j < n; ++j) {
                const unsigned long long k = first + j - t0;
                if (k < log_len) enq_log[k] = items[j];
            }
        }
        const unsigned total = __reduce_add_sync(TQ_FULL_MASK, n);
        for (unsigned got = 0; got < total && !bail; got += 32) {
            const bool hungry = lane < min(32u, total - got);
            const unsigned long long t = tq_warp_dequeue_n(q, hungry, &atomics);
            bool stop = false;
            if (hungry) {
                for (;;) {
                    unsigned item = 0;
                    bool ok;
                    if (use_poll) {
                        // the arrival check alone, then the caller's take
                        ok = tq_poll(q, t, &item);
                        if (ok) tq_st_relaxed(q.slots + (t & q.mask), (unsigned long long)(unsigned)(t + q.mask + 1));
                    } else {
                        ok = tq_take(q, t, &item);
                    }
                    if (ok) {
                        const unsigned long long k = t - t0;
                        if (k < log_len) deq_log[k] = item;
                        atomicAdd(out + 1, 1ull);
                        break;
                    }
                    if (tq_status_read(q, warp) != TQ_RUNNING) {
                        stop = true;
                        break;
                    }
                    if (tq_globaltimer() > deadline) {
                        tq_status_set_thread(q, TQ_ABORTED_TIMEOUT);
                        stop = true;
                        break;
                    }
                }
            }
            bail = __any_sync(TQ_FULL_MASK, stop);
        }
        if (first != TQ_NO_TICKET) atomicAdd(out + 0, (unsigned long long)n);
        bail = bail || __any_sync(TQ_FULL_MASK, first == TQ_NO_TICKET);
    }
    if (lane == 0) atomicAdd(out + 2, (unsigned long long)atomics);
}

}  // namespace

extern "C" int devapi_run(const tq_device_view *v, int warps, int rounds, const unsigned *nmine,
                          unsigned long long t0, unsigned *enq_log, unsigned *deq_log,
                          unsigned long long log_len, int use_poll, double timeout_s, unsigned long long *out,
                          void *stream)
{
    if (!v || warps < 1 || rounds < 1 || !nmine || !out) return -1;
    const int wpb = warps < 8 ? warps : 8;
    if (warps % wpb) return -1;
    devapi_kernel<<<warps / wpb, 32 * wpb, 0, (cudaStream_t)stream>>>(
        *v, rounds, nmine, t0, enq_log, deq_log, log_len, use_poll,
        (unsigned long long)(timeout_s * 1e9), out);
    if (cudaGetLastError() != cudaSuccess) return -2;
    return cudaStreamSynchronize((cudaStream_t)stream) == cudaSuccess ? 0 : -2;
}
