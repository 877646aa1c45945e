/*
 * microbench.cu — measured ceilings for the roofline: the 64-bit atomicCAS /
 * coherent-load rate on distinct words (L2-resident and HBM-resident arrays, coalesced and
 * random patterns) and the cost of one grid barrier of the persistent replay kernel.  Timed
 * with CUDA events on the caller's stream.  Not part of the checking path.
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace.h"
#include "hirace_device.cuh"
#include "internal.h"
#include "kernel_common.cuh"

namespace hirace_impl {
namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t x)
{
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    x *= 0xc4ceb9fe1a85ec53ull;
    x ^= x >> 33;
    return x;
}

/* op 0: CAS that always succeeds (expected value tracked per word), 1: atomicAdd, 2: coherent
 * load, 3: load + CAS (the replay's read-modify-write pair) */
__global__ void __launch_bounds__(256) k_mb_atomics(unsigned long long *a, uint64_t nwords, uint64_t per_thread,
                                                    int random, int op, unsigned long long *sink)
{
    const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t nthreads = (uint64_t)gridDim.x * blockDim.x;
    unsigned long long acc = 0;
    for (uint64_t k = 0; k < per_thread; k++) {
        const uint64_t j = k * nthreads + tid;
        const uint64_t w = random ? mix64(j) % nwords : j % nwords;
        unsigned long long *p = a + w;
        if (op == 0) {
            acc += atomicCAS(p, 0ull, 0ull);
        } else if (op == 1) {
            acc += atomicAdd(p, 1ull);
        } else if (op == 2) {
            acc += hirace::ld_coherent(p);
        } else {
            const unsigned long long o = hirace::ld_coherent(p);
            acc += atomicCAS(p, o, o + 1);
        }
    }
    if (acc == 0x123456789ull)
        *sink = acc;
}

/* barrier variants: 0 = grid_sync (library), 1 = no sleep while polling, 2 = last arriver
 * flips a separate generation flag that the others poll */
__device__ __forceinline__ void grid_sync_variant(unsigned int *bar, unsigned int nctas, unsigned int &epoch,
                                                  int mode)
{
    if (mode == 0) {
        grid_sync(bar, nctas, epoch);
        return;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        epoch++;
        if (mode == 1) {
            const unsigned int target = epoch * nctas;
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
            unsigned int v;
            do {
                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
            } while (v < target);
        } else {
            unsigned int *flag = bar + 32; /* another 128-byte line */
            unsigned int old;
            asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(bar) : "memory");
            if (old == epoch * nctas - 1) {
                asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag), "r"(epoch) : "memory");
            } else {
                unsigned int v;
                do {
                    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
                } while (v < epoch);
            }
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kReplayThreads) k_mb_grid_sync(unsigned int *bar, int iters, int mode)
{
    unsigned int epoch = 0;
    for (int i = 0; i < iters; i++)
        grid_sync_variant(bar, gridDim.x, epoch, mode);
}

/* the words listed in idx[0..n), grid-stride (consecutive threads take consecutive list
 * entries): op 2 = coherent load, 3 = load + CAS.  The list's order is the access pattern
 * (random, sorted, window-major ...), chosen by the caller. */
__global__ void __launch_bounds__(256) k_mb_indexed(unsigned long long *a, const unsigned long long *__restrict__ idx,
                                                    uint64_t n, int op, unsigned long long *sink)
{
    unsigned long long acc = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long *p = a + __ldcs(idx + i);
        const unsigned long long o = hirace::ld_coherent(p);
        if (op == 3)
            acc += atomicCAS(p, o, o + 1);
        else
            acc += o;
    }
    if (acc == 0x123456789ull)
        *sink = acc;
}

} // namespace
} // namespace hirace_impl

using namespace hirace_impl;

extern "C" hirace_status hirace_microbench_indexed(int device, void *words, const void *idx, uint64_t n, int op,
                                                   int ctas_per_sm, double *ms_out, void *stream)
{
    if (!ms_out || !words || (n && !idx) || (op != 2 && op != 3) || ctas_per_sm < 1)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaSetDevice(device) != cudaSuccess)
        return HIRACE_E_CUDA;
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0, st);
    k_mb_indexed<<<sms * ctas_per_sm, 256, 0, st>>>((unsigned long long *)words, (const unsigned long long *)idx, n, op,
                                                    (unsigned long long *)words);
    cudaEventRecord(e1, st);
    float ms = 0;
    hirace_status s = HIRACE_OK;
    if (cudaEventSynchronize(e1) != cudaSuccess || cudaEventElapsedTime(&ms, e0, e1) != cudaSuccess)
        s = HIRACE_E_CUDA;
    *ms_out = ms;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    return s;
}

extern "C" hirace_status hirace_microbench_atomics(int device, uint64_t nwords, int random, int op, uint64_t nops,
                                                   double *ops_per_s, void *stream)
{
    if (!ops_per_s || nwords == 0 || op < 0 || op > 3)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaSetDevice(device) != cudaSuccess)
        return HIRACE_E_CUDA;
    unsigned long long *a = nullptr, *sink = nullptr;
    if (cudaMalloc(&a, nwords * 8) != cudaSuccess)
        return HIRACE_E_NOMEM;
    cudaMalloc(&sink, 8);
    cudaMemsetAsync(a, 0, nwords * 8, st);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    const int grid = sms * 8;
    const uint64_t nthreads = (uint64_t)grid * 256;
    const uint64_t per = (nops + nthreads - 1) / nthreads;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_mb_atomics<<<grid, 256, 0, st>>>(a, nwords, per, random, op, sink); /* warm-up */
    cudaEventRecord(e0, st);
    k_mb_atomics<<<grid, 256, 0, st>>>(a, nwords, per, random, op, sink);
    cudaEventRecord(e1, st);
    hirace_status s = HIRACE_OK;
    float ms = 0;
    if (cudaEventSynchronize(e1) != cudaSuccess || cudaEventElapsedTime(&ms, e0, e1) != cudaSuccess)
        s = HIRACE_E_CUDA;
    else
        *ops_per_s = (double)per * nthreads / (ms * 1e-3);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(a);
    cudaFree(sink);
    return s;
}

extern "C" hirace_status hirace_microbench_grid_sync(int device, int iters, int mode, double *us_per_barrier,
                                                     void *stream)
{
    if (!us_per_barrier || iters < 1)
        return HIRACE_E_INVAL;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaSetDevice(device) != cudaSuccess)
        return HIRACE_E_CUDA;
    unsigned int *bar = nullptr;
    if (cudaMalloc(&bar, 64 * sizeof(unsigned int)) != cudaSuccess)
        return HIRACE_E_NOMEM;
    const int grid = replay_max_grid(device);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms[2] = {0, 0};
    hirace_status s = HIRACE_OK;
    for (int rep = 0; rep < 2; rep++) { /* iters and 1 barrier: the difference is the barrier cost */
        int it = rep == 0 ? iters : 1;
        void *args[] = {&bar, &it, &mode};
        cudaMemsetAsync(bar, 0, 64 * sizeof(unsigned int), st);
        cudaEventRecord(e0, st);
        if (cudaLaunchCooperativeKernel((const void *)k_mb_grid_sync, dim3(grid), dim3(kReplayThreads), args, 0, st) !=
            cudaSuccess)
            s = HIRACE_E_CUDA;
        cudaEventRecord(e1, st);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms[rep], e0, e1);
    }
    if (s == HIRACE_OK)
        *us_per_barrier = (ms[0] - ms[1]) * 1e3 / (iters - 1 > 0 ? iters - 1 : 1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(bar);
    return s;
}
