/* kernel_common.cuh — device helpers shared by the library's kernels (sm_100a). */
#ifndef HIRACE_KERNEL_COMMON_CUH
#define HIRACE_KERNEL_COMMON_CUH

#include <cuda_runtime.h>
#include <stdint.h>

#include "hirace.h"

#ifndef HIRACE_BAR_ACQLOAD
#define HIRACE_BAR_ACQLOAD 1
#endif

namespace hirace_impl {

/* batch key (g,b,w) of event p = meta >> 5 */
__device__ __forceinline__ uint32_t batch_key_at(const hirace_event *ev, uint32_t p)
{
    return __ldg(&ev[p].meta) >> 5;
}

/* Grid-wide barrier for a cooperative launch (all CTAs co-resident): monotone arrival counter,
 * release on arrive, acquire on the spin, so shadow CASes before the barrier are visible to
 * every CTA after it (batch order = a linear extension of happens-before). */
__device__ __forceinline__ void grid_sync(unsigned int *bar, unsigned int nctas, unsigned int &epoch)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        epoch++;
        const unsigned int target = epoch * nctas;
        /* bar.sync above orders the CTA's accesses before this release (cumulativity) */
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
        unsigned int v;
        for (;;) { /* relaxed busy poll (no sleep: 1.5 vs 2.9 us per barrier on B200, no L1
                      * invalidation per poll), one acquire fence after */
            asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
            if (v >= target)
                break;
#ifdef HIRACE_BAR_SLEEP
            __nanosleep(HIRACE_BAR_SLEEP);
#endif
        }
#if HIRACE_BAR_ACQLOAD
        /* one acquire load of the counter: it reads the last arrival's value, so it synchronises
         * with every red.release of the release sequence (instead of a full acq_rel fence) */
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
#else
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
    }
    __syncthreads();
}

/* ---- mbarrier + 1-D bulk async copy (TMA engine, no tensor map needed) -------------------- */

__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init()
{
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t *bar)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
    uint32_t done = 0;
    while (!done) {
        asm volatile("{\n\t.reg .pred p;\n\t"
                     "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done)
                     : "r"(smem_u32(bar)), "r"(parity)
                     : "memory");
    }
}

/* global -> shared bulk copy completing on an mbarrier (bytes % 16 == 0, 16-B aligned) */
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar)
{
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

} // namespace hirace_impl

#endif
