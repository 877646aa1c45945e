/* record.cuh — the two shadow-record layouts behind one interface, so the replay and collect
 * kernels are written once and instantiated per layout:
 *   Rec<unsigned long long>  8-byte record (hirace_device.cuh: state:5 | g:8 | b:10 | w:9 | tid:32)
 *   Rec<unsigned int>        compact 4-byte record (hirace_shadow_alloc_compact, SURVEY §8(f) f1:
 *                            state:5 | g | b | w | tid, widths from the declared epoch limits;
 *                            PAPER.md L289, L419-423).
 * Both feed the same raw-flag FSM table (label_raw layout); the fields hold the same values,
 * so every transition is the same. */
#ifndef HIRACE_RECORD_CUH
#define HIRACE_RECORD_CUH

#include <stdint.h>

#include "hirace_device.cuh"

namespace hirace_impl {

template <typename R> struct Rec;

template <> struct Rec<unsigned long long> {
    __device__ __forceinline__ explicit Rec(const hirace_dev_ctx &) {}
    __device__ __forceinline__ uint32_t ep(uint32_t g, uint32_t b, uint32_t w) const
    {
        return (g << hirace::SH_G) | (b << hirace::SH_B) | (w << hirace::SH_W);
    }
    __device__ __forceinline__ bool fits(uint32_t, uint32_t, uint32_t) const { return true; }
    __device__ __forceinline__ uint32_t label(unsigned long long o, uint32_t tid, uint32_t kind, uint32_t ep,
                                              const hirace::geom &G) const
    {
        return hirace::label_raw_ep(o, tid, kind, ep, G);
    }
    __device__ __forceinline__ unsigned long long next(unsigned long long o, uint32_t e, uint32_t tid,
                                                       uint32_t ep) const
    {
        return (e & hirace::E_KEEP) ? ((o & ~31ull) | (e & hirace::E_STATE))
                                    : (((unsigned long long)tid << hirace::SH_TID) | ep | (e & hirace::E_STATE));
    }
    __device__ __forceinline__ uint32_t g(unsigned long long o) const { return hirace::g_of(o); }
    __device__ __forceinline__ uint32_t tid(unsigned long long o) const { return hirace::tid_of(o); }
    static __device__ __forceinline__ unsigned long long load(const unsigned long long *p)
    {
        return hirace::ld_coherent(p);
    }
    static __device__ __forceinline__ unsigned long long cas_if(unsigned long long *p, unsigned long long cmp,
                                                                unsigned long long val, bool pred)
    {
        return hirace::cas64_if(p, cmp, val, pred);
    }
    static __device__ __forceinline__ unsigned long long cas(unsigned long long *p, unsigned long long cmp,
                                                             unsigned long long val)
    {
        return atomicCAS(p, cmp, val);
    }
};

template <> struct Rec<unsigned int> {
    hirace::clay L;
    __device__ __forceinline__ explicit Rec(const hirace_dev_ctx &c) : L(hirace::clay_of(c)) {}
    __device__ __forceinline__ uint32_t ep(uint32_t g, uint32_t b, uint32_t w) const
    {
        return hirace::c_epochs(L, g, b, w);
    }
    __device__ __forceinline__ bool fits(uint32_t g, uint32_t b, uint32_t w) const { return hirace::c_fits(L, g, b, w); }
    __device__ __forceinline__ uint32_t label(unsigned int o, uint32_t tid, uint32_t kind, uint32_t ep,
                                              const hirace::geom &G) const
    {
        return hirace::label_raw_c(o, tid, kind, ep, L, G);
    }
    __device__ __forceinline__ unsigned int next(unsigned int o, uint32_t e, uint32_t tid, uint32_t ep) const
    {
        return hirace::next_c(o, e, tid, ep, L);
    }
    __device__ __forceinline__ uint32_t g(unsigned int o) const { return hirace::c_g(o, L); }
    __device__ __forceinline__ uint32_t tid(unsigned int o) const { return hirace::c_tid(o, L); }
    static __device__ __forceinline__ unsigned int load(const unsigned int *p) { return hirace::ld_coherent32(p); }
    static __device__ __forceinline__ unsigned int cas_if(unsigned int *p, unsigned int cmp, unsigned int val, bool pred)
    {
        return hirace::cas32_if(p, cmp, val, pred);
    }
    static __device__ __forceinline__ unsigned int cas(unsigned int *p, unsigned int cmp, unsigned int val)
    {
        return atomicCAS(p, cmp, val);
    }
};

template <typename R> __device__ __forceinline__ R *shadow_as(const hirace_dev_ctx &c)
{
    return reinterpret_cast<R *>(c.shadow);
}

} // namespace hirace_impl

#endif
