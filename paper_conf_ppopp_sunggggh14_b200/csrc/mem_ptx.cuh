// mem_ptx.cuh -- explicit-PTX global/shared memory accessors used by the libipt kernels.
#pragma once
#include <stdint.h>

namespace ipt {

// W-byte raw vector types (raw bit moves; no floating point anywhere).
template <int W> struct VecT;
template <> struct VecT<16> { using type = uint4; };
template <> struct VecT<8> { using type = uint2; };
template <> struct VecT<4> { using type = uint32_t; };
template <> struct VecT<2> { using type = uint32_t; };  // low 16 bits used
template <> struct VecT<1> { using type = uint32_t; };  // low 8 bits used

// L2-cached (L1-bypassing) loads/stores: every position is touched ~once per stage, and
// the claim protocol relies on reading the coherent (L2) copy.
template <int W> __device__ __forceinline__ typename VecT<W>::type ld_cg(const void *p);
template <> __device__ __forceinline__ uint4 ld_cg<16>(const void *p) {
    uint4 v;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint2 ld_cg<8>(const void *p) {
    uint2 v;
    asm volatile("ld.global.cg.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_cg<4>(const void *p) {
    uint32_t v;
    asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_cg<2>(const void *p) {
    uint16_t v;
    asm volatile("ld.global.cg.u16 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_cg<1>(const void *p) {
    uint16_t v;
    asm volatile("ld.global.cg.u8 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
    return v;
}

// Acquire loads (gpu scope): later memory operations of this thread are ordered after them.
template <int W> __device__ __forceinline__ typename VecT<W>::type ld_acq(const void *p);
template <> __device__ __forceinline__ uint4 ld_acq<16>(const void *p) {
    uint4 v;
    asm volatile("ld.acquire.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint2 ld_acq<8>(const void *p) {
    uint2 v;
    asm volatile("ld.acquire.gpu.global.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_acq<4>(const void *p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_acq<2>(const void *p) {
    uint16_t v;
    asm volatile("ld.acquire.gpu.global.u16 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
    return v;
}
template <> __device__ __forceinline__ uint32_t ld_acq<1>(const void *p) {
    uint16_t v;
    asm volatile("ld.acquire.gpu.global.u8 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
    return v;
}

template <int W> __device__ __forceinline__ void st_cg(void *p, const typename VecT<W>::type &v);
template <> __device__ __forceinline__ void st_cg<16>(void *p, const uint4 &v) {
    asm volatile("st.global.cg.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
template <> __device__ __forceinline__ void st_cg<8>(void *p, const uint2 &v) {
    asm volatile("st.global.cg.v2.u32 [%0], {%1,%2};" :: "l"(p), "r"(v.x), "r"(v.y) : "memory");
}
template <> __device__ __forceinline__ void st_cg<4>(void *p, const uint32_t &v) {
    asm volatile("st.global.cg.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
template <> __device__ __forceinline__ void st_cg<2>(void *p, const uint32_t &v) {
    uint16_t h = (uint16_t)v;
    asm volatile("st.global.cg.u16 [%0], %1;" :: "l"(p), "h"(h) : "memory");
}
template <> __device__ __forceinline__ void st_cg<1>(void *p, const uint32_t &v) {
    uint16_t h = (uint16_t)(v & 0xff);
    asm volatile("st.global.cg.u8 [%0], %1;" :: "l"(p), "h"(h) : "memory");
}

// OR-fold of a vector into 32 bits (feeds the address dependency below).
__device__ __forceinline__ uint32_t fold(const uint4 &v) { return v.x | v.y | v.z | v.w; }
__device__ __forceinline__ uint32_t fold(const uint2 &v) { return v.x | v.y; }
__device__ __forceinline__ uint32_t fold(const uint32_t &v) { return v; }

// Opaque zero that data-depends on x: the compiler cannot fold it away, and the hardware
// cannot issue a load whose address uses it before x has arrived.  This orders the start
// walker's flag re-check after its data loads.
__device__ __forceinline__ uint32_t dep_zero(uint32_t x) {
    uint32_t z;
    asm volatile("and.b32 %0, %1, 0;" : "=r"(z) : "r"(x));
    return z;
}

// Coherent (gpu-scope) read of a flag word: always served by L2.
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Claim: atomic OR returning the previous word (gpu scope).
__device__ __forceinline__ uint32_t atom_or_u32(uint32_t *p, uint32_t bits) {
    uint32_t old;
    asm volatile("atom.relaxed.gpu.global.or.b32 %0, [%1], %2;"
                 : "=r"(old) : "l"(p), "r"(bits) : "memory");
    return old;
}

__device__ __forceinline__ uint32_t atom_or_acq_u32(uint32_t *p, uint32_t bits) {
    uint32_t old;
    asm volatile("atom.acquire.gpu.global.or.b32 %0, [%1], %2;"
                 : "=r"(old) : "l"(p), "r"(bits) : "memory");
    return old;
}

__device__ __forceinline__ void fence_acq_rel_gpu() {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}

__device__ __forceinline__ void prefetch_l2(const void *p) {
    asm volatile("prefetch.global.L2 [%0];" :: "l"(p));
}

// ------------------------------------------------------------ mbarrier / bulk copy
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count)
                 : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;"
                 :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// Raise the expected transaction bytes of the current phase without arriving.
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;"
                 :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// Shared address overload of the 1-D bulk copy.
__device__ __forceinline__ void bulk_g2s_u32(uint32_t sdst, const void *gsrc, uint32_t bytes,
                                             uint32_t sbar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        :: "r"(sdst), "l"(gsrc), "r"(bytes), "r"(sbar) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
// Non-blocking probe of a phase.
__device__ __forceinline__ bool mbar_test_wait(uint64_t *bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
// The mbarrier receives one arrival once all of this thread's prior cp.async copies have
// landed (no pending-count increment: the barrier is initialised with the thread count).
__device__ __forceinline__ void cp_async_mbar_arrive(uint64_t *bar) {
    asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
// 1-D bulk copy global -> shared (TMA engine, "UBLKCP"), completion on an mbarrier.
__device__ __forceinline__ void bulk_g2s(void *sdst, const void *gsrc, uint32_t bytes,
                                         uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        :: "r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ uint4 lds128(uint32_t saddr) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(saddr) : "memory");
    return v;
}
#ifndef IPT_ST_HINT
#define IPT_ST_HINT 0
#endif
__device__ __forceinline__ void stg128_na(void *p, const uint4 &v) {
#if IPT_ST_HINT == 1
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
#elif IPT_ST_HINT == 2 || IPT_ST_HINT == 3
    asm volatile("{\n\t.reg .b64 pol;\n\t"
#if IPT_ST_HINT == 2
                 "createpolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\t"
#else
                 "createpolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\t"
#endif
                 "st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, pol;\n\t}"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
#else
    asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
#endif
}

}  // namespace ipt
