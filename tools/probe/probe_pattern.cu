// Diagnostic (not product code): DRAM efficiency of the tile stage's access pattern.
// Work unit (tile t, slice k): read `rows` chunks of C bytes (row stride X) from
// src + t*T + k*C, write rows*C contiguous bytes to dst + t*T + k*rows*C.
#include <cuda_runtime.h>
#include <stdint.h>
__device__ __forceinline__ uint4 ldcg(const void *p) {
    uint4 v; asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory"); return v; }
template <int H> __device__ __forceinline__ uint4 ldh(const void *p) {
    uint4 v;
    if (H == 0) return ldcg(p);
    if (H == 1) asm volatile("{.reg .b64 pol; createpolicy.fractional.L2::evict_first.b64 pol, 1.0;\n\tld.global.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], pol;}" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    if (H == 2) asm volatile("{.reg .b64 pol; createpolicy.fractional.L2::evict_last.b64 pol, 1.0;\n\tld.global.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], pol;}" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    if (H == 3) asm volatile("ld.global.cs.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void stna(void *p, uint4 v) {
    asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory"); }
template <int U, int H>
__global__ void __launch_bounds__(512, 1) pattern(const char *src, char *dst, uint64_t nunits, uint32_t K,
                                                  uint64_t T, uint32_t rows, uint64_t X, uint32_t C, int mode) {
    const uint32_t cv = C / 16, nv = rows * cv;
    for (uint64_t u = blockIdx.x; u < nunits; u += gridDim.x) {
        const uint64_t t = u / K, k = u % K;
        const char *s = src + t * T + k * C;
        const uint64_t nt = nunits / K;
        const uint64_t tw = mode == 2 ? (t + nt / 2) % nt : t;
        char *d = dst + tw * T + k * (uint64_t)rows * C;
        char *drmw = dst + t * T + k * C;
        for (uint32_t e0 = threadIdx.x; e0 < nv; e0 += U * blockDim.x) {
            uint4 v[U];
#pragma unroll
            for (int i = 0; i < U; ++i) {
                uint32_t e = e0 + i * blockDim.x;
                if (e < nv) v[i] = ldh<H>(s + (uint64_t)(e / cv) * X + (e % cv) * 16);
            }
#pragma unroll
            for (int i = 0; i < U; ++i) {
                uint32_t e = e0 + i * blockDim.x;
                if (e < nv) {
                    if (mode == 1) stna(drmw + (uint64_t)(e / cv) * X + (e % cv) * 16, v[i]);
                    else stna(d + (uint64_t)e * 16, v[i]);
                }
            }
        }
    }
}
extern "C" int probe_pattern(const void *src, void *dst, uint64_t nunits, uint32_t K, uint64_t T,
                             uint32_t rows, uint64_t X, uint32_t C, int grid, int H, int mode, void *stream) {
    auto k = H == 0 ? pattern<16, 0> : H == 1 ? pattern<16, 1> : H == 2 ? pattern<16, 2> : pattern<16, 3>;
    k<<<grid, 512, 0, (cudaStream_t)stream>>>((const char *)src, (char *)dst, nunits, K, T, rows, X, C, mode);
    return (int)cudaGetLastError();
}
