// regxpose.cuh -- in-register V x V transposes of 16-byte vectors (V = 16 / elem bytes),
// shared by the on-chip tile kernels (tile_onchip.cu) and the square swap kernel
// (square_swap.cu).  Raw bit moves only.
#pragma once
#include <stdint.h>

namespace ipt {

// ---------------------------------------------------------------- register transposes
// Rotate x[0..V) so that out[e] = x[(e - off) mod V], with `off` per lane (select net).
template <int V, typename E>
__device__ __forceinline__ void rotate_sel(E (&x)[V], int off) {
#pragma unroll
    for (int sh = 1; sh < V; sh <<= 1) {
        const bool f = (off & sh) != 0;
        E y[V];
#pragma unroll
        for (int e = 0; e < V; ++e) y[e] = f ? x[(e - sh + V) % V] : x[e];
#pragma unroll
        for (int e = 0; e < V; ++e) x[e] = y[e];
    }
}

template <int EB> struct Elem;
template <> struct Elem<4> { using T = uint32_t; };
template <> struct Elem<8> { using T = unsigned long long; };
template <> struct Elem<16> { using T = uint4; };

template <int EB>
__device__ __forceinline__ void unpack(const uint4 &v, typename Elem<EB>::T (&e)[16 / EB]);
template <> __device__ __forceinline__ void unpack<4>(const uint4 &v, uint32_t (&e)[4]) {
    e[0] = v.x; e[1] = v.y; e[2] = v.z; e[3] = v.w;
}
template <> __device__ __forceinline__ void unpack<8>(const uint4 &v, unsigned long long (&e)[2]) {
    e[0] = ((unsigned long long)v.y << 32) | v.x;
    e[1] = ((unsigned long long)v.w << 32) | v.z;
}
template <> __device__ __forceinline__ void unpack<16>(const uint4 &v, uint4 (&e)[1]) { e[0] = v; }

template <int EB>
__device__ __forceinline__ uint4 pack(const typename Elem<EB>::T (&e)[16 / EB]);
template <> __device__ __forceinline__ uint4 pack<4>(const uint32_t (&e)[4]) {
    return make_uint4(e[0], e[1], e[2], e[3]);
}
template <> __device__ __forceinline__ uint4 pack<8>(const unsigned long long (&e)[2]) {
    return make_uint4((uint32_t)e[0], (uint32_t)(e[0] >> 32), (uint32_t)e[1], (uint32_t)(e[1] >> 32));
}
template <> __device__ __forceinline__ uint4 pack<16>(const uint4 (&e)[1]) { return e[0]; }

__device__ __forceinline__ void sts128(uint32_t saddr, const uint4 &v) {
    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};"
                 :: "r"(saddr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

}  // namespace ipt
