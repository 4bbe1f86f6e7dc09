// Diagnostic (not product code): DRAM efficiency of random S-byte block read-then-write
// traffic -- the memory pattern of a cycle-following stage without its atomics/chains.
#include <cuda_runtime.h>
#include <stdint.h>
__device__ __forceinline__ uint4 ldcg(const void *p) {
    uint4 v; asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory"); return v; }
__device__ __forceinline__ void stcg(void *p, uint4 v) {
    asm volatile("st.global.cg.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory"); }
template <int U, int R>
__global__ void __launch_bounds__(256) rmw_blocks(char *base, const uint32_t *perm, uint32_t nblk, uint32_t S) {
    const int lane = threadIdx.x & 31;
    const uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
    const uint32_t nv = S / 16;
    for (uint32_t i0 = w * U; i0 < nblk; i0 += nw * U) {
        uint4 v[U][R];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            uint32_t i = i0 + u; if (i >= nblk) break;
            char *a = base + (size_t)perm[i] * S;
#pragma unroll
            for (int r = 0; r < R; ++r) { uint32_t e = lane + 32 * r; if (e < nv) v[u][r] = ldcg(a + e * 16); }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            uint32_t i = i0 + u; if (i >= nblk) break;
            char *a = base + (size_t)perm[i] * S;
#pragma unroll
            for (int r = 0; r < R; ++r) { uint32_t e = lane + 32 * r; if (e < nv) { uint4 x = v[u][r]; x.x ^= 1; stcg(a + e * 16, x); } }
        }
    }
}
extern "C" int probe_rmw(void *base, const void *perm, uint32_t nblk, uint32_t S, int U, int sms, void *stream) {
    cudaStream_t st = (cudaStream_t)stream;
    int grid = sms * 8;
    int R = (S + 511) / 512;
#define GO(u, r) if (U == u && R == r) { rmw_blocks<u, r><<<grid, 256, 0, st>>>((char *)base, (const uint32_t *)perm, nblk, S); return (int)cudaGetLastError(); }
    GO(1,1) GO(2,1) GO(4,1) GO(1,2) GO(2,2) GO(4,2) GO(1,4) GO(2,4) GO(4,4)
    return -1;
}
