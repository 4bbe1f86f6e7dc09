// Diagnostic (not product code): a copy through shared memory with the group tile
// kernel's pipeline shape, to isolate what costs bandwidth.  Each CTA (1 per SM, 512
// threads) owns chunk c = blockIdx.x + k*gridDim.x of CH bytes; iteration k issues the
// cp.async loads of chunk k+1 into the other slot, waits for chunk k, optionally joins a
// global barrier of all CTAs (sync = 1: arrive + spin on one counter, as the group
// kernel), then writes chunk k from shared memory with 16-byte stores to dst (= src for
// in place).
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void __launch_bounds__(512, 1) cp_pipe(const char *src, char *dst, uint64_t nch, uint32_t ch,
                                                  int sync, unsigned int *ctr) {
    extern __shared__ __align__(128) unsigned char sm[];
    const uint32_t s0 = su32(sm);
    auto issue = [&](uint64_t c, uint32_t slot) {
        const char *g = src + c * ch;
        for (uint32_t e = threadIdx.x; e < ch / 16; e += blockDim.x)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(s0 + slot * ch + e * 16), "l"(g + (uint64_t)e * 16) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    uint32_t it = 0;
    const uint64_t nit = (nch - blockIdx.x + gridDim.x - 1) / gridDim.x;
    const uint64_t nit_all = (nch + gridDim.x - 1) / gridDim.x;
    if (blockIdx.x < nch) issue(blockIdx.x, 0);
    for (uint64_t k = 0; k < nit_all; ++k, ++it) {
        const uint64_t c = blockIdx.x + k * gridDim.x;
        if (k + 1 < nit) issue(c + gridDim.x, (it + 1) & 1);
        else asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 1;" ::: "memory");
        // sync 1: thread 0 (a writer) arrives with release; 2: relaxed arrival and poll;
        // 3: the last warp (no stores) arrives with release and polls with acquire
        const uint32_t ctl = (sync == 3) ? blockDim.x - 32 : 0;
        const uint32_t nwr = (sync == 3) ? blockDim.x - 32 : blockDim.x;
        if (sync) {
            __syncthreads();
            if (threadIdx.x == ctl) {
                if (sync == 2) asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
                else asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
                const uint32_t target = (uint32_t)((k + 1) * gridDim.x);
                uint32_t v;
                do {
                    if (sync == 2) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
                    else asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
                } while (v < target);
            }
        }
        __syncthreads();
        if (k < nit && threadIdx.x < nwr) {
            char *d = dst + c * ch;
            for (uint32_t e = threadIdx.x; e < ch / 16; e += nwr) {
                uint4 v;
                asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(s0 + (it & 1) * ch + e * 16));
                asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(d + (uint64_t)e * 16), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
            }
        }
        __syncthreads();
    }
}

extern "C" int probe_copy(const void *src, void *dst, uint64_t bytes, uint32_t ch, int grid, int sync,
                          void *ctr, void *stream) {
    cudaStream_t st = (cudaStream_t)stream;
    cudaFuncSetAttribute(cp_pipe, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * ch);
    cudaMemsetAsync(ctr, 0, 4, st);
    cp_pipe<<<grid, 512, 2 * ch, st>>>((const char *)src, (char *)dst, bytes / ch, ch, sync, (unsigned int *)ctr);
    return (int)cudaGetLastError();
}
