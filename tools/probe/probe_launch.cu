// Launch floor of a whole-GPU kernel shaped like tile_group_rf: 148 CTAs x 512 threads,
// up to 227 KB of dynamic shared memory, optionally cooperative and with a 512-column TMEM
// allocation -- back-to-back launches timed with events (tools/probe_launch.py).
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

template <bool TMEM>
__global__ void __launch_bounds__(512, 1) empty_kernel(int *out) {
    extern __shared__ unsigned char smem[];
    __shared__ uint32_t base;
    if (TMEM) {
        if (threadIdx.x < 32) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;"
                         :: "r"((uint32_t)__cvta_generic_to_shared(&base)) : "memory");
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
        }
        __syncthreads();
        if (threadIdx.x < 32)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(base) : "memory");
    }
    if (threadIdx.x == 0 && blockIdx.x == 0 && out) out[0] = smem[0];
}

extern "C" float probe_launch(int smem, int coop, int tmem, int reps) {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    void *k = tmem ? (void *)empty_kernel<true> : (void *)empty_kernel<false>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(sms);
    cfg.blockDim = dim3(512);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = coop ? 1 : 0;
    int *out = nullptr;
    void *args[] = {&out};
    for (int i = 0; i < 10; ++i) cudaLaunchKernelExC(&cfg, k, args);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    for (int i = 0; i < reps; ++i) cudaLaunchKernelExC(&cfg, k, args);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (cudaGetLastError() != cudaSuccess) return -1;
    return 1000.f * ms / reps;
}
