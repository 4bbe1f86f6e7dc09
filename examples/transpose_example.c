/*
 * transpose_example.c -- using libipt from C (no torch): in-place transposition of an
 * M x N matrix of 4-byte elements in device memory, checked on the host.
 *
 *   gcc -O2 -I include examples/transpose_example.c \
 *       -L paper_conf_ppopp_sunggggh14_b200 -lipt -Wl,-rpath,$PWD/paper_conf_ppopp_sunggggh14_b200 \
 *       -I /usr/local/cuda/include -L /usr/local/cuda/lib64 -lcudart -o transpose_example
 *   ./transpose_example 1800 7200
 *
 * The C ABI (include/ipt.h) takes plain device pointers and a cudaStream_t passed as void*.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include "ipt.h"

int main(int argc, char **argv) {
    const int64_t M = argc > 1 ? atoll(argv[1]) : 1800, N = argc > 2 ? atoll(argv[2]) : 7200;
    const size_t bytes = (size_t)(M * N) * sizeof(uint32_t);
    uint32_t *h = (uint32_t *)malloc(bytes), *d = NULL;
    if (!h) return 1;
    for (int64_t k = 0; k < M * N; ++k) h[k] = (uint32_t)k;     /* A(i, j) = i*N + j */
    if (cudaMalloc((void **)&d, bytes) != cudaSuccess) { fprintf(stderr, "no device\n"); return 1; }
    cudaMemcpy(d, h, bytes, cudaMemcpyHostToDevice);

    ipt_plan_t plan;
    ipt_status s = ipt_plan(M, N, (int)sizeof(uint32_t), 0, &plan);
    if (s != IPT_OK) { fprintf(stderr, "ipt_plan: %s\n", ipt_status_string(s)); return 1; }
    printf("plan m=%lld n=%lld stages=%d variants=%d,%d,%d workspace=%llu B\n", (long long)plan.m,
           (long long)plan.n, plan.n_stages, plan.variant[0], plan.variant[1], plan.variant[2],
           (unsigned long long)plan.workspace_bytes);

    s = ipt_transpose(d, M, N, (int)sizeof(uint32_t), NULL);       /* A -> A^T, same storage */
    if (s != IPT_OK) { fprintf(stderr, "ipt_transpose: %s (%s)\n", ipt_status_string(s), ipt_last_cuda_error()); return 1; }
    cudaMemcpy(h, d, bytes, cudaMemcpyDeviceToHost);

    int64_t bad = 0;                                              /* A^T(j, i) = A(i, j) */
    for (int64_t j = 0; j < N; ++j)
        for (int64_t i = 0; i < M; ++i)
            bad += h[j * M + i] != (uint32_t)(i * N + j);
    printf("%s: %lld mismatches (%s)\n", bad ? "FAIL" : "ok", (long long)bad, ipt_version());
    cudaFree(d);
    free(h);
    return bad != 0;
}
