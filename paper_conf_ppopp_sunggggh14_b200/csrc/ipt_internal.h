// ipt_internal.h -- internal declarations shared by the libipt translation units.
// Not part of the ABI (include/ipt.h is).  No oracle code is included or reachable.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>

#include "../../include/ipt.h"

namespace ipt {

// -------------------------------------------------------------- fast 64-bit division
// Division by a run-time invariant divisor d via a multiply-high (Granlund & Montgomery,
// "Division by invariant integers using multiplication", Fig. 4.1, N = 64):
//   l = ceil(log2 d),  m = floor(2^64 (2^l - d) / d) + 1,
//   t = mulhi(m, n),   q = (t + ((n - t) >> s1)) >> s2,  s1 = min(l, 1), s2 = max(l - 1, 0).
// Exact for every 64-bit n.  Used for the index maps of every kernel so that no 64-bit
// '%' or '/' appears in an inner loop (SURVEY.md Sec. 7 "64-bit index space").
struct FastDiv {
    uint64_t d;
    uint64_t m;
    uint32_t s1, s2;
};

FastDiv make_fastdiv(uint64_t d);  // host

__host__ __device__ __forceinline__ uint64_t mulhi64(uint64_t a, uint64_t b) {
#if defined(__CUDA_ARCH__)
    return __umul64hi(a, b);
#else
    return (uint64_t)(((unsigned __int128)a * b) >> 64);
#endif
}

__host__ __device__ __forceinline__ uint64_t fdiv(uint64_t n, const FastDiv &f) {
    uint64_t t = mulhi64(n, f.m);
    return (t + ((n - t) >> f.s1)) >> f.s2;
}

__host__ __device__ __forceinline__ void fdivmod(uint64_t n, const FastDiv &f, uint64_t &q,
                                                 uint64_t &r) {
    q = fdiv(n, f);
    r = n - q * f.d;
}

// 32-bit variant (same algorithm, N = 32), for indices known to fit 32 bits.
struct FastDiv32 {
    uint32_t d, m, s1, s2;
};

FastDiv32 make_fastdiv32(uint32_t d);  // host

__host__ __device__ __forceinline__ void fdivmod32(uint32_t n, const FastDiv32 &f, uint32_t &q,
                                          uint32_t &r) {
#if defined(__CUDA_ARCH__)
    const uint32_t t = __umulhi(n, f.m);
#else
    const uint32_t t = (uint32_t)(((uint64_t)n * f.m) >> 32);
#endif
    q = (t + ((n - t) >> f.s1)) >> f.s2;
    r = n - q * f.d;
}

// ------------------------------------------------------------------ stage descriptor
// One elementary transposition P(batch, A, B, s): batch x [A x B x s] -> batch x [B x A x s]
// (SURVEY.md R5).  The batch index T is split as T = to * inner + ti: item T starts at
// base + to * ostride + ti * (A*B*s*eb) bytes, so that batched calls with an arbitrary
// matrix stride fold into one launch.
struct StageDesc {
    char *base;
    int64_t outer, inner;   // batch = outer * inner
    int64_t ostride;        // bytes between outer items (>= inner * A*B*s*eb)
    int64_t A, B, s;
    int eb;                 // element bytes
};

// ---------------------------------------------------------------- kernel launchers
// All launchers return cudaSuccess or the launch error; they only enqueue work.

// Cycle following over super-elements with a global flag bitmap (PTTWAC over
// super-elements, P:200-224 / SURVEY K5+K6).  `ws` must hold cycle_ws_bytes(desc).
size_t cycle_ws_bytes(const StageDesc &d);
cudaError_t launch_cycle_global(const StageDesc &d, void *ws, cudaStream_t st, int device);

// Segmented cycle following (cycle_seg.cu): equal-length segments of the cycles computed
// on the host (cached per shape), one grid barrier, no flags.  Needs S*eb % 16 == 0 and
// 16-byte aligned data; uses the first 4 bytes of `ws` (>= 256 B) as barrier counter.
// Returns cudaErrorNotSupported when not applicable (caller falls back to flags).
cudaError_t launch_cycle_seg(const StageDesc &d, void *ws, cudaStream_t st, int device);
uint64_t cycle_seg_walkers(int64_t S_bytes, int device);
uint64_t cycle_seg_est_len(int64_t units_per_item, int64_t items, int64_t S_bytes, int device);
bool cycle_prefer_seg(int64_t units, int64_t items, int64_t S_bytes, int device);   // plan.cpp

// Whole-tile on-chip transposition (BS kernel, Fig. 1): s must be 1
// and an A x B tile must fit in shared memory (tile_onchip_fits()).
bool tile_onchip_fits(int64_t A, int64_t B, int eb, int device);
// 0: does not fit, 1: generic element path, 2: 16-byte path in one CTA,
// 3: 16-byte path split over a thread-block cluster (tile_cluster_k CTAs),
// 4: element path split over a thread-block cluster,
// 5: 16-byte path split over a co-resident group of CTAs (double-buffered slices),
// 6: element path (4/8-byte elements) split over a co-resident group of CTAs,
// 7: 16-byte path over every SM, slices in shared memory + registers (tile_group_rf)
int tile_onchip_path(int64_t A, int64_t B, int eb, int device);
int tile_cluster_k(int64_t A, int64_t B, int eb, int device);
int tile_generic_cluster_k(int64_t A, int64_t B, int eb, int device);
bool tile_group_split(int64_t A, int64_t B, int eb, int device);
bool tile_rf_fits(int64_t A, int64_t B, int eb, int device);   // whole-GPU smem + register tiles
bool tile_group_generic_split(int64_t A, int64_t B, int eb, int device);
// Group split of `count` tiles: CTAs per tile (0 = does not fit) and groups in flight.
int tile_group_k(int64_t A, int64_t B, int eb, uint64_t count, int device, int *groups,
                 bool *tma = nullptr, int *nbuf = nullptr);
// Kernel names the launchers will run for a stage (diagnostics, ipt__stage_kernel).
const char *tile_kernel_name(const StageDesc &d, int device);
const char *cycle_kernel_name(const StageDesc &d, int device);
const char *square_kernel_name(const StageDesc &d);
// Workspace of a tile stage: the group split's arrival counters (one per group and slice
// buffer, kGroupCtrStride bytes apart, at most 256).  `ws` may be NULL for the other paths.
constexpr uint32_t kGroupCtrStride = 32;
constexpr size_t kTileWsBytes = 256 * kGroupCtrStride;
cudaError_t launch_tile_onchip(const StageDesc &d, void *ws, cudaStream_t st, int device);

// Square items P(batch, g, g, 1) by symmetric block-pair swaps: any g, no
// workspace.  square_swap_vec_path: the 16-byte path applies (else the element path).
cudaError_t launch_square_swap(const StageDesc &d, cudaStream_t st, int device);
bool square_swap_vec_path(const StageDesc &d);
bool prefer_square_swap(int64_t batch, int64_t g, int eb, int device);   // plan.cpp

// Device properties used by planner and launchers (cached).
struct DevProps {
    int sms;
    int smem_optin;     // max dynamic shared memory per block (bytes)
    int smem_per_sm;
    int max_threads_sm;
    int l2_bytes;
    bool valid;
};
DevProps dev_props(int device);   // device < 0 -> nominal B200 values

// Launch accounting (ipt_kernel_launch_count).
void note_launch();

// Environment-variable integer override (tuning knobs for tests / sweeps).
long env_int(const char *name, long dflt);
uint64_t env_hash();   // hash of the IPT_* variables set (cache keys of env-dependent plans)

}  // namespace ipt
