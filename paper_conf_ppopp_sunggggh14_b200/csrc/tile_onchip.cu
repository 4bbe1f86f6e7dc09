// tile_onchip.cu -- elementary transposition P(batch, A, B, 1): every contiguous A x B
// tile -> B x A in place, with the whole tile staged in shared memory.
//
// Paper: the Barrier-sync (BS) kernel of Fig. 1: "one work-group transposes a
// matrix that fits the on-chip memory" -- every element is copied into an on-chip temp
// array at its transposed position, a barrier, and the temp array is copied back.  The
// 0010! stage applies it to the N'M' independent m x n tiles; BS is the fastest
// 010! "if the tile (m x n) fits into shared memory".
//
// B200 design:
//   * Fast path (elem 4/8/16 B, m and n multiples of V = 16/elem): persistent CTAs, two
//     shared-memory tile buffers.  Each tile row (n*elem bytes, contiguous in HBM) is
//     fetched by the TMA engine with a 1-D bulk copy (cp.async.bulk, completion on an
//     mbarrier) into a row-padded layout; the next tile is prefetched while the current
//     one is written out.  The padded pitch q (in 16-byte units) is odd.
//   * Write-out: each thread owns a V x V block, reads V 16-byte row pieces from shared
//     memory in a lane-rotated order (conflict-free: every 8-lane phase hits 8 distinct
//     16-byte bank groups because q is odd and the row order is rotated by the lane's
//     position), transposes the block in registers with a select-network rotation, and
//     writes V fully coalesced 16-byte stores (a warp writes 512 contiguous bytes per
//     output row piece).
//   * Generic path (any elem size / any m, n that fit): one tile per iteration, plain
//     coalesced element loads into an odd-pitch shared array, barrier, coalesced element
//     stores from the transposed position -- Fig. 1 written for a CUDA block.
#include "ipt_internal.h"
#include "mem_ptx.cuh"

#include <map>
#include <mutex>

namespace ipt {

struct TileParams {
    char *base;
    uint64_t ostride;     // bytes between outer items
    uint64_t tile_bytes;  // m*n*eb (= inner stride)
    uint64_t count;       // total tiles = outer * inner
    FastDiv divInner;
    uint32_t m, n;        // tile rows / cols (input view)
    uint32_t q;           // fast path: padded pitch in 16-byte units (odd)
    uint32_t pitch;       // generic path: padded pitch in elements (odd)
    uint32_t buf_bytes;   // bytes of one smem tile buffer
    FastDiv divM, divN, divMV;  // m, n and m/V
};

__device__ __forceinline__ char *tile_ptr(const TileParams &p, uint64_t t) {
    uint64_t to, ti;
    fdivmod(t, p.divInner, to, ti);
    return p.base + to * p.ostride + ti * p.tile_bytes;
}

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

// ---------------------------------------------------------------------- fast kernel
template <int EB>
__global__ void __launch_bounds__(256) tile_onchip_fast(const TileParams p) {
    constexpr int V = 16 / EB;               // elements per 16-byte vector
    constexpr int ROT = (V >= 8) ? 1 : 8 / V; // lanes sharing one rotation
    using E = typename Elem<EB>::T;
    extern __shared__ __align__(128) unsigned char smem[];
    uint64_t *bar = reinterpret_cast<uint64_t *>(smem);
    unsigned char *const buf0 = smem + 128;
    const int tid = threadIdx.x;
    const int nthr = blockDim.x;
    const int lane = tid & 31;
    const uint32_t mv = p.m / V, nv = p.n / V;
    const uint32_t nblk = mv * nv;
    const uint32_t row_bytes = p.n * EB;

    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        fence_mbar_init();
    }
    __syncthreads();

    auto issue = [&](uint64_t t, int b) {
        // warp 0 only: lane 0 arms the barrier, then all lanes issue row copies
        const char *g = tile_ptr(p, t);
        if (lane == 0) mbar_arrive_expect_tx(&bar[b], (uint32_t)p.tile_bytes);
        __syncwarp();
        for (uint32_t i = lane; i < p.m; i += 32)
            bulk_g2s(buf0 + (size_t)b * p.buf_bytes + (size_t)i * p.q * 16, g + (size_t)i * row_bytes, row_bytes, &bar[b]);
    };

    uint64_t t = blockIdx.x;
    if (t < p.count && tid < 32) issue(t, 0);
    for (int it = 0; t < p.count; t += gridDim.x, ++it) {
        const int b = it & 1;
        const uint64_t tn = t + gridDim.x;
        if (tn < p.count && tid < 32) issue(tn, b ^ 1);
        mbar_wait(&bar[b], (uint32_t)((it >> 1) & 1));

        char *g = tile_ptr(p, t);
        const uint32_t sbase = smem_u32(buf0) + (uint32_t)b * p.buf_bytes;
        for (uint32_t blk = tid; blk < nblk; blk += nthr) {
            uint64_t bj64, bi64;
            fdivmod(blk, p.divMV, bj64, bi64);
            const uint32_t bi = (uint32_t)bi64, bj = (uint32_t)bj64;
            const int off = (int)((bi / ROT) % V);
            E x[V][V];
#pragma unroll
            for (int kk = 0; kk < V; ++kk) {
                const uint32_t rho = (uint32_t)((kk + off) % V);
                const uint4 v = lds128(sbase + ((bi * V + rho) * p.q + bj) * 16);
                unpack<EB>(v, x[kk]);
            }
            // x[kk][c] = tile[bi*V + (kk+off)%V][bj*V + c]; output row c gets column c.
#pragma unroll
            for (int c = 0; c < V; ++c) {
                E col[V];
#pragma unroll
                for (int kk = 0; kk < V; ++kk) col[kk] = x[kk][c];
                rotate_sel<V, E>(col, off);    // col[e] = tile[bi*V + e][bj*V + c]
                stg128_na(g + ((size_t)(bj * V + c) * p.m + (size_t)bi * V) * EB, pack<EB>(col));
            }
        }
        __syncthreads();   // buffer b fully consumed before it is refilled (it + 2)
    }
    (void)lane;
}

// ------------------------------------------------------------------- generic kernel
template <typename T>
__global__ void __launch_bounds__(256) tile_onchip_generic(const TileParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T *s = reinterpret_cast<T *>(smem_raw);
    const uint32_t mn = p.m * p.n;
    for (uint64_t t = blockIdx.x; t < p.count; t += gridDim.x) {
        T *g = reinterpret_cast<T *>(tile_ptr(p, t));
        for (uint32_t e = threadIdx.x; e < mn; e += blockDim.x) {
            uint64_t i, j;
            fdivmod(e, p.divN, i, j);
            s[i * p.pitch + j] = g[e];
        }
        __syncthreads();
        for (uint32_t o = threadIdx.x; o < mn; o += blockDim.x) {
            uint64_t r, c;
            fdivmod(o, p.divM, r, c);    // output row r < n, column c < m
            g[o] = s[c * p.pitch + r];
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------ host side
namespace {

bool fast_ok(const StageDesc &d) {
    const int eb = d.eb;
    if (eb != 4 && eb != 8 && eb != 16) return false;
    const int V = 16 / eb;
    if (d.A % V || d.B % V) return false;
    if (((uintptr_t)d.base & 15) != 0) return false;
    if (d.outer > 1 && (d.ostride & 15) != 0) return false;
    if (env_int("IPT_TILE_GENERIC", 0)) return false;
    return true;
}

uint32_t fast_q(const StageDesc &d) {
    uint32_t q = (uint32_t)(d.B * d.eb / 16);
    return (q & 1) ? q : q + 1;
}

size_t fast_smem(const StageDesc &d) {
    return 128 + 2 * (size_t)d.A * fast_q(d) * 16;
}

uint32_t generic_pitch(const StageDesc &d) {
    uint32_t P = (uint32_t)d.B;
    return (P & 1) ? P : P + 1;
}

size_t generic_smem(const StageDesc &d) { return (size_t)d.A * generic_pitch(d) * d.eb; }

template <typename K>
int occupancy(K kern, size_t smem, int device) {
    static std::mutex mu;
    static std::map<std::pair<const void *, std::pair<int, size_t>>, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_pair((const void *)kern, std::make_pair(device, smem));
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    int n = 0;
    // one attribute value per kernel: the device maximum (a lower value set for one
    // shape would make a later, larger launch fail)
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         dev_props(device).smem_optin);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, 256, smem) != cudaSuccess) n = 1;
    if (n < 1) n = 1;
    cache[key] = n;
    return n;
}

template <typename K>
cudaError_t go(K kern, const TileParams &p, size_t smem, cudaStream_t st, int device) {
    DevProps dp = dev_props(device);
    int per_sm = occupancy(kern, smem, device);
    uint64_t grid = (uint64_t)dp.sms * per_sm;
    if (p.count < grid) grid = p.count;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, 256, smem, st>>>(p);
    note_launch();
    return cudaGetLastError();
}

}  // namespace

int tile_onchip_path(int64_t A, int64_t B, int eb, int device) {
    DevProps dp = dev_props(device);
    StageDesc d{};
    d.A = A; d.B = B; d.s = 1; d.eb = eb; d.outer = 1; d.inner = 1;
    d.base = nullptr;
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    const bool vec = (eb == 4 || eb == 8 || eb == 16) && A % (16 / eb) == 0 && B % (16 / eb) == 0
                     && !env_int("IPT_TILE_GENERIC", 0);
    if (vec && (long)fast_smem(d) <= budget) return 2;
    if ((long)generic_smem(d) <= budget && A * B < (1ll << 31)) return 1;
    return 0;
}

bool tile_onchip_fits(int64_t A, int64_t B, int eb, int device) {
    return tile_onchip_path(A, B, eb, device) != 0;
}

cudaError_t launch_tile_onchip(const StageDesc &d, cudaStream_t st, int device) {
    DevProps dp = dev_props(device);
    TileParams p{};
    p.base = d.base;
    p.ostride = (uint64_t)d.ostride;
    p.tile_bytes = (uint64_t)d.A * d.B * d.eb;
    p.count = (uint64_t)d.outer * d.inner;
    p.divInner = make_fastdiv((uint64_t)d.inner);
    p.m = (uint32_t)d.A;
    p.n = (uint32_t)d.B;
    p.divM = make_fastdiv((uint64_t)d.A);
    p.divN = make_fastdiv((uint64_t)d.B);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    if (fast_ok(d) && (long)fast_smem(d) <= budget) {
        p.q = fast_q(d);
        p.buf_bytes = (uint32_t)((size_t)d.A * p.q * 16);
        p.divMV = make_fastdiv((uint64_t)(d.A / (16 / d.eb)));
        const size_t smem = fast_smem(d);
        switch (d.eb) {
            case 4: return go(tile_onchip_fast<4>, p, smem, st, device);
            case 8: return go(tile_onchip_fast<8>, p, smem, st, device);
            case 16: return go(tile_onchip_fast<16>, p, smem, st, device);
        }
    }
    p.pitch = generic_pitch(d);
    const size_t smem = generic_smem(d);
    if ((long)smem > budget) return cudaErrorInvalidValue;
    switch (d.eb) {
        case 1: return go(tile_onchip_generic<uint8_t>, p, smem, st, device);
        case 2: return go(tile_onchip_generic<uint16_t>, p, smem, st, device);
        case 4: return go(tile_onchip_generic<uint32_t>, p, smem, st, device);
        case 8: return go(tile_onchip_generic<unsigned long long>, p, smem, st, device);
        case 16: return go(tile_onchip_generic<uint4>, p, smem, st, device);
    }
    return cudaErrorInvalidValue;
}

}  // namespace ipt
