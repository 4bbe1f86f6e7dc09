// tile_onchip.cu -- elementary transposition P(batch, A, B, 1): every contiguous A x B
// tile -> B x A in place, with the whole tile staged in shared memory.
//
// Paper: the Barrier-sync (BS) kernel of Fig. 1: "one work-group transposes a
// matrix that fits the on-chip memory" -- every element is copied into an on-chip temp
// array at its transposed position, a barrier, and the temp array is copied back.  The
// 0010! stage applies it to the N'M' independent m x n tiles; BS is the fastest
// 010! "if the tile (m x n) fits into shared memory".
//
// B200 design.  Fast paths (elem 4/8/16 B, m and n multiples of
// V = 16/elem, 16-B aligned tiles) share the write-out and differ in how a tile reaches
// shared memory:
//   * "tma": persistent CTAs with an NB-deep ring of tile buffers; each tile row
//     (n*elem contiguous bytes) is fetched by the TMA engine with a 1-D bulk copy
//     (cp.async.bulk, completion on an mbarrier) into a row-padded layout, NB-1 tiles
//     ahead of the one being written out.
//   * "ldg": each thread issues a batch of 16-byte loads into registers (many bytes in
//     flight per thread), stores them to the padded layout, barrier, write-out; several
//     CTAs per SM overlap each other's load and store phases.
//   Shared layout: row pitch q (16-byte units) is odd.  Write-out: each thread owns a
//   V x V block, reads its V row pieces with a lane-rotated order (every 8-lane phase
//   of an LDS.128 hits 8 distinct 16-byte bank groups), transposes the block in
//   registers with a select-network rotation, and issues V coalesced 16-byte stores
//   (a warp writes 512 contiguous bytes per output row piece).
// Generic path (any elem size / any m, n that fit): coalesced element loads into an
// odd-pitch shared array, barrier, coalesced element stores -- Fig. 1 for a CUDA block.
#include "ipt_internal.h"
#include "mem_ptx.cuh"
#include "regxpose.cuh"

#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdio>
#include <map>
#include <mutex>
#include <tuple>

namespace ipt {

struct TileParams {
    char *base;
    uint64_t ostride;     // bytes between outer items
    uint64_t tile_bytes;  // m*n*eb (= inner stride)
    uint64_t count;       // total tiles = outer * inner
    FastDiv divInner;
    uint32_t m, n;        // tile rows / cols (input view)
    uint32_t q;           // fast paths: padded pitch in 16-byte units (odd)
    uint32_t pitch;       // generic path: padded pitch in elements (odd)
    uint32_t buf_bytes;   // bytes of one smem tile buffer
    uint32_t nbuf;        // tma path: ring depth
    FastDiv divM, divN, divMV, divNV;  // m, n, m/V, n/V
    FastDiv32 divM32, divN32, divMV32, divMVK32, divNV32;   // m, n, m/V, (m/V)/K, n/V
    uint32_t K;           // cluster path: CTAs per tile
    int colsplit;         // generic cluster path: split columns (1) or rows (0)
    uint32_t ralign;      // generic cluster row split: slice boundaries in multiples of this
    uint32_t gb;          // streaming kernel: V-row blocks per group (0 = automatic)
    uint32_t *gbar;       // group-split kernel: one arrival counter per group (workspace)
    uint32_t *gexit;      // group-split kernel: per-group exit counters (self-resetting
                          // library-owned counters; nullptr = gbar zeroed by a memset)
    int vec16;            // generic path: tiles 16-byte aligned, 16-byte loads
    int arrive_release;   // group kernels: release-ordered arrivals (default relaxed)
    uint32_t box_rows;    // tile_group_tma: rows per 2-D TMA box (divides the slice rows)
    uint32_t npan;        // tile_group_tma: column panels per slice (width q vectors each)
    uint32_t pstride;     // tile_group_tma: bytes between panels (128-byte multiple)
    uint32_t rres;        // tile_group_rf: 1 = 3-D tensor map (strided batch of single tiles)
    int diag;             // group kernels, measurement only (IPT_TILE_DIAG; results invalid):
                          // 1 = no group wait, 2 = no stores, 4 = no loads, 32 = stores
                          // to a second buffer after the data; 16 = timeline
                          // trace (results valid, see ipt__tile_trace)
    unsigned long long *trace;
    uint32_t rows_a;      // tile_group_rf: slice rows staged in shared memory by TMA (rest: TMEM)
    uint32_t rows_b;      // tile_group_rf: rows per chunk of the TMEM part
    uint32_t cpan;        // tile_group_rf: panels per chunk of the TMEM part
    uint32_t zero;        // 0 at run time, opaque to the compiler (load-completion dependency)
    uint32_t gcols;       // tile_group_generic: > 1 = 2-D slice grid, K / gcols row bands x gcols
                          // column pieces (rank = band * gcols + piece)
};

__device__ __forceinline__ char *tile_ptr(const TileParams &p, uint64_t t) {
    uint64_t to, ti;
    fdivmod(t, p.divInner, to, ti);
    return p.base + to * p.ostride + ti * p.tile_bytes;
}

// Write the transposed tile from padded shared memory to global g.  The CTA holds the
// block rows [bi0, bi0 + mvp) x block columns [bj0, bj0 + nbj) of the tile (V x V blocks):
// buffer row bil*V + r, 16-byte column bjl (pitch q) holds tile row (bi0+bil)*V + r,
// columns (bj0+bjl)*V .. +V-1.  Whole tile for one CTA; a row or column slice per cluster CTA.
struct NoProbe {
    __device__ void operator()() const {}
};

template <int EB, typename Probe = NoProbe>
__device__ __forceinline__ void write_out(const TileParams &p, uint32_t sbase, char *g, uint32_t q,
                                          uint32_t bi0, uint32_t mvp, const FastDiv32 &divmvp,
                                          uint32_t bj0, uint32_t nbj, Probe probe = Probe()) {
    constexpr int V = 16 / EB;
    constexpr int ROT = (V >= 8) ? 1 : 8 / V;   // lanes sharing one rotation
    using E = typename Elem<EB>::T;
    const uint32_t nblk = mvp * nbj;
    for (uint32_t blk = threadIdx.x; blk < nblk; blk += blockDim.x) {
        probe();
        uint32_t bjl, bil;
        fdivmod32(blk, divmvp, bjl, bil);
        const uint32_t bi = bi0 + bil, bj = bj0 + bjl;
        const int off = (int)((bil / ROT) % V);
        E x[V][V];
#pragma unroll
        for (int kk = 0; kk < V; ++kk) {
            const uint32_t rho = (uint32_t)((kk + off) % V);
            const uint4 v = lds128(sbase + ((bil * V + rho) * q + bjl) * 16);
            unpack<EB>(v, x[kk]);
        }
        // x[kk][c] = tile[bi*V + (kk+off)%V][bj*V + c]; output row bj*V+c gets column c.
#pragma unroll
        for (int c = 0; c < V; ++c) {
            E col[V];
#pragma unroll
            for (int kk = 0; kk < V; ++kk) col[kk] = x[kk][c];
            rotate_sel<V, E>(col, off);    // col[e] = tile[bi*V + e][bj*V + c]
            stg128_na(g + ((size_t)(bj * V + c) * p.m + (size_t)bi * V) * EB, pack<EB>(col));
        }
    }
}

template <int EB>
__device__ __forceinline__ void write_out(const TileParams &p, uint32_t sbase, char *g) {
    write_out<EB>(p, sbase, g, p.q, 0, p.m / (16 / EB), p.divMV32, 0, p.n / (16 / EB));
}

// As write_out, for a slice held as column panels (tile_group_tma): 16-byte column bjl
// lives in panel bjl / pw at sbase + panel * pstride, row pitch pw vectors.  SWZ: one panel
// of 128-byte rows in the TMA 128-byte swizzle (vector c of row r at chunk c ^ (r & 7);
// sbase 1024-byte aligned).
template <int EB, typename Probe, bool SWZ = false>
__device__ __forceinline__ void write_out_pan(const TileParams &p, uint32_t sbase, char *g, uint32_t pw,
                                              const FastDiv32 &divpw, uint32_t pstride, uint32_t bi0,
                                              uint32_t mvp, const FastDiv32 &divmvp, uint32_t bj0,
                                              uint32_t nbj, Probe probe) {
    constexpr int V = 16 / EB;
    constexpr int ROT = (V >= 8) ? 1 : 8 / V;
    using E = typename Elem<EB>::T;
    const uint32_t nblk = mvp * nbj;
    for (uint32_t blk = threadIdx.x; blk < nblk; blk += blockDim.x) {
        probe();
        uint32_t bjl, bil, pan, pc;
        fdivmod32(blk, divmvp, bjl, bil);
        fdivmod32(bjl, divpw, pan, pc);
        const uint32_t bi = bi0 + bil, bj = bj0 + bjl;
        // lane rotation of the V rows a thread reads (undone by rotate_sel): (bil / ROT) mod V
        // is conflict-free for runs of >= 8 consecutive V-row blocks at any quarter-warp
        // alignment; for V = 4 and mvp = 4 mod 8 blocks per column (the rf row slices' part A
        // of 4 blocks), 2(bil/2) + bil/4 takes 1.31-1.5 wavefronts per access to 1.0 (bank
        // model over all quarter-warp alignments, odd pitches and the 128-byte swizzle;
        // it is worse for other block counts, e.g. 450: 1.17 vs 1.01).  rf 4096x3000:
        // 5.11 -> 5.19 TB/s
        const int off = (V == 4 && (mvp & 7) == 4) ? (int)((((bil >> 1) << 1) + (bil >> 2)) & 3)
                                                   : (int)((bil / ROT) % V);
        const uint32_t pb = sbase + pan * pstride + pc * 16;
        E x[V][V];
#pragma unroll
        for (int kk = 0; kk < V; ++kk) {
            const uint32_t rho = (uint32_t)((kk + off) % V), row = bil * V + rho;
            const uint4 v = SWZ ? lds128(sbase + row * 128 + ((pc ^ (row & 7)) << 4)) : lds128(pb + row * pw * 16);
            unpack<EB>(v, x[kk]);
        }
#pragma unroll
        for (int c = 0; c < V; ++c) {
            E col[V];
#pragma unroll
            for (int kk = 0; kk < V; ++kk) col[kk] = x[kk][c];
            rotate_sel<V, E>(col, off);
            stg128_na(g + ((size_t)(bj * V + c) * p.m + (size_t)bi * V) * EB, pack<EB>(col));
        }
    }
}

// ------------------------------------------------------------ register-staged kernel
template <int EB, int U, int MINB = 2>
__global__ void __launch_bounds__(512, MINB) tile_onchip_ldg(const TileParams p) {
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t sbase = smem_u32(smem);
    const uint32_t nvec = (uint32_t)(p.tile_bytes / 16);
    for (uint64_t t = blockIdx.x; t < p.count; t += gridDim.x) {
        char *g = tile_ptr(p, t);
        for (uint32_t e0 = threadIdx.x; e0 < nvec; e0 += U * blockDim.x) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t e = e0 + u * blockDim.x;
                if (e < nvec) v[u] = ld_cg<16>(g + (size_t)e * 16);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t e = e0 + u * blockDim.x;
                if (e < nvec) {
                    uint32_t i, j;
                    fdivmod32(e, p.divNV32, i, j);
                    sts128(sbase + (i * p.q + j) * 16, v[u]);
                }
            }
        }
        __syncthreads();
        write_out<EB>(p, sbase, g);
        __syncthreads();
    }
}

__device__ __forceinline__ FastDiv32 make_fastdiv32_dev(uint32_t d) {
    FastDiv32 f;
    if (d == 0) d = 1;
    f.d = d;
    const uint32_t l = (d > 1) ? 32 - __clz(d - 1) : 0;
    const uint64_t two_l = (uint64_t)1 << l;
    f.m = (uint32_t)((((two_l - d) << 32) / d) + 1);
    f.s1 = l ? 1 : 0;
    f.s2 = l ? l - 1 : 0;
    return f;
}

// -------------------------------------------------------------- cluster-split kernel
// Tiles larger than one CTA's shared memory: a thread-block cluster of K CTAs (K SMs)
// owns one tile; CTA k holds tile rows [k*m/K, (k+1)*m/K) and writes exactly the output
// columns those rows become (every output row is [slice 0 | slice 1 | ... ]), so no
// distributed-shared-memory traffic is needed.  The only cross-CTA hazard is in-place:
// no CTA may store into the tile before every CTA of the cluster has finished loading
// it -- one cluster barrier (release/acquire) per tile.  This lifts the paper's on-chip
// tile limit to K x 227 KB, which lets stages 1 and 3 use larger
// super-elements.
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int EB, int U, int MINB = 2>
__global__ void __launch_bounds__(512, MINB) tile_onchip_cluster(const TileParams p) {
    constexpr int V = 16 / EB;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t sbase = smem_u32(smem);
    const uint32_t K = p.K;
    const uint32_t rank = cluster_rank();
    const uint32_t cid = blockIdx.x / K, ncl = gridDim.x / K;
    const uint32_t mv = p.m / V, nvr = p.n / V;    // V-row blocks, 16-byte vectors per row
    uint32_t b0, b1, c0, c1, q;
    if (!p.colsplit) {   // rows [b0, b1) (V-row blocks), all columns
        b0 = (uint32_t)((uint64_t)rank * mv / K);
        b1 = (uint32_t)((uint64_t)(rank + 1) * mv / K);
        c0 = 0; c1 = nvr; q = p.q;
    } else {             // all rows, 16-byte columns [c0, c1) (one vector = V columns)
        b0 = 0; b1 = mv;
        c0 = (uint32_t)((uint64_t)rank * nvr / K);
        c1 = (uint32_t)((uint64_t)(rank + 1) * nvr / K);
        q = (c1 - c0) | 1u;
    }
    const uint32_t rows = (b1 - b0) * V, cvec = c1 - c0;
    const uint32_t nvec = rows * cvec;
    const FastDiv32 divmvp = make_fastdiv32_dev(b1 - b0);
    const FastDiv32 divc = make_fastdiv32_dev(cvec);
    for (uint64_t t = cid; t < p.count; t += ncl) {
        char *g = tile_ptr(p, t);
        const char *src = g + ((size_t)b0 * V * nvr + c0) * 16;
        for (uint32_t e0 = threadIdx.x; e0 < nvec; e0 += U * blockDim.x) {
            uint4 v[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t e = e0 + u * blockDim.x;
                if (e < nvec) {
                    uint32_t i, j;
                    fdivmod32(e, divc, i, j);
                    v[u] = ld_cg<16>(src + ((size_t)i * nvr + j) * 16);
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t e = e0 + u * blockDim.x;
                if (e < nvec) {
                    uint32_t i, j;
                    fdivmod32(e, divc, i, j);
                    sts128(sbase + (i * q + j) * 16, v[u]);
                }
            }
        }
        cluster_sync_all();     // every slice of tile t is on chip before anyone stores
        write_out<EB>(p, sbase, g, q, b0, b1 - b0, divmvp, c0, cvec);
        __syncthreads();        // shared slice consumed before the next tile's loads
    }
}

// Element loads of `cnt` contiguous elements (row length via divN) into an odd-pitch
// shared array, U loads in flight per thread.
template <typename T, int U = 8>
__device__ __forceinline__ void load_slice_scalar(T *s, const T *src, uint32_t cnt, uint32_t pitch,
                                                  const FastDiv32 &divN) {
    for (uint32_t e0 = threadIdx.x; e0 < cnt; e0 += U * blockDim.x) {
        T v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t e = e0 + u * blockDim.x;
            if (e < cnt) v[u] = src[e];
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t e = e0 + u * blockDim.x;
            if (e < cnt) {
                uint32_t i, j;
                fdivmod32(e, divN, i, j);
                s[i * pitch + j] = v[u];
            }
        }
    }
}

// Same with 16-byte vector loads (src 16-byte aligned, cnt * sizeof(T) % 16 == 0).
template <typename T, int U = 4>
__device__ __forceinline__ void load_slice_vec(T *s, const T *src, uint32_t cnt, uint32_t pitch,
                                               uint32_t n, const FastDiv32 &divN) {
    constexpr int PV = 16 / sizeof(T) > 0 ? 16 / sizeof(T) : 1;
    const uint32_t nvec = cnt / PV;
    for (uint32_t e0 = threadIdx.x; e0 < nvec; e0 += U * blockDim.x) {
        uint4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t e = e0 + u * blockDim.x;
            if (e < nvec) v[u] = ld_cg<16>(reinterpret_cast<const char *>(src) + (size_t)e * 16);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t e = e0 + u * blockDim.x;
            if (e < nvec) {
                union { uint4 w; T x[PV]; } uu;
                uu.w = v[u];
                uint32_t i, j;
                fdivmod32(e * PV, divN, i, j);
#pragma unroll
                for (int k = 0; k < PV; ++k) {
                    s[i * pitch + j] = uu.x[k];
                    if (++j == n) { j = 0; ++i; }
                }
            }
        }
    }
}

// ------------------------------------------------------------ streaming slice kernel
// One CTA per SM (slices > 113 KB, single CTA or cluster row split): the write-out of
// tile t and the load of tile t + 1 are overlapped inside the CTA.  The slice is processed
// in groups of 8 V-row blocks (each group writes 8*V*elem = 128 contiguous bytes into
// every output row); as soon as a group has been written out, the same group of the
// next tile is fetched into the freed shared memory with cp.async (no registers, so the
// stores of the following groups keep flowing).  The in-place rule is unchanged: no
// store into tile t+1 before every CTA of the cluster has finished loading it.
__device__ __forceinline__ void cp_async16(uint32_t sdst, const void *gsrc) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(sdst), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

template <int EB>
__global__ void __launch_bounds__(512, 1) tile_onchip_stream(const TileParams p) {
    constexpr int V = 16 / EB;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t sbase = smem_u32(smem);
    const uint32_t K = p.K ? p.K : 1;
    const uint32_t rank = (K > 1) ? cluster_rank() : 0;
    const uint32_t cid = blockIdx.x / K, ncl = gridDim.x / K;
    const uint32_t mv = p.m / V, nvr = p.n / V;
    uint32_t b0, b1, c0, c1, q;
    if (!p.colsplit) {   // row split: V-row blocks [b0, b1), all 16-byte columns
        b0 = (uint32_t)((uint64_t)rank * mv / K);
        b1 = (uint32_t)((uint64_t)(rank + 1) * mv / K);
        c0 = 0; c1 = nvr; q = p.q;
    } else {             // column split: all rows, 16-byte columns [c0, c1)
        b0 = 0; b1 = mv;
        c0 = (uint32_t)((uint64_t)rank * nvr / K);
        c1 = (uint32_t)((uint64_t)(rank + 1) * nvr / K);
        q = (c1 - c0) | 1u;
    }
    const uint32_t nb = b1 - b0, cvec = c1 - c0;
    // V-row blocks per group (measured, tools/tile_sweep.py with IPT_TILE_GROUP): 8 for
    // column slices, 16 for row slices (32 when rows are narrow)
    const uint32_t GB = p.gb ? p.gb : (p.colsplit ? 8u : (cvec >= 24 ? 16u : 32u));
    const uint32_t ngroups = (nb + GB - 1) / GB;
    const FastDiv32 divc = make_fastdiv32_dev(cvec);

    auto load_group = [&](const char *g, uint32_t grp) {   // cp.async rows of one group
        const uint32_t bl0 = grp * GB, bl1 = min(nb, bl0 + GB);
        const uint32_t rows = (bl1 - bl0) * V;
        const uint32_t cnt = rows * cvec;
        const char *src = g + ((size_t)(b0 + bl0) * V * nvr + c0) * 16;
        const uint32_t srow0 = bl0 * V;
        for (uint32_t e = threadIdx.x; e < cnt; e += blockDim.x) {
            uint32_t i, j;
            fdivmod32(e, divc, i, j);
            cp_async16(sbase + ((srow0 + i) * q + j) * 16, src + ((size_t)i * nvr + j) * 16);
        }
    };

    uint64_t t = cid;
    if (t < p.count) {
        const char *g = tile_ptr(p, t);
        for (uint32_t grp = 0; grp < ngroups; ++grp) load_group(g, grp);
        cp_async_commit();
    }
    for (; t < p.count; t += ncl) {
        char *g = tile_ptr(p, t);
        cp_async_wait_all();
        __syncthreads();
        if (K > 1) cluster_sync_all();   // all slices of tile t on chip before any store
        const uint64_t tn = t + ncl;
        const char *gn = (tn < p.count) ? tile_ptr(p, tn) : nullptr;
        for (uint32_t grp = 0; grp < ngroups; ++grp) {
            const uint32_t bl0 = grp * GB, cntb = min(nb, bl0 + GB) - bl0;
            const FastDiv32 dv = make_fastdiv32_dev(cntb);
            write_out<EB>(p, sbase + bl0 * V * q * 16, g, q, b0 + bl0, cntb, dv, c0, cvec);
            __syncthreads();                 // group consumed -> refill with tile t + 1
            if (gn) load_group(gn, grp);
            cp_async_commit();
        }
    }
    cp_async_wait_all();
}

// -------------------------------------------------- group-split double-buffered kernel
// Tiles too large for a cluster's shared memory with double buffering: a group of K
// co-resident CTAs anywhere on the GPU (cooperative launch; clusters are confined to one
// GPC, which leaves up to a quarter of the SMs idle at K = 16) owns one tile at a time;
// CTA k holds slice k (as the cluster kernel) in one of two buffers.  While tile t is
// written out from one buffer, tile t + groups is fetched into the other with cp.async.
// In-place rule: a CTA arrives on the group's counter once its slice of a tile is on
// chip, and stores into that tile only after all K have arrived.  Arrival for the next
// tile is signalled half-way through the current write-out, so the wait is normally
// already satisfied (a CTA only arrives for tile i+1 after passing the wait for tile i,
// hence the cumulative count K*(i+1) identifies tile i).
// Memory ordering: an arrival reports that this CTA's READS of the tile have completed
// (their data is in shared memory; the CTA observed that through the mbarrier), and the
// waiters then WRITE the tile -- a load-buffering shape, not message passing.  A release
// would only order this CTA's earlier *writes* (the previous tile's write-out, which no
// waiter reads) and costs a MEMBAR.GPU that drains them: 25 % of a copy pipeline's
// bandwidth (tools/probe_copy.py, 4.7 vs 5.9 TB/s).  So the arrival is relaxed; the
// waiter's acquire poll keeps its stores after the observed count (stores are never
// performed before the loop exit they depend on).  IPT_TILE_ARRIVE_RELEASE=1 restores it.
__device__ __forceinline__ void group_arrive(uint32_t *ctr, bool release) {
    if (release) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
    else asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" :: "l"(ctr) : "memory");
}
__device__ __forceinline__ uint64_t global_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Spin until the counter reaches `target`.  Co-residency is guaranteed by the cooperative
// launch; the watchdog turns a violated guarantee into a launch error instead of a hang.
__device__ __forceinline__ void group_wait(const uint32_t *ctr, uint32_t target) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
    if (v >= target) return;
    const uint64_t t0 = global_ns();
    do {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
        if (global_ns() - t0 > 20000000000ull) __trap();   // 20 s
    } while (v < target);
}

constexpr uint32_t kGroupMaxBuf = 4;
constexpr uint32_t kTraceIters = 64;   // diag trace: iterations recorded per CTA
constexpr size_t kTraceBytes = 1024 * kTraceIters * 4 * 8;
static unsigned long long *g_trace = nullptr;

// Ring of p.nbuf slice buffers shared by the group kernels.  Iteration j of a group
// handles tile gid + j*groups in buffer j % nbuf; the loads of tile j + nbuf - 1 are
// issued at the start of iteration j, so a slice has nbuf - 1 write-outs to land.  Its
// cp.async copies arrive on the buffer's mbarrier (cp.async.mbarrier.arrive: no warp
// stalls on them); thread 0 probes the barriers while writing and signals the group, in
// tile order, once each slice has landed.  One counter per (group, buffer): a CTA arrives
// for tile j + nbuf only after finishing tile j, i.e. after all K arrivals for tile j, so
// counter j % nbuf reaching K * (j / nbuf + 1) means exactly "every slice of tile j is on
// chip".
struct GroupPipe {
    uint64_t *mbar;     // nbuf mbarriers in shared memory
    uint32_t *ctr;      // this group's counters, kGroupCtrStride bytes apart
    uint32_t K, nbuf;
    bool release;       // arrive with release semantics (IPT_TILE_ARRIVE_RELEASE=1)
    uint32_t na = 0;    // thread 0: next iteration to arrive for
    __device__ void init() {
        if (threadIdx.x == 0) {
            for (uint32_t b = 0; b < nbuf; ++b) mbar_init(&mbar[b], blockDim.x);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
        __syncthreads();
    }
    __device__ uint32_t *slot(uint32_t j) const { return ctr + (j % nbuf) * (kGroupCtrStride / 4); }
    __device__ void issued(uint32_t j) { cp_async_mbar_arrive(&mbar[j % nbuf]); }
    __device__ bool landed(uint32_t j) { return mbar_test_wait(&mbar[j % nbuf], (j / nbuf) & 1); }
    __device__ void wait_landed(uint32_t j) { mbar_wait(&mbar[j % nbuf], (j / nbuf) & 1); }
    __device__ void probe(uint32_t limit) {          // thread 0
        while (na < limit && landed(na)) group_arrive(slot(na++), release);
    }
    __device__ void force(uint32_t j) {              // thread 0: arrivals up to j
        while (na <= j) {
            wait_landed(na);
            group_arrive(slot(na++), release);
        }
    }
    __device__ void wait_group(uint32_t j) { group_wait(slot(j), K * (j / nbuf + 1)); }
};

// Main loop of a group kernel: load(tile pointer, buffer address) issues the cp.async
// copies of one slice; write(tile pointer, buffer address, probe) writes one out, calling
// probe() now and then.  (Waiting for the next slice half-way through the write-out and
// arriving then, with all warps, measured 2-8 % slower than thread 0 probing.)
template <typename Load, typename Write>
__device__ __forceinline__ void group_loop(const TileParams &p, uint32_t s0, uint64_t *mbar,
                                           Load load, Write write) {
    const uint32_t K = p.K, gid = blockIdx.x / K, ng = gridDim.x / K;
    GroupPipe pipe;
    pipe.mbar = mbar;
    pipe.ctr = p.gbar + gid * p.nbuf * (kGroupCtrStride / 4);
    pipe.K = K;
    pipe.nbuf = p.nbuf;
    pipe.release = p.arrive_release != 0;
    pipe.init();
    const uint32_t nt = gid < p.count ? (uint32_t)((p.count - gid + ng - 1) / ng) : 0;
    auto issue = [&](uint32_t j) {
        if (!(p.diag & 4)) load(tile_ptr(p, gid + (uint64_t)j * ng), s0 + (j % p.nbuf) * p.buf_bytes);
        pipe.issued(j);
    };
    for (uint32_t j = 0; j + 1 < p.nbuf && j < nt; ++j) issue(j);
    // timeline trace (diag 16): per CTA and iteration, globaltimer at start, own slice
    // landed, group complete, write-out done
    unsigned long long *tr = (p.diag & 16) && threadIdx.x == 0 ? p.trace + (uint64_t)blockIdx.x * kTraceIters * 4 : nullptr;
    for (uint32_t i = 0; i < nt; ++i) {
        if (tr && i < kTraceIters - 1) tr[i * 4 + 0] = global_ns();
        const uint32_t jn = i + p.nbuf - 1;
        if (jn < nt) issue(jn);
        const uint32_t lim = min(nt, jn + 1);
        pipe.wait_landed(i);                         // own slice of tile i on chip
        if (threadIdx.x == 0) {
            if (tr && i < kTraceIters - 1) tr[i * 4 + 1] = global_ns();
            pipe.force(i);
            if (!(p.diag & 1)) pipe.wait_group(i);   // every slice of tile i on chip
            if (tr && i < kTraceIters - 1) tr[i * 4 + 2] = global_ns();
        }
        __syncthreads();
        if (!(p.diag & 2)) write(tile_ptr(p, gid + (uint64_t)i * ng) + ((p.diag & 32) ? p.count * p.tile_bytes : 0),
              s0 + (i % p.nbuf) * p.buf_bytes,
              [&]() { if (threadIdx.x == 0) pipe.probe(lim); });
        __syncthreads();                             // buffer i % nbuf free
        if (tr && i < kTraceIters - 1) tr[i * 4 + 3] = global_ns();
    }
    if (tr) {   // last trace slot: the SM this CTA ran on
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        tr[(kTraceIters - 1) * 4] = smid;
    }
    if (p.gexit && threadIdx.x == 0) {
        // self-resetting counters: the last CTA of the group to finish (no CTA of it polls
        // any more) zeroes the group's arrival counters and its exit counter, so the next
        // launch on this stream starts from zero without a memset node
        uint32_t *ex = p.gexit + gid * (kGroupCtrStride / 4);
        if (atomicAdd(ex, 1u) == K - 1) {
            for (uint32_t b = 0; b < p.nbuf; ++b) atomicExch(pipe.slot(b), 0u);
            atomicExch(ex, 0u);
        }
    }
}

template <int EB>
__global__ void __launch_bounds__(512, 1) tile_group_db(const TileParams p) {
    constexpr int V = 16 / EB;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t s0 = smem_u32(smem);
    const uint32_t K = p.K;
    const uint32_t rank = blockIdx.x % K;
    const uint32_t mv = p.m / V, nvr = p.n / V;
    uint32_t b0, b1, c0, c1, q;
    if (!p.colsplit) {
        b0 = (uint32_t)((uint64_t)rank * mv / K);
        b1 = (uint32_t)((uint64_t)(rank + 1) * mv / K);
        c0 = 0; c1 = nvr; q = p.q;
    } else {
        b0 = 0; b1 = mv;
        c0 = (uint32_t)((uint64_t)rank * nvr / K);
        c1 = (uint32_t)((uint64_t)(rank + 1) * nvr / K);
        q = (c1 - c0) | 1u;
    }
    const uint32_t nb = b1 - b0, cvec = c1 - c0;
    const uint32_t cnt = nb * V * cvec;
    const FastDiv32 divc = make_fastdiv32_dev(cvec), divnb = make_fastdiv32_dev(nb);
    __shared__ __align__(8) uint64_t mbar[kGroupMaxBuf];
    group_loop(p, s0, mbar,
        [&](const char *g, uint32_t sb) {
            const char *src = g + ((size_t)b0 * V * nvr + c0) * 16;
            for (uint32_t e = threadIdx.x; e < cnt; e += blockDim.x) {
                uint32_t i, j;
                fdivmod32(e, divc, i, j);
                cp_async16(sb + (i * q + j) * 16, src + ((size_t)i * nvr + j) * 16);
            }
        },
        [&](char *g, uint32_t sb, auto probe) {
            write_out<EB>(p, sb, g, q, b0, nb, divnb, c0, cvec, probe);
        });
}

// --------------------------------------------------- group-split kernel, TMA slices
// As tile_group_db, but each slice is fetched by 2-D tensor copies (cp.async.bulk.tensor,
// the TMA engine) from a tensor map over the stacked tiles ((count*m) rows x n columns):
// one copy per box of box_rows rows x (q*V) columns lands the slice at an odd pitch of q
// 16-byte vectors (columns beyond n are zero-filled, columns of the neighbour slice are
// read but never written), so no thread issues per-vector loads.
__device__ __forceinline__ void tma_load_2d(uint32_t sdst, const CUtensorMap *tm, int32_t x, int32_t y,
                                            uint32_t sbar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        :: "r"(sdst), "l"(tm), "r"(x), "r"(y), "r"(sbar) : "memory");
}

template <int EB>
__global__ void __launch_bounds__(512, 1) tile_group_tma(const TileParams p, const __grid_constant__ CUtensorMap tmap) {
    constexpr int V = 16 / EB;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t s0 = smem_u32(smem);
    const uint32_t K = p.K;
    const uint32_t rank = blockIdx.x % K;
    const uint32_t mv = p.m / V, nvr = p.n / V;
    uint32_t b0, b1, c0, c1;
    if (!p.colsplit) {
        b0 = (uint32_t)((uint64_t)rank * mv / K);
        b1 = (uint32_t)((uint64_t)(rank + 1) * mv / K);
        c0 = 0; c1 = nvr;
    } else {
        b0 = 0; b1 = mv;
        c0 = (uint32_t)((uint64_t)rank * nvr / K);
        c1 = (uint32_t)((uint64_t)(rank + 1) * nvr / K);
    }
    const uint32_t q = p.q;   // panel width in vectors (odd), the same for every CTA
    const uint32_t nb = b1 - b0, cvec = c1 - c0;
    const uint32_t rows = p.colsplit ? p.m : (uint32_t)(((uint64_t)mv + K - 1) / K) * V;  // rows fetched
    const uint32_t pstride = p.pstride;
    const FastDiv32 divnb = make_fastdiv32_dev(nb), divq = make_fastdiv32_dev(q);
    __shared__ __align__(8) uint64_t mbar[kGroupMaxBuf];
    group_loop(p, s0, mbar,
        [&](const char *g, uint32_t sb) {
            if (threadIdx.x == 0) {
                const uint64_t row0 = (uint64_t)(g - p.base) / ((uint64_t)p.n * EB) + (uint64_t)b0 * V;
                uint64_t *bar = &mbar[(sb - s0) / p.buf_bytes];
                mbar_expect_tx(bar, p.npan * rows * q * 16);
                const uint32_t sbar = smem_u32(bar);
                for (uint32_t pn = 0; pn < p.npan; ++pn)
                    for (uint32_t r = 0; r < rows; r += p.box_rows)
                        tma_load_2d(sb + pn * pstride + r * q * 16, &tmap, (int32_t)((c0 + pn * q) * V),
                                    (int32_t)(row0 + r), sbar);
            }
        },
        [&](char *g, uint32_t sb, auto probe) {
            write_out_pan<EB>(p, sb, g, q, divq, pstride, b0, nb, divnb, c0, cvec, probe);
        });
}

// ------------------- whole-GPU tiles held in shared memory AND tensor memory (rf)
// Tiles too large even for single-buffered slices over every SM (e.g. one 4096 x 3000 or
// 1800 x 7200 float32 matrix, 49-52 MB, as ONE tile: the plan m = M, n = N, stages 1 and 3
// identities -- P:315's "tile fits on chip" taken to the whole B200).  The aggregate
// on-chip storage of 148 SMs is shared memory (148 x 227 KB) plus Blackwell's tensor memory
// (TMEM, 148 x 256 KB, otherwise the MMA accumulator store; here plain staging).  A group of
// K CTAs (one per SM, 512 threads) owns a tile; CTA k's slice (row or column split, as
// tile_group_tma) is held as
//   part A: its first rows_a rows, fetched by 2-D TMA boxes into the column-panel layout;
//   part B: the remaining rows, loaded by the threads with 16-byte loads (consecutive
//           threads, consecutive vectors of a row) and parked in TMEM with tcgen05.st --
//           each thread owns 128 columns of its warp's lane quarter (512 B, RV <= 32
//           vectors), so no register is held across the write-out.
// In-place rule as the group kernels: the CTA arrives on the group counter once part A has
// landed (mbarrier) and every part-B load has returned (its value was stored to TMEM), and
// no CTA stores into the tile before all K arrived.  Write-out: part A from shared memory
// (write_out_pan: transposed V x V register blocks, coalesced 16-byte stores), then part B
// is brought back (tcgen05.ld), stored into the freed shared memory in the same panel layout
// and written out the same way.  Tiles of a group run one after another (a batch: the
// spread of the CTAs overlaps one tile's stores with the next tile's loads across the GPU).
__device__ __forceinline__ void tma_load_3d_t(uint32_t sdst, const CUtensorMap *tm, int32_t x, int32_t y,
                                              int32_t z, uint32_t sbar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
        :: "r"(sdst), "l"(tm), "r"(x), "r"(y), "r"(z), "r"(sbar) : "memory");
}
__device__ __forceinline__ void tm_st4(uint32_t taddr, const uint4 &v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};"
                 :: "r"(taddr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ uint4 tm_ld4(uint32_t taddr) {
    uint4 v;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(taddr) : "memory");
    return v;
}

constexpr int kRfBatch = 8;   // part-B vectors per thread in registers at a time
// Part-B loads in flight per thread on the one-chunk path: half of the thread's vectors
// (two round trips), at least 8 -- rv = 24: 12 per batch, measured C5 4.92 -> 5.01 TB/s
// (8: 4.92, 10: 4.89, 12: 5.01, 14: 4.93, 16: 4.88, 24: 4.92; 512 matrices)
constexpr int rf_load_batch(int rv) { return rv / 2 < 8 ? 8 : rv / 2; }

// Part B is handled in chunks (cb rows x cpan panels of the slice, staged through a
// region of shared memory after part A's): chunk k's vectors are numbered consecutively
// from base_k (E = base_k + row * ncols_k + col; every base a multiple of 512, so no
// thread's TMEM column group is shared by two chunks -- tcgen05.st writes all 32 lanes),
// thread E % 512 holds vector E in its TMEM columns 4 * (E / 512) .. +3.
struct RfChunk {
    uint32_t r0, nr, c0, nc, base;   // rows / vector columns of part B, first E
};
__device__ __forceinline__ RfChunk rf_chunk(const TileParams &p, uint32_t k, uint32_t rb, uint32_t cvec) {
    const uint32_t cw = p.cpan * p.q;                              // chunk width (vectors)
    const uint32_t npc = (cvec + cw - 1) / cw;                     // panel chunks per row chunk
    RfChunk c{};
    uint32_t base = 0;
    for (uint32_t j = 0; j <= k; ++j) {
        const uint32_t kr = j / npc, kc = j % npc;
        c.r0 = kr * p.rows_b;
        c.nr = min(p.rows_b, rb - c.r0);
        c.c0 = kc * cw;
        c.nc = min(cw, cvec - c.c0);
        c.base = base;
        base += (c.nr * c.nc + 511) / 512 * 512;
    }
    return c;
}

template <int EB, int RV, bool CH, bool SWZ = false>
__global__ void __launch_bounds__(512, 1) tile_group_rf(const TileParams p, const __grid_constant__ CUtensorMap tmap) {
    constexpr int V = 16 / EB;
    static_assert(RV % kRfBatch == 0 && RV <= 32, "TMEM holds 32 vectors per thread");
    static_assert(!(SWZ && CH), "swizzled slices are staged in one chunk");
    extern __shared__ __align__(128) unsigned char smem[];
    // SWZ: column slices of exactly 8 vectors (one 128-byte line per row) in the TMA 128-byte
    // swizzle, whose pattern repeats every 1024 bytes of shared memory address
    const uint32_t s0 = SWZ ? (smem_u32(smem) + 1023u) & ~1023u : smem_u32(smem);
    const uint32_t K = p.K, rank = blockIdx.x % K, gid = blockIdx.x / K, ng = gridDim.x / K;
    const uint32_t warp = threadIdx.x >> 5, tid = threadIdx.x;
    const uint32_t mv = p.m / V, nvr = p.n / V;
    uint32_t b0, b1, c0, c1;
    if (!p.colsplit) {   // row slices in units of ralign V-row blocks (sector-aligned pieces)
        const uint32_t ra_ = p.ralign ? p.ralign : 1u, units = mv / ra_;
        b0 = (uint32_t)((uint64_t)rank * units / K) * ra_;
        b1 = rank + 1 == K ? mv : (uint32_t)((uint64_t)(rank + 1) * units / K) * ra_;
        c0 = 0; c1 = nvr;
    } else {             // column slices in units of ralign vectors (sector-aligned pieces)
        const uint32_t ra_ = p.ralign ? p.ralign : 1u, units = nvr / ra_;
        b0 = 0; b1 = mv;
        c0 = (uint32_t)((uint64_t)rank * units / K) * ra_;
        c1 = rank + 1 == K ? nvr : (uint32_t)((uint64_t)(rank + 1) * units / K) * ra_;
    }
    const uint32_t q = p.q, cvec = c1 - c0;
    const uint32_t rows = (b1 - b0) * V, r0 = b0 * V;
    const uint32_t ra = min(p.rows_a, rows), rb = rows - ra;        // rows in smem / TMEM
    const uint32_t nvb = rb * cvec;                                    // part-B vectors of the slice
    // CH: part B in several chunks (compiled separately: the one-chunk kernel stays lean)
    const uint32_t nchunk = !rb ? 0 : (!CH ? 1 : ((rb + p.rows_b - 1) / p.rows_b) *
                                                 ((cvec + p.cpan * q - 1) / (p.cpan * q)));
    const uint32_t pstride_b = (((CH ? p.rows_b : rb) * q * 16) + 127) & ~127u;
    const FastDiv32 divq = make_fastdiv32_dev(q), divc = make_fastdiv32_dev(cvec);
    const FastDiv32 diva = make_fastdiv32_dev(ra / V), divb = make_fastdiv32_dev(rb / V);
    __shared__ __align__(8) uint64_t mbar;
    __shared__ uint32_t tmem_base;
    if (warp == 0) {   // all 512 TMEM columns of this SM (one CTA per SM)
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;"
                     :: "r"(smem_u32(&tmem_base)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    if (tid == 0) {
        mbar_init(&mbar, 1);
        fence_mbar_init();
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    // this thread's 128 columns in its warp's lane quarter
    const uint32_t taddr = tmem_base + ((32u * (warp & 3)) << 16) + (warp >> 2) * 128u;
    uint32_t *ctr = p.gbar + gid * (kGroupCtrStride / 4);
    const uint32_t nt = gid < p.count ? (uint32_t)((p.count - gid + ng - 1) / ng) : 0;
    // timeline trace (IPT_TILE_DIAG=16; tools/rf_trace.py): per CTA and tile, globaltimer at
    // start, part B parked, part A landed, group complete, A written, B staged, B written
    unsigned long long *tr = (p.diag & 16) && tid == 0 ? p.trace + (uint64_t)blockIdx.x * 256 : nullptr;
    auto mark = [&](uint32_t i, int k) { if (tr && i < 31) tr[i * 8 + k] = global_ns(); };
    if (tr) {   // last slot: the SM this CTA runs on
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        tr[31 * 8] = smid;
    }
    for (uint32_t i = 0; i < nt; ++i) {
        const uint64_t t = gid + (uint64_t)i * ng;
        char *g = tile_ptr(p, t);
        mark(i, 0);
        // ---- part A: TMA boxes (rows_a rows of every panel; boxes may read past the slice)
        if (tid == 0) {
            mbar_arrive_expect_tx(&mbar, p.npan * p.rows_a * q * 16);
            const uint32_t sbar = smem_u32(&mbar);
            for (uint32_t pn = 0; pn < p.npan; ++pn)
                for (uint32_t r = 0; r < p.rows_a; r += p.box_rows) {
                    const int32_t x = (int32_t)((c0 + pn * q) * V);
                    const uint32_t dst = s0 + pn * p.pstride + r * q * 16;
                    if (p.rres)   // strided batch: 3-D map (columns, rows, tiles)
                        tma_load_3d_t(dst, &tmap, x, (int32_t)(r0 + r), (int32_t)t, sbar);
                    else          // tiles stacked: 2-D map (columns, rows of all tiles)
                        tma_load_2d(dst, &tmap, x, (int32_t)(t * p.m + r0 + r), sbar);
                }
        }
        // ---- part B: 16-byte loads parked in TMEM (thread E % 512 holds vector E in its
        // columns 4 * (E / 512); with several chunks, chunk k's vectors start at base_k)
        if (!(p.diag & 4) && !CH) {   // one chunk: every thread's vectors E < nvb
            // (batches of LB loads, each parked before the next is issued: all of a thread's
            // loads in flight measured slower -- 4.39 vs 4.34 TB/s on C5, 3.3 vs 3.0 on one
            // C1 matrix, first version)
            const char *gb = g + ((size_t)(r0 + ra) * nvr + c0) * 16;
#pragma unroll 1
            constexpr int LB = rf_load_batch(RV);
            for (int u0 = 0; u0 < RV; u0 += LB) {
                if ((uint32_t)u0 * 512 >= nvb) break;
                uint4 v[LB];
#pragma unroll
                for (int j = 0; j < LB; ++j) {
                    const uint32_t e = tid + (uint32_t)(u0 + j) * 512;
                    v[j] = make_uint4(0, 0, 0, 0);
                    if (u0 + j < RV && e < nvb) {
                        uint32_t r, c;
                        fdivmod32(e, divc, r, c);
                        v[j] = ld_cg<16>(gb + ((size_t)r * nvr + c) * 16);
                    }
                }
#pragma unroll
                for (int j = 0; j < LB; ++j)
                    if (u0 + j < RV) tm_st4(taddr + 4u * (uint32_t)(u0 + j), v[j]);
            }
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
            mark(i, 1);
        } else if (!(p.diag & 4)) {
            for (uint32_t k = 0; CH && k < nchunk; ++k) {
                const RfChunk c = rf_chunk(p, k, rb, cvec);
                const uint32_t n = c.nr * c.nc, uhi = (c.base + n + 511) / 512;
                const FastDiv32 dnc = make_fastdiv32_dev(c.nc);
                const char *gb = g + ((size_t)(r0 + ra + c.r0) * nvr + c0 + c.c0) * 16;
#pragma unroll 1
                for (uint32_t u0 = c.base / 512; u0 < uhi; u0 += kRfBatch) {
                    uint4 v[kRfBatch];
#pragma unroll
                    for (int j = 0; j < kRfBatch; ++j) {
                        const uint32_t E = tid + (u0 + j) * 512;
                        v[j] = make_uint4(0, 0, 0, 0);
                        if (E >= c.base && E < c.base + n) {
                            uint32_t r, cc;
                            fdivmod32(E - c.base, dnc, r, cc);
                            v[j] = ld_cg<16>(gb + ((size_t)r * nvr + cc) * 16);
                        }
                    }
#pragma unroll
                    for (int j = 0; j < kRfBatch; ++j)
                        if (u0 + j < uhi) tm_st4(taddr + 4u * (u0 + j), v[j]);   // warp-uniform bound
                }
            }
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        }
        mbar_wait(&mbar, i & 1);            // part A has landed
        mark(i, 2);
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        if (tid == 0) {
            group_arrive(ctr, p.arrive_release != 0);
            if (!(p.diag & 1)) group_wait(ctr, K * (i + 1));   // all slices of the tile on chip
        }
        mark(i, 3);
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        // ---- write-out: part A, then part B (chunk by chunk) through the freed shared memory
        // diag 32 (measurement): stores to a second buffer after the data (out of place)
        char *const gw = (p.diag & 32) ? g + p.count * p.tile_bytes : g;
        if (ra && !(p.diag & 2))
            write_out_pan<EB, NoProbe, SWZ>(p, s0, gw, q, divq, p.pstride, r0 / V, ra / V, diva, c0, cvec, NoProbe());
        __syncthreads();
        mark(i, 4);
        if (!CH && nchunk) {   // one chunk: the whole part B through the freed shared memory
#pragma unroll 1
            for (int u0 = 0; u0 < RV; u0 += kRfBatch) {
                if ((uint32_t)u0 * 512 >= nvb) break;
                uint4 v[kRfBatch];
#pragma unroll
                for (int j = 0; j < kRfBatch; ++j) v[j] = tm_ld4(taddr + 4u * (uint32_t)(u0 + j));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
                for (int j = 0; j < kRfBatch; ++j) {
                    const uint32_t e = tid + (uint32_t)(u0 + j) * 512;
                    if (e < nvb) {
                        uint32_t r, c, pn, pc;
                        fdivmod32(e, divc, r, c);
                        fdivmod32(c, divq, pn, pc);
                        sts128(SWZ ? s0 + r * 128 + ((pc ^ (r & 7)) << 4) : s0 + pn * pstride_b + (r * q + pc) * 16, v[j]);
                    }
                }
            }
            __syncthreads();
            mark(i, 5);
            if (!(p.diag & 2))
                write_out_pan<EB, NoProbe, SWZ>(p, s0, gw, q, divq, pstride_b, (r0 + ra) / V, rb / V, divb, c0, cvec, NoProbe());
        }
        for (uint32_t k = 0; CH && k < nchunk; ++k) {
            const RfChunk c = rf_chunk(p, k, rb, cvec);
            const uint32_t n = c.nr * c.nc, uhi = (c.base + n + 511) / 512;
            const FastDiv32 dnc = make_fastdiv32_dev(c.nc);
#pragma unroll 1
            for (uint32_t u0 = c.base / 512; u0 < uhi; u0 += kRfBatch) {
                uint4 v[kRfBatch];
#pragma unroll
                for (int j = 0; j < kRfBatch; ++j)
                    if (u0 + j < uhi) v[j] = tm_ld4(taddr + 4u * (u0 + j));
                asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
                for (int j = 0; j < kRfBatch; ++j) {
                    const uint32_t E = tid + (u0 + j) * 512;
                    if (u0 + j < uhi && E >= c.base && E < c.base + n) {
                        uint32_t r, cc, pn, pc;
                        fdivmod32(E - c.base, dnc, r, cc);
                        fdivmod32(cc, divq, pn, pc);
                        sts128(s0 + pn * pstride_b + (r * q + pc) * 16, v[j]);
                    }
                }
            }
            __syncthreads();
            if (!(p.diag & 2))
                write_out_pan<EB>(p, s0, gw, q, divq, pstride_b, (r0 + ra + c.r0) / V, c.nr / V,
                                  make_fastdiv32_dev(c.nr / V), c0 + c.c0, c.nc, NoProbe());
            __syncthreads();
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        mark(i, 6);
    }
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem_base) : "memory");
    if (p.gexit && tid == 0) {   // self-resetting counters (see group_loop)
        uint32_t *ex = p.gexit + gid * (kGroupCtrStride / 4);
        if (atomicAdd(ex, 1u) == K - 1) {
            atomicExch(ctr, 0u);
            atomicExch(ex, 0u);
        }
    }
}

// --------------------------------- group-split element path with TMA slices (aligned rows)
// Element-path tiles whose INPUT rows are 16-byte aligned (n * elem % 16 == 0, row split)
// while the output rows are not (m % (16/elem) != 0, e.g. 9998 x 192 or 14803 x 128
// panels): slices are fetched as tile_group_tma does (2-D TMA boxes into column panels of q
// odd vectors; boxes may cover the next tile's first rows -- read, never used), the
// write-out reads one aligned LDS.128 per lane and 4 columns (no realignment) and stores one
// element per lane and output row (32 consecutive output elements per warp store).
template <int EB>
__global__ void __launch_bounds__(512, 1) tile_group_tma_elem(const TileParams p, const __grid_constant__ CUtensorMap tmap) {
    constexpr uint32_t V = 16 / EB;
    using E = typename Elem<EB>::T;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t s0 = smem_u32(smem);
    const uint32_t K = p.K, rank = blockIdx.x % K;
    const uint32_t mvc = (p.m + V - 1) / V;                    // V-row blocks (last partial)
    const uint32_t b0 = (uint32_t)((uint64_t)rank * mvc / K), b1 = (uint32_t)((uint64_t)(rank + 1) * mvc / K);
    const uint32_t r0 = b0 * V, r1 = min(b1 * V, p.m);
    const uint32_t rows = r1 > r0 ? r1 - r0 : 0;
    const uint32_t frows = ((mvc + K - 1) / K) * V;            // rows fetched per slice
    const uint32_t q = p.q, nvr = p.n / V;
    constexpr uint32_t CH = 8;                                   // vector columns per task
    const uint32_t nrb = (rows + 31) / 32, nch = (nvr + CH - 1) / CH, ntask = nrb * nch;
    const FastDiv32 divrb = make_fastdiv32_dev(nrb ? nrb : 1), divq = make_fastdiv32_dev(q);
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    const uint64_t mEB = (uint64_t)p.m * EB;
    __shared__ __align__(8) uint64_t mbar[kGroupMaxBuf];
    group_loop(p, s0, mbar,
        [&](const char *g, uint32_t sb) {
            if (threadIdx.x == 0) {
                const uint64_t row0 = (uint64_t)(g - p.base) / ((uint64_t)p.n * EB) + r0;
                uint64_t *bar = &mbar[(sb - s0) / p.buf_bytes];
                mbar_expect_tx(bar, p.npan * frows * q * 16);
                const uint32_t sbar = smem_u32(bar);
                for (uint32_t pn = 0; pn < p.npan; ++pn)
                    for (uint32_t r = 0; r < frows; r += p.box_rows)
                        tma_load_2d(sb + pn * p.pstride + r * q * 16, &tmap, (int32_t)(pn * q * V),
                                    (int32_t)(row0 + r), sbar);
            }
        },
        [&](char *g, uint32_t sb, auto probe) {
            for (uint32_t task = warp; task < ntask; task += nw) {
                probe();
                uint32_t ch, rb;
                fdivmod32(task, divrb, ch, rb);
                const uint32_t i = rb * 32 + lane;
                if (i >= rows) continue;
                char *out = g + ((uint64_t)(ch * CH) * V * p.m + r0 + i) * EB;
#pragma unroll 2
                for (uint32_t cbl = 0; cbl < CH; ++cbl) {
                    const uint32_t cv = ch * CH + cbl;
                    if (cv >= nvr) break;
                    uint32_t pan, pc;
                    fdivmod32(cv, divq, pan, pc);
                    E x[V];
                    unpack<EB>(lds128(sb + pan * p.pstride + (i * q + pc) * 16), x);
                    char *oc = out + (uint64_t)cbl * V * mEB;
#pragma unroll
                    for (uint32_t k = 0; k < V; ++k) *reinterpret_cast<E *>(oc + k * mEB) = x[k];
                }
            }
        });
}

// ------------------------------------------------- group-split element-path kernel
// Tiles whose sides are not multiples of 16/elem (e.g. 64 x 9998 or 14803 x 32 floats),
// 4- and 8-byte elements, over a CTA group as tile_group_db.  A slice is a set of row
// pieces: rows [r0, r1) x columns [c0, c1) (row split: all columns; column split: all
// rows).  Each piece is fetched with cp.async as the 16-byte vectors covering it, kept at
// its global 16-byte phase (sh = first element's offset in its vector) in a shared row of
// Q vectors (Q odd).  Write-out: a warp takes 32 consecutive rows x PV consecutive
// columns; each lane reads the two vectors holding its PV elements, aligns them with a
// select network, and the warp stores PV runs of 32 consecutive output elements.
template <int EB>
__global__ void __launch_bounds__(512, 1) tile_group_generic(const TileParams p) {
    constexpr uint32_t PV = 16 / EB;
    using E = typename Elem<EB>::T;
    extern __shared__ __align__(128) unsigned char smem[];
    const uint32_t s0 = smem_u32(smem);
    const uint32_t K = p.K;
    const uint32_t rank = blockIdx.x % K;
    uint32_t r0, r1, c0, c1;
    if (p.gcols > 1) {   // 2-D grid: output pieces of (m / gr) elements, input pieces n / gc
        const uint32_t gc = p.gcols, gr = K / gc, ri = rank / gc, ci = rank % gc;
        r0 = (uint32_t)((uint64_t)ri * p.m / gr);
        r1 = (uint32_t)((uint64_t)(ri + 1) * p.m / gr);
        c0 = (uint32_t)((uint64_t)ci * p.n / gc);
        c1 = (uint32_t)((uint64_t)(ci + 1) * p.n / gc);
    } else if (p.colsplit) {
        r0 = 0; r1 = p.m;
        c0 = (uint32_t)((uint64_t)rank * p.n / K);
        c1 = (uint32_t)((uint64_t)(rank + 1) * p.n / K);
    } else {
        c0 = 0; c1 = p.n;
        r0 = (uint32_t)((uint64_t)rank * p.m / K);
        r1 = (uint32_t)((uint64_t)(rank + 1) * p.m / K);
    }
    const uint32_t rows = r1 - r0, L = c1 - c0, Q = p.q;
    const uint32_t QV = (L + 2 * PV - 2) / PV;            // covering vectors, worst phase
    const FastDiv32 divq = make_fastdiv32_dev(QV);
    constexpr uint32_t CH = 8;                            // column blocks per write task
    const uint32_t nrb = (rows + 31) / 32, ncb = (L + PV - 1) / PV, nch = (ncb + CH - 1) / CH;
    const uint32_t ntask = nrb * nch;
    const FastDiv32 divrb = make_fastdiv32_dev(nrb);
    const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    const uint64_t mEB = (uint64_t)p.m * EB;
    __shared__ __align__(8) uint64_t mbar[kGroupMaxBuf];

    auto load = [&](const char *g, uint32_t sb) {
        const uint32_t cnt = rows * QV;
        for (uint32_t e = threadIdx.x; e < cnt; e += blockDim.x) {
            uint32_t i, j;
            fdivmod32(e, divq, i, j);
            const uintptr_t a = (uintptr_t)(g + ((uint64_t)(r0 + i) * p.n + c0) * EB);
            const uint32_t sh = (uint32_t)(a & 15) / EB;
            if (j * PV < sh + L) cp_async16(sb + (i * Q + j) * 16, (const void *)((a & ~(uintptr_t)15) + j * 16));
        }
    };
    // Task (column chunk ch, row block rb), row blocks fastest: the warps of a CTA write
    // adjacent 32-element runs of the same output rows.  Per lane: one row, CH x PV columns.
    auto write = [&](char *g, uint32_t sb, auto probe) {
        for (uint32_t task = warp; task < ntask; task += nw) {
            probe();
            uint32_t ch, rb;
            fdivmod32(task, divrb, ch, rb);
            const uint32_t i = rb * 32 + lane;
            if (i >= rows) continue;
            const uintptr_t a = (uintptr_t)(g + ((uint64_t)(r0 + i) * p.n + c0) * EB);
            const uint32_t sh = (uint32_t)(a & 15) / EB;
            const uint32_t srow = sb + i * Q * 16;
            const uint32_t cfirst = ch * CH * PV;
            char *out = g + ((uint64_t)(c0 + cfirst) * p.m + r0 + i) * EB;
            // the phase o is the row's (c is a multiple of PV): consecutive column blocks
            // share a vector -- carried instead of loaded twice
            const uint32_t o = sh % PV, v0 = (sh + cfirst) / PV;
            uint4 cur = lds128(srow + v0 * 16);
#pragma unroll 2
            for (uint32_t cbl = 0; cbl < CH; ++cbl) {
                const uint32_t c = cfirst + cbl * PV;
                if (c >= L) break;
                const uint4 nxt = lds128(srow + (v0 + cbl + 1) * 16);
                E x[2 * PV];
                {
                    E ex[PV], ey[PV];
                    unpack<EB>(cur, ex);
                    unpack<EB>(nxt, ey);
                    cur = nxt;
#pragma unroll
                    for (uint32_t k = 0; k < PV; ++k) { x[k] = ex[k]; x[PV + k] = ey[k]; }
                }
#pragma unroll
                for (uint32_t sft = 1; sft < PV; sft <<= 1) {   // x[k] <- x[k + o]
                    const bool f = (o & sft) != 0;
#pragma unroll
                    for (uint32_t k = 0; k + sft < 2 * PV; ++k) x[k] = f ? x[k + sft] : x[k];
                }
                char *oc = out + (uint64_t)cbl * PV * mEB;
#pragma unroll
                for (uint32_t k = 0; k < PV; ++k)
                    if (c + k < L) *reinterpret_cast<E *>(oc + k * mEB) = x[k];
            }
        }
    };
    group_loop(p, s0, mbar, load, write);
}

// ------------------------------------------------------------------- generic kernel
// Any element size and any m x n that fits (Fig. 1 for a CUDA block).  The tile is
// contiguous, so when it is 16-byte aligned it is loaded with 16-byte vectors; elements
// land in an odd-pitch shared array (conflict-free transposed reads) and are written
// back with coalesced element stores (an output row of m elements is rarely 16-byte
// aligned).  All index maps use 32-bit multiply-high division.
template <typename T>
__global__ void __launch_bounds__(512) tile_onchip_generic(const TileParams p) {
    constexpr int PV = 16 / sizeof(T) > 0 ? 16 / sizeof(T) : 1;   // elements per 16 B
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T *s = reinterpret_cast<T *>(smem_raw);
    const uint32_t mn = p.m * p.n;
    for (uint64_t t = blockIdx.x; t < p.count; t += gridDim.x) {
        T *g = reinterpret_cast<T *>(tile_ptr(p, t));
        if (p.vec16) {
            const uint32_t nvec = mn / PV;
            for (uint32_t e = threadIdx.x; e < nvec; e += blockDim.x) {
                union { uint4 v; T x[PV]; } u;
                u.v = ld_cg<16>(reinterpret_cast<const char *>(g) + (size_t)e * 16);
                uint32_t i, j;
                fdivmod32(e * PV, p.divN32, i, j);
#pragma unroll
                for (int k = 0; k < PV; ++k) {
                    s[i * p.pitch + j] = u.x[k];
                    if (++j == p.n) { j = 0; ++i; }
                }
            }
        } else {
            load_slice_scalar<T>(s, g, mn, p.pitch, p.divN32);
        }
        __syncthreads();
        for (uint32_t o = threadIdx.x; o < mn; o += blockDim.x) {
            uint32_t r, c;
            fdivmod32(o, p.divM32, r, c);   // output row r < n, column c < m
            g[o] = s[c * p.pitch + r];
        }
        __syncthreads();
    }
}

// ------------------------------------------------------ cluster-split generic kernel
// Element path for tiles larger than one CTA (e.g. m = 9998 = 2 x 4999 rows): CTA k of a
// K-CTA cluster holds rows [k*m/K, (k+1)*m/K) (uneven slices allowed) and writes the
// matching column segment of every output row with coalesced element stores.  One
// cluster barrier per tile separates all loads of the tile from all stores into it.

template <typename T>
__global__ void __launch_bounds__(512, 1) tile_generic_cluster(const TileParams p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T *s = reinterpret_cast<T *>(smem_raw);
    const uint32_t K = p.K;
    const uint32_t rank = cluster_rank();
    const uint32_t cid = blockIdx.x / K, ncl = gridDim.x / K;
    if (!p.colsplit) {
        // row split: CTA k holds rows [r0, r1); writes that column segment of every output
        // row.  Slice boundaries are rounded to RA rows so that every slice starts on a
        // 16-byte boundary (16-byte slice loads), and -- when output rows are 16-byte
        // multiples -- the column segments are written with 16-byte stores.
        constexpr uint32_t PV = 16 / sizeof(T) > 0 ? 16 / sizeof(T) : 1;
        const uint32_t ra = p.ralign ? p.ralign : 1;
        const uint32_t units = p.m / ra;
        const uint32_t r0 = (uint32_t)((uint64_t)rank * units / K) * ra;
        const uint32_t r1 = (rank + 1 == K) ? p.m : (uint32_t)((uint64_t)(rank + 1) * units / K) * ra;
        const uint32_t rows = r1 - r0;
        const uint32_t cnt = rows * p.n;
        const FastDiv32 divRows = make_fastdiv32_dev(rows);
        const bool vec = p.vec16 && (((uint64_t)r0 * p.n * sizeof(T)) % 16 == 0) &&
                         (((uint64_t)cnt * sizeof(T)) % 16 == 0);
        const bool vecst = p.vec16 && PV > 1 && ((uint64_t)p.m * sizeof(T)) % 16 == 0 &&
                           ((uint64_t)r0 * sizeof(T)) % 16 == 0 && rows % PV == 0;
        const uint32_t rowsv = rows / PV;
        const FastDiv32 divRowsV = make_fastdiv32_dev(rowsv ? rowsv : 1);
        for (uint64_t t = cid; t < p.count; t += ncl) {
            T *g = reinterpret_cast<T *>(tile_ptr(p, t));
            const T *src = g + (size_t)r0 * p.n;
            if (vec)
                load_slice_vec<T>(s, src, cnt, p.pitch, p.n, p.divN32);
            else
                load_slice_scalar<T>(s, src, cnt, p.pitch, p.divN32);
            cluster_sync_all();     // all slices loaded before any store into the tile
            if (vecst) {
                const uint32_t cntv = rowsv * p.n;
                for (uint32_t o = threadIdx.x; o < cntv; o += blockDim.x) {
                    uint32_t r, clv;
                    fdivmod32(o, divRowsV, r, clv);   // output row r, columns r0 + PV*clv ..
                    union { uint4 w; T x[PV]; } u;
#pragma unroll
                    for (uint32_t k = 0; k < PV; ++k) u.x[k] = s[(clv * PV + k) * p.pitch + r];
                    stg128_na(g + (size_t)r * p.m + r0 + clv * PV, u.w);
                }
            } else {
                for (uint32_t o = threadIdx.x; o < cnt; o += blockDim.x) {
                    uint32_t r, cl;
                    fdivmod32(o, divRows, r, cl);   // output row r < n, column r0 + cl
                    g[(size_t)r * p.m + r0 + cl] = s[cl * p.pitch + r];
                }
            }
            __syncthreads();
        }
    } else {
        // column split (few, long rows): CTA k holds columns [c0, c1) of every row and
        // writes output rows [c0, c1) -- one contiguous range
        const uint32_t c0 = (uint32_t)((uint64_t)rank * p.n / K);
        const uint32_t c1 = (uint32_t)((uint64_t)(rank + 1) * p.n / K);
        const uint32_t cols = c1 - c0;
        const uint32_t P = cols | 1u;
        const uint32_t cnt = p.m * cols;
        const FastDiv32 divCols = make_fastdiv32_dev(cols);
        for (uint64_t t = cid; t < p.count; t += ncl) {
            T *g = reinterpret_cast<T *>(tile_ptr(p, t));
            constexpr int U = 8;
            for (uint32_t e0 = threadIdx.x; e0 < cnt; e0 += U * blockDim.x) {
                T v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const uint32_t e = e0 + u * blockDim.x;
                    if (e < cnt) {
                        uint32_t i, jl;
                        fdivmod32(e, divCols, i, jl);
                        v[u] = g[(size_t)i * p.n + c0 + jl];
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const uint32_t e = e0 + u * blockDim.x;
                    if (e < cnt) {
                        uint32_t i, jl;
                        fdivmod32(e, divCols, i, jl);
                        s[i * P + jl] = v[u];
                    }
                }
            }
            cluster_sync_all();
            T *dst = g + (size_t)c0 * p.m;
            for (uint32_t o = threadIdx.x; o < cnt; o += blockDim.x) {
                uint32_t rl, c;
                fdivmod32(o, p.divM32, rl, c);   // output row c0 + rl, column c
                dst[o] = s[c * P + rl];
            }
            __syncthreads();
        }
    }
}

// ------------------------------------------------------------------------ host side
namespace {

int tile_threads(uint64_t tile_bytes) {
    // small tiles: 256 threads (fewer idle threads in the write-out), else 512
    long t = env_int("IPT_TILE_THREADS", tile_bytes < 48 * 1024 ? 256 : 512);
    return (t == 256 || t == 512) ? (int)t : 512;
}

bool vec_ok(int64_t A, int64_t B, int eb) {
    if (eb != 4 && eb != 8 && eb != 16) return false;
    const int V = 16 / eb;
    if (A % V || B % V) return false;
    return !env_int("IPT_TILE_GENERIC", 0);
}

bool fast_ok(const StageDesc &d) {
    if (!vec_ok(d.A, d.B, d.eb)) return false;
    if (((uintptr_t)d.base & 15) != 0) return false;
    if (d.outer > 1 && (d.ostride & 15) != 0) return false;
    return true;
}

uint32_t fast_q(int64_t B, int eb) {
    uint32_t q = (uint32_t)(B * eb / 16);
    return (q & 1) ? q : q + 1;
}

size_t fast_smem(int64_t A, int64_t B, int eb) {
    return (size_t)A * fast_q(B, eb) * 16;
}

uint32_t generic_pitch(int64_t B) {
    uint32_t P = (uint32_t)B;
    return (P & 1) ? P : P + 1;
}

size_t generic_smem(int64_t A, int64_t B, int eb) { return (size_t)A * generic_pitch(B) * eb; }

template <typename K>
int occupancy(K kern, int threads, size_t smem, int device) {
    static std::mutex mu;
    static std::map<std::pair<const void *, std::pair<int, std::pair<int, size_t>>>, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_pair((const void *)kern, std::make_pair(device, std::make_pair(threads, smem)));
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    int n = 0;
    // one attribute value per kernel: the device maximum (a lower value set for one
    // shape would make a later, larger launch fail)
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         dev_props(device).smem_optin);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, threads, smem) != cudaSuccess) n = 1;
    if (n < 1) n = 1;
    cache[key] = n;
    return n;
}

template <typename K>
cudaError_t go(K kern, const TileParams &p, size_t smem, cudaStream_t st, int device) {
    DevProps dp = dev_props(device);
    const int threads = tile_threads(p.tile_bytes);
    int per_sm = occupancy(kern, threads, smem, device);
    uint64_t grid = (uint64_t)dp.sms * per_sm;
    if (p.count < grid) grid = p.count;
    if (grid < 1) grid = 1;
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile m=%u n=%u smem=%zu threads=%d per_sm=%d grid=%llu tiles=%llu\n",
                p.m, p.n, smem, threads, per_sm, (unsigned long long)grid,
                (unsigned long long)p.count);
    kern<<<(unsigned)grid, threads, smem, st>>>(p);
    note_launch();
    return cudaGetLastError();
}

template <typename K_>
cudaError_t go_cluster(K_ kern, const TileParams &p, size_t smem, int K, cudaStream_t st,
                       int device) {
    DevProps dp = dev_props(device);
    const int threads = tile_threads(smem);
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, dp.smem_optin);
    cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(threads, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = K;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int per_sm = occupancy(kern, threads, smem, device);
    uint64_t clusters = (uint64_t)dp.sms * per_sm / K;
    cfg.gridDim = dim3((unsigned)(clusters * K), 1, 1);
    int maxc = 0;   // co-resident clusters (cluster placement may strand SMs)
    if (cudaOccupancyMaxActiveClusters(&maxc, kern, &cfg) == cudaSuccess && maxc > 0) {
        if ((uint64_t)maxc < clusters && (uint64_t)maxc * 2 >= clusters) clusters = (uint64_t)maxc;
    } else {
        cudaGetLastError();
    }
    if (p.count < clusters) clusters = p.count;
    if (clusters < 1) clusters = 1;
    cfg.gridDim = dim3((unsigned)(clusters * K), 1, 1);
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile_cluster m=%u n=%u K=%d colsplit=%d smem=%zu threads=%d per_sm=%d maxc=%d clusters=%llu tiles=%llu\n",
                p.m, p.n, K, p.colsplit, smem, threads, per_sm, maxc, (unsigned long long)clusters, (unsigned long long)p.count);
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, p);
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

// Fast-path cluster/group split: column split when the tile has fewer rows than columns
// (each CTA then writes whole contiguous output rows), else row split.
static bool fast_colsplit(int64_t A, int64_t B, int eb) {
    // row-split write segments are ~A*eb/K bytes: only short rows (< 1 KB) favour columns
    return A < B && A * eb < 1024 && env_int("IPT_TILE_FAST_COLSPLIT", 1);
}

// Slice geometry of tile_group_tma: the vectors a slice row needs are fetched as npan
// column panels of q vectors (odd, q*V <= 256 elements per box row), each as boxes of br
// rows (br divides the fetched rows).  ok = false when the TMA path does not apply.
struct TmaGeom {
    bool ok = false;
    uint32_t q = 0, npan = 0, rows = 0, br = 0;
    size_t pstride = 0, bytes = 0;   // panel stride (128-byte aligned), slice bytes
};

static TmaGeom tma_geom(int64_t A, int64_t B, int eb, int K, bool cs) {
    TmaGeom t;
    if ((eb != 4 && eb != 8) || !env_int("IPT_TILE_GROUP_TMA", 1)) return t;
    const int V = 16 / eb;
    const int64_t mv = A / V, nvr = B / V;
    const uint32_t need = (uint32_t)(cs ? (nvr + K - 1) / K : nvr);
    t.rows = (uint32_t)(cs ? A : ((mv + K - 1) / K) * V);
    const uint32_t maxw = 256 / V - 1;
    t.npan = (need + maxw - 1) / maxw;
    t.q = ((need + t.npan - 1) / t.npan) | 1u;
    // box destinations must be 128-byte aligned: several boxes per panel need br % 8 == 0
    for (uint32_t b = std::min<uint32_t>(t.rows, 256); b >= 1; --b)
        if (t.rows % b == 0 && (b == t.rows || b % 8 == 0)) { t.br = b; break; }
    if (t.br == 0 || (t.br < 16 && t.br != t.rows)) return t;
    t.pstride = (((size_t)t.rows * t.q * 16) + 127) & ~(size_t)127;
    t.bytes = (size_t)t.npan * t.pstride;
    t.ok = true;
    return t;
}


// Group split (tile_group_db / tile_group_generic): K CTAs per tile, `groups` tiles in
// flight, nbuf slice buffers per CTA.  K minimises waves x (slice + 4 KB barrier
// allowance); a larger K must win by 3 % (fewer CTAs per barrier, longer pieces).
// Split direction (measured, tools/tile_big.py): a row split reads contiguous slices and
// writes A*eb/K-byte pieces of every output row; it is preferred while those pieces are
// >= 64 B (e.g. 720 x 720: 5.2 vs 4.4 TB/s, 600 x 1200: 4.9 vs 4.7), else the column
// split (contiguous writes; 120 x 7200: 4.9 vs 3.3).
constexpr long kGroupStaticSmem = 256;   // mbarriers

struct GroupCfg {
    int K = 0, groups = 0, nbuf = 0;
    int gcols = 0;          // element path: > 1 = 2-D slice grid (K / gcols bands x gcols pieces)
    size_t slice = 0;
    bool colsplit = false;
};

// Slice buffers per CTA (2; 3 or 4 measured 10-40 % slower: smaller slices, larger K).
static int group_nbuf() {
    const long b = env_int("IPT_TILE_GROUP_NBUF", 2);
    return b < 2 ? 2 : (b > (long)kGroupMaxBuf ? (int)kGroupMaxBuf : (int)b);
}

// Best K for one split direction; `generic`: element-path slices of row pieces with one
// padding vector (the aligner may read one vector past the last row).
static GroupCfg group_search_nb(int64_t A, int64_t B, int eb, uint64_t count, int device, bool cs,
                                bool generic, int nb);

// Double-buffered slices when they fit; otherwise ONE buffer per CTA (no overlap of a
// tile's write-out with the next tile's fetch, but twice the on-chip capacity: tiles of up
// to ~33 MB over all 148 SMs -- e.g. a whole 1009 x 7001 float32 matrix in one pass).
static GroupCfg group_search(int64_t A, int64_t B, int eb, uint64_t count, int device, bool cs,
                             bool generic) {
    GroupCfg g = group_search_nb(A, B, eb, count, device, cs, generic, group_nbuf());
    if (!g.K && env_int("IPT_TILE_GROUP_SINGLE", 1))
        g = group_search_nb(A, B, eb, count, device, cs, generic, 1);
    return g;
}

static GroupCfg group_search_nb(int64_t A, int64_t B, int eb, uint64_t count, int device, bool cs,
                                bool generic, int nb) {
    GroupCfg g;
    const DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    const int V = 16 / eb;
    const int kfix = (int)env_int("IPT_TILE_GROUP_K", 0);
    const uint64_t cnt = std::max<uint64_t>(count, 1);
    g.nbuf = nb;
    g.colsplit = cs;
    double best = 1e300;
    for (int K = 2; K <= dp.sms; ++K) {
        if (kfix && K != kfix) continue;
        size_t slice;
        if (generic) {
            if ((cs ? B : A) < (int64_t)K * (cs ? V : 1)) break;
            const int64_t L = cs ? (B + K - 1) / K : B;
            const int64_t rows = cs ? A : (A + K - 1) / K;
            slice = (size_t)(rows * (((L + 2 * V - 2) / V) | 1) + 1) * 16;
        } else {
            const int64_t mv = A / V, nvr = B / V;
            if ((cs ? nvr : mv) < K) break;
            slice = cs ? (size_t)A * (size_t)(((nvr + K - 1) / K) | 1) * 16
                       : (size_t)((mv + K - 1) / K) * V * fast_q(B, eb) * 16;
        }
        if (!generic) {   // room for the TMA panel layout when that path applies
            const TmaGeom t = tma_geom(A, B, eb, K, cs);
            if (t.ok) slice = std::max(slice, t.bytes);
        } else {
            if (!cs && (B * eb) % 16 == 0 && env_int("IPT_TILE_GEN_TMAA", 1)) {   // tile_group_tma_elem
                const TmaGeom te = tma_geom((A + V - 1) / V * V, B, eb, K, false);
                if (te.ok) slice = std::max(slice, te.bytes);
            }
        }
        slice = (slice + 127) & ~(size_t)127;
        if ((long)(nb * slice) + kGroupStaticSmem > budget) continue;
        const int64_t groups = std::min<int64_t>(dp.sms / K, (int64_t)cnt);
        const double waves = (double)((cnt + groups - 1) / groups);
        const double cost = waves * ((double)slice + 4096.0);
        if (cost < best * 0.97) {
            best = cost;
            g.K = K;
            g.groups = (int)groups;
            g.slice = slice;
        }
    }
    return g;
}

static GroupCfg group_choose_uncached(int64_t A, int64_t B, int eb, uint64_t count, int device, bool generic);

// Group configurations are searched over every K (and both split directions): cached per
// (shape, count, device, IPT_* knobs) so that a launch or a plan evaluation costs a lookup.
static GroupCfg group_choose(int64_t A, int64_t B, int eb, uint64_t count, int device, bool generic) {
    static std::mutex mu;
    static std::map<std::tuple<int64_t, int64_t, int, uint64_t, int, bool, uint64_t>, GroupCfg> cache;
    const auto key = std::make_tuple(A, B, eb, count, device, generic, env_hash());
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
    }
    const GroupCfg g = group_choose_uncached(A, B, eb, count, device, generic);
    std::lock_guard<std::mutex> lk(mu);
    cache[key] = g;
    return g;
}

// Element path: estimated time of a group configuration, in slice bytes.  Waves x (slice
// + 4 KB barrier allowance) x a piece factor: every slice is written as pieces of output
// rows and read as pieces of input rows, and each piece costs ~48 bytes of partial 32-byte
// sectors at its two ends (fit on 21 stage-2 tiles of the sweep, tools/group_tile_time.py:
// e.g. 1181 x 1453: column split, 67-byte input pieces 2.44 TB/s -> 4 x 18 grid 4.39);
// a single slice buffer (no overlap of write-out and fetch) x 1.25.
static double group_est(const GroupCfg &g, int64_t A, int64_t B, int eb, uint64_t count) {
    if (!g.K) return 1e300;
    double out_b, in_b;
    if (g.gcols > 1) {
        const int64_t gr = g.K / g.gcols;
        out_b = (double)((A + gr - 1) / gr * eb);
        in_b = (double)((B + g.gcols - 1) / g.gcols * eb);
    } else if (g.colsplit) {
        out_b = (double)(A * eb);
        in_b = (double)((B + g.K - 1) / g.K * eb);
    } else {
        out_b = (double)((A + g.K - 1) / g.K * eb);
        in_b = (double)(B * eb);
    }
    auto f = [](double pb) { return (pb + 48.0) / pb; };
    const uint64_t cnt = std::max<uint64_t>(count, 1);
    const double waves = (double)((cnt + g.groups - 1) / g.groups);
    return waves * ((double)g.slice + 4096.0) * (0.5 * f(out_b) + 0.5 * f(in_b)) * (g.nbuf == 1 ? 1.25 : 1.0);
}

// Element path, 2-D slice grid: K = gr x gc CTAs, CTA (band, piece) holds rows
// [band * A / gr, ..) x columns [piece * B / gc, ..).  For tiles where neither 1-D split
// gives long pieces on both sides: a row split of a 1279 x 6353 float32 tile writes
// 34-byte pieces of every output row and its column split does not fit; 4 x 37 writes
// 1280-byte pieces and reads 172-byte ones (2.86 -> 4.15 TB/s).  Smallest group_est.
static GroupCfg group_search_2d(int64_t A, int64_t B, int eb, uint64_t count, int device, int nb) {
    GroupCfg g;
    const DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    const int V = 16 / eb;
    const uint64_t cnt = std::max<uint64_t>(count, 1);
    const int64_t fgr = env_int("IPT_TILE_GROUP_GR", 0);
    double best = 1e300;
    for (int64_t gr = 2; gr <= dp.sms / 2; ++gr) {
        if (fgr && gr != fgr) continue;
        if (A < gr) break;
        for (int64_t gc = 2; gr * gc <= dp.sms; ++gc) {
            if (B < gc) break;
            const int64_t rows = (A + gr - 1) / gr, L = (B + gc - 1) / gc;
            size_t slice = (size_t)(rows * (((L + 2 * V - 2) / V) | 1) + 1) * 16;
            slice = (slice + 127) & ~(size_t)127;
            if ((long)(nb * slice) + kGroupStaticSmem > budget) continue;
            GroupCfg c;
            c.K = (int)(gr * gc);
            c.gcols = (int)gc;
            c.groups = (int)std::min<int64_t>(dp.sms / c.K, (int64_t)cnt);
            c.slice = slice;
            c.nbuf = nb;
            const double e = group_est(c, A, B, eb, count);
            if (e < best * 0.99) {
                best = e;
                g = c;
            }
        }
    }
    return g;
}

static GroupCfg group_choose_uncached(int64_t A, int64_t B, int eb, uint64_t count, int device, bool generic) {
    const long f = env_int("IPT_TILE_GROUP_COLSPLIT", -1);
    if (f >= 0 && f != 2) return group_search(A, B, eb, count, device, f != 0, generic);
    const bool grid2d = generic && env_int("IPT_TILE_GROUP_2D", 1);
    auto search2d = [&]() {
        GroupCfg g = group_search_2d(A, B, eb, count, device, group_nbuf());
        if (!g.K && env_int("IPT_TILE_GROUP_SINGLE", 1)) g = group_search_2d(A, B, eb, count, device, 1);
        return g;
    };
    if (f == 2 && grid2d) {   // tests: the 2-D grid whenever one fits
        const GroupCfg g = search2d();
        if (g.K) return g;
    }
    const GroupCfg row = group_search(A, B, eb, count, device, false, generic);
    if (!grid2d) {
        if (row.K && A * eb / row.K >= 64) return row;
        const GroupCfg col = group_search(A, B, eb, count, device, true, generic);
        return col.K ? col : row;
    }
    // element path: the row split, the column split and the best 2-D grid by group_est
    const GroupCfg col = group_search(A, B, eb, count, device, true, generic);
    const GroupCfg g2 = search2d();
    double er = group_est(row, A, B, eb, count);
    const double ec = group_est(col, A, B, eb, count), e2 = group_est(g2, A, B, eb, count);
    // a row split with 16-byte aligned input rows fetches its slices by TMA
    // (tile_group_tma_elem, ~15 % faster: 9998 x 256 4.38 vs 4.18 TB/s on the 2-D grid)
    const int V = 16 / eb;
    if (row.K && (B * eb) % 16 == 0 && env_int("IPT_TILE_GEN_TMAA", 1) &&
        tma_geom((A + V - 1) / V * V, B, eb, row.K, false).ok)
        er *= 0.85;
    if (e2 < er && e2 < ec) return g2;
    return ec < er ? col : row;
}

GroupCfg group_cfg(int64_t A, int64_t B, int eb, uint64_t count, int device) {
    if (!vec_ok(A, B, eb)) return GroupCfg{};
    return group_choose(A, B, eb, count, device, false);
}

GroupCfg group_cfg_generic(int64_t A, int64_t B, int eb, uint64_t count, int device) {
    if (eb != 4 && eb != 8) return GroupCfg{};
    return group_choose(A, B, eb, count, device, true);
}

// Tensor map + box geometry for tile_group_tma (IPT_TILE_GROUP_TMA, default on): 4- and 8-byte elements,
// tiles stacked contiguously, a uniform odd box width of at most 256 elements, and a box
// height dividing the fetched slice rows.  Returns false when the TMA path does not apply.
static PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void *f = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)f;
    });
    return fn;
}

template <int EB>
bool group_tma_setup(const StageDesc &d, TileParams &p, const GroupCfg &g, CUtensorMap *tm) {
    if (EB != 4 && EB != 8) return false;
    if (d.outer > 1 && d.ostride != d.inner * (int64_t)p.tile_bytes) return false;
    const TmaGeom t = tma_geom(d.A, d.B, EB, g.K, g.colsplit);
    if (!t.ok || t.bytes > g.slice) return false;
    auto enc = tensor_map_encoder();
    if (!enc) return false;
    const int V = 16 / EB;
    const uint64_t total_rows = (uint64_t)(d.outer * d.inner) * (uint64_t)d.A;
    cuuint64_t dims[2] = {(cuuint64_t)d.B, (cuuint64_t)total_rows};
    cuuint64_t strides[1] = {(cuuint64_t)(d.B * EB)};
    cuuint32_t box[2] = {t.q * V, t.br};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(tm, EB == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 2, d.base,
                     dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        if (env_int("IPT_DEBUG", 0)) fprintf(stderr, "[ipt] tensor map encode failed (%d)\n", (int)r);
        return false;
    }
    p.q = t.q;
    p.box_rows = t.br;
    p.npan = t.npan;
    p.pstride = (uint32_t)t.pstride;
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile_group_tma q=%u npan=%u rows=%u box=%ux%u\n", t.q, t.npan, t.rows, t.q * V, t.br);
    return true;
}

// Tensor map + geometry for tile_group_tma_elem: as group_tma_setup, rows counted in
// ceil(m / V) blocks (the last one partial), row split only, 16-byte aligned input rows.
template <int EB>
bool group_tma_setup_elem(const StageDesc &d, TileParams &p, const GroupCfg &g, CUtensorMap *tm,
                          size_t *slice, int device) {
    if (EB != 4 && EB != 8) return false;
    const int V = 16 / EB;
    if (g.colsplit || (d.B * EB) % 16 || ((uintptr_t)d.base & 15)) return false;
    if (d.outer > 1 && d.ostride != d.inner * (int64_t)p.tile_bytes) return false;
    if (!env_int("IPT_TILE_GEN_TMAA", 1)) return false;
    const int64_t Ac = (d.A + V - 1) / V * V;                  // rows in whole V-blocks
    const TmaGeom t = tma_geom(Ac, d.B, EB, g.K, false);
    if (!t.ok) return false;
    // the boxes cover whole V-blocks and 128-byte aligned panels: the slice buffers may
    // grow a little beyond the element layout's, within the opt-in shared memory
    if (t.bytes > g.slice && (size_t)g.nbuf * t.bytes + 4096 > (size_t)dev_props(device).smem_optin) return false;
    auto enc = tensor_map_encoder();
    if (!enc) return false;
    const uint64_t total_rows = (uint64_t)(d.outer * d.inner) * (uint64_t)d.A;
    cuuint64_t dims[2] = {(cuuint64_t)d.B, (cuuint64_t)total_rows};
    cuuint64_t strides[1] = {(cuuint64_t)(d.B * EB)};
    cuuint32_t box[2] = {t.q * (uint32_t)V, t.br};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(tm, EB == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 2, d.base,
                     dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { cudaGetLastError(); return false; }
    p.q = t.q;
    p.box_rows = t.br;
    p.npan = t.npan;
    p.pstride = (uint32_t)t.pstride;
    if (t.bytes > *slice) *slice = t.bytes;
    p.buf_bytes = (uint32_t)*slice;
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile_group_tma_elem q=%u npan=%u rows=%u box=%ux%u slice=%zu\n", t.q, t.npan,
                t.rows, t.q * V, t.br, *slice);
    return true;
}


// Library-owned group counters per (device, stream): arrivals (kTileWsBytes) then per-group
// exit counters (kTileWsBytes), zeroed once ON that stream, re-zeroed by each launch's last
// CTA of every group.  Never used by captured launches (create == false -> the call's
// workspace with a memset node): a graph may be replayed on another stream concurrently
// with direct calls on the capture stream.
static uint32_t *group_counters(int device, cudaStream_t st, bool create) {
    static std::mutex mu;
    static std::map<std::pair<int, cudaStream_t>, uint32_t *> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_pair(device, st);
    auto it = cache.find(key);
    if (it != cache.end()) return it->second;
    if (!create) return nullptr;
    void *p = nullptr;
    if (cudaMalloc(&p, 2 * kTileWsBytes) != cudaSuccess ||
        cudaMemsetAsync(p, 0, 2 * kTileWsBytes, st) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    cache[key] = (uint32_t *)p;
    return (uint32_t *)p;
}

// Group-split launch: groups x K CTAs, all co-resident (cooperative launch); the arrival
// counters (kGroupCtrStride bytes apart) are library-owned and self-resetting, or the
// call's workspace zeroed on the stream first.
template <int EB, bool GENERIC>
cudaError_t launch_group_db(const StageDesc &d, TileParams p, const GroupCfg &g, void *ws,
                            cudaStream_t st, int device) {
    if (!ws || !g.K) return cudaErrorInvalidValue;
    if (GENERIC) {
        const int64_t L = g.gcols > 1 ? (d.B + g.gcols - 1) / g.gcols : g.colsplit ? (d.B + g.K - 1) / g.K : d.B;
        p.q = (uint32_t)(((L + 2 * (16 / EB) - 2) / (16 / EB)) | 1);
        p.gcols = (uint32_t)std::max(g.gcols, 0);
    } else {
        p.q = fast_q(d.B, d.eb);
    }
    p.colsplit = g.colsplit ? 1 : 0;
    p.K = (uint32_t)g.K;
    p.nbuf = (uint32_t)g.nbuf;
    p.buf_bytes = (uint32_t)g.slice;
    p.gbar = (uint32_t *)ws;
    if ((size_t)g.groups * g.nbuf * kGroupCtrStride > kTileWsBytes) return cudaErrorInvalidValue;
    // self-resetting counters owned by the library per (device, stream) when available
    p.gexit = nullptr;
    if (env_int("IPT_TILE_RESET", 1)) {
        cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
        if (cudaStreamIsCapturing(st, &cap) != cudaSuccess) { cudaGetLastError(); cap = cudaStreamCaptureStatusActive; }
        if (uint32_t *c = cap == cudaStreamCaptureStatusNone ? group_counters(device, st, true) : nullptr) {
            p.gbar = c;
            p.gexit = c + kTileWsBytes / 4;
        }
    }
    auto kern = GENERIC ? tile_group_generic<EB> : tile_group_db<EB>;
    CUtensorMap tmap;
    // element path with 16-byte aligned input rows: TMA slices + element write-out
    size_t slice = g.slice;
    const bool grid2d = g.gcols > 1;   // cp.async slices only
    const bool tma_elem = GENERIC && !grid2d && group_tma_setup_elem<EB>(d, p, g, &tmap, &slice, device);
    const bool tma = tma_elem || (!GENERIC && group_tma_setup<EB>(d, p, g, &tmap));
    cudaError_t e = cudaSuccess;
    if (!p.gexit) {
        e = cudaMemsetAsync(ws, 0, (size_t)g.groups * g.nbuf * kGroupCtrStride, st);
        if (e != cudaSuccess) return e;
    }
    auto set_smem = [&](const void *k) {   // dynamic + static shared memory within the opt-in maximum
        static std::mutex mu;
        static std::map<std::pair<const void *, int>, bool> done;
        std::lock_guard<std::mutex> lk(mu);
        if (!done[std::make_pair(k, device)]) {
            cudaFuncAttributes fa{};
            cudaFuncGetAttributes(&fa, k);
            cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 dev_props(device).smem_optin - (int)fa.sharedSizeBytes);
            done[std::make_pair(k, device)] = true;
        }
    };
    set_smem((const void *)kern);
    auto tkern = tma_elem ? tile_group_tma_elem<EB> : tile_group_tma<EB>;
    if (tma) set_smem((const void *)tkern);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(g.groups * g.K), 1, 1);
    cfg.blockDim = dim3(512, 1, 1);
    cfg.dynamicSmemBytes = g.nbuf * slice;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile_group%s m=%u n=%u K=%d groups=%d colsplit=%d gcols=%d nbuf=%d smem=%zu tiles=%llu\n",
                GENERIC ? "_generic" : "", p.m, p.n, g.K, g.groups, p.colsplit, g.gcols, g.nbuf, g.nbuf * g.slice,
                (unsigned long long)p.count);
    e = tma ? cudaLaunchKernelEx(&cfg, tkern, p, tmap) : cudaLaunchKernelEx(&cfg, kern, p);
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

// Whole-GPU tiles in shared memory + registers (tile_group_rf): K = every SM, one group.
struct RfCfg {
    int K = 0, rv = 0;
    bool colsplit = false;
    bool swz = false;      // column slices of one 128-byte line per row, TMA 128-byte swizzle
    uint32_t q = 0, npan = 0, rows_a = 0, rows_b = 0, cpan = 0, box_rows = 0, ralign = 0;
    size_t pstride = 0, smem = 0;
};
constexpr int kRfThreads = 512;
constexpr int kRfMaxRV = 32;   // part-B vectors per thread in TMEM (128 columns x 4 B)

// Configuration of tile_group_rf: the largest part A in shared memory (TMA boxes of <= 256
// rows, 128-byte aligned), part B in TMEM (at most 32 vectors per thread, every chunk
// padded to 512 vectors) staged through part A's region after its write-out, in row (or
// panel) chunks as large as shared memory allows.
static RfCfg rf_search(int64_t A, int64_t B, int eb, int device, bool cs, bool chunks, int64_t ral) {
    RfCfg c;
    const DevProps dp = dev_props(device);
    const int K = dp.sms, V = 16 / eb;
    const int64_t mv = A / V, nvr = B / V;
    const int64_t sv = cs ? nvr : mv;   // split dimension in V-blocks / vectors
    if (sv % ral || sv / ral < K) return c;
    // max slice (split in units of ral V-blocks / vectors; the last CTA takes the remainder)
    const int64_t smax = std::max((sv / ral + K - 1) / K * ral, sv - (sv / ral) * (K - 1) / K * ral);
    const int64_t rows = cs ? A : smax * V;
    const int64_t cvec = cs ? smax : nvr;                                // max slice vectors per row
    const uint32_t maxw = 256 / V - 1;
    const uint32_t npan = (uint32_t)((cvec + maxw - 1) / maxw);
    const uint32_t q = (uint32_t)(((cvec + npan - 1) / npan) | 1);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin) - 1024;
    const int64_t maxchunks = 32;
    auto pst = [&](int64_t r) { return (int64_t)((r * q * 16 + 127) & ~(int64_t)127); };
    for (int64_t ra = rows / V * V; ra >= V; ra -= V) {
        const int64_t abytes = npan * pst(ra);
        if (abytes > budget) continue;
        uint32_t br = 0;                                   // TMA box rows (128-B aligned boxes)
        if (ra <= 256) br = (uint32_t)ra;
        else
            for (uint32_t b = 256; b >= 16; b -= 8)
                if (ra % b == 0) { br = b; break; }
        if (!br) continue;
        const int64_t rb = rows - ra;
        if ((rb * cvec + kRfThreads - 1) / kRfThreads > kRfMaxRV) return c;   // smaller A only adds TMEM
        const int64_t room = budget;
        const int64_t maxvec = INT64_MAX;   // vectors per chunk
        int64_t cb = 0, cp = 0;
        if (rb > 0 && !chunks) {   // part B staged at once (one chunk)
            if (npan * pst(rb) > room) continue;
            cb = rb;
            cp = npan;
        } else if (rb > 0) {
            if (npan * pst(V) <= room && npan * V * cvec <= maxvec) {   // chunks of whole rows
                cp = npan;
                cb = V;
                while (cb + V <= rb && npan * pst(cb + V) <= room && (cb + V) * cvec <= maxvec) cb += V;
            } else if (pst(rb) <= room) {                                 // chunks of whole panels
                cb = rb;
                cp = std::max<int64_t>(1, std::min<int64_t>(room / pst(rb), maxvec / (rb * q)));
                if (rb * q > maxvec) continue;
            } else {
                continue;
            }
            const int64_t cw = cp * q;
            const int64_t nch = ((rb + cb - 1) / cb) * ((cvec + cw - 1) / cw);
            if (nch > maxchunks) continue;
            int64_t cols = 0;   // TMEM columns: every chunk padded to a multiple of 512 vectors
            for (int64_t r = 0; r < rb; r += cb)
                for (int64_t cc = 0; cc < cvec; cc += cw)
                    cols += (std::min(cb, rb - r) * std::min(cw, cvec - cc) + kRfThreads - 1) / kRfThreads;
            if (cols > kRfMaxRV) continue;
        }
        c.K = K;
        c.colsplit = cs;
        c.ralign = (uint32_t)ral;
        c.q = q;
        c.npan = npan;
        c.rows_a = (uint32_t)ra;
        c.rows_b = (uint32_t)std::max<int64_t>(cb, V);
        c.cpan = (uint32_t)std::max<int64_t>(cp, 1);
        c.box_rows = br;
        c.rv = (int)((rb * cvec + kRfThreads - 1) / kRfThreads);
        c.pstride = (size_t)pst(ra);
        c.smem = (size_t)std::max<int64_t>(abytes, rb > 0 ? std::min<int64_t>(cp, npan) * pst(cb) : 0);
        return c;
    }
    return c;
}

// Column slices of exactly one 128-byte line per row (8 vectors): K = B*eb/128 CTAs, which
// must be at least 3/4 of the SMs (the rest idle).  Part A lands by TMA in the 128-byte
// swizzle (conflict-free write-out reads at pitch 128 B), part B is restaged through the
// same region in one chunk.  Every CTA's pieces of the input rows are whole lines -- no
// sector is shared between two CTAs.
static RfCfg rf_search_swz(int64_t A, int64_t B, int eb, int device) {
    RfCfg c;
    const DevProps dp = dev_props(device);
    const int V = 16 / eb;
    const int64_t nvr = B / V;
    if (nvr % 8) return c;
    const int64_t K = nvr / 8;
    if (K > dp.sms || 4 * K < 3 * (int64_t)dp.sms) return c;
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin) - 2048;   // + 1 KB alignment slack
    for (int64_t ra = std::min<int64_t>(A, budget / 128) / 8 * 8; ra >= 8; ra -= 8) {
        uint32_t br = 0;
        for (uint32_t b = 256; b >= 8; b -= 8)
            if (ra % b == 0) { br = b; break; }
        if (!br) continue;
        const int64_t rb = A - ra;
        if (rb * 8 > (int64_t)kRfThreads * kRfMaxRV || rb * 128 > budget) return c;   // smaller A: more B
        c.K = (int)K;
        c.colsplit = true;
        c.swz = true;
        c.ralign = 8;
        c.q = 8;
        c.npan = 1;
        c.rows_a = (uint32_t)ra;
        c.rows_b = (uint32_t)std::max<int64_t>(rb, V);
        c.cpan = 1;
        c.box_rows = br;
        c.rv = (int)((rb * 8 + kRfThreads - 1) / kRfThreads);
        c.pstride = (size_t)ra * 128;
        c.smem = 1024 + (size_t)std::max(ra, rb) * 128;
        return c;
    }
    return c;
}

static RfCfg rf_cfg(int64_t A, int64_t B, int eb, int device) {
    if ((eb != 4 && eb != 8) || !vec_ok(A, B, eb) || !env_int("IPT_TILE_RF", 1)) return RfCfg{};
    static std::mutex mu;
    static std::map<std::tuple<int64_t, int64_t, int, int, uint64_t>, RfCfg> cache;
    const auto key = std::make_tuple(A, B, eb, device, env_hash());
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
    }
    const int K = dev_props(device).sms;
    // split the longer side (tools/rf_sweep.py per orientation, column vs row split:
    // 3000 x 4096 4.19 vs 3.99 TB/s, 3200 x 4000 3.33 vs 3.00, 4096 x 3000 3.67 vs 4.85),
    // and rows only while the row-split pieces are >= 64 B
    const bool row_first = A >= B && A * eb / K >= 64;
    // the natural split direction first, unchunked configurations before chunked ones
    // (2500 x 5100: column split in one chunk 3.4 TB/s vs row split in chunks 2.8)
    // Row slices start on 32-byte boundaries of the output rows when that fits
    // (IPT_TILE_RF_RALIGN, bytes; 0 = any 16-byte V-block boundary): every CTA writes a piece
    // of every output row, and pieces starting mid-sector made some CTAs' write-out ~40 %
    // slower (tools/rf_trace.py: exactly the CTAs whose pieces start 16 bytes before a line
    // boundary), holding up the next tile's group barrier.  C5: 4.40 -> 4.63 TB/s (64 B:
    // 4.50, 128 B: 4.40 -- coarser units unbalance the slices).
    const int64_t rab = env_int("IPT_TILE_RF_RALIGN", 32);
    const int64_t ral = rab > 16 ? rab / 16 : 1;   // V-blocks are 16 bytes of an output row
    RfCfg c;
    const long fcs = env_int("IPT_TILE_RF_CS", -1);   // measurement: force the split direction
    if (!row_first && fcs != 0 && env_int("IPT_TILE_RF_SWZ", 1)) c = rf_search_swz(A, B, eb, device);
    for (int pass = 0; pass < 4 && !c.K; ++pass) {
        const bool cs = (pass & 1) ? row_first : !row_first;
        if (fcs >= 0 && cs != (fcs != 0)) continue;
        // column slices stay on 16-byte boundaries: 32-byte column units measured slower
        // (3000 x 4096: 3.97 vs 4.40 TB/s)
        if (!cs && ral > 1) c = rf_search(A, B, eb, device, cs, pass >= 2, ral);
        if (!c.K) c = rf_search(A, B, eb, device, cs, pass >= 2, 1);
    }
    std::lock_guard<std::mutex> lk(mu);
    cache[key] = c;
    return c;
}

template <int EB>
cudaError_t launch_group_rf(const StageDesc &d, TileParams p, const RfCfg &c, void *ws, cudaStream_t st,
                            int device) {
    if (!ws || !c.K) return cudaErrorInvalidValue;
    const bool packed = d.outer <= 1 || d.ostride == d.inner * (int64_t)p.tile_bytes;
    if (!packed && d.inner != 1) return cudaErrorNotSupported;
    auto enc = tensor_map_encoder();
    if (!enc) return cudaErrorNotSupported;
    const int V = 16 / EB;
    CUtensorMap tm;
    CUresult r;
    if (packed) {   // tiles stacked: (columns, rows of all tiles)
        const uint64_t total_rows = (uint64_t)(d.outer * d.inner) * (uint64_t)d.A;
        cuuint64_t dims[2] = {(cuuint64_t)d.B, (cuuint64_t)total_rows};
        cuuint64_t strides[1] = {(cuuint64_t)(d.B * EB)};
        cuuint32_t box[2] = {c.q * (uint32_t)V, c.box_rows};
        cuuint32_t estr[2] = {1, 1};
        r = enc(&tm, EB == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 2, d.base,
                dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                c.swz ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        p.rres = 0;
    } else {        // strided batch of single tiles: (columns, rows, tiles), tile stride ostride
        if (d.ostride % 16) return cudaErrorNotSupported;
        cuuint64_t dims[3] = {(cuuint64_t)d.B, (cuuint64_t)d.A, (cuuint64_t)d.outer};
        cuuint64_t strides[2] = {(cuuint64_t)(d.B * EB), (cuuint64_t)d.ostride};
        cuuint32_t box[3] = {c.q * (uint32_t)V, c.box_rows, 1};
        cuuint32_t estr[3] = {1, 1, 1};
        r = enc(&tm, EB == 4 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_INT64, 3, d.base,
                dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                c.swz ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        p.rres = 1;
    }
    if (r != CUDA_SUCCESS) return cudaErrorNotSupported;
    p.q = c.q;
    p.npan = c.npan;
    p.pstride = (uint32_t)c.pstride;
    p.box_rows = c.box_rows;
    p.rows_a = c.rows_a;
    p.rows_b = c.rows_b;
    p.cpan = c.cpan;
    p.ralign = c.ralign;
    p.colsplit = c.colsplit ? 1 : 0;
    p.K = (uint32_t)c.K;
    p.nbuf = 1;
    p.zero = 0;
    p.gbar = (uint32_t *)ws;
    p.gexit = nullptr;
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(st, &cap) != cudaSuccess) { cudaGetLastError(); cap = cudaStreamCaptureStatusActive; }
    if (env_int("IPT_TILE_RESET", 1) && cap == cudaStreamCaptureStatusNone) {
        if (uint32_t *ctr = group_counters(device, st, true)) {
            p.gbar = ctr;
            p.gexit = ctr + kTileWsBytes / 4;
        }
    }
    if (!p.gexit) {
        const cudaError_t e = cudaMemsetAsync(ws, 0, kGroupCtrStride, st);
        if (e != cudaSuccess) return e;
    }
    const void *kern = nullptr;
    const int rv = std::max(kRfBatch, (c.rv + kRfBatch - 1) / kRfBatch * kRfBatch);
    const int64_t ral = c.ralign ? c.ralign : 1, mvv = d.A / V;
    const int64_t rmax = c.colsplit ? d.A
        : std::max((mvv / ral + c.K - 1) / c.K * ral, mvv - (mvv / ral) * (c.K - 1) / c.K * ral) * V;
    const int64_t rbm = rmax - (int64_t)c.rows_a;   // max rows in TMEM
    const bool ch = rbm > (int64_t)c.rows_b || c.cpan < c.npan;
#define IPT_RF(R) if (!kern && rv == R) kern = c.swz ? (ch ? nullptr : (const void *)tile_group_rf<EB, R, false, true>) \
        : ch ? (const void *)tile_group_rf<EB, R, true> : (const void *)tile_group_rf<EB, R, false>;
    IPT_RF(8) IPT_RF(16) IPT_RF(24) IPT_RF(32)
#undef IPT_RF
    if (!kern) return cudaErrorNotSupported;
    {
        static std::mutex mu;
        static std::map<std::pair<const void *, int>, bool> done;
        std::lock_guard<std::mutex> lk(mu);
        if (!done[std::make_pair(kern, device)]) {
            cudaFuncAttributes fa{};
            cudaFuncGetAttributes(&fa, kern);
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 dev_props(device).smem_optin - (int)fa.sharedSizeBytes);
            done[std::make_pair(kern, device)] = true;
        }
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)c.K, 1, 1);
    cfg.blockDim = dim3(kRfThreads, 1, 1);
    cfg.dynamicSmemBytes = c.smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] tile_group_rf m=%u n=%u K=%d colsplit=%d q=%u npan=%u rows_a=%u chunk=%ux%u box=%u rv=%d smem=%zu tiles=%llu\n",
                p.m, p.n, c.K, p.colsplit, c.q, c.npan, c.rows_a, c.rows_b, c.cpan, c.box_rows, rv, c.smem,
                (unsigned long long)p.count);
    void *args[] = {&p, &tm};
    p.diag = (int)env_int("IPT_TILE_DIAG", 0);
    cudaError_t e = cudaLaunchKernelExC(&cfg, kern, args);
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace

// Cluster size for a tile that does not fit one CTA (0 = none): the smallest K in
// {2, 4, 8, 16} whose slice fits 113 KB (two CTAs per SM), else the smallest that fits.

int tile_cluster_k(int64_t A, int64_t B, int eb, int device) {
    if (!vec_ok(A, B, eb) || !env_int("IPT_TILE_CLUSTER", 1)) return 0;
    DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    const int V = 16 / eb;
    const bool cs = fast_colsplit(A, B, eb);
    int fit = 0;
    for (int K : {2, 4, 8, 16}) {
        size_t slice;
        if (cs) {
            const int64_t nvr = B / V;
            if (nvr < K) break;
            slice = (size_t)A * (size_t)(((nvr + K - 1) / K) | 1) * 16;
        } else {
            if (A / V < K) break;
            slice = (size_t)((A / V + K - 1) / K) * V * (size_t)fast_q(B, eb) * 16;
        }
        if (slice <= 113 * 1024) return K;
        if (!fit && (long)slice <= budget) fit = K;
    }
    return fit;
}

// Cluster size for the element path when the tile does not fit one CTA (0 = none).
// Row split by default (16-byte slice loads; measured faster even for 32 x 9998 tiles);
// IPT_TILE_COLSPLIT=1 selects the column split for tiles with more columns than rows.
static bool generic_colsplit(int64_t A, int64_t B) {
    return env_int("IPT_TILE_COLSPLIT", 0) && B > A;
}

// Row-slice alignment of the element-path cluster split: 16 / gcd(n * eb, 16) rows start
// every slice on a 16-byte boundary (1 when that does not divide the rows evenly).
static uint32_t generic_ralign(int64_t A, int64_t B, int eb, int K) {
    uint32_t x = 16, g = (uint32_t)((B * eb) & 15);
    if (g == 0) g = 16;
    while (g) { uint32_t t = x % g; x = g; g = t; }
    const uint32_t a = 16 / x;
    return (A % a == 0 && A / a >= K) ? a : 1;
}

static int64_t generic_slice_rows(int64_t A, int64_t B, int eb, int K) {
    const int64_t ra = generic_ralign(A, B, eb, K);
    return ((A / ra + K - 1) / K) * ra;
}

int tile_generic_cluster_k(int64_t A, int64_t B, int eb, int device) {
    if (!env_int("IPT_TILE_CLUSTER", 1) || A * B >= (1ll << 31)) return 0;
    DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    const bool cs = generic_colsplit(A, B);
    for (int K : {2, 4, 8, 16}) {
        size_t bytes;
        if (cs) {
            if (B < K) break;
            bytes = (size_t)A * (size_t)(((B + K - 1) / K) | 1) * eb;
        } else {
            if (A < K) break;
            bytes = (size_t)generic_slice_rows(A, B, eb, K) * generic_pitch(B) * eb;
        }
        if ((long)bytes <= budget) return K;
    }
    return 0;
}

// Group split instead of a cluster (measured, tools/tile_big.py): when no cluster fits, when
// the cluster's slices need one CTA per SM (streaming kernel), and for K >= 8 (clusters of
// 8 and 16 strand SMs: 14 co-resident 16-CTA clusters at two CTAs per SM, 7 at one).
// Clusters of 2 or 4 with two CTAs per SM are as fast or faster and need no workspace.
bool tile_group_split(int64_t A, int64_t B, int eb, int device) {
    if (!vec_ok(A, B, eb) || !env_int("IPT_TILE_GROUP_SPLIT", 1)) return false;
    const DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    if ((long)fast_smem(A, B, eb) <= budget) return false;
    const int K = tile_cluster_k(A, B, eb, device);
    if (K && K < 8) {
        const int V = 16 / eb;
        const size_t slice = fast_colsplit(A, B, eb)
            ? (size_t)A * (size_t)((((B / V) + K - 1) / K) | 1) * 16
            : (size_t)(((A / V) + K - 1) / K) * V * (size_t)fast_q(B, eb) * 16;
        if (slice <= 113 * 1024) return false;
    }
    return group_cfg(A, B, eb, (uint64_t)dp.sms, device).K != 0;
}

// Element path over a CTA group (4- and 8-byte elements) when the tile needs more than
// 113 KB of one CTA (measured faster than the single-CTA and cluster element kernels).
bool tile_group_generic_split(int64_t A, int64_t B, int eb, int device) {
    if ((eb != 4 && eb != 8) || !env_int("IPT_TILE_GROUP_GENERIC", 1)) return false;
    if ((size_t)generic_smem(A, B, eb) <= 113 * 1024) return false;
    return group_cfg_generic(A, B, eb, (uint64_t)dev_props(device).sms, device).K != 0;
}

int tile_group_k(int64_t A, int64_t B, int eb, uint64_t count, int device, int *groups, bool *tma,
                 int *nbuf) {
    const bool fast = vec_ok(A, B, eb);
    const GroupCfg g = fast ? group_cfg(A, B, eb, count, device)
                            : group_cfg_generic(A, B, eb, count, device);
    if (groups) *groups = g.groups;
    if (nbuf) *nbuf = g.nbuf;
    if (tma) *tma = fast && g.K && tma_geom(A, B, eb, g.K, g.colsplit).ok;
    return g.K;
}

int tile_onchip_path(int64_t A, int64_t B, int eb, int device) {
    DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    if (env_int("IPT_TILE_RF_FORCE", 0) && tile_rf_fits(A, B, eb, device)) return 7;   // tests
    if (vec_ok(A, B, eb) && (long)fast_smem(A, B, eb) <= budget) return 2;
    if (tile_group_split(A, B, eb, device)) return 5;
    if (tile_cluster_k(A, B, eb, device)) return 3;
    if (!vec_ok(A, B, eb) && tile_group_generic_split(A, B, eb, device)) return 6;
    if ((long)generic_smem(A, B, eb) > budget && tile_generic_cluster_k(A, B, eb, device)) return 4;
    if ((long)generic_smem(A, B, eb) <= budget && A * B < (1ll << 31)) return 1;
    if (tile_rf_fits(A, B, eb, device)) return 7;
    return 0;
}

// A tile held over every SM in shared memory + registers (tile_group_rf)?
bool tile_rf_fits(int64_t A, int64_t B, int eb, int device) { return rf_cfg(A, B, eb, device).K != 0; }

// Name of the kernel launch_tile_onchip runs for this stage (diagnostics: the bench's
// per-kernel roofline and the ncu launch lists use the same names).  Mirrors the launcher's
// decisions; the TMA choices are made on geometry (a tensor-map encode failure at launch
// falls back to the cp.async kernel of the same family).
const char *tile_kernel_name(const StageDesc &d, int device) {
    const DevProps dp = dev_props(device);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    if (env_int("IPT_TILE_RF_FORCE", 0) && fast_ok(d) && (d.eb == 4 || d.eb == 8) && rf_cfg(d.A, d.B, d.eb, device).K)
        return "tile_group_rf";
    if (fast_ok(d) && (long)fast_smem(d.A, d.B, d.eb) <= budget) {
        const size_t smem = fast_smem(d.A, d.B, d.eb);
        if (smem > 113 * 1024 && env_int("IPT_TILE_STREAM", 1))
            return "tile_onchip_stream";
        return "tile_onchip_ldg";
    }
    const uint64_t count = (uint64_t)(d.outer * d.inner);
    const bool packed = d.outer <= 1 || d.ostride == d.inner * d.A * d.B * d.eb;
    if (fast_ok(d) && tile_group_split(d.A, d.B, d.eb, device)) {
        const GroupCfg g = group_cfg(d.A, d.B, d.eb, count, device);
        const TmaGeom t = tma_geom(d.A, d.B, d.eb, g.K, g.colsplit);
        return (packed && t.ok && t.bytes <= g.slice) ? "tile_group_tma" : "tile_group_db";
    }
    if (!fast_ok(d) && tile_group_generic_split(d.A, d.B, d.eb, device)) {
        const GroupCfg g = group_cfg_generic(d.A, d.B, d.eb, count, device);
        const int V = 16 / d.eb;
        if (g.gcols > 1) return "tile_group_generic";   // 2-D grid: cp.async slices
        if (!g.colsplit && (d.B * d.eb) % 16 == 0 && ((uintptr_t)d.base & 15) == 0 && packed &&
            env_int("IPT_TILE_GEN_TMAA", 1) && tma_geom((d.A + V - 1) / V * V, d.B, d.eb, g.K, false).ok)
            return "tile_group_tma_elem";
        return "tile_group_generic";
    }
    if (fast_ok(d) && (long)fast_smem(d.A, d.B, d.eb) > budget && tile_cluster_k(d.A, d.B, d.eb, device))
        return "tile_onchip_cluster";
    if (fast_ok(d) && (d.eb == 4 || d.eb == 8) && (long)generic_smem(d.A, d.B, d.eb) > budget &&
        (packed || d.inner == 1) && rf_cfg(d.A, d.B, d.eb, device).K)
        return "tile_group_rf";
    if ((long)generic_smem(d.A, d.B, d.eb) > budget) return "tile_generic_cluster";
    return "tile_onchip_generic";
}

bool tile_onchip_fits(int64_t A, int64_t B, int eb, int device) {
    return tile_onchip_path(A, B, eb, device) != 0;
}

cudaError_t launch_tile_onchip(const StageDesc &d, void *ws, cudaStream_t st, int device) {
    if (d.s != 1) return cudaErrorInvalidValue;   // tile-local transposition of elements only
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
    p.gb = (uint32_t)env_int("IPT_TILE_GROUP", 0);
    p.diag = (int)env_int("IPT_TILE_DIAG", 0);
    if (p.diag & 16) {
        if (!g_trace && cudaMalloc(&g_trace, kTraceBytes) != cudaSuccess) g_trace = nullptr;
        if (g_trace) cudaMemsetAsync(g_trace, 0, kTraceBytes, st);
        p.trace = g_trace;
        if (!g_trace) p.diag &= ~16;
    }
    p.arrive_release = (int)env_int("IPT_TILE_ARRIVE_RELEASE", 0);
    const long budget = env_int("IPT_TILE_SMEM_MAX", dp.smem_optin);
    if (env_int("IPT_TILE_RF_FORCE", 0) && fast_ok(d) && (d.eb == 4 || d.eb == 8)) {   // tests
        const RfCfg c = rf_cfg(d.A, d.B, d.eb, device);
        if (c.K) return d.eb == 4 ? launch_group_rf<4>(d, p, c, ws, st, device)
                                  : launch_group_rf<8>(d, p, c, ws, st, device);
    }
    if (fast_ok(d) && (long)fast_smem(d.A, d.B, d.eb) <= budget) {
        const int V = 16 / d.eb;
        p.q = fast_q(d.B, d.eb);
        p.buf_bytes = (uint32_t)((size_t)d.A * p.q * 16);
        p.divMV = make_fastdiv((uint64_t)(d.A / V));
        p.divNV = make_fastdiv((uint64_t)(d.B / V));
        p.divNV32 = make_fastdiv32((uint32_t)(d.B / V));
        p.divMV32 = make_fastdiv32((uint32_t)(d.A / V));
        const size_t smem = fast_smem(d.A, d.B, d.eb);
        const bool big = smem > 113 * 1024 && env_int("IPT_TILE_BIGU", 1);
        if (smem > 113 * 1024 && env_int("IPT_TILE_STREAM", 1)) {
            p.K = 1;
            p.colsplit = 0;
            switch (d.eb) {
                case 4: return go(tile_onchip_stream<4>, p, smem, st, device);
                case 8: return go(tile_onchip_stream<8>, p, smem, st, device);
                case 16: return go(tile_onchip_stream<16>, p, smem, st, device);
            }
        }
        switch (d.eb) {
            // one CTA per SM for > 113 KB: twice the loads in flight per thread
            case 4: return big ? go(tile_onchip_ldg<4, 16, 1>, p, smem, st, device)
                               : go(tile_onchip_ldg<4, 8>, p, smem, st, device);
            case 8: return big ? go(tile_onchip_ldg<8, 16, 1>, p, smem, st, device)
                               : go(tile_onchip_ldg<8, 8>, p, smem, st, device);
            case 16: return big ? go(tile_onchip_ldg<16, 16, 1>, p, smem, st, device)
                                : go(tile_onchip_ldg<16, 8>, p, smem, st, device);
        }
    }
    if (fast_ok(d) && tile_group_split(d.A, d.B, d.eb, device)) {
        const GroupCfg g = group_cfg(d.A, d.B, d.eb, p.count, device);
        switch (d.eb) {
            case 4: return launch_group_db<4, false>(d, p, g, ws, st, device);
            case 8: return launch_group_db<8, false>(d, p, g, ws, st, device);
            case 16: return launch_group_db<16, false>(d, p, g, ws, st, device);
        }
    }
    if (!fast_ok(d) && tile_group_generic_split(d.A, d.B, d.eb, device)) {
        const GroupCfg g = group_cfg_generic(d.A, d.B, d.eb, p.count, device);
        switch (d.eb) {
            case 4: return launch_group_db<4, true>(d, p, g, ws, st, device);
            case 8: return launch_group_db<8, true>(d, p, g, ws, st, device);
        }
    }
    if (fast_ok(d) && (d.eb == 4 || d.eb == 8) && !tile_cluster_k(d.A, d.B, d.eb, device) &&
        (long)generic_smem(d.A, d.B, d.eb) > budget) {
        const RfCfg c = rf_cfg(d.A, d.B, d.eb, device);
        if (c.K) {
            cudaError_t e = d.eb == 4 ? launch_group_rf<4>(d, p, c, ws, st, device)
                                      : launch_group_rf<8>(d, p, c, ws, st, device);
            if (e != cudaErrorNotSupported) return e;
            cudaGetLastError();
        }
    }
    if (fast_ok(d) && (long)fast_smem(d.A, d.B, d.eb) > budget) {
        const int K = tile_cluster_k(d.A, d.B, d.eb, device);
        if (K) {
            const int V = 16 / d.eb;
            p.q = fast_q(d.B, d.eb);
            p.K = (uint32_t)K;
            p.colsplit = fast_colsplit(d.A, d.B, d.eb) ? 1 : 0;
            const int64_t nvr = d.B / V;
            const size_t smem = p.colsplit
                ? (size_t)d.A * (size_t)(((nvr + K - 1) / K) | 1) * 16
                : (size_t)((d.A / V + K - 1) / K) * V * p.q * 16;
            const bool big = smem > 113 * 1024 && env_int("IPT_TILE_BIGU", 1);
            if (big && env_int("IPT_TILE_STREAM", 1)) {
                p.divNV32 = make_fastdiv32((uint32_t)nvr);
                switch (d.eb) {
                    case 4: return go_cluster(tile_onchip_stream<4>, p, smem, K, st, device);
                    case 8: return go_cluster(tile_onchip_stream<8>, p, smem, K, st, device);
                    case 16: return go_cluster(tile_onchip_stream<16>, p, smem, K, st, device);
                }
            }
            switch (d.eb) {
                case 4: return big ? go_cluster(tile_onchip_cluster<4, 16, 1>, p, smem, K, st, device)
                                   : go_cluster(tile_onchip_cluster<4, 8>, p, smem, K, st, device);
                case 8: return big ? go_cluster(tile_onchip_cluster<8, 16, 1>, p, smem, K, st, device)
                                   : go_cluster(tile_onchip_cluster<8, 8>, p, smem, K, st, device);
                case 16: return big ? go_cluster(tile_onchip_cluster<16, 16, 1>, p, smem, K, st, device)
                                    : go_cluster(tile_onchip_cluster<16, 8>, p, smem, K, st, device);
            }
        }
    }
    p.pitch = generic_pitch(d.B);
    p.divM32 = make_fastdiv32((uint32_t)d.A);
    p.divN32 = make_fastdiv32((uint32_t)d.B);
    p.vec16 = (((uintptr_t)d.base & 15) == 0) && (p.tile_bytes % 16 == 0) &&
              (d.outer <= 1 || (d.ostride & 15) == 0) && d.eb <= 16;
    const size_t smem = generic_smem(d.A, d.B, d.eb);
    if ((long)smem > budget) {
        const int K = tile_generic_cluster_k(d.A, d.B, d.eb, device);
        if (!K) return cudaErrorInvalidValue;
        p.K = (uint32_t)K;
        p.colsplit = generic_colsplit(d.A, d.B) ? 1 : 0;
        p.ralign = generic_ralign(d.A, d.B, d.eb, K);
        const size_t cs = p.colsplit
            ? (size_t)d.A * (size_t)(((d.B + K - 1) / K) | 1) * d.eb
            : (size_t)generic_slice_rows(d.A, d.B, d.eb, K) * p.pitch * d.eb;
        switch (d.eb) {
            case 1: return go_cluster(tile_generic_cluster<uint8_t>, p, cs, K, st, device);
            case 2: return go_cluster(tile_generic_cluster<uint16_t>, p, cs, K, st, device);
            case 4: return go_cluster(tile_generic_cluster<uint32_t>, p, cs, K, st, device);
            case 8: return go_cluster(tile_generic_cluster<unsigned long long>, p, cs, K, st, device);
            case 16: return go_cluster(tile_generic_cluster<uint4>, p, cs, K, st, device);
        }
        return cudaErrorInvalidValue;
    }
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

// Internal diagnostic hook (not in the ABI): copy the last group-kernel timeline trace
// (IPT_TILE_DIAG=16; [CTA][iteration][4] globaltimer ns) to host memory.
extern "C" int ipt__tile_trace(void *host, size_t bytes) {
    if (!ipt::g_trace) return -1;
    cudaDeviceSynchronize();
    return (int)cudaMemcpy(host, ipt::g_trace, bytes < ipt::kTraceBytes ? bytes : ipt::kTraceBytes,
                           cudaMemcpyDeviceToHost);
}
