// cycle_seg.cu -- elementary transposition P(batch, A, B, s) by cycle following along
// precomputed, equal-length cycle segments (no flag bits).
//
// Paper: the 100! / 0100! stages shift super-elements along the cycles of Eq. (1)
// (Sec. 5.2).  PTTWAC lets work-items start anywhere and
// stop at a flag set by another work-item; the paper notes that cycles alone give too
// little and too irregular parallelism ("load imbalance"), which PTTWAC's flags
// repair dynamically.  For small, latency-bound stages (e.g. the 52 MB configs[0]
// matrix: one dependent global round trip per chain step, walker chains of random
// length) the makespan is set by the LONGEST chain segment, not by bandwidth.
//
// B200 design (beyond the paper): the planner walks the cycles of the stage's
// permutation once on the host (O(units), cached per shape -- like a plan) and cuts
// every cycle into segments of at most L units, L chosen so that every segment of every
// batch item and chunk gets its own walker (tasks <= co-resident walkers).  The kernel
// runs all segments in two phases separated by ONE grid-wide barrier:
//   phase 1: each walker loads the super-element (chunk) at its segment's first
//            position x into registers;
//   phase 2: it carries it along the segment: d = next(cur), load A[d], store the carried
//            data into d, carry A[d] on; the last step stores into the next segment's
//            first position WITHOUT reading it (its content was taken in phase 1).
// Every position is read once and written once; a position is only written after it was
// read (its own walker, program order; or the next segment's walker, phase 1 < barrier),
// so no flags, atomics or start re-checks are needed and every walker does <= L steps.
// Walkers are G-lane groups holding R 16-byte vectors per lane (units with S % 16 == 0
// and 16-byte aligned data only; the flag-based cycle_global covers the rest).
#include "ipt_internal.h"
#include "mem_ptx.cuh"

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <tuple>
#include <vector>

namespace ipt {

struct SegParams {
    char *base;
    uint64_t ostride, istride;   // bytes between outer / inner batch items
    uint64_t S;                  // unit (super-element) bytes, multiple of 16
    uint64_t A;
    FastDiv divB, divInner, divNch, divNseg;
    uint64_t nch;                // chunks per unit
    uint64_t chunk;              // bytes per chunk (G * R * 16)
    const ulonglong2 *segs;      // {first position, length} per segment
    uint64_t nseg, tasks;        // tasks = items * nseg * nch
    unsigned int *bar;           // grid barrier counters [arrive, exit]
    int self_reset;              // counters start at 0 and the last CTA re-zeroes them
    int store_after_load;        // IPT_SEG_SAL (default 1)
    uint32_t zero;               // 0 at run time, opaque to the compiler
    int diag;                    // measurement only (results invalid): 1 no barrier, 2 no phase 2,
                                 // 4 no phase-2 stores, 8 no phase-2 loads
};

template <int G, int R>
__global__ void __launch_bounds__(256, 4) cycle_seg_kernel(const SegParams p) {
    const uint64_t gtid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t w = gtid / G;
    const uint32_t l = threadIdx.x % G;
    const bool act = w < p.tasks;
    uint4 D[R], Bk[R];
#pragma unroll
    for (int v = 0; v < R; ++v) D[v] = make_uint4(0, 0, 0, 0);
    char *ib = nullptr;
    uint64_t cur = 0, len = 0, off0 = 0;
    bool valid[R];
    if (act) {
        uint64_t rest, ch, item, seg, to, ti;
        fdivmod(w, p.divNch, rest, ch);          // chunk fastest: a warp's walkers cover
        fdivmod(rest, p.divNseg, item, seg);     // adjacent chunks of one unit
        fdivmod(item, p.divInner, to, ti);
        ib = p.base + to * p.ostride + ti * p.istride;
        const ulonglong2 sg = p.segs[seg];
        cur = sg.x;
        len = sg.y;
        off0 = ch * p.chunk + (uint64_t)l * 16;
#pragma unroll
        for (int v = 0; v < R; ++v) {
            const uint64_t off = off0 + (uint64_t)v * G * 16;
            valid[v] = off < (ch + 1) * p.chunk && off < p.S;
            if (valid[v]) D[v] = ld_cg<16>(ib + cur * p.S + off);
        }
    }
    // phase-1 loads must have returned before this thread passes the barrier
    uint32_t f = 0;
#pragma unroll
    for (int v = 0; v < R; ++v) f |= fold(D[v]);
    if ((f & p.zero) != 0) __trap();
    __syncthreads();
    if (threadIdx.x == 0 && !(p.diag & 1)) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        atomicAdd(p.bar, 1u);
        uint32_t seen = 0;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(seen) : "l"(p.bar) : "memory");
        } while (seen < gridDim.x);
        if (p.self_reset && atomicAdd(p.bar + 1, 1u) == gridDim.x - 1) {
            // every CTA has left the spin: zero both counters for the next launch on this
            // stream (stream order makes them visible to it), no memset node needed
            atomicExch(p.bar, 0u);
            atomicExch(p.bar + 1, 0u);
        }
    }
    __syncthreads();
    if (!act || (p.diag & 2)) return;
    for (uint64_t i = 1; i <= len; ++i) {
        uint64_t q, r;
        fdivmod(cur, p.divB, q, r);
        const uint64_t d = r * p.A + q;           // Eq. (1) on units: (k mod B) * A + k / B
        char *gd = ib + d * p.S;
        uint32_t z = 0;
        if (i < len && !(p.diag & 8)) {
#pragma unroll
            for (int v = 0; v < R; ++v)
                if (valid[v]) Bk[v] = ld_cg<16>(gd + off0 + (uint64_t)v * G * 16);
            // Store only after the backup has arrived (address dependency): a store racing
            // its own line's pending fill in L2 stalls the slice (measured 2.5 vs 5.8 TB/s).
            if (p.store_after_load) {
                uint32_t f2 = 0;
#pragma unroll
                for (int v = 0; v < R; ++v) f2 |= valid[v] ? fold(Bk[v]) : 0u;
                z = f2 & p.zero;   // runtime zero: ptxas cannot fold it (and.b32 x, 0 it can)
            }
        }
        if (!(p.diag & 4)) {
#pragma unroll
            for (int v = 0; v < R; ++v)
                if (valid[v]) st_cg<16>(gd + z + off0 + (uint64_t)v * G * 16, D[v]);
        }
        if (i < len) {
#pragma unroll
            for (int v = 0; v < R; ++v) D[v] = Bk[v];
        }
        cur = d;
    }
}

// ------------------------------------------------- unaligned units (S % 16 != 0, S % 4 == 0)
// Same schedule for units whose start addresses have different 16-byte phases (e.g.
// m = 127 floats: 508-byte units).  A walker is a group of G lanes (G | 32; several walkers
// per warp for small units) holding one chunk of a unit as the 16-byte vectors COVERING it
// at its source position (vector v = r*G + gl), plus the chunk's word phase o (0..3) there.
// Storing into a target of phase p shifts the carried words by d = p - o words across the
// vector frame (one funnel step between neighbouring vectors: a shuffle inside the group,
// the group's edge lanes taking the neighbouring register); interior vectors are written
// with 16-byte stores, the two edge vectors word by word (their other words belong to the
// neighbouring units, moved by their own walkers).  The backup loaded from the target (its
// covering vectors, phase p) becomes the carried chunk.  Walkers of a warp may diverge
// (different segment lengths / shifts): every shuffle uses the walker's own lane mask.
// Vector v + dir (dir = +-1) of the group's frame, for v = r*G + gl.
template <int G, int R>
__device__ __forceinline__ uint4 group_vec_nb(const uint4 (&a)[R], int r, uint32_t gl, int dir, unsigned gmask) {
    const int src = ((int)gl + dir + G) % G;
    // the neighbouring register (compile-time indices: no local-memory array).  Lane s's
    // only receiver is lane s - dir; the receiver that wraps around the group (lane G-1
    // for dir = +1, lane 0 for dir = -1) wants the sender's neighbouring register, so the
    // edge sender (lane 0, resp. G-1) sends that one instead: one shuffle per word.
    const uint4 o = dir > 0 ? a[r + 1 < R ? r + 1 : R - 1] : a[r > 0 ? r - 1 : 0];
    const bool edge = R > 1 && (dir > 0 ? gl == 0 : gl == G - 1);
    const uint4 snd = edge ? o : a[r];
    uint4 x;
    x.x = __shfl_sync(gmask, snd.x, src, G);
    x.y = __shfl_sync(gmask, snd.y, src, G);
    x.z = __shfl_sync(gmask, snd.z, src, G);
    x.w = __shfl_sync(gmask, snd.w, src, G);
    return x;
}
__device__ __forceinline__ uint32_t w4(const uint4 &v, int k) {
    return k == 0 ? v.x : (k == 1 ? v.y : (k == 2 ? v.z : v.w));
}
// Words k of the shifted vector: out[k] = cat(lo, hi)[k + s], s in 0..3.
__device__ __forceinline__ uint4 funnel4(const uint4 &lo, const uint4 &hi, int s) {
    switch (s) {
        case 0: return lo;
        case 1: return make_uint4(lo.y, lo.z, lo.w, hi.x);
        case 2: return make_uint4(lo.z, lo.w, hi.x, hi.y);
        default: return make_uint4(lo.w, hi.x, hi.y, hi.z);
    }
}

struct SegUaParams {
    char *base;
    uint64_t ostride, istride;   // bytes between outer / inner batch items
    uint64_t S;                  // unit bytes (multiple of 4)
    uint64_t A;
    FastDiv divB, divInner, divNch, divNseg;
    uint64_t nch;                // chunks per unit
    uint32_t cw;                 // words per (full) chunk, multiple of 4
    uint32_t nw;                 // words per unit
    const ulonglong2 *segs;
    uint64_t nseg, tasks;
    unsigned int *bar;
    int self_reset;
    uint32_t zero;
};

template <int G, int R>
__global__ void __launch_bounds__(256, (R >= 5 ? 3 : 4)) cycle_seg_ua_kernel(const SegUaParams p) {
    const uint32_t gl = threadIdx.x % G;
    const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << ((threadIdx.x & 31) - gl));
    const uint64_t w = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / G;
    const bool act = w < p.tasks;
    uint4 D[R], Bk[R];
#pragma unroll
    for (int r = 0; r < R; ++r) D[r] = Bk[r] = make_uint4(0, 0, 0, 0);
    char *ib = nullptr;
    uint64_t cur = 0, len = 0, coff = 0;   // coff: byte offset of the chunk in its unit
    uint32_t nwc = 0;                      // words in this chunk
    int o = 0;                             // word phase of the carried chunk
    if (act) {
        uint64_t rest, ch, item, seg, to, ti;
        fdivmod(w, p.divNch, rest, ch);
        fdivmod(rest, p.divNseg, item, seg);
        fdivmod(item, p.divInner, to, ti);
        ib = p.base + to * p.ostride + ti * p.istride;
        const ulonglong2 sg = p.segs[seg];
        cur = sg.x;
        len = sg.y;
        coff = ch * (uint64_t)p.cw * 4;
        nwc = (uint32_t)min((uint64_t)p.cw, (uint64_t)p.nw - ch * p.cw);
        const uintptr_t a = (uintptr_t)(ib + cur * p.S + coff);
        o = (int)((a & 15) >> 2);
        const char *vb = (const char *)(a & ~(uintptr_t)15);
        const uint32_t nvv = (o + nwc + 3) >> 2;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const uint32_t v = r * G + gl;
            if (v < nvv) D[r] = ld_cg<16>(vb + (size_t)v * 16);
        }
    }
    uint32_t f = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) f |= fold(D[r]);
    if ((f & p.zero) != 0) __trap();
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
        atomicAdd(p.bar, 1u);
        uint32_t seen = 0;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(seen) : "l"(p.bar) : "memory");
        } while (seen < gridDim.x);
        if (p.self_reset && atomicAdd(p.bar + 1, 1u) == gridDim.x - 1) {
            atomicExch(p.bar, 0u);
            atomicExch(p.bar + 1, 0u);
        }
    }
    __syncthreads();
    if (!act) return;   // whole walkers: a group's lanes share one task
    for (uint64_t i = 1; i <= len; ++i) {
        uint64_t q, rr;
        fdivmod(cur, p.divB, q, rr);
        const uint64_t d = rr * p.A + q;             // Eq. (1) on units
        const uintptr_t a = (uintptr_t)(ib + d * p.S + coff);
        const int pt = (int)((a & 15) >> 2);         // target phase
        char *vb = (char *)(a & ~(uintptr_t)15);
        const uint32_t nvt = (pt + nwc + 3) >> 2;    // covering vectors of the target
        uint32_t z = 0;
        if (i < len) {
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const uint32_t v = r * G + gl;
                if (v < nvt) Bk[r] = ld_cg<16>(vb + (size_t)v * 16);
            }
            uint32_t f2 = 0;   // stores wait for the backup (see cycle_seg_kernel)
#pragma unroll
            for (int r = 0; r < R; ++r) f2 |= fold(Bk[r]);
            z = f2 & p.zero;
        }
        vb += z;
        // target vector v, word k = carried chunk word (4v + k - pt) = carried covering word
        // (4v + k - dsh), dsh = pt - o: from vectors (v, v+1) at shift -dsh, or (v-1, v) at
        // shift 4 - dsh
        const int dsh = pt - o;
        const int dir = dsh <= 0 ? 1 : -1;
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const uint4 nb = group_vec_nb<G, R>(D, r, gl, dir, gmask);
            const uint4 outv = dsh <= 0 ? funnel4(D[r], nb, -dsh) : funnel4(nb, D[r], 4 - dsh);
            const uint32_t v = r * G + gl;
            if (v < nvt) {
                const int t0 = (int)(4 * v) - pt;      // chunk word held by component 0
                char *dst = vb + (size_t)v * 16;
                if (t0 >= 0 && t0 + 3 < (int)nwc) {
                    st_cg<16>(dst, outv);
                } else {
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        if (t0 + k >= 0 && t0 + k < (int)nwc) st_cg<4>(dst + 4 * k, w4(outv, k));
                }
            }
        }
        if (i < len) {
#pragma unroll
            for (int r = 0; r < R; ++r) D[r] = Bk[r];
            o = pt;
        }
        cur = d;
    }
}

// ------------------------------------------------------------------------ host side
namespace {

struct SegPlan {
    bool ok = false;
    uint64_t L = 0, nseg = 0;
    void *dev = nullptr;   // ulonglong2[nseg], library-owned, never freed (plan cache)
    // The list is uploaded asynchronously on the stream of the first call (pinned staging
    // buffer, event `ready`): a later launch on another stream waits for the event; once it
    // has been seen complete (`landed`), the staging buffer is freed and no wait is needed.
    cudaEvent_t ready = nullptr;
    void *staging = nullptr;
    std::atomic<bool> landed{false};
};

// Walk the cycles of k -> (k mod B) * A + k / B on n = A*B units; cut each non-trivial
// cycle into segments of <= L units with L the smallest length whose segment count fits
// `max_seg`.  Returns false when even one segment per cycle does not fit.
bool build_segments(uint64_t A, uint64_t B, uint64_t max_seg, std::vector<ulonglong2> &out,
                    uint64_t &L) {
    const uint64_t n = A * B;
    std::vector<uint64_t> seen((n + 63) / 64, 0);
    auto next = [A, B](uint64_t k) { return (k % B) * A + k / B; };
    std::vector<std::pair<uint64_t, uint64_t>> cycles;   // (leader, length), length >= 2
    for (uint64_t k = 0; k < n; ++k) {
        if (seen[k >> 6] >> (k & 63) & 1) continue;
        uint64_t c = k, len = 0;
        do {
            seen[c >> 6] |= 1ull << (c & 63);
            c = next(c);
            ++len;
        } while (c != k);
        if (len >= 2) cycles.push_back({k, len});
    }
    if (cycles.empty()) { L = 0; out.clear(); return true; }
    if (cycles.size() > max_seg) return false;
    uint64_t lo = 1, hi = 0;
    for (auto &c : cycles) hi = std::max(hi, c.second);
    auto count = [&](uint64_t len) {
        uint64_t s = 0;
        for (auto &c : cycles) s += (c.second + len - 1) / len;
        return s;
    };
    while (lo < hi) {   // smallest L with count(L) <= max_seg
        const uint64_t mid = lo + (hi - lo) / 2;
        if (count(mid) <= max_seg) hi = mid; else lo = mid + 1;
    }
    L = lo;
    out.clear();
    out.reserve(count(L));
    for (auto &c : cycles) {
        uint64_t pos = c.first;
        for (uint64_t done = 0; done < c.second; done += L) {
            const uint64_t len = std::min(L, c.second - done);
            out.push_back(make_ulonglong2(pos, len));
            for (uint64_t j = 0; j < len; ++j) pos = next(pos);
        }
    }
    return true;
}

struct SegCfg {
    int G, R;
    uint64_t nch, chunk;
    bool ua = false;     // unaligned units: cycle_seg_ua_kernel, chunk = cw words
    uint32_t cw = 0;
};

// Unaligned units: a walker of G lanes x R vectors covers cap = G*R vectors; a chunk of cw
// words covers at most (cw + 6) / 4 of them at any phase, so cw + 3 <= 4 cap.  Units are cut
// into the fewest equal chunks (multiples of 4 words) that fit the largest walker (32 x 6),
// and each chunk gets the walker of the smallest cap that holds it (ties: fewest lanes,
// i.e. most walkers per warp).  R = 3, 5, 6 [r2]: with powers of two only, sizes just above
// a power-of-two cap (508 B = 33 covering vectors: 16 x 4 = 64 lanes-vectors, half idle)
// ran ~30 % below their neighbours (IPT_SEG_UA_R2=1 restores the {1, 2, 4} set).
constexpr int kSegUaRs[] = {1, 2, 3, 4, 5, 6};
SegCfg seg_cfg_ua(uint64_t S) {
    const uint64_t nw = S / 4;
    const long gmin = env_int("IPT_SEG_UA_G", 8);   // smallest walker width considered
    const bool pow2 = env_int("IPT_SEG_UA_R2", 0) != 0;
    const int rmax = pow2 ? 4 : 6;
    // words per chunk on the largest walker: cw + 3 <= 4 cap with cw a multiple of 4
    const uint64_t maxw = 4ull * 32 * rmax - 4;
    SegCfg c{32, rmax, (nw + maxw - 1) / maxw, 0, true, 0};
    if (pow2 && nw > 508) {   // round-1 rule: greedy 508-word chunks
        c.cw = 508;
        c.nch = (nw + 507) / 508;
        c.chunk = (uint64_t)c.cw * 4;
        return c;
    }
    const uint64_t cw = ((nw + c.nch - 1) / c.nch + 3) & ~3ull;   // balanced, 4-word multiple
    uint64_t best = ~0ull;
    for (int G : {8, 16, 32})
        if (G >= gmin)
            for (int R : kSegUaRs) {
                if (R > rmax || (pow2 && (R == 3 || R > 4))) continue;
                const uint64_t cap = (uint64_t)G * R;
                if (cw + 3 <= 4 * cap && cap < best) {
                    best = cap;
                    c.G = G;
                    c.R = R;
                }
            }
    c.cw = (uint32_t)cw;
    c.chunk = (uint64_t)c.cw * 4;
    return c;
}

// Is a stage with S-byte units run by the unaligned kernel?  (S % 16 != 0, or data not
// 16-byte aligned; 4-byte granular units only.)
bool seg_unaligned(uint64_t S, uintptr_t base, bool strided, uint64_t ostride) {
    return S % 16 || (base & 15) || (strided && (ostride & 15));
}

SegCfg seg_cfg(uint64_t S, bool ua = false) {
    if (ua || S % 16) return seg_cfg_ua(S);
    const uint64_t nv = S / 16;
    static const int Gs[3] = {8, 16, 32};
    SegCfg best{32, 4, (nv + 127) / 128, 32 * 4 * 16};
    if (nv > 128) {
        if (env_int("IPT_CYC_CHUNK256", 2) == 1) {
            // balanced chunks on 256-byte boundaries (16 vectors), at most 2 KB each; the
            // default is greedy 2 KB chunks (equal or faster, tools/seg_sweep.py)
            uint64_t cv = (nv + best.nch - 1) / best.nch;
            cv = (cv + 15) / 16 * 16;
            if (cv > 128) cv = 128;
            best.nch = (nv + cv - 1) / cv;
            best.R = (int)((cv + 31) / 32);
            best.chunk = cv * 16;
        }
        return best;
    }
    uint64_t bestcap = ~0ull;
    for (int G : Gs)
        for (int R = 1; R <= 4; ++R) {
            const uint64_t cap = (uint64_t)G * R;
            if (cap >= nv && cap < bestcap) { bestcap = cap; best = SegCfg{G, R, 1, cap * 16}; }
        }
    return best;
}

template <int G, int R>
void *seg_kernel_ptr() { return (void *)cycle_seg_kernel<G, R>; }

void *seg_kernel(int G, int R, bool ua = false) {
    if (ua) {
#define IPT_SEG_UA(g) if (G == g) switch (R) { \
        case 1: return (void *)cycle_seg_ua_kernel<g, 1>; case 2: return (void *)cycle_seg_ua_kernel<g, 2>; \
        case 3: return (void *)cycle_seg_ua_kernel<g, 3>; case 4: return (void *)cycle_seg_ua_kernel<g, 4>; \
        case 5: return (void *)cycle_seg_ua_kernel<g, 5>; case 6: return (void *)cycle_seg_ua_kernel<g, 6>; }
        IPT_SEG_UA(8) IPT_SEG_UA(16) IPT_SEG_UA(32)
#undef IPT_SEG_UA
        return nullptr;
    }
#define IPT_SEG_K(g, r) if (G == g && R == r) return seg_kernel_ptr<g, r>();
    IPT_SEG_K(8, 1) IPT_SEG_K(8, 2) IPT_SEG_K(8, 3) IPT_SEG_K(8, 4)
    IPT_SEG_K(16, 1) IPT_SEG_K(16, 2) IPT_SEG_K(16, 3) IPT_SEG_K(16, 4)
    IPT_SEG_K(32, 1) IPT_SEG_K(32, 2) IPT_SEG_K(32, 3) IPT_SEG_K(32, 4)
#undef IPT_SEG_K
    return nullptr;
}

int seg_blocks_per_sm(void *k) {
    static std::mutex mu;
    static std::map<void *, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(k);
    if (it != cache.end()) return it->second;
    int n = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, k, 256, 0) != cudaSuccess) {
        cudaGetLastError();
        n = 0;
    }
    cache[k] = n;
    return n;
}

std::mutex g_seg_mu;
std::map<std::tuple<int, uint64_t, uint64_t, uint64_t>, std::shared_ptr<SegPlan>> g_seg_cache;

// Self-resetting barrier counters, one zero-initialised pair per (device, stream); created
// on first use, never freed.  Never used by captured launches: a graph may be replayed on
// another stream concurrently with direct calls on this one (the workspace + memset path
// is captured instead).
std::mutex g_ctr_mu;
std::map<std::pair<int, cudaStream_t>, unsigned int *> g_ctr;

unsigned int *seg_counters(int device, cudaStream_t st) {
    std::lock_guard<std::mutex> lk(g_ctr_mu);
    auto key = std::make_pair(device, st);
    auto it = g_ctr.find(key);
    if (it != g_ctr.end()) return it->second;
    void *p = nullptr;
    // zeroed ON the stream that uses the pair (a legacy-stream cudaMemset is not ordered
    // before work on a non-blocking stream -- found on the host pipeline's compute stream)
    if (cudaMalloc(&p, 256) != cudaSuccess || cudaMemsetAsync(p, 0, 256, st) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    g_ctr[key] = (unsigned int *)p;
    return (unsigned int *)p;
}

bool seg_plan_cached(int device, uint64_t A, uint64_t B, uint64_t max_seg) {
    std::lock_guard<std::mutex> lk(g_seg_mu);
    return g_seg_cache.count(std::make_tuple(device, A, B, max_seg)) != 0;
}

std::shared_ptr<SegPlan> seg_plan(int device, uint64_t A, uint64_t B, uint64_t max_seg, cudaStream_t st) {
    const auto key = std::make_tuple(device, A, B, max_seg);
    {
        std::lock_guard<std::mutex> lk(g_seg_mu);
        auto it = g_seg_cache.find(key);
        if (it != g_seg_cache.end()) return it->second;
    }
    auto sp = std::make_shared<SegPlan>();
    std::vector<ulonglong2> segs;
    uint64_t L = 0;
    if (build_segments(A, B, max_seg, segs, L)) {
        sp->L = L;
        sp->nseg = segs.size();
        sp->ok = true;
        sp->landed = segs.empty();
        if (!segs.empty()) {
            // asynchronous upload on the caller's stream: no host stall on unrelated device
            // work (the first call of a shape may come from an asynchronous API)
            const size_t bytes = segs.size() * sizeof(ulonglong2);
            if (cudaMalloc(&sp->dev, bytes) != cudaSuccess || cudaMallocHost(&sp->staging, bytes) != cudaSuccess ||
                cudaEventCreateWithFlags(&sp->ready, cudaEventDisableTiming) != cudaSuccess) {
                cudaGetLastError();
                sp->ok = false;
            } else {
                std::memcpy(sp->staging, segs.data(), bytes);
                if (cudaMemcpyAsync(sp->dev, sp->staging, bytes, cudaMemcpyHostToDevice, st) != cudaSuccess ||
                    cudaEventRecord(sp->ready, st) != cudaSuccess) {
                    cudaGetLastError();
                    sp->ok = false;
                }
            }
        }
    }
    std::lock_guard<std::mutex> lk(g_seg_mu);
    g_seg_cache[key] = sp;
    return sp;
}

// Order a launch on `st` after the plan's upload.  Returns false when that cannot be done
// under stream capture (upload not yet seen complete): the caller uses the flag kernel.
bool seg_plan_ready(SegPlan &sp, cudaStream_t st, bool capturing) {
    if (sp.landed) return true;
    std::lock_guard<std::mutex> lk(g_seg_mu);
    if (sp.landed) return true;
    if (capturing) return false;
    const cudaError_t q = cudaEventQuery(sp.ready);
    if (q == cudaSuccess) {
        cudaFreeHost(sp.staging);
        sp.staging = nullptr;
        sp.landed = true;
        return true;
    }
    cudaGetLastError();   // cudaErrorNotReady
    return cudaStreamWaitEvent(st, sp.ready, 0) == cudaSuccess;
}

}  // namespace

// Walkers a launch can keep co-resident for a stage with S-byte units (0: not applicable).
uint64_t cycle_seg_walkers(int64_t S_bytes, int device) {
    if (S_bytes % 4 || (S_bytes % 16 && !env_int("IPT_SEG_UA", 1))) return 0;
    const SegCfg c = seg_cfg((uint64_t)S_bytes);
    void *k = seg_kernel(c.G, c.R, c.ua);
    const int per_sm = device >= 0 ? seg_blocks_per_sm(k) : 4;
    return (uint64_t)dev_props(device).sms * per_sm * 256 / c.G;
}

// Host cycle walk bound: ~10 ns per unit, once per shape; beyond 2^26 units (~0.7 s) the
// flag kernel is used instead.
constexpr uint64_t kSegMaxUnits = 1ull << 26;

bool stage_unaligned(const StageDesc &d) {
    return seg_unaligned((uint64_t)(d.s * d.eb), (uintptr_t)d.base, d.outer > 1, (uint64_t)d.ostride);
}

bool cycle_seg_applicable(const StageDesc &d) {
    const uint64_t S = (uint64_t)(d.s * d.eb);
    if ((uint64_t)(d.A * d.B) > kSegMaxUnits) return false;
    if (!stage_unaligned(d)) return true;
    // unaligned units: 4-byte granular (the walker moves whole words)
    if (S % 4 || ((uintptr_t)d.base & 3) || (d.outer > 1 && (d.ostride & 3))) return false;
    return env_int("IPT_SEG_UA", 1) != 0;
}

size_t cycle_seg_ws_bytes() { return 256; }

// Returns cudaErrorNotSupported when the stage does not fit one round of walkers (the
// caller then uses the flag-based cycle_global).
cudaError_t launch_cycle_seg(const StageDesc &d, void *ws, cudaStream_t st, int device) {
    if (!cycle_seg_applicable(d)) return cudaErrorNotSupported;
    const uint64_t S = (uint64_t)(d.s * d.eb);
    const bool ua = stage_unaligned(d);
    const SegCfg c = seg_cfg(S, ua);
    void *k = seg_kernel(c.G, c.R, ua);
    const int per_sm = seg_blocks_per_sm(k);
    if (per_sm < 1) return cudaErrorNotSupported;
    const uint64_t items = (uint64_t)(d.outer * d.inner);
    const uint64_t walkers = (uint64_t)dev_props(device).sms * per_sm * 256 / c.G;
    const uint64_t per_item = walkers / (items * c.nch);
    if (per_item < 1) return cudaErrorNotSupported;
    // building a segment plan allocates and copies synchronously: not during stream capture
    // (a captured call uses an already cached plan, else the flag kernel)
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(st, &cap) != cudaSuccess) { cudaGetLastError(); cap = cudaStreamCaptureStatusActive; }
    if (cap != cudaStreamCaptureStatusNone && !seg_plan_cached(device, (uint64_t)d.A, (uint64_t)d.B, per_item))
        return cudaErrorNotSupported;
    auto sp = seg_plan(device, (uint64_t)d.A, (uint64_t)d.B, per_item, st);
    if (!sp->ok) return cudaErrorNotSupported;
    if (sp->nseg == 0) return cudaSuccess;   // identity permutation
    if (!seg_plan_ready(*sp, st, cap != cudaStreamCaptureStatusNone)) return cudaErrorNotSupported;
    unsigned int *ctr = nullptr;
    if (env_int("IPT_SEG_RESET", 1))
        ctr = cap == cudaStreamCaptureStatusNone ? seg_counters(device, st) : nullptr;   // captured: workspace
    if (!ctr) {
        const cudaError_t e = cudaMemsetAsync(ws, 0, 2 * sizeof(unsigned int), st);
        if (e != cudaSuccess) return e;
    }
    if (ua) {
        SegUaParams u{};
        u.base = d.base;
        u.ostride = (uint64_t)d.ostride;
        u.istride = (uint64_t)(d.A * d.B) * S;
        u.S = S;
        u.A = (uint64_t)d.A;
        u.divB = make_fastdiv((uint64_t)d.B);
        u.divInner = make_fastdiv((uint64_t)d.inner);
        u.divNch = make_fastdiv(c.nch);
        u.divNseg = make_fastdiv(sp->nseg);
        u.nch = c.nch;
        u.cw = c.cw;
        u.nw = (uint32_t)(S / 4);
        u.segs = (const ulonglong2 *)sp->dev;
        u.nseg = sp->nseg;
        u.tasks = items * sp->nseg * c.nch;
        u.bar = ctr ? ctr : (unsigned int *)ws;
        u.self_reset = ctr ? 1 : 0;
        u.zero = 0;
        const uint64_t blocks_needed = (u.tasks * c.G + 255) / 256;
        const unsigned grid = (unsigned)std::min<uint64_t>(blocks_needed, (uint64_t)dev_props(device).sms * per_sm);
        if (env_int("IPT_DEBUG", 0))
            fprintf(stderr, "[ipt] cycle_seg_ua A=%lld B=%lld S=%llu G=%d R=%d cw=%u nch=%llu L=%llu nseg=%llu grid=%u\n",
                    (long long)d.A, (long long)d.B, (unsigned long long)S, c.G, c.R, c.cw,
                    (unsigned long long)c.nch, (unsigned long long)sp->L, (unsigned long long)sp->nseg, grid);
        void *args[] = {&u};
        cudaError_t e = cudaLaunchCooperativeKernel(k, dim3(grid), dim3(256), args, 0, st);
        if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
            cudaGetLastError();
            return cudaErrorNotSupported;
        }
        note_launch();
        return e != cudaSuccess ? e : cudaGetLastError();
    }
    SegParams p{};
    p.base = d.base;
    p.ostride = (uint64_t)d.ostride;
    p.istride = (uint64_t)(d.A * d.B) * S;
    p.S = S;
    p.A = (uint64_t)d.A;
    p.divB = make_fastdiv((uint64_t)d.B);
    p.divInner = make_fastdiv((uint64_t)d.inner);
    p.divNch = make_fastdiv(c.nch);
    p.divNseg = make_fastdiv(sp->nseg);
    p.nch = c.nch;
    p.chunk = c.chunk;
    p.segs = (const ulonglong2 *)sp->dev;
    p.nseg = sp->nseg;
    p.tasks = items * sp->nseg * c.nch;
    p.store_after_load = (int)env_int("IPT_SEG_SAL", 1);
    p.zero = 0;
    p.diag = (int)env_int("IPT_SEG_DIAG", 0);
    // barrier counters: a library-owned, self-resetting pair per (device, stream) -- no memset
    // node per launch (2 us of a ~40 us configs[0] transposition); the caller's workspace
    // with a memset (above) when the pair cannot be used (stream capture, IPT_SEG_RESET=0)
    cudaError_t e = cudaSuccess;
    p.bar = ctr ? ctr : (unsigned int *)ws;
    p.self_reset = ctr ? 1 : 0;
    const uint64_t blocks_needed = (p.tasks * c.G + 255) / 256;
    const unsigned grid = (unsigned)std::min<uint64_t>(blocks_needed, (uint64_t)dev_props(device).sms * per_sm);
    if (env_int("IPT_DEBUG", 0))
        fprintf(stderr, "[ipt] cycle_seg A=%lld B=%lld S=%llu G=%d R=%d nch=%llu L=%llu nseg=%llu tasks=%llu grid=%u\n",
                (long long)d.A, (long long)d.B, (unsigned long long)S, c.G, c.R,
                (unsigned long long)c.nch, (unsigned long long)sp->L, (unsigned long long)sp->nseg,
                (unsigned long long)p.tasks, grid);
    void *args[] = {&p};
    e = cudaLaunchCooperativeKernel(k, dim3(grid), dim3(256), args, 0, st);
    if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
        cudaGetLastError();            // co-residency not available here: flag kernel instead
        return cudaErrorNotSupported;  // (the counter memset above is harmless)
    }
    note_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
}

const char *cycle_seg_name(const StageDesc &d) { return stage_unaligned(d) ? "cycle_seg_ua" : "cycle_seg"; }

// Would launch_cycle_seg run this stage (diagnostics)?  Without a cached segment plan the
// cycles are not walked here: a stage with more cycles than walkers (rare) is reported as
// segmented although the launcher then falls back to the flag kernel.
bool cycle_seg_would_launch(const StageDesc &d, int device) {
    if (!cycle_seg_applicable(d)) return false;
    const bool ua = stage_unaligned(d);
    const SegCfg c = seg_cfg((uint64_t)(d.s * d.eb), ua);
    const int per_sm = seg_blocks_per_sm(seg_kernel(c.G, c.R, ua));
    if (per_sm < 1) return false;
    const uint64_t items = (uint64_t)(d.outer * d.inner);
    const uint64_t walkers = (uint64_t)dev_props(device).sms * per_sm * 256 / c.G;
    return walkers / (items * c.nch) >= 1;
}

// Planner estimate of the segment length L (units per walker) without walking cycles.
uint64_t cycle_seg_est_len(int64_t units_per_item, int64_t items, int64_t S_bytes, int device) {
    if ((uint64_t)units_per_item > kSegMaxUnits) return 0;
    const uint64_t w = cycle_seg_walkers(S_bytes, device);
    if (!w) return 0;
    const SegCfg c = seg_cfg((uint64_t)S_bytes);
    const uint64_t per_item = w / ((uint64_t)items * c.nch);
    if (per_item < 1) return 0;
    return ((uint64_t)units_per_item + per_item - 1) / per_item;
}

}  // namespace ipt

// Test hook (host only, not part of the ABI in include/ipt.h): build the segments of the
// A x B unit permutation for at most max_seg walkers and verify them the way the kernel
// uses them -- every non-fixed position is read exactly once (a segment's first position
// in phase 1, the others as backups) and written exactly once (positions 1..len of the
// segment); fixed points are untouched.  Returns the number of segments (L in *L_out), -1
// if the segments do not fit max_seg, -2 if the coverage check fails.
extern "C" int64_t ipt__seg_check(uint64_t A, uint64_t B, uint64_t max_seg, uint64_t *L_out) {
    std::vector<ulonglong2> segs;
    uint64_t L = 0;
    if (!ipt::build_segments(A, B, max_seg, segs, L)) return -1;
    if (L_out) *L_out = L;
    const uint64_t n = A * B;
    std::vector<uint8_t> rd(n, 0), wr(n, 0);
    auto next = [A, B](uint64_t k) { return (k % B) * A + k / B; };
    for (const ulonglong2 &sg : segs) {
        if (sg.y < 1 || sg.y > L || sg.x >= n) return -2;
        uint64_t cur = sg.x;
        ++rd[cur];
        for (uint64_t i = 1; i <= sg.y; ++i) {
            const uint64_t d = next(cur);
            if (i < sg.y) ++rd[d];
            ++wr[d];
            cur = d;
        }
    }
    for (uint64_t k = 0; k < n; ++k) {
        const bool fixed = next(k) == k;
        if (fixed ? (rd[k] || wr[k]) : (rd[k] != 1 || wr[k] != 1)) return -2;
    }
    return (int64_t)segs.size();
}
