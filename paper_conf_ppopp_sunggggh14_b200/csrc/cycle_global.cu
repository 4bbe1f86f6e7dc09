// cycle_global.cu -- elementary transposition P(batch, A, B, s) by cycle following of
// super-elements coordinated through a packed global flag bitmap.
//
// Paper: the 100! / 0100! transpositions ("every m-element tile is treated as a
// super-element that is then shifted"; Sec. 5.2) shift super-elements along
// the cycles of Eq. (1) applied to the A x B matrix of super-elements; many
// work-items share a cycle and coordinate with atomically set flag bits (PTTWAC, P:117,
// P:172-174); "only one bit per super-element is needed".  Sec. 5.2.1
// moves one super-element per SIMD unit (warp) instead of one per work-group, with the
// super-element held in registers when its size allows ("register tiling").
//
// B200 design:
//   * A "walker" is a group of G lanes (G | 32) holding one super-element (or one chunk
//     of it) in registers as W-byte vectors (W = 16 when alignment permits), R vectors per
//     lane.  A warp runs 32/G walkers in lock-step, so a warp keeps 32/G independent
//     chains in flight (Little's law); a persistent grid fills every SM.  With G = 32 all
//     control flow is warp-uniform.
//   * Super-elements larger than one walker's capacity are split into `nchunk` chunks
//     that follow the SAME permutation independently (moving chunk c of every
//     super-element is itself a valid permutation), each with its own flag bit.
//   * Start units are handed out 32 at a time (one flag word, which doubles as a
//     pre-check so claimed units are never re-read) from a global work counter: in
//     increasing order for one matrix (adjacent work-items start at adjacent elements,
//     P:172), scrambled across a batch so that all matrices' start frontiers advance
//     together (fewer, longer chains).
//   * Claim protocol (P1; modelled in tools/protocol_sim.py): flag bit u =
//     "unit u has received its final value".  Chain step from cur: d = next(cur); load
//     backup = A[d] and claim bit d (atomic OR, acquire) concurrently; a lost claim ends
//     the chain, a won claim stores the carried data into d (after the claim) and carries
//     the backup on.  A cycle that closes at the walker's own start is claimed like any
//     other target (its backup is not re-read).  A chain start at x loads A[x], fences,
//     and re-checks bit x; if set, the start is abandoned (the claimer of x carries A[x]).
//   * Index maps use multiply-high division (no '%' or '/' in the loop), in 32-bit
//     arithmetic whenever every index fits (I = uint32_t), else 64-bit.
#include "ipt_internal.h"
#include "mem_ptx.cuh"

#include <map>
#include <mutex>

namespace ipt {

__device__ __forceinline__ void fdivmod_t(uint32_t n, const FastDiv32 &f, const FastDiv &,
                                          uint32_t &q, uint32_t &r) {
    fdivmod32(n, f, q, r);
}
__device__ __forceinline__ void fdivmod_t(uint64_t n, const FastDiv32 &, const FastDiv &f,
                                          uint64_t &q, uint64_t &r) {
    fdivmod(n, f, q, r);
}

struct Div2 {
    FastDiv d64;
    FastDiv32 d32;
};

struct CycParams {
    char *base;
    uint64_t ostride;   // bytes between outer batch items
    uint64_t istride;   // bytes between inner batch items (= A*B*S)
    uint64_t S;         // super-element bytes
    uint64_t A, AB;
    uint64_t nchunk;    // chunks per super-element
    uint64_t cvec;      // vectors per (full) chunk
    uint64_t nvec;      // vectors per super-element
    uint64_t units;     // batch * A*B * nchunk
    uint64_t nwords;    // flag words
    uint64_t wstride;   // start-order scramble (coprime to nwords)
    uint64_t nfetch;    // fetches = nwords << segsh (a fetch is a segment of a flag word)
    uint32_t segsh;     // log2(segments per flag word): small stages hand out fewer units
    Div2 divB, divAB, divInner, divNchunk, divNwords;
    uint32_t *flags;
    unsigned long long *counter;
    int refresh;        // re-read the flag word after a chain ends before the next start
    int fence;          // 1: PTX-model fences on both sides of the claim protocol
    uint32_t zero;      // 0 at run time, opaque to the compiler (address-dependency knob)
    unsigned long long *stats;  // optional diagnostics (IPT_CYC_STATS=1): round counts
    int fastloop;       // steady-state chain loop (IPT_CYC_FASTLOOP, default on)
    int sal;            // chain stores wait for the target's backup load (IPT_CYC_SAL)
};

enum : int { M_FETCH = 0, M_SCAN = 1, M_START = 2, M_CHAIN = 3, M_REFRESH = 4, M_DONE = 5 };

// Register budget -> resident warps: the kernel is latency-bound (one dependent round
// trip per chain step), so it is compiled for full occupancy (8 x 256 threads = 64 warps
// per SM, <= 32 registers) when a walker's payload is <= 16 bytes per lane.
template <int W, int R> struct CycMinBlocks {
    static constexpr int value = (W * R <= 16) ? 8 : ((W * R <= 32) ? 6 : (W * R <= 64 ? 4 : 2));
};

template <int W, int G, int R, typename I>
__global__ void __launch_bounds__(256, CycMinBlocks<W, R>::value)
cycle_global_kernel(const CycParams p) {
    using V = typename VecT<W>::type;
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31;
    const int gl = lane % G;          // lane within walker group
    const int g0 = lane - gl;         // first lane of the group
    const unsigned gmask = (G == 32) ? FULL : (((1u << G) - 1u) << g0);
    const I A = (I)p.A, nchunk = (I)p.nchunk, nwords = (I)p.nwords;

    int mode = M_FETCH;
#ifdef IPT_CYC_STATS
    // round statistics (diagnostic build: nvcc -DIPT_CYC_STATS, tools/cyc_stats.py)
    uint32_t st_start = 0, st_abort = 0, st_step = 0, st_lost = 0, st_refresh = 0, st_iter = 0;
#endif
    I word = 0;            // flag word (= 32 start units) being scanned
    uint32_t cw = 0;       // cached copy of that flag word
    int nb = 0;            // next bit to consider in the word
    char *item = nullptr;  // start of the current batch item (+ chunk offset)
    I ubase = 0;           // unit index of (item, k = 0, chunk)
    I k = 0, k0 = 0;
    int nv = 0;            // vectors in this chunk
    V data[R], in[R];
#pragma unroll
    for (int r = 0; r < R; ++r) { data[r] = V(); in[r] = V(); }

    auto next_of = [&](I x) -> I {
        I q, r;
        fdivmod_t(x, p.divB.d32, p.divB.d64, q, r);
        return r * A + q;                              // Eq. (1) on super-element offsets
    };

    // One round: work acquisition (if needed), then one memory round trip; `in` receives
    // the target's content.  (A variant that also loaded the chain's following target one
    // round early -- valid, since a won claim means nobody else ever wrote it -- measured
    // 10-25 % slower on B200: more registers, fewer warps, DRAM already saturated.)
    auto round = [&]() -> bool {
        // ----------------------------------------------- steady state: every walker chains
        // Chains average ~30 steps, so most rounds of a warp are pure chain steps; this
        // loop runs them without the acquisition / start / refresh logic (the kernel is
        // issue-bound for small super-elements).  Same protocol as the general round.
        if (p.fastloop && __all_sync(FULL, mode == M_CHAIN)) {
            for (;;) {
                const I tgt = next_of(k);
                const bool back_home = (tgt == k0);
                const I ut = ubase + tgt * nchunk;
                const uint32_t bit = 1u << ((uint32_t)ut & 31);
                char *addr = item + (uint64_t)tgt * p.S;
                if (!back_home) {
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int v = gl + r * G;
                        if (v < nv) in[r] = ld_cg<W>(addr + (size_t)v * W);
                    }
                }
                uint32_t old = 0;
                if (gl == 0) {
                    uint32_t *fwp = p.flags + (ut >> 5);
                    old = p.fence ? atom_or_acq_u32(fwp, bit) : atom_or_u32(fwp, bit);
                }
                old = __shfl_sync(FULL, old, g0);
                __syncwarp();
                if (!(old & bit)) {
                    if (p.sal && !back_home) {   // store after the backup arrived (cycle_seg.cu)
                        uint32_t acc = 0;
#pragma unroll
                        for (int r = 0; r < R; ++r) {
                            const int v = gl + r * G;
                            if (v < nv) acc |= fold(in[r]);
                        }
                        addr += (acc & p.zero);
                    }
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int v = gl + r * G;
                        if (v < nv) st_cg<W>(addr + (size_t)v * W, data[r]);
                    }
                    if (back_home) {
                        mode = M_SCAN;
                    } else {
#pragma unroll
                        for (int r = 0; r < R; ++r) data[r] = in[r];
                        k = tgt;
                    }
                } else {
                    mode = p.refresh ? M_REFRESH : M_SCAN;
                }
#ifdef IPT_CYC_STATS
                if (p.stats) { st_step += !(old & bit); st_lost += (old & bit) != 0; ++st_iter; }
#endif
                if (!__all_sync(FULL, mode == M_CHAIN)) break;
            }
            return true;
        }
        // ------------------------------------------------ work acquisition (no data moved)
        for (;;) {
            const unsigned need = __ballot_sync(FULL, mode == M_FETCH && gl == 0);
            if (need) {
                const int leader = __ffs(need) - 1;
                unsigned long long wb = 0;
                if (lane == leader) wb = atomicAdd(p.counter, (unsigned long long)__popc(need));
                wb = __shfl_sync(FULL, wb, leader);
                const uint64_t f = wb + __popc(need & ((1u << g0) - 1u));
                const bool have = f < p.nfetch;
                const uint64_t mine64 = f >> p.segsh;
                const uint32_t seg = (uint32_t)(f & ((1u << p.segsh) - 1u));
                I mine = (I)mine64;
                if (have && p.wstride != 1) {
                    uint64_t q, r;
                    fdivmod(mine64 * p.wstride, p.divNwords.d64, q, r);
                    mine = (I)r;
                }
                const uint32_t F = 32u >> p.segsh;
                const uint32_t segmask = (F == 32) ? 0xffffffffu : (((1u << F) - 1u) << (seg * F));
                uint32_t fw = 0;
                if (mode == M_FETCH && have) fw = ld_relaxed_u32(p.flags + mine);
                fw = __shfl_sync(FULL, fw, g0);
                if (mode == M_FETCH) {
                    word = mine;
                    if (!have) {
                        mode = M_DONE;
                    } else {
                        cw = fw | ~segmask;     // bits outside this segment: not ours
                        nb = 0;
                        mode = M_SCAN;
                    }
                }
            }
            // Scan the cached word for the next unit that still needs a start walker.
            while (mode == M_SCAN) {
                uint32_t valid = 0xffffffffu;
                if (word == nwords - 1 && (p.units & 31)) valid = (1u << (p.units & 31)) - 1u;
                const uint32_t cand = ~cw & valid & (nb >= 32 ? 0u : (0xffffffffu << nb));
                if (!cand) { mode = M_FETCH; break; }
                const int b = __ffs(cand) - 1;
                nb = b + 1;
                const I u = word * 32 + (I)b;
                I tk = u, ch = 0;
                if (p.nchunk > 1) fdivmod_t(u, p.divNchunk.d32, p.divNchunk.d64, tk, ch);
                I T, kk;
                fdivmod_t(tk, p.divAB.d32, p.divAB.d64, T, kk);
                if (next_of(kk) == kk) continue;        // fixed point of Eq. (1): nothing moves
                I to, ti;
                fdivmod_t(T, p.divInner.d32, p.divInner.d64, to, ti);
                item = p.base + (uint64_t)to * p.ostride + (uint64_t)ti * p.istride +
                       (uint64_t)ch * p.cvec * W;
                ubase = T * (I)p.AB * nchunk + ch;
                nv = (int)((ch == nchunk - 1) ? (p.nvec - (uint64_t)ch * p.cvec) : p.cvec);
                k = k0 = kk;
                mode = M_START;
            }
            const unsigned pending = __ballot_sync(FULL, mode == M_FETCH || mode == M_SCAN);
            if (!pending) break;
        }
        if (!__ballot_sync(FULL, mode != M_DONE)) {
#ifdef IPT_CYC_STATS
            if (p.stats && gl == 0) {
                atomicAdd(p.stats + 0, (unsigned long long)st_start);
                atomicAdd(p.stats + 1, (unsigned long long)st_abort);
                atomicAdd(p.stats + 2, (unsigned long long)st_step);
                atomicAdd(p.stats + 3, (unsigned long long)st_lost);
                atomicAdd(p.stats + 4, (unsigned long long)st_refresh);
                if (lane == 0) atomicAdd(p.stats + 5, (unsigned long long)st_iter);
            }
#endif
            return false;
        }
#ifdef IPT_CYC_STATS
        ++st_iter;
#endif

        // --------------------------------------------------------------- memory round
        const I tgt = (mode == M_CHAIN) ? next_of(k) : k;
        // Cycle closed at our own start x: x must still be CLAIMED (another walker carrying
        // A[prev(x)] -- the start walker of prev(x) -- may race for it), but its backup is
        // the value this walker already delivered, so it is not re-read.
        const bool back_home = (mode == M_CHAIN) && (tgt == k0);
        const I ut = ubase + tgt * nchunk;             // flag index of the target unit
        const uint32_t bit = 1u << ((uint32_t)ut & 31);
        uint32_t *fwp = p.flags + (ut >> 5);
        char *addr = item + (uint64_t)tgt * p.S;
        const bool moving = (mode == M_START || mode == M_CHAIN) && !back_home;

        if (moving) {
            // a start's data loads are acquire loads: its flag re-check below is ordered
            // after them without a full fence
            const bool acq = (mode == M_START) && p.fence;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int v = gl + r * G;
                if (v < nv) in[r] = acq ? ld_acq<W>(addr + (size_t)v * W) : ld_cg<W>(addr + (size_t)v * W);
            }
        }
        uint32_t old = 0;
        if (mode == M_CHAIN && gl == 0)
            old = p.fence ? atom_or_acq_u32(fwp, bit) : atom_or_u32(fwp, bit);
        uint32_t fw = 0;
        if (mode == M_START) {
            if (!p.fence) {   // address dependency on the loaded data instead of acquire
                uint32_t acc = 0;
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const int v = gl + r * G;
                    if (v < nv) acc |= fold(in[r]);
                }
                fwp += (acc & p.zero);
            }
            fw = ld_relaxed_u32(fwp);
        } else if (mode == M_REFRESH) {
            fw = ld_relaxed_u32(p.flags + word);
        }

        // ------------------------------------------------------------------- resolve
        uint32_t fw0;
        bool start_lost;
        if (G == 32) {
            old = __shfl_sync(FULL, old, 0);
            __syncwarp();   // orders lane 0's (acquire) claim before the other lanes' stores
            start_lost = __any_sync(FULL, (fw & bit) != 0);
            fw0 = fw;
        } else {
            old = __shfl_sync(FULL, old, g0);
            __syncwarp();
            const unsigned seen = __ballot_sync(FULL, mode == M_START && (fw & bit));
            start_lost = (seen & gmask) != 0;
            fw0 = __shfl_sync(FULL, fw, g0);
        }
#ifdef IPT_CYC_STATS
        if (p.stats) {
            st_start += (mode == M_START);
            st_abort += (mode == M_START && start_lost);
            st_step += (mode == M_CHAIN && !(old & bit));
            st_lost += (mode == M_CHAIN && (old & bit));
            st_refresh += (mode == M_REFRESH);
        }
#endif
        if (mode == M_START) {
            cw |= fw0;
            if (start_lost) {
                mode = M_SCAN;                         // already claimed: its claimer carries A[x]
            } else {
#pragma unroll
                for (int r = 0; r < R; ++r) data[r] = in[r];
                mode = M_CHAIN;
            }
        } else if (mode == M_CHAIN) {
            if (!(old & bit)) {
                if (p.sal && !back_home) {
                    uint32_t acc = 0;
#pragma unroll
                    for (int r = 0; r < R; ++r) {
                        const int v = gl + r * G;
                        if (v < nv) acc |= fold(in[r]);
                    }
                    addr += (acc & p.zero);
                }
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const int v = gl + r * G;
                    if (v < nv) st_cg<W>(addr + (size_t)v * W, data[r]);
                }
                if (back_home) {
                    mode = M_SCAN;
                } else {
#pragma unroll
                    for (int r = 0; r < R; ++r) data[r] = in[r];
                    k = tgt;
                }
            } else {
                mode = p.refresh ? M_REFRESH : M_SCAN; // lost the claim: chain ends here
            }
        } else if (mode == M_REFRESH) {
            cw |= fw0;
            mode = M_SCAN;
        }
        return true;
    };

    while (round()) {
    }
}

// ------------------------------------------------------------ unaligned super-elements
// Super-elements whose size is a multiple of 4 but not of 16 bytes (e.g. m = 131 floats):
// their start addresses have different 16-byte phases, so the carried data cannot keep a
// fixed lane/vector mapping.  A warp walker (G = 32) loads the 16-byte vectors COVERING
// the target, keeps the carried super-element word-aligned in a per-warp shared buffer,
// and writes it back realigned: whole 16-byte vectors inside, per-word stores at the two
// partial ends.  Same claim protocol and start schedule as cycle_global_kernel.
template <int R, typename I>
__global__ void __launch_bounds__(256, 6) cycle_ua_kernel(const CycParams p) {
    constexpr unsigned FULL = 0xffffffffu;
    __shared__ uint32_t carry_all[8][R * 128];
    const int lane = threadIdx.x & 31;
    uint32_t *carry = carry_all[threadIdx.x >> 5];
    const I A = (I)p.A, nchunk = (I)p.nchunk, nwords = (I)p.nwords;

    int mode = M_FETCH;
    I word = 0;
    uint32_t cw = 0;
    int nb = 0;
    char *item = nullptr;
    I ubase = 0, k = 0, k0 = 0;
    int nw = 0;                          // 4-byte words in this chunk
    uint4 in[R];
#pragma unroll
    for (int r = 0; r < R; ++r) in[r] = make_uint4(0, 0, 0, 0);

    for (;;) {
        // ------------------------------------------------ work acquisition (warp-uniform)
        for (; mode == M_FETCH || mode == M_SCAN;) {
            if (mode == M_FETCH) {
                unsigned long long wb = 0;
                if (lane == 0) wb = atomicAdd(p.counter, 1ull);
                wb = __shfl_sync(FULL, wb, 0);
                if (wb >= p.nfetch) { mode = M_DONE; break; }
                uint64_t mine = wb >> p.segsh;
                const uint32_t seg = (uint32_t)(wb & ((1u << p.segsh) - 1u));
                if (p.wstride != 1) {
                    uint64_t q, r;
                    fdivmod(mine * p.wstride, p.divNwords.d64, q, r);
                    mine = r;
                }
                word = (I)mine;
                const uint32_t F = 32u >> p.segsh;
                const uint32_t segmask = (F == 32) ? 0xffffffffu : (((1u << F) - 1u) << (seg * F));
                cw = ld_relaxed_u32(p.flags + word) | ~segmask;
                cw = __shfl_sync(FULL, cw, 0);
                nb = 0;
                mode = M_SCAN;
            }
            uint32_t valid = 0xffffffffu;
            if (word == nwords - 1 && (p.units & 31)) valid = (1u << (p.units & 31)) - 1u;
            const uint32_t cand = ~cw & valid & (nb >= 32 ? 0u : (0xffffffffu << nb));
            if (!cand) { mode = M_FETCH; continue; }
            const int b = __ffs(cand) - 1;
            nb = b + 1;
            const I u = word * 32 + (I)b;
            I tk = u, ch = 0;
            if (p.nchunk > 1) fdivmod_t(u, p.divNchunk.d32, p.divNchunk.d64, tk, ch);
            I T, kk, q, r;
            fdivmod_t(tk, p.divAB.d32, p.divAB.d64, T, kk);
            fdivmod_t(kk, p.divB.d32, p.divB.d64, q, r);
            if (r * A + q == kk) continue;              // fixed point of Eq. (1)
            I to, ti;
            fdivmod_t(T, p.divInner.d32, p.divInner.d64, to, ti);
            item = p.base + (uint64_t)to * p.ostride + (uint64_t)ti * p.istride +
                   (uint64_t)ch * p.cvec * 4;
            ubase = T * (I)p.AB * nchunk + ch;
            nw = (int)((ch == nchunk - 1) ? (p.nvec - (uint64_t)ch * p.cvec) : p.cvec);
            k = k0 = kk;
            mode = M_START;
            break;
        }
        if (mode == M_DONE) break;

        // --------------------------------------------------------------- memory round
        I tgt = k;
        if (mode == M_CHAIN) {
            I q, r;
            fdivmod_t(k, p.divB.d32, p.divB.d64, q, r);
            tgt = r * A + q;
        }
        const bool back_home = (mode == M_CHAIN) && (tgt == k0);
        const I ut = ubase + tgt * nchunk;
        const uint32_t bit = 1u << ((uint32_t)ut & 31);
        uint32_t *fwp = p.flags + (ut >> 5);
        const uintptr_t a = (uintptr_t)(item + (uint64_t)tgt * p.S);
        const int o = (int)((a & 15) >> 2);             // word phase of the target
        const char *vb = (const char *)(a - (uintptr_t)(o * 4));
        const int nvv = (o + nw + 3) >> 2;              // covering 16-byte vectors
        if ((mode == M_START || mode == M_CHAIN) && !back_home) {
            const bool acq = (mode == M_START) && p.fence;   // see cycle_global_kernel
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int j = lane + 32 * r;
                if (j < nvv) in[r] = acq ? ld_acq<16>(vb + (size_t)j * 16) : ld_cg<16>(vb + (size_t)j * 16);
            }
        }
        uint32_t old = 0;
        if (mode == M_CHAIN && lane == 0)
            old = p.fence ? atom_or_acq_u32(fwp, bit) : atom_or_u32(fwp, bit);
        uint32_t fw = 0;
        if (mode == M_START) {
            fw = ld_relaxed_u32(fwp);
        } else if (mode == M_REFRESH) {
            fw = ld_relaxed_u32(p.flags + word);
        }
        old = __shfl_sync(FULL, old, 0);
        __syncwarp();
        const bool start_lost = __any_sync(FULL, (fw & bit) != 0);

        auto carry_from_in = [&]() {            // carry[t] = word t of the loaded target
            __syncwarp();
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int j = lane + 32 * r;
                if (j < nvv) {
                    const uint32_t w4[4] = {in[r].x, in[r].y, in[r].z, in[r].w};
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int t = 4 * j + i - o;
                        if (t >= 0 && t < nw) carry[t] = w4[i];
                    }
                }
            }
            __syncwarp();
        };

        if (mode == M_START) {
            cw |= fw;
            if (start_lost) {
                mode = M_SCAN;
            } else {
                carry_from_in();
                mode = M_CHAIN;
            }
        } else if (mode == M_CHAIN) {
            if (!(old & bit)) {
                // store the carried words into the target, realigned to its phase o
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const int j = lane + 32 * r;
                    if (j < nvv) {
                        char *dst = (char *)vb + (size_t)j * 16;
                        const int t0 = 4 * j - o;
                        if (t0 >= 0 && t0 + 3 < nw) {
                            st_cg<16>(dst, make_uint4(carry[t0], carry[t0 + 1], carry[t0 + 2], carry[t0 + 3]));
                        } else {
#pragma unroll
                            for (int i = 0; i < 4; ++i) {
                                const int t = t0 + i;
                                if (t >= 0 && t < nw) st_cg<4>(dst + 4 * i, carry[t]);
                            }
                        }
                    }
                }
                if (back_home) {
                    __syncwarp();
                    mode = M_SCAN;
                } else {
                    carry_from_in();            // the displaced content is carried on
                    k = tgt;
                }
            } else {
                mode = p.refresh ? M_REFRESH : M_SCAN;
            }
        } else if (mode == M_REFRESH) {
            cw |= fw;
            mode = M_SCAN;
        }
    }
}

// ------------------------------------------------------------------------- host side
namespace {

struct Choice { int W, G, R; uint64_t cvec, nchunk; bool ua; };

int pick_vec_bytes(const StageDesc &d) {
    const uint64_t S = (uint64_t)d.s * d.eb;
    const uint64_t inner_bytes = (uint64_t)d.A * d.B * S;
    uint64_t g = (uint64_t)(uintptr_t)d.base | S | inner_bytes;
    if (d.outer > 1) g |= (uint64_t)d.ostride;
    for (int W = 16; W > 1; W >>= 1)
        if ((g & (uint64_t)(W - 1)) == 0) return W;
    return 1;
}

Choice choose(const StageDesc &d) {
    Choice c;
    const uint64_t S = (uint64_t)d.s * d.eb;
    c.W = pick_vec_bytes(d);
    c.ua = false;
    if ((c.W == 4 || c.W == 8) && S >= 64 && env_int("IPT_CYC_UA", 1)) {
        // 4-byte granular super-elements with mixed 16-byte phases: realigning walker
        c.ua = true;
        c.W = 4;
        const uint64_t nw = S / 4;
        c.nchunk = (nw + 508) / 509;
        c.cvec = (nw + c.nchunk - 1) / c.nchunk;              // words per chunk
        c.G = 32;
        c.R = c.cvec <= 125 ? 1 : (c.cvec <= 253 ? 2 : 4);
        return c;
    }
    const uint64_t nvec = S / c.W;
    const long max_chunk = env_int("IPT_CYC_MAXVEC", 128);   // vectors per walker chunk
    uint64_t cap = (uint64_t)(max_chunk < 1 ? 1 : max_chunk);
    c.nchunk = (nvec + cap - 1) / cap;
    c.cvec = (nvec + c.nchunk - 1) / c.nchunk;                // balanced chunks
    // Chunks of super-elements larger than one walker (16-byte vectors): greedy full 2 KB
    // chunks and a partial last one (default, IPT_CYC_CHUNK256=2) run 5-10 % faster than
    // balanced chunks (0; e.g. 6400 B as 4 x 1600 B: 5.36 vs 5.67 TB/s, 5120 B: 5.43 vs
    // 5.95) -- chunk boundaries on 2 KB multiples; (1) balanced on 256-byte multiples.
    const long ck = env_int("IPT_CYC_CHUNK256", 2);
    if (c.W == 16 && c.nchunk > 1 && ck == 2) {
        c.cvec = cap;
    } else if (c.W == 16 && c.nchunk > 1 && cap >= 16 && ck == 1) {
        c.cvec = (c.cvec + 15) / 16 * 16;
        if (c.cvec > cap) c.cvec = cap;
        c.nchunk = (nvec + c.cvec - 1) / c.cvec;
    }
    // walker shape: G lanes x R vectors >= cvec
    const int Gs16[] = {1, 2, 4, 8, 16, 32};
    const int Gs[] = {1, 4, 32};
    c.G = 32; c.R = 4;
    long fg = env_int("IPT_CYC_G", 0), fr = env_int("IPT_CYC_R", 0);
    bool done = false;
    if (fg > 0 && fr > 0 && (uint64_t)(fg * fr) >= c.cvec) {
        c.G = (int)fg; c.R = (int)fr; done = true;
    }
    if (!done) {
        if (c.cvec <= 32) {
            c.R = 1;
            if (c.W == 16) { for (int g : Gs16) if ((uint64_t)g >= c.cvec) { c.G = g; break; } }
            else if (c.W >= 4) { for (int g : Gs) if ((uint64_t)g >= c.cvec) { c.G = g; break; } }
            else c.G = (c.cvec <= 1) ? 1 : 32;
        } else if (c.cvec <= 64) {
            c.G = 32; c.R = 2;
            if (c.W < 4) c.R = 4;
        } else {
            c.G = 32; c.R = 4;
        }
    }
    return c;
}

template <int W, int G, int R, typename I>
cudaError_t launch_t(const CycParams &p, cudaStream_t st, int device) {
    auto kern = cycle_global_kernel<W, G, R, I>;
    static std::mutex mu;
    static std::map<int, int> occ_cache;
    int per_sm = 0;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = occ_cache.find(device);
        if (it == occ_cache.end()) {
            cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0);
            if (e != cudaSuccess) return e;
            occ_cache[device] = per_sm;
        } else {
            per_sm = it->second;
        }
    }
    DevProps dp = dev_props(device);
    long occ_cap = env_int("IPT_CYC_BLOCKS_PER_SM", 0);
    if (occ_cap > 0 && occ_cap < per_sm) per_sm = (int)occ_cap;
    uint64_t grid = (uint64_t)dp.sms * (uint64_t)(per_sm > 0 ? per_sm : 1);
    const uint64_t groups_per_block = 8ull * (32 / G);
    const uint64_t need = (p.nfetch + groups_per_block - 1) / groups_per_block;
    if (need < grid) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, 256, 0, st>>>(p);
    note_launch();
    return cudaGetLastError();
}

template <int R, typename I>
cudaError_t launch_ua(const CycParams &p, cudaStream_t st, int device) {
    auto kern = cycle_ua_kernel<R, I>;
    static std::mutex mu;
    static std::map<int, int> occ_cache;
    int per_sm = 0;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = occ_cache.find(device);
        if (it == occ_cache.end()) {
            cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0);
            if (e != cudaSuccess) return e;
            occ_cache[device] = per_sm;
        } else {
            per_sm = it->second;
        }
    }
    DevProps dp = dev_props(device);
    uint64_t grid = (uint64_t)dp.sms * (uint64_t)(per_sm > 0 ? per_sm : 1);
    const uint64_t need = (p.nfetch + 7) / 8;
    if (need < grid) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, 256, 0, st>>>(p);
    note_launch();
    return cudaGetLastError();
}

typedef cudaError_t (*LaunchFn)(const CycParams &, cudaStream_t, int);

template <int W, int G, int R>
LaunchFn pick_idx(bool idx32) {
    return idx32 ? &launch_t<W, G, R, uint32_t> : &launch_t<W, G, R, uint64_t>;
}

#define IPT_CASE(W_, G_, R_) \
    if (c.W == W_ && c.G == G_ && c.R == R_) return pick_idx<W_, G_, R_>(idx32);

LaunchFn lookup(const Choice &c, bool idx32) {
    if (c.ua) {
        if (c.R == 1) return idx32 ? &launch_ua<1, uint32_t> : &launch_ua<1, uint64_t>;
        if (c.R == 2) return idx32 ? &launch_ua<2, uint32_t> : &launch_ua<2, uint64_t>;
        return idx32 ? &launch_ua<4, uint32_t> : &launch_ua<4, uint64_t>;
    }
    // W = 16: every group width
    IPT_CASE(16, 1, 1) IPT_CASE(16, 2, 1) IPT_CASE(16, 4, 1) IPT_CASE(16, 8, 1)
    IPT_CASE(16, 16, 1) IPT_CASE(16, 32, 1) IPT_CASE(16, 32, 2) IPT_CASE(16, 32, 4)
    IPT_CASE(16, 16, 2) IPT_CASE(16, 16, 4) IPT_CASE(16, 8, 2) IPT_CASE(16, 8, 4)
    IPT_CASE(16, 4, 2) IPT_CASE(16, 4, 4)
    // W = 8 / 4
    IPT_CASE(8, 1, 1) IPT_CASE(8, 4, 1) IPT_CASE(8, 32, 1) IPT_CASE(8, 32, 2) IPT_CASE(8, 32, 4)
    IPT_CASE(4, 1, 1) IPT_CASE(4, 4, 1) IPT_CASE(4, 32, 1) IPT_CASE(4, 32, 2) IPT_CASE(4, 32, 4)
    // W = 2 / 1 (1- and 2-byte elements with odd super-elements)
    IPT_CASE(2, 1, 1) IPT_CASE(2, 32, 1) IPT_CASE(2, 32, 4)
    IPT_CASE(1, 1, 1) IPT_CASE(1, 32, 1) IPT_CASE(1, 32, 4)
    return nullptr;
}
#undef IPT_CASE

Div2 make_div2(uint64_t d) {
    Div2 x;
    x.d64 = make_fastdiv(d);
    x.d32 = make_fastdiv32((uint32_t)(d < (1ull << 32) ? d : 1));
    return x;
}

}  // namespace

size_t cycle_ws_bytes(const StageDesc &d) {
    Choice c = choose(d);
    const uint64_t units = (uint64_t)d.outer * d.inner * d.A * d.B * c.nchunk;
    const uint64_t nwords = (units + 31) / 32;
    return 256 + nwords * 4;
}

bool cycle_seg_would_launch(const StageDesc &d, int device);   // cycle_seg.cu
const char *cycle_seg_name(const StageDesc &d);

const char *cycle_kernel_name(const StageDesc &d, int device) {
    if (cycle_prefer_seg(d.A * d.B, d.outer * d.inner, d.s * d.eb, device) && cycle_seg_would_launch(d, device))
        return cycle_seg_name(d);
    return choose(d).ua ? "cycle_ua" : "cycle_global";
}

cudaError_t launch_cycle_global(const StageDesc &d, void *ws, cudaStream_t st, int device) {
    // Segmented cycle following (cycle_seg.cu): precomputed equal-length segments, no flags,
    // where the planner's model predicts it faster (IPT_CYC_SEG: 0 never, 2 always).
    if (cycle_prefer_seg(d.A * d.B, d.outer * d.inner, d.s * d.eb, device)) {
        cudaError_t e = launch_cycle_seg(d, ws, st, device);
        if (e != cudaErrorNotSupported) return e;
        cudaGetLastError();
    }
    Choice c = choose(d);
    const uint64_t units = (uint64_t)d.outer * d.inner * d.A * d.B * c.nchunk;
    // 32-bit indices when every unit index (and word * 32 + 31) fits
    const bool idx32 = units + 64 < (1ull << 32) && !env_int("IPT_CYC_IDX64", 0);
    LaunchFn fn = lookup(c, idx32);
    if (!fn) {  // unsupported forced shape: fall back to the widest generic walker
        c.G = 32; c.R = 4;
        if ((uint64_t)c.G * c.R < c.cvec) return cudaErrorInvalidValue;
        fn = lookup(c, idx32);
        if (!fn) return cudaErrorInvalidValue;
    }
    CycParams p;
    p.base = d.base;
    p.S = (uint64_t)d.s * d.eb;
    p.A = (uint64_t)d.A;
    p.AB = (uint64_t)d.A * d.B;
    p.istride = p.AB * p.S;
    p.ostride = (uint64_t)d.ostride;
    p.nvec = p.S / c.W;
    p.nchunk = c.nchunk;
    p.cvec = c.cvec;
    p.units = units;
    p.nwords = (p.units + 31) / 32;
    {
        // Small stages: hand out segments of a flag word so that every resident walker
        // gets a start (parallelism = fetches, not words).
        const DevProps dp = dev_props(device);
        const uint64_t walkers = (uint64_t)dp.sms * 64 * (c.ua ? 1 : (32 / c.G));
        long forced = env_int("IPT_CYC_SEGSH", -1);
        uint32_t sh = 0;
        // target fetches = walkers / 2 (measured, tools/cyc_knobs.py: 1-2x starve the fetch
        // counter -- one contended atomic per fetch -- on C1-sized stages: -20..-45 %)
        const uint64_t target = walkers * (uint64_t)env_int("IPT_CYC_SEGF", 50) / 100;
        while (sh < 5 && (p.nwords << sh) < target) ++sh;
        if (forced >= 0 && forced <= 5) sh = (uint32_t)forced;
        p.segsh = sh;
        p.nfetch = p.nwords << sh;
    }
    p.wstride = 1;
    {
        const uint64_t batch = (uint64_t)d.outer * d.inner;
        const long mode = env_int("IPT_CYC_SCRAMBLE", 2);
        auto gcd = [](uint64_t a, uint64_t b) { while (b) { uint64_t t = a % b; a = b; b = t; } return a; };
        if (mode && batch > 1 && p.nwords > batch && p.nwords < (1ull << 32)) {
            uint64_t s = (p.nwords + batch - 1) / batch;
            while (gcd(s, p.nwords) != 1) ++s;
            p.wstride = s;
        } else if (mode == 2 && p.nwords > 64 && p.nwords < (1ull << 32)) {
            // single matrix: golden-ratio stride spreads concurrently started chains
            uint64_t s = (uint64_t)(0.6180339887 * (double)p.nwords);
            while (gcd(s, p.nwords) != 1) ++s;
            p.wstride = s;
        }
    }
    p.divNwords = make_div2(p.nwords ? p.nwords : 1);
    p.divB = make_div2((uint64_t)d.B);
    p.divAB = make_div2(p.AB);
    p.divInner = make_div2((uint64_t)d.inner);
    p.divNchunk = make_div2(c.nchunk);
    p.counter = (unsigned long long *)ws;
    p.flags = (uint32_t *)((char *)ws + 256);
    p.refresh = (int)env_int("IPT_CYC_REFRESH", 1);
    p.fence = (int)env_int("IPT_CYC_FENCE", 1);
    p.zero = 0;
    p.fastloop = (int)env_int("IPT_CYC_FASTLOOP", 1);
    p.sal = (int)env_int("IPT_CYC_SAL", 0);
    p.stats = env_int("IPT_CYC_STATS", 0) ? (unsigned long long *)ws + 8 : nullptr;
    cudaError_t e = cudaMemsetAsync(ws, 0, 256 + p.nwords * 4, st);
    if (e != cudaSuccess) return e;
    return fn(p, st, device);
}

}  // namespace ipt
