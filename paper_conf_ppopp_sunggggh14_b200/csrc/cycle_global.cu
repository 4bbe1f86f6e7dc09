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
//     chains in flight (Little's law); a persistent grid fills every SM.
//   * Super-elements larger than one walker's capacity are split into `nchunk` chunks
//     that follow the SAME permutation independently (moving chunk c of every
//     super-element is itself a valid permutation), each with its own flag bit.
//   * Start positions are handed out in increasing order, 32 units (one flag word) at a
//     time, from a global work counter (adjacent work-items start at adjacent
//     elements); the flag word doubles as a pre-check so claimed units are never
//     re-read.
//   * Claim protocol (P1): flag bit u = "unit u has received its final
//     value".  Chain step from cur: d = next(cur); load backup = A[d] and atomicOr(bit d)
//     concurrently; if the bit was already set the chain ends, else store carried data
//     into d and carry the backup on.  A chain start at x loads A[x] and then re-checks
//     bit x with a load whose address depends on the loaded data (so it is ordered after
//     it); if set, the start is abandoned (the claimer of x carries A[x]).
//   * Index maps use 64-bit indices and multiply-high division (no 64-bit '%').
#include "ipt_internal.h"
#include "mem_ptx.cuh"

#include <mutex>
#include <map>

namespace ipt {

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
    FastDiv divB, divAB, divInner, divNchunk;
    uint32_t *flags;
    unsigned long long *counter;
    int refresh;        // re-read the flag word after a chain ends before the next start
    uint32_t zero;      // always 0 at run time; opaque to the compiler (see dep_zero use)
    int fence;          // 1: PTX-model fences on both sides of the claim protocol
    int pf;             // chain look-ahead depth (L2 prefetch of the next targets)
    uint64_t wstride;   // start-order scramble (coprime to nwords)
    FastDiv divNwords;
};

enum : int { M_FETCH = 0, M_SCAN = 1, M_START = 2, M_CHAIN = 3, M_REFRESH = 4, M_DONE = 5 };

template <int W, int G, int R>
__global__ void __launch_bounds__(256) cycle_global_kernel(const CycParams p) {
    using V = typename VecT<W>::type;
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31;
    const int gl = lane % G;          // lane within walker group
    const int g0 = lane - gl;         // first lane of the group
    const unsigned gmask = (G == 32) ? FULL : (((1u << G) - 1u) << g0);

    int mode = M_FETCH;
    uint64_t word = 0;     // flag word (= chunk of 32 start units) being scanned
    uint32_t cw = 0;       // cached copy of that flag word
    int nb = 0;            // next bit to consider in the word
    char *item = nullptr;  // start of the current batch item (+ chunk offset)
    uint64_t ubase = 0;    // unit index of (item, k = 0, chunk)
    uint64_t k = 0, k0 = 0;
    int nv = 0;            // vectors in this chunk
    V data[R], in[R];
#pragma unroll
    for (int r = 0; r < R; ++r) { data[r] = V(); in[r] = V(); }

    for (;;) {
        // ------------------------------------------------ work acquisition (no data moved)
        for (;;) {
            const unsigned need = __ballot_sync(FULL, mode == M_FETCH && gl == 0);
            if (need) {
                const int leader = __ffs(need) - 1;
                unsigned long long wb = 0;
                if (lane == leader) wb = atomicAdd(p.counter, (unsigned long long)__popc(need));
                wb = __shfl_sync(FULL, wb, leader);
                uint64_t mine = wb + __popc(need & ((1u << g0) - 1u));
                const bool have = mine < p.nwords;
                // Start order: fetch i scans flag word (i * wstride) mod nwords.  For a
                // batch of small independent matrices wstride ~ words per matrix, so the
                // start frontier advances through all matrices at once (like one big
                // matrix) instead of bursting through one at a time, which keeps chains
                // long and PTTWAC's redundant start reads low.
                if (have && p.wstride != 1) {
                    uint64_t q, r;
                    fdivmod(mine * p.wstride, p.divNwords, q, r);
                    mine = r;
                }
                uint32_t fw = 0;
                if (mode == M_FETCH && have) fw = ld_relaxed_u32(p.flags + mine);
                fw = __shfl_sync(FULL, fw, g0);
                if (mode == M_FETCH) {
                    word = mine;
                    if (!have) {
                        mode = M_DONE;
                    } else {
                        cw = fw;
                        nb = 0;
                        mode = M_SCAN;
                    }
                }
            }
            // Scan the cached word for the next unit that still needs a start walker.
            while (mode == M_SCAN) {
                uint32_t valid = 0xffffffffu;
                if (word == p.nwords - 1 && (p.units & 31)) valid = (1u << (p.units & 31)) - 1u;
                const uint32_t cand = ~cw & valid & (nb >= 32 ? 0u : (0xffffffffu << nb));
                if (!cand) { mode = M_FETCH; break; }
                const int b = __ffs(cand) - 1;
                nb = b + 1;
                const uint64_t u = word * 32 + (uint64_t)b;
                uint64_t tk = u, ch = 0;
                if (p.nchunk > 1) fdivmod(u, p.divNchunk, tk, ch);
                uint64_t T, kk;
                fdivmod(tk, p.divAB, T, kk);
                uint64_t q, r;
                fdivmod(kk, p.divB, q, r);
                if (r * p.A + q == kk) continue;        // fixed point of Eq. (1): nothing moves
                uint64_t to, ti;
                fdivmod(T, p.divInner, to, ti);
                item = p.base + to * p.ostride + ti * p.istride + ch * p.cvec * W;
                ubase = T * p.AB * p.nchunk + ch;
                nv = (int)((ch == p.nchunk - 1) ? (p.nvec - ch * p.cvec) : p.cvec);
                k = k0 = kk;
                mode = M_START;
            }
            const unsigned pending = __ballot_sync(FULL, mode == M_FETCH || mode == M_SCAN);
            if (!pending) break;
        }
        if (!__ballot_sync(FULL, mode != M_DONE)) break;

        // --------------------------------------------------------------- memory round
        uint64_t tgt = k;
        if (mode == M_CHAIN) {
            uint64_t q, r;
            fdivmod(k, p.divB, q, r);
            tgt = r * p.A + q;                         // Eq. (1) on super-element offsets
        }
        // Cycle closed at our own start x: x must still be CLAIMED (another walker carrying
        // A[prev(x)] -- the start walker of prev(x) -- may race for it), but its backup is
        // the value this walker already delivered, so it is not re-read.
        const bool back_home = (mode == M_CHAIN) && (tgt == k0);
        const uint64_t ut = ubase + tgt * p.nchunk;    // flag index of the target unit
        const uint32_t bit = 1u << (ut & 31);
        char *addr = item + tgt * p.S;

        if ((mode == M_START || mode == M_CHAIN) && !back_home) {
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int v = gl + r * G;
                if (v < nv) in[r] = ld_cg<W>(addr + (size_t)v * W);
            }
            // Look-ahead: the chain's next positions are known from Eq. (1) alone, so the
            // lines of the next `pf` targets are prefetched into L2 now; their backup reads
            // (issued in later rounds, only by whoever claims them) then hit L2 instead of
            // paying a DRAM round trip per chain step.  No data is consumed early, so the
            // claim protocol is unchanged; a prefetch is wasted only at a chain's true end
            // (the winner of a lost claim walks the same targets).
            uint64_t la = tgt;
            for (int j = 0; j < p.pf; ++j) {
                uint64_t q, r;
                fdivmod(la, p.divB, q, r);
                la = r * p.A + q;
                if (la == k0) break;
                const uintptr_t lo = (uintptr_t)(item + la * p.S);
                const uintptr_t first = lo & ~(uintptr_t)127;
                const uintptr_t last = (lo + (uintptr_t)nv * W - 1) & ~(uintptr_t)127;
                for (uintptr_t line = first + (uintptr_t)gl * 128; line <= last; line += (uintptr_t)G * 128)
                    prefetch_l2((const void *)line);
            }
        }
        uint32_t old = 0;
        if (mode == M_CHAIN && gl == 0)
            old = p.fence ? atom_or_acq_u32(p.flags + (ut >> 5), bit)
                          : atom_or_u32(p.flags + (ut >> 5), bit);
        uint32_t fw = 0;
        if (mode == M_START) {
            if (p.fence) fence_acq_rel_gpu();
            uint32_t acc = 0;
#pragma unroll
            for (int r = 0; r < R; ++r) {
                const int v = gl + r * G;
                if (v < nv) acc |= fold(in[r]);
            }
            fw = ld_relaxed_u32(p.flags + (ut >> 5) + (acc & p.zero));
        } else if (mode == M_REFRESH) {
            fw = ld_relaxed_u32(p.flags + word);
        }

        // ------------------------------------------------------------------- resolve
        old = __shfl_sync(FULL, old, g0);
        __syncwarp();   // orders lane 0's (acquire) claim before the other lanes' stores
        const unsigned seen = __ballot_sync(FULL, mode == M_START && (fw & bit));
        const uint32_t fw0 = __shfl_sync(FULL, fw, g0);
        if (mode == M_START) {
            cw |= fw0;
            if (seen & gmask) {
                mode = M_SCAN;                         // already claimed: its claimer carries A[x]
            } else {
#pragma unroll
                for (int r = 0; r < R; ++r) data[r] = in[r];
                mode = M_CHAIN;
            }
        } else if (mode == M_CHAIN) {
            if (!(old & bit)) {
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
    }
}

// ------------------------------------------------------------------------- host side
namespace {

struct Choice { int W, G, R; uint64_t cvec, nchunk; };

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
    const uint64_t nvec = S / c.W;
    const long max_chunk = env_int("IPT_CYC_MAXVEC", 128);   // vectors per walker chunk
    uint64_t cap = (uint64_t)(max_chunk < 1 ? 1 : max_chunk);
    c.nchunk = (nvec + cap - 1) / cap;
    c.cvec = (nvec + c.nchunk - 1) / c.nchunk;                // balanced chunks
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

template <int W, int G, int R>
cudaError_t launch_t(const CycParams &p, cudaStream_t st, int device) {
    auto kern = cycle_global_kernel<W, G, R>;
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
    const uint64_t need = (p.nwords + groups_per_block - 1) / groups_per_block;
    if (need < grid) grid = need;
    if (grid < 1) grid = 1;
    kern<<<(unsigned)grid, 256, 0, st>>>(p);
    note_launch();
    return cudaGetLastError();
}

typedef cudaError_t (*LaunchFn)(const CycParams &, cudaStream_t, int);

#define IPT_CASE(W_, G_, R_) \
    if (c.W == W_ && c.G == G_ && c.R == R_) return &launch_t<W_, G_, R_>;

LaunchFn lookup(const Choice &c) {
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

}  // namespace

size_t cycle_ws_bytes(const StageDesc &d) {
    const uint64_t S = (uint64_t)d.s * d.eb;
    Choice c = choose(d);
    (void)S;
    const uint64_t units = (uint64_t)d.outer * d.inner * d.A * d.B * c.nchunk;
    const uint64_t nwords = (units + 31) / 32;
    return 256 + nwords * 4;
}

cudaError_t launch_cycle_global(const StageDesc &d, void *ws, cudaStream_t st, int device) {
    Choice c = choose(d);
    LaunchFn fn = lookup(c);
    if (!fn) {  // unsupported forced shape: fall back to the widest generic walker
        c.G = 32; c.R = 4;
        if ((uint64_t)c.G * c.R < c.cvec) return cudaErrorInvalidValue;
        fn = lookup(c);
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
    p.units = (uint64_t)d.outer * d.inner * p.AB * c.nchunk;
    p.nwords = (p.units + 31) / 32;
    p.wstride = 1;
    {
        const uint64_t batch = (uint64_t)d.outer * d.inner;
        const long mode = env_int("IPT_CYC_SCRAMBLE", 1);
        if (mode && batch > 1 && p.nwords > batch && p.nwords < (1ull << 32)) {
            uint64_t st = (p.nwords + batch - 1) / batch;
            auto gcd = [](uint64_t a, uint64_t b) { while (b) { uint64_t t = a % b; a = b; b = t; } return a; };
            while (gcd(st, p.nwords) != 1) ++st;
            p.wstride = st;
        }
    }
    p.divNwords = make_fastdiv(p.nwords ? p.nwords : 1);
    p.divB = make_fastdiv((uint64_t)d.B);
    p.divAB = make_fastdiv(p.AB);
    p.divInner = make_fastdiv((uint64_t)d.inner);
    p.divNchunk = make_fastdiv(c.nchunk);
    p.counter = (unsigned long long *)ws;
    p.flags = (uint32_t *)((char *)ws + 256);
    p.refresh = (int)env_int("IPT_CYC_REFRESH", 1);
    p.zero = 0;
    p.fence = (int)env_int("IPT_CYC_FENCE", 1);
    p.pf = (int)env_int("IPT_CYC_PF", 0);
    cudaError_t e = cudaMemsetAsync(ws, 0, 256 + p.nwords * 4, st);
    if (e != cudaSuccess) return e;
    return fn(p, st, device);
}

}  // namespace ipt
