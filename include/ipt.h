/*
 * ipt.h -- C ABI of libipt, a B200-native (sm_100a) in-place matrix transposition
 * library following Sung, Gomez-Luna, Gonzalez-Linares, Guil, Hwu, "In-Place
 * Transposition of Rectangular Matrices on Accelerators", PPoPP'14.
 *
 * Citations "P:<line>" refer to the paper text line, with the section /
 * equation it falls in.  SURVEY.md 8(b) is the contract this header implements.
 *
 * THE OPERATION (Sec. 3).  A is an M x N row-major array of elements of
 * `elem_bytes` bytes; after ipt_transpose the same storage holds A^T, the N x M
 * row-major array with A^T(j, i) = A(i, j); i.e. the byte content of offset
 * k = i*N + j moves to k' = j*M + i (Eq. (1)).  Elements are moved as raw
 * bytes (no floating-point operation; NaN payloads survive).
 *
 * THE METHOD (Sec. 4.2).  With M = M'*m and N = N'*n the transpose is
 * the composition of three elementary tiled transpositions ("stages"):
 *   stage 1  100!  : M x N' x n        -> N' x M x n
 *   stage 2  0010! : N' x M' x m x n   -> N' x M' x n x m
 *   stage 3  0100! : N' x M' x n x m   -> N' x n x M' x m
 * Every elementary transposition swaps two adjacent dimensions of a row-major array,
 * so all of them are instances of one operation:
 *   P(batch, A, B, s) : batch x [A x B x s]  ->  batch x [B x A x s]
 * ("super-elements" of s contiguous elements are shifted as a whole).
 *
 * CONVENTIONS (the paper is silent):
 *   - Ownership: the caller owns every data pointer; libipt never allocates or frees it.
 *   - Device pointers ("d_"): CUDA device memory of the current device.  Host pointers
 *     ("h_"): host memory (pinned or pageable).
 *   - Asynchrony: every device call is stream-ordered on `stream` (a cudaStream_t; NULL =
 *     legacy default stream) and returns after enqueueing.  Host calls (ipt_*_host)
 *     return after the result is back in host memory.
 *   - Validation: all arguments are checked BEFORE any launch; an error return other
 *     than IPT_ERR_CUDA means nothing was enqueued and the data is untouched.
 *   - Errors after launch return IPT_ERR_CUDA; the data is then undefined (an in-place
 *     permutation is not resumable: the flag bitmap is the only progress record).
 *   - elem_bytes in {1, 2, 4, 8, 16}; the data pointer must be aligned to elem_bytes.
 *     16-byte vector paths are selected automatically when alignment permits.
 *   - Workspace: cycle-following stages need one flag bit per moved unit plus a work
 *     counter ("only one bit per super-element is needed").  Pass a device
 *     buffer of ipt_workspace_bytes() bytes, or NULL to use an internal per-(device,
 *     stream) cache (a cached buffer that must grow is retired, never freed, so work or
 *     graphs already holding it stay valid; under stream capture a NULL workspace is a
 *     graph-owned allocation instead, see ipt_graph_create).  libipt zeroes the flags
 *     itself before every stage.  Host-delegated calls (ipt_transpose_host*) refuse
 *     stream capture (IPT_ERR_INVALID_ARG).
 *   - Thread safety: concurrent calls on distinct buffers with distinct workspaces (or
 *     distinct streams when using the internal cache) are safe.
 *   - M == 1 or N == 1 (and empty batches) are successful no-ops.
 */
#ifndef IPT_H
#define IPT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    IPT_OK = 0,
    IPT_ERR_INVALID_ARG = 1,      /* a size < 0 / < 1, NULL pointer, overflow          */
    IPT_ERR_UNSUPPORTED_ELEM = 2, /* elem_bytes not in {1,2,4,8,16}                    */
    IPT_ERR_MISALIGNED = 3,       /* data pointer / stride not aligned to elem_bytes   */
    IPT_ERR_NO_MEMORY = 4,        /* workspace too small / internal allocation failed  */
    IPT_ERR_CUDA = 5,             /* a CUDA call failed (data undefined if after launch) */
    IPT_ERR_NO_DEVICE = 6         /* device query failed (no CUDA device)              */
} ipt_status;

/* How one stage is executed. */
typedef enum {
    IPT_VAR_IDENTITY = 0,      /* stage elided: a swapped dimension is 1 */
    IPT_VAR_TILE_ONCHIP = 1,   /* whole tile staged on chip (BS, Fig. 1): one CTA, a
                                  cluster, a group of CTAs, or every SM with shared memory +
                                  tensor memory (tiles up to ~70 MB) */
    /* 2: reserved -- the paper's in-tile PTTWAC with flags in local memory (Sec. 5.1,
       P:172-198) is not built on B200: every tile that fits an on-chip flag bitmap also
       fits on chip itself; plans with variant 2 are rejected */
    IPT_VAR_CYCLE_GLOBAL = 3,  /* PTTWAC over super-elements, flag bits in global memory */
    IPT_VAR_SQUARE_SWAP = 4    /* square tiles (m == n, any size): symmetric swaps across the
                                  diagonal, cycles of length 2; with m = M = N = n the
                                  whole transposition is this single pass */
} ipt_variant;

/* A plan for the 3-stage transposition of one M x N matrix (Sec. 4.2 + Sec. 7.4). */
typedef struct {
    int64_t M, N;          /* matrix shape                                     */
    int64_t m, n;          /* tile sizes: M = Mp*m, N = Np*n            */
    int64_t Mp, Np;        /* M' and N'                                         */
    int32_t elem_bytes;
    int32_t n_stages;      /* number of non-identity stages (S in the roofline) */
    int32_t variant[3];    /* ipt_variant of stage 1, 2, 3                      */
    int32_t reserved;
    int64_t flag_bits[3];  /* flag bits used by each stage for ONE matrix       */
    uint64_t workspace_bytes; /* device workspace for ONE matrix (max over stages) */
} ipt_plan_t;

/* ---------------------------------------------------------------- planning (host) */

/* Tile-size planner (Sec. 7.4): factors M and N and picks (m, n) and a
 * variant per stage from a cost model of the B200 kernels.  Host-only, deterministic
 * for a given (M, N, elem_bytes, device properties).  device < 0 plans for a nominal
 * B200 (148 SMs, 227 KB shared memory per block) without touching the GPU. */
ipt_status ipt_plan(int64_t M, int64_t N, int elem_bytes, int device, ipt_plan_t *out);

/* Same with forced tile sizes m | M and n | N (IPT_ERR_INVALID_ARG otherwise). */
ipt_status ipt_plan_with_tiles(int64_t M, int64_t N, int64_t m, int64_t n, int elem_bytes,
                               int device, ipt_plan_t *out);

/* Measured plan choice: the cost model's best `candidates` plans (plus the best plan of
 * every other stage count) each transpose the matrix at d_ptr (M x N) and the model-best
 * N x M plan transposes it back, timed with CUDA events on `stream`; the data is
 * unchanged on return (synchronous).  The fastest plan is returned and remembered for
 * (M, N, elem_bytes, device): later ipt_plan / ipt_transpose calls use it.
 * candidates < 2 returns ipt_plan's choice without timing.  Jobs <= 256 MB time at least
 * 12 candidates; jobs smaller than L2 are timed cold (a library-owned scratch buffer of
 * twice the L2 size, allocated on first use, is overwritten before every repetition). */
ipt_status ipt_plan_autotune(void *d_ptr, int64_t M, int64_t N, int elem_bytes, int candidates,
                             void *stream, ipt_plan_t *out);

/* Same for a batch (timed with ipt_transpose_batched_plan on all `count` matrices); the
 * result is returned, not remembered (single-matrix plans may differ). */
ipt_status ipt_plan_autotune_batched(void *d_base, int64_t count, int64_t stride_bytes,
                                     int64_t M, int64_t N, int elem_bytes, int candidates,
                                     void *stream, ipt_plan_t *out);

/* Device workspace bytes for executing `plan` on a batch of `batch` matrices. */
size_t ipt_workspace_bytes(const ipt_plan_t *plan, int64_t batch);

/* ------------------------------------------------------------ full transposition */

/* A (M x N, row-major, at d_ptr) -> A^T (N x M) in the same storage. */
ipt_status ipt_transpose(void *d_ptr, int64_t M, int64_t N, int elem_bytes, void *stream);

/* Executes a given plan.  d_workspace may be NULL (internal cache); otherwise it must
 * hold ipt_workspace_bytes(plan, 1) bytes (ws_bytes). */
ipt_status ipt_transpose_plan(void *d_ptr, const ipt_plan_t *plan, void *d_workspace,
                              size_t ws_bytes, void *stream);

/* As ipt_transpose_plan, and records `events` (cudaEvent_t[4], each may be NULL) on the
 * stream: events[0] before stage 1, events[i] right after stage i (identity stages
 * record at the same point).  Used to time each stage live. */
ipt_status ipt_transpose_plan_events(void *d_ptr, const ipt_plan_t *plan, void *d_workspace,
                                     size_t ws_bytes, void *stream, void *const *events);

/* `count` independent M x N matrices, matrix t at d_base + t*stride_bytes
 * (stride_bytes >= M*N*elem_bytes, multiple of elem_bytes).  The batch is folded into
 * each stage (the instances are independent), so each stage is one launch. */
ipt_status ipt_transpose_batched(void *d_base, int64_t count, int64_t stride_bytes,
                                 int64_t M, int64_t N, int elem_bytes, void *stream);

ipt_status ipt_transpose_batched_plan(void *d_base, int64_t count, int64_t stride_bytes,
                                      const ipt_plan_t *plan, void *d_workspace,
                                      size_t ws_bytes, void *stream);

/* As ipt_transpose_batched_plan, recording `events` (cudaEvent_t[4], each may be NULL)
 * around the stages as ipt_transpose_plan_events does. */
ipt_status ipt_transpose_batched_plan_events(void *d_base, int64_t count, int64_t stride_bytes,
                                             const ipt_plan_t *plan, void *d_workspace,
                                             size_t ws_bytes, void *stream,
                                             void *const *events);

/* The paper's 4-stage Gustavson/Karlsson baseline (Fig. 2): 0100!, 0010!, 1000!,
 * 0100! on the 4-D view M' x m x N' x n, with the same kernels.  m | M, n | N, or 0 to
 * take the 3-stage planner's tiles.  Kept to reproduce the paper's 3-stage vs 4-stage
 * comparison (Table 2); same conventions as ipt_transpose_plan. */
ipt_status ipt_transpose_4stage(void *d_ptr, int64_t M, int64_t N, int64_t m, int64_t n,
                                int elem_bytes, void *d_workspace, size_t ws_bytes,
                                void *stream);

/* ----------------------------------------------- host-delegated transposition (Sec. 6) */

/* In-place transposition of a HOST array executed on the GPU (Fig. 4/5):
 * host->device copy, stage 1 on `stream`, then stages 2-3 and the device->host copy split
 * into `queues` groups of output panels on separate streams so that transfers overlap the
 * remaining stages (Fig. 5b; queues = 1 is the synchronous scheme of Fig. 5a).  h_ptr is
 * read and overwritten with A^T (N x M); pinned host memory is required for overlap.
 * d_buffer (device, may be NULL = internal cache) must hold at least M*N*elem_bytes plus
 * the flag workspace (IPT_ERR_NO_MEMORY otherwise).  Returns after the result is in
 * host memory. */
ipt_status ipt_transpose_host(void *h_ptr, int64_t M, int64_t N, int elem_bytes, int queues,
                              void *d_buffer, size_t d_buffer_bytes, void *stream);

/* Asynchronous form: everything is enqueued and ordered on `stream` (completion of the
 * D2H of every panel is joined back onto `stream`); returns after enqueueing.  The host
 * buffer and the device buffer (internal cache: one per (device, stream)) must not be
 * reused until the stream has reached this point.  Calls on different streams overlap,
 * e.g. the H2D of one matrix with the D2H of the previous one (both PCIe directions). */
ipt_status ipt_transpose_host_async(void *h_ptr, int64_t M, int64_t N, int elem_bytes,
                                    int queues, void *d_buffer, size_t d_buffer_bytes,
                                    void *stream);

/* Host-delegated transposition of `count` host matrices (h_ptrs[i]: Ms[i] x Ns[i],
 * elem_bytes each; pinned memory for overlap) as a copy/compute pipeline across matrices
 * (Sec. 6's overlap applied between matrices): the H2D of matrix i+1 and the D2H of matrix
 * i-1 overlap the stages of matrix i, with two device slots, one copy-in, one compute and
 * one copy-out stream (internal, per caller stream).  Every h_ptrs[i] is overwritten with
 * its transpose.  d_buffer (may be NULL = internal cache) must hold 2 slots of the largest
 * matrix (256-byte aligned) plus the stage workspace (IPT_ERR_NO_MEMORY otherwise).
 * Asynchronous: ordered after prior work on `stream`, and `stream` continues after the
 * last copy-out; host buffers must not be touched before that. */
ipt_status ipt_transpose_host_pipeline(void *const *h_ptrs, const int64_t *Ms, const int64_t *Ns,
                                       int count, int elem_bytes, void *d_buffer,
                                       size_t d_buffer_bytes, void *stream);

/* ------------------------------------------------------------------- CUDA graphs */

/* Capture the launches of `plan` applied to `count` matrices at d_base (stride_bytes apart;
 * ignored for count == 1) into an executable CUDA graph; *out receives an opaque handle.
 * Replaying it (ipt_graph_launch) transposes those matrices in place with one
 * cudaGraphLaunch -- no per-call planning, validation or kernel-launch overhead.  The graph
 * is bound to the pointers.  Workspace: the caller's d_workspace (>= ipt_workspace_bytes;
 * then replays must not overlap each other or other calls using it), or NULL = a buffer
 * owned by the graph (allocated here, freed by ipt_graph_destroy), so replays never share
 * flags or counters with direct calls or other graphs (replays of ONE graph must be
 * stream-ordered with each other).  A libipt call captured by the caller (e.g.
 * torch.cuda.graph) with a NULL workspace instead allocates and frees its flags inside the
 * captured sequence (memory allocation nodes; costlier per replay).  Captured
 * launches never use the library's per-stream self-resetting counters (they zero their
 * counters with memset nodes).  Segment lists of segmented cycle stages are used only if a
 * direct call built them already (else the flag kernel is captured): run the plan once
 * before capturing to get identical kernels.  ipt_graph_destroy frees everything the
 * handle owns (the caller synchronises first).  Note that an M x N graph replayed twice
 * applies the M x N transposition twice; pair it with an N x M graph. */
ipt_status ipt_graph_create(void *d_base, int64_t count, int64_t stride_bytes, const ipt_plan_t *plan,
                            void *d_workspace, size_t ws_bytes, void **out);
ipt_status ipt_graph_launch(void *graph, void *stream);
ipt_status ipt_graph_destroy(void *graph);

/* ------------------------------------------------ elementary transpositions */

/* Device workspace bytes for P(batch, A, B, s) with elem_bytes elements (for s == 1 it
 * also covers the on-chip tile kernels' group counters, 8 KB). */
size_t ipt_stage_workspace_bytes(int64_t batch, int64_t A, int64_t B, int64_t s,
                                 int elem_bytes);

/* 100! (SoA -> ASTA, Sec. 5.2): batch x [A x B x s] -> batch x [B x A x s] by
 * cycle following of s-element super-elements with one global flag bit each (PTTWAC);
 * small stages of 16-byte-multiple super-elements instead follow equal-length cycle
 * segments precomputed on the host on the first call for a shape (cached; the first
 * call then synchronises with the device once), with no flags. */
ipt_status ipt_100(void *d_ptr, int64_t batch, int64_t A, int64_t B, int64_t s,
                   int elem_bytes, void *d_workspace, size_t ws_bytes, void *stream);

/* 010! (AoS -> ASTA, Sec. 5.1): batch x [A x B] -> batch x [B x A] (tile-local
 * transposes; on-chip when a tile fits the shared memory of one CTA, a cluster or a
 * co-resident group of CTAs (up to ~16 MB of 16-byte-vectorisable tiles), square tiles
 * (A == B, any size) by symmetric block-pair swaps, else cycle following).  A
 * given workspace must hold ipt_stage_workspace_bytes(batch, A, B, 1). */
ipt_status ipt_010(void *d_ptr, int64_t batch, int64_t A, int64_t B, int elem_bytes,
                   void *d_workspace, size_t ws_bytes, void *stream);

/* 0010! on a 4-D array d0 x d1 x d2 x d3 -> d0 x d1 x d3 x d2 (= ipt_010(d0*d1, d2, d3)). */
ipt_status ipt_0010(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3,
                    int elem_bytes, void *d_workspace, size_t ws_bytes, void *stream);

/* 0100! on a 4-D array d0 x d1 x d2 x d3 -> d0 x d2 x d1 x d3 (= ipt_100(d0, d1, d2, d3)). */
ipt_status ipt_0100(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3,
                    int elem_bytes, void *d_workspace, size_t ws_bytes, void *stream);

/* 1000! on a 4-D array d0 x d1 x d2 x d3 -> d1 x d0 x d2 x d3 (= ipt_100(1, d0, d1, d2*d3));
 * the third stage of the 4-stage Gustavson/Karlsson scheme. */
ipt_status ipt_1000(void *d_ptr, int64_t d0, int64_t d1, int64_t d2, int64_t d3,
                    int elem_bytes, void *d_workspace, size_t ws_bytes, void *stream);

/* ------------------------------------ layout marshaling (Sung et al.'s DL system) */
/* AoS: M structures of N fields (row-major M x N).  SoA: N x M.  ASTA (Array of Structures
 * of Tiled Arrays) with tiles of m structures (m | M): M/m x N x m.  AoS -> ASTA is 010!
 * on (M/m) x m x N; SoA -> ASTA is 100! on N x (M/m) x m.  The *_to_aos / *_to_soa
 * calls are the inverse transformations.  Same conventions as ipt_010 / ipt_100. */
ipt_status ipt_aos_to_asta(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream);
ipt_status ipt_asta_to_aos(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream);
ipt_status ipt_soa_to_asta(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream);
ipt_status ipt_asta_to_soa(void *d_ptr, int64_t M, int64_t N, int64_t m, int elem_bytes,
                           void *d_workspace, size_t ws_bytes, void *stream);

/* ------------------------------------------------------------------- diagnostics */

const char *ipt_status_string(ipt_status s);

/* Number of libipt kernels launched by this process so far (all devices). */
uint64_t ipt_kernel_launch_count(void);

/* Description of the CUDA error behind the calling thread's last IPT_ERR_CUDA. */
const char *ipt_last_cuda_error(void);

/* Library version string. */
const char *ipt_version(void);

#ifdef __cplusplus
}
#endif

#endif /* IPT_H */
