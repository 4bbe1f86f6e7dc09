/*
 * ipt_oracle.c -- CPU ORACLE for in-place transposition (Sung et al., PPoPP'14).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_ppopp_sunggggh14_b200/, libipt.so) never links, loads or calls it,
 * and it shares no code, header, table or constant with the CUDA path.
 *
 * Plain, single-threaded, obviously-correct C.  Every function follows a passage of
 * /root/reference/PAPER.md ("P:<line>"):
 *
 *   - Eq. (1), P:84-89 (Sec. 3): in a row-major M x N array the element at offset k
 *     moves to k' = k*M mod (MN-1) for 0 <= k < MN-1, and k' = MN-1 for k = MN-1.
 *     Computed literally, with 128-bit intermediates so k*M cannot overflow.
 *   - P:107 (Sec. 3) and P:113 (Sec. 4): the permutation is a set of cycles ("chains of
 *     shifting"); the content of the destination is saved before it is overwritten and
 *     carried to the next location.
 *   - P:70 (Sec. 2.1): Berman's bit table -- one "visited" bit per element -- marks the
 *     cycles that have been shifted.
 *   - P:140, P:156-158 (Sec. 4.1/4.2): the elementary tiled transpositions.  Every one of
 *     them swaps two adjacent dimensions of a row-major array, so all are instances of
 *     one operation:
 *        P(batch, A, B, s):  batch x [A x B x s]  ->  batch x [B x A x s]
 *     i.e. `batch` independent transpositions of an A x B matrix whose elements are
 *     "super-elements" of s consecutive elements ("every m-element tile is treated
 *     as a super-element that is then shifted").  Eq. (1) is applied to super-element
 *     offsets with (M, N) := (A, B).
 *        100!  (stage 1)  = P(1, M, N', n)
 *        0010! (stage 2)  = P(N'M', m, n, 1)
 *        0100! (stage 3)  = P(N', M', n, m)
 *        1000! (4-stage)  = P(1, M', N', m*n)  (on the 4-D view of that stage)
 *
 * Values are moved as raw bytes (memcpy); there is no floating-point operation anywhere,
 * so NaN payloads and signed zeros are preserved bit for bit.
 *
 * Return codes: 0 = ok, -1 = invalid argument, -2 = out of memory.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef unsigned __int128 u128;

/* Eq. (1), applied to an A x B array: destination of offset k (0 <= k < A*B). */
int64_t oracle_eq1_dest(int64_t k, int64_t A, int64_t B)
{
    int64_t calM = A * B - 1;                 /* the paper's script-M = M*N - 1 */
    if (k == calM) return calM;               /* second case of Eq. (1)          */
    return (int64_t)(((u128)(uint64_t)k * (u128)(uint64_t)A) % (u128)(uint64_t)calM);
}

/* P(batch, A, B, s) in place by sequential cycle following with a visited bit table
 * (P:70 Berman, P:107 chains of shifting, P:113 worked example).  Super-elements are
 * s*elem_bytes contiguous bytes; batch items are contiguous (A*B*s elements each). */
int oracle_permute_inplace(void *data, int64_t batch, int64_t A, int64_t B, int64_t s,
                           int elem_bytes)
{
    if (!data || batch < 0 || A < 1 || B < 1 || s < 1 || elem_bytes < 1) return -1;
    if (batch == 0 || A == 1 || B == 1) return 0;       /* 1 x B or A x 1: identity */
    const int64_t n_units = A * B;
    const size_t se = (size_t)s * (size_t)elem_bytes;   /* super-element bytes */
    unsigned char *tmp = (unsigned char *)malloc(se);
    unsigned char *sav = (unsigned char *)malloc(se);
    unsigned char *visited = (unsigned char *)malloc((size_t)((n_units + 7) / 8));
    if (!tmp || !sav || !visited) { free(tmp); free(sav); free(visited); return -2; }

    for (int64_t t = 0; t < batch; ++t) {
        unsigned char *a = (unsigned char *)data + (size_t)t * (size_t)n_units * se;
        memset(visited, 0, (size_t)((n_units + 7) / 8));
        for (int64_t start = 0; start < n_units; ++start) {
            if (visited[start >> 3] & (1u << (start & 7))) continue;
            /* carry the content of `start` around its cycle */
            memcpy(tmp, a + (size_t)start * se, se);
            int64_t cur = start;
            do {
                int64_t nx = oracle_eq1_dest(cur, A, B);
                memcpy(sav, a + (size_t)nx * se, se);   /* save destination's content */
                memcpy(a + (size_t)nx * se, tmp, se);   /* shift carried content in   */
                memcpy(tmp, sav, se);                   /* carry the saved content on */
                visited[nx >> 3] |= (unsigned char)(1u << (nx & 7));
                cur = nx;
            } while (cur != start);
        }
    }
    free(tmp); free(sav); free(visited);
    return 0;
}

/* Full in-place transpose of a row-major M x N array: the single-stage
 * algorithm, i.e. P(1, M, N, 1). */
int oracle_transpose_inplace(void *data, int64_t M, int64_t N, int elem_bytes)
{
    return oracle_permute_inplace(data, 1, M, N, 1, elem_bytes);
}

/* The paper's 3-stage algorithm, Sec. 4.2, in the paper's order:
 *   1. M x N' x n  -> N' x M x n          (100!,  P:156)
 *   2. N' x M' x m x n -> N' x M' x n x m (0010!)
 *   3. N' x M' x n x m -> N' x n x M' x m (0100!)
 * Requires M = M'm, N = N'n. */
int oracle_transpose_3stage(void *data, int64_t M, int64_t N, int64_t m, int64_t n,
                            int elem_bytes)
{
    if (m < 1 || n < 1 || M % m || N % n) return -1;
    const int64_t Mp = M / m, Np = N / n;
    int rc;
    if ((rc = oracle_permute_inplace(data, 1, M, Np, n, elem_bytes))) return rc;
    if ((rc = oracle_permute_inplace(data, Np * Mp, m, n, 1, elem_bytes))) return rc;
    return oracle_permute_inplace(data, Np, Mp, n, m, elem_bytes);
}

/* The 4-stage Gustavson/Karlsson sequence of Fig. 2 / P:142 on the 4-D view
 * M' x m x N' x n:  0100! -> 0010! -> 1000! -> 0100!. */
int oracle_transpose_4stage(void *data, int64_t M, int64_t N, int64_t m, int64_t n,
                            int elem_bytes)
{
    if (m < 1 || n < 1 || M % m || N % n) return -1;
    const int64_t Mp = M / m, Np = N / n;
    int rc;
    /* M' x m x N' x n -> M' x N' x m x n : M' instances of m x N' with super-element n */
    if ((rc = oracle_permute_inplace(data, Mp, m, Np, n, elem_bytes))) return rc;
    /* M' x N' x m x n -> M' x N' x n x m : M'N' instances of m x n */
    if ((rc = oracle_permute_inplace(data, Mp * Np, m, n, 1, elem_bytes))) return rc;
    /* M' x N' x n x m -> N' x M' x n x m : one M' x N' array of (n*m)-super-elements */
    if ((rc = oracle_permute_inplace(data, 1, Mp, Np, n * m, elem_bytes))) return rc;
    /* N' x M' x n x m -> N' x n x M' x m : N' instances of M' x n with super-element m */
    return oracle_permute_inplace(data, Np, Mp, n, m, elem_bytes);
}

/* Cycle structure of the M x N transposition (the count is Cate & Twigg's
 * theorem): number of cycles, of fixed points (length-1 cycles) and the length
 * of the longest cycle, by walking every cycle once with a visited table. */
int oracle_cycle_stats(int64_t M, int64_t N, int64_t *cycles, int64_t *fixed,
                       int64_t *longest)
{
    if (M < 1 || N < 1 || !cycles || !fixed || !longest) return -1;
    const int64_t n_units = M * N;
    unsigned char *visited = (unsigned char *)calloc((size_t)((n_units + 7) / 8), 1);
    if (!visited) return -2;
    int64_t c = 0, f = 0, L = 0;
    for (int64_t start = 0; start < n_units; ++start) {
        if (visited[start >> 3] & (1u << (start & 7))) continue;
        int64_t len = 0, cur = start;
        do {
            visited[cur >> 3] |= (unsigned char)(1u << (cur & 7));
            cur = (n_units == 1) ? cur : oracle_eq1_dest(cur, M, N);
            ++len;
        } while (cur != start);
        ++c;
        if (len == 1) ++f;
        if (len > L) L = len;
    }
    free(visited);
    *cycles = c; *fixed = f; *longest = L;
    return 0;
}

/* Writes the cycles of the M x N transposition as in P:113: each cycle listed from its
 * smallest offset (the order cycle following meets them), members in shifting order,
 * cycles separated by -1.  Returns the number of int64 written, or -1 if cap is too
 * small. */
int64_t oracle_cycles_list(int64_t M, int64_t N, int64_t *out, int64_t cap)
{
    if (M < 1 || N < 1 || !out) return -1;
    const int64_t n_units = M * N;
    unsigned char *visited = (unsigned char *)calloc((size_t)((n_units + 7) / 8), 1);
    if (!visited) return -1;
    int64_t w = 0;
    for (int64_t start = 0; start < n_units; ++start) {
        if (visited[start >> 3] & (1u << (start & 7))) continue;
        int64_t cur = start;
        do {
            if (w >= cap) { free(visited); return -1; }
            out[w++] = cur;
            visited[cur >> 3] |= (unsigned char)(1u << (cur & 7));
            cur = (n_units == 1) ? cur : oracle_eq1_dest(cur, M, N);
        } while (cur != start);
        if (w >= cap) { free(visited); return -1; }
        out[w++] = -1;
    }
    free(visited);
    return w;
}
