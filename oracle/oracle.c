/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.  The plain CPU definition of the TTLG
 * tensor transposition that the CUDA path is checked against.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code, header, table or helper with
 * paper_conf_ipps_veduradasskhpkn18_b200/ (the product), and the product never
 * calls it.
 *
 * What it computes (§I, Eq. 1):
 *     B[rho(i0, i1, ..., i_{d-1})] <- A[i0, i1, ..., i_{d-1}]
 * written as "the d-nested loop that reads each element from the input tensor
 * and writes it to the output tensor element corresponding to the permuted
 * indexing".
 *
 * Conventions (readings R1, R2):
 *   - extents[0] is the fastest-varying index (MATLAB/Fortran notation,
 *     PAPER.md L284-286 footnote 1);
 *   - perm[i] = j means output dimension i is input dimension j
 *     (§VI); so B has extents m[i] = extents[perm[i]].
 *
 * Elements are moved as uint32_t / uint64_t bit patterns, never through
 * floating-point registers, so NaN payloads, -0.0, subnormals and inf are
 * preserved (reading R3: a transposition does no arithmetic, so the
 * result is unique bit for bit).
 *
 * Pins (tests/test_oracle.py): identity, inverse, composition, the 2-D matrix
 * transpose of PAPER.md L43-48, brute-force dict enumeration on tiny shapes,
 * exactly-once under index encoding, NumPy's transpose, hand-derived tiny
 * vectors, and the independently computed digests of SURVEY.md §8(c).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_MAX_RANK 15

typedef struct {
    int elem_bytes, rank;
    int64_t n[ORACLE_MAX_RANK];     /* input extents, n[0] fastest            */
    int32_t perm[ORACLE_MAX_RANK];  /* output dim i = input dim perm[i]       */
    int64_t sA[ORACLE_MAX_RANK];    /* input strides                          */
    int64_t sB[ORACLE_MAX_RANK];    /* output strides (of output dim i)       */
    const void *A;
    void *B;
    int64_t lo, hi;                 /* range of the outermost input index     */
} job_t;

/* Step 1 of SURVEY §8(c): strides.  sA[0]=1, sA[k]=sA[k-1]*n[k-1];
 * m[i]=n[perm[i]]; sB[0]=1, sB[i]=sB[i-1]*m[i-1]. */
static int setup(job_t *j, int elem_bytes, int rank, const int64_t *extents,
                 const int32_t *perm) {
    int seen[ORACLE_MAX_RANK] = {0};
    if (rank < 1 || rank > ORACLE_MAX_RANK) return 1;
    if (elem_bytes != 4 && elem_bytes != 8) return 1;
    j->elem_bytes = elem_bytes;
    j->rank = rank;
    for (int k = 0; k < rank; k++) {
        if (extents[k] < 1) return 1;
        if (perm[k] < 0 || perm[k] >= rank || seen[perm[k]]) return 1;
        seen[perm[k]] = 1;
        j->n[k] = extents[k];
        j->perm[k] = perm[k];
    }
    j->sA[0] = 1;
    for (int k = 1; k < rank; k++) j->sA[k] = j->sA[k - 1] * j->n[k - 1];
    j->sB[0] = 1;
    for (int i = 1; i < rank; i++) j->sB[i] = j->sB[i - 1] * j->n[j->perm[i - 1]];
    return 0;
}

/* Step 2-3: walk every input multi-index with an odometer (i0 fastest),
 * lin_A = sum_k i_k sA[k], lin_B = sum_i i_{perm[i]} sB[i]; B[lin_B] = A[lin_A]. */
static void *run(void *arg) {
    job_t *j = (job_t *)arg;
    const int d = j->rank;
    int64_t idx[ORACLE_MAX_RANK];
    if (j->lo >= j->hi) return NULL;
    for (int k = 0; k < d; k++) idx[k] = 0;
    idx[d - 1] = j->lo;
    for (;;) {
        int64_t linA = 0, linB = 0;
        for (int k = 0; k < d; k++) linA += idx[k] * j->sA[k];
        for (int i = 0; i < d; i++) linB += idx[j->perm[i]] * j->sB[i];
        if (j->elem_bytes == 8)
            ((uint64_t *)j->B)[linB] = ((const uint64_t *)j->A)[linA];
        else
            ((uint32_t *)j->B)[linB] = ((const uint32_t *)j->A)[linA];
        /* odometer increment, i0 fastest */
        int k = 0;
        while (k < d) {
            idx[k]++;
            if (k == d - 1) {
                if (idx[k] < j->hi) break;
                return NULL;
            }
            if (idx[k] < j->n[k]) break;
            idx[k] = 0;
            k++;
        }
    }
}

/* Out-of-place transposition, B = T(A).  Returns 0 on success, 1 on bad args.
 * nthreads > 1 splits the outermost input index across POSIX threads (the
 * only parallelism; no blocking, no reordering of the definition). */
int oracle_transpose(int elem_bytes, int rank, const int64_t *extents,
                     const int32_t *perm, const void *A, void *B, int nthreads) {
    job_t base;
    if (setup(&base, elem_bytes, rank, extents, perm)) return 1;
    base.A = A;
    base.B = B;
    const int64_t outer = base.n[rank - 1];
    if (nthreads < 1) nthreads = 1;
    if (nthreads > outer) nthreads = (int)outer;
    if (nthreads == 1) {
        base.lo = 0;
        base.hi = outer;
        run(&base);
        return 0;
    }
    job_t *jobs = (job_t *)malloc(sizeof(job_t) * (size_t)nthreads);
    pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)nthreads);
    for (int t = 0; t < nthreads; t++) {
        jobs[t] = base;
        jobs[t].lo = outer * t / nthreads;
        jobs[t].hi = outer * (t + 1) / nthreads;
        pthread_create(&th[t], NULL, run, &jobs[t]);
    }
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    free(jobs);
    free(th);
    return 0;
}

/* The sub-tensor form (the library's ttlg_plan_strided; used by the fused
 * sharded exchange): the same d-nested loop with given strides (elements),
 * lin_A = a_off + sum_k i_k in_strides[k], lin_B = b_off + sum_i
 * i_{perm[i]} out_strides[i].  Writes only the addressed positions of B. */
int oracle_transpose_strided(int elem_bytes, int rank, const int64_t *extents,
                             const int32_t *perm, const int64_t *in_strides,
                             const int64_t *out_strides, const void *A, int64_t a_off,
                             void *B, int64_t b_off) {
    job_t j;
    if (setup(&j, elem_bytes, rank, extents, perm)) return 1;
    for (int k = 0; k < rank; k++) {
        j.sA[k] = in_strides[k];
        j.sB[k] = out_strides[k];
    }
    j.A = (const char *)A + a_off * elem_bytes;
    j.B = (char *)B + b_off * elem_bytes;
    j.lo = 0;
    j.hi = j.n[rank - 1];
    run(&j);
    return 0;
}

/* The same definition read backwards, for sampled checks at sizes the full
 * loop cannot hold: for each output linear index lin_B, decode the output
 * multi-index o (o_0 fastest, extents m[i] = n[perm[i]]), set
 * i_{perm[i]} = o_i, and return lin_A = sum_k i_k sA[k]. */
int oracle_source_index(int rank, const int64_t *extents, const int32_t *perm,
                        const int64_t *linB, int64_t *linA, int64_t count) {
    job_t j;
    if (setup(&j, 8, rank, extents, perm)) return 1;
    for (int64_t e = 0; e < count; e++) {
        int64_t rem = linB[e];
        int64_t in_idx[ORACLE_MAX_RANK];
        for (int i = 0; i < rank; i++) {
            int64_t m = j.n[j.perm[i]];
            in_idx[j.perm[i]] = rem % m;
            rem /= m;
        }
        int64_t a = 0;
        for (int k = 0; k < rank; k++) a += in_idx[k] * j.sA[k];
        linA[e] = a;
    }
    return 0;
}
