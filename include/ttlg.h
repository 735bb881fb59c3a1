/*
 * ttlg.h -- C ABI of the B200-native TTLG tensor-transposition library.
 *
 * Operation (§I, Eq. 1): out-of-place transposition
 *     B[rho(i0, ..., i_{d-1})] <- A[i0, ..., i_{d-1}]
 * of a dense rank-d tensor of fp32 or fp64 elements, moved as bit patterns
 * (no arithmetic, so the result is unique bit for bit).
 *
 * Conventions (readings R1, R2):
 *   - extents[0] is the fastest-varying index (FVI): the element with
 *     multi-index (i0..i_{d-1}) lives at linear offset sum_k i_k * prod_{k'<k} n_k'
 *     (MATLAB/Fortran notation, PAPER.md L284-286 footnote 1);
 *   - perm[i] = j means output dimension i is input dimension j (PAPER.md
 *     L1883-1886, §VI).  B therefore has extents m[i] = extents[perm[i]]; the
 *     paper's rho is perm^{-1}.
 *
 * Usage modes (§VI): "repeated use" = ttlg_plan once +
 * ttlg_execute many times; "single use" = ttlg_transpose (plan cost counts).
 * ttlg_predict_time is the performance-model query for higher-level optimisers
 * such as a TTGT contraction engine (PAPER.md L11-21 Abstract, L60-63 §I).
 *
 * Threading / ownership:
 *   - the caller owns extents/perm (copied into the plan) and A/B (device
 *     memory, N*s bytes each, N = prod extents, s = 4 or 8);
 *   - a plan is immutable host memory; it is bound to the CUDA device that was
 *     current when it was created (TTLG_ERR_DEVICE if executed elsewhere); all
 *     kernel parameters are captured at launch, so a plan may be destroyed as
 *     soon as ttlg_execute returns and one plan may be executed concurrently
 *     on several streams;
 *   - ttlg_execute / ttlg_transpose are asynchronous in stream order and never
 *     synchronise the host; launch failures return TTLG_ERR_CUDA.
 *   - planning makes no CUDA calls other than cached device-attribute queries;
 *     with no CUDA device present a virtual B200 profile (148 SMs, 227 KB
 *     shared memory per block) is used, so ttlg_plan / ttlg_predict_time work
 *     on a CPU-only host (ttlg_execute then returns TTLG_ERR_DEVICE).
 */
#ifndef TTLG_H_
#define TTLG_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define TTLG_MAX_RANK 15 /* rank-specialised code "until rank 15" */
#define TTLG_VERSION 100

typedef enum { TTLG_F32 = 0, TTLG_F64 = 1 } ttlg_dtype;

typedef enum {
  TTLG_OK = 0,
  TTLG_ERR_INVALID_VALUE = 1, /* bad rank/extent/perm/dtype, null or misaligned pointer */
  TTLG_ERR_ALIASING = 2,      /* [A, A+N*s) overlaps [B, B+N*s): op is out-of-place (L91) */
  TTLG_ERR_DEVICE = 3,        /* no CUDA device, or executed on another device than planned */
  TTLG_ERR_CUDA = 4,          /* a CUDA launch / runtime call failed */
  TTLG_ERR_NO_MEMORY = 5,     /* host allocation failed */
  TTLG_ERR_INTERNAL = 6,      /* planner could not build a legal plan (bug) */
  TTLG_ERR_UNSUPPORTED = 7    /* e.g. a forced schema that does not apply */
} ttlg_status;

/* Kernel schemas (§III-IV, Alg. 1; flowchart L686-697).
 * COPY is the fused-rank-1 case (identity after index fusion). */
typedef enum {
  TTLG_SCHEMA_AUTO = -1,
  TTLG_SCHEMA_COPY = 0,
  TTLG_SCHEMA_FML = 1, /* FVI-Match-Large, Alg. 7 */
  TTLG_SCHEMA_FMS = 2, /* FVI-Match-Small, Alg. 6 */
  TTLG_SCHEMA_OD = 3,  /* Orthogonal-Distinct, Alg. 2 */
  TTLG_SCHEMA_OA = 4   /* Orthogonal-Arbitrary, Alg. 4/5 L868-1020 */
} ttlg_schema;

typedef struct ttlg_plan_s *ttlg_plan_t;

/* Optional planning hints (tests, calibration, model-regret studies).
 * Initialise with ttlg_plan_hints_init() (everything "auto"), then set what
 * you want forced. */
typedef struct {
  int32_t schema;                        /* TTLG_SCHEMA_AUTO (-1) = model choice        */
  int32_t in_dim;                        /* -1 = auto; else last fused input dim of the
                                            input slice (Alg. 3 dimsIn)                   */
  int64_t in_block;                      /* blocking factor of that dim (blockA), 0=auto */
  int32_t out_dim;                       /* -1 = auto; position b of the last output dim
                                            of the output slice (Alg. 3 dimsOut)          */
  int64_t out_block;                     /* blockB, 0 = auto                             */
  int32_t elem_bytes_override;           /* 0 = auto widening; else 4/8/16 access width
                                            (pins the width: no k_quad 16-byte chunks)   */
  int32_t threads;                       /* 0 = auto; else threads per block (k_bulk:
                                            consumer threads, 256 or 512)                 */
  int32_t grid;                          /* 0 = auto (persistent); else blocks           */
  int32_t no_fusion;                     /* 1 = skip index fusion (tests)                */
  int32_t variant;                       /* staged kernel: 0 = model choice, 1 = k_tile
                                            (one tile per CTA), 2 = k_pipe (persistent,
                                            double-buffered), 3 = k_quad (OD in 16-byte
                                            chunks, K x K register transpose), 4 = k_deint
                                            / k_inter ([n0,M(,nb)] perm (1 0 (2)) with
                                            2 <= n0 <= 8 and M a multiple of 16/s, or
                                            2 <= M <= 8 and n0 a multiple of 16/s:
                                            16-byte accesses both ways through a per-warp
                                            staging buffer), 5 = k_bulk with quad
                                            consumers (OD; TMA bulk row loads into an
                                            mbarrier ring), 6 = k_bulk with gather
                                            consumers (any schema), 7 = k_vec (16-byte
                                            cp.async loads, 16-byte stores gathered from
                                            16/s element reads); 5-7 need every A-row
                                            (6, 7: and B-row) 16-byte aligned and whole
                                            16-byte chunks, else TTLG_ERR_UNSUPPORTED;
                                            8 = k_phase (k_tile's slice with 16-byte
                                            loads at any row alignment); 9 = k_blk (the
                                            fused perm's leading dims 0..c-1, c >= 2,
                                            map onto output positions 0..c-1 and form a
                                            block of 32 chunks .. 8 KB contiguous in A
                                            and B: one warp per block, chunk loads and
                                            gathered chunk stores), 10 = k_tmap (OD:
                                            the tile loaded by TMA tensor-map box copies,
                                            cp.async.bulk.tensor, swizzled; fused
                                            rank <= 5, 16-byte aligned A strides and
                                            k_quad's chunk alignment), else
                                            TTLG_ERR_UNSUPPORTED.  The automatic choice
                                            considers 0-4, 7 and 9 (env TTLG_VEC=0 drops
                                            7; TTLG_BULK=1 adds 5, 6; TTLG_PHASE=1 adds
                                            8; TTLG_TMA=1 adds 10)                         */
} ttlg_plan_hints;

/* Everything a test or benchmark may want to know about a plan. */
typedef struct {
  int32_t schema;                         /* ttlg_schema actually used                   */
  int32_t dtype;                          /* ttlg_dtype                                  */
  int32_t rank;                           /* rank as given                               */
  int32_t fused_rank;                     /* rank after squeeze + fusion (L666-685)      */
  int64_t fused_extents[TTLG_MAX_RANK];   /* in units of the access element (below)      */
  int32_t fused_perm[TTLG_MAX_RANK];
  int32_t access_bytes;                   /* 4, 8 or 16: element width after widening    */
  int64_t tile_extents[TTLG_MAX_RANK];    /* per fused dim; 1 = not in the slice         */
  int32_t in_dim, out_dim;                /* last dims of the input / output slice       */
  int64_t in_run, out_run;                /* contiguous run lengths (access elements)    */
  int64_t tile_volume;                    /* elements per slice (tile)                   */
  int64_t num_tiles;
  int32_t grid, threads, smem_bytes;
  int64_t bytes;                          /* algorithmic bytes 2*N*s                     */
  double predicted_seconds;               /* performance-model prediction                */
  int32_t candidates;                     /* number of candidates the model scored       */
  int32_t param_bytes;                    /* kernel-parameter blob size                  */
  int32_t kernel;                         /* 0 k_direct (FML/COPY), 1 k_tile, 2 k_pipe,
                                             3 k_quad, 4 k_deint / k_inter, 5 k_bulk
                                             (quad consumers), 6 k_bulk (gather
                                             consumers), 7 k_vec, 8 k_phase, 9 k_blk
                                             (closed leading block, one warp per block)  */
  int32_t occupancy;                      /* resident CTAs per SM assumed by the model   */
  int32_t num_features;                   /* model feature vector (§V features, B200)    */
  double features[12];
  int32_t stages;                         /* k_bulk: tile buffers in the ring; else 0    */
} ttlg_plan_info;

void ttlg_plan_hints_init(ttlg_plan_hints *hints);

/* Create a plan (Alg. 1 taxonomy + Alg. 3 slice/block search + §V model).
 * extents: [rank] int64, each >= 1; perm: [rank] permutation of 0..rank-1;
 * rank in [1, 15].  Returns TTLG_ERR_INVALID_VALUE on bad arguments. */
ttlg_status ttlg_plan(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                      const int32_t *perm);

/* As ttlg_plan, with hints (may be NULL). Forced choices that do not apply
 * return TTLG_ERR_UNSUPPORTED. */
ttlg_status ttlg_plan_ex(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                         const int32_t *perm, const ttlg_plan_hints *hints);

/* Sub-tensor transposition (the general strided form; used by the fused
 * sharded exchange): the same operation as ttlg_plan on
 * extents/perm, but element (i0..i_{d-1}) is read from
 *     A + sum_k i_k * in_strides[k]
 * and written to
 *     B + sum_i o_i * out_strides[i],   o_i = i_{perm[i]},
 * strides in ELEMENTS (in_strides per input dim, out_strides per output dim;
 * either may be NULL = dense, which is exactly ttlg_plan_ex).  Extent-1 dims
 * ignore their stride.  Requirements: every stride of a non-unit dim >= 1; the
 * fastest non-unit dim of A has in_stride 1 and the first non-unit output dim
 * has out_stride 1 (else TTLG_ERR_UNSUPPORTED: the kernels move contiguous
 * runs along both FVIs); B must be injective -- sorted by stride, each output
 * dim's stride >= the previous stride x extent (else TTLG_ERR_INVALID_VALUE).
 * Index fusion (L666-685) joins two dims only where both tensors are dense
 * across them.  Aliasing is checked on the spanned byte ranges
 * [A, A + s*(1 + sum (n_k-1)*in_strides[k])) and likewise for B.
 * ttlg_execute_host rejects strided plans (TTLG_ERR_UNSUPPORTED). */
ttlg_status ttlg_plan_strided(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                              const int32_t *perm, const int64_t *in_strides,
                              const int64_t *out_strides, const ttlg_plan_hints *hints);

/* Repeated-use execution: one asynchronous kernel launch on `stream`
 * (a cudaStream_t; NULL = legacy default stream).  A and B are device
 * pointers, element-aligned, non-overlapping. */
ttlg_status ttlg_execute(ttlg_plan_t plan, const void *A, void *B, void *stream);

/* Batched repeated-use execution: the same plan on `count` (A[i], B[i]) pairs
 * in ONE kernel launch (grid.y = count, at most TTLG_MAX_BATCH pairs per
 * launch; larger counts take ceil(count / TTLG_MAX_BATCH) launches).  Used by
 * the fused sharded exchange, where rank p's P sub-transpositions have the
 * same shape and differ only in the A sub-box and the destination (peer) B
 * slab.  Arrays are caller-owned host arrays of device pointers; every pair
 * obeys ttlg_execute's rules, and no A[i] may overlap any B[j]
 * (TTLG_ERR_ALIASING).  Outputs B[i] must not overlap each other (not
 * checked: the result would depend on the write order).  count < 1 or NULL
 * arrays -> TTLG_ERR_INVALID_VALUE. */
#define TTLG_MAX_BATCH 16
ttlg_status ttlg_execute_batch(ttlg_plan_t plan, int32_t count, const void *const *A,
                               void *const *B, void *stream);

ttlg_status ttlg_plan_destroy(ttlg_plan_t plan);

/* Single-use: plan + execute + destroy, no caching, no host sync. */
ttlg_status ttlg_transpose(ttlg_dtype dt, int rank, const int64_t *extents, const int32_t *perm,
                           const void *A, void *B, void *stream);

/* Host-buffer end-to-end path: A_host -> A_dev, transpose, B_dev -> B_host.
 * A is split along one input dim into up to 32 chunks (>= 16 MiB each); the
 * dim is chosen so that the narrower of the chunk's host-side row widths (its
 * slab of A, a strided 2-D region; its slab of B, likewise) is as wide as
 * possible.  Each chunk is copied densely (cudaMemcpy2DAsync), transposed
 * with a sub-plan, and copied back -- H2D, kernels and D2H of successive
 * chunks run on internal streams so both PCIe directions overlap.  Ordered
 * after prior work on `stream`; `stream` waits for completion (no host sync).
 * A_host/B_host should be pinned; A_dev/B_dev are device scratch of N*s bytes
 * each (their contents are chunk slabs afterwards, not A / B).  Small or
 * unsplittable tensors: one stream, in order.  Dense plans only. */
ttlg_status ttlg_execute_host(ttlg_plan_t plan, const void *A_host, void *B_host, void *A_dev,
                              void *B_dev, void *stream);

/* Performance-model query (§V): predicted seconds of the
 * plan the library would choose.  No CUDA calls beyond cached attributes. */
ttlg_status ttlg_predict_time(ttlg_dtype dt, int rank, const int64_t *extents,
                              const int32_t *perm, double *seconds);

ttlg_status ttlg_plan_describe(ttlg_plan_t plan, ttlg_plan_info *info);

/* Measure-mode refinement (the cuTT "measure" idea, PAPER.md L130-136,
 * L1575-1579): executes up to max_candidates (<= 16) of the model's
 * ranked short list on A -> B (B is overwritten with the correct result; A is
 * read only), times each with CUDA events on `stream` (synchronises the
 * stream), and replaces *plan by the fastest (the old plan is destroyed).
 * best_seconds (may be NULL) receives the measured time. */
ttlg_status ttlg_plan_tune(ttlg_plan_t *plan, const void *A, void *B, void *stream,
                           int32_t max_candidates, double *best_seconds);

/* Every candidate the planner scores for this problem (Alg. 3's enumeration),
 * with its model features and predicted time -- for calibration (§V) and
 * measure-mode / model-regret studies.  Writes up to max_out entries to out and
 * the number written to *n_out.  Any candidate can be executed by passing its
 * schema / in_dim / tile_extents[in_dim] / out_dim / tile_extents[perm[out_dim]]
 * as hints to ttlg_plan_ex. */
ttlg_status ttlg_plan_candidates(ttlg_dtype dt, int rank, const int64_t *extents,
                                 const int32_t *perm, const ttlg_plan_hints *hints,
                                 ttlg_plan_info *out, int32_t max_out, int32_t *n_out);

/* Peer memory for the fused sharded exchange (not in the
 * paper): rank p's sub-tensor transpositions store straight into the B slabs
 * of the other ranks over NVLink/NVSwitch (CUDA IPC mappings; every rank runs
 * one process per GPU, PyTorch supplies the process group that moves the
 * handles).
 *   ttlg_ipc_export: handle (TTLG_IPC_HANDLE_BYTES bytes, caller-owned) of the
 *     device allocation containing `ptr`, and ptr's byte offset in it;
 *   ttlg_ipc_open: map another process's allocation on the current device
 *     (peer access enabled lazily); *ptr = mapped base + offset;
 *   ttlg_ipc_close: unmap (pass the pointer and offset ttlg_ipc_open used).
 * Errors: TTLG_ERR_INVALID_VALUE for null arguments, TTLG_ERR_CUDA when the
 * runtime refuses (e.g. handle opened in the exporting process itself). */
#define TTLG_IPC_HANDLE_BYTES 64
ttlg_status ttlg_ipc_export(const void *ptr, void *handle, int64_t *offset);
ttlg_status ttlg_ipc_open(const void *handle, int64_t offset, void **ptr);
ttlg_status ttlg_ipc_close(void *ptr, int64_t offset);

const char *ttlg_status_string(ttlg_status s);
const char *ttlg_schema_name(int schema);
int ttlg_version(void);
/* Provenance of the performance-model coefficients compiled in (calibration tag). */
const char *ttlg_model_source(void);

#ifdef __cplusplus
}
#endif
#endif /* TTLG_H_ */
