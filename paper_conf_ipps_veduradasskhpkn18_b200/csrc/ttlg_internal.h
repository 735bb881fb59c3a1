// ttlg_internal.h -- plan and kernel-parameter layout shared by the host
// planner (planner.cpp), the C ABI (api.cpp) and the sm_100a kernels
// (kernels.cu).  Product code; never includes anything from oracle/.
#pragma once

#include <stdint.h>

#include <atomic>

#include "../../include/ttlg.h"

#define TTLG_MAXD TTLG_MAX_RANK

namespace ttlg {

// Fast unsigned division by a run-time constant (multiply-high + shift).
// Valid for dividends n < 2^31 (tile indices and row indices always are).
// quotient = (umulhi(n, mul) + (mul_hi_bit ? n : 0)) >> shr; we use the
// 31+ceil(log2 d) formulation so that mul fits in 32 bits.
struct FastDiv {
  uint32_t div;
  uint32_t mul;
  uint32_t shr;
};

inline FastDiv make_fastdiv(uint32_t d) {
  FastDiv f;
  f.div = d;
  if (d <= 1) {
    f.mul = 0;
    f.shr = 0;
    return f;
  }
  const uint32_t l = 32 - (uint32_t)__builtin_clz(d - 1);  // ceil(log2 d), d >= 2
  uint32_t p = 31 + l;
  f.mul = (uint32_t)(((1ull << p) + d - 1) / d);
  f.shr = p - 32;
  return f;
}

inline uint32_t fastdiv_host(uint32_t n, const FastDiv &f) {
  if (f.div <= 1) return n;
  return (uint32_t)((((uint64_t)n * f.mul) >> 32) >> f.shr);
}

// Kernel kinds.
enum KernelKind : int32_t {
  KK_DIRECT = 0,  // FML / COPY: contiguous input run -> rows of the output run, no smem staging
  KK_TILE = 1,    // OD / OA / FMS: register-staged, one tile per CTA (k_tile)
  KK_PIPE = 2,    // OD / OA / FMS: cp.async double-buffered, persistent (k_pipe)
  KK_QUAD = 3,    // OD: 16-byte chunks in and out, K x K register transpose (k_quad)
  KK_DEINT = 4,   // [n0, M(, nb)] perm (1 0 (2)) with n0 <= 8 (k_deint, AoS -> SoA) or
                  // n1 <= 8 (k_inter, SoA -> AoS): 16-byte accesses both ways
  KK_BULKQ = 5,   // OD: TMA bulk row loads into an mbarrier ring, K x K register transposes,
                  // 16-byte stores (k_bulk, consumer mode quad)
  KK_BULKG = 6,   // any schema: TMA bulk row loads, 16-byte stores gathered from K
                  // element reads (k_bulk, consumer mode gather)
  KK_VEC = 7,     // any schema with 16-byte aligned rows: 16-byte cp.async loads, 16-byte
                  // stores gathered from K element reads (k_vec)
  KK_PHASE = 8,   // k_tile's slice with 16-byte loads at any row alignment (per-row phase
                  // in shared memory) and element stores (k_phase)
  KK_BLK = 9,     // closed leading block (<= 8 KB, contiguous in A and B): one warp per
                  // block, WC-byte chunk loads and gathered WC-byte stores (k_blk)
  KK_TMA = 10,    // OD: TMA tensor-map tile loads (cp.async.bulk.tensor, 128-byte swizzle)
                  // into an mbarrier ring, k_bulk's quad consumers (k_tmap)
  KK_NUM = 11,
};

// Everything one launch needs, passed by value as a __grid_constant__ kernel
// parameter (lives in the constant bank; replaces the paper's texture-bound
// offset arrays, and its rank-specialised macro code,
// L1138-1155: loops over these arrays are unrolled to TTLG_MAXD with guards so
// every index is a compile-time constant).
//
// Tile ("slice" in the paper) geometry, all in access-element units:
//   the tile is the box prod_k t[k] over fused input dims; the input run is
//   the input-prefix dims 0..a (a possibly blocked), contiguous in A, length LA;
//   the output run is the output-prefix dims perm[0..b] (perm[b] possibly
//   blocked), contiguous in B, length LB.  A-rows enumerate the tile digits
//   outside the input run (RA = V/LA), B-rows those outside the output run
//   (RB = V/LB).  Per-row tables (built in shared memory once per CTA) hold the
//   relative global offset and the shared-memory offset of each row.
struct TileParams {
  // ---- tile grid (tile index -> tile base), grid dims in input order, first fastest
  uint32_t num_tiles;
  int32_t ng;
  FastDiv gdiv[TTLG_MAXD];
  int64_t gsA[TTLG_MAXD];  // t[k] * strideA[k]
  int64_t gsB[TTLG_MAXD];  // t[k] * strideB[k]
  // ---- partial tiles: the two blockable dims (a = last input-run dim, pb = perm[b])
  int32_t blkA_g, blkB_g;  // grid-dim index of dim a / dim pb, -1 if never partial
  int32_t blkA_n, blkA_t, blkB_n, blkB_t;
  // ---- run geometry
  int32_t V;               // tile volume
  int32_t LA, RA, LAunit;  // LAlim = LAunit * lim_a
  int32_t LB, RB, LBunit;  // LBlim = LBunit * lim_pb
  // ---- A-row digits (tile dims outside the input run), input order
  int32_t nra, ra_blk;     // ra_blk: which A-row digit is dim pb (-1: none)
  int32_t ra_ext[TTLG_MAXD];
  int32_t ra_sG[TTLG_MAXD];  // stride in A
  int32_t ra_sS[TTLG_MAXD];  // stride in the smem tile
  FastDiv ra_div[TTLG_MAXD];  // fast division by ra_ext
  // ---- B-row digits (tile dims outside the output run), input order
  int32_t nrb, rb_blk;     // rb_blk: which B-row digit is dim a (-1: none)
  int32_t rb_ext[TTLG_MAXD];
  int32_t rb_sG[TTLG_MAXD];  // stride in B
  int32_t rb_sS[TTLG_MAXD];
  FastDiv rb_div[TTLG_MAXD];
  // ---- output-run digits, output order (-> smem column offsets)
  int32_t nj;
  int32_t j_ext[TTLG_MAXD];
  int32_t j_sS[TTLG_MAXD];
  FastDiv j_div[TTLG_MAXD];
  // ---- input-run digits, input order (-> smem offsets when the run is padded)
  int32_t xtab, ni;        // xtab: 1 = input run padded in smem, read icol table
  FastDiv i_div[TTLG_MAXD];
  int32_t i_sS[TTLG_MAXD];
  int32_t off_icol;
  // ---- shared-memory layout (bytes) and per-thread stepping
  int32_t smem_elems;      // data tile elements incl. padding
  int32_t off_tabB, off_jcol, off_digB, off_digA, off_ctx, off_data, off_data2, smem_bytes;
  int32_t drA, dxA, drB, dxB;  // divmod(threads, LA) and divmod(threads, LB)
  int32_t rsB;                 // B-rows per pass of the store walk (threads / LB; 0: LB > threads)
  FastDiv fd_LA, fd_LB, fd_NT, fd_rsB;  // per-thread walk setup without hardware division
  int32_t qk, qnj;             // k_quad: chunk elements K (0: scalar kernels), column slots
  int32_t tpc;                 // tiles per CTA (consecutive tile indices)
  int32_t deint_n0;            // k_deint: n0 (the structure size, 2..8); k_inter: n1
  int32_t deint_inter;         // 1: k_inter (SoA -> AoS, the small dim is dim 1)
  // k_bulk: ring of nstage tile buffers (stage_bytes apart, from off_data),
  // 2 * nstage mbarriers at off_bar (full[s], empty[s]); warp 0 produces
  int32_t nstage, stage_bytes, off_bar;
  int32_t tma_rows;  // 1: one TMA bulk copy per A-row; 0: 16-byte cp.async chunks
  // k_phase: A-offset phase (mod 16/W) contributed by each B-row digit and each
  // output-run digit (0 for input-run dims); elements of A (end-of-tensor guard)
  int32_t rb_sP[TTLG_MAXD];
  int32_t j_sP[TTLG_MAXD];
  int64_t a_elems;
  int32_t blk_cpl;  // k_blk: chunks per lane (template instance)
  int32_t blk_swz;  // k_blk: chunk-slot XOR swizzle shift (0: row padding RA instead)
  // k_tmap: the tile box as a TMA tensor map over A's fused dims in "map order"
  // (input-run dims 0..a, then the output-run dims in output order, then the
  // other dims).  The input run is split into tm_np panels of tm_pa elements
  // of dim a (tm_pw bytes per box row, <= 128); panel p is one box load of
  // tm_pbytes to stage + p * tm_pbytes, swizzled with the span of one row.  Grid dim g
  // contributes coordinate (digit * tm_gt[g]) to map dim tm_gmap[g].
  int32_t tm_rank, tm_np, tm_pa, tm_pw, tm_pbytes, tm_adim;
  int32_t tm_swz;  // XOR mask the swizzle applies to (byte offset >> 3): 0x70 / 0x30 / 0x10 / 0
                   // for box rows of 128 / 64 / 32 / 16 bytes (SWIZZLE_128B / 64B / 32B / none)
  int32_t tm_gmap[TTLG_MAXD], tm_gt[TTLG_MAXD];
  // host side (encoded per launch with the operand's address, kernels.cu)
  int64_t tm_dim[TTLG_MAXD];     // globalDim, map order
  int64_t tm_stride[TTLG_MAXD];  // globalStrides in bytes of map dims 1..rank-1
  int32_t tm_box[TTLG_MAXD];     // boxDim (dim a: tm_pa)
};

// Operand pointers of one launch: entry blockIdx.y (grid.y = n <= kMaxBatch;
// ttlg_execute_batch) -- a __grid_constant__ kernel parameter like TileParams.
constexpr int kMaxBatch = TTLG_MAX_BATCH;
struct BatchPtrs {
  const void *A[kMaxBatch];
  void *B[kMaxBatch];
};

struct Problem {
  int esize;       // bytes per element as given (4/8)
  int W;           // access-element bytes after widening (4/8/16)
  int d;           // fused rank
  int64_t n[TTLG_MAXD];
  int32_t p[TTLG_MAXD];
  // strides per fused INPUT dim, in access elements: offset in A of digit k
  // is i_k * sA[k], offset in B is i_k * sB[k] (dense tensors: prefix
  // products; sub-tensors: ttlg_plan_strided).  sA[0] = sB[p[0]] = 1.
  int64_t sA[TTLG_MAXD], sB[TTLG_MAXD];
  // largest input-run dim a / output-run position b whose prefix is dense
  // (a tile's input and output runs must stay contiguous)
  int denseA, denseB;
  // largest K in {2, 4} (k_quad chunk elements) dividing every row stride
  // that a chunk must stay aligned to (A: dims >= 1; B: dims != p[0])
  int kalign;
};

struct DeviceProfile {
  int sms;
  int smem_per_block_optin;
  int smem_per_sm;
  int max_threads_per_sm;
  int regs_per_sm;
  double hbm_gbs;  // measured copy bandwidth used by the model
  bool virt;       // true: no device, virtual B200
};

}  // namespace ttlg

struct ttlg_plan_s {
  int device;  // -1 when planned against the virtual profile
  int kind;    // ttlg::KernelKind
  int W;       // access bytes
  int align;   // pointer alignment the kernel needs (W, or 16 for k_quad)
  int threads;
  int grid;
  int variant;  // reserved (hints->variant)
  int64_t nbytes;  // N * s
  int64_t spanA, spanB;  // bytes from the base pointer to one past the last element
  ttlg::TileParams kp;
  ttlg_plan_info info;
  // original request (for the misaligned-pointer fallback)
  int dt, rank;
  int64_t ext[TTLG_MAXD];
  int32_t perm[TTLG_MAXD];
  ttlg_plan_hints hints;
  bool has_hints;
  // sub-tensor (ttlg_plan_strided) request: strides in elements as given
  bool strided;
  int64_t in_strides[TTLG_MAXD], out_strides[TTLG_MAXD];
  // element-width plan for pointers not aligned to `align` (api.cpp execute):
  // built once, on first use, and owned by this plan
  mutable std::atomic<ttlg_plan_s *> fallback{nullptr};

  ttlg_plan_s() = default;
  ttlg_plan_s(const ttlg_plan_s &) = delete;
  ttlg_plan_s &operator=(const ttlg_plan_s &) = delete;
  ~ttlg_plan_s() { delete fallback.load(std::memory_order_acquire); }
};

namespace ttlg {
// collects every scored candidate (ttlg_plan_candidates: calibration, regret studies)
struct CandidateSink {
  ttlg_plan_info *out;
  int max;
  int n;
  bool shortlist;  // false: every scored candidate; true: the ranked short list
};
constexpr int kModelFeatureCount = 10;
// planner.cpp
ttlg_status validate(ttlg_dtype dt, int rank, const int64_t *ext, const int32_t *perm);
// fast = the single-use effort level.  1: the same screen, refinement and
// tree ranking as a repeated-use plan (so both pick the same kernel), minus
// the shared-memory padding search and the reported-prediction tree pass;
// 2 (passes shorter than a plan, e.g. 15^6 fp64): also refine only the
// linear screen's best kFast2Refine and rank kFast2TopK with the trees
constexpr int kFastRefine = 32, kFastTopK = 16;
constexpr int kFast2Refine = 8, kFast2TopK = 6;
// in_strides / out_strides (elements; NULL = dense): the sub-tensor form of
// ttlg_plan_strided -- in_strides[k] per input dim, out_strides[i] per output dim
ttlg_status make_plan(ttlg_plan_s *plan, ttlg_dtype dt, int rank, const int64_t *ext,
                      const int32_t *perm, const ttlg_plan_hints *hints, const DeviceProfile &dev,
                      CandidateSink *sink = nullptr, int fast = 0,
                      const int64_t *in_strides = nullptr, const int64_t *out_strides = nullptr);
// api.cpp
const DeviceProfile &device_profile(int device);
// kernels.cu
// n pairs (1 <= n <= kMaxBatch) in one launch: grid (plan->grid, n)
ttlg_status launch(const ttlg_plan_s *plan, int n, const void *const *A, void *const *B,
                   void *stream);
int kernel_regs(int kind, int W);  // registers per thread of a kernel variant (cached; 0 if unknown)
int blk_regs(int S, int WC, int cpl);  // the same for a k_blk instance
}  // namespace ttlg
