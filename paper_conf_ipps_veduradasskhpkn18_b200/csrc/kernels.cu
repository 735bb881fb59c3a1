// kernels.cu -- sm_100a transposition kernels of the B200 TTLG library.
//
// Two kernel families, templated on the access width W = 4/8/16 bytes:
//
//  k_direct  (FML / COPY; Alg. 7): the tile is a
//            contiguous run of A (input dims 0..a, a blocked); elements are
//            read with coalesced streaming loads, U per thread in flight, and
//            written straight to their output row (output run = the matching
//            FVI, dim 0).  No shared memory for data, only the row table.
//
//  k_pipe    (OD / OA / FMS; Alg. 2, Alg. 4/5 L868-1020, Alg. 6
//            L1022-1107): the tile (the paper's "slice") is the union of an
//            input-prefix group and an output-prefix group.  Load phase: A-rows
//            of LA contiguous elements are copied global -> shared with cp.async
//            (LDGSTS, predicated PTX); store phase: B-rows of LB
//            contiguous elements are read from shared memory through the column
//            offsets and written coalesced.  Rows are processed warp-wise: a
//            warp (or a power-of-two lane group of G <= 32 lanes when the run is
//            short) owns a row, so the row-table lookup is a broadcast and the
//            column offsets are register-resident -- the B200 form of the
//            paper's compile-time-constant indexing (L1138-1155).  The
//            shared-memory layout pads every output-only dim so that output
//            position j lands in bank j mod (128/W): conflict-free column reads
//            (generalising the 32x33 pad, L747-749, and FMS's pad, L1104-1107).
//
// Two grid strategies compete per candidate: PERSIST = false ("k_tile"): one
// CTA per tile (or a few consecutive tiles, `tpc`), single buffer, many CTAs
// per SM; PERSIST = true ("k_pipe"): persistent CTAs with a double-buffered
// cp.async ring.  k_direct uses one CTA per tile.  Every CTA builds its row tables in shared memory
// (the paper's texture-mapped offset arrays, L737-745) and decodes its tile
// index with fast-divmod (the paper's decode/compute_base, L725-737).
#include <cuda_runtime.h>

#include <mutex>

#include "ttlg_internal.h"

namespace ttlg {

template <int W>
struct Vec;
template <>
struct Vec<4> {
  using T = unsigned int;
};
template <>
struct Vec<8> {
  using T = uint2;
};
template <>
struct Vec<16> {
  using T = uint4;
};

template <bool CS, typename T>
__device__ __forceinline__ T ld_stream(const T *p) {
  if constexpr (CS)
    return __ldcs(p);
  else
    return *p;
}
template <bool CS, typename T>
__device__ __forceinline__ void st_stream(T *p, T v) {
  if constexpr (CS)
    __stcs(p, v);
  else
    *p = v;
}

// cp.async (LDGSTS): global -> shared without a register round trip.  No
// "memory" clobber on the copy itself (ordering is enforced by commit/wait +
// __syncthreads), so the compiler may keep addresses and table values in
// registers across it.
template <int W>
__device__ __forceinline__ void cp_async(uint32_t s, const void *gptr) {
  if constexpr (W == 16)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gptr));
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;\n" ::"r"(s), "l"(gptr), "n"(W));
}
// predicated forms (the predicate goes into the PTX guard, so predicated-off
// lanes cost no branch / reconvergence)
template <int W>
__device__ __forceinline__ void cp_async_p(uint32_t s, const void *gptr, bool p) {
  if constexpr (W == 16)
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n"
                 " @q cp.async.cg.shared.global [%0], [%1], 16;\n}\n" ::"r"(s),
                 "l"(gptr), "r"((int)p));
  else
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n"
                 " @q cp.async.ca.shared.global [%0], [%1], %3;\n}\n" ::"r"(s),
                 "l"(gptr), "r"((int)p), "n"(W));
}
__device__ __forceinline__ void stcs_p(unsigned int *a, unsigned int v, bool p) {
  asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %2, 0;\n @q st.global.cs.u32 [%0], %1;\n}\n"
               ::"l"(a), "r"(v), "r"((int)p) : "memory");
}
__device__ __forceinline__ void stcs_p(uint2 *a, uint2 v, bool p) {
  asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %3, 0;\n"
               " @q st.global.cs.v2.u32 [%0], {%1, %2};\n}\n"
               ::"l"(a), "r"(v.x), "r"(v.y), "r"((int)p) : "memory");
}
__device__ __forceinline__ void stcs_p(uint4 *a, uint4 v, bool p) {
  asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %5, 0;\n"
               " @q st.global.cs.v4.u32 [%0], {%1, %2, %3, %4};\n}\n"
               ::"l"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"((int)p) : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

__device__ __forceinline__ uint32_t fdiv(uint32_t n, const FastDiv &f) {
  return __umulhi(n, f.mul) >> f.shr;  // grid divisors are always >= 2
}

struct TileCtx {
  int64_t bA, bB;
  int limA, limB;
};

// decode(blockid) + compute_base (Alg. 2 lines 6-7): tile index -> tile
// coordinates (mixed radix over the grid dims, first fastest) -> base offsets
// and the extents of the two blockable dims inside this tile.
__device__ __forceinline__ TileCtx decode_tile(const TileParams &P, uint32_t tile) {
  TileCtx c;
  c.bA = 0;
  c.bB = 0;
  c.limA = P.blkA_t;
  c.limB = P.blkB_t;
  uint32_t rem = tile;
#pragma unroll
  for (int g = 0; g < TTLG_MAXD; g++) {
    if (g < P.ng) {
      const uint32_t q = fdiv(rem, P.gdiv[g]);
      const int cg = (int)(rem - q * P.gdiv[g].div);
      rem = q;
      c.bA += (int64_t)cg * P.gsA[g];
      c.bB += (int64_t)cg * P.gsB[g];
      if (g == P.blkA_g) c.limA = min(P.blkA_t, P.blkA_n - cg * P.blkA_t);
      if (g == P.blkB_g) c.limB = min(P.blkB_t, P.blkB_n - cg * P.blkB_t);
    }
  }
  return c;
}

// Row tables (Alg. 4's input_offset / output_offset, separated into a per-row
// part and a per-column part): decode row index i over the row digits.
// Digit extents are >= 2, so the multiply-shift division applies.
__device__ __forceinline__ void build_rows(int R, int nr, const FastDiv *ext, const int32_t *sG,
                                           const int32_t *sS, int blk, int2 *tab, int *dig) {
  for (int i = threadIdx.x; i < R; i += blockDim.x) {
    int rem = i, g = 0, s = 0, dg = 0;
    for (int k = 0; k < nr; k++) {
      const int cq = (int)fdiv((uint32_t)rem, ext[k]);
      const int c = rem - cq * (int)ext[k].div;
      rem = cq;
      g += c * sG[k];
      s += c * sS[k];
      if (k == blk) dg = c;
    }
    tab[i] = make_int2(g, s);
    dig[i] = dg;
  }
}

template <int W, int U, bool CS>
__global__ void __launch_bounds__(512) k_direct(const __grid_constant__ TileParams P,
                                                const void *__restrict__ Av,
                                                void *__restrict__ Bv) {
  using T = typename Vec<W>::T;
  extern __shared__ __align__(16) unsigned char smem[];
  int2 *tabB = reinterpret_cast<int2 *>(smem + P.off_tabB);
  int *digA = reinterpret_cast<int *>(smem + P.off_digA);
  const T *A = reinterpret_cast<const T *>(Av);
  T *B = reinterpret_cast<T *>(Bv);

  build_rows(P.RB, P.nrb, P.rb_div, P.rb_sG, P.rb_sS, P.rb_blk, tabB, digA);
  __syncthreads();

  const int NT = blockDim.x, tid = threadIdx.x;
  const int r0 = tid / P.LB, j0 = tid % P.LB;
  for (int it = 0; it < P.tpc; it++) {
    const uint32_t tile = blockIdx.x * (uint32_t)P.tpc + it;
    if (tile >= P.num_tiles) break;
    const TileCtx c = decode_tile(P, tile);
    const int lim = P.LAunit * c.limA;  // the blocked dim a is the tile's outermost
    const T *Ab = A + c.bA;
    T *Bb = B + c.bB;
    int e = tid, r = r0, j = j0;
    while (e < lim) {
      T v[U];
      int ob[U];
#pragma unroll
      for (int u = 0; u < U; u++) {
        ob[u] = -1;
        if (e < lim) {
          v[u] = ld_stream<CS>(Ab + e);
          ob[u] = tabB[r].x + j;
        }
        e += NT;
        j += P.dxB;
        r += P.drB;
        if (j >= P.LB) {
          j -= P.LB;
          r++;
        }
      }
#pragma unroll
      for (int u = 0; u < U; u++)
        if (ob[u] >= 0) st_stream<CS>(Bb + ob[u], v[u]);
    }
  }
}

// shared-memory helpers on 32-bit shared addresses (no generic->shared
// conversion per access)
__device__ __forceinline__ int2 lds_int2(uint32_t a) {
  int2 v;
  asm volatile("ld.shared.v2.s32 {%0, %1}, [%2];\n" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ int lds_int(uint32_t a) {
  int v;
  asm volatile("ld.shared.s32 %0, [%1];\n" : "=r"(v) : "r"(a));
  return v;
}
template <typename T>
__device__ __forceinline__ T lds_T(uint32_t a);
template <>
__device__ __forceinline__ unsigned int lds_T<unsigned int>(uint32_t a) {
  unsigned int v;
  asm volatile("ld.shared.u32 %0, [%1];\n" : "=r"(v) : "r"(a));
  return v;
}
template <>
__device__ __forceinline__ uint2 lds_T<uint2>(uint32_t a) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];\n" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
template <>
__device__ __forceinline__ uint4 lds_T<uint4>(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];\n"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "r"(a));
  return v;
}

// k_pipe template parameters:
//   GA32 / GB32: the A-row / B-row lane group is a whole warp (run >= 32), so
//                lane offsets along a row are compile-time immediates;
//   NJ > 0:      every lane owns at most NJ output-run positions of a B-row
//                (LB <= NJ * G_B) and keeps their shared-memory column offsets
//                in registers; NJ = 0: column offsets read from the table.
// Loop trip counts are warp-uniform and the bodies predicated, so no
// divergence/reconvergence bookkeeping is generated in the hot loops.
template <int W, int NJ, bool GA32, bool GB32, bool PERSIST, bool XT>
__global__ void __launch_bounds__(512) k_pipe(const __grid_constant__ TileParams P,
                                              const void *__restrict__ Av,
                                              void *__restrict__ Bv) {
  using T = typename Vec<W>::T;
  extern __shared__ __align__(16) unsigned char smem[];
  const uint32_t s0 = (uint32_t)__cvta_generic_to_shared(smem);
  const uint32_t s_tabA = s0, s_tabB = s0 + P.off_tabB, s_jcol = s0 + P.off_jcol;
  const uint32_t s_digB = s0 + P.off_digB, s_digA = s0 + P.off_digA;
  const uint32_t s_buf0 = s0 + P.off_data, s_buf1 = s0 + P.off_data2;
  const T *A = reinterpret_cast<const T *>(Av);
  T *B = reinterpret_cast<T *>(Bv);

  build_rows(P.RA, P.nra, P.ra_div, P.ra_sG, P.ra_sS, P.ra_blk,
             reinterpret_cast<int2 *>(smem), reinterpret_cast<int *>(smem + P.off_digB));
  build_rows(P.RB, P.nrb, P.rb_div, P.rb_sG, P.rb_sS, P.rb_blk,
             reinterpret_cast<int2 *>(smem + P.off_tabB),
             reinterpret_cast<int *>(smem + P.off_digA));
  for (int j = threadIdx.x; j < P.LB; j += blockDim.x) {
    int rem = j, s = 0;
    for (int k = 0; k < P.nj; k++) {
      const int cq = (int)fdiv((uint32_t)rem, P.j_div[k]);
      s += (rem - cq * (int)P.j_div[k].div) * P.j_sS[k];
      rem = cq;
    }
    reinterpret_cast<int *>(smem + P.off_jcol)[j] = s * W;  // byte offset
  }
  if constexpr (XT) {
    for (int x = threadIdx.x; x < P.LA; x += blockDim.x) {
      int rem = x, s = 0;
      for (int k = 0; k < P.ni; k++) {
        const int cq = (int)fdiv((uint32_t)rem, P.i_div[k]);
        s += (rem - cq * (int)P.i_div[k].div) * P.i_sS[k];
        rem = cq;
      }
      reinterpret_cast<int *>(smem + P.off_icol)[x] = s * W;  // byte offset
    }
  }
  const uint32_t s_icol = s0 + P.off_icol;
  __syncthreads();

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int lgA = GA32 ? 5 : P.lgA, lgB = GB32 ? 5 : P.lgB;
  const int gA = 1 << lgA, gB = 1 << lgB;
  const int xA0 = lane & (gA - 1), rA0 = warp * (32 >> lgA) + (lane >> lgA);
  const int rAstep = nw * (32 >> lgA);
  const int xB0 = lane & (gB - 1), rB0 = warp * (32 >> lgB) + (lane >> lgB);
  const int rBstep = nw * (32 >> lgB);
  const int RA = P.RA, RB = P.RB, LA = P.LA, LB = P.LB;
  const int kA = (LA + gA - 1) >> lgA;  // uniform per-row trip count (load)
  const int kB = (LB + gB - 1) >> lgB;  // uniform per-row trip count (store)
  const uint32_t jstrideW = (P.nj == 1 ? (uint32_t)P.j_sS[0] : 0u) * W;  // chunked long runs
  int jc[NJ > 0 ? NJ : 1];
  if constexpr (NJ > 0) {
#pragma unroll
    for (int i = 0; i < NJ; i++) {
      const int j = xB0 + i * gB;
      jc[i] = j < LB ? lds_int(s_jcol + 4 * j) : 0;
    }
  }

  // load phase of one tile: A-row r -> smem, cp.async, lanes stride the run
  auto issue = [&](const TileCtx &c, uint32_t sbuf) {
    const bool full = (c.limA == P.blkA_t) && (c.limB == P.blkB_t);
    const int lim = full ? LA : P.LAunit * c.limA;
    const T *Ab = A + c.bA + xA0;
    const uint32_t sb = sbuf + xA0 * W;
    for (int r = rA0; r < RA; r += rAstep) {
      const int2 t = lds_int2(s_tabA + 8 * r);
      const bool rok = full || lds_int(s_digB + 4 * r) < c.limB;
      const T *src = Ab + t.x;
      if constexpr (XT) {
        // padded input run: smem offset of run position x from the icol table
        const uint32_t rowS = sbuf + t.y * W;
        for (int k = 0; k < kA; k++) {
          const int x = xA0 + (k << lgA);
          const int off = x < LA ? lds_int(s_icol + 4 * x) : 0;
          cp_async_p<W>(rowS + off, src + (k << lgA), rok && x < lim);
        }
      } else {
        const uint32_t dst = sb + t.y * W;
        for (int k = 0; k < kA; k++)
          cp_async_p<W>(dst + (k << lgA) * W, src + (k << lgA), rok && xA0 + (k << lgA) < lim);
      }
    }
  };
  // store phase of one tile: B-row r <- smem through the column offsets
  auto drain = [&](const TileCtx &c, uint32_t sbuf) {
    const bool full = (c.limA == P.blkA_t) && (c.limB == P.blkB_t);
    const int lim = full ? LB : P.LBunit * c.limB;
    T *Bb = B + c.bB + xB0;
    for (int r = rB0; r < RB; r += rBstep) {
      const int2 t = lds_int2(s_tabB + 8 * r);
      const bool rok = full || lds_int(s_digA + 4 * r) < c.limA;
      T *dst = Bb + t.x;
      const uint32_t src = sbuf + t.y * W;
      if constexpr (NJ > 0) {
        if (LB <= (NJ << lgB)) {
#pragma unroll
          for (int i = 0; i < NJ; i++) {
            if (i < kB)
              stcs_p(dst + (i << lgB), lds_T<T>(src + jc[i]), rok && xB0 + (i << lgB) < lim);
          }
        } else
        // runs longer than NJ lane-slots (single output digit only, so the
        // column offset is linear in j) take several uniform chunks
        for (int jb = 0; jb < lim; jb += NJ << lgB) {
          const uint32_t cb = (uint32_t)jb * jstrideW;
#pragma unroll
          for (int i = 0; i < NJ; i++) {
            if (i < kB) {
              const bool ok = rok && jb + xB0 + (i << lgB) < lim;
              // predicated-off lanes read a valid address (no OOB smem access)
              stcs_p(dst + jb + (i << lgB), lds_T<T>(src + (ok ? cb + jc[i] : 0u)), ok);
            }
          }
        }
      } else {
#pragma unroll 4
        for (int i = 0; i < kB; i++) {
          const int j = xB0 + (i << lgB);
          const int off = j < LB ? lds_int(s_jcol + 4 * j) : 0;
          stcs_p(dst + (i << lgB), lds_T<T>(src + off), rok && j < lim);
        }
      }
    }
  };

  if constexpr (!PERSIST) {
    // k_tile: one tile (or tpc consecutive tiles) per CTA, single buffer, many
    // CTAs per SM -- the cp.async skeleton that reaches the D2D copy rate
    // (tools/copybench.cu: 6.4-6.6 TB/s vs 5.4-5.8 TB/s persistent)
    for (int it = 0; it < P.tpc; it++) {
      const uint32_t tile = blockIdx.x * (uint32_t)P.tpc + it;
      if (tile >= P.num_tiles) break;
      const TileCtx c = decode_tile(P, tile);
      if (it > 0) __syncthreads();
      issue(c, s_buf0);
      cp_async_commit();
      cp_async_wait<0>();
      __syncthreads();
      drain(c, s_buf0);
    }
  } else {
    uint32_t tile = blockIdx.x;
    TileCtx cur = decode_tile(P, tile < P.num_tiles ? tile : 0);
    if (tile < P.num_tiles) issue(cur, s_buf0);
    cp_async_commit();
    for (int k = 0; tile < P.num_tiles; k++) {
      const uint32_t next = tile + gridDim.x;
      TileCtx nx = cur;
      if (next < P.num_tiles) {
        nx = decode_tile(P, next);
        issue(nx, (k & 1) ? s_buf0 : s_buf1);
      }
      cp_async_commit();
      cp_async_wait<1>();
      __syncthreads();
      drain(cur, (k & 1) ? s_buf1 : s_buf0);
      __syncthreads();
      cur = nx;
      tile = next;
    }
    cp_async_wait<0>();
  }
}

// ---------------------------------------------------------------------------
// launch plumbing
template <int W, bool GA32, bool PERSIST, bool XT>
static const void *kernel_ptr_pipe(int nj, bool gb32) {
  if (!gb32) return (const void *)k_pipe<W, 1, GA32, false, PERSIST, XT>;  // LB < 32: one slot
  switch (nj) {
    case 1: return (const void *)k_pipe<W, 1, GA32, true, PERSIST, XT>;
    case 2: return (const void *)k_pipe<W, 2, GA32, true, PERSIST, XT>;
    case 4: return (const void *)k_pipe<W, 4, GA32, true, PERSIST, XT>;
    case 8: return (const void *)k_pipe<W, 8, GA32, true, PERSIST, XT>;
  }
  return (const void *)k_pipe<W, 16, GA32, true, PERSIST, XT>;  // LB <= 512 (planner cap)
}

template <int W, bool XT>
static const void *kernel_ptr_x(int kind, int nj, bool ga32, bool gb32) {
  if (kind == KK_PIPE)
    return ga32 ? kernel_ptr_pipe<W, true, true, XT>(nj, gb32)
                : kernel_ptr_pipe<W, false, true, XT>(nj, gb32);
  return ga32 ? kernel_ptr_pipe<W, true, false, XT>(nj, gb32)
              : kernel_ptr_pipe<W, false, false, XT>(nj, gb32);
}

template <int W>
static const void *kernel_ptr_w(int kind, int nj, bool ga32, bool gb32, bool xt) {
  if (kind == KK_DIRECT) return (const void *)k_direct<W, 8, true>;
  return xt ? kernel_ptr_x<W, true>(kind, nj, ga32, gb32)
            : kernel_ptr_x<W, false>(kind, nj, ga32, gb32);
}

static int pow2_at_least(int k) {
  int p = 1;
  while (p < k) p <<= 1;
  return p;
}

// per-lane elements of a B-row (NJ <= 16)
static int nj_of(const TileParams &K) {
  const int k = pow2_at_least((K.LB + (1 << K.lgB) - 1) >> K.lgB);
  return k <= 16 ? k : 16;  // longer runs: single output digit, chunked (planner rule)
}

static const void *kernel_ptr(int kind, int W, int nj, bool ga32, bool gb32, bool xt) {
  switch (W) {
    case 4: return kernel_ptr_w<4>(kind, nj, ga32, gb32, xt);
    case 8: return kernel_ptr_w<8>(kind, nj, ga32, gb32, xt);
    case 16: return kernel_ptr_w<16>(kind, nj, ga32, gb32, xt);
  }
  return nullptr;
}

static int widx(int W) { return W == 4 ? 0 : (W == 8 ? 1 : 2); }

int kernel_regs(int kind, int W) {
  static int regs[KK_NUM][3] = {{-1, -1, -1}, {-1, -1, -1}, {-1, -1, -1}};
  static std::mutex mu;
  std::lock_guard<std::mutex> g(mu);
  int &r = regs[kind][widx(W)];
  if (r < 0) {
    cudaFuncAttributes attr;
    if (cudaFuncGetAttributes(&attr, kernel_ptr(kind, W, 4, true, true, false)) == cudaSuccess) {
      r = attr.numRegs;
    } else {
      cudaGetLastError();
      r = 0;
    }
  }
  return r;
}

ttlg_status launch(const ttlg_plan_s *plan, const void *A, void *B, void *stream) {
  const void *fn = kernel_ptr(plan->kind, plan->W, nj_of(plan->kp), plan->kp.lgA == 5,
                              plan->kp.lgB == 5, plan->kp.xtab != 0);
  if (!fn) return TTLG_ERR_INTERNAL;
  const int smem = plan->kp.smem_bytes;
  if (smem > 48 * 1024) {
    // opt in once per (kernel instantiation, device)
    static std::mutex mu;
    static const void *done[64][16];
    static int ndone[16];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 16) return TTLG_ERR_DEVICE;
    std::lock_guard<std::mutex> g(mu);
    bool found = false;
    for (int i = 0; i < ndone[dev]; i++) found |= done[i][dev] == fn;
    if (!found) {
      if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024) !=
          cudaSuccess)
        return TTLG_ERR_CUDA;
      if (ndone[dev] < 64) done[ndone[dev]++][dev] = fn;
    }
  }
  TileParams kp = plan->kp;
  void *args[] = {(void *)&kp, (void *)&A, (void *)&B};
  cudaError_t e = cudaLaunchKernel(fn, dim3(plan->grid), dim3(plan->threads), args, smem,
                                   (cudaStream_t)stream);
  if (e != cudaSuccess) return TTLG_ERR_CUDA;
  return TTLG_OK;
}

}  // namespace ttlg
