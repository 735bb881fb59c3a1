// kernels.cu -- sm_100a transposition kernels of the B200 TTLG library.
//
// Two kernel families (templated on the access width W = 4/8/16 bytes):
//
//  k_direct  (FML / COPY; Alg. 7): the tile is a
//            contiguous run of A (input dims 0..a, a blocked); every element is
//            read with a coalesced streaming load and written straight to its
//            output row (output run = dim 0, the matching FVI) -- no shared
//            memory for data, only the per-CTA row-offset table.
//
//  k_staged  (OD / OA / FMS; Alg. 2, Alg. 4/5 L868-1020, Alg. 6
//            L1022-1107): the tile (the paper's "slice") is the union of an
//            input-prefix group and an output-prefix group.  Load phase: A-rows
//            of LA contiguous elements -> shared memory; store phase: B-rows of
//            LB contiguous elements <- shared memory through the column table.
//            The shared-memory layout pads every output-only dim so that output
//            position j lands in bank j mod (128/W): conflict-free column reads
//            (generalising the 32x33 pad, L747-749, and FMS's pad, L1104-1107).
//
// Both are persistent: grid = min(tiles, SMs x resident CTAs); every CTA builds
// its row tables once in shared memory (replacing texture-mapped offset arrays,
// L737-745) and then strides over tiles, decoding each tile index with
// fast-divmod (the paper's decode/compute_base, L725-737) and adding strides.
// Loads are issued U at a time before their stores (memory-level parallelism).
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

__device__ __forceinline__ uint32_t fdiv(uint32_t n, const FastDiv &f) {
  return __umulhi(n, f.mul) >> f.shr;  // grid divisors are always >= 2
}

template <bool CS, typename T>
__device__ __forceinline__ T ld_stream(const T *p) {
  if constexpr (CS) return __ldcs(p);
  else return *p;
}
template <bool CS, typename T>
__device__ __forceinline__ void st_stream(T *p, T v) {
  if constexpr (CS) __stcs(p, v);
  else *p = v;
}

// cp.async (LDGSTS): global -> shared without a register round trip.
template <int W>
__device__ __forceinline__ void cp_async(void *smem_ptr, const void *gptr) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem_ptr);
  if constexpr (W == 16)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gptr) : "memory");
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;\n" ::"r"(s), "l"(gptr), "n"(W)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}

struct TileCtx {
  int64_t bA, bB;
  int limA, limB;
};

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

// Row tables: decode row index i over the row digits (first fastest).
#define TTLG_BUILD_ROWS(R, NR, EXT, SG, SS, BLK, TAB, DIG)                   \
  for (int i = threadIdx.x; i < (R); i += blockDim.x) {                      \
    int rem = i, g = 0, s = 0, dg = 0;                                       \
    _Pragma("unroll") for (int k = 0; k < TTLG_MAXD; k++) {                  \
      if (k < (NR)) {                                                        \
        const int e = (EXT)[k];                                              \
        const int cq = rem / e;                                              \
        const int c = rem - cq * e;                                          \
        rem = cq;                                                            \
        g += c * (SG)[k];                                                    \
        s += c * (SS)[k];                                                    \
        if (k == (BLK)) dg = c;                                              \
      }                                                                      \
    }                                                                        \
    (TAB)[i] = make_int2(g, s);                                              \
    (DIG)[i] = dg;                                                           \
  }

template <int W, int U, bool CS>
__global__ void __launch_bounds__(256) k_direct(const __grid_constant__ TileParams P,
                                                const void *__restrict__ Av,
                                                void *__restrict__ Bv) {
  using T = typename Vec<W>::T;
  extern __shared__ __align__(16) unsigned char smem[];
  int2 *tabB = reinterpret_cast<int2 *>(smem + P.off_tabB);
  int *digA = reinterpret_cast<int *>(smem + P.off_digA);
  const T *A = reinterpret_cast<const T *>(Av);
  T *B = reinterpret_cast<T *>(Bv);

  TTLG_BUILD_ROWS(P.RB, P.nrb, P.rb_ext, P.rb_sG, P.rb_sS, P.rb_blk, tabB, digA);
  __syncthreads();

  const int NT = blockDim.x, tid = threadIdx.x;
  const int r0 = tid / P.LB, j0 = tid % P.LB;
  for (uint32_t tile = blockIdx.x; tile < P.num_tiles; tile += gridDim.x) {
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

template <int W, int U, bool CS>
__global__ void __launch_bounds__(256) k_staged(const __grid_constant__ TileParams P,
                                                const void *__restrict__ Av,
                                                void *__restrict__ Bv) {
  using T = typename Vec<W>::T;
  extern __shared__ __align__(16) unsigned char smem[];
  int2 *tabA = reinterpret_cast<int2 *>(smem);
  int2 *tabB = reinterpret_cast<int2 *>(smem + P.off_tabB);
  int *jcol = reinterpret_cast<int *>(smem + P.off_jcol);
  int *digB = reinterpret_cast<int *>(smem + P.off_digB);
  int *digA = reinterpret_cast<int *>(smem + P.off_digA);
  T *data = reinterpret_cast<T *>(smem + P.off_data);
  const T *A = reinterpret_cast<const T *>(Av);
  T *B = reinterpret_cast<T *>(Bv);

  TTLG_BUILD_ROWS(P.RA, P.nra, P.ra_ext, P.ra_sG, P.ra_sS, P.ra_blk, tabA, digB);
  TTLG_BUILD_ROWS(P.RB, P.nrb, P.rb_ext, P.rb_sG, P.rb_sS, P.rb_blk, tabB, digA);
  for (int j = threadIdx.x; j < P.LB; j += blockDim.x) {
    int rem = j, s = 0;
#pragma unroll
    for (int k = 0; k < TTLG_MAXD; k++) {
      if (k < P.nj) {
        const int e = P.j_ext[k];
        const int cq = rem / e;
        s += (rem - cq * e) * P.j_sS[k];
        rem = cq;
      }
    }
    jcol[j] = s;
  }
  __syncthreads();

  const int tid = threadIdx.x;
  const int rA0 = tid / P.LA, xA0 = tid % P.LA;
  const int rB0 = tid / P.LB, xB0 = tid % P.LB;
  for (uint32_t tile = blockIdx.x; tile < P.num_tiles; tile += gridDim.x) {
    const TileCtx c = decode_tile(P, tile);
    const bool full = (c.limA == P.blkA_t) && (c.limB == P.blkB_t);
    const int LAlim = P.LAunit * c.limA, LBlim = P.LBunit * c.limB;
    // ---- load phase: coalesced A-row reads -> shared memory
    {
      const T *Ab = A + c.bA;
      int r = rA0, x = xA0;
      while (r < P.RA) {
        T v[U];
        int so[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
          so[u] = -1;
          if (r < P.RA && (full || (x < LAlim && digB[r] < c.limB))) {
            const int2 t = tabA[r];
            v[u] = ld_stream<CS>(Ab + t.x + x);
            so[u] = t.y + x;
          }
          x += P.dxA;
          r += P.drA;
          if (x >= P.LA) {
            x -= P.LA;
            r++;
          }
        }
#pragma unroll
        for (int u = 0; u < U; u++)
          if (so[u] >= 0) data[so[u]] = v[u];
      }
    }
    __syncthreads();
    // ---- store phase: shared memory -> coalesced B-row writes
    {
      T *Bb = B + c.bB;
      int r = rB0, j = xB0;
      while (r < P.RB) {
#pragma unroll
        for (int u = 0; u < U; u++) {
          if (r < P.RB && (full || (j < LBlim && digA[r] < c.limA))) {
            const int2 t = tabB[r];
            st_stream<CS>(Bb + t.x + j, data[t.y + jcol[j]]);
          }
          j += P.dxB;
          r += P.drB;
          if (j >= P.LB) {
            j -= P.LB;
            r++;
          }
        }
      }
    }
    __syncthreads();
  }
}

// k_pipe: the staged schema with the load phase issued as cp.async into one
// of two shared-memory buffers, one tile ahead: tile k+1 streams in while
// tile k is written out, so every CTA keeps a whole tile of loads in flight
// (the B200 replacement of the paper's coarsening for latency hiding, L1115-1136).
template <int W, int U, bool CS>
__global__ void __launch_bounds__(256) k_pipe(const __grid_constant__ TileParams P,
                                              const void *__restrict__ Av,
                                              void *__restrict__ Bv) {
  using T = typename Vec<W>::T;
  extern __shared__ __align__(16) unsigned char smem[];
  int2 *tabA = reinterpret_cast<int2 *>(smem);
  int2 *tabB = reinterpret_cast<int2 *>(smem + P.off_tabB);
  int *jcol = reinterpret_cast<int *>(smem + P.off_jcol);
  int *digB = reinterpret_cast<int *>(smem + P.off_digB);
  int *digA = reinterpret_cast<int *>(smem + P.off_digA);
  T *buf0 = reinterpret_cast<T *>(smem + P.off_data);
  T *buf1 = reinterpret_cast<T *>(smem + P.off_data2);
  const T *A = reinterpret_cast<const T *>(Av);
  T *B = reinterpret_cast<T *>(Bv);

  TTLG_BUILD_ROWS(P.RA, P.nra, P.ra_ext, P.ra_sG, P.ra_sS, P.ra_blk, tabA, digB);
  TTLG_BUILD_ROWS(P.RB, P.nrb, P.rb_ext, P.rb_sG, P.rb_sS, P.rb_blk, tabB, digA);
  for (int j = threadIdx.x; j < P.LB; j += blockDim.x) {
    int rem = j, s = 0;
#pragma unroll
    for (int k = 0; k < TTLG_MAXD; k++) {
      if (k < P.nj) {
        const int e = P.j_ext[k];
        const int cq = rem / e;
        s += (rem - cq * e) * P.j_sS[k];
        rem = cq;
      }
    }
    jcol[j] = s;
  }
  __syncthreads();

  const int tid = threadIdx.x;
  const int rA0 = tid / P.LA, xA0 = tid % P.LA;
  const int rB0 = tid / P.LB, xB0 = tid % P.LB;

  auto issue = [&](const TileCtx &c, T *buf) {
    const bool full = (c.limA == P.blkA_t) && (c.limB == P.blkB_t);
    const int LAlim = P.LAunit * c.limA;
    const T *Ab = A + c.bA;
    int r = rA0, x = xA0;
    while (r < P.RA) {
      if (full || (x < LAlim && digB[r] < c.limB)) {
        const int2 t = tabA[r];
        cp_async<W>(buf + t.y + x, Ab + t.x + x);
      }
      x += P.dxA;
      r += P.drA;
      if (x >= P.LA) {
        x -= P.LA;
        r++;
      }
    }
  };

  uint32_t tile = blockIdx.x;
  TileCtx cur = decode_tile(P, tile < P.num_tiles ? tile : 0);
  if (tile < P.num_tiles) issue(cur, buf0);
  cp_async_commit();
  for (int k = 0; tile < P.num_tiles; k++) {
    const uint32_t next = tile + gridDim.x;
    TileCtx nx = cur;
    if (next < P.num_tiles) {
      nx = decode_tile(P, next);
      issue(nx, (k & 1) ? buf0 : buf1);
    }
    cp_async_commit();
    cp_async_wait<1>();
    __syncthreads();
    {
      const T *data = (k & 1) ? buf1 : buf0;
      const bool full = (cur.limA == P.blkA_t) && (cur.limB == P.blkB_t);
      const int LBlim = P.LBunit * cur.limB;
      T *Bb = B + cur.bB;
      int r = rB0, j = xB0;
      while (r < P.RB) {
#pragma unroll
        for (int u = 0; u < U; u++) {
          if (r < P.RB && (full || (j < LBlim && digA[r] < cur.limA))) {
            const int2 t = tabB[r];
            st_stream<CS>(Bb + t.x + j, data[t.y + jcol[j]]);
          }
          j += P.dxB;
          r += P.drB;
          if (j >= P.LB) {
            j -= P.LB;
            r++;
          }
        }
      }
    }
    __syncthreads();
    cur = nx;
    tile = next;
  }
  cp_async_wait<0>();
}

// ---------------------------------------------------------------------------
// launch plumbing
template <int W, bool CS>
static const void *kernel_ptr_w(int kind) {
  constexpr int U = (W == 16) ? 4 : 8;
  switch (kind) {
    case KK_DIRECT: return (const void *)k_direct<W, U, CS>;
    case KK_STAGED: return (const void *)k_staged<W, U, CS>;
    case KK_PIPE: return (const void *)k_pipe<W, U, CS>;
  }
  return nullptr;
}

static const void *kernel_ptr(int kind, int W, bool cs) {
  switch (W) {
    case 4: return cs ? kernel_ptr_w<4, true>(kind) : kernel_ptr_w<4, false>(kind);
    case 8: return cs ? kernel_ptr_w<8, true>(kind) : kernel_ptr_w<8, false>(kind);
    case 16: return cs ? kernel_ptr_w<16, true>(kind) : kernel_ptr_w<16, false>(kind);
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
    if (cudaFuncGetAttributes(&attr, kernel_ptr(kind, W, true)) == cudaSuccess) {
      r = attr.numRegs;
    } else {
      cudaGetLastError();
      r = 0;
    }
  }
  return r;
}

ttlg_status launch(const ttlg_plan_s *plan, const void *A, void *B, void *stream) {
  const bool cs = !(plan->variant & 2);
  const void *fn = kernel_ptr(plan->kind, plan->W, cs);
  if (!fn) return TTLG_ERR_INTERNAL;
  const int smem = plan->kp.smem_bytes;
  if (smem > 48 * 1024) {
    // opt in once per (kernel variant, device)
    static bool done[KK_NUM][3][2][16];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 16) return TTLG_ERR_DEVICE;
    bool &d = done[plan->kind][widx(plan->W)][cs][dev];
    if (!d) {
      if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024) !=
          cudaSuccess)
        return TTLG_ERR_CUDA;
      d = true;
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
