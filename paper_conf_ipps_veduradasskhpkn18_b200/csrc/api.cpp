// api.cpp -- the C ABI declared in include/ttlg.h.
#include <cuda_runtime.h>

#include <cstdlib>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <mutex>
#include <new>

#include "model_coeffs.h"
#include "model_gbt.h"
#include "ttlg_internal.h"

namespace ttlg {

// Virtual B200 profile (no device): 148 SMs, 227 KB opt-in smem per block,
// 228 KB per SM, 2048 threads and 64K registers per SM; HBM copy bandwidth as
// measured by the driver on this pool (MEASURED_PEAKS.json hbm_gbs).
static DeviceProfile virtual_b200() {
  DeviceProfile d;
  d.sms = 148;
  d.smem_per_block_optin = 227 * 1024;
  d.smem_per_sm = 228 * 1024;
  d.max_threads_per_sm = 2048;
  d.regs_per_sm = 65536;
  d.hbm_gbs = 6555.5;
  d.virt = true;
  return d;
}

const DeviceProfile &device_profile(int device) {
  static DeviceProfile cache[16];
  static bool have[16] = {false};
  static DeviceProfile virt = virtual_b200();
  static std::mutex mu;
  if (device < 0 || device >= 16) return virt;
  std::lock_guard<std::mutex> g(mu);
  if (!have[device]) {
    DeviceProfile d = virtual_b200();
    int v;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device) == cudaSuccess) {
      d.sms = v;
      d.virt = false;
      if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, device) ==
          cudaSuccess)
        d.smem_per_block_optin = v;
      if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerMultiprocessor, device) ==
          cudaSuccess)
        d.smem_per_sm = v;
      if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxThreadsPerMultiProcessor, device) ==
          cudaSuccess)
        d.max_threads_per_sm = v;
      if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxRegistersPerMultiprocessor, device) ==
          cudaSuccess)
        d.regs_per_sm = v;
    } else {
      cudaGetLastError();
    }
    cache[device] = d;
    have[device] = true;
  }
  return cache[device];
}

static int current_device() {
  static int ndev = -2;
  if (ndev == -2) {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) {
      cudaGetLastError();
      n = 0;
    }
    ndev = n;
  }
  if (ndev <= 0) return -1;
  int dev = -1;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  return dev;
}

constexpr double kFastPlanSeconds = 150e-6;
// passes shorter than a fast-effort plan: the second fast level (refine 8 /
// rank 6) below 35 us, and below 45 us for rank >= 4 problems, whose level-1
// plans take ~40 us on the GPU box's CPU: 16^6 fp64 (41-us passes) measured
// single/repeated mean 1.034, max 1.08 on level 2 vs 1.042 / 1.51 on level 1
// (r2e40); rank-3 problems of the same size plan fast enough on level 1 and
// lose on level 2 (r2e41: [2, 4096, 4096] fp32 `2 1 0` 1.01 -> 1.18)
constexpr double kFast2PlanSeconds = 35e-6;
constexpr double kFast2PlanSecondsHighRank = 45e-6;

static ttlg_status plan_into(ttlg_plan_s *p, ttlg_dtype dt, int rank, const int64_t *ext,
                             const int32_t *perm, const ttlg_plan_hints *hints,
                             int fast = 0, const int64_t *in_strides = nullptr,
                             const int64_t *out_strides = nullptr) {
  const int dev = current_device();
  ttlg_status st = make_plan(p, dt, rank, ext, perm, hints, device_profile(dev), nullptr, fast,
                             in_strides, out_strides);
  if (st != TTLG_OK) return st;
  p->strided = in_strides || out_strides;
  {
    int64_t acc = 1;
    for (int k = 0; k < rank; k++) {
      p->in_strides[k] = in_strides ? in_strides[k] : acc;
      acc *= ext[k];
    }
    acc = 1;
    for (int i = 0; i < rank; i++) {
      p->out_strides[i] = out_strides ? out_strides[i] : acc;
      acc *= ext[perm[i]];
    }
  }
  p->device = dev;
  p->dt = dt;
  p->rank = rank;
  for (int k = 0; k < rank; k++) {
    p->ext[k] = ext[k];
    p->perm[k] = perm[k];
  }
  p->has_hints = hints != nullptr;
  if (hints) p->hints = *hints;
  return TTLG_OK;
}

// TTLG_SYNC=1: synchronise and check after every launch (debug mode).
static bool getenv_sync() {
  static int v = -1;
  if (v < 0) {
    const char *e = getenv("TTLG_SYNC");
    v = (e && e[0] == '1') ? 1 : 0;
  }
  return v == 1;
}

// n (A, B) pairs of one plan (1 <= n <= kMaxBatch): one launch with grid.y = n
static ttlg_status execute_n(const ttlg_plan_s *p, int n, const void *const *Av,
                             void *const *Bv, void *stream) {
  if (!p || n < 1 || n > kMaxBatch || !Av || !Bv) return TTLG_ERR_INVALID_VALUE;
  const int s = p->dt == TTLG_F64 ? 8 : 4;
  uintptr_t any = 0;
  for (int i = 0; i < n; i++) {
    const uintptr_t a = (uintptr_t)Av[i], b = (uintptr_t)Bv[i];
    if (!a || !b || a % s || b % s) return TTLG_ERR_INVALID_VALUE;
    any |= a | b;
  }
  for (int i = 0; i < n; i++)
    for (int j = 0; j < n; j++) {
      const uintptr_t a = (uintptr_t)Av[i], b = (uintptr_t)Bv[j];
      if (a < b + (uintptr_t)p->spanB && b < a + (uintptr_t)p->spanA) return TTLG_ERR_ALIASING;
    }
  if (p->device < 0) return TTLG_ERR_DEVICE;
  int dev = -1;
  if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) {
    cudaGetLastError();
    return TTLG_ERR_DEVICE;
  }
  if (any % (uintptr_t)p->align) {
    // widened / 16-byte-vector access needs aligned pointers: run the plan's
    // element-width twin (elem_bytes_override also rules out k_quad and
    // k_deint), planned once on first use and kept in the plan.  Only the
    // caller's schema / no_fusion hints carry over: slice, kernel and block
    // hints describe the widened problem (ttlg_plan_tune's winners carry them).
    ttlg_plan_s *q = p->fallback.load(std::memory_order_acquire);
    if (!q) {
      q = new (std::nothrow) ttlg_plan_s;
      if (!q) return TTLG_ERR_NO_MEMORY;
      ttlg_plan_hints h;
      ttlg_plan_hints_init(&h);
      h.elem_bytes_override = s;
      if (p->has_hints) {
        h.schema = p->hints.schema;
        h.no_fusion = p->hints.no_fusion;
      }
      const int64_t *isx = p->strided ? p->in_strides : nullptr;
      const int64_t *osx = p->strided ? p->out_strides : nullptr;
      ttlg_status st = plan_into(q, (ttlg_dtype)p->dt, p->rank, p->ext, p->perm, &h, false, isx, osx);
      if (st != TTLG_OK && h.schema != TTLG_SCHEMA_AUTO) {
        // a schema of the widened problem (e.g. OD on a squeezed pencil) need
        // not exist at element width; the bytes are the same under any schema
        h.schema = TTLG_SCHEMA_AUTO;
        st = plan_into(q, (ttlg_dtype)p->dt, p->rank, p->ext, p->perm, &h, false, isx, osx);
      }
      if (st != TTLG_OK) {
        delete q;
        return st;
      }
      ttlg_plan_s *expected = nullptr;
      if (!p->fallback.compare_exchange_strong(expected, q, std::memory_order_acq_rel)) {
        delete q;  // another thread installed one first
        q = expected;
      }
    }
    ttlg_status st = launch(q, n, Av, Bv, stream);
    if (st == TTLG_OK && getenv_sync()) {
      if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return TTLG_ERR_CUDA;
    }
    return st;
  }
  ttlg_status st = launch(p, n, Av, Bv, stream);
  if (st == TTLG_OK && getenv_sync()) {
    if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) return TTLG_ERR_CUDA;
  }
  return st;
}


static ttlg_status execute(const ttlg_plan_s *p, const void *A, void *B, void *stream) {
  return execute_n(p, 1, &A, &B, stream);
}

// ---- host-buffer pipeline (ttlg_execute_host) --------------------------------
// A is split along one input dim cd into C chunks.  Chunk k's input slab is
// i_cd in [c0, c0+cc): rows of (prod_{j<cd} n_j) * cc elements at pitch
// prod_{j<=cd} n_j (one contiguous block when cd = d-1), copied densely with
// cudaMemcpy2DAsync; its transposition is the same permutation on extents
// with n_cd -> cc, and its output is B restricted to o_pos in [c0, c0+cc)
// (pos = position of cd in perm): rows of (prod_{i<pos} m_i) * cc elements at
// pitch prod_{i<=pos} m_i (contiguous when pos = d-1).  cd maximises the
// narrower of the two row widths (PCIe DMA of narrow rows is slow), so e.g. a
// full reversal splits a middle dim.  H2D, kernel and D2H of successive
// chunks run on three internal streams joined by events, so the
// host->device and device->host PCIe directions overlap.
namespace {
constexpr int kMaxChunks = 32;
struct HostPipe {
  cudaStream_t h2d = nullptr, comp = nullptr, d2h = nullptr;
  cudaEvent_t start = nullptr, done = nullptr, evA[kMaxChunks], evB[kMaxChunks];
  bool ok = false;
  std::once_flag init;
  std::mutex mu;
};
HostPipe g_pipes[16];

// The device's pipe (streams and events created once, on that device: the
// caller has checked that `dev` is current).
HostPipe *host_pipe(int dev) {
  if (dev < 0 || dev >= 16) return nullptr;
  HostPipe &p = g_pipes[dev];
  std::call_once(p.init, [&p]() {
    bool good = cudaStreamCreateWithFlags(&p.h2d, cudaStreamNonBlocking) == cudaSuccess &&
                cudaStreamCreateWithFlags(&p.comp, cudaStreamNonBlocking) == cudaSuccess &&
                cudaStreamCreateWithFlags(&p.d2h, cudaStreamNonBlocking) == cudaSuccess &&
                cudaEventCreateWithFlags(&p.start, cudaEventDisableTiming) == cudaSuccess &&
                cudaEventCreateWithFlags(&p.done, cudaEventDisableTiming) == cudaSuccess;
    for (int i = 0; good && i < kMaxChunks; i++)
      good = cudaEventCreateWithFlags(&p.evA[i], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&p.evB[i], cudaEventDisableTiming) == cudaSuccess;
    if (!good) cudaGetLastError();
    p.ok = good;
  });
  return p.ok ? &p : nullptr;
}
}  // namespace

static ttlg_status execute_host(const ttlg_plan_s *p, const void *A_host, void *B_host,
                                void *A_dev, void *B_dev, cudaStream_t s) {
  const int esize = p->dt == TTLG_F64 ? 8 : 4;
  const int d = p->rank;
  int64_t N = 1, m[TTLG_MAXD];
  for (int k = 0; k < d; k++) N *= p->ext[k];
  for (int i = 0; i < d; i++) m[i] = p->ext[p->perm[i]];
  const int64_t nbytes = N * esize;
  if (p->device < 0) return TTLG_ERR_DEVICE;
  {
    int dev = -1;  // before any stream / event of the device's pipe is touched
    if (cudaGetDevice(&dev) != cudaSuccess || dev != p->device) {
      cudaGetLastError();
      return TTLG_ERR_DEVICE;
    }
  }
  const int64_t want = std::min<int64_t>((int64_t)kMaxChunks, nbytes / (16ll << 20));
  // the split dim: widest narrower row (contiguous side = unbounded)
  int cd = -1, pos = -1;
  int64_t C = 0;
  double best = 0.0;
  for (int k = 0; k < d; k++) {
    const int64_t Ck = std::min<int64_t>(p->ext[k], want);
    if (Ck < 2) continue;
    int pk = 0;
    while (p->perm[pk] != k) pk++;
    int64_t inA = 1, inB = 1;
    for (int j = 0; j < k; j++) inA *= p->ext[j];
    for (int i = 0; i < pk; i++) inB *= m[i];
    const int64_t cc = p->ext[k] / Ck;
    const double wA = (k == d - 1) ? 1e300 : (double)inA * cc * esize;
    const double wB = (pk == d - 1) ? 1e300 : (double)inB * cc * esize;
    const double w = std::min(wA, wB);
    if (w > best) {
      best = w;
      cd = k;
      pos = pk;
      C = Ck;
    }
  }
  HostPipe *hp = (cd >= 0 && best >= 2048.0) ? host_pipe(p->device) : nullptr;
  if (!hp) {  // small, unsplittable or too narrow: one stream, in order
    if (cudaMemcpyAsync(A_dev, A_host, (size_t)nbytes, cudaMemcpyHostToDevice, s) != cudaSuccess)
      return TTLG_ERR_CUDA;
    ttlg_status st = execute(p, A_dev, B_dev, s);
    if (st != TTLG_OK) return st;
    if (cudaMemcpyAsync(B_host, B_dev, (size_t)nbytes, cudaMemcpyDeviceToHost, s) != cudaSuccess)
      return TTLG_ERR_CUDA;
    return TTLG_OK;
  }
  std::lock_guard<std::mutex> g(hp->mu);
  const int64_t nc = p->ext[cd];
  int64_t inA = 1, inB = 1;
  for (int j = 0; j < cd; j++) inA *= p->ext[j];
  for (int i = 0; i < pos; i++) inB *= m[i];
  const int64_t rowsA = N / (inA * nc), rowsB = N / (inB * nc);
  // at most two distinct chunk extents -> two sub-plans
  const int64_t base = nc / C, rem = nc % C;
  ttlg_plan_s sub[2];
  const int64_t subc[2] = {base, base + 1};
  for (int v = 0; v < 2; v++) {
    if (subc[v] == 0 || (v == 1 && rem == 0)) continue;
    int64_t e[TTLG_MAXD];
    for (int k = 0; k < d; k++) e[k] = p->ext[k];
    e[cd] = subc[v];
    ttlg_status st = plan_into(&sub[v], (ttlg_dtype)p->dt, d, e, p->perm,
                               p->has_hints ? &p->hints : nullptr);
    if (st != TTLG_OK) return st;
  }
  if (cudaEventRecord(hp->start, s) != cudaSuccess) return TTLG_ERR_CUDA;
  cudaStreamWaitEvent(hp->h2d, hp->start, 0);
  cudaStreamWaitEvent(hp->comp, hp->start, 0);
  cudaStreamWaitEvent(hp->d2h, hp->start, 0);
  const int64_t per = N / nc;  // elements per index of the split dim
  const unsigned char *Ah = (const unsigned char *)A_host;
  unsigned char *Bh = (unsigned char *)B_host;
  int64_t c0 = 0;
  for (int64_t k = 0; k < C; k++) {
    const int v = k < rem ? 1 : 0;
    const int64_t cc = subc[v];
    unsigned char *a_slab = (unsigned char *)A_dev + c0 * per * esize;
    unsigned char *b_chunk = (unsigned char *)B_dev + c0 * per * esize;
    const size_t wa = (size_t)(inA * cc * esize), wb = (size_t)(inB * cc * esize);
    cudaError_t e = cudaMemcpy2DAsync(a_slab, wa, Ah + c0 * inA * esize,
                                      (size_t)(inA * nc * esize), wa, (size_t)rowsA,
                                      cudaMemcpyHostToDevice, hp->h2d);
    if (e != cudaSuccess) return TTLG_ERR_CUDA;
    cudaEventRecord(hp->evA[k], hp->h2d);
    cudaStreamWaitEvent(hp->comp, hp->evA[k], 0);
    ttlg_status st = execute(&sub[v], a_slab, b_chunk, hp->comp);
    if (st != TTLG_OK) return st;
    cudaEventRecord(hp->evB[k], hp->comp);
    cudaStreamWaitEvent(hp->d2h, hp->evB[k], 0);
    e = cudaMemcpy2DAsync(Bh + c0 * inB * esize, (size_t)(inB * nc * esize), b_chunk, wb, wb,
                          (size_t)rowsB, cudaMemcpyDeviceToHost, hp->d2h);
    if (e != cudaSuccess) return TTLG_ERR_CUDA;
    c0 += cc;
  }
  if (cudaEventRecord(hp->done, hp->d2h) != cudaSuccess) return TTLG_ERR_CUDA;
  if (cudaStreamWaitEvent(s, hp->done, 0) != cudaSuccess) return TTLG_ERR_CUDA;
  return TTLG_OK;
}

}  // namespace ttlg

using namespace ttlg;

extern "C" {

void ttlg_plan_hints_init(ttlg_plan_hints *h) {
  if (!h) return;
  memset(h, 0, sizeof(*h));
  h->schema = TTLG_SCHEMA_AUTO;
  h->in_dim = -1;
  h->out_dim = -1;
}

ttlg_status ttlg_plan_ex(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                         const int32_t *perm, const ttlg_plan_hints *hints) {
  if (!out) return TTLG_ERR_INVALID_VALUE;
  *out = nullptr;
  ttlg_plan_s *p = new (std::nothrow) ttlg_plan_s;
  if (!p) return TTLG_ERR_NO_MEMORY;
  ttlg_status st = plan_into(p, dt, rank, extents, perm, hints);
  if (st != TTLG_OK) {
    delete p;
    return st;
  }
  *out = p;
  return TTLG_OK;
}

ttlg_status ttlg_plan_strided(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                              const int32_t *perm, const int64_t *in_strides,
                              const int64_t *out_strides, const ttlg_plan_hints *hints) {
  if (!out) return TTLG_ERR_INVALID_VALUE;
  *out = nullptr;
  ttlg_plan_s *p = new (std::nothrow) ttlg_plan_s;
  if (!p) return TTLG_ERR_NO_MEMORY;
  ttlg_status st = plan_into(p, dt, rank, extents, perm, hints, false, in_strides, out_strides);
  if (st != TTLG_OK) {
    delete p;
    return st;
  }
  *out = p;
  return TTLG_OK;
}

ttlg_status ttlg_plan(ttlg_plan_t *out, ttlg_dtype dt, int rank, const int64_t *extents,
                      const int32_t *perm) {
  return ttlg_plan_ex(out, dt, rank, extents, perm, nullptr);
}

ttlg_status ttlg_execute(ttlg_plan_t plan, const void *A, void *B, void *stream) {
  return execute(plan, A, B, stream);
}

ttlg_status ttlg_execute_batch(ttlg_plan_t plan, int32_t count, const void *const *A,
                               void *const *B, void *stream) {
  if (!plan || count < 1 || !A || !B) return TTLG_ERR_INVALID_VALUE;
  // validate every pair (and cross-pair aliasing) before the first launch
  for (int i = 0; i < count; i++)
    for (int j = 0; j < count; j++) {
      const uintptr_t a = (uintptr_t)A[i], b = (uintptr_t)B[j];
      if (!a || !b) return TTLG_ERR_INVALID_VALUE;
      if (a < b + (uintptr_t)plan->spanB && b < a + (uintptr_t)plan->spanA)
        return TTLG_ERR_ALIASING;
    }
  for (int32_t i0 = 0; i0 < count; i0 += kMaxBatch) {
    const int n = (int)std::min<int32_t>(kMaxBatch, count - i0);
    ttlg_status st = execute_n(plan, n, A + i0, B + i0, stream);
    if (st != TTLG_OK) return st;
  }
  return TTLG_OK;
}

ttlg_status ttlg_plan_destroy(ttlg_plan_t plan) {
  delete plan;
  return TTLG_OK;
}

ttlg_status ttlg_transpose(ttlg_dtype dt, int rank, const int64_t *extents, const int32_t *perm,
                           const void *A, void *B, void *stream) {
  ttlg_plan_s p;  // single use: no heap, no cache
  // the plan must hide behind the previous launch: when one pass over the
  // data is short (< kFastPlanSeconds at the profile's copy bandwidth) use the
  // fast effort level
  ttlg_status st = validate(dt, rank, extents, perm);
  if (st != TTLG_OK) return st;
  double bytes = 2.0 * (dt == TTLG_F64 ? 8 : 4);
  for (int k = 0; k < rank; k++) bytes *= (double)extents[k];
  const double pass = bytes / (device_profile(current_device()).hbm_gbs * 1e9);
  const double fast2 = rank >= 4 ? kFast2PlanSecondsHighRank : kFast2PlanSeconds;
  int fast = pass < fast2 ? 2 : (pass < kFastPlanSeconds ? 1 : 0);
  static const int forced = [] {  // TTLG_FAST_LEVEL=0/1/2 pins the level (experiments)
    const char *e = getenv("TTLG_FAST_LEVEL");
    return (e && e[0] >= '0' && e[0] <= '2') ? e[0] - '0' : -1;
  }();
  if (forced >= 0) fast = forced;
  st = plan_into(&p, dt, rank, extents, perm, nullptr, fast);
  if (st != TTLG_OK) return st;
  return execute(&p, A, B, stream);
}

ttlg_status ttlg_execute_host(ttlg_plan_t plan, const void *A_host, void *B_host, void *A_dev,
                              void *B_dev, void *stream) {
  if (!plan || !A_host || !B_host || !A_dev || !B_dev) return TTLG_ERR_INVALID_VALUE;
  if (plan->strided) return TTLG_ERR_UNSUPPORTED;  // dense tensors only
  return execute_host(plan, A_host, B_host, A_dev, B_dev, (cudaStream_t)stream);
}

ttlg_status ttlg_predict_time(ttlg_dtype dt, int rank, const int64_t *extents,
                              const int32_t *perm, double *seconds) {
  if (!seconds) return TTLG_ERR_INVALID_VALUE;
  ttlg_plan_s p;
  ttlg_status st = plan_into(&p, dt, rank, extents, perm, nullptr);
  if (st != TTLG_OK) return st;
  *seconds = p.info.predicted_seconds;
  return TTLG_OK;
}

ttlg_status ttlg_plan_candidates(ttlg_dtype dt, int rank, const int64_t *extents,
                                 const int32_t *perm, const ttlg_plan_hints *hints,
                                 ttlg_plan_info *out, int32_t max_out, int32_t *n_out) {
  if (!out || !n_out || max_out < 0) return TTLG_ERR_INVALID_VALUE;
  ttlg_plan_s p;
  CandidateSink sink{out, max_out, 0, false};
  ttlg_status st = make_plan(&p, dt, rank, extents, perm, hints,
                             device_profile(current_device()), &sink);
  *n_out = sink.n;
  return st;
}

ttlg_status ttlg_plan_tune(ttlg_plan_t *plan, const void *A, void *B, void *stream,
                           int32_t max_candidates, double *best_seconds) {
  if (!plan || !*plan || !A || !B || max_candidates < 1) return TTLG_ERR_INVALID_VALUE;
  ttlg_plan_s *p = *plan;
  if (p->device < 0) return TTLG_ERR_DEVICE;
  // the model's ranked short list
  ttlg_plan_info list[kGbtTopK];
  CandidateSink sink{list, std::min<int>(max_candidates, kGbtTopK), 0, true};
  ttlg_plan_s scratch;
  const int64_t *isx = p->strided ? p->in_strides : nullptr;
  const int64_t *osx = p->strided ? p->out_strides : nullptr;
  ttlg_status st = make_plan(&scratch, (ttlg_dtype)p->dt, p->rank, p->ext, p->perm,
                             p->has_hints ? &p->hints : nullptr, device_profile(p->device), &sink,
                             false, isx, osx);
  if (st != TTLG_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess)
    return TTLG_ERR_CUDA;
  ttlg_plan_s *best = nullptr;
  float best_ms = 1e30f;
  for (int i = 0; i < sink.n; i++) {
    const ttlg_plan_info &ci = list[i];
    ttlg_plan_hints h;
    ttlg_plan_hints_init(&h);
    h.schema = ci.schema == TTLG_SCHEMA_COPY ? TTLG_SCHEMA_FML : ci.schema;
    h.in_dim = ci.in_dim;
    h.in_block = ci.tile_extents[ci.in_dim];
    h.out_dim = ci.out_dim;
    h.out_block = ci.tile_extents[ci.fused_perm[ci.out_dim]];
    h.threads = ci.threads;
    h.variant = ci.kernel == KK_TILE    ? 1
                : ci.kernel == KK_PIPE  ? 2
                : ci.kernel == KK_QUAD  ? 3
                : ci.kernel == KK_BULKQ ? 5
                : ci.kernel == KK_BULKG ? 6
                : ci.kernel == KK_VEC   ? 7
                : ci.kernel == KK_TMA   ? 10
                                        : 0;
    if (ci.kernel == KK_BULKQ || ci.kernel == KK_BULKG || ci.kernel == KK_TMA)
      h.threads = ci.threads - 32;  // consumers
    if (ci.kernel == KK_DEINT || ci.kernel == KK_BLK) {  // no slice parameters: the
      ttlg_plan_hints_init(&h);                         // structure fixes the slice
      h.variant = ci.kernel == KK_DEINT ? 4 : 9;
    }
    ttlg_plan_s *q = new (std::nothrow) ttlg_plan_s;
    if (!q) break;
    if (plan_into(q, (ttlg_dtype)p->dt, p->rank, p->ext, p->perm, &h, false, isx, osx) !=
        TTLG_OK) {
      delete q;
      continue;
    }
    float ms = 1e30f;
    bool ok = execute(q, A, B, stream) == TTLG_OK;  // warm-up
    for (int r = 0; ok && r < 3; r++) {
      ok = cudaEventRecord(e0, s) == cudaSuccess && execute(q, A, B, stream) == TTLG_OK &&
           cudaEventRecord(e1, s) == cudaSuccess && cudaEventSynchronize(e1) == cudaSuccess;
      float t = 0;
      if (ok && cudaEventElapsedTime(&t, e0, e1) == cudaSuccess) ms = std::min(ms, t);
    }
    if (ok && ms < best_ms) {
      delete best;
      best = q;
      best_ms = ms;
    } else {
      delete q;
    }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (!best) return TTLG_ERR_INTERNAL;
  best->info.predicted_seconds = best_ms * 1e-3;  // measured
  delete *plan;
  *plan = best;
  if (best_seconds) *best_seconds = best_ms * 1e-3;
  return TTLG_OK;
}

ttlg_status ttlg_plan_describe(ttlg_plan_t plan, ttlg_plan_info *info) {
  if (!plan || !info) return TTLG_ERR_INVALID_VALUE;
  *info = plan->info;
  return TTLG_OK;
}

// ---- peer memory (CUDA IPC) for the fused sharded exchange --------------------
// The allocation base comes from the driver's cuMemGetAddressRange, reached
// through the runtime's entry-point query (no link-time libcuda dependency, so
// the library still loads on a host without a driver).
typedef int (*MemGetAddressRangeFn)(unsigned long long *, size_t *, unsigned long long);

static MemGetAddressRangeFn mem_range_fn() {
  static MemGetAddressRangeFn fn = nullptr;
  static bool tried = false;
  if (!tried) {
    tried = true;
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (MemGetAddressRangeFn)f;
    else
      cudaGetLastError();
  }
  return fn;
}

ttlg_status ttlg_ipc_export(const void *ptr, void *handle, int64_t *offset) {
  if (!ptr || !handle || !offset) return TTLG_ERR_INVALID_VALUE;
  static_assert(sizeof(cudaIpcMemHandle_t) <= TTLG_IPC_HANDLE_BYTES, "IPC handle size");
  MemGetAddressRangeFn fn = mem_range_fn();
  if (!fn) return TTLG_ERR_CUDA;
  unsigned long long base = 0;
  size_t size = 0;
  if (fn(&base, &size, (unsigned long long)(uintptr_t)ptr) != 0) return TTLG_ERR_CUDA;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, (void *)(uintptr_t)base) != cudaSuccess) {
    cudaGetLastError();
    return TTLG_ERR_CUDA;
  }
  memset(handle, 0, TTLG_IPC_HANDLE_BYTES);
  memcpy(handle, &h, sizeof(h));
  *offset = (int64_t)((uintptr_t)ptr - (uintptr_t)base);
  return TTLG_OK;
}

ttlg_status ttlg_ipc_open(const void *handle, int64_t offset, void **ptr) {
  if (!handle || !ptr || offset < 0) return TTLG_ERR_INVALID_VALUE;
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  void *base = nullptr;
  if (cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
    cudaGetLastError();
    return TTLG_ERR_CUDA;
  }
  *ptr = (unsigned char *)base + offset;
  return TTLG_OK;
}

ttlg_status ttlg_ipc_close(void *ptr, int64_t offset) {
  if (!ptr || offset < 0) return TTLG_ERR_INVALID_VALUE;
  if (cudaIpcCloseMemHandle((unsigned char *)ptr - offset) != cudaSuccess) {
    cudaGetLastError();
    return TTLG_ERR_CUDA;
  }
  return TTLG_OK;
}

const char *ttlg_status_string(ttlg_status s) {
  switch (s) {
    case TTLG_OK: return "TTLG_OK";
    case TTLG_ERR_INVALID_VALUE: return "TTLG_ERR_INVALID_VALUE";
    case TTLG_ERR_ALIASING: return "TTLG_ERR_ALIASING";
    case TTLG_ERR_DEVICE: return "TTLG_ERR_DEVICE";
    case TTLG_ERR_CUDA: return "TTLG_ERR_CUDA";
    case TTLG_ERR_NO_MEMORY: return "TTLG_ERR_NO_MEMORY";
    case TTLG_ERR_INTERNAL: return "TTLG_ERR_INTERNAL";
    case TTLG_ERR_UNSUPPORTED: return "TTLG_ERR_UNSUPPORTED";
  }
  return "TTLG_ERR_UNKNOWN";
}

const char *ttlg_schema_name(int schema) {
  switch (schema) {
    case TTLG_SCHEMA_COPY: return "COPY";
    case TTLG_SCHEMA_FML: return "FML";
    case TTLG_SCHEMA_FMS: return "FMS";
    case TTLG_SCHEMA_OD: return "OD";
    case TTLG_SCHEMA_OA: return "OA";
  }
  return "AUTO";
}

int ttlg_version(void) { return TTLG_VERSION; }

const char *ttlg_model_source(void) { return kModelSource; }

}  // extern "C"
