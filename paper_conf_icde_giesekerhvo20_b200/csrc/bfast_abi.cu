// bfast_abi.cu -- host side of libbfast.so: argument validation, plans
// (design matrix in fp64 -> fp32 device constants), kernel launches, the
// host-buffer (end-to-end) path and the multi-device shard driver.
// Declarations and contracts: include/bfast.h.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <map>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/bfast.h"
#include "monitor_simt.cuh"
#include "monitor_fused.cuh"
#include "refit_fp64.cuh"
#include "preprocess.cuh"

namespace {

thread_local std::string g_err;
thread_local int g_launches = 0;
thread_local bool g_prof_on = false;
thread_local std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_prof;

int fail(int status, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return status;
}

#define CUDA_TRY(expr)                                                                 \
  do {                                                                                 \
    cudaError_t e_ = (expr);                                                           \
    if (e_ != cudaSuccess)                                                             \
      return fail(e_ == cudaErrorMemoryAllocation ? BFAST_ENOMEM : BFAST_ECUDA,        \
                  "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

constexpr int kMaxSmem = 227 * 1024;    // per CTA
constexpr size_t kSmemPerSM = 228 * 1024;  // per SM (B200)

int validate_scalar(int64_t N, const double *dates, int32_t n_hist, int32_t k, float h,
                    float lambda) {
  if (N < 2) return fail(BFAST_EINVAL, "N=%lld < 2", (long long)N);
  if (N > 32767) return fail(BFAST_EUNSUPPORTED, "N=%lld > 32767 dates", (long long)N);
  if (n_hist < 1 || n_hist > N - 1)
    return fail(BFAST_EINVAL, "n_hist=%d outside [1, N-1]", n_hist);
  if (k < 0) return fail(BFAST_EINVAL, "k=%d < 0", k);
  if (!(h > 0.f && h <= 1.f)) return fail(BFAST_EINVAL, "h=%g outside (0, 1]", (double)h);
  if (!(lambda > 0.f) || !std::isfinite(lambda))
    return fail(BFAST_EINVAL, "lambda=%g must be finite and > 0", (double)lambda);
  if (!dates) return fail(BFAST_EINVAL, "dates is NULL");
  for (int64_t t = 0; t < N; ++t) {
    if (!std::isfinite(dates[t])) return fail(BFAST_EINVAL, "dates[%lld] not finite", (long long)t);
    if (t && !(dates[t] > dates[t - 1]))
      return fail(BFAST_EINVAL, "dates not strictly increasing at %lld", (long long)t);
  }
  if (k > BFAST_K_MAX_HARMONICS)
    return fail(BFAST_EUNSUPPORTED, "k=%d > %d", k, BFAST_K_MAX_HARMONICS);
  return BFAST_OK;
}

int host_window(int nbar, float hf) {  // Fig. 12 L516 in f32, as the kernel
  volatile float prod = (float)nbar * hf;
  return (int)prod;
}

}  // namespace

struct bfast_plan {
  int device = 0;
  int64_t N = 0;
  int32_t n = 0, k = 0, K = 0, KP = 0;
  float hf = 0.f, lambda = 0.f;
  std::vector<double> dates;
  double tc = 0.0, ts = 1.0;
  int hcap = 1;
  float *dX = nullptr;      // [N][KP] fp32
  double *dX64 = nullptr;   // [N][K] fp64
  int32_t *dcount = nullptr;
  int *dprobe = nullptr;  // window probe result (max h over a sample)
  int64_t *dlist = nullptr;
  int64_t list_cap = 0;
  cudaEvent_t scratch_free = nullptr;  // orders executions sharing the refit scratch
  // bfast_monitor_host: double-buffered device slabs, a copy and a compute
  // stream, and their events, owned by the plan and reused across calls
  // (allocated on first use, grown when a call needs a wider slab)
  struct HostPath {
    int64_t slab = 0;
    float *dY[2] = {nullptr, nullptr};
    int32_t *dB[2] = {nullptr, nullptr};
    float *dM[2] = {nullptr, nullptr};
    // pinned staging of each slab's results: a D2H into pageable caller
    // memory would block the host thread until the slab's kernel is done and
    // so serialise the next slab's upload behind it
    int32_t *hB[2] = {nullptr, nullptr};
    float *hM[2] = {nullptr, nullptr};
    cudaStream_t cs = nullptr, ks = nullptr;
    cudaEvent_t loaded[2] = {nullptr, nullptr}, done[2] = {nullptr, nullptr};
  } host;
  // fused kernel (monitor_fused.cuh): per-chunk tables of passes A, B, C
  uint8_t *dtabf = nullptr;
  size_t tabfB_off = 0, tabfC_off = 0;
  // NaN-free history: the Cholesky factor of the
  // common Gram sum_{t<n} x_t x_t^T, fp64 on the host, in the kernel's
  // register layout (FzTables::shared); nullptr when the history Gram is
  // singular
  float *dshared = nullptr;
  int nch = 0, ncm = 0;
  int mode = 0;  // 0 fused tensor-core kernel, 1 SIMT kernel only (BFAST_KERNEL=simt at plan creation)
  std::mutex mu;
  ~bfast_plan() {
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    cudaFree(dX);
    cudaFree(dX64);
    cudaFree(dcount);
    cudaFree(dprobe);
    cudaFree(dlist);
    cudaFree(dtabf);
    cudaFree(dshared);
    if (scratch_free) cudaEventDestroy(scratch_free);
    for (int i = 0; i < 2; ++i) {
      cudaFree(host.dY[i]);
      cudaFree(host.dB[i]);
      cudaFree(host.dM[i]);
      cudaFreeHost(host.hB[i]);
      cudaFreeHost(host.hM[i]);
      if (host.loaded[i]) cudaEventDestroy(host.loaded[i]);
      if (host.done[i]) cudaEventDestroy(host.done[i]);
    }
    if (host.cs) cudaStreamDestroy(host.cs);
    if (host.ks) cudaStreamDestroy(host.ks);
    if (prev >= 0) cudaSetDevice(prev);
  }
};

namespace {

// Design matrix of Eq. (3) (L65-L68) in fp64, with the trend regressor
// centred and scaled, t' = (t - tc)/ts; rows padded
// to KP columns.
void build_design(const bfast_plan &pl, std::vector<float> &X, std::vector<double> &X64) {
  const double two_pi = 6.283185307179586476925286766559;
  X.assign((size_t)pl.N * pl.KP, 0.f);
  X64.assign((size_t)pl.N * pl.K, 0.0);
  for (int64_t t = 0; t < pl.N; ++t) {
    double row[2 + 2 * BFAST_K_MAX_HARMONICS];
    row[0] = 1.0;
    row[1] = ((double)(t + 1) - pl.tc) / pl.ts;
    for (int j = 1; j <= pl.k; ++j) {
      double F = two_pi * (double)j * pl.dates[t];
      row[2 * j] = std::sin(F);
      row[2 * j + 1] = std::cos(F);
    }
    for (int i = 0; i < pl.K; ++i) {
      X[(size_t)t * pl.KP + i] = (float)row[i];
      X64[(size_t)t * pl.K + i] = row[i];
    }
  }
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no
// link-time dependency on libcuda).
typedef CUresult (*PFN_encodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                    const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
PFN_encodeTiled get_encode() {
  static PFN_encodeTiled fn = nullptr;
  static std::once_flag once;
  std::call_once(once, []() {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_encodeTiled)f;
  });
  return fn;
}

// Tensor map of the stack range [p0, p0+P) x [0, N): box `pix` px x 16 dates
// (one tile), out-of-bounds elements read as NaN (= missing).
bool make_stack_map(CUtensorMap *m, const void *Y, int64_t ldY, int64_t P, int64_t N, int pix, int dates = 16,
                    bool i16 = false) {
  PFN_encodeTiled enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)P, (cuuint64_t)N};
  cuuint64_t strides[1] = {(cuuint64_t)ldY * (i16 ? 2 : 4)};
  cuuint32_t box[2] = {(cuuint32_t)pix, (cuuint32_t)dates};
  cuuint32_t es[2] = {1, 1};
  // float32: out-of-bounds elements read as NaN (= missing); int16 codes:
  // zero (the kernel marks a period's dates past its end itself)
  return enc(m, i16 ? CU_TENSOR_MAP_DATA_TYPE_UINT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)Y, dims, strides,
             box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             i16 ? CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE : CU_TENSOR_MAP_FLOAT_OOB_FILL_NAN_REQUEST_ZERO_FMA) ==
         CUDA_SUCCESS;
}

uint16_t bf16_rne(double v) {
  float f = (float)v;
  uint32_t u;
  std::memcpy(&u, &f, 4);
  if ((u & 0x7f800000u) == 0x7f800000u) return (uint16_t)(u >> 16);
  u += 0x7fffu + ((u >> 16) & 1u);
  return (uint16_t)(u >> 16);
}
double bf16_val(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  std::memcpy(&f, &u, 4);
  return (double)f;
}
void split3(double v, uint16_t &h, uint16_t &m, uint16_t &l) {
  h = bf16_rne(v);
  m = bf16_rne(v - bf16_val(h));
  l = bf16_rne(v - bf16_val(h) - bf16_val(m));
}
inline size_t kmaj(int row, int k, int rows) { return sm100::kmajor_off(row, k, rows) / 2; }

// Chunk tables of the fused kernel (monitor_fused.cuh), B operands in the
// canonical K-major layout, fp64 values split into bf16 parts:
//   A[c] (history chunk c, pass A): F_hi | F_mid | F_lo ([NGn x 16] each;
//        row q = moment function f_q, the last one the constant 1; column d
//        = date 16c + d) | x_hi | x_mid ([KBn x 16] each, the first moment);
//   B[c] (history chunk c, pass B): the yhat table [16 x KY] (row d = date;
//        K index = 6 blocks of K: x_hi | x_mid | x_lo | x_hi | x_mid | x_hi,
//        paired in the GEMM with beta hi | hi | hi | mid | mid | lo) | x_hi |
//        x_mid | x_lo ([KBn x 16] each, the refinement moment);
//   C[c] (monitoring chunk c): the yhat table of dates n + 16c + d.
template <int K>
void build_fz_tables(const bfast_plan &pl, std::vector<uint16_t> &tab, size_t &offB, size_t &offC) {
  using C = bfast::FzCfg<K>;
  const int k = pl.k, n = pl.n, N = (int)pl.N, DC = C::DC;
  const int nch = (n + DC - 1) / DC, ncm = (N - n + DC - 1) / DC;
  const double two_pi = 6.283185307179586476925286766559;
  auto xrow = [&](int t, double *x) {
    const double tau = ((double)(t + 1) - pl.tc) / pl.ts, th = two_pi * pl.dates[t];
    x[0] = 1.0;
    x[1] = tau;
    for (int j = 1; j <= k; ++j) {
      x[2 * j] = std::sin(j * th);
      x[2 * j + 1] = std::cos(j * th);
    }
  };
  auto frow = [&](int t, double *f) {  // tau, tau^2, tau sin_j, tau cos_j, sin_m, cos_m, 1
    const double tau = ((double)(t + 1) - pl.tc) / pl.ts, th = two_pi * pl.dates[t];
    f[0] = tau;
    f[1] = tau * tau;
    for (int j = 1; j <= k; ++j) {
      f[2 + 2 * (j - 1)] = tau * std::sin(j * th);
      f[3 + 2 * (j - 1)] = tau * std::cos(j * th);
    }
    for (int m = 1; m <= 2 * k; ++m) {
      f[2 + 2 * k + 2 * (m - 1)] = std::sin(m * th);
      f[3 + 2 * k + 2 * (m - 1)] = std::cos(m * th);
    }
    f[C::NF] = 1.0;  // the constant function: its masked moment is nbar
  };
  const size_t TA = C::TABA / 2, TB = C::TABB / 2, TC = C::TABC / 2;
  tab.assign((size_t)nch * (TA + TB) + (size_t)ncm * TC, 0);
  offB = (size_t)nch * TA;
  offC = offB + (size_t)nch * TB;
  double x[2 + 2 * BFAST_K_MAX_HARMONICS], f[3 + 6 * BFAST_K_MAX_HARMONICS];
  auto put_b3 = [&](uint16_t *b3, int d, const double *xv) {  // [16 x KY]: xh|xm|xl|xh|xm|xh
    for (int i = 0; i < K; ++i) {
      uint16_t h, m, l;
      split3(xv[i], h, m, l);
      const uint16_t blk[6] = {h, m, l, h, m, h};
      for (int b = 0; b < 6; ++b) b3[kmaj(d, b * K + i, C::DC)] = blk[b];
    }
  };
  auto put_bx = [&](uint16_t *bx, int d, const double *xv, int parts) {  // parts x [KBn x 16]
    for (int i = 0; i < K; ++i) {
      uint16_t h, m, l;
      split3(xv[i], h, m, l);
      const uint16_t prt[3] = {h, m, l};
      for (int e = 0; e < parts; ++e) bx[e * C::BX_BYTES / 2 + kmaj(i, d, C::KBn)] = prt[e];
    }
  };
  for (int c = 0; c < nch; ++c) {
    uint16_t *ta = tab.data() + (size_t)c * TA;
    uint16_t *tb = tab.data() + offB + (size_t)c * TB;
    for (int d = 0; d < DC; ++d) {
      const int t = c * DC + d;
      if (t >= n) continue;
      xrow(t, x);
      frow(t, f);
      for (int q = 0; q <= C::NF; ++q) {
        uint16_t h, m, l;
        split3(f[q], h, m, l);
        const uint16_t prt[3] = {h, m, l};
        for (int e = 0; e < 3; ++e) ta[e * C::BF_BYTES / 2 + kmaj(q, d, C::NGn)] = prt[e];
      }
      put_bx(ta + 3 * C::BF_BYTES / 2, d, x, 2);
      put_b3(tb, d, x);
      put_bx(tb + C::B3_BYTES / 2, d, x, 3);
    }
  }
  for (int c = 0; c < ncm; ++c) {
    uint16_t *tcp = tab.data() + offC + (size_t)c * TC;
    for (int d = 0; d < DC; ++d) {
      const int t = n + c * DC + d;
      if (t >= N) continue;
      xrow(t, x);
      put_b3(tcp, d, x);
    }
  }
}

// f3 (the [27] special case): every pixel whose
// history has no missing value shares the Gram A = sum_{t<n} x_t x_t^T, so
// its factor is computed once: Cholesky in fp64, rounded to fp32 in the
// layout fz_chol leaves (Tri<K>: idx(j, j) = A_jj, idx(q, i) = L_iq for q <
// i), then the K reciprocal pivots, the smallest pivot ratio d_j / A_jj and
// the largest variance inflation factor A_jj (A^-1)_jj (the fused kernel's
// fp64-refit triggers, here exact).  Returns false if A is not positive
// definite (the kernel then factors every pixel itself).
bool shared_factor(const bfast_plan &pl, std::vector<float> &out) {
  const int K = pl.K;
  std::vector<float> Xf;
  std::vector<double> X64;
  build_design(pl, Xf, X64);
  std::vector<double> A((size_t)K * K, 0.0), L((size_t)K * K, 0.0);
  for (int t = 0; t < pl.n; ++t)
    for (int i = 0; i < K; ++i)
      for (int j = 0; j < K; ++j) A[i * K + j] += X64[(size_t)t * K + i] * X64[(size_t)t * K + j];
  double minratio = 1.0;
  for (int j = 0; j < K; ++j) {
    double d = A[j * K + j];
    for (int q = 0; q < j; ++q) d -= L[j * K + q] * L[j * K + q];
    if (!(d > 0.0)) return false;
    minratio = std::min(minratio, d / A[j * K + j]);
    L[j * K + j] = std::sqrt(d);
    for (int i = j + 1; i < K; ++i) {
      double v = A[j * K + i];
      for (int q = 0; q < j; ++q) v -= L[i * K + q] * L[j * K + q];
      L[i * K + j] = v / L[j * K + j];
    }
  }
  // (A^-1)_jj = sum_i (L^-1)_ij^2
  double vif = 0.0;
  for (int j = 0; j < K; ++j) {
    std::vector<double> m(K, 0.0);
    m[j] = 1.0 / L[j * K + j];
    double ss = m[j] * m[j];
    for (int i = j + 1; i < K; ++i) {
      double v = 0.0;
      for (int q = j; q < i; ++q) v += L[i * K + q] * m[q];
      m[i] = -v / L[i * K + i];
      ss += m[i] * m[i];
    }
    vif = std::max(vif, ss * A[j * K + j]);
  }
  const int kN = K * (K + 1) / 2;
  out.assign((size_t)kN + K + 2, 0.f);
  auto tri = [&](int i, int j) { return i * K - i * (i - 1) / 2 + (j - i); };  // Tri<K>::idx, i <= j
  for (int j = 0; j < K; ++j) {
    out[tri(j, j)] = (float)A[j * K + j];
    for (int i = j + 1; i < K; ++i) out[tri(j, i)] = (float)L[i * K + j];
    out[kN + j] = (float)(1.0 / L[j * K + j]);
  }
  out[kN + K] = (float)minratio;
  out[kN + K + 1] = (float)vif;
  return true;
}

int build_fz(bfast_plan &pl) {
  {
    std::vector<float> sf;
    if (shared_factor(pl, sf)) {
      CUDA_TRY(cudaMalloc(&pl.dshared, sf.size() * sizeof(float)));
      CUDA_TRY(cudaMemcpy(pl.dshared, sf.data(), sf.size() * sizeof(float), cudaMemcpyHostToDevice));
    }
  }
  std::vector<uint16_t> tab;
  size_t ob = 0, oc = 0;
  switch (pl.k) {
    case 0: build_fz_tables<2>(pl, tab, ob, oc); break;
    case 1: build_fz_tables<4>(pl, tab, ob, oc); break;
    case 2: build_fz_tables<6>(pl, tab, ob, oc); break;
    case 3: build_fz_tables<8>(pl, tab, ob, oc); break;
    case 4: build_fz_tables<10>(pl, tab, ob, oc); break;
    case 5: build_fz_tables<12>(pl, tab, ob, oc); break;
    case 6: build_fz_tables<14>(pl, tab, ob, oc); break;
    default: return BFAST_EUNSUPPORTED;
  }
  pl.tabfB_off = ob * 2;
  pl.tabfC_off = oc * 2;
  CUDA_TRY(cudaMalloc(&pl.dtabf, tab.size() * 2));
  CUDA_TRY(cudaMemcpy(pl.dtabf, tab.data(), tab.size() * 2, cudaMemcpyHostToDevice));
  return BFAST_OK;
}

size_t simt_smem(const bfast_plan &pl, int bp) {
  return (size_t)pl.N * pl.KP * sizeof(float) + (size_t)pl.hcap * bp * (sizeof(float) + sizeof(int16_t));
}

// The fused kernel (monitor_fused.cuh): T tiles of 128 pixels per CTA, the
// largest T whose shared memory fits (the MOSUM ring grows with the window
// hcap = floor(hf * n)), as many CTAs per SM as shared memory, TMEM and
// registers admit, and a persistent grid over the tile groups.
// Returns BFAST_OK with `done` = false when the stack cannot be read by TMA
// (row pitch not a multiple of 16 bytes): the caller falls back to SIMT.
// the kernel argument of single-period launches (unused there)
const bfast::FzMulti &no_multi() {
  static const bfast::FzMulti m{};
  return m;
}

template <int K, bool I16, bool MULTI, bool CLAMP = false, bool DENSE = false>
int fused_config(int device, cudaFuncAttributes &fa) {
  static thread_local int configured_dev = -1;
  CUDA_TRY(cudaFuncGetAttributes(&fa, bfast::monitor_fused_kernel<K, I16, MULTI, CLAMP, DENSE>));
  if (configured_dev != device) {
    CUDA_TRY(cudaFuncSetAttribute(bfast::monitor_fused_kernel<K, I16, MULTI, CLAMP, DENSE>,
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmem - (int)fa.sharedSizeBytes));
    CUDA_TRY(cudaFuncSetAttribute(bfast::monitor_fused_kernel<K, I16, MULTI, CLAMP, DENSE>,
                                  cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared));
    configured_dev = device;
  }
  return BFAST_OK;
}

template <int K, bool I16>
int launch_fused(const bfast_plan &pl, const bfast::MonitorParams &prm, cudaStream_t st, bool &done) {
  using C = bfast::FzCfg<K>;
  done = false;
  cudaFuncAttributes fa{};
  {
    const int rc = fused_config<K, I16, false>(pl.device, fa);
    if (rc) return rc;
  }
  const int static_smem = (int)fa.sharedSizeBytes;
  constexpr int esz = I16 ? 2 : 4;
  const void *Ybase = I16 ? (const void *)(prm.Y16 + prm.p0) : (const void *)(prm.Y + prm.p0);
  if (!pl.dtabf || (prm.ldY * esz) % 16 != 0 || ((uintptr_t)Ybase % 16) != 0) return BFAST_OK;
  // tiles per CTA and stack stages: the most tiles that fit with 3 stack
  // stages, else with 2
  int T = C::TMAX, sc = C::SCMAX;
  if (const char *e = std::getenv("BFAST_FZ_T")) T = std::max(1, std::min(C::TMAX, std::atoi(e)));
  if (const char *e = std::getenv("BFAST_FZ_SC")) sc = std::max(2, std::min(C::SCMAX, std::atoi(e)));
  int hcap = pl.hcap;  // MOSUM ring slots per pixel
  auto fits = [&](int t, int c) { return C::smem_bytes(t, hcap, c, esz) + static_smem <= (size_t)kMaxSmem; };
  // the ring sized for a complete history (h = floor(hf n)) costs tiles:
  // size it from the widest window of a sample of the stack (+ a margin;
  // wider windows go to the fp64 refit).  Synchronises the stream once.
  const char *wpe = std::getenv("BFAST_WINDOW_PROBE");
  if (!fits(T, 2) && prm.P >= 32 * 64 && pl.dprobe && !(wpe && wpe[0] == '0')) {
    const int64_t groups = std::min<int64_t>(2048, prm.P / 32);
    const int64_t gstride = prm.P / groups;
    CUDA_TRY(cudaMemsetAsync(pl.dprobe, 0, sizeof(int), st));
    if (I16)
      bfast::window_probe_kernel<int16_t><<<(unsigned)groups, 32, 0, st>>>(
          prm.Y16 + prm.p0, prm.ldY, prm.P, pl.n, pl.hf, gstride, prm.nodata, pl.dprobe);
    else
      bfast::window_probe_kernel<float><<<(unsigned)groups, 32, 0, st>>>(prm.Y + prm.p0, prm.ldY, prm.P, pl.n,
                                                                         pl.hf, gstride, 0, pl.dprobe);
    CUDA_TRY(cudaGetLastError());
    int hmax = 0;
    CUDA_TRY(cudaMemcpyAsync(&hmax, pl.dprobe, sizeof(int), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    hcap = std::min(pl.hcap, std::max(std::min(pl.hcap, 8), hmax + std::max(8, hmax / 8)));
  }
  while (T > 1 && !fits(T, 2)) --T;
  T = std::max(C::TPC, T / C::TPC * C::TPC);  // whole control groups
  if (!fits(T, sc)) sc = 2;
  const size_t smem = C::smem_bytes(T, hcap, sc, esz);
  if (smem + static_smem > (size_t)kMaxSmem)
    return fail(BFAST_EUNSUPPORTED, "fused kernel: shared memory %zu B for window %d", smem, hcap);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, pl.device);
  // CTAs per SM: shared memory (228 KB per SM, 1 KB reserved per CTA), TMEM
  // (512 columns), registers, threads
  const int threads = 128 * (T + 1);  // T consumer warpgroups + the control warpgroup
  const int by_smem = (int)(kSmemPerSM / (smem + static_smem + 1024));
  const int by_tmem = 512 / C::pow2cols(T * C::TCOLS);
  const int by_regs = 65536 / (threads * std::max(fa.numRegs, 1));
  const int by_thr = 2048 / threads;
  const int per_sm = std::max(1, std::min(std::min(by_smem, by_tmem), std::min(by_regs, by_thr)));
  // full stack; history only (dates >= n out of bounds -> NaN); L2 prefetch boxes
  CUtensorMap ymap, hmap, pmap;
  if (!make_stack_map(&ymap, Ybase, prm.ldY, prm.P, pl.N, 128 * C::TPC, 16, I16) ||
      !make_stack_map(&hmap, Ybase, prm.ldY, prm.P, pl.n, 128 * C::TPC, 16, I16) ||
      !make_stack_map(&pmap, Ybase, prm.ldY, prm.P, pl.N, 128 * C::TPC, C::PFB, I16))
    return BFAST_OK;
  // L2 prefetch of first-touch dates ahead of the TMA loads: off (measured
  // -1..-5% without it across the configs in round 2; BFAST_FZ_PFD=128 re-enables)
  int pfd = 0;
  if (const char *e = std::getenv("BFAST_FZ_PFD")) pfd = std::max(0, std::atoi(e)) / C::PFB * C::PFB;
  bfast::FzTables tb{};
  tb.tabA = pl.dtabf;
  tb.tabB = pl.dtabf + pl.tabfB_off;
  tb.tabC = pl.dtabf + pl.tabfC_off;
  // the float an int16 nodata code turns into (monitor_fused.cuh fz_code)
  {
    const uint32_t u = (((uint32_t)(uint16_t)prm.nodata) ^ 0x8000u) | 0x4B000000u;
    std::memcpy(&tb.fnd, &u, 4);
  }
  // f3: BFAST_SHARED_FACTOR=1 launches the instantiation in which warps of
  // complete histories use the plan's fp64 factor (off by default: its warp
  // test costs the cloudy scenes)
  const char *sfe = std::getenv("BFAST_SHARED_FACTOR");
  const bool dense = !I16 && sfe && sfe[0] == '1' && pl.dshared;
  tb.shared = dense ? pl.dshared : nullptr;
  tb.nch = pl.nch;
  tb.ncm = pl.ncm;
  tb.T = T;
  tb.hcap = hcap;
  tb.pfd = pfd;
  tb.sc = sc;
  tb.ntg = (prm.P + 128 * T - 1) / (128 * T);
  const int64_t grid = std::min<int64_t>(tb.ntg, (int64_t)sms * per_sm);
  if (std::getenv("BFAST_VERBOSE"))
    std::fprintf(stderr, "bfast: fused k=%d T=%d sc=%d smem=%zu+%d regs=%d per_sm=%d grid=%lld tile groups=%lld "
                 "ring=%d of %d\n", pl.k, T, sc, smem, static_smem, fa.numRegs, per_sm, (long long)grid,
                 (long long)tb.ntg, hcap, pl.hcap);
  if (dense && hcap == pl.hcap) {
    cudaFuncAttributes fd{};
    const int rc = fused_config<K, false, false, false, true>(pl.device, fd);
    if (rc) return rc;
    bfast::monitor_fused_kernel<K, false, false, false, true><<<(unsigned)grid, threads, smem, st>>>(
        prm, tb, ymap, hmap, pmap, no_multi());
  } else if (hcap < pl.hcap) {  // the sampled ring: the instantiation that clamps windows
    cudaFuncAttributes fc{};
    const int rc = fused_config<K, I16, false, true>(pl.device, fc);
    if (rc) return rc;
    bfast::monitor_fused_kernel<K, I16, false, true><<<(unsigned)grid, threads, smem, st>>>(prm, tb, ymap, hmap,
                                                                                          pmap, no_multi());
  } else {
    bfast::monitor_fused_kernel<K, I16, false><<<(unsigned)grid, threads, smem, st>>>(prm, tb, ymap, hmap, pmap,
                                                                                     no_multi());
  }
  CUDA_TRY(cudaGetLastError());
  done = true;
  return BFAST_OK;
}

template <int K>
int launch_refit(const bfast_plan &pl, const bfast::MonitorParams &prm, cudaStream_t st, int sms);

template <int K>
int launch_k(const bfast_plan &pl, const bfast::MonitorParams &prm, cudaStream_t st) {
  static thread_local int configured_dev = -1;
  int bp = 128;
  while (bp > 32 && simt_smem(pl, bp) > (size_t)kMaxSmem) bp >>= 1;
  const size_t smem = simt_smem(pl, bp);
  if (configured_dev != pl.device) {
    CUDA_TRY(cudaFuncSetAttribute(bfast::monitor_simt_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  kMaxSmem));
    CUDA_TRY(cudaFuncSetAttribute(bfast::refit_fp64_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  kMaxSmem));
    configured_dev = pl.device;
  }
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, pl.device);
  // the refit list/counter are plan scratch: order executions on any stream
  CUDA_TRY(cudaStreamWaitEvent(st, pl.scratch_free, 0));
  CUDA_TRY(cudaMemsetAsync(prm.refit_count, 0, sizeof(int32_t), st));
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (g_prof_on) {
    CUDA_TRY(cudaEventCreate(&e0));
    CUDA_TRY(cudaEventCreate(&e1));
    CUDA_TRY(cudaEventRecord(e0, st));
  }
  int launches = 0;
  bool fused = false;
  if (pl.mode == 0) {
    const int rc = prm.Y16 ? launch_fused<K, true>(pl, prm, st, fused) : launch_fused<K, false>(pl, prm, st, fused);
    if (rc) return rc;
  }
  if (!fused && prm.Y16 && prm.P > 0) {
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
    return fail(BFAST_EUNSUPPORTED, "int16 stacks run on the fused kernel only (ldY %% 8 == 0, 16-byte aligned Y)");
  }
  {
    launches += fused ? 1 : 0;
  }
  // SIMT kernel: forced (BFAST_KERNEL=simt), or a stack the TMA cannot read
  // (row pitch not a multiple of 16 bytes)
  if (!fused && prm.P > 0) {
    if (smem > (size_t)kMaxSmem) return fail(BFAST_EUNSUPPORTED, "shared memory %zu B too large", smem);
    const int64_t blocks = (prm.P + bp - 1) / bp;
    bfast::monitor_simt_kernel<K><<<(unsigned)blocks, bp, smem, st>>>(prm);
    CUDA_TRY(cudaGetLastError());
    ++launches;
  }
  if (g_prof_on) {
    CUDA_TRY(cudaEventRecord(e1, st));
    g_prof.emplace_back(e0, e1);
  }
  const int rc = launch_refit<K>(pl, prm, st, sms);
  if (rc) return rc;
  g_launches = launches + 1;
  return BFAST_OK;
}

// fp64 refit of the pixels the fused / SIMT kernel flagged (the plan's list);
// exits at once when the list is empty.  Releases the plan's refit scratch.
template <int K>
int launch_refit(const bfast_plan &pl, const bfast::MonitorParams &prm, cudaStream_t st, int sms) {
#ifndef BFAST_REFIT_WARPS
#define BFAST_REFIT_WARPS 4
#endif
  static thread_local int configured_dev = -1;
  if (configured_dev != pl.device) {
    CUDA_TRY(cudaFuncSetAttribute(bfast::refit_fp64_kernel<K>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  kMaxSmem));
    configured_dev = pl.device;
  }
  int rwarps = BFAST_REFIT_WARPS;  // fewer warps per CTA where a long series needs the room
  const size_t rwsmem = bfast::refit_warp_doubles((int)pl.N) * sizeof(double);
  while (rwarps > 1 && (size_t)rwarps * rwsmem > (size_t)kMaxSmem) rwarps >>= 1;
  const size_t rsmem = (size_t)rwarps * rwsmem;
  if (rsmem > (size_t)kMaxSmem) return fail(BFAST_EUNSUPPORTED, "refit smem too large");
  // one resident wave: each warp walks its items with the next column in
  // flight, so extra (waiting) blocks would only break that pipeline
  int rblocks = 0;
  CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rblocks, bfast::refit_fp64_kernel<K>, rwarps * 32,
                                                         rsmem));
  bfast::refit_fp64_kernel<K><<<sms * std::max(rblocks, 1), rwarps * 32, rsmem, st>>>(prm);
  CUDA_TRY(cudaGetLastError());
  CUDA_TRY(cudaEventRecord(pl.scratch_free, st));
  return BFAST_OK;
}

// f1: several monitoring periods in ONE fused launch (monitor_fused.cuh
// FzMulti): period i = plans[i] with its MonitorParams; then the fp64 refit
// of each period's flagged pixels.  Every plan has the same k and pixel range.
template <int K>
int launch_multi_k(const std::vector<bfast_plan *> &pls, const std::vector<bfast::MonitorParams> &prms,
                   cudaStream_t st) {
  using C = bfast::FzCfg<K>;
  const int M = (int)pls.size();
  const bfast_plan &p0 = *pls[0];
  const bfast::MonitorParams &q0 = prms[0];
  cudaFuncAttributes fa{};
  {
    const int rc = fused_config<K, false, true>(p0.device, fa);
    if (rc) return rc;
  }
  const int static_smem = (int)fa.sharedSizeBytes;
  int hcap = 1, hfull = 1;
  const bfast_plan *plong = pls[0];  // the period with the longest history
  for (auto *pl : pls) {
    hfull = std::max(hfull, pl->hcap);
    if (pl->n > plong->n) plong = pl;
  }
  hcap = hfull;
  int T = bfast::FzTiles<K, true>::TM, sc = C::SCMAX;
  if (const char *e = std::getenv("BFAST_FZ_T")) T = std::max(1, std::min(T, std::atoi(e)));
  if (const char *e = std::getenv("BFAST_FZ_SC")) sc = std::max(2, std::min(C::SCMAX, std::atoi(e)));
  auto fits = [&](int t, int c) { return C::smem_bytes(t, hcap, c) + static_smem <= (size_t)kMaxSmem; };
  // the ring from a sample of the longest history's windows (as launch_fused)
  const char *wpe = std::getenv("BFAST_WINDOW_PROBE");
  if (!fits(T, 2) && q0.P >= 32 * 64 && plong->dprobe && !(wpe && wpe[0] == '0')) {
    const int64_t groups = std::min<int64_t>(2048, q0.P / 32);
    CUDA_TRY(cudaMemsetAsync(plong->dprobe, 0, sizeof(int), st));
    bfast::window_probe_kernel<float><<<(unsigned)groups, 32, 0, st>>>(q0.Y + q0.p0, q0.ldY, q0.P, plong->n,
                                                                       plong->hf, q0.P / groups, 0, plong->dprobe);
    CUDA_TRY(cudaGetLastError());
    int hmax = 0;
    CUDA_TRY(cudaMemcpyAsync(&hmax, plong->dprobe, sizeof(int), cudaMemcpyDeviceToHost, st));
    CUDA_TRY(cudaStreamSynchronize(st));
    hcap = std::min(hfull, std::max(std::min(hfull, 8), hmax + std::max(8, hmax / 8)));
  }
  while (T > 1 && !fits(T, 2)) --T;
  T = std::max(C::TPC, T / C::TPC * C::TPC);  // whole control groups
  if (!fits(T, sc)) sc = 2;
  const size_t smem = C::smem_bytes(T, hcap, sc);
  if (smem + static_smem > (size_t)kMaxSmem)
    return fail(BFAST_EUNSUPPORTED, "fused kernel: shared memory %zu B for window %d", smem, hcap);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, p0.device);
  const int threads = 128 * (T + 1);
  const int by_smem = (int)(kSmemPerSM / (smem + static_smem + 1024));
  const int by_tmem = 512 / C::pow2cols(T * C::TCOLS);
  const int by_regs = 65536 / (threads * std::max(fa.numRegs, 1));
  const int per_sm = std::max(1, std::min(std::min(by_smem, by_tmem), std::min(by_regs, 2048 / threads)));
  auto mp = std::make_unique<bfast::FzMulti>();
  std::memset(mp.get(), 0, sizeof(bfast::FzMulti));
  mp->M = M;
  mp->Lg = 0;
  for (int i = 0; i < M; ++i) {
    const bfast_plan &pl = *pls[i];
    bfast::FzPeriod &fp = mp->per[i];
    fp.prm = prms[i];
    fp.tabA = pl.dtabf;
    fp.tabB = pl.dtabf + pl.tabfB_off;
    fp.tabC = pl.dtabf + pl.tabfC_off;
    fp.shared = nullptr;  // f3 is not part of the multi-period kernel
    fp.nch = pl.nch;
    fp.ncm = pl.ncm;
    mp->Lg += 2 * pl.nch + pl.ncm;
    if (!make_stack_map(&fp.h, prms[i].Y + prms[i].p0, prms[i].ldY, prms[i].P, pl.n, 128 * C::TPC, 16) ||
        !make_stack_map(&fp.y, prms[i].Y + prms[i].p0, prms[i].ldY, prms[i].P, pl.N, 128 * C::TPC, 16))
      return fail(BFAST_EUNSUPPORTED, "tensor maps of the stack");
  }
  int64_t Nmax = 0;
  for (auto *pl : pls) Nmax = std::max<int64_t>(Nmax, pl->N);
  CUtensorMap pmap;
  if (!make_stack_map(&pmap, q0.Y + q0.p0, q0.ldY, q0.P, Nmax, 128 * C::TPC, C::PFB))
    return fail(BFAST_EUNSUPPORTED, "tensor maps of the stack");
  for (auto *pl : pls) CUDA_TRY(cudaStreamWaitEvent(st, pl->scratch_free, 0));
  for (int i = 0; i < M; ++i) CUDA_TRY(cudaMemsetAsync(prms[i].refit_count, 0, sizeof(int32_t), st));
  bfast::FzTables tb{};
  tb.tabA = mp->per[0].tabA;
  tb.tabB = mp->per[0].tabB;
  tb.tabC = mp->per[0].tabC;
  tb.nch = p0.nch;
  tb.ncm = p0.ncm;
  tb.T = T;
  tb.hcap = hcap;
  // no L2 prefetch in the multi-period kernel: most of its reads are L2
  // re-reads of earlier periods (measured -3% on 4 and 7 yearly periods)
  tb.pfd = 0;
  if (const char *e = std::getenv("BFAST_FZ_PFD")) tb.pfd = std::max(0, std::atoi(e)) / C::PFB * C::PFB;
  tb.sc = sc;
  tb.ntg = (q0.P + 128 * T - 1) / (128 * T);
  tb.shared = nullptr;
  if (std::getenv("BFAST_VERBOSE"))
    std::fprintf(stderr, "bfast: multi k=%d M=%d T=%d sc=%d smem=%zu hcap=%d\n", p0.k, M, T, sc, smem, hcap);
  const int64_t grid = std::min<int64_t>(tb.ntg, (int64_t)sms * per_sm);
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  if (g_prof_on) {
    CUDA_TRY(cudaEventCreate(&e0));
    CUDA_TRY(cudaEventCreate(&e1));
    CUDA_TRY(cudaEventRecord(e0, st));
  }
  if (hcap < hfull) {  // the sampled ring: windows wider than it go to the refit
    cudaFuncAttributes fc{};
    const int rc = fused_config<K, false, true, true>(p0.device, fc);
    if (rc) return rc;
    bfast::monitor_fused_kernel<K, false, true, true><<<(unsigned)grid, threads, smem, st>>>(
        q0, tb, mp->per[0].y, mp->per[0].h, pmap, *mp);
  } else {
    bfast::monitor_fused_kernel<K, false, true><<<(unsigned)grid, threads, smem, st>>>(q0, tb, mp->per[0].y,
                                                                                      mp->per[0].h, pmap, *mp);
  }
  CUDA_TRY(cudaGetLastError());
  if (g_prof_on) {
    CUDA_TRY(cudaEventRecord(e1, st));
    g_prof.emplace_back(e0, e1);
  }
  for (int i = 0; i < M; ++i) {
    const int rc = launch_refit<K>(*pls[i], prms[i], st, sms);
    if (rc) return rc;
  }
  g_launches = 1 + M;
  return BFAST_OK;
}

int launch_multi(const std::vector<bfast_plan *> &pls, const std::vector<bfast::MonitorParams> &prms,
                 cudaStream_t st) {
  switch (pls[0]->k) {
    case 0: return launch_multi_k<2>(pls, prms, st);
    case 1: return launch_multi_k<4>(pls, prms, st);
    case 2: return launch_multi_k<6>(pls, prms, st);
    case 3: return launch_multi_k<8>(pls, prms, st);
    case 4: return launch_multi_k<10>(pls, prms, st);
    case 5: return launch_multi_k<12>(pls, prms, st);
    case 6: return launch_multi_k<14>(pls, prms, st);
  }
  return fail(BFAST_EUNSUPPORTED, "k=%d", pls[0]->k);
}

int launch(const bfast_plan &pl, const bfast::MonitorParams &prm, cudaStream_t st) {
  switch (pl.k) {
    case 0: return launch_k<2>(pl, prm, st);
    case 1: return launch_k<4>(pl, prm, st);
    case 2: return launch_k<6>(pl, prm, st);
    case 3: return launch_k<8>(pl, prm, st);
    case 4: return launch_k<10>(pl, prm, st);
    case 5: return launch_k<12>(pl, prm, st);
    case 6: return launch_k<14>(pl, prm, st);
  }
  return fail(BFAST_EUNSUPPORTED, "k=%d", pl.k);
}

// --- one-shot plan cache (bfast_monitor / bfast_monitor_ex / host paths)
// Plans are shared_ptr: a caller holds its reference for the whole
// execution, so evicting the plan from the cache (a 17th key, possibly from
// another thread) cannot free it under a running call.
std::mutex g_cache_mu;
std::vector<std::shared_ptr<bfast_plan>> g_cache;

int env_mode() {
  const char *m = std::getenv("BFAST_KERNEL");
  return !m ? 0 : (std::strcmp(m, "simt") == 0 ? 1 : 0);
}

bool same_plan(const bfast_plan &pl, int dev, int64_t N, const double *dates, int32_t n, int32_t k,
               float h, float lambda) {
  return pl.device == dev && pl.N == N && pl.n == n && pl.k == k && pl.hf == h &&
         pl.lambda == lambda && std::memcmp(pl.dates.data(), dates, sizeof(double) * N) == 0;
}

int cached_plan(int dev, int64_t N, const double *dates, int32_t n, int32_t k, float h, float lambda,
                std::shared_ptr<bfast_plan> &out) {
  std::lock_guard<std::mutex> g(g_cache_mu);
  for (auto &p : g_cache)
    if (same_plan(*p, dev, N, dates, n, k, h, lambda) && p->mode == env_mode()) {
      out = p;
      return BFAST_OK;
    }
  bfast_plan *pl = nullptr;
  int rc = bfast_plan_create(&pl, dev, N, dates, n, k, h, lambda);
  if (rc) return rc;
  if (g_cache.size() >= 16) g_cache.erase(g_cache.begin());
  g_cache.emplace_back(pl);
  out = g_cache.back();
  return BFAST_OK;
}

int ensure_list(bfast_plan &pl, int64_t P) {
  if (P <= pl.list_cap) return BFAST_OK;
  cudaFree(pl.dlist);
  pl.dlist = nullptr;
  pl.list_cap = 0;
  CUDA_TRY(cudaMalloc(&pl.dlist, sizeof(int64_t) * (size_t)std::max<int64_t>(P, 1)));
  pl.list_cap = P;
  return BFAST_OK;
}

// Pixel ranges of at most 2^30 pixels per launch set: TMA box coordinates
// and the kernels' tile arithmetic are 32-bit.
constexpr int64_t kMaxLaunchPixels = (int64_t)1 << 30;

int execute_one(bfast_plan &pl, const bfast_args *a, int64_t p0, int64_t P, const bfast_codec_i16 *codec);

int execute_range(bfast_plan &pl, const bfast_args *a, int64_t p0, int64_t P,
                  const bfast_codec_i16 *codec = nullptr) {
  if (P == 0) {
    g_launches = 0;
    return BFAST_OK;
  }
  int total = 0;
  for (int64_t b = 0; b < P; b += kMaxLaunchPixels) {
    const int rc = execute_one(pl, a, p0 + b, std::min(kMaxLaunchPixels, P - b), codec);
    if (rc) return rc;
    total += g_launches;
  }
  g_launches = total;
  return BFAST_OK;
}

int execute_one(bfast_plan &pl, const bfast_args *a, int64_t p0, int64_t P, const bfast_codec_i16 *codec) {
  int rc = ensure_list(pl, P);
  if (rc) return rc;
  bfast::MonitorParams prm{};
  prm.Y = codec ? nullptr : a->Y;
  if (codec) {
    prm.Y16 = codec->Y;
    prm.dscale = codec->scale;
    prm.doffset = codec->offset;
    prm.nodata = codec->nodata;
  }
  prm.ldY = a->ldY;
  prm.P = P;
  prm.p0 = p0;
  prm.N = (int)pl.N;
  prm.n = pl.n;
  prm.X = pl.dX;
  prm.X64 = pl.dX64;
  prm.KP = pl.KP;
  prm.hf = pl.hf;
  prm.lambda = pl.lambda;
  prm.hcap = pl.hcap;
  prm.tc = pl.tc;
  prm.ts = pl.ts;
  prm.out_break = a->out_break;
  prm.out_mag = a->out_magnitude;
  prm.out_beta = a->out_beta;
  prm.out_sigma = a->out_sigma;
  prm.out_nbar = a->out_nbar;
  prm.out_flags = a->out_flags;
  prm.refit_list = pl.dlist;
  prm.refit_count = pl.dcount;
  return launch(pl, prm, (cudaStream_t)a->stream);
}

int validate_args(const bfast_args *a) {
  if (!a) return fail(BFAST_EINVAL, "args is NULL");
  int rc = validate_scalar(a->N, a->dates, a->n_hist, a->k, a->h, a->lambda);
  if (rc) return rc;
  if (a->P < 0) return fail(BFAST_EINVAL, "P < 0");
  if (a->ldY < a->P) return fail(BFAST_EINVAL, "ldY < P");
  if (a->P > 0 && (!a->Y || !a->out_break || !a->out_magnitude))
    return fail(BFAST_EINVAL, "NULL Y/out_break/out_magnitude");
  if ((a->N - 1) * (double)a->ldY + a->P > 9.0e18) return fail(BFAST_EINVAL, "stack too large");
  return BFAST_OK;
}

}  // namespace

extern "C" {

#ifdef BFAST_FZ_TIMING
// diagnostics build only: the fused kernel's cycle accounting (copied, then reset)
int bfast_debug_fz_timing(unsigned long long *out, int n) {
  unsigned long long h[16] = {0};
  CUDA_TRY(cudaMemcpyFromSymbol(h, bfast::fz_timing, sizeof h));
  const unsigned long long z[16] = {0};
  CUDA_TRY(cudaMemcpyToSymbol(bfast::fz_timing, z, sizeof z));
  for (int i = 0; i < n && i < 16; ++i) out[i] = h[i];
  return BFAST_OK;
}
#endif

int bfast_abi_version(void) { return BFAST_ABI_VERSION; }

const char *bfast_last_error(void) { return g_err.c_str(); }

int bfast_last_launch_count(void) { return g_launches; }

int bfast_profile_enable(int on) {
  g_prof_on = on != 0;
  if (!g_prof_on) {
    for (auto &e : g_prof) {
      cudaEventDestroy(e.first);
      cudaEventDestroy(e.second);
    }
    g_prof.clear();
  }
  return BFAST_OK;
}

int bfast_profile_collect(float *ms_out, int max) {
  int n = 0;
  int rc = BFAST_OK;
  for (auto &e : g_prof) {
    float ms = 0.f;
    if (rc == BFAST_OK) {
      cudaError_t err = cudaEventSynchronize(e.second);
      if (err == cudaSuccess) err = cudaEventElapsedTime(&ms, e.first, e.second);
      if (err != cudaSuccess) rc = fail(BFAST_ECUDA, "profile: %s", cudaGetErrorString(err));
    }
    if (rc == BFAST_OK && ms_out && n < max) ms_out[n++] = ms;
    cudaEventDestroy(e.first);
    cudaEventDestroy(e.second);
  }
  g_prof.clear();
  return rc == BFAST_OK ? n : rc;
}

const char *bfast_status_string(int s) {
  switch (s) {
    case BFAST_OK: return "BFAST_OK";
    case BFAST_EINVAL: return "BFAST_EINVAL";
    case BFAST_EUNSUPPORTED: return "BFAST_EUNSUPPORTED";
    case BFAST_ECUDA: return "BFAST_ECUDA";
    case BFAST_ENOMEM: return "BFAST_ENOMEM";
  }
  return "unknown status";
}

void bfast_shard_range(int64_t P, int rank, int world, int64_t *begin, int64_t *end) {
  if (world < 1 || rank < 0 || rank >= world || P <= 0) {
    *begin = *end = 0;
    return;
  }
  const int64_t tiles = (P + 127) / 128;
  const int64_t b = tiles * rank / world, e = tiles * (rank + 1) / world;
  *begin = std::min(P, b * 128);
  *end = std::min(P, e * 128);
}

int bfast_plan_create(bfast_plan **out, int device, int64_t N, const double *dates, int32_t n_hist,
                      int32_t k, float h, float lambda) {
  if (!out) return fail(BFAST_EINVAL, "out is NULL");
  *out = nullptr;
  int rc = validate_scalar(N, dates, n_hist, k, h, lambda);
  if (rc) return rc;
  std::unique_ptr<bfast_plan> pl(new bfast_plan());
  pl->device = device;
  pl->N = N;
  pl->n = n_hist;
  pl->k = k;
  pl->K = 2 + 2 * k;
  pl->KP = (pl->K + 3) / 4 * 4;
  pl->hf = h;
  pl->lambda = lambda;
  pl->dates.assign(dates, dates + N);
  pl->tc = 0.5 * ((double)n_hist + 1.0);
  pl->ts = n_hist > 1 ? 0.5 * ((double)n_hist - 1.0) : 1.0;
  pl->hcap = std::max(1, host_window(n_hist, h));
  if (simt_smem(*pl, 32) > (size_t)kMaxSmem)
    return fail(BFAST_EUNSUPPORTED, "N=%lld with window %d exceeds shared memory", (long long)N,
                pl->hcap);
  if (bfast::refit_warp_doubles((int)N) * sizeof(double) > (size_t)kMaxSmem)
    return fail(BFAST_EUNSUPPORTED, "N=%lld too large for the refit kernel", (long long)N);
  {
    const char *mode = std::getenv("BFAST_KERNEL");
    pl->mode = !mode ? 0 : (std::strcmp(mode, "simt") == 0 ? 1 : 0);
  }
  std::vector<float> X;
  std::vector<double> X64;
  build_design(*pl, X, X64);
  int prev = -1;
  CUDA_TRY(cudaGetDevice(&prev));
  CUDA_TRY(cudaSetDevice(device));
  cudaError_t e = cudaMalloc(&pl->dX, X.size() * sizeof(float));
  if (e == cudaSuccess) e = cudaMalloc(&pl->dX64, X64.size() * sizeof(double));
  if (e == cudaSuccess) e = cudaMalloc(&pl->dcount, sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&pl->dprobe, sizeof(int));
  if (e == cudaSuccess) e = cudaMemcpy(pl->dX, X.data(), X.size() * sizeof(float), cudaMemcpyHostToDevice);
  if (e == cudaSuccess)
    e = cudaMemcpy(pl->dX64, X64.data(), X64.size() * sizeof(double), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemset(pl->dcount, 0, sizeof(int32_t));
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&pl->scratch_free, cudaEventDisableTiming);
  int trc = BFAST_OK;
  if (e == cudaSuccess && trc == BFAST_OK && pl->mode == 0) trc = build_fz(*pl);
  pl->nch = (n_hist + 15) / 16;
  pl->ncm = ((int)N - n_hist + 15) / 16;
  cudaSetDevice(prev);
  if (trc != BFAST_OK) return trc;
  if (e != cudaSuccess)
    return fail(e == cudaErrorMemoryAllocation ? BFAST_ENOMEM : BFAST_ECUDA, "plan: %s",
                cudaGetErrorString(e));
  *out = pl.release();
  return BFAST_OK;
}

void bfast_plan_destroy(bfast_plan *plan) { delete plan; }

int bfast_plan_execute(const bfast_plan *plan, const bfast_args *a) {
  if (!plan) return fail(BFAST_EINVAL, "plan is NULL");
  int rc = validate_args(a);
  if (rc) return rc;
  bfast_plan &pl = const_cast<bfast_plan &>(*plan);
  if (!same_plan(pl, pl.device, a->N, a->dates, a->n_hist, a->k, a->h, a->lambda))
    return fail(BFAST_EINVAL, "args do not match the plan");
  std::lock_guard<std::mutex> g(pl.mu);
  int prev = -1;
  CUDA_TRY(cudaGetDevice(&prev));
  if (prev != pl.device) CUDA_TRY(cudaSetDevice(pl.device));
  rc = execute_range(pl, a, 0, a->P);
  if (prev != pl.device) cudaSetDevice(prev);
  return rc;
}

int bfast_monitor_ex(const bfast_args *a) {
  int rc = validate_args(a);
  if (rc) return rc;
  int dev = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  std::shared_ptr<bfast_plan> pl;
  rc = cached_plan(dev, a->N, a->dates, a->n_hist, a->k, a->h, a->lambda, pl);
  if (rc) return rc;
  std::lock_guard<std::mutex> g(pl->mu);
  return execute_range(*pl, a, 0, a->P);
}

int bfast_monitor_periods(const bfast_args *a, const int32_t *n_hist, const int32_t *N_end, int32_t M) {
  if (!a || !n_hist || !N_end) return fail(BFAST_EINVAL, "args, n_hist or N_end NULL");
  if (M < 1) return fail(BFAST_EINVAL, "M=%d < 1", M);
  if (M > bfast::kMaxPeriods) return fail(BFAST_EUNSUPPORTED, "M=%d > %d periods", M, bfast::kMaxPeriods);
  bfast_args v = *a;
  v.n_hist = n_hist[0];
  int rc = validate_args(&v);
  if (rc) return rc;
  for (int i = 0; i < M; ++i) {
    if (N_end[i] > a->N || N_end[i] < 2) return fail(BFAST_EINVAL, "N_end[%d]=%d outside [2, N]", i, N_end[i]);
    rc = validate_scalar(N_end[i], a->dates, n_hist[i], a->k, a->h, a->lambda);
    if (rc) return fail(rc, "period %d: %s", i, g_err.c_str());
    for (int j = 0; j < i; ++j)
      if (n_hist[j] == n_hist[i] && N_end[j] == N_end[i]) return fail(BFAST_EINVAL, "periods %d and %d equal", j, i);
  }
  if (a->P == 0) {
    g_launches = 0;
    return BFAST_OK;
  }
  int dev = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  std::vector<std::shared_ptr<bfast_plan>> hold(M);
  std::vector<bfast_plan *> pls(M);
  for (int i = 0; i < M; ++i) {
    rc = cached_plan(dev, N_end[i], a->dates, n_hist[i], a->k, a->h, a->lambda, hold[i]);
    if (rc) return rc;
    pls[i] = hold[i].get();
    if (pls[i]->mode != 0 || !pls[i]->dtabf)
      return fail(BFAST_EUNSUPPORTED, "several periods run on the fused kernel only");
  }
  if (a->ldY % 4 != 0 || ((uintptr_t)a->Y) % 16 != 0)
    return fail(BFAST_EUNSUPPORTED, "several periods: Y must be 16-byte aligned and ldY %% 4 == 0 (TMA)");
  std::vector<bfast_plan *> order(pls);
  std::sort(order.begin(), order.end());
  std::vector<std::unique_lock<std::mutex>> locks;
  for (auto *pl : order) locks.emplace_back(pl->mu);
  const int K = 2 + 2 * a->k;
  int total = 0;
  for (int64_t b = 0; b < a->P; b += kMaxLaunchPixels) {
    const int64_t w = std::min(kMaxLaunchPixels, a->P - b);
    std::vector<bfast::MonitorParams> prms(M);
    for (int i = 0; i < M; ++i) {
      bfast_plan &pl = *pls[i];
      rc = ensure_list(pl, w);
      if (rc) return rc;
      bfast::MonitorParams &q = prms[i];
      q = bfast::MonitorParams{};
      q.Y = a->Y;
      q.ldY = a->ldY;
      q.P = w;
      q.p0 = b;
      q.N = (int)pl.N;
      q.n = pl.n;
      q.X = pl.dX;
      q.X64 = pl.dX64;
      q.KP = pl.KP;
      q.hf = pl.hf;
      q.lambda = pl.lambda;
      q.hcap = pl.hcap;
      q.tc = pl.tc;
      q.ts = pl.ts;
      // outputs [M][P]: period i's map starts at i * P (the kernel indexes by absolute pixel)
      q.out_break = a->out_break + (size_t)i * a->P;
      q.out_mag = a->out_magnitude + (size_t)i * a->P;
      q.out_beta = a->out_beta ? a->out_beta + (size_t)i * a->P * K : nullptr;
      q.out_sigma = a->out_sigma ? a->out_sigma + (size_t)i * a->P : nullptr;
      q.out_nbar = a->out_nbar ? a->out_nbar + (size_t)i * a->P : nullptr;
      q.out_flags = a->out_flags ? a->out_flags + (size_t)i * a->P : nullptr;
      q.refit_list = pl.dlist;
      q.refit_count = pl.dcount;
    }
    // one period: the single-period kernel (the same arithmetic, no period
    // tables).  BFAST_PERIODS=split runs every period as its own launch
    // (each reads its slice of the stack from HBM): on this issue-bound
    // kernel that is the faster schedule (f1)
    const char *pm = std::getenv("BFAST_PERIODS");
    if (M == 1 || (pm && std::strcmp(pm, "split") == 0)) {
      for (int i = 0; i < M; ++i) {
        rc = launch(*pls[i], prms[i], (cudaStream_t)a->stream);
        if (rc) return rc;
        total += g_launches;
      }
    } else {
      rc = launch_multi(pls, prms, (cudaStream_t)a->stream);
      if (rc) return rc;
      total += g_launches;
    }
  }
  g_launches = total;
  return BFAST_OK;
}

int bfast_monitor_i16(const bfast_codec_i16 *codec, const bfast_args *a) {
  if (!codec || !a) return fail(BFAST_EINVAL, "codec or args NULL");
  if (a->Y) return fail(BFAST_EINVAL, "args->Y must be NULL (the stack is codec->Y)");
  if (!(codec->scale != 0.f) || !std::isfinite(codec->scale) || !std::isfinite(codec->offset))
    return fail(BFAST_EINVAL, "codec scale must be finite and non-zero, offset finite");
  if (codec->nodata < -32768 || codec->nodata > 32767) return fail(BFAST_EINVAL, "nodata outside int16");
  bfast_args v = *a;
  v.Y = reinterpret_cast<const float *>(codec->Y);  // validated as the stack pointer
  int rc = validate_args(&v);
  if (rc) return rc;
  if (a->P > 0 && (((uintptr_t)codec->Y) % 16 != 0 || a->ldY % 8 != 0))
    return fail(BFAST_EUNSUPPORTED, "int16 stack: Y must be 16-byte aligned and ldY %% 8 == 0 (TMA)");
  int dev = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  std::shared_ptr<bfast_plan> pl;
  rc = cached_plan(dev, a->N, a->dates, a->n_hist, a->k, a->h, a->lambda, pl);
  if (rc) return rc;
  if (pl->mode != 0) return fail(BFAST_EUNSUPPORTED, "int16 stacks run on the fused kernel only");
  std::lock_guard<std::mutex> g(pl->mu);
  return execute_range(*pl, &v, 0, a->P, codec);
}

int bfast_monitor(const float *Y, int64_t N, int64_t P, const double *dates, int32_t n_hist,
                  int32_t k, float h, float lambda, int32_t *out_break, float *out_magnitude) {
  bfast_args a{};
  a.Y = Y;
  a.N = N;
  a.P = P;
  a.ldY = P;
  a.dates = dates;
  a.n_hist = n_hist;
  a.k = k;
  a.h = h;
  a.lambda = lambda;
  a.out_break = out_break;
  a.out_magnitude = out_magnitude;
  int rc = bfast_monitor_ex(&a);
  if (rc) return rc;
  CUDA_TRY(cudaStreamSynchronize(nullptr));
  return BFAST_OK;
}

// End-to-end on host buffers: pixel slabs, double-buffered H2D on a copy
// stream overlapping the kernel on the compute stream.  The device slabs,
// streams and events are the plan's (bfast_plan::HostPath), kept across
// calls: a stream of tiles pays the allocations once.
int host_path_ensure(bfast_plan &pl, int64_t slab) {
  auto &hp = pl.host;
  if (!hp.cs) {
    CUDA_TRY(cudaStreamCreateWithFlags(&hp.cs, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&hp.ks, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CUDA_TRY(cudaEventCreateWithFlags(&hp.loaded[i], cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&hp.done[i], cudaEventDisableTiming));
    }
  }
  if (slab <= hp.slab) return BFAST_OK;
  CUDA_TRY(cudaStreamSynchronize(hp.ks));
  CUDA_TRY(cudaStreamSynchronize(hp.cs));
  for (int i = 0; i < 2; ++i) {
    cudaFree(hp.dY[i]);
    cudaFree(hp.dB[i]);
    cudaFree(hp.dM[i]);
    cudaFreeHost(hp.hB[i]);
    cudaFreeHost(hp.hM[i]);
    hp.dY[i] = nullptr;
    hp.dB[i] = nullptr;
    hp.dM[i] = nullptr;
    hp.hB[i] = nullptr;
    hp.hM[i] = nullptr;
  }
  hp.slab = 0;
  for (int i = 0; i < 2; ++i) {
    CUDA_TRY(cudaMalloc(&hp.dY[i], sizeof(float) * (size_t)pl.N * slab));
    CUDA_TRY(cudaMalloc(&hp.dB[i], sizeof(int32_t) * slab));
    CUDA_TRY(cudaMalloc(&hp.dM[i], sizeof(float) * slab));
    CUDA_TRY(cudaMallocHost(&hp.hB[i], sizeof(int32_t) * slab));
    CUDA_TRY(cudaMallocHost(&hp.hM[i], sizeof(float) * slab));
  }
  hp.slab = slab;
  return BFAST_OK;
}

int bfast_monitor_host(const float *Y_host, int64_t N, int64_t P, int64_t ldY, const double *dates,
                       int32_t n_hist, int32_t k, float h, float lambda, int32_t *out_break_host,
                       float *out_magnitude_host, int device) {
  int rc = validate_scalar(N, dates, n_hist, k, h, lambda);
  if (rc) return rc;
  if (P < 0 || ldY < P) return fail(BFAST_EINVAL, "P < 0 or ldY < P");
  if (P == 0) {
    g_launches = 0;
    return BFAST_OK;
  }
  if (!Y_host || !out_break_host || !out_magnitude_host) return fail(BFAST_EINVAL, "NULL pointer");
  int prev = 0;
  CUDA_TRY(cudaGetDevice(&prev));
  const int dev = device < 0 ? prev : device;
  CUDA_TRY(cudaSetDevice(dev));
  struct Restore {
    int d;
    ~Restore() { cudaSetDevice(d); }
  } restore{prev};
  std::shared_ptr<bfast_plan> pl;
  rc = cached_plan(dev, N, dates, n_hist, k, h, lambda, pl);
  if (rc) return rc;
  // slab width: ~1 GiB of stack per buffer, multiple of 128 pixels
  int64_t slab = std::max<int64_t>(128, ((int64_t)1 << 28) / N / 128 * 128);
  slab = std::min<int64_t>(slab, (P + 127) / 128 * 128);
  std::lock_guard<std::mutex> g(pl->mu);
  rc = host_path_ensure(*pl, slab);
  if (rc) return rc;
  auto &hp = pl->host;
  slab = hp.slab;
  int launches = 0;
  cudaError_t e = cudaSuccess;
  int slot = 0;
  // results of the previous slab, drained to the caller's arrays from the
  // pinned staging once its D2H is done (while the next upload runs)
  int64_t pend_b = -1, pend_w = 0;
  int pend_slot = 0;
  auto drain = [&]() -> cudaError_t {
    if (pend_b < 0) return cudaSuccess;
    const cudaError_t ee = cudaEventSynchronize(hp.done[pend_slot]);
    if (ee != cudaSuccess) return ee;
    std::memcpy(out_break_host + pend_b, hp.hB[pend_slot], sizeof(int32_t) * pend_w);
    std::memcpy(out_magnitude_host + pend_b, hp.hM[pend_slot], sizeof(float) * pend_w);
    pend_b = -1;
    return cudaSuccess;
  };
  for (int64_t b0 = 0; b0 < P && rc == BFAST_OK; b0 += slab, slot ^= 1) {
    const int64_t w = std::min(slab, P - b0);
    // the buffer is free once the kernel that used it two slabs ago is done
    e = cudaStreamWaitEvent(hp.cs, hp.done[slot], 0);
    if (e == cudaSuccess)
      e = cudaMemcpy2DAsync(hp.dY[slot], sizeof(float) * w, Y_host + b0, sizeof(float) * ldY, sizeof(float) * w,
                            N, cudaMemcpyHostToDevice, hp.cs);
    if (e == cudaSuccess) e = cudaEventRecord(hp.loaded[slot], hp.cs);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(hp.ks, hp.loaded[slot], 0);
    if (e != cudaSuccess) break;
    bfast_args a{};
    a.Y = hp.dY[slot];
    a.N = N;
    a.P = w;
    a.ldY = w;
    a.dates = dates;
    a.n_hist = n_hist;
    a.k = k;
    a.h = h;
    a.lambda = lambda;
    a.out_break = hp.dB[slot];
    a.out_magnitude = hp.dM[slot];
    a.stream = hp.ks;
    rc = execute_range(*pl, &a, 0, w);
    launches += g_launches;
    if (rc) break;
    e = cudaMemcpyAsync(hp.hB[slot], hp.dB[slot], sizeof(int32_t) * w, cudaMemcpyDeviceToHost, hp.ks);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(hp.hM[slot], hp.dM[slot], sizeof(float) * w, cudaMemcpyDeviceToHost, hp.ks);
    if (e == cudaSuccess) e = cudaEventRecord(hp.done[slot], hp.ks);
    if (e == cudaSuccess) e = drain();  // the slab before this one
    if (e != cudaSuccess) break;
    pend_b = b0;
    pend_w = w;
    pend_slot = slot;
  }
  if (e == cudaSuccess && rc == BFAST_OK) e = drain();
  const cudaError_t es = cudaStreamSynchronize(hp.ks);
  if (rc) return rc;
  if (e == cudaSuccess) e = es;
  if (e != cudaSuccess) return fail(BFAST_ECUDA, "host path: %s", cudaGetErrorString(e));
  g_launches = launches;
  return BFAST_OK;
}

int bfast_monitor_multi(const float *Y_host, int64_t N, int64_t P, int64_t ldY, const double *dates,
                        int32_t n_hist, int32_t k, float h, float lambda, const int *devices, int ndev,
                        int32_t *out_break_host, float *out_magnitude_host) {
  int rc = validate_scalar(N, dates, n_hist, k, h, lambda);
  if (rc) return rc;
  if (!devices || ndev < 1) return fail(BFAST_EINVAL, "no devices");
  if (P < 0 || ldY < P) return fail(BFAST_EINVAL, "P < 0 or ldY < P");
  if (P > 0 && (!Y_host || !out_break_host || !out_magnitude_host))
    return fail(BFAST_EINVAL, "NULL pointer");
  std::vector<int> status(ndev, BFAST_OK);
  std::vector<std::string> errs(ndev);
  std::vector<int> launches(ndev, 0);
  std::vector<std::thread> th;
  for (int r = 0; r < ndev; ++r) {
    th.emplace_back([&, r]() {
      int64_t b, e;
      bfast_shard_range(P, r, ndev, &b, &e);
      if (e > b)
        status[r] = bfast_monitor_host(Y_host + b, N, e - b, ldY, dates, n_hist, k, h, lambda,
                                       out_break_host + b, out_magnitude_host + b, devices[r]);
      errs[r] = g_err;
      launches[r] = g_launches;
    });
  }
  for (auto &t : th) t.join();
  int total = 0;
  for (int r = 0; r < ndev; ++r) {
    if (status[r]) return fail(status[r], "device %d: %s", devices[r], errs[r].c_str());
    total += launches[r];
  }
  g_launches = total;
  return BFAST_OK;
}

// ---- f2: host-pipeline preprocessing -----------------
int bfast_valid_dates(const float *Y, int64_t N, int64_t P, int64_t ldY, int32_t *keep, void *stream) {
  if (N < 0 || P < 0 || ldY < P) return fail(BFAST_EINVAL, "N < 0, P < 0 or ldY < P");
  if (N == 0) {
    g_launches = 0;
    return BFAST_OK;
  }
  if (!keep || (P > 0 && !Y)) return fail(BFAST_EINVAL, "NULL pointer");
  const int64_t nseg = (P + bfast::kScanSeg - 1) / bfast::kScanSeg;
  if (N > 0x7fffffff || nseg > 65535) return fail(BFAST_EUNSUPPORTED, "stack too large for one scan");
  cudaStream_t st = (cudaStream_t)stream;
  CUDA_TRY(cudaMemsetAsync(keep, 0, sizeof(int32_t) * N, st));
  g_launches = 0;
  if (P == 0) return BFAST_OK;
  const int vec4 = (ldY % 4 == 0) && ((uintptr_t)Y % 16 == 0);
  bfast::slice_any_kernel<<<dim3((unsigned)N, (unsigned)nseg), bfast::kScanThreads, 0, st>>>(Y, P, ldY, keep, vec4);
  CUDA_TRY(cudaGetLastError());
  g_launches = 1;
  return BFAST_OK;
}

int bfast_gather_dates(const float *Y, int64_t N, int64_t ldY, int64_t P, const int32_t *idx, int64_t Nc,
                       float *Yc, int64_t ldYc, void *stream) {
  if (N < 0 || P < 0 || Nc < 0 || ldY < P || ldYc < P)
    return fail(BFAST_EINVAL, "N < 0, P < 0, Nc < 0, ldY < P or ldYc < P");
  g_launches = 0;
  if (P == 0 || Nc == 0) return BFAST_OK;
  if (!Y || !idx || !Yc) return fail(BFAST_EINVAL, "NULL pointer");
  if (Nc > 65535) return fail(BFAST_EUNSUPPORTED, "Nc=%lld > 65535", (long long)Nc);
  const int vec4 = (ldY % 4 == 0) && (ldYc % 4 == 0) && ((uintptr_t)Y % 16 == 0) && ((uintptr_t)Yc % 16 == 0);
  int dev = 0, sms = 148;
  CUDA_TRY(cudaGetDevice(&dev));
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // about 8 resident blocks per SM over all rows
  const int64_t per_row = std::max<int64_t>(1, std::min<int64_t>((P / (vec4 ? 4 : 1) + 255) / 256,
                                                               std::max<int64_t>(1, 8 * sms / Nc)));
  bfast::gather_dates_kernel<<<dim3((unsigned)per_row, (unsigned)Nc), 256, 0, (cudaStream_t)stream>>>(
      Y, N, ldY, P, idx, Yc, ldYc, vec4);
  CUDA_TRY(cudaGetLastError());
  g_launches = 1;
  return BFAST_OK;
}

int bfast_monitor_host_resume(const float *Y_host, int64_t N, int64_t P, int64_t ldY, const double *dates,
                              int32_t n_hist, int32_t k, float h, float lambda, int32_t *out_break_host,
                              float *out_magnitude_host, int device, int64_t tile, int64_t max_tiles,
                              int64_t *done) {
  if (!done || *done < 0 || *done > P || tile < 1)
    return fail(BFAST_EINVAL, "done NULL or outside [0, P], or tile < 1");
  int launches = 0;
  for (int64_t t = 0; *done < P && (max_tiles < 0 || t < max_tiles); ++t) {
    const int64_t b = *done, w = std::min(tile, P - b);
    const int rc = bfast_monitor_host(Y_host + b, N, w, ldY, dates, n_hist, k, h, lambda, out_break_host + b,
                                      out_magnitude_host + b, device);
    if (rc) return rc;
    launches += g_launches;
    *done = b + w;  // the tile's results are in the host arrays
  }
  g_launches = launches;
  return BFAST_OK;
}

}  // extern "C"
namespace {
std::mutex g_ipc_mu;
std::map<void *, void *> g_ipc_base;  // mapped pointer -> opened allocation base
}  // namespace
extern "C" {

int bfast_monitor_shards(const float *const *Y_dev, const int64_t *P, const int64_t *ldY, const int *devices,
                         int nshards, int64_t N, const double *dates, int32_t n_hist, int32_t k, float h,
                         float lambda, int gather_device, int32_t *out_break, float *out_magnitude) {
  int rc = validate_scalar(N, dates, n_hist, k, h, lambda);
  if (rc) return rc;
  if (!Y_dev || !P || !ldY || !devices || nshards < 1) return fail(BFAST_EINVAL, "no shards");
  int64_t total = 0;
  for (int i = 0; i < nshards; ++i) {
    if (P[i] < 0 || ldY[i] < P[i]) return fail(BFAST_EINVAL, "shard %d: P < 0 or ldY < P", i);
    if (P[i] > 0 && !Y_dev[i]) return fail(BFAST_EINVAL, "shard %d: NULL stack", i);
    total += P[i];
  }
  if (total > 0 && (!out_break || !out_magnitude)) return fail(BFAST_EINVAL, "NULL outputs");
  std::vector<int> status(nshards, BFAST_OK);
  std::vector<std::string> errs(nshards);
  std::vector<int> launches(nshards, 0);
  std::vector<std::thread> th;
  int64_t off = 0;
  for (int i = 0; i < nshards; ++i) {
    th.emplace_back([&, i, off]() {
      if (P[i] == 0) return;
      int st = BFAST_OK;
      cudaError_t e = cudaSetDevice(devices[i]);
      if (e == cudaSuccess && devices[i] != gather_device) {
        // the shard's epilogue stores go straight to the gather device
        e = cudaDeviceEnablePeerAccess(gather_device, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) {
          cudaGetLastError();
          e = cudaSuccess;
        }
      }
      std::shared_ptr<bfast_plan> pl;
      cudaStream_t s = nullptr;
      if (e == cudaSuccess) st = cached_plan(devices[i], N, dates, n_hist, k, h, lambda, pl);
      if (e == cudaSuccess && st == BFAST_OK) e = cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
      if (e == cudaSuccess && st == BFAST_OK) {
        bfast_args a{};
        a.Y = Y_dev[i];
        a.N = N;
        a.P = P[i];
        a.ldY = ldY[i];
        a.dates = dates;
        a.n_hist = n_hist;
        a.k = k;
        a.h = h;
        a.lambda = lambda;
        a.out_break = out_break + off;
        a.out_magnitude = out_magnitude + off;
        a.stream = s;
        std::lock_guard<std::mutex> g(pl->mu);
        st = execute_range(*pl, &a, 0, P[i]);
        launches[i] = g_launches;
        if (st == BFAST_OK) e = cudaStreamSynchronize(s);
      }
      if (s) cudaStreamDestroy(s);
      if (st == BFAST_OK && e != cudaSuccess) st = fail(BFAST_ECUDA, "%s", cudaGetErrorString(e));
      status[i] = st;
      errs[i] = g_err;
    });
    off += P[i];
  }
  for (auto &t : th) t.join();
  int total_l = 0;
  for (int i = 0; i < nshards; ++i) {
    if (status[i]) return fail(status[i], "shard %d (device %d): %s", i, devices[i], errs[i].c_str());
    total_l += launches[i];
  }
  g_launches = total_l;
  return BFAST_OK;
}

// The IPC handle: the CUDA handle of the allocation containing dev_ptr (a
// caching allocator hands out sub-blocks of larger cudaMalloc segments)
// followed by dev_ptr's byte offset in it.
typedef CUresult (*PFN_getAddressRange)(CUdeviceptr *, size_t *, CUdeviceptr);
int bfast_ipc_export(const void *dev_ptr, unsigned char *handle) {
  if (!dev_ptr || !handle) return fail(BFAST_EINVAL, "NULL pointer");
  static PFN_getAddressRange range = nullptr;
  static std::once_flag once;
  std::call_once(once, []() {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      range = (PFN_getAddressRange)f;
  });
  if (!range) return fail(BFAST_ECUDA, "cuMemGetAddressRange unavailable");
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, (CUdeviceptr)(uintptr_t)dev_ptr) != CUDA_SUCCESS)
    return fail(BFAST_EINVAL, "not a device allocation");
  cudaIpcMemHandle_t hnd;
  CUDA_TRY(cudaIpcGetMemHandle(&hnd, (void *)(uintptr_t)base));
  static_assert(sizeof(hnd) + sizeof(int64_t) == BFAST_IPC_HANDLE_BYTES, "handle size");
  const int64_t off = (int64_t)((uintptr_t)dev_ptr - (uintptr_t)base);
  std::memcpy(handle, &hnd, sizeof(hnd));
  std::memcpy(handle + sizeof(hnd), &off, sizeof(off));
  return BFAST_OK;
}

int bfast_ipc_open(const unsigned char *handle, int device, void **dev_ptr) {
  if (!handle || !dev_ptr) return fail(BFAST_EINVAL, "NULL pointer");
  *dev_ptr = nullptr;
  int prev = 0;
  CUDA_TRY(cudaGetDevice(&prev));
  if (device >= 0) CUDA_TRY(cudaSetDevice(device));
  cudaIpcMemHandle_t hnd;
  int64_t off = 0;
  std::memcpy(&hnd, handle, sizeof(hnd));
  std::memcpy(&off, handle + sizeof(hnd), sizeof(off));
  void *base = nullptr;
  const cudaError_t e = cudaIpcOpenMemHandle(&base, hnd, cudaIpcMemLazyEnablePeerAccess);
  cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(BFAST_ECUDA, "cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
  *dev_ptr = static_cast<char *>(base) + off;
  std::lock_guard<std::mutex> g(g_ipc_mu);
  g_ipc_base[*dev_ptr] = base;
  return BFAST_OK;
}

int bfast_ipc_close(void *dev_ptr) {
  if (!dev_ptr) return BFAST_OK;
  void *base = dev_ptr;
  {
    std::lock_guard<std::mutex> g(g_ipc_mu);
    auto it = g_ipc_base.find(dev_ptr);
    if (it == g_ipc_base.end()) return fail(BFAST_EINVAL, "not a pointer from bfast_ipc_open");
    base = it->second;
    g_ipc_base.erase(it);
  }
  CUDA_TRY(cudaIpcCloseMemHandle(base));
  return BFAST_OK;
}

}  // extern "C"
