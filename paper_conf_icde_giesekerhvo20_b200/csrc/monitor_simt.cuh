// monitor_simt.cuh -- fused one-pass BFAST-Monitor kernel, thread per pixel.
//
// One thread owns one pixel for the whole of Algorithm 1;
// a CTA owns a tile of `blockDim.x` consecutive pixels, so every load of
// the time-major stack Y[t*ldY + p] by a warp is one 128-byte row segment
// (the paper needed a transposition for this, L185/L276; our Y is already
// the paper's Y^T).  The paper's ten kernels (Fig. 12, ker 1-10) become
// stages of this single pass; no intermediate (Xsqr, beta, yhat, rbar, I)
// ever touches HBM.
//
//   pass 1, t in [0,n):   masked Gram A = sum v x x^T and moment
//                         b = sum v (y-c) x in fp32 (Alg. 1 l.2 and l.4 /
//                         Fig. 4 with the mask as a select, L181 reading R10)
//   solve:                fp64 register Cholesky of A (Alg. 1 l.3-4; the
//                         paper's Gauss-Jordan, Fig. 5, on an SPD matrix)
//   pass 2, t in [0,n):   residuals, sigma-hat (L513-L515), MOSUM seed
//                         (m^fst, L518)
//   pass 2, t in [n,N):   residuals, order-preserving rank (filterNaNsWKeys,
//                         L483-L490, as a per-thread counter), MOSUM window
//                         (L520-L525) over a shared-memory ring of the last
//                         h residuals, boundary (Alg. 1 l.10), first break
//                         (L527-L534) and the mean (L526, reading R8).
//
// Numerics: the trend column of X is centred and
// scaled by the plan and each pixel's first valid value c is subtracted
// before accumulating (the intercept absorbs it), which keeps the fp32 Gram
// well conditioned; pixels whose Cholesky pivot ratio shows conditioning
// worse than kRefitRatio are appended to a list and refitted in fp64 by
// refit_fp64.cuh.
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

namespace bfast {

struct MonitorParams {
  const float *Y;
  int64_t ldY, P, p0;  // pixels [p0, p0 + P) of the stack
  int N, n;
  const float *X;      // [N][KP] fp32, centred basis
  const double *X64;   // [N][K] fp64, same basis (refit)
  int KP;
  float hf, lambda;
  int hcap;            // ring capacity (>= max window)
  double tc, ts;       // trend centring: t' = (t - tc) / ts, t 1-based
  int32_t *out_break;
  float *out_mag, *out_beta, *out_sigma;
  int32_t *out_nbar;
  uint8_t *out_flags;
  int64_t *refit_list;   // absolute pixel indices (int64: P may exceed 2^31 across launches)
  int32_t *refit_count;
  // int16 codec (Y16 == nullptr: the float32 stack Y):
  // y = fmaf(dscale, (float)code, doffset), code == nodata -> missing
  const int16_t *Y16;
  float dscale, doffset;
  int32_t nodata;
};

// Pivot-ratio thresholds of the fp32 solve.
constexpr double kRefitRatio = 3e-2;   // worse conditioning -> fp64 refit
// |m_j|/B_j within kTieTol of 1 at some j <= j* -> the break decision is
// re-taken in fp64 by the refit kernel
constexpr float kTieTol = 1e-4f;
// reading R4: sigma-hat <= kSigmaTol * max|y_hist| is an exact fit
// (fp64 rounding residue), decided in fp64 by the refit kernel only
constexpr double kSigmaTol = 1e-10;

__device__ __forceinline__ float ld_keep(const float *p) {
  // history values are read twice: keep them in L2 (default policy)
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ float ld_stream(const float *p) {
  // monitoring values are read once
  return __ldcs(p);
}

// Window width of Fig. 12, h = t32(r32(nbar) * hf), in f32 (R3).
__device__ __forceinline__ int window_h(int nbar, float hf) {
  return (int)__fmul_rn(__int2float_rn(nbar), hf);
}

// Boundary of Alg. 1 l.10 for the 1-based compacted rank `rank1`:
// lambda * sqrt(log+(rank1 / nbar)), log+(x) = max(1, ln x) (R6).
__device__ __forceinline__ float boundary_f32(float lambda, int rank1, int nbar) {
  float x = __fdiv_rn(__int2float_rn(rank1), __int2float_rn(nbar));
  float l = logf(x);
  return lambda * sqrtf(fmaxf(l, 1.0f));
}

template <int K>
struct Tri {
  static constexpr int kN = K * (K + 1) / 2;
  __host__ __device__ static constexpr int idx(int i, int j) {  // i <= j, row-major upper
    return i * K - i * (i - 1) / 2 + (j - i);
  }
};

// Compile-time loop: f(std::integral_constant<int, I>) for I in [B, E), so
// every register-array index below is a constant (no local memory).
template <int B, int E>
struct SFor {
  template <class F>
  __device__ __forceinline__ static void run(F &&f) {
    if constexpr (B < E) {
      f(std::integral_constant<int, B>{});
      SFor<B + 1, E>::run(f);
    }
  }
};
template <int B, int E>
struct SForDown {  // I = E-1 down to B
  template <class F>
  __device__ __forceinline__ static void run(F &&f) {
    if constexpr (B < E) {
      f(std::integral_constant<int, E - 1>{});
      SForDown<B, E - 1>::run(f);
    }
  }
};

// Cholesky factorisation in place of the packed SPD matrix A (upper
// triangle, row-major): on return A holds L^T (A[idx(q,i)] = l_iq).  Returns
// the smallest pivot ratio d_j / A_jj (1 - R^2 of column j on the previous
// ones), a cheap conditioning proxy; <= 0 means not positive definite.
template <int K, typename T>
__device__ __forceinline__ T chol_factor(T (&A)[Tri<K>::kN]) {
  T minratio = T(1);
  SFor<0, K>::run([&](auto jc) {
    constexpr int j = decltype(jc)::value;
    T d = A[Tri<K>::idx(j, j)];
    SFor<0, j>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      d -= A[Tri<K>::idx(q, j)] * A[Tri<K>::idx(q, j)];
    });
    const T ratio = d / A[Tri<K>::idx(j, j)];
    minratio = ratio < minratio ? ratio : minratio;
    const T ljj = sqrt(d > T(1e-30) ? d : T(1e-30));
    const T inv = T(1) / ljj;
    A[Tri<K>::idx(j, j)] = ljj;
    SFor<j + 1, K>::run([&](auto ic) {
      constexpr int i = decltype(ic)::value;
      T s = A[Tri<K>::idx(j, i)];
      SFor<0, j>::run([&](auto qc) {
        constexpr int q = decltype(qc)::value;
        s -= A[Tri<K>::idx(q, i)] * A[Tri<K>::idx(q, j)];
      });
      A[Tri<K>::idx(j, i)] = s * inv;
    });
  });
  return minratio;
}

// Solve L L^T x = b with the factor of chol_factor.
template <int K, typename T>
__device__ __forceinline__ void chol_solve(const T (&L)[Tri<K>::kN], const T (&b)[K], T (&x)[K]) {
  T z[K];
  SFor<0, K>::run([&](auto ic) {
    constexpr int i = decltype(ic)::value;
    T s = b[i];
    SFor<0, i>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      s -= L[Tri<K>::idx(q, i)] * z[q];
    });
    z[i] = s / L[Tri<K>::idx(i, i)];
  });
  SForDown<0, K>::run([&](auto ic) {
    constexpr int i = decltype(ic)::value;
    T s = z[i];
    SFor<i + 1, K>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      s -= L[Tri<K>::idx(i, q)] * x[q];
    });
    x[i] = s / L[Tri<K>::idx(i, i)];
  });
}

// Back-transform from the centred basis with offset c to the ABI basis
// (1, t, sin, cos, ...), t 1-based.
template <int K, typename T>
__device__ __forceinline__ void store_beta(const MonitorParams &p, int64_t pix, const T (&beta)[K],
                                           T c, bool valid) {
  if (!p.out_beta) return;
  float *o = p.out_beta + pix * K;
  if (!valid) {
#pragma unroll
    for (int i = 0; i < K; ++i) o[i] = __int_as_float(0x7fc00000);
    return;
  }
  o[0] = (float)(beta[0] - beta[1] * (T)(p.tc / p.ts) + c);
  o[1] = (float)(beta[1] / (T)p.ts);
#pragma unroll
  for (int i = 2; i < K; ++i) o[i] = (float)beta[i];
}

constexpr int kUnroll = 8;

template <int K>
__global__ void __launch_bounds__(128, K >= 12 ? 2 : 4) monitor_simt_kernel(MonitorParams p) {
  extern __shared__ float4 smem4[];
  const int KP = p.KP;
  float *sX = reinterpret_cast<float *>(smem4);
  float *ring = sX + (size_t)p.N * KP;
  {
    const float4 *g = reinterpret_cast<const float4 *>(p.X);
    const int n4 = p.N * KP / 4;
    for (int i = threadIdx.x; i < n4; i += blockDim.x) smem4[i] = g[i];
  }
  __syncthreads();

  const int BP = blockDim.x;
  const int tid = threadIdx.x;
  const int64_t lp = (int64_t)blockIdx.x * BP + tid;  // local pixel
  const bool active = lp < p.P;
  const int64_t pix = p.p0 + (active ? lp : 0);
  const float *ycol = p.Y + pix;
  const int64_t ldY = p.ldY;
  const int n = p.n, N = p.N;
  const float qnan = __int_as_float(0x7fc00000);

  // ---------------- pass 1: masked Gram and moment (Alg. 1 l.2, l.4)
  float A[Tri<K>::kN];
  float b[K];
#pragma unroll
  for (int i = 0; i < Tri<K>::kN; ++i) A[i] = 0.f;
#pragma unroll
  for (int i = 0; i < K; ++i) b[i] = 0.f;
  int nbar = 0;
  float c0 = 0.f, ymax = 0.f;
  bool have = false;

  for (int t0 = 0; t0 < n; t0 += kUnroll) {
    float yv[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      int t = t0 + u;
      yv[u] = (active && t < n) ? ld_keep(ycol + (int64_t)t * ldY) : qnan;
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int t = t0 + u;
      if (t >= n) break;
      const float y = yv[u];
      const bool v = (y == y);
      if (v && !have) { c0 = y; have = true; }
      const float yp = v ? (y - c0) : 0.f;
      ymax = v ? fmaxf(ymax, fabsf(y)) : ymax;
      nbar += v ? 1 : 0;
      float x[K];
      const float *xr = sX + (size_t)t * KP;
#pragma unroll
      for (int i = 0; i < K; i += 2) {
        float2 xx = *reinterpret_cast<const float2 *>(xr + i);
        x[i] = xx.x;
        x[i + 1] = xx.y;
      }
#pragma unroll
      for (int i = 0; i < K; ++i) {
        const float w = v ? x[i] : 0.f;
#pragma unroll
        for (int j = i; j < K; ++j) A[Tri<K>::idx(i, j)] = fmaf(w, x[j], A[Tri<K>::idx(i, j)]);
        b[i] = fmaf(yp, x[i], b[i]);
      }
    }
  }

  // ---------------- solve (Alg. 1 l.3-4): Cholesky of the SPD Gram in
  // fp32 registers; the factor is kept for the refinement step below
  const int h = window_h(nbar, p.hf);
  bool deg = (nbar < K + 1) || (h < 1);
  float beta[K];
  bool refit = false;
  {
    const float minratio = chol_factor<K, float>(A);
    chol_solve<K, float>(A, b, beta);
    if (!deg && !(minratio >= (float)kRefitRatio)) refit = true;
    if (deg) {
#pragma unroll
      for (int i = 0; i < K; ++i) beta[i] = 0.f;
    }
  }

  // ---------------- pass 2a: history residuals r0 = y' - x'beta0, their
  // moment db = sum v r0 x (one step of iterative refinement of the fp32
  // normal equations), sigma-hat, and the ring of the last residuals with
  // their date indices (for the MOSUM seed m^fst, L518)
  const int hh = deg ? 1 : h;
  const int hcap = p.hcap;
  float *myring = ring + tid;
  int16_t *mydate = reinterpret_cast<int16_t *>(ring + (size_t)hcap * BP) + tid;
  float s2 = 0.f;
  float db[K];
#pragma unroll
  for (int i = 0; i < K; ++i) db[i] = 0.f;
  int cr = 0, ws = 0;  // compacted rank, ring write slot (= cr mod hcap)
  for (int t0 = 0; t0 < n; t0 += kUnroll) {
    float yv[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      int t = t0 + u;
      yv[u] = (active && t < n) ? ld_keep(ycol + (int64_t)t * ldY) : qnan;
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int t = t0 + u;
      if (t >= n) break;
      const float y = yv[u];
      const float *xr = sX + (size_t)t * KP;
      float x[K];
#pragma unroll
      for (int i = 0; i < K; i += 2) {
        float2 xx = *reinterpret_cast<const float2 *>(xr + i);
        x[i] = xx.x;
        x[i + 1] = xx.y;
      }
      float yhat = 0.f;
#pragma unroll
      for (int i = 0; i < K; ++i) yhat = fmaf(beta[i], x[i], yhat);
      const bool v = (y == y);
      const float r = v ? (y - c0) - yhat : 0.f;
#pragma unroll
      for (int i = 0; i < K; ++i) db[i] = fmaf(r, x[i], db[i]);
      s2 = fmaf(r, r, s2);
      if (v) {
        myring[ws * BP] = r;
        mydate[ws * BP] = (int16_t)t;
        ws = (ws + 1 == hcap) ? 0 : ws + 1;
        ++cr;
      }
    }
  }
  // refined fit beta = beta0 + A^-1 db (same factor); sigma-hat of the
  // refined residuals: sum (r0 - x'dbeta)^2 = s2 - dbeta.db (A dbeta = db)
  float sigma;
  float dbf[K];
  {
    chol_solve<K, float>(A, db, dbf);
    float lin = 0.f;
#pragma unroll
    for (int i = 0; i < K; ++i) {
      if (deg) dbf[i] = 0.f;
      lin = fmaf(dbf[i], db[i], lin);
      beta[i] += dbf[i];
    }
    sigma = sqrtf(fmaxf(s2 - lin, 0.f) / (float)(nbar - K));
    // sigma^2 = s2 - lin cancels when the refinement step is large next to
    // the residual sum: the fp32 sigma-hat is then unreliable -> fp64 refit
    if (!(lin <= 1e-2f * s2)) refit = true;
  }
  // noise within 2e-3 of the signal scale: fp32 fitted values (~1e-7 |y|)
  // are no longer negligible next to sigma-hat -> fp64 refit (R12), which
  // also takes the sigma-hat ~ 0 decision of reading R4 in fp64
  if (!deg && !(sigma > 2e-3f * ymax)) refit = true;
  const float inv_scale = 1.0f / (sigma * sqrtf((float)nbar));
  // MOSUM seed: the last h-1 history residuals (ranks nbar-h+1 .. nbar-1),
  // corrected to the refined fit in the ring, summed into W
  float W = 0.f;
  {
    const int nseed = deg ? 0 : hh - 1;
    int slot = ws - nseed;
    slot += (slot < 0) ? hcap : 0;
    for (int q = 0; q < nseed; ++q) {
      const int t = mydate[slot * BP];
      const float *xr = sX + (size_t)t * KP;
      float corr = 0.f;
#pragma unroll
      for (int i = 0; i < K; i += 2) {
        float2 xx = *reinterpret_cast<const float2 *>(xr + i);
        corr = fmaf(dbf[i], xx.x, corr);
        corr = fmaf(dbf[i + 1], xx.y, corr);
      }
      const float r = myring[slot * BP] - corr;
      myring[slot * BP] = r;
      W += r;
      slot = (slot + 1 == hcap) ? 0 : slot + 1;
    }
  }

  // ---------------- pass 2b: monitoring (Alg. 1 l.6-12, Fig. 12 ker 9-10)
  float msum = 0.f;
  int brk = -1;
  const float lam = p.lambda;
  const float lam_lo = lam * (1.0f - kTieTol);
  bool tie = false;
  for (int t0 = n; t0 < N; t0 += kUnroll) {
    float yv[kUnroll];
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      int t = t0 + u;
      yv[u] = (active && t < N) ? ld_stream(ycol + (int64_t)t * ldY) : qnan;
    }
#pragma unroll
    for (int u = 0; u < kUnroll; ++u) {
      const int t = t0 + u;
      if (t >= N) break;
      const float y = yv[u];
      const float *xr = sX + (size_t)t * KP;
      float yhat = 0.f;
#pragma unroll
      for (int i = 0; i < K; i += 2) {
        float2 xx = *reinterpret_cast<const float2 *>(xr + i);
        yhat = fmaf(beta[i], xx.x, yhat);
        yhat = fmaf(beta[i + 1], xx.y, yhat);
      }
      const float r = (y - c0) - yhat;
      if (y == y) {
        if (cr > nbar) {  // j >= 1: the window drops rank cr - h
          int rs = ws - hh;
          rs += (rs < 0) ? hcap : 0;
          W -= myring[rs * BP];
        }
        W += r;
        myring[ws * BP] = r;
        ws = (ws + 1 == hcap) ? 0 : ws + 1;
        const float m = W * inv_scale;
        msum += m;
        if (brk < 0 && fabsf(m) > lam_lo) {
          const float B = boundary_f32(lam, cr + 1, nbar);
          const float am = fabsf(m);
          tie |= fabsf(am - B) <= kTieTol * B;
          if (am > B) brk = t - n;
        }
        ++cr;
      }
    }
  }
  const int Nbar = cr;
  if (Nbar - nbar < 1) deg = true;

  if (!active) return;
  const bool fit_ok = !((nbar < K + 1) || (h < 1) || (Nbar - nbar < 1));
  p.out_break[pix] = deg ? -2 : brk;
  p.out_mag[pix] = deg ? qnan : msum / (float)(Nbar - nbar);
  if (p.out_sigma) p.out_sigma[pix] = fit_ok ? sigma : qnan;
  if (p.out_nbar) p.out_nbar[pix] = nbar;
  if (p.out_flags) p.out_flags[pix] = deg ? 1u : 0u;
  store_beta<K, float>(p, pix, beta, c0, fit_ok);
  if ((refit || tie) && fit_ok && !(nbar < K + 1)) {
    // warp-aggregated append to the fp64 refit list
    const unsigned mask = __activemask();
    const int leader = __ffs(mask) - 1;
    const int lane = tid & 31;
    int base = 0;
    if (lane == leader) base = atomicAdd(p.refit_count, __popc(mask));
    base = __shfl_sync(mask, base, leader);
    p.refit_list[base + __popc(mask & ((1u << lane) - 1))] = pix;
  }
}

}  // namespace bfast
