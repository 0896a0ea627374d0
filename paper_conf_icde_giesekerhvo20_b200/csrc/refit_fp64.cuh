// refit_fp64.cuh -- fp64 recomputation of the pixels the fp32 pass flagged
// as ill-conditioned (pivot ratio < kRefitRatio), one warp per pixel.
//
// Same definitions as the fused pass (Algorithm 1; Fig. 12
// L478-L537), organised for a warp instead of a thread:
//   - lanes take 32 consecutive dates; validity is a warp ballot and the
//     order-preserving compaction of filterNaNsWKeys (L483-L490) is the
//     popc-prefix of that ballot (the scan+scatter of Fig. 12 in one
//     instruction pair);
//   - the masked Gram / moment (Alg. 1 l.2, l.4) are accumulated per lane in
//     fp64 and reduced with xor-shuffles;
//   - every lane solves the same fp64 system (Cholesky, rank test on the
//     unit-diagonal pivots as the oracle's reading R4 does);
//   - compacted residuals go to a per-warp shared-memory array; the MOSUM
//     windows (Eq. (4)) are prefix-sum differences; the first
//     break is a ballot over j in order (the (bool, idx) reduce of
//     L532-L534) and the mean a shuffle reduction.
#pragma once
#include "monitor_simt.cuh"

namespace bfast {

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// shared memory per warp, in doubles: prefix sums [N + 1], kRefitBufs
// column buffers [N] f32 (the current pixel's and the next ones', in
// flight) and the compacted date list Ic [N] u16
#ifndef BFAST_REFIT_BUFS
#define BFAST_REFIT_BUFS 2
#endif
constexpr int kRefitBufs = BFAST_REFIT_BUFS;
__host__ __device__ constexpr size_t refit_warp_doubles(int N) {
  return (size_t)(N + 1) + ((size_t)kRefitBufs * N + 1) / 2 + ((size_t)N + 3) / 4;
}

// one 4-byte global -> shared copy through the LSU's asynchronous path
// (cp.async, no register staging); completion tracked per thread by groups
__device__ __forceinline__ void cp_async4(float *dst, const float *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_prev() {
  asm volatile("cp.async.wait_group %0;" ::"n"(kRefitBufs - 1) : "memory");
}

// the pixel's column is N strided 4-byte reads (one DRAM burst each): every
// lane issues its N/32 copies at once, straight into shared memory
__device__ __forceinline__ void refit_fetch_column(float *Yc, const float *Y, int64_t pix, int N, int64_t ldY,
                                                   int lane) {
  const float *ycol = Y + pix;
  for (int t = lane; t < N; t += 32) cp_async4(Yc + t, ycol + (int64_t)t * ldY);
}

// an int16-coded stack (f4): the column decoded exactly as the oracle does,
// y = fmaf(scale, code, offset) (one rounding), the nodata code -> NaN; plain
// loads (cp.async has no 2-byte form), ordered by the caller's __syncwarp
__device__ __forceinline__ void refit_decode_column(float *Yc, const MonitorParams &p, int64_t pix, int N, int lane) {
  const int16_t *ycol = p.Y16 + pix;
  for (int t = lane; t < N; t += 32) {
    const int v = ycol[(int64_t)t * p.ldY];
    Yc[t] = v == p.nodata ? __int_as_float(0x7fc00000) : fmaf(p.dscale, (float)v, p.doffset);
  }
}
__device__ __forceinline__ void refit_column(float *Yc, const MonitorParams &p, int64_t pix, int N, int lane) {
  if (p.Y16)
    refit_decode_column(Yc, p, pix, N, lane);
  else
    refit_fetch_column(Yc, p.Y, pix, N, p.ldY, lane);
}

template <int K>
__global__ void __launch_bounds__(128) refit_fp64_kernel(MonitorParams p) {
  // per warp: [N + 1] compacted residual prefix sums (fp64), then
  // kRefitBufs column buffers [N] (fp32): the column of item i is used
  // while the columns of the next kRefitBufs - 1 items are being copied in
  // (software pipeline over the warp's items), then the date list Ic
  extern __shared__ double rbuf_all[];
  const int lane = threadIdx.x & 31;
  const int wib = threadIdx.x >> 5;
  const int wpb = blockDim.x >> 5;
  double *S = rbuf_all + (size_t)wib * refit_warp_doubles(p.N);
  float *Ybuf = reinterpret_cast<float *>(S + p.N + 1);
  uint16_t *Ic = reinterpret_cast<uint16_t *>(Ybuf + kRefitBufs * p.N);
  const int count = *p.refit_count;
  const int n = p.n, N = p.N;
  const int64_t ldY = p.ldY;
  const double qnan = __longlong_as_double(0x7ff8000000000000ll);
  const int stride = gridDim.x * wpb;

  int item = blockIdx.x * wpb + wib;
#pragma unroll
  for (int q = 0; q < kRefitBufs - 1; ++q) {  // prologue: the first kRefitBufs - 1 columns
    const int it = item + q * stride;
    if (it < count) refit_column(Ybuf + q * N, p, p.refit_list[it], N, lane);
    cp_async_commit();
  }
  for (int buf = 0; item < count; item += stride, buf = buf + 1 == kRefitBufs ? 0 : buf + 1) {
    const int64_t pix = p.refit_list[item];  // absolute pixel index
    const int ahead = item + (kRefitBufs - 1) * stride;
    // the buffer this column goes to was read by the previous item (whose
    // trailing __syncwarp ordered those reads before these copies)
    const int abuf = buf == 0 ? kRefitBufs - 1 : buf - 1;
    if (ahead < count) refit_column(Ybuf + abuf * N, p, p.refit_list[ahead], N, lane);
    cp_async_commit();
    cp_async_wait_prev();  // this lane's copies of the current column landed
    __syncwarp();          // ... and every other lane's
    const float *Yc = Ybuf + buf * N;
    // ---- order-preserving compaction (filterNaNsWKeys, L483-L490): Ic[c]
    // = date of the c-th valid value, c < Nbar; the ranks are the popc
    // prefix of the validity ballot, so every later loop runs over the
    // N̄ valid dates only, all lanes busy
    int cr = 0, nbar = 0;
#pragma unroll 1
    for (int t0 = 0; t0 < N; t0 += 32) {
      const int t = t0 + lane;
      const bool v = t < N && Yc[t] == Yc[t];
      const unsigned bal = __ballot_sync(0xffffffffu, v);
      if (v) Ic[cr + __popc(bal & ((1u << lane) - 1))] = (uint16_t)t;
      if (t0 < n) nbar += __popc(bal & (t0 + 32 <= n ? 0xffffffffu : ((1u << (n - t0)) - 1u)));
      cr += __popc(bal);
    }
    const int Nbar = cr;
    __syncwarp();  // Ic is read across lanes below
    // ---- history: offset c0 = first valid history value, Gram, moment (fp64)
    double A[Tri<K>::kN], b[K];
#pragma unroll
    for (int i = 0; i < Tri<K>::kN; ++i) A[i] = 0.0;
#pragma unroll
    for (int i = 0; i < K; ++i) b[i] = 0.0;
    const double c0 = nbar > 0 ? (double)Yc[Ic[0]] : 0.0;
    double ymax = 0.0;
#pragma unroll 1
    for (int c = lane; c < nbar; c += 32) {
      const int t = Ic[c];
      const float yf = Yc[t];
      const double y = (double)yf - c0;
      ymax = fmax(ymax, fabs((double)yf));
      const double *x = p.X64 + (size_t)t * K;
      double xr[K];
#pragma unroll
      for (int i = 0; i < K; ++i) xr[i] = x[i];
#pragma unroll
      for (int i = 0; i < K; ++i) {
#pragma unroll
        for (int j = i; j < K; ++j) A[Tri<K>::idx(i, j)] = fma(xr[i], xr[j], A[Tri<K>::idx(i, j)]);
        b[i] = fma(y, xr[i], b[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < Tri<K>::kN; ++i) A[i] = warp_sum(A[i]);
#pragma unroll
    for (int i = 0; i < K; ++i) b[i] = warp_sum(b[i]);
#pragma unroll
    for (int o = 16; o; o >>= 1) ymax = fmax(ymax, __shfl_xor_sync(0xffffffffu, ymax, o));

    double beta[K];
    const double minratio = chol_factor<K, double>(A);
    chol_solve<K, double>(A, b, beta);
    const int h = window_h(nbar, p.hf);
    bool deg = !(minratio > 1e-9);  // rank test (reading R4)

    // ---- residuals of the valid dates in compacted order, as prefix sums S
    double s2 = 0.0;
    if (lane == 0) S[0] = 0.0;
    __syncwarp();  // S[0] is read by every lane below
#pragma unroll 1
    for (int c0i = 0; c0i < Nbar; c0i += 32) {
      const int c = c0i + lane;
      double r = 0.0;
      if (c < Nbar) {
        const int t = Ic[c];
        const double *x = p.X64 + (size_t)t * K;
        double yhat = 0.0;
#pragma unroll
        for (int i = 0; i < K; ++i) yhat = fma(x[i], beta[i], yhat);
        r = ((double)Yc[t] - c0) - yhat;
      }
      if (c < nbar) s2 += r * r;
      // inclusive warp scan of r (lanes past N̄ carry 0)
      double sc = r;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        double up = __shfl_up_sync(0xffffffffu, sc, o);
        if (lane >= o) sc += up;
      }
      const double base = S[c0i];
      __syncwarp();
      if (c < Nbar) S[c + 1] = base + sc;
      __syncwarp();
    }
    s2 = warp_sum(s2);
    const double sigma = sqrt(s2 / (double)(nbar - K));
    // reading R4: sigma-hat at fp64 rounding level of an exact fit (the
    // oracle's ORACLE_SIGMA_TOL rule; PAPER.md L515/L524 divide by it)
    if (!(sigma > kSigmaTol * ymax)) deg = true;
    // ---- MOSUM by prefix differences, first break, mean
    const double scale = sigma * sqrt((double)nbar);
    double msum = 0.0;
    int jstar = -1;
    const int J = Nbar - nbar;
    for (int j0 = 0; j0 < J; j0 += 32) {
      const int j = j0 + lane;
      bool hit = false;
      if (j < J) {
        const double m = (S[nbar + j + 1] - S[nbar + j - h + 1]) / scale;
        msum += m;
        const double x = (double)(nbar + 1 + j) / (double)nbar;
        const double B = (double)p.lambda * sqrt(fmax(1.0, log(x)));
        hit = fabs(m) > B;
      }
      const unsigned hb = __ballot_sync(0xffffffffu, hit);
      if (jstar < 0 && hb) jstar = j0 + __ffs(hb) - 1;
    }
    msum = warp_sum(msum);
    // original date index of compacted rank nbar + jstar (REMAPINDICES)
    const int brk = jstar >= 0 ? (int)Ic[nbar + jstar] - n : -1;
    if (lane == 0) {
      p.out_break[pix] = deg ? -2 : brk;
      p.out_mag[pix] = deg ? (float)qnan : (float)(msum / (double)J);
      if (p.out_sigma) p.out_sigma[pix] = (float)sigma;
#ifdef BFAST_REFIT_WHY
      if (p.out_flags) p.out_flags[pix] = (uint8_t)((p.out_flags[pix] & 0xF0u) | (deg ? 1u : 0u) | 2u);
#else
      if (p.out_flags) p.out_flags[pix] = (uint8_t)((deg ? 1u : 0u) | 2u);
#endif
      if (p.out_beta) {
        float *o = p.out_beta + pix * K;
        const bool rank_def = !(minratio > 1e-9);
        o[0] = rank_def ? (float)qnan : (float)(beta[0] - beta[1] * p.tc / p.ts + c0);
        o[1] = rank_def ? (float)qnan : (float)(beta[1] / p.ts);
#pragma unroll
        for (int i = 2; i < K; ++i) o[i] = rank_def ? (float)qnan : (float)beta[i];
      }
    }
    __syncwarp();
  }
}

}  // namespace bfast
