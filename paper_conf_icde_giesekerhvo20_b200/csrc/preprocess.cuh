// preprocess.cuh -- the step before the hot path in the paper's pipeline
// (after a chunk is copied to the GPU,
// "removal of slices only containing NaN values"; L379: Africa, 6873 dates
// of which about 350 slices hold any data per image).
//
//   slice_any_kernel    keep[t] = 1 iff some pixel of date slice t holds a
//                       value (y == y); HBM-bound scan of the stack, a slice
//                       stops being read as soon as one value is found
//   gather_dates_kernel Yc[i][p] = Y[idx[i]][p]: the kept slices, in order,
//                       as a compact time-major stack (HBM copy)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bfast {

constexpr int kScanThreads = 256;
constexpr int kScanPerThread = 32;  // floats per thread per segment (8 x float4)
constexpr int64_t kScanSeg = (int64_t)kScanThreads * kScanPerThread;

// grid (N slices, segments of kScanSeg pixels): the slice index varies
// fastest, so the first wave reads segment 0 of every slice and a block
// whose slice is already known to hold a value returns without reading it
// (a slice with data costs about one segment, an empty one the full scan).
__global__ void __launch_bounds__(kScanThreads) slice_any_kernel(const float *__restrict__ Y, int64_t P, int64_t ldY,
                                                                 int32_t *keep, int vec4) {
  const int64_t t = blockIdx.x;
  if (*(volatile int32_t *)(keep + t)) return;
  const float *row = Y + t * ldY;
  const int64_t p0 = (int64_t)blockIdx.y * kScanSeg;
  bool any = false;
  if (vec4 && p0 + kScanSeg <= P) {
    const float4 *r4 = reinterpret_cast<const float4 *>(row + p0);
#pragma unroll
    for (int i = 0; i < kScanPerThread / 4; ++i) {
      const float4 v = __ldcs(r4 + i * kScanThreads + threadIdx.x);  // read once
      any |= (v.x == v.x) | (v.y == v.y) | (v.z == v.z) | (v.w == v.w);
    }
  } else {
    for (int i = 0; i < kScanPerThread; ++i) {
      const int64_t p = p0 + (int64_t)i * kScanThreads + threadIdx.x;
      if (p < P) {
        const float v = __ldcs(row + p);
        any |= (v == v);
      }
    }
  }
  if (__syncthreads_or(any) && threadIdx.x == 0) keep[t] = 1;
}

// grid (column blocks, Nc rows): row i of Yc = row idx[i] of Y, columns [0,
// P); an index outside [0, N) gives a row of NaN
__global__ void __launch_bounds__(256) gather_dates_kernel(const float *__restrict__ Y, int64_t N, int64_t ldY,
                                                           int64_t P, const int32_t *__restrict__ idx,
                                                           float *__restrict__ Yc, int64_t ldYc, int vec4) {
  const int64_t i = blockIdx.y;
  const int32_t t = idx[i];
  float *dst = Yc + i * ldYc;
  const int64_t step = (int64_t)gridDim.x * blockDim.x;
  if (t < 0 || t >= N) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < P; p += step)
      dst[p] = __int_as_float(0x7fc00000);
    return;
  }
  const float *src = Y + (int64_t)t * ldY;
  if (vec4) {
    const int64_t P4 = P / 4;
    const float4 *s4 = reinterpret_cast<const float4 *>(src);
    float4 *d4 = reinterpret_cast<float4 *>(dst);
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < P4; q += step) __stcs(d4 + q, __ldcs(s4 + q));
    for (int64_t p = 4 * P4 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < P; p += step)
      dst[p] = src[p];
  } else {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < P; p += step) dst[p] = __ldcs(src + p);
  }
}

// The fused kernel's MOSUM ring holds h = floor(hf * nbar) residuals per
// pixel; the plan sizes it for nbar = n (a complete history), which on a
// cloudy scene wastes most of it and can cost a tile per CTA.  This probe
// finds max h over a sample of 32-pixel groups spread over the stack (one
// warp per group, coalesced rows); the launcher sizes the ring from it (plus
// a margin) and the kernel hands any pixel whose window does not fit to the
// fp64 refit.  E = float (NaN missing) or int16_t (code == nodata missing).
template <typename E>
__global__ void __launch_bounds__(32) window_probe_kernel(const E *__restrict__ Y, int64_t ldY, int64_t P, int n,
                                                          float hf, int64_t gstride, int32_t nodata, int *hmax) {
  const int64_t p = (int64_t)blockIdx.x * gstride + threadIdx.x;
  int cnt = 0;
  if (p < P)
    for (int t = 0; t < n; ++t) {
      const E v = Y[(int64_t)t * ldY + p];
      if constexpr (sizeof(E) == 2)
        cnt += (int)v != nodata;
      else
        cnt += v == v;
    }
  int h = (int)__fmul_rn(__int2float_rn(cnt), hf);  // Fig. 12 L516 in f32 (R3)
#pragma unroll
  for (int o = 16; o; o >>= 1) h = max(h, __shfl_xor_sync(0xffffffffu, h, o));
  if (threadIdx.x == 0) atomicMax(hmax, h);
}

}  // namespace bfast
