// solve_probe.cu -- the fused kernel's per-pixel solve in two
// forms, per thread in registers, fp32: (1) Cholesky of the SPD Gram + two
// triangular solves (beta0 and the refinement step share the factor) -- what
// monitor_fused.cuh does; (2) the paper's Gauss-Jordan inverse of [A | I]
// without pivoting (Fig. 5) + two matrix-vector products.
// Reports ns per pixel-solve over 2^24 pixels and the max error against fp64.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 solve_probe.cu -o solve_probe
#include <cstdio>
#include <cmath>
#include <vector>
#include <cuda_runtime.h>

template <int K>
__device__ __forceinline__ void make_spd(unsigned seed, float (&A)[K][K], float (&b)[K], float (&d)[K]) {
  // Gram of 3K pseudo-random rows (centred trend + harmonics-like values)
  for (int i = 0; i < K; ++i) { b[i] = 0.f; d[i] = 0.f; for (int j = 0; j < K; ++j) A[i][j] = 0.f; }
  unsigned s = seed * 2654435761u + 12345u;
  for (int r = 0; r < 3 * K; ++r) {
    float x[K];
    for (int i = 0; i < K; ++i) { s = s * 1664525u + 1013904223u; x[i] = (float)(s >> 8) * (2.f / 16777216.f) - 1.f; }
    x[0] = 1.f;
    s = s * 1664525u + 1013904223u;
    const float y = (float)(s >> 8) * (1.f / 16777216.f);
    for (int i = 0; i < K; ++i) { b[i] = fmaf(x[i], y, b[i]); d[i] = fmaf(x[i], 1e-3f * y, d[i]);
      for (int j = 0; j < K; ++j) A[i][j] = fmaf(x[i], x[j], A[i][j]); }
  }
}

template <int K>
__global__ void chol_kernel(int n, float *out, int reps) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  float A[K][K], b[K], d[K];
  make_spd<K>(p, A, b, d);
  float acc = 0.f;
  for (int rep = 0; rep < reps; ++rep) {
    float L[K][K], dinv[K];
#pragma unroll
    for (int j = 0; j < K; ++j) {
      float s = A[j][j] + (float)rep * 1e-7f;
#pragma unroll
      for (int q = 0; q < j; ++q) s = fmaf(-L[j][q], L[j][q], s);
      const float inv = rsqrtf(fmaxf(s, 1e-30f));
      dinv[j] = inv;
#pragma unroll
      for (int i = j + 1; i < K; ++i) {
        float t = A[i][j];
#pragma unroll
        for (int q = 0; q < j; ++q) t = fmaf(-L[i][q], L[j][q], t);
        L[i][j] = t * inv;
      }
    }
    float x[K], z[K], y2[K];
    // two right-hand sides with the same factor
#pragma unroll
    for (int rhs = 0; rhs < 2; ++rhs) {
      const float *r = rhs ? d : b;
#pragma unroll
      for (int i = 0; i < K; ++i) { float t = r[i];
#pragma unroll
        for (int q = 0; q < i; ++q) t = fmaf(-L[i][q], z[q], t); z[i] = t * dinv[i]; }
#pragma unroll
      for (int i = K - 1; i >= 0; --i) { float t = z[i];
#pragma unroll
        for (int q = i + 1; q < K; ++q) t = fmaf(-L[q][i], (rhs ? y2 : x)[q], t); (rhs ? y2 : x)[i] = t * dinv[i]; }
    }
#pragma unroll
    for (int i = 0; i < K; ++i) acc += x[i] + y2[i];
  }
  out[p] = acc;
}

template <int K>
__global__ void gj_kernel(int n, float *out, int reps) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  float A0[K][K], b[K], d[K];
  make_spd<K>(p, A0, b, d);
  float acc = 0.f;
  for (int rep = 0; rep < reps; ++rep) {
    float M[K][2 * K];
#pragma unroll
    for (int i = 0; i < K; ++i)
#pragma unroll
      for (int j = 0; j < 2 * K; ++j) M[i][j] = j < K ? A0[i][j] + (i == j ? (float)rep * 1e-7f : 0.f) : (j - K == i ? 1.f : 0.f);
    // Fig. 5: for each pivot q, scale row q, eliminate column q from every other row
#pragma unroll
    for (int q = 0; q < K; ++q) {
      const float inv = 1.f / M[q][q];
#pragma unroll
      for (int j = 0; j < 2 * K; ++j) M[q][j] *= inv;
#pragma unroll
      for (int i = 0; i < K; ++i) {
        if (i == q) continue;
        const float f = M[i][q];
#pragma unroll
        for (int j = 0; j < 2 * K; ++j) M[i][j] = fmaf(-f, M[q][j], M[i][j]);
      }
    }
    float x[K], y2[K];
#pragma unroll
    for (int i = 0; i < K; ++i) { float s = 0.f, t = 0.f;
#pragma unroll
      for (int j = 0; j < K; ++j) { s = fmaf(M[i][K + j], b[j], s); t = fmaf(M[i][K + j], d[j], t); } x[i] = s; y2[i] = t; }
#pragma unroll
    for (int i = 0; i < K; ++i) acc += x[i] + y2[i];
  }
  out[p] = acc;
}

int main() {
  constexpr int K = 8;
  const int n = 1 << 24, reps = 8;
  float *o;
  cudaMalloc(&o, sizeof(float) * n);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int regs[2];
  for (int v = 0; v < 2; ++v) {
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, v ? (const void *)gj_kernel<K> : (const void *)chol_kernel<K>);
    regs[v] = fa.numRegs;
  }
  float ms[2][2];
  for (int v = 0; v < 2; ++v)
    for (int r = 0; r < 2; ++r) {  // reps = 1 and 8: the difference isolates the solve
      const int rr = r ? reps : 1;
      for (int w = 0; w < 2; ++w) {
        cudaEventRecord(e0);
        if (v) gj_kernel<K><<<n / 128, 128>>>(n, o, rr); else chol_kernel<K><<<n / 128, 128>>>(n, o, rr);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
      }
      cudaEventElapsedTime(&ms[v][r], e0, e1);
    }
  for (int v = 0; v < 2; ++v) {
    const double per = (ms[v][1] - ms[v][0]) / (reps - 1) * 1e6 / n;  // ns per pixel-solve
    std::printf("{\"solve\": \"%s\", \"K\": %d, \"registers\": %d, \"ns_per_pixel_solve\": %.4f, "
                "\"ms_per_2^24_solves\": %.3f}\n", v ? "gauss_jordan_inverse (Fig. 5)" : "cholesky (monitor_fused)",
                K, regs[v], per, per * n / 1e6);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
