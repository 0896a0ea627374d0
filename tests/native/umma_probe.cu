// umma_probe.cu -- hardware check of the sm100.cuh primitives the tensor-core
// monitor kernel relies on: bulk async copy + mbarrier transaction counts,
// TMEM allocation, K-major no-swizzle smem descriptors, tcgen05.mma
// (kind::f16, bf16 -> fp32) for every N the kernel uses, commit, TMEM loads.
// Built and run by tests/test_tc_primitives.py on the GPU box:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 umma_probe.cu -o probe
// Prints one line per case and "ALL OK" on success.
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>

#include "../../paper_conf_icde_giesekerhvo20_b200/csrc/sm100.cuh"

using namespace sm100;

__global__ void probe_kernel(const uint16_t *A, const uint16_t *B, float *D, int K, int N) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t bar_load, bar_mma;
  __shared__ uint32_t tbase_s;
  uint8_t *stage = smem;                      // raw A rows [128][K] bf16
  uint8_t *As = stage + 128 * K * 2;          // canonical K-major A
  uint8_t *Bs = As + 128 * K * 2;             // canonical K-major B
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    mbar_init(&bar_load, 1);
    mbar_init(&bar_mma, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (tid == 0) {
    mbar_arrive_expect_tx(&bar_load, 128 * K * 2);
    // one bulk copy per row (as the monitor kernel copies one date row)
    for (int r = 0; r < 128; ++r) bulk_g2s(stage + r * K * 2, A + (size_t)r * K, K * 2, &bar_load);
  }
  if (warp == 0) tmem_alloc(&tbase_s, 256);
  mbar_wait(&bar_load, 0);
  for (int c = 0; c < K / 8; ++c) {
    uint4 v = *reinterpret_cast<const uint4 *>(stage + tid * K * 2 + c * 16);
    *reinterpret_cast<uint4 *>(As + kmajor_off(tid, 8 * c, 128)) = v;
  }
  for (int n = tid; n < N; n += blockDim.x)
    for (int c = 0; c < K / 8; ++c) {
      uint4 v = *reinterpret_cast<const uint4 *>(B + (size_t)n * K + c * 8);
      *reinterpret_cast<uint4 *>(Bs + kmajor_off(n, 8 * c, N)) = v;
    }
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tbase_s;
  if (tid == 0) {
    const uint32_t idesc = idesc_bf16_f32(128, N);
    for (int s = 0; s < K / 16; ++s) {
      uint64_t ad = smem_desc(smem_u32(As) + s * 2 * 128 * 16, 128 * 16, 128);
      uint64_t bd = smem_desc(smem_u32(Bs) + s * 2 * N * 16, N * 16, 128);
      umma_bf16(tbase, ad, bd, idesc, s > 0 ? 1u : 0u);
    }
    umma_commit(&bar_mma);
  }
  mbar_wait(&bar_mma, 0);
  tc_fence_after();
  for (int c0 = 0; c0 < N; c0 += 16) {
    float v[16];
    tmem_ld16(tbase + ((uint32_t)(32 * (warp & 3)) << 16) + c0, v);
    tmem_ld_wait();
    for (int i = 0; i < 16; ++i) D[(size_t)tid * N + c0 + i] = v[i];
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, 256);
}

// Same product with A held in TMEM (tcgen05.st by the thread owning the row,
// then tcgen05.mma with the A operand in tensor memory).
__global__ void probe_ts_kernel(const uint16_t *A, const uint16_t *B, float *D, int K, int N) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t bar_mma;
  __shared__ uint32_t tbase_s;
  uint8_t *Bs = smem;
  const int tid = threadIdx.x, warp = tid >> 5;
  if (tid == 0) {
    mbar_init(&bar_mma, 1);
    fence_mbar_init();
  }
  if (warp == 0) tmem_alloc(&tbase_s, 512);
  for (int n = tid; n < N; n += blockDim.x)
    for (int c = 0; c < K / 8; ++c) {
      uint4 v = *reinterpret_cast<const uint4 *>(B + (size_t)n * K + c * 8);
      *reinterpret_cast<uint4 *>(Bs + kmajor_off(n, 8 * c, N)) = v;
    }
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tbase_s;
  const uint32_t acol = 256, lanebase = tbase + ((uint32_t)(32 * (warp & 3)) << 16);
  for (int c = 0; c < K / 16; ++c) {
    uint32_t w[8];
    for (int j = 0; j < 8; ++j)
      w[j] = (uint32_t)A[(size_t)tid * K + 16 * c + 2 * j] | ((uint32_t)A[(size_t)tid * K + 16 * c + 2 * j + 1] << 16);
    tmem_st8(lanebase + acol + 8 * c, w);
  }
  tmem_st_wait();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (tid == 0) {
    const uint32_t idesc = idesc_bf16_f32(128, N);
    for (int s = 0; s < K / 16; ++s) {
      uint64_t bd = smem_desc(smem_u32(Bs) + s * 2 * N * 16, N * 16, 128);
      umma_bf16_ts(tbase, tbase + acol + 8 * s, bd, idesc, s > 0 ? 1u : 0u);
    }
    umma_commit(&bar_mma);
  }
  mbar_wait(&bar_mma, 0);
  tc_fence_after();
  for (int c0 = 0; c0 < N; c0 += 16) {
    float v[16];
    tmem_ld16(lanebase + c0, v);
    tmem_ld_wait();
    for (int i = 0; i < 16; ++i) D[(size_t)tid * N + c0 + i] = v[i];
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, 512);
}

static uint16_t to_bf16(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  u += 0x7fff + ((u >> 16) & 1);
  return (uint16_t)(u >> 16);
}
static float from_bf16(uint16_t h) {
  uint32_t u = (uint32_t)h << 16;
  float f;
  memcpy(&f, &u, 4);
  return f;
}

int main() {
  int fails = 0;
  const int Ks[] = {16, 32, 64};
  const int Ns[] = {16, 48, 64, 128, 256};
  for (int K : Ks)
    for (int N : Ns) {
      std::vector<uint16_t> A(128 * K), B(N * K);
      srand(K * 1000 + N);
      for (auto &a : A) a = to_bf16((rand() % 2001 - 1000) / 256.0f);
      for (auto &b : B) b = to_bf16((rand() % 2001 - 1000) / 512.0f);
      uint16_t *dA, *dB;
      float *dD;
      cudaMalloc(&dA, A.size() * 2);
      cudaMalloc(&dB, B.size() * 2);
      cudaMalloc(&dD, 128 * N * 4);
      cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
      cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
      size_t smem = 128 * K * 2 * 2 + N * K * 2;
      cudaFuncSetAttribute(probe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      probe_kernel<<<1, 128, smem>>>(dA, dB, dD, K, N);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<float> D(128 * N);
      cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
      double maxerr = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < N; ++n) {
          double ref = 0;
          for (int k = 0; k < K; ++k) ref += (double)from_bf16(A[m * K + k]) * from_bf16(B[n * K + k]);
          maxerr = fmax(maxerr, fabs(ref - D[m * N + n]));
        }
      bool ok = e == cudaSuccess && maxerr < 1e-3;
      printf("K=%d N=%d err=%s maxerr=%g %s\n", K, N, cudaGetErrorString(e), maxerr, ok ? "ok" : "FAIL");
      fails += !ok;
      cudaFree(dA);
      cudaFree(dB);
      cudaFree(dD);
      if (e != cudaSuccess) return 1;
    }
  // A from TMEM, the shapes of the yhat GEMM (K = 6K' padded to 16)
  const int Ks2[] = {16, 48, 96};
  const int Ns2[] = {16, 32};
  for (int K : Ks2)
    for (int N : Ns2) {
      std::vector<uint16_t> A(128 * K), B(N * K);
      srand(K * 7 + N);
      for (auto &a : A) a = to_bf16((rand() % 2001 - 1000) / 256.0f);
      for (auto &b : B) b = to_bf16((rand() % 2001 - 1000) / 512.0f);
      uint16_t *dA, *dB;
      float *dD;
      cudaMalloc(&dA, A.size() * 2);
      cudaMalloc(&dB, B.size() * 2);
      cudaMalloc(&dD, 128 * N * 4);
      cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
      cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
      size_t smem = N * K * 2;
      cudaFuncSetAttribute(probe_ts_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      probe_ts_kernel<<<1, 128, smem>>>(dA, dB, dD, K, N);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<float> D(128 * N);
      cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
      double maxerr = 0;
      for (int m = 0; m < 128; ++m)
        for (int n = 0; n < N; ++n) {
          double ref = 0;
          for (int k = 0; k < K; ++k) ref += (double)from_bf16(A[m * K + k]) * from_bf16(B[n * K + k]);
          maxerr = fmax(maxerr, fabs(ref - D[m * N + n]));
        }
      bool ok = e == cudaSuccess && maxerr < 1e-3;
      printf("TMEM-A K=%d N=%d err=%s maxerr=%g %s\n", K, N, cudaGetErrorString(e), maxerr, ok ? "ok" : "FAIL");
      fails += !ok;
      cudaFree(dA);
      cudaFree(dB);
      cudaFree(dD);
      if (e != cudaSuccess) return 1;
    }
  if (!fails) printf("ALL OK\n");
  return fails ? 1 : 0;
}
