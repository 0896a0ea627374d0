#include <cstdio>
__global__ void k(unsigned long long *out, int ns) {
  unsigned long long t0 = clock64(), it = 0;
  while (clock64() - t0 < 2000000ull) { __nanosleep(ns); ++it; }
  out[0] = it;
}
int main() {
  unsigned long long *d, h;
  cudaMalloc(&d, 8);
  for (int ns : {32, 64, 128, 256, 512, 1024}) {
    k<<<1, 1>>>(d, ns); cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    printf("nanosleep(%d): %llu iterations in 2e6 cycles -> %.1f cycles/iter\n", ns, h, 2e6 / h);
  }
}
