// fp64 pipe throughput microbenchmark (DFMA, DADD, DMUL, DDIV, DSQRT) on
// sm_100a, to set the fp64 roofline (MEASURED_PEAKS has no fp64).
#include <cstdio>
#include <cuda_runtime.h>
template <int OP>
__global__ void k(double* out, int iters, double a, double b) {
  double x0 = threadIdx.x * 1e-3 + 1.0, x1 = x0 + 0.1, x2 = x0 + 0.2, x3 = x0 + 0.3;
  double x4 = x0 + 0.4, x5 = x0 + 0.5, x6 = x0 + 0.6, x7 = x0 + 0.7;
#pragma unroll 1
  for (int i = 0; i < iters; ++i) {
#define S(x) if (OP == 0) x = fma(x, a, b); else if (OP == 1) x = __dadd_rn(x, b); else if (OP == 2) x = __dmul_rn(x, a); else if (OP == 3) x = b / x; else x = sqrt(x + b);
    S(x0) S(x1) S(x2) S(x3) S(x4) S(x5) S(x6) S(x7)
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}
template <int OP>
double run(const char* name, int iters) {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out; cudaMalloc(&out, sizeof(double) * sms * 8 * 256);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<OP><<<sms * 8, 256>>>(out, iters / 10, 0.999999, 1e-7);
  cudaEventRecord(e0);
  k<OP><<<sms * 8, 256>>>(out, iters, 0.999999, 1e-7);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double ops = (double)sms * 8 * 256 * iters * 8;
  printf("{\"op\": \"%s\", \"gops_per_s\": %.1f, \"ms\": %.3f}\n", name, ops / ms / 1e6, ms);
  cudaFree(out);
  return ops / ms / 1e6;
}
int main() {
  run<0>("dfma", 20000); run<1>("dadd", 20000); run<2>("dmul", 20000);
  run<3>("ddiv", 2000); run<4>("dsqrt", 2000);
  return 0;
}
