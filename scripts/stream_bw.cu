// Bandwidth of the row-streaming access pattern used by the step kernels:
// NI input fields read and NO output fields written per cell, one thread per
// column walking KS rows, blocks of TB threads; optional 2 columns/thread
// (16-B vector accesses).  Prints achieved GB/s (read+write bytes).
#include <cstdio>
#include <cuda_runtime.h>
constexpr int NX = 3840, NY = 3840, PITCH = 3872, ROWS = NY + 8;
template <int NI, int NO, int KS, int VEC>
__global__ void k_stream(const double* __restrict__ in, double* __restrict__ out) {
  const int j = (blockIdx.x * blockDim.x + threadIdx.x) * VEC;
  if (j >= NX) return;
  const int k0 = blockIdx.y * KS;
  for (int k = k0; k < k0 + KS && k < NY; ++k) {
    const size_t i = (size_t)(k + 2) * PITCH + j + 16;
    if (VEC == 1) {
      double s = 0;
#pragma unroll
      for (int f = 0; f < NI; ++f) s += in[(size_t)f * PITCH * ROWS + i];
#pragma unroll
      for (int f = 0; f < NO; ++f) out[(size_t)f * PITCH * ROWS + i] = s + f;
    } else {
      double2 s = {0, 0};
#pragma unroll
      for (int f = 0; f < NI; ++f) {
        const double2 v = *reinterpret_cast<const double2*>(in + (size_t)f * PITCH * ROWS + i);
        s.x += v.x; s.y += v.y;
      }
#pragma unroll
      for (int f = 0; f < NO; ++f)
        *reinterpret_cast<double2*>(out + (size_t)f * PITCH * ROWS + i) = make_double2(s.x + f, s.y + f);
    }
  }
}
template <int NI, int NO, int KS, int VEC>
void run(const char* name, int tb, double* in, double* out) {
  dim3 grid((NX / VEC + tb - 1) / tb, (NY + KS - 1) / KS);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) k_stream<NI, NO, KS, VEC><<<grid, tb>>>(in, out);
  cudaEventRecord(a);
  const int reps = 10;
  for (int r = 0; r < reps; ++r) k_stream<NI, NO, KS, VEC><<<grid, tb>>>(in, out);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  const double bytes = (double)NX * NY * 8 * (NI + NO);
  printf("%-28s tb=%4d  %.3f ms  %.0f GB/s\n", name, tb, ms / reps, bytes / (ms / reps * 1e-3) / 1e9);
}
int main() {
  double *in, *out;
  const size_t fsz = (size_t)PITCH * ROWS;
  cudaMalloc(&in, fsz * 8 * 6); cudaMalloc(&out, fsz * 8 * 4);
  cudaMemset(in, 0, fsz * 8 * 6);
  run<4, 3, 32, 1>("in4 out3 ks32 vec1", 128, in, out);
  run<4, 3, 32, 1>("in4 out3 ks32 vec1", 256, in, out);
  run<4, 3, 32, 1>("in4 out3 ks32 vec1", 512, in, out);
  run<4, 3, 8, 1>("in4 out3 ks8 vec1", 128, in, out);
  run<4, 3, 128, 1>("in4 out3 ks128 vec1", 128, in, out);
  run<4, 3, 32, 2>("in4 out3 ks32 vec2", 128, in, out);
  run<4, 3, 32, 2>("in4 out3 ks32 vec2", 256, in, out);
  run<5, 2, 32, 1>("in5 out2 ks32 vec1", 128, in, out);
  run<5, 6, 32, 1>("in5 out6 ks32 vec1", 128, in, out);
  run<1, 1, 32, 1>("in1 out1 ks32 vec1 (copy)", 128, in, out);
  run<1, 1, 32, 2>("in1 out1 ks32 vec2 (copy)", 256, in, out);
  return 0;
}
