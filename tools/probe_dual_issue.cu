// Measurement aid: how FP64 (16-lane pipe, 2 cycles/warp) co-issues with
// ALU-pipe (LOP3), FMA-pipe integer (IMAD) and FP32 (FFMA) work on one SMSP.
// Each group = 8 independent lanes of work per op kind; all chains independent.
#include <cstdio>
#include <cuda_runtime.h>

// bit flags: 1 DFMA, 2 LOP3, 4 IMAD, 8 FFMA, 16 second LOP3, 32 second IMAD, 64 IADD
template <int MODE>
__global__ void mix(double* out, unsigned* iout, long long* cyc, int iters) {
  double d[8];
  unsigned u[8], w[8], z[8];
  float f[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { d[i] = threadIdx.x * 1e-9 + i; u[i] = threadIdx.x + i; w[i] = u[i] * 3; z[i] = u[i] ^ 5; f[i] = i * 0.5f; }
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE & 1) d[i] = fma(d[i], 1.0000001, 1e-9);
      if (MODE & 2) asm volatile("lop3.b32 %0, %0, 0x1234, 0x5a5a5a5a, 0x96;" : "+r"(u[i]));
      if (MODE & 4) asm volatile("mad.lo.u32 %0, %0, 0x9E3779B9, 7;" : "+r"(w[i]));
      if (MODE & 8) asm volatile("fma.rn.f32 %0, %0, 0f3F800001, 0f3F800000;" : "+f"(f[i]));
      if (MODE & 16) asm volatile("lop3.b32 %0, %0, 0x4321, 0x0a5a5a5a, 0x96;" : "+r"(z[i]));
      if (MODE & 32) asm volatile("mad.lo.u32 %0, %0, 0x1E3779B9, 5;" : "+r"(z[i]));
      if (MODE & 64) asm volatile("add.u32 %0, %0, 0x1234567;" : "+r"(z[i]));
    }
  }
  long long t1 = clock64();
  double s = 0; unsigned us = 0; float fs = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i]; us ^= u[i] ^ w[i] ^ z[i]; fs += f[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s + fs;
  iout[blockIdx.x * blockDim.x + threadIdx.x] = us;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int MODE>
void run(const char* name, int sms, double* d, unsigned* u, long long* c) {
  const int threads = 1024, iters = 2048;
  mix<MODE><<<sms, threads>>>(d, u, c, 8);
  cudaDeviceSynchronize();
  mix<MODE><<<sms, threads>>>(d, u, c, iters);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, c, 8, cudaMemcpyDeviceToHost);
  double warps_per_smsp = threads / 32.0 / 4.0;
  printf("%-34s cycles per group per warp per SMSP: %6.2f\n", name, double(h[0]) / iters / warps_per_smsp);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* d; unsigned* u; long long* c;
  cudaMalloc(&d, sms * 1024 * 8); cudaMalloc(&u, sms * 1024 * 4); cudaMalloc(&c, sms * 8);
  run<1>("8 DFMA", sms, d, u, c);
  run<2>("8 LOP3", sms, d, u, c);
  run<4>("8 IMAD", sms, d, u, c);
  run<8>("8 FFMA", sms, d, u, c);
  run<64>("8 IADD", sms, d, u, c);
  run<2 | 4>("8 LOP3 + 8 IMAD", sms, d, u, c);
  run<2 | 8>("8 LOP3 + 8 FFMA", sms, d, u, c);
  run<2 | 16>("16 LOP3", sms, d, u, c);
  run<1 | 2>("8 DFMA + 8 LOP3", sms, d, u, c);
  run<1 | 4>("8 DFMA + 8 IMAD", sms, d, u, c);
  run<1 | 8>("8 DFMA + 8 FFMA", sms, d, u, c);
  run<1 | 2 | 16>("8 DFMA + 16 LOP3", sms, d, u, c);
  run<1 | 4 | 32>("8 DFMA + 16 IMAD", sms, d, u, c);
  run<1 | 2 | 4>("8 DFMA + 8 LOP3 + 8 IMAD", sms, d, u, c);
  run<1 | 2 | 8>("8 DFMA + 8 LOP3 + 8 FFMA", sms, d, u, c);
  run<1 | 4 | 8>("8 DFMA + 8 IMAD + 8 FFMA", sms, d, u, c);
  run<1 | 64>("8 DFMA + 8 IADD", sms, d, u, c);
  run<1 | 2 | 64>("8 DFMA + 8 LOP3 + 8 IADD", sms, d, u, c);
  return 0;
}
