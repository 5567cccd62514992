// Measurement aid: is the SMSP limited by register-file operand reads
// (~2 x 32-bit per lane per clock)?  Same instruction counts, different
// numbers of register source operands.
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(1024, 1) k(double* out, unsigned* iout, long long* cyc, int iters) {
  double d[8], e[8];
  unsigned u[8], w[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    d[i] = threadIdx.x * 1e-9 + i; e[i] = 1.0 + i * 1e-12 + threadIdx.x * 1e-15;
    u[i] = threadIdx.x * 7 + i; w[i] = u[i] * 13 + 1;
  }
  double c1 = e[0] * 0.5, c2 = e[1] * 0.25;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE == 1) { asm volatile("add.f64 %0, %0, 0d3E112E0BE826D695;" : "+d"(d[i]));
                       asm volatile("lop3.b32 %0, %0, 0x1234, 0x5a5a5a5a, 0x96;" : "+r"(u[i])); }
      if (MODE == 2) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d[i]) : "d"(e[i]), "d"(e[(i + 3) & 7]));
      if (MODE == 3) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d[i]) : "d"(c1), "d"(c2));
      if (MODE == 4) { asm volatile("mul.rn.f64 %0, %0, %1;" : "+d"(d[i]) : "d"(e[i]));
                       asm volatile("add.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i])); }
      if (MODE == 5) { asm volatile("mul.rn.f64 %0, %0, %1;" : "+d"(d[i]) : "d"(e[i]));
                       asm volatile("add.u32 %0, %0, 0x1234567;" : "+r"(u[i])); }
      if (MODE == 6) asm volatile("add.f64 %0, %0, 0d3E112E0BE826D695;" : "+d"(d[i]));
      if (MODE == 7) asm volatile("mul.rn.f64 %0, %0, %1;" : "+d"(d[i]) : "d"(e[i]));
      if (MODE == 8) { asm volatile("mul.rn.f64 %0, %0, %1;" : "+d"(d[i]) : "d"(e[i]));
                       asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(u[i]) : "r"(w[i]), "r"(w[(i + 1) & 7])); }
    }
  }
  long long t1 = clock64();
  double s = c1 + c2; unsigned us = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i] + e[i]; us ^= u[i] ^ w[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  iout[blockIdx.x * blockDim.x + threadIdx.x] = us;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int MODE>
void run(const char* name, int sms, double* d, unsigned* u, long long* c, int threads) {
  const int iters = 1024;
  k<MODE><<<sms, threads>>>(d, u, c, 8);
  cudaDeviceSynchronize();
  k<MODE><<<sms, threads>>>(d, u, c, iters);
  if (cudaDeviceSynchronize() != cudaSuccess) { printf("%s failed\n", name); return; }
  long long h[1];
  cudaMemcpy(h, c, 8, cudaMemcpyDeviceToHost);
  printf("threads=%4d %-40s %6.2f cycles per group of 8\n", threads, name, double(h[0]) / iters / (threads / 128.0));
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* d; unsigned* u; long long* c;
  cudaMalloc(&d, sms * 1024 * 8); cudaMalloc(&u, sms * 1024 * 4); cudaMalloc(&c, sms * 8);
  for (int t : {512, 1024}) {
    run<6>("DADD(R,imm)            [2 reads]", sms, d, u, c, t);
    run<7>("DMUL(R,R)              [4 reads]", sms, d, u, c, t);
    run<1>("DADD(R,imm)+LOP3(R)    [2+1 reads]", sms, d, u, c, t);
    run<2>("DFMA(R,R,R) distinct   [6 reads]", sms, d, u, c, t);
    run<3>("DFMA(R,c1,c2) shared   [2-6 reads]", sms, d, u, c, t);
    run<4>("DMUL(R,R)+IADD(R,R)    [4+2 reads]", sms, d, u, c, t);
    run<5>("DMUL(R,R)+IADD(R,imm)  [4+1 reads]", sms, d, u, c, t);
    run<8>("DMUL(R,R)+LOP3(R,R,R)  [4+3 reads]", sms, d, u, c, t);
  }
  return 0;
}
