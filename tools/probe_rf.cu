// Measurement aid: does register-operand count of FP64 instructions limit
// co-issue with integer work (register-file read bandwidth)?
#include <cstdio>
#include <cuda_runtime.h>

// MODE bits: 1 = DFMA 3 distinct reg operands, 2 = DFMA 2 regs + imm, 4 = DMUL 2 regs,
//            8 = add 8 LOP3 (1 reg + imm), 16 = add 8 LOP3 with 3 reg operands,
//            32 = add 8 IMAD (reg, reg, reg)
template <int MODE>
__global__ void k(double* out, unsigned* iout, long long* cyc, int iters) {
  double d[8], e[8], f[8];
  unsigned u[8], w[8], z[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    d[i] = threadIdx.x * 1e-9 + i; e[i] = 1.0 + i * 1e-12 + threadIdx.x * 1e-15; f[i] = 1e-9 * (i + 1);
    u[i] = threadIdx.x * 7 + i; w[i] = u[i] * 13; z[i] = u[i] ^ 0x55;
  }
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE & 1) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d[i]) : "d"(e[i]), "d"(f[i]));
      if (MODE & 2) asm volatile("fma.rn.f64 %0, %0, %1, 0d3FF0000000000000;" : "+d"(d[i]) : "d"(e[i]));
      if (MODE & 4) asm volatile("mul.rn.f64 %0, %0, %1;" : "+d"(d[i]) : "d"(e[i]));
      if (MODE & 8) asm volatile("lop3.b32 %0, %0, 0x1234, 0x5a5a5a5a, 0x96;" : "+r"(u[i]));
      if (MODE & 16) asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(u[i]) : "r"(w[i]), "r"(z[i]));
      if (MODE & 32) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(w[i]) : "r"(z[i]), "r"(u[(i + 3) & 7]));
    }
  }
  long long t1 = clock64();
  double s = 0; unsigned us = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i] + e[i] + f[i]; us ^= u[i] ^ w[i] ^ z[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  iout[blockIdx.x * blockDim.x + threadIdx.x] = us;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int MODE>
void run(const char* name, int sms, double* d, unsigned* u, long long* c) {
  const int threads = 1024, iters = 2048;
  k<MODE><<<sms, threads>>>(d, u, c, 8);
  cudaDeviceSynchronize();
  k<MODE><<<sms, threads>>>(d, u, c, iters);
  cudaDeviceSynchronize();
  long long h[1];
  cudaMemcpy(h, c, 8, cudaMemcpyDeviceToHost);
  printf("%-36s cycles/group/warp/SMSP: %6.2f\n", name, double(h[0]) / iters / (threads / 128.0));
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* d; unsigned* u; long long* c;
  cudaMalloc(&d, sms * 1024 * 8); cudaMalloc(&u, sms * 1024 * 4); cudaMalloc(&c, sms * 8);
  run<1>("8 DFMA(3 reg)", sms, d, u, c);
  run<2>("8 DFMA(2 reg+imm)", sms, d, u, c);
  run<4>("8 DMUL(2 reg)", sms, d, u, c);
  run<8>("8 LOP3(1 reg)", sms, d, u, c);
  run<16>("8 LOP3(3 reg)", sms, d, u, c);
  run<32>("8 IMAD(3 reg)", sms, d, u, c);
  run<1 | 8>("8 DFMA(3 reg) + 8 LOP3(1 reg)", sms, d, u, c);
  run<1 | 16>("8 DFMA(3 reg) + 8 LOP3(3 reg)", sms, d, u, c);
  run<2 | 8>("8 DFMA(2 reg) + 8 LOP3(1 reg)", sms, d, u, c);
  run<2 | 16>("8 DFMA(2 reg) + 8 LOP3(3 reg)", sms, d, u, c);
  run<4 | 16>("8 DMUL + 8 LOP3(3 reg)", sms, d, u, c);
  run<1 | 32>("8 DFMA(3 reg) + 8 IMAD(3 reg)", sms, d, u, c);
  run<1 | 8 | 32>("8 DFMA(3) + 8 LOP3(1) + 8 IMAD(3)", sms, d, u, c);
  run<2 | 8 | 32>("8 DFMA(2) + 8 LOP3(1) + 8 IMAD(3)", sms, d, u, c);
  run<1 | 16 | 32>("8 DFMA(3) + 8 LOP3(3) + 8 IMAD(3)", sms, d, u, c);
  return 0;
}
