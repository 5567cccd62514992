// Measurement aid: marginal SMSP cycles of one non-FP64 instruction issued
// alongside DFMA-heavy code (8 independent DFMA chains with 3 register
// operands + 8 independent ops of one kind per group).  Guides the EP
// kernel's instruction mix.
#include <cstdio>
#include <cuda_runtime.h>

template <int OP>
__global__ void __launch_bounds__(1024, 1) k(double* out, unsigned* iout, long long* cyc, int iters, const double2* gtab) {
  __shared__ double2 tab[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) tab[i] = gtab[i];
  __syncthreads();
  double d[8], e[8], f[8];
  unsigned u[8], w[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    d[i] = threadIdx.x * 1e-9 + i; e[i] = 1.0 + i * 1e-12 + threadIdx.x * 1e-15; f[i] = 1e-9 * (i + 1 + threadIdx.x);
    u[i] = threadIdx.x * 7 + i; w[i] = u[i] * 13 + 1;
  }
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (OP != 99) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d[i]) : "d"(e[i]), "d"(f[i]));
      if (OP == 1) asm volatile("lop3.b32 %0, %0, 0x1234, 0x5a5a5a5a, 0x96;" : "+r"(u[i]));
      if (OP == 2) asm volatile("add.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i]));
      if (OP == 3) { unsigned r; asm volatile("{.reg .pred p; setp.lt.u32 p, %1, %2; selp.u32 %0, 1, 0, p;}" : "=r"(r) : "r"(u[i]), "r"(w[i])); u[i] += r; }
      if (OP == 4) asm volatile("prmt.b32.b4e %0, %0, %1, %2;" : "+r"(u[i]) : "r"(w[i]), "r"(u[(i + 1) & 7]));
      if (OP == 5) { unsigned r; asm volatile("cvt.rzi.u32.f64 %0, %1;" : "=r"(r) : "d"(d[i])); u[i] ^= r; }
      if (OP == 6) { double y; asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(e[i])); e[i] = y; }
      if (OP == 7) { double2 t; asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(t.x), "=d"(t.y) : "r"((unsigned)__cvta_generic_to_shared(&tab[u[i] & 255]))); f[i] = t.x; u[i] += __double2hiint(t.y); }
      if (OP == 8) asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(*(unsigned long long*)&d[i]) : "r"(u[i]), "r"(w[i]));
      if (OP == 9) asm volatile("mad.lo.u32 %0, %0, %1, 7;" : "+r"(u[i]) : "r"(w[i]));
      if (OP == 10) asm volatile("max.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i]));
      if (OP == 11) asm volatile("shr.u32 %0, %0, 3;" : "+r"(u[i]));
      if (OP == 12) asm volatile("mov.b32 %0, %1;" : "=r"(u[i]) : "r"(w[(i + 3) & 7]));
      if (OP == 13) { asm volatile("lop3.b32 %0, %0, 0x1234, 0x5a5a5a5a, 0x96;" : "+r"(u[i]));
                      asm volatile("lop3.b32 %0, %0, 0x4321, 0x0a5a5a5a, 0x96;" : "+r"(w[i])); }
      if (OP == 14) asm volatile("add.f64 %0, %0, %1;" : "+d"(f[i]) : "d"(e[i]));
    }
  }
  long long t1 = clock64();
  double s = 0; unsigned us = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i] + e[i] + f[i]; us ^= u[i] ^ w[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  iout[blockIdx.x * blockDim.x + threadIdx.x] = us;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char* name, int sms, double* d, unsigned* u, long long* c, const double2* tab, int threads) {
  const int iters = 1024;
  k<OP><<<sms, threads>>>(d, u, c, 8, tab);
  cudaDeviceSynchronize();
  k<OP><<<sms, threads>>>(d, u, c, iters, tab);
  if (cudaDeviceSynchronize() != cudaSuccess || cudaGetLastError() != cudaSuccess) { printf("%s: launch failed\n", name); return; }
  long long h[1];
  cudaMemcpy(h, c, 8, cudaMemcpyDeviceToHost);
  double v = double(h[0]) / iters / (threads / 128.0);
  printf("threads=%4d  8 DFMA + 8 %-22s %6.2f cycles  (marginal %.2f / op)\n", threads, name, v, (v - 16.0) / 8.0);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* d; unsigned* u; long long* c; double2* tab;
  cudaMalloc(&d, sms * 1024 * 8); cudaMalloc(&u, sms * 1024 * 4); cudaMalloc(&c, sms * 8);
  cudaMalloc(&tab, 256 * 16); cudaMemset(tab, 0, 256 * 16);
  for (int threads : {256, 512, 1024}) {
    run<0>("(nothing)", sms, d, u, c, tab, threads);
    run<1>("LOP3 (1 reg)", sms, d, u, c, tab, threads);
    run<2>("IADD (2 reg)", sms, d, u, c, tab, threads);
    run<3>("ISETP+SEL+IADD", sms, d, u, c, tab, threads);
    run<4>("PRMT (3 reg)", sms, d, u, c, tab, threads);
    run<5>("F2I.F64", sms, d, u, c, tab, threads);
    run<6>("MUFU.RSQ64H", sms, d, u, c, tab, threads);
    run<7>("LDS.128 + LEA + IADD", sms, d, u, c, tab, threads);
    run<8>("IMAD.WIDE", sms, d, u, c, tab, threads);
    run<9>("IMAD (2 reg)", sms, d, u, c, tab, threads);
    run<10>("VIMNMX", sms, d, u, c, tab, threads);
    run<11>("SHF (1 reg)", sms, d, u, c, tab, threads);
    run<12>("MOV", sms, d, u, c, tab, threads);
    run<13>("2x LOP3", sms, d, u, c, tab, threads);
    run<14>("DADD (2 reg) [fp64]", sms, d, u, c, tab, threads);
  }
  return 0;
}
