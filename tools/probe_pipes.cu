// Measurement aid: SMSP cost of integer / FP32 / XU instructions issued next
// to an FP64 (DFMA) stream, with NO data dependence between the two streams
// (tools/probe_mix.cu's IMAD.WIDE/F2I/MUFU/LDS cases shared registers with
// the DFMA chains and measured latency).  Each group per thread: 8 DFMA on 8
// independent chains (R,R,R operands, like the EP transform) + N ops of one
// kind on 8 independent integer/FP32 chains.  Reported: SMSP cycles per group
// per warp; 16.0 = the FP64 pipe alone.
#include <cstdio>
#include <cuda_runtime.h>

template <int OP, int N>
__global__ void __launch_bounds__(512, 1) k(double* out, unsigned* iout, long long* cyc, int iters) {
  double d[8], e[8], f[8];
  unsigned u[8], w[8], z[8];
  unsigned long long q[8];
  float g[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    d[i] = threadIdx.x * 1e-9 + i; e[i] = 1.0 + i * 1e-12 + threadIdx.x * 1e-15; f[i] = 1e-9 * (i + 1 + threadIdx.x);
    u[i] = 0x3F000000u + threadIdx.x * 7 + i; w[i] = u[i] * 13 + 1; z[i] = u[i] ^ 0x5555; q[i] = u[i]; g[i] = 1.0f + i;
  }
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(d[i]) : "d"(e[i]), "d"(f[i]));
#pragma unroll
      for (int r = 0; r < N; ++r) {
        if (OP == 1) asm volatile("lop3.b32 %0, %0, 0xfffff, %1, 0xea;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 2) asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(u[i]) : "r"(w[i]), "r"(z[i]));
        if (OP == 3) asm volatile("mad.wide.u32 %0, %1, %2, %0;" : "+l"(q[i]) : "r"(unsigned(q[i])), "r"(w[i]));
        if (OP == 4) asm volatile("mad.hi.u32 %0, %0, %1, %0;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 5) { unsigned r2; asm volatile("{.reg .pred p; setp.lt.u32 p, %1, %2; selp.u32 %0, 1, 0, p;}" : "=r"(r2) : "r"(u[i]), "r"(w[i])); u[i] ^= r2; }
        if (OP == 6) asm volatile("max.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 7) asm volatile("shr.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 8) asm volatile("prmt.b32.b4e %0, %1, 0, %0;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 9) asm volatile("add.rm.f32 %0, %0, 0f497FFFE4;" : "+f"(g[i]));
        if (OP == 10) asm volatile("max.NaN.f32 %0, %0, %1, 0f3FE00000;" : "+f"(g[i]) : "f"(__int_as_float(w[i])));
        if (OP == 11) asm volatile("add.u32 %0, %0, 0x1234567;" : "+r"(u[i]));
        if (OP == 12) asm volatile("add.u32 %0, %0, %1;" : "+r"(u[i]) : "r"(w[i]));
        if (OP == 13) { unsigned r2; asm volatile("cvt.rzi.u32.f64 %0, %1;" : "=r"(r2) : "d"(__hiloint2double(0x40000000, int(u[i])))); u[i] += r2; }
        if (OP == 14) { double y; asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(__hiloint2double(int(u[i]), 0))); u[i] = unsigned(__double2hiint(y)); }
        if (OP == 15) asm volatile("fma.rn.f32 %0, %0, %1, 0f3F800000;" : "+f"(g[i]) : "f"(g[(i + 1) & 7]));
        if (OP == 16) asm volatile("min.u32 %0, %0, 0x2001;" : "+r"(u[i]));
        if (OP == 17) asm volatile("{.reg .f64 t; cvt.rn.f64.s64 t, %0; mov.b64 %0, t;}" : "+l"(q[i]));
        if (OP == 18) asm volatile("add.rn.f64 %0, %0, %1;" : "+d"(e[i]) : "d"(f[(i + 1) & 7]));
        if (OP == 19) asm volatile("{.reg .f64 t; cvt.rn.f64.u32 t, %0; mov.b64 %1, t;}" : "+r"(u[i]), "+l"(q[i]));
        if (OP == 20) { asm volatile("lop3.b32 %0, %0, 0xfffff, %1, 0xea;" : "+r"(u[i]) : "r"(w[i]));
                        asm volatile("add.rn.f64 %0, %0, %1;" : "+d"(e[i]) : "d"(f[(i + 1) & 7])); }
      }
    }
  }
  long long t1 = clock64();
  double s = 0; unsigned us = 0; float gs = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) { s += d[i] + e[i] + f[i]; us ^= u[i] ^ w[i] ^ unsigned(q[i]) ^ unsigned(q[i] >> 32); gs += g[i]; }
  out[blockIdx.x * blockDim.x + threadIdx.x] = s + gs;
  iout[blockIdx.x * blockDim.x + threadIdx.x] = us;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int OP, int N>
void run(const char* name, int sms, double* d, unsigned* u, long long* c) {
  const int iters = 1024, threads = 512;
  k<OP, N><<<sms, threads>>>(d, u, c, 8);
  cudaDeviceSynchronize();
  k<OP, N><<<sms, threads>>>(d, u, c, iters);
  if (cudaDeviceSynchronize() != cudaSuccess) { printf("%s: failed\n", name); return; }
  long long h[1];
  cudaMemcpy(h, c, 8, cudaMemcpyDeviceToHost);
  const double v = double(h[0]) / iters / (threads / 128.0);
  printf("8 DFMA(R,R,R) + %d x 8 %-16s %6.2f cycles/group  (+%.2f per op)\n", N, name, v, (v - 16.0) / (8.0 * N));
}

#define RUN(OP, NAME) run<OP, 1>(NAME, sms, d, u, c); run<OP, 2>(NAME, sms, d, u, c);

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* d; unsigned* u; long long* c;
  cudaMalloc(&d, sms * 1024 * 8); cudaMalloc(&u, sms * 1024 * 4); cudaMalloc(&c, sms * 8);
  run<0, 1>("(nothing)", sms, d, u, c);
  RUN(1, "LOP3 R,imm,R");
  RUN(2, "IMAD R,R,R");
  RUN(3, "IMAD.WIDE");
  RUN(4, "IMAD.HI R,R,R");
  RUN(5, "ISETP+SEL");
  RUN(6, "VIMNMX R,R");
  RUN(16, "VIMNMX R,imm");
  RUN(7, "SHF R,R");
  RUN(8, "PRMT");
  RUN(9, "FADD.RM");
  RUN(10, "FMNMX3.NAN");
  RUN(13, "F2I.U32.F64");
  RUN(14, "MUFU.RSQ64H");
  RUN(15, "FFMA");
  RUN(17, "I2F.F64.S64");
  RUN(18, "DADD R,R");
  RUN(19, "I2F.F64.U32");
  RUN(20, "LOP3+DADD");
  return 0;
}
