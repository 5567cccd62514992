// Measurement aid: FP64 pipe throughput and MUFU-based
// approximation accuracy on the box's B200. Not part of the product path.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_fp64 probe_fp64.cu
//   ./probe_fp64
//
// Prints DFMA lane-ops per SM clock (clock64-normalised, so throttling does not
// distort it) and the max relative error of rsqrt.approx.f64 / rcp.approx.f64.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); return 1; } } while (0)

template <int CHAINS>
__global__ void dfma_loop(double* out, long long* cyc, int iters, double m, double c) {
  double v[CHAINS];
#pragma unroll
  for (int i = 0; i < CHAINS; ++i) v[i] = threadIdx.x * 1e-9 + i;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int k = 0; k < 16; ++k)
#pragma unroll
      for (int i = 0; i < CHAINS; ++i) v[i] = fma(v[i], m, c);
  }
  __syncthreads();
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < CHAINS; ++i) s += v[i];
  if (s == 12345.0) out[0] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

__global__ void rsqrt_err(const double* x, double* rel_rs, double* rel_rc, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double v = x[i], y, z;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(v));
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(z) : "d"(v));
  double ref = 1.0 / sqrt(v);  // ~1 ulp
  rel_rs[i] = fabs(y - ref) / ref;
  rel_rc[i] = fabs(z - 1.0 / v) * v;
}


// Dependent-chain latencies (one warp): cycles per dependent instruction.
__global__ void lat_kernel(double* out, long long* cyc, double x, int n) {
  __shared__ double2 sm[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) sm[i] = make_double2(1.0 + i * 1e-3, 0.5);
  __syncthreads();
  double a = x + threadIdx.x * 1e-9, b = a;
  unsigned u = threadIdx.x;
  long long t0, t1;
  // DFMA chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { a = fma(a, 0.999999, 1e-7); a = fma(a, 0.999999, 1e-7); a = fma(a, 0.999999, 1e-7); a = fma(a, 0.999999, 1e-7); }
  t1 = clock64(); if (threadIdx.x == 0) cyc[0] = (t1 - t0);
  // DADD chain
  t0 = clock64();
  for (int i = 0; i < n; ++i) { b = b + 1e-7; b = b + 1e-7; b = b + 1e-7; b = b + 1e-7; }
  t1 = clock64(); if (threadIdx.x == 0) cyc[1] = (t1 - t0);
  // MUFU.RSQ64H chain (+1 DADD to keep it positive and dependent)
  double c = a;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { double y; asm volatile("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(c)); c = y; }
  t1 = clock64(); if (threadIdx.x == 0) cyc[2] = (t1 - t0);
  // F2I + I2F chain-ish: F2I then IADD then use as LDS index
  double d = a;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { unsigned k = __double2uint_rz(d); double2 e = sm[k & 255]; d = e.x; }
  t1 = clock64(); if (threadIdx.x == 0) cyc[3] = (t1 - t0);
  // LDS.128 chain via integer index
  t0 = clock64();
  for (int i = 0; i < n; ++i) { double2 e = sm[u & 255]; u = __double_as_longlong(e.y) >> 40; u += (unsigned)__double_as_longlong(e.x); }
  t1 = clock64(); if (threadIdx.x == 0) cyc[4] = (t1 - t0);
  // IMAD.WIDE chain
  unsigned long long w = u | 1;
  t0 = clock64();
  for (int i = 0; i < n; ++i) { w = w * 1220703125ull; w = w * 1220703125ull; w = w * 1220703125ull; w = w * 1220703125ull; }
  t1 = clock64(); if (threadIdx.x == 0) cyc[5] = (t1 - t0);
  out[threadIdx.x] = a + b + c + d + (double)u + (double)w;
}

int main() {
  cudaDeviceProp p;
  CK(cudaGetDeviceProperties(&p, 0));
  printf("device %s sm_%d%d SMs=%d clockRate(kHz)=%d\n", p.name, p.major, p.minor,
         p.multiProcessorCount, p.clockRate);
  double* dout; long long* dcyc;
  int blocks = p.multiProcessorCount;
  CK(cudaMalloc(&dout, 8));
  CK(cudaMalloc(&dcyc, sizeof(long long) * blocks * 8));
  const int iters = 4096;
  for (int threads : {256, 512, 1024}) {
    for (int bps : {1, 2}) {
      if (threads * bps > 2048) continue;
      int nb = blocks * bps;
      dfma_loop<8><<<nb, threads>>>(dout, dcyc, 16, 1.0000001, 1e-7);
      CK(cudaDeviceSynchronize());
      cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
      cudaEventRecord(e0);
      dfma_loop<8><<<nb, threads>>>(dout, dcyc, iters, 1.0000001, 1e-7);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      std::vector<long long> cyc(nb);
      CK(cudaMemcpy(cyc.data(), dcyc, 8 * nb, cudaMemcpyDeviceToHost));
      long long cmax = 0; for (auto c : cyc) cmax = c > cmax ? c : cmax;
      double ops_per_block = double(threads) * iters * 16 * 8;
      double lanes_per_clk_sm = ops_per_block * bps / double(cmax);
      double tflops = 2.0 * ops_per_block * nb / (ms * 1e-3) / 1e12;
      printf("DFMA threads=%d blocks/SM=%d : %.2f lane-FMA/clk/SM (clock64), %.2f TFLOP/s, ms=%.3f, implied MHz=%.0f\n",
             threads, bps, lanes_per_clk_sm, tflops, ms, cmax / (ms * 1e3));
    }
  }
  {
    long long* dc; double* dd;
    CK(cudaMalloc(&dc, 64)); CK(cudaMalloc(&dd, 8 * 1024));
    const int n = 4096;
    lat_kernel<<<1, 32>>>(dd, dc, 1.5, n);
    CK(cudaDeviceSynchronize());
    long long hc[8];
    CK(cudaMemcpy(hc, dc, 48, cudaMemcpyDeviceToHost));
    printf("latency (cycles/dep op): DFMA %.2f  DADD %.2f  MUFU.RSQ64H %.2f  F2I+LDS %.2f  LDS.128+int %.2f  64b-mul %.2f\n",
           hc[0] / (4.0 * n), hc[1] / (4.0 * n), hc[2] / double(n), hc[3] / double(n), hc[4] / double(n), hc[5] / (4.0 * n));
  }
  // approximation accuracy
  const int n = 1 << 22;
  std::vector<double> hx(n);
  uint64_t s = 88172645463325252ull;
  for (int i = 0; i < n; ++i) {
    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
    double u = (s >> 11) * (1.0 / 9007199254740992.0);
    hx[i] = std::ldexp(1.0 + u, int(s % 200) - 100);
  }
  double *dx, *dr, *dc;
  CK(cudaMalloc(&dx, 8 * n)); CK(cudaMalloc(&dr, 8 * n)); CK(cudaMalloc(&dc, 8 * n));
  CK(cudaMemcpy(dx, hx.data(), 8 * n, cudaMemcpyHostToDevice));
  rsqrt_err<<<(n + 255) / 256, 256>>>(dx, dr, dc, n);
  CK(cudaDeviceSynchronize());
  std::vector<double> hr(n), hc(n);
  CK(cudaMemcpy(hr.data(), dr, 8 * n, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hc.data(), dc, 8 * n, cudaMemcpyDeviceToHost));
  double mr = 0, mc = 0;
  for (int i = 0; i < n; ++i) { mr = fmax(mr, hr[i]); mc = fmax(mc, hc[i]); }
  printf("rsqrt.approx.ftz.f64 max rel err = %.3e (2^%.2f)\n", mr, std::log2(mr));
  printf("rcp.approx.ftz.f64   max rel err = %.3e (2^%.2f)\n", mc, std::log2(mc));
  return 0;
}
