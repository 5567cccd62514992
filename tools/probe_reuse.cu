// Measurement aid: does the operand reuse cache survive warp interleaving?
// Each thread runs CH dependent chains v = fma(v, m, c) with m, c loop-invariant
// registers (3-register DFMA).  With CH = 1 every DFMA depends on the previous
// one, so consecutive instructions of a warp are separated by other warps'
// issues; with CH = 4 the chains interleave inside the warp.  If reuse works
// in both cases, both reach ~2 cycles per warp-DFMA per SMSP (64 lanes/clk/SM);
// if only the 6-register-read form is possible, ~3 cycles.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_reuse probe_reuse.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int CH, int MODE>
__global__ void k(double* out, long long* cyc, int iters, double m0, double c0) {
  double v[CH];
  double m = m0 + threadIdx.x * 1e-18, c = c0 + threadIdx.x * 1e-19;
  double m2 = m * 0.5, c2 = c * 0.25;
#pragma unroll
  for (int i = 0; i < CH; ++i) v[i] = threadIdx.x * 1e-9 + i;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 16; ++j)
#pragma unroll
      for (int i = 0; i < CH; ++i) {
        if (MODE == 0) v[i] = fma(v[i], m, c);                       // shared m, c (reusable)
        else v[i] = fma(v[i], (j & 1) ? m2 : m, (j & 1) ? c2 : c);   // alternating: no reuse
      }
  }
  __syncthreads();
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += v[i];
  if (s == 12345.0) out[0] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

template <int CH, int MODE>
void run(const char* name, int threads) {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out;
  long long* cyc;
  cudaMalloc(&out, 8);
  cudaMalloc(&cyc, sizeof(long long) * sms);
  const int iters = 4096 / CH;
  k<CH, MODE><<<sms, threads>>>(out, cyc, 16, 1.0000001, 1e-9);
  k<CH, MODE><<<sms, threads>>>(out, cyc, iters, 1.0000001, 1e-9);
  cudaDeviceSynchronize();
  long long c;
  cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
  const double dfma_per_smsp = double(iters) * 16 * CH * (threads / 32) / 4.0;
  printf("%-34s threads=%4d  %.2f cycles per warp-DFMA per SMSP\n", name, threads, c / dfma_per_smsp);
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int thr : {256, 512, 1024}) {
    run<1, 0>("1 chain, shared m,c", thr);
    run<1, 1>("1 chain, alternating m,c", thr);
    run<4, 0>("4 chains, shared m,c", thr);
    run<4, 1>("4 chains, alternating m,c", thr);
  }
  return 0;
}
