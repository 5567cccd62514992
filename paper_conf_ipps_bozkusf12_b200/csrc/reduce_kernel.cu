// reduce_kernel.cu — F2: the paper's reduction benchmark, "the addition of
// 16M single-precision floating point values" (SHOC,
// PAPER.md:793-795), as an HBM-bound sm_100a kernel.
//
// One launch: a grid of at most one resident wave streams the input with
// 16-byte loads (8 independent float4 per thread per round in flight, the
// thread count chosen so the rounds cover the input), accumulates in
// FP64 (reading R11: the sum is defined exactly; FP64 accumulation keeps the
// error ~1e-14 of sum|x| at any size), then warp shuffle -> per-warp shared
// memory -> per-block partial -> last-block fixed-order finalize (the EP
// kernel's reduction pattern, deterministic).
#include <cuda_runtime.h>

#include <cstdint>

#include "reduce_launch.h"

namespace hplep {

#ifndef RED_THREADS_CFG
#define RED_THREADS_CFG 512
#endif
#ifndef RED_UNROLL
#define RED_UNROLL 8   // independent 16-B loads in flight per thread (4: -25 % at 16M floats)
#endif
#ifndef RED_BPS
#define RED_BPS 2      // blocks per SM (one wave)
#endif
constexpr int RED_THREADS = RED_THREADS_CFG;

__global__ void __launch_bounds__(RED_THREADS)
reduce_sum_f32_kernel(const float* __restrict__ in, int64_t n, double* __restrict__ partials,
                      unsigned* __restrict__ counter, double* __restrict__ out) {
  __shared__ double s_w[RED_THREADS / 32];
  __shared__ int s_last;
  const int64_t tid = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const int64_t T = int64_t(gridDim.x) * blockDim.x;
  // scalar head up to 16-byte alignment, vector body, scalar tail
  const int64_t mis = (reinterpret_cast<uintptr_t>(in) >> 2) & 3;
  const int64_t head = mis ? (4 - mis < n ? 4 - mis : n) : 0;
  double acc = 0.0;
  if (tid < head) acc += double(__ldcs(in + tid));
  const float4* v = reinterpret_cast<const float4*>(in + head);
  const int64_t nv = (n - head) / 4;
  // full rounds of RED_UNROLL independent 16-B loads per thread (the grid is
  // sized so that the rounds cover the input), then a short remainder
  int64_t i = tid;
#ifdef RED_FLOOR  // timing study only (result wrong): skip the stream, keep launch + tree + fold
  i = nv;
#endif
  for (; i + (RED_UNROLL - 1) * T < nv; i += RED_UNROLL * T) {
    float4 r[RED_UNROLL];
#pragma unroll
    for (int k = 0; k < RED_UNROLL; ++k) r[k] = __ldcs(v + i + k * T);
#pragma unroll
    for (int k = 0; k < RED_UNROLL; ++k) acc += (double(r[k].x) + double(r[k].y)) + (double(r[k].z) + double(r[k].w));
  }
  for (; i < nv; i += T) {
    const float4 a = __ldcs(v + i);
    acc += (double(a.x) + double(a.y)) + (double(a.z) + double(a.w));
  }
  const int64_t tail0 = head + 4 * nv;
  if (tid < n - tail0) acc += double(__ldcs(in + tail0 + tid));

#pragma unroll
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xFFFFFFFFu, acc, off);
  if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double b = 0.0;
    for (unsigned w = 0; w < blockDim.x / 32; ++w) b += s_w[w];
    partials[blockIdx.x] = b;
    __threadfence();
    // acquiring ticket: the last block's loads below (after the barrier) are
    // ordered after every block's fence + ticket (no second fence)
    unsigned ticket;
    asm volatile("atom.add.acquire.gpu.global.u32 %0, [%1], 1;" : "=r"(ticket) : "l"(counter) : "memory");
    s_last = ticket == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  // last block: all threads fold the partials (strided, fixed order), then
  // the same warp/block tree — deterministic, and no serial 600-load chain
  double s = 0.0;
  for (unsigned b = threadIdx.x; b < gridDim.x; b += blockDim.x) s += __ldcg(partials + b);
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xFFFFFFFFu, s, off);
  __syncthreads();
  if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (unsigned w = 0; w < blockDim.x / 32; ++w) t += s_w[w];
    *out = t;
    *counter = 0;
  }
}

int launch_reduce_sum_f32(const float* in, int64_t n, double* out, ReduceWorkspace& ws, int sms,
                          cudaStream_t stream) {
  // at most one resident wave (sms * RED_BPS blocks); within it, as few
  // threads as make every thread's work whole rounds of RED_UNROLL loads
  const int64_t tmax = int64_t(sms) * RED_BPS * RED_THREADS, nv = n / 4;
  const int64_t rounds = (nv + RED_UNROLL * tmax - 1) / (RED_UNROLL * tmax);
  const int64_t t = rounds > 0 ? (nv + RED_UNROLL * rounds - 1) / (RED_UNROLL * rounds) : 1;
  int blocks = int((t + RED_THREADS - 1) / RED_THREADS);
  if (blocks < 1) blocks = 1;
  if (blocks > sms * RED_BPS) blocks = sms * RED_BPS;
  if (blocks > ws.capacity) return set_error(HPL_EINVAL, "reduce workspace too small");
  reduce_sum_f32_kernel<<<blocks, RED_THREADS, 0, stream>>>(in, n, ws.partials, ws.counter, out);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, "reduce_sum_f32_kernel launch");
  return 0;
}

}  // namespace hplep
