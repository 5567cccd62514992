// transpose_kernel.cu — F4: the paper's matrix-transpose benchmark, "the
// transposition of a 16K x 16K matrix" (AMD APP SDK,
// PAPER.md:791-793), as an HBM-bound sm_100a kernel.
//
// dst (w x h, row-major) = transpose of src (h x w, row-major):
//   dst[j][i] = src[i][j]   — Fig. 10(b)'s dest[idy][idx] = src[idx][idy]
//    with the blocked structure the benchmark itself uses:
//   "contiguous reads and transposing blocks of the matrix in the local memory
//   shared by each group of threads".
//
// One CTA moves one 64 x 64 tile per iteration: four 16-byte streaming loads
// per thread (16 KB in flight per CTA, up to 8 CTAs per SM),
// scalar stores into a 64 x 65 shared tile (the pad makes both the row-wise
// stores and the column-wise reads bank-conflict free), then each warp writes
// 128 contiguous bytes of a dst row per store instruction.  Pure data
// movement: results are bit-exact by construction.  Edge tiles (h or w not a
// multiple of 64, or rows not 16-byte aligned) take guarded scalar paths.
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/hpl.h"

namespace hplep {

int set_error(int code, const char* fmt, ...);
int set_cuda_error(cudaError_t e, const char* what);

constexpr int TT = 64;          // tile edge (elements)
constexpr int TR_THREADS = 256; // 8 warps

__global__ void __launch_bounds__(TR_THREADS, 8)  // <= 32 registers: 8 CTAs (2048 threads) per SM
k_transpose_f32(const float* __restrict__ src, float* __restrict__ dst, int64_t h, int64_t w,
                int64_t tiles_w, int64_t ntiles, int vec_ok) {
  __shared__ float tile[TT][TT + 1];
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  for (int64_t id = blockIdx.x; id < ntiles; id += gridDim.x) {
    const int64_t r0 = (id / tiles_w) * TT, c0 = (id % tiles_w) * TT;
    const bool full = vec_ok && r0 + TT <= h && c0 + TT <= w;
    // ---- load: per pass k, lane (g, q) = (t & 7, (t >> 3) & 3) of warp w reads
    //      float4 group g + 8 (k & 1) of row 4 w + q + 32 (k >> 1): every warp
    //      instruction covers four full 128-B row segments, and the scalar
    //      shared stores hit 32 distinct banks (row + 4 g + e, pad 65)
    if (full) {
      float4 v[4];
      const int g = t & 7, rr = t >> 3;
#pragma unroll
      for (int k = 0; k < 4; ++k)
        v[k] = __ldcs(reinterpret_cast<const float4*>(src + (r0 + rr + 32 * (k >> 1)) * w + c0 +
                                                     4 * (g + 8 * (k & 1))));
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float* row = tile[rr + 32 * (k >> 1)] + 4 * (g + 8 * (k & 1));
        row[0] = v[k].x;
        row[1] = v[k].y;
        row[2] = v[k].z;
        row[3] = v[k].w;
      }
    } else {
      // scalar, guarded: warp reads 32 consecutive floats of a row
      for (int k = 0; k < TT * TT / TR_THREADS; ++k) {
        const int e = t + k * TR_THREADS, r = e >> 6, c = e & 63;
        if (r0 + r < h && c0 + c < w) tile[r][c] = __ldcs(src + (r0 + r) * w + c0 + c);
      }
    }
    __syncthreads();
    // ---- store: warp writes 32 consecutive floats of dst row c0 + j:
    //      dst[c0 + j][r0 + i] = tile[i][j], i = lane (+ 32), j = warp + 8 m
    const bool rows_in = r0 + TT <= h;
#pragma unroll 4
    for (int m = 0; m < TT / 8; ++m) {
      const int j = warp + 8 * m;
      if (c0 + j >= w) break;
      float* drow = dst + (c0 + j) * h + r0;
      if (rows_in) {
        __stcs(drow + lane, tile[lane][j]);
        __stcs(drow + lane + 32, tile[lane + 32][j]);
      } else {
        if (r0 + lane < h) __stcs(drow + lane, tile[lane][j]);
        if (r0 + lane + 32 < h) __stcs(drow + lane + 32, tile[lane + 32][j]);
      }
    }
    __syncthreads();  // tile reused by the next iteration
  }
}

int launch_transpose_f32(const float* src, float* dst, int64_t h, int64_t w, int sms, cudaStream_t stream) {
  const int64_t tiles_h = (h + TT - 1) / TT, tiles_w = (w + TT - 1) / TT, ntiles = tiles_h * tiles_w;
  // 16-byte row loads need 16-byte aligned rows: w % 4 == 0 and src aligned
  const int vec_ok = (w % 4 == 0) && (reinterpret_cast<uintptr_t>(src) % 16 == 0);
#ifndef TR_PERSIST
#define TR_PERSIST 0  // 1: one resident wave (8 CTAs per SM) looping over tiles; 0: one CTA per tile
#endif
  int64_t blocks = ntiles;
  if (TR_PERSIST && blocks > int64_t(sms) * 8) blocks = int64_t(sms) * 8;
  if (blocks > 0x7FFFFFFF) blocks = 0x7FFFFFFF;  // the kernel loops over the rest
  if (blocks == 0) return 0;
  k_transpose_f32<<<unsigned(blocks), TR_THREADS, 0, stream>>>(src, dst, h, w, tiles_w, ntiles, vec_ok);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, "k_transpose_f32 launch");
  return 0;
}

}  // namespace hplep
