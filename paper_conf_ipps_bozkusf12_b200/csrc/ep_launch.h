// ep_launch.h — internal interface between the C ABI (hpl_runtime.cpp) and the
// EP kernels (ep_kernel.cu).  Not installed; include/hpl.h is the public API.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/hpl.h"
#include "ep_common.cuh"

namespace hplep {

constexpr int HPL_VARIANT_LEAN = HPL_EP_LEAN;
constexpr int HPL_VARIANT_LIBDEVICE = HPL_EP_LIBDEVICE;
#ifndef EP_DEFAULT_THREADS_CFG
#define EP_DEFAULT_THREADS_CFG 384  // 12 warps x 4 pairs in lockstep (round 2: +2.1 % over 16 warps x 3)
#endif
constexpr int EP_DEFAULT_THREADS = EP_DEFAULT_THREADS_CFG;
#ifndef EP_MIN_PPT
#define EP_MIN_PPT 8   // min pairs per thread before the grid grows (64 -> 8: -8 us at 2^16 pairs, session 3)
#endif
constexpr uint64_t EP_MIN_PAIRS_PER_THREAD = EP_MIN_PPT;

struct EPConfig {
  int variant = HPL_VARIANT_LEAN;
  int threads_per_block = 0;  // 0 = EP_DEFAULT_THREADS
  int blocks_per_sm = 0;      // 0 = occupancy-derived
};

struct JumpTable {
  uint64_t j[NJUMP];
};

// error plumbing (hpl_runtime.cpp): record detail, return the code
int set_error(int code, const char* fmt, ...);
int set_cuda_error(cudaError_t e, const char* what);

void build_jump_table(uint64_t a, uint64_t* J);
uint64_t host_jump(uint64_t x, uint64_t k, const uint64_t* J);

int launch_shape(int device, uint64_t npairs, const EPConfig& cfg, int* blocks, int* threads, int* smem);
int launch_ep(int device, uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t npairs,
              const EPConfig& cfg, double* dev_out13, cudaStream_t stream,
              const CommParams* comm = nullptr);
int launch_lcg_states(uint64_t seed, uint64_t a, uint64_t offset, uint64_t n, uint64_t* dev_out,
                      cudaStream_t stream);
unsigned long long launch_count();
int release_ep_state();
int launch_pairs_debug(int device, uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t n,
                       double* dev_out, cudaStream_t stream);

}  // namespace hplep
