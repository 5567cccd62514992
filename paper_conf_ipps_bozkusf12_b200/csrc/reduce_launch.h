// reduce_launch.h — internal interface of the HBM-bound kernels: the F2
// reduction and the F4 transpose.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/hpl.h"

namespace hplep {

int set_error(int code, const char* fmt, ...);
int set_cuda_error(cudaError_t e, const char* what);

struct ReduceWorkspace {
  double* partials = nullptr;
  unsigned* counter = nullptr;
  int capacity = 0;
};

int launch_reduce_sum_f32(const float* in, int64_t n, double* out, ReduceWorkspace& ws, int sms,
                          cudaStream_t stream);

// F4 transpose (transpose_kernel.cu): dst (w x h) = src (h x w) transposed.
int launch_transpose_f32(const float* src, float* dst, int64_t h, int64_t w, int sms, cudaStream_t stream);

}  // namespace hplep
