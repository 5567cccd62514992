// reduce_launch.h — internal interface of the F2 reduction kernel.
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

}  // namespace hplep
