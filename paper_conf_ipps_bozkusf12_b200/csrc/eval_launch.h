// eval_launch.h — internal interface of the generic hpl_eval (F1).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/hpl.h"

namespace hplep {

int set_error(int code, const char* fmt, ...);

// A resolved index domain: unused dimensions have global = local = 1.
struct EvalDomain {
  int ndim;
  int64_t global[3];
  int64_t local[3];
};

// Registered kernel: name, argument signature (see hpl_kernel_info), launcher
// (ptrs[i] = device pointer of array argument i, or nullptr for scalars) and
// the element count each array argument must hold for a domain.
struct KernelDesc {
  const char* name;
  const char* signature;
  int (*launch)(const EvalDomain& D, void* const* ptrs, const hpl_arg* args, cudaStream_t s);
  int64_t (*need)(const EvalDomain& D, int arg);
};

int kernel_count();
const KernelDesc* kernel_at(int i);
const KernelDesc* kernel_find(const char* name);

}  // namespace hplep
