// ep_common.cuh — shared host/device definitions of the CUDA EP path.
// (CUDA path only: nothing here is shared with oracle/.)
#pragma once
#include <cstdint>

#ifdef __CUDACC__
#define EP_HD __host__ __device__ __forceinline__
#else
#define EP_HD inline
#endif

namespace hplep {

// ---- LCG (NPB randdp.f, reading R2): x_{k+1} = a x_k mod 2^46 -------------
// Exact 64-bit wraparound arithmetic.  For x, a < 2^46 the low 64 bits of
// a*x determine a*x mod 2^46, so `(a * x) & MASK46` is bit-identical to
// NPB's double-split randlc (tests/test_oracle.py pins the oracle's randlc
// to the same identity; tests/test_gpu_parity.py pins this code's states).
constexpr uint64_t MASK46 = (uint64_t(1) << 46) - 1;
constexpr uint64_t MASK52 = (uint64_t(1) << 52) - 1;
constexpr uint64_t EXP_ONE = 0x3FF0000000000000ull;  // bits of 1.0

EP_HD uint64_t mulmod46(uint64_t x, uint64_t y) { return (x * y) & MASK46; }

// The kernel keeps the state as the bit pattern of the double v = 1 + x*2^-46:
// v = EXP_ONE | (x << 6).  Because a*(EXP_ONE) is a multiple of 2^52, one LCG
// step is  v' = ((a * v) & MASK52) | EXP_ONE  — three integer instructions,
// and v' is directly the double 1 + u, so x1 = 2u - 1 = 2v - 3 is one exact
// DFMA.  (Design note in DESIGN.md §4.1.)
EP_HD uint64_t state_to_v(uint64_t x) { return EXP_ONE | (x << 6); }
EP_HD uint64_t v_to_state(uint64_t v) { return (v & MASK52) >> 6; }
EP_HD uint64_t step_v(uint64_t v, uint64_t a) { return ((a * v) & MASK52) | EXP_ONE; }

// Jump table J[i] = a^(2^i) mod 2^46, i = 0..45.
constexpr int NJUMP = 46;

// ---- lean-log table ---------------------------------------
// -2 ln t for t in (0, 1] is computed as T[u] + r * q(r) where
// u indexes (exponent, top LOG_K mantissa bits) of t rounded to the nearest
// bucket centre, inv[u] is a float-exact approximation of 1/centre,
// r = fma(t, inv[u], -1) and T[u] = RN(2 ln inv[u]).
constexpr int LOG_K = 8;                       // mantissa bits per exponent
constexpr int LOG_EMIN = -16;                  // smallest exponent in the table
constexpr int LOG_SHIFT = 20 - LOG_K;          // hi-word shift to the index
constexpr uint32_t LOG_IDX_MIN = uint32_t(1023 + LOG_EMIN) << LOG_K;
constexpr uint32_t LOG_IDX_MAX = uint32_t(1023) << LOG_K;  // bucket of t = 1.0
constexpr uint32_t LOG_N = LOG_IDX_MAX - LOG_IDX_MIN + 1;  // 4097 entries
// u = (hi(t) + LOG_ADD) >> LOG_SHIFT  (mod 2^32), valid iff u < LOG_N
constexpr uint32_t LOG_ADD = (uint32_t(1) << (LOG_SHIFT - 1)) - (LOG_IDX_MIN << LOG_SHIFT);

struct LogEntry {
  double T;    // RN(2 ln inv)
  double inv;  // float-representable ~1/centre
};

// ---- partial results ------------------------------------------------------
struct EPPartial {
  double sx, sy;
  unsigned long long q[10];
  unsigned long long big;  // l >= 10 (HPL_ERANGE)
};

struct EPParams {
  uint64_t jump[NJUMP];  // a^(2^i) mod 2^46
  uint64_t a;            // multiplier
  uint64_t x_begin;      // state before the first uniform of this launch's range
  uint64_t npairs;       // pairs in this launch
  uint64_t base;         // pairs per thread (floor)
  uint64_t extra;        // threads [0, extra) take base + 1 pairs
  const LogEntry* table; // global copy of the lean-log table (LOG_N entries)
  EPPartial* partials;   // [gridDim.x]
  unsigned int* counter; // last-block-done ticket, left at 0 after each launch
  double* out13;         // result
};

}  // namespace hplep
