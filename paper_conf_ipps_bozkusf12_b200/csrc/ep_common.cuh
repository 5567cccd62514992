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

// The I2F form (EP_I2F, the default): y = x 2^18 - 2^63 as a signed 64-bit
// integer, i.e. the state in the top 46 bits with the sign bit flipped.  For
// odd a, a (y + 2^63) + 2^63 = a y + (a + 1) 2^63 = a y (mod 2^64), so one LCG
// step is y' = a y mod 2^64 (two integer instructions, the low 18 bits stay
// 0), and the exact conversion I2F.F64.S64(y) = (x - 2^45) 2^18 = x' 2^64 is
// NPB's x/2 = u - 1/2 scaled by a power of two.
constexpr uint64_t SIGN64 = uint64_t(1) << 63;
EP_HD uint64_t state_to_y(uint64_t x) { return (x << 18) ^ SIGN64; }
EP_HD uint64_t y_to_state(uint64_t y) { return (y ^ SIGN64) >> 18; }

// Jump table J[i] = a^(2^i) mod 2^46, i = 0..45.
constexpr int NJUMP = 46;

// ---- lean-log table ---------------------------------------
// The kernel works with t' = t/4 in (0, 1/4] (x' = x/2, exact).  -2 ln t is
// computed as T[u] + r * q(r) where u indexes (exponent, top LOG_K mantissa
// bits) of t' rounded to the nearest bucket centre c, inv[u] is a
// float-exact approximation of 1/c, r = fma(t', inv[u], -1) (|r| <= 2^-9) and
// T[u] = RN(2 ln(inv[u] / 4)), so that -2 ln t = T[u] - 2 ln(1 + r).
#ifndef EP_LOG_K
#define EP_LOG_K 9
#endif
#ifndef EP_LOG_EMIN
#define EP_LOG_EMIN -16
#endif
constexpr int LOG_K = EP_LOG_K;                // mantissa bits per exponent (8: |r| <= 2^-9, 9: 2^-10)
constexpr int LOG_EMIN = EP_LOG_EMIN;          // table covers t >= ~2^LOG_EMIN
constexpr int LOG_SHIFT = 20 - LOG_K;          // hi-word shift to the index
constexpr uint32_t LOG_BIAS_TOP = 1023 - 2;    // biased exponent of t' = 1/4
constexpr uint32_t LOG_IDX_MIN = uint32_t(int(LOG_BIAS_TOP) + LOG_EMIN) << LOG_K;
constexpr uint32_t LOG_IDX_MAX = uint32_t(LOG_BIAS_TOP) << LOG_K;  // bucket of t' = 1/4
constexpr uint32_t LOG_N = LOG_IDX_MAX - LOG_IDX_MIN + 1;  // 4097 real entries
// u = (hi(t') + LOG_ADD) >> LOG_SHIFT  (mod 2^32), valid iff u < LOG_N
constexpr uint32_t LOG_ADD = (uint32_t(1) << (LOG_SHIFT - 1)) - (LOG_IDX_MIN << LOG_SHIFT);
// Entries LOG_N .. LOG_N + 511 are reject sentinels {T = 2^1000, inv = 0}: they
// cover every rejected t' in (~1/4, 1/2) and make t2 ~ 2^500, so X, Y are huge
// (l >= 4 and, in the FP32 binning, a selector >= 2^21).  Entry LOG_TINY =
// LOG_N + 512 is the sentinel for t' below the table (the index wraps around
// and is clamped onto it): {T = 60, inv = 0} gives L ~ 64.6 and hence
// max(|X|,|Y|) in [5.6, 8.1], routing the pair to the exact rare path.
// (The older acceptance mode clamps at LOG_N, whose entry is a reject sentinel.)
constexpr uint32_t LOG_TINY = LOG_N + 512;
constexpr uint32_t LOG_TAB = LOG_TINY + 1;

// Truncating index (EP_IDX_TRUNC=1, the default): entry j of the table holds
// the bucket of every t' whose high word H has H >> LOG_SHIFT == j + TRUNC_J0,
// i.e. [lo_j, lo_j + w) with the reference point at its centre (so |r| has the
// same bound as with round-to-nearest buckets).  Entry 0 (j0 = IDX_MIN - 1) is
// the "below the table" sentinel {T = 60, inv = 0}, reached through the clamp
// max(H, TRUNC_HLO); the two buckets around t' = 1/4 ([1/4 - w, 1/4) and
// [1/4, 1/4 + w)) take 1/4 itself as reference point (inv = 4, T = 0, r exact),
// so L = -2 ln(1 + r) never cancels against T as t' -> 1/4; t' = 1/4 gives
// L = 0 (X = Y = 0, bin 0) and every t' > 1/4 a negative L (NaN -> rare path
// -> exact reject); the entries above are reject sentinels up to t' = 1/2.  Address = ((max(H, HLO) >> 11) << 4) + base':
// VIMNMX + SHF + LEA, no recentring add.
constexpr uint32_t TRUNC_J0 = LOG_IDX_MIN - 1;
constexpr uint32_t TRUNC_HLO = TRUNC_J0 << LOG_SHIFT;
constexpr uint32_t TRUNC_TAB = ((LOG_BIAS_TOP + 1) << LOG_K) - TRUNC_J0 + 1;  // up to t' = 1/2
static_assert(TRUNC_TAB == LOG_TAB, "same table footprint in both index modes");

struct LogEntry {
  double T;    // RN(2 ln(inv / 4))
  double inv;  // float-representable ~1/centre
};

// ---- partial results ------------------------------------------------------
struct EPPartial {
  double sx, sy;
  unsigned long long q[10];
  unsigned long long big;  // l >= 10 (HPL_ERANGE)
};

// ---- fused cross-GPU combine ---------------------------
// Every rank owns one CommInbox in its own device memory; peers write into it
// over NVLink (CUDA IPC mappings).  slot[epoch & 1][r] holds rank r's 13-word
// partial {sx, sy, q0..q9, big} in words 0..12 and, in word COMM_TAG, the
// epoch (1, 2, ... per fused call) of the call that wrote it, stored with a
// system-scope release after the data.
constexpr int COMM_MAX_RANKS = 8;
constexpr int COMM_TAG = 13;
struct CommInbox {
  double slot[2][COMM_MAX_RANKS][16];
  unsigned long long stale;     // calls whose tags changed during the fold (a peer ran ahead)
  unsigned long long timeouts;  // calls whose wait gave up (peer missing)
};
struct CommParams {
  CommInbox* inbox[COMM_MAX_RANKS];  // peer inboxes mapped into this process (own at [rank])
  int rank, nranks;                   // nranks == 0: no fused combine
  unsigned long long epoch;           // 1, 2, ... per fused call of this comm
  unsigned long long timeout_ns;      // give up waiting after this long (word 0 := NaN)
};

struct EPParams {
  uint64_t jump[NJUMP];  // a^(2^i) mod 2^46
  double coef[6];        // lean constants (kept in the parameter bank, not registers)
  uint64_t a;            // multiplier
  unsigned a_lo, a_hi;   // its 32-bit halves
  unsigned apow_lo[8], apow_hi[8];  // a^(k+1) mod 2^46, k = 0..7 (parallel LCG steps)
  uint64_t x_begin;      // state before the first uniform of this launch's range
  uint64_t npairs;       // pairs in this launch
  uint64_t base;         // pairs per thread (floor)
  uint64_t extra;        // threads [0, extra) take base + 1 pairs
  const LogEntry* table; // global copy of the lean-log table (LOG_TAB entries)
  EPPartial* partials;   // [gridDim.x]
  unsigned int* counter; // last-block-done ticket, left at 0 after each launch
  double* out13;         // result
  CommParams comm;       // fused cross-GPU combine (comm.nranks == 0: off)
};

}  // namespace hplep
