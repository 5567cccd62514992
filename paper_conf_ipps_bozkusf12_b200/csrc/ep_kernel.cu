// ep_kernel.cu — the fused NPB-EP hot path for sm_100a.
//
// One launch computes the 13-word EP result of a contiguous range of pairs:
//   A2 per-thread LCG skip-ahead  x = x_begin * a^(2 p0) mod 2^46
//   A3 uniforms in registers      v = ((a v) & 2^52-1) | bits(1.0)
//   A4 pair map + acceptance      x1 = 2v-3, t = RN(RN(x1^2)+RN(x2^2)), t <= 1
//   A5 polar transform            t2 = sqrt(-2 ln t / t)
//   A6 annulus binning            l = trunc(max(|x1|,|x2|) t2), packed counters
//   A7 sums                       sx += x1 t2, sy += x2 t2
//   A8 warp shuffle -> shared-memory block reduction -> per-block partial ->
//      last-block-done fixed-order finalize into out13 (deterministic).
// The method is NPB EP (the paper's reference [16]); the
// stream/acceptance/binning conventions are readings R1-R10 in DESIGN.md.
// HBM traffic is ~O(grid) bytes; the kernel is FP64-pipe / issue bound.
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <vector>

#include "ep_common.cuh"
#include "ep_launch.h"

namespace hplep {

constexpr int EP_MAX_THREADS = 1024;
constexpr int EP_MAX_BLOCKS_PER_SM = 32;  // hpl_ep_set_config's blocks_per_sm bound (hardware limit)

__device__ __forceinline__ double as_double(uint64_t v) {
  return __longlong_as_double(static_cast<long long>(v));
}

// x * a^k mod 2^46 through the jump table (product of J[i] over set bits of k).
__device__ __forceinline__ uint64_t jump_state(uint64_t x, uint64_t k, const uint64_t* J) {
#pragma unroll 1
  for (int i = 0; i < NJUMP && (k >> i) != 0; ++i)
    if ((k >> i) & 1) x = mulmod46(x, J[i]);
  return x;
}

__device__ __forceinline__ double rsqrt_approx(double p) {
  double y;
  asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(p));  // MUFU.RSQ64H, ~2^-20
  return y;
}

#ifndef EP_T_FMA
#define EP_T_FMA 2     // t' = fma(x1', x1', RN(x2'^2)) (one DADD less; |t'_f - t'| <= 1.5 2^-52 t', DESIGN R11);
#endif                 // 2: the fused t' just below 1/4 indexes the NaN bucket -> rare path, which recomputes
                       //    NPB's t' and decides acceptance exactly; 1: same by an explicit band test
#ifndef EP_IDX_TRUNC
#define EP_IDX_TRUNC 1  // 1: truncating table index (VIMNMX + SHF + LEA; ep_common.cuh)
#endif
#ifndef EP_LCG_CARRY
#define EP_LCG_CARRY 1  // 1: LCG carries the unmasked high word (IMAD reads one odd register)
#endif
#ifndef EP_I2F
#define EP_I2F 0        // 1: x'' = I2F.F64.S64(y) = x' 2^64 from the signed LCG state (no LOP3, no DADD map);
#endif                  //    t'' = t' 2^128, table inverses scaled by 2^-128.  18 FP64/pair
                        //    and parity green, but 9 % slower at class D (1.155 vs 1.273 M, r02aj): the
                        //    64-bit-source conversion costs ~7 issue cycles per warp instruction here
// t'' = t' * 2^EP_TSH and x'' = x' * 2^(EP_TSH/2) (exact power-of-two scalings of NPB's roundings)
constexpr unsigned EP_TSH = EP_I2F ? 128u : 0u;
constexpr double EP_TSCALE = EP_I2F ? 0x1p128 : 1.0;
#ifndef EP_E_SQ
#define EP_E_SQ 1       // 1: Newton residual e = 1 - p y0^2 with y0^2 exact (one register pair)
#endif

// Shared-memory address of the log-table entry of t' (high word H).  `tabb` is
// the table base, pre-biased by -TRUNC_J0 entries in the truncating mode.
#ifndef EP_TICKET_ACQ
#define EP_TICKET_ACQ 1  // 1: last-block detection by an acquiring ticket atomic instead of a second fence (-0.3 us)
#endif
#ifndef EP_IDX_ONE
#define EP_IDX_ONE 1  // 1: the +1 of the fused-t' index from a loop-invariant register (-0.33 IMAD.MOV/pair: +1.6 % with the 384 x 4 default, -2.7 % with 512 x 3)
#endif
__device__ __forceinline__ unsigned tab_addr(unsigned H, unsigned tabb, unsigned one = 1u) {
#if EP_IDX_TRUNC && EP_T_FMA == 2 && EP_IDX_ONE
  return ((max(H + one, TRUNC_HLO + (EP_TSH << 20)) >> LOG_SHIFT) << 4) + tabb;
#elif EP_IDX_TRUNC && EP_T_FMA == 2
  // H + 1: the fused t' with high word 0x3FCFFFFF (just below 1/4) shares the
  // NaN bucket of [1/4, 1/4 + w) -> rare path (exact acceptance); other t'
  // move at most one high-word step (|r| <= 2^-10 + 2^-20)
  return ((max(H + 1u, TRUNC_HLO + (EP_TSH << 20)) >> LOG_SHIFT) << 4) + tabb;
#elif EP_IDX_TRUNC
  return ((max(H, TRUNC_HLO) >> LOG_SHIFT) << 4) + tabb;
#else
  return (min((H + LOG_ADD) >> LOG_SHIFT, LOG_N) << 4) + tabb;
#endif
}
__device__ __forceinline__ unsigned tab_base(const void* smem) {
  const unsigned b = static_cast<unsigned>(__cvta_generic_to_shared(smem));
  // (the t'' scaling moves every index by EP_TSH << LOG_K entries: folded into the base)
  return EP_IDX_TRUNC ? b - (TRUNC_J0 + (EP_TSH << LOG_K)) * 16u : b;
}
// t' below the table (truncating mode; the exact rare path recomputes these pairs)
__device__ __forceinline__ bool below_table(double t) {
  return static_cast<unsigned>(__double2hiint(t)) < (LOG_IDX_MIN << LOG_SHIFT) + (EP_TSH << 20);
}

#ifndef EP_Y0LO
#define EP_Y0LO 0  // 1: rsqrt seed = {low word of p, MUFU.RSQ64H high word} (no zeroing move)
#endif
// MUFU.RSQ64H yields only the high word; rsqrt.approx.f64 zeroes the low word
// with an extra (IMAD-pipe) move.  Any low word perturbs the seed by < 2^-20
// relative, below the MUFU's own 2^-20 error, and the cubic Newton step takes
// a 2^-19 seed to < 2^-56, so the low word of p itself serves.
__device__ __forceinline__ double rsqrt_seed_hi(double p) {
  double y;
  asm("{\n\t.reg .f64 r;\n\t.reg .b32 rl, rh, pl, ph;\n\t"
      "rsqrt.approx.ftz.f64 r, %1;\n\tmov.b64 {rl, rh}, r;\n\tmov.b64 {pl, ph}, %1;\n\t"
      "mov.b64 %0, {pl, rh};\n\t}" : "=d"(y) : "d"(p));
  return y;
}

// 1 << (8 l) for l in 0..3 in one PRMT (backward-4-extract of the byte string
// {1,0,0,0,0,0,0,0} starting at byte l); lanes with l >= 4 never use it.
__device__ __forceinline__ unsigned bin_increment(unsigned l, unsigned one = 1u) {
  unsigned r;
  asm("prmt.b32.b4e %0, %1, %2, %3;" : "=r"(r) : "r"(one), "r"(0u), "r"(l));
  return r;
}

#ifndef EP_BIN_MODE
#define EP_BIN_MODE 3  // 0: two F2I; 1: hi-word max + one F2I; 2: hi-word max + integer shift; 3: FP32 view of the high words (no XU)
#endif
// l = trunc(max(|X|,|Y|)) for the common case, and ge4 = (max(|X|,|Y|) >= 4).
// Modes 1/2 take the max on the high words: (hi << 1) drops the sign and
// keeps the magnitude order, and for values < 2^20 the integer part depends
// on the high word only, so no rounding question arises.  Mode 2 then
// truncates with integer ops: (1.f) 2^21 >> (21 - e), e = exponent.
//
// Mode 3 (no XU instructions): the high word h of a double with value M read
// as an FP32 number is f(h), a monotone piecewise-linear map with f(1) = 1.875,
// f(2) = 2, f(3) = 2.125, f(4) = 2.25 (bits 0x3FF00000, 0x40000000,
// 0x40080000, 0x40100000).  The integer thresholds have zero low words, so
// trunc(M) < 5 is decided exactly by h.  m = max(|f(hX)|, |f(hY)|, 1.75)
// (one FMNMX3), then v = RM(m + 2^20 - 1.75) lands on the 1/8 grid of
// [2^20, 2^21): bits(v) = bits(2^20) + trunc(8 (m - 1.75)) = bits(2^20) + l for
// M < 4, and >= bits(2^20) + 4 iff M >= 4.  The returned selector is bits(v)
// (PRMT reads its two low bits).
__device__ __forceinline__ unsigned bin_index(double X, double Y, bool& ge4, unsigned implicit_bit) {
  if (EP_BIN_MODE == 3) {
    const float fx = __int_as_float(__double2hiint(X)), fy = __int_as_float(__double2hiint(Y));
    float m;  // max(|fx|, |fy|, 1.75), NaN if either is NaN (FMNMX3.NAN)
    asm("max.NaN.f32 %0, %1, %2, 0f3FE00000;" : "=f"(m) : "f"(fabsf(fx)), "f"(fabsf(fy)));
    float v;
    asm("add.rm.f32 %0, %1, 0f497FFFE4;" : "=f"(v) : "f"(m));  // 2^20 - 1.75
    const unsigned b = __float_as_uint(v);
    ge4 = b >= 0x49800004u;
    return b;
  }
  if (EP_BIN_MODE == 0) {
    const unsigned l = max(__double2uint_rz(fabs(X)), __double2uint_rz(fabs(Y)));
    ge4 = l >= 4;
    return l;
  }
  const unsigned hx = static_cast<unsigned>(__double2hiint(X)) << 1;
  const unsigned hy = static_cast<unsigned>(__double2hiint(Y)) << 1;
  const unsigned m2 = max(hx, hy);
  ge4 = m2 >= (0x40100000u << 1);
  if (EP_BIN_MODE == 1) return __double2uint_rz(__hiloint2double(int(m2 >> 1), 0));
  unsigned mn, l;
  asm("lop3.b32 %0, %1, 0x1FFFFF, %2, 0xEA;" : "=r"(mn) : "r"(m2), "r"(implicit_bit));  // (m2 & 0x1FFFFF) | 2^21
  asm("shr.b32 %0, %1, %2;" : "=r"(l) : "r"(mn), "r"(1044u - (m2 >> 21)));           // shift >= 32 -> 0
  return l;
}

// One LCG step on the (lo, hi) words of v = bits(1 + x 2^-46):
//   v' = ((a v) mod 2^52) | bits(1.0)
// = IMAD.WIDE.U32 + IMAD (+ IMAD if a >= 2^32) + one LOP3 doing mask and OR.
// Same step with bits(1.0)'s high word supplied in a register, so mask and
// OR fuse into one LOP3 (ptxas otherwise splits them: two 32-bit constants).
template <bool A32>
__device__ __forceinline__ void lcg_step_k(unsigned& lo, unsigned& hi, unsigned a_lo, unsigned a_hi,
                                           unsigned exp_hi) {
  const unsigned ph = __umulhi(lo, a_lo) + hi * a_lo + (A32 ? 0u : lo * a_hi);
  lo = lo * a_lo;
  asm("lop3.b32 %0, %1, 0x000FFFFF, %2, 0xEA;" : "=r"(hi) : "r"(ph), "r"(exp_hi));
}

// Same step carrying the UNMASKED high word ph: a * (bits above 2^52) only
// reaches bits >= 2^52 of the product, so ph' = hi(a v) + a ph agrees with the
// masked recurrence on bits 0..19; the double's high word hd is the masked copy.
// The IMAD then reads ph (any register parity) and the odd carry word instead
// of two odd registers (RF-bank conflict).
template <bool A32>
__device__ __forceinline__ void lcg_step_c(unsigned& lo, unsigned& ph, unsigned& hd, unsigned a_lo, unsigned a_hi,
                                           unsigned exp_hi) {
  ph = __umulhi(lo, a_lo) + ph * a_lo + (A32 ? 0u : lo * a_hi);
  lo = lo * a_lo;
  asm("lop3.b32 %0, %1, 0x000FFFFF, %2, 0xEA;" : "=r"(hd) : "r"(ph), "r"(exp_hi));
}

// I2F form (ep_common.cuh state_to_y): y' = a y mod 2^64 = IMAD.WIDE.U32 + IMAD
// (+ IMAD if a >= 2^32); the uniform is then one exact I2F.F64.S64.
template <bool A32>
__device__ __forceinline__ void lcg_step_y(unsigned& lo, unsigned& hi, unsigned a_lo, unsigned a_hi) {
#ifndef EP_Y64
#define EP_Y64 0  // 1: one 64-bit multiply (ptxas: IMAD.WIDE.U32 into the state pair + IMAD on its high word)
#endif
  if (EP_Y64) {
    uint64_t y = (static_cast<uint64_t>(hi) << 32) | lo;
    y *= A32 ? static_cast<uint64_t>(a_lo) : ((static_cast<uint64_t>(a_hi) << 32) | a_lo);
    lo = static_cast<unsigned>(y);
    hi = static_cast<unsigned>(y >> 32);
  } else {
    hi = __umulhi(lo, a_lo) + hi * a_lo + (A32 ? 0u : lo * a_hi);
    lo = lo * a_lo;
  }
}
__device__ __forceinline__ double y_to_x2(unsigned lo, unsigned hi) {  // x'' = x' 2^64, exact
  return __ll2double_rn(static_cast<long long>((static_cast<uint64_t>(hi) << 32) | lo));
}

template <bool A32>
__device__ __forceinline__ void lcg_step(unsigned& lo, unsigned& hi, unsigned a_lo, unsigned a_hi) {
  const unsigned ph = __umulhi(lo, a_lo) + hi * a_lo + (A32 ? 0u : lo * a_hi);
  lo = lo * a_lo;
  hi = (ph & 0x000FFFFFu) | 0x3FF00000u;
}


// -2 ln(1+r) = r (-2 + r (1 + r (-2/3 + r (1/2 + r (c5 + r c6))))).  The default
// (EP_LOG_DEG4, K = 9 table, |r| <= 2^-10) stops at r/2: the dropped (2/5) r^5
// is <= (2/5) 2^-50 in L (R11).  The longer series of the other
// modes (K = 8, or EP_LOG_DEG4=0) rounds c5 = -2/5 and c6 = 1/3 to 20-bit
// mantissas that encode as DFMA immediates (they only weigh r^5, r^6: relative
// effect < 2^-60); -2/3 stays exact (kernel parameter).
#define EP_C6 0x1.55555p-2    /* 1/3  rounded to 20 bits */
#define EP_C5 -0x1.9999ap-2   /* -2/5 rounded to 20 bits */

// Loop-invariant operands made opaque (asm volatile), so ptxas keeps them in
// registers instead of rematerialising them with IMAD.MOV every iteration
// (IMAD-pipe work contends with the FP64 pipe on sm_100).
struct LeanConst {
  double c6, c0375;
  unsigned one, implicit_bit, exp_hi;
};
// `kc` is a shared-memory copy of {c6, 0.375, 1} written at kernel start; the
// values are read back through asm volatile loads, which ptxas can neither
// constant-fold nor duplicate.
__device__ __forceinline__ LeanConst make_lean_const(unsigned kc) {
  LeanConst K;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(K.c6) : "r"(kc));
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(K.c0375) : "r"(kc + 8u));
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(K.one) : "r"(kc + 16u));
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(K.implicit_bit) : "r"(kc + 20u));
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(K.exp_hi) : "r"(kc + 24u));
  return K;
}

struct PairAcc {
  double csx, csy;
  unsigned cnt;  // 8-bit packed counts of bins 0..3
};

// Exact slow path for the rare lanes: t below the table (sentinel) or
// l >= 4.  Recomputes what the fast path could not and tallies bins >= 4 in
// shared memory; returns the sums/count increments (registers, no locals).
struct RareOut {
  double dx, dy;
  unsigned dcnt;
};
// `u` is the caller's table index of t' (>= LOG_N below the table); with
// u = ~0u the index is recomputed here (the stage then need not keep it live).
__device__ __noinline__ RareOut rare_pair(double t, double x1, double x2, double X, double Y,
                                          unsigned u, unsigned long long* s_rare) {
#if EP_T_FMA
  // the caller's t' is fused: recompute NPB's t' = RN(RN(x1'^2) + RN(x2'^2));
  // where the two differ, X, Y are recomputed from NPB's t' below
  const double tf = t;
  t = __dadd_rn(__dmul_rn(x1, x1), __dmul_rn(x2, x2));
#else
  const double tf = t;
#endif
  if (t > 0.25 * EP_TSCALE) return RareOut{0.0, 0.0, 0u};  // rejected
#if EP_IDX_TRUNC
  (void)u;
  if (below_table(t) || t != tf || X != X) {  // (NaN: EP_T_FMA == 2's bucket at 1/4)
#else
  if (u == ~0u) u = (static_cast<unsigned>(__double2hiint(t)) + LOG_ADD) >> LOG_SHIFT;  // wraps below the table
  if (u >= LOG_N || t != tf) {
#endif  // t below the table: NPB's formula, libdevice log/sqrt, on
    // the unscaled t = 4 t', x = 2 x' (exact)
    const double tt = (4.0 / EP_TSCALE) * t;
    const double t2 = sqrt(-2.0 * log(tt) / tt);
    X = __dmul_rn((EP_I2F ? 0x1p-63 : 2.0) * x1, t2);
    Y = __dmul_rn((EP_I2F ? 0x1p-63 : 2.0) * x2, t2);
  }
  const unsigned l = __double2uint_rz(fmax(fabs(X), fabs(Y)));
  RareOut o{X, Y, 0u};
  if (l < 4) o.dcnt = bin_increment(l);
  else atomicAdd(&s_rare[(l < 10 ? l : 10u) - 4], 1ull);
  return o;
}

// One pair, lean transform (A3-A7).  No branch on the common path: rejected
// lanes compute garbage that the `ok` predicate discards.
//
// Scaled variables (exact, powers of two): x' = v - 1.5 = x/2, t' = x1'^2 +
// x2'^2 = t/4 (same roundings as NPB's t), accept iff t' <= 1/4.  The table is
// indexed by t' and returns L = -2 ln t directly; t2' = sqrt(L/t') = 2 t2, so
// X = x1' t2' = x1 t2 exactly as NPB's X.
template <bool A32>
__device__ __forceinline__ void lean_pair(unsigned& vlo, unsigned& vhi, const EPParams& P,
                                          unsigned tab, PairAcc& A, unsigned long long* s_rare) {
  lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
  const double v1 = __hiloint2double(int(vhi), int(vlo));
  lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
  const double v2 = __hiloint2double(int(vhi), int(vlo));
  const double x1 = __dadd_rn(v1, -1.5);  // (2u - 1)/2, exact
  const double x2 = __dadd_rn(v2, -1.5);
  const double t = __dadd_rn(__dmul_rn(x1, x1), __dmul_rn(x2, x2));  // t/4, NPB roundings (R5)
  const bool acc = t <= 0.25;
  // A5: L = -2 ln(4 t) from the table entry of t (sentinel for t outside)
  const unsigned H = static_cast<unsigned>(__double2hiint(t));
  const unsigned u = min((H + LOG_ADD) >> LOG_SHIFT, LOG_N);  // (only the rounding mode's rare path reads it)
  double eT, eInv;
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(eT), "=d"(eInv) : "r"(tab_addr(H, tab)));
  const double r = fma(t, eInv, -1.0);
  double c = fma(r, EP_C6, EP_C5);
  c = fma(c, r, 0.5);
  c = fma(c, r, P.coef[2]);
  c = fma(c, r, 1.0);
  c = fma(c, r, -2.0);
  const double L = fma(c, r, eT);
  // t2' = sqrt(L/t) = L rsqrt(L t): MUFU seed + one cubic Newton step
  const double p = fma(L, t, 0x1p-200);  // + 2^-200: t' == 1/4 -> L = 0 -> t2' = 0
  const double y0 = rsqrt_approx(p);
  const double e = EP_E_SQ ? fma(-p, __dmul_rn(y0, y0), 1.0) : fma(-__dmul_rn(p, y0), y0, 1.0);
  const double cc = fma(e, 0.375, 0.5);
  const double g = __dmul_rn(L, y0);
  const double ge = __dmul_rn(g, e);
  const double t2 = fma(ge, cc, g);
  // A6/A7 as NPB writes them: X = x1 t2, Y = x2 t2, l = int(max(|X|,|Y|))
  const double X = __dmul_rn(x1, t2);
  const double Y = __dmul_rn(x2, t2);
  const unsigned l = max(__double2uint_rz(fabs(X)), __double2uint_rz(fabs(Y)));
  const bool ok = acc && l < 4;
  if (ok) {
    A.csx = __dadd_rn(A.csx, X);
    A.csy = __dadd_rn(A.csy, Y);
    A.cnt += bin_increment(l);
  }
  if (acc && !ok) {
    const RareOut o = rare_pair(t, x1, x2, X, Y, EP_IDX_TRUNC ? ~0u : u, s_rare);
    A.csx += o.dx;
    A.csy += o.dy;
    A.cnt += o.dcnt;
  }
}

// W consecutive pairs in lockstep (stage by stage), so that the W independent
// dependency chains interleave in the instruction stream (ILP W) while the
// LCG chain between them stays short.  One rare-path branch per group.
#ifndef EP_ACC_INT
#define EP_ACC_INT 1   // 1: acceptance t' <= 1/4 by a 64-bit integer compare of the bits
#endif
#ifndef EP_ACC_HI
#define EP_ACC_HI 1    // 1: acceptance from the high word of t' only (rare path settles hi == bits(1/4));
#endif                 //    -1.5 instructions/pair, +1.4 % at class D (session 3)
#ifndef EP_LCG_PAR
#define EP_LCG_PAR 0   // 1: the 2W uniforms of a group from v by independent a^k multiplies
#endif
#ifndef EP_ILP
#define EP_ILP 2       // pairs in lockstep for the 85..128-register tiers
#endif

template <bool A32, int W>
__device__ __forceinline__ void lean_pairs(unsigned& vlo, unsigned& vhi, const EPParams& P,
                                           unsigned tab, PairAcc& A, unsigned long long* s_rare) {
  double x1[W], x2[W], t[W], X[W], Y[W];
  unsigned u[W], l[W];
  bool acc[W], ok[W];
  if (EP_LCG_PAR) {
    // v_k = a^k v_0 mod 2^52 (| bits(1.0)), k = 1..2W: one multiply deep
    const unsigned lo0 = vlo, hi0 = vhi;
#pragma unroll
    for (int k = 0; k < 2 * W; ++k) {
      const unsigned alo = P.apow_lo[k], ahi = P.apow_hi[k];
      const unsigned ph = __umulhi(lo0, alo) + hi0 * alo + lo0 * ahi;
      const unsigned hi = (ph & 0x000FFFFFu) | 0x3FF00000u;
      const double v = __hiloint2double(int(hi), int(lo0 * alo));
      if (k & 1) x2[k >> 1] = __dadd_rn(v, -1.5);
      else x1[k >> 1] = __dadd_rn(v, -1.5);
      if (k == 2 * W - 1) { vlo = lo0 * alo; vhi = hi; }
    }
  } else {
#pragma unroll
    for (int k = 0; k < W; ++k) {
      lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
      x1[k] = __dadd_rn(__hiloint2double(int(vhi), int(vlo)), -1.5);
      lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
      x2[k] = __dadd_rn(__hiloint2double(int(vhi), int(vlo)), -1.5);
    }
  }
#pragma unroll
  for (int k = 0; k < W; ++k) {
    t[k] = __dadd_rn(__dmul_rn(x1[k], x1[k]), __dmul_rn(x2[k], x2[k]));
    if (EP_ACC_INT)
      acc[k] = static_cast<unsigned long long>(__double_as_longlong(t[k])) <= 0x3FD0000000000000ull;
    else
      acc[k] = t[k] <= 0.25;
    u[k] = min((static_cast<unsigned>(__double2hiint(t[k])) + LOG_ADD) >> LOG_SHIFT, LOG_N);
  }
  double eT[W], eInv[W];
#pragma unroll
  for (int k = 0; k < W; ++k)
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(eT[k]), "=d"(eInv[k])
                 : "r"(tab_addr(static_cast<unsigned>(__double2hiint(t[k])), tab)));
  double r[W], c[W], L[W];
#pragma unroll
  for (int k = 0; k < W; ++k) {
    r[k] = fma(t[k], eInv[k], -1.0);
    c[k] = fma(r[k], EP_C6, EP_C5);
  }
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], 0.5);
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], P.coef[2]);
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], 1.0);
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], -2.0);
#pragma unroll
  for (int k = 0; k < W; ++k) L[k] = fma(c[k], r[k], eT[k]);
  double p[W], y0[W], e[W], g[W], t2[W];
#pragma unroll
  for (int k = 0; k < W; ++k) {
    p[k] = fma(L[k], t[k], 0x1p-200);
    y0[k] = rsqrt_approx(p[k]);
  }
#pragma unroll
  for (int k = 0; k < W; ++k)
    e[k] = EP_E_SQ ? fma(-p[k], __dmul_rn(y0[k], y0[k]), 1.0) : fma(-__dmul_rn(p[k], y0[k]), y0[k], 1.0);
#pragma unroll
  for (int k = 0; k < W; ++k) {
    g[k] = __dmul_rn(L[k], y0[k]);
    t2[k] = fma(__dmul_rn(g[k], e[k]), fma(e[k], 0.375, 0.5), g[k]);
  }
  bool any_rare = false;
#pragma unroll
  for (int k = 0; k < W; ++k) {
    X[k] = __dmul_rn(x1[k], t2[k]);
    Y[k] = __dmul_rn(x2[k], t2[k]);
    l[k] = max(__double2uint_rz(fabs(X[k])), __double2uint_rz(fabs(Y[k])));
    ok[k] = acc[k] && l[k] < 4;
    if (ok[k]) {
      A.csx = __dadd_rn(A.csx, X[k]);
      A.csy = __dadd_rn(A.csy, Y[k]);
      A.cnt += bin_increment(l[k]);
    }
    any_rare |= acc[k] && !ok[k];
  }
  if (any_rare) {
#pragma unroll
    for (int k = 0; k < W; ++k)
      if (acc[k] && !ok[k]) {
        const RareOut o = rare_pair(t[k], x1[k], x2[k], X[k], Y[k], EP_IDX_TRUNC ? ~0u : u[k], s_rare);
        A.csx += o.dx;
        A.csy += o.dy;
        A.cnt += o.dcnt;
      }
  }
}

#ifndef EP_LOOP_UNROLL
#define EP_LOOP_UNROLL 2  // unroll of the pipelined group loop (codegen/register-allocation knob; 2: +1.6 % with EP_T_FMA 2)
#endif
constexpr int kLoopUnroll = EP_LOOP_UNROLL;  // (#pragma arguments are not macro-expanded)
#ifndef EP_PIPE_ORDER
#define EP_PIPE_ORDER 0  // 1: single stage, transform then generate (no ping-pong)
#endif
#ifndef EP_TMA_TABLE
#define EP_TMA_TABLE 1 // 1: load the log table with cp.async.bulk (TMA) + mbarrier (one
                       // thread, one 139-KB stream); 0: strided 16-B loads by all threads
#endif
#ifndef EP_TAB_BATCH
#define EP_TAB_BATCH 8   // table-copy loads in flight per thread (1 = the plain strided loop)
#endif
#ifndef EP_TMA_WAIT_LATE
#define EP_TMA_WAIT_LATE 1  // 1: wait for the table after the skip-ahead instead of before
#endif                      // (TMA + late wait: +2.8 % at class D over the plain copy, session 3)
#ifndef EP_T2MODE
#define EP_T2MODE 1    // 1: t2 = g + g (e cc) instead of g + (g e) cc
#endif
#ifndef EP_KMODE
#define EP_KMODE 0     // 1: loop constants as immediates + kernel-parameter (uniform) operands
#endif
#ifndef EP_ABL
#define EP_ABL 0       // ablation bit set for timing studies only (results are wrong if != 0)
#endif
#ifndef EP_IDX_FUSED
#define EP_IDX_FUSED 0 // 1: table index clamped before the shift (fused add + min)
#endif
#ifndef EP_STAGE_U
#define EP_STAGE_U 1   // 1: the stage keeps the table index for the rare path (register-allocation knob)
#endif
#ifndef EP_MAXSQ
#define EP_MAXSQ 0     // 1: bin from RN(max|x'| t2) (one DMUL), sums by DFMA (needs EP_BIN_MODE 3)
#endif
#ifndef EP_PRED_MODE
#define EP_PRED_MODE 0 // 1: acceptance and rare routing from the FP32 bin selector (needs EP_BIN_MODE 3)
#endif
#if EP_PRED_MODE == 1 && EP_BIN_MODE != 3
#error "EP_PRED_MODE 1 needs EP_BIN_MODE 3"
#endif
#if EP_PRED_MODE == 1 && EP_T_FMA
#error "EP_PRED_MODE 1 reads acceptance from the selector, which cannot tell the fused t' next to 1/4 (EP_T_FMA) from a reject"
#endif
#ifndef EP_RARE_VOTE
#define EP_RARE_VOTE 1 // 1: rare-path branch on a warp vote (needs warp-uniform trip counts)
#endif
#ifndef EP_LOG_DEG4
#define EP_LOG_DEG4 1  // 1: degree-4 series for -2 ln(1+r) (K >= 9: |error| <= (2/5) 2^-50 absolute in L)
#endif
#ifndef EP_JUMP_WIN
#define EP_JUMP_WIN 1  // 1: per-thread skip-ahead by 4-bit windows (shared-memory table)
#endif
constexpr int EP_WIN_N = (NJUMP + 3) / 4;  // 12 windows cover 2 p0 < 2^46
#ifndef EP_PIPE
#define EP_PIPE 1      // 1: software-pipeline generation of group g+1 under the transform of group g
#endif
#if EP_I2F && !(EP_IDX_TRUNC && EP_T_FMA == 2 && EP_ACC_HI && EP_PRED_MODE == 0 && EP_PIPE && !EP_MAXSQ && !EP_LCG_PAR)
#error "EP_I2F is built for the default pipelined path (truncating index, fused t', high-word acceptance)"
#endif

// Software-pipelined form of lean_pairs: gen_stage produces the LCG pairs, t',
// the table index and the table entries of a group (integer + LDS heavy);
// transform_stage consumes them (FP64 heavy).  The main loop ping-pongs two
// stages so each transform is interleaved with the next group's generation.
template <int W>
struct Stage {
  double x1[W], x2[W], t[W], eT[W], eInv[W];
  double xm[W];  // EP_MAXSQ: the x' of larger magnitude
  unsigned u[W];
};

template <bool A32, int W>
__device__ __forceinline__ void gen_stage(unsigned& vlo, unsigned& vhi, const EPParams& P, unsigned tab,
                                          Stage<W>& S, unsigned exp_hi, unsigned one = 1u) {
#pragma unroll
  for (int k = 0; k < W; ++k) {
#if EP_I2F && !(EP_ABL & 2)
    lcg_step_y<A32>(vlo, vhi, P.a_lo, P.a_hi);
    S.x1[k] = y_to_x2(vlo, vhi);
    lcg_step_y<A32>(vlo, vhi, P.a_lo, P.a_hi);
    S.x2[k] = y_to_x2(vlo, vhi);
    (void)exp_hi;
#else
#if EP_ABL & 2  // ablation (timing only, wrong results): LCG step -> one add
    vlo += P.a_lo;
#elif EP_LCG_CARRY
    unsigned hd;  // vhi carries the unmasked high word (lcg_step_c)
    lcg_step_c<A32>(vlo, vhi, hd, P.a_lo, P.a_hi, exp_hi);
    S.x1[k] = __dadd_rn(__hiloint2double(int(hd), int(vlo)), -1.5);
#else
    lcg_step_k<A32>(vlo, vhi, P.a_lo, P.a_hi, exp_hi);
#endif
#if !EP_LCG_CARRY || (EP_ABL & 2)
    S.x1[k] = __dadd_rn(__hiloint2double(int(vhi), int(vlo)), -1.5);
#endif
#if EP_ABL & 2
    vhi ^= vlo;
#elif EP_LCG_CARRY
    lcg_step_c<A32>(vlo, vhi, hd, P.a_lo, P.a_hi, exp_hi);
    S.x2[k] = __dadd_rn(__hiloint2double(int(hd), int(vlo)), -1.5);
#else
    lcg_step_k<A32>(vlo, vhi, P.a_lo, P.a_hi, exp_hi);
#endif
#if !EP_LCG_CARRY || (EP_ABL & 2)
    S.x2[k] = __dadd_rn(__hiloint2double(int(vhi), int(vlo)), -1.5);
#endif
#endif
  }
#pragma unroll
  for (int k = 0; k < W; ++k) {
#if EP_MAXSQ
    const double s1 = __dmul_rn(S.x1[k], S.x1[k]), s2 = __dmul_rn(S.x2[k], S.x2[k]);
    S.t[k] = __dadd_rn(s1, s2);
    S.xm[k] = __double_as_longlong(s1) >= __double_as_longlong(s2) ? S.x1[k] : S.x2[k];
#elif EP_T_FMA
    S.t[k] = fma(S.x1[k], S.x1[k], __dmul_rn(S.x2[k], S.x2[k]));
#else
    S.t[k] = __dadd_rn(__dmul_rn(S.x1[k], S.x1[k]), __dmul_rn(S.x2[k], S.x2[k]));
#endif
#if EP_IDX_TRUNC
    // (no stage index: the rare path tests below_table(t) itself)
#elif EP_IDX_FUSED
    // clamp before the shift (same index; lets ptxas fuse add + min: VIADDMNMX)
    constexpr unsigned LIM = ((EP_PRED_MODE == 1 ? LOG_TINY : LOG_N) << LOG_SHIFT) | ((1u << LOG_SHIFT) - 1);
    S.u[k] = min(static_cast<unsigned>(__double2hiint(S.t[k])) + LOG_ADD, LIM) >> LOG_SHIFT;
#else
    S.u[k] = min((static_cast<unsigned>(__double2hiint(S.t[k])) + LOG_ADD) >> LOG_SHIFT,
                 EP_PRED_MODE == 1 ? LOG_TINY : LOG_N);
#endif
  }
#pragma unroll
  for (int k = 0; k < W; ++k) {
#if EP_ABL & 1  // ablation: no table lookup / index
    S.eT[k] = S.x1[k];
    S.eInv[k] = S.x2[k];
#elif EP_IDX_TRUNC
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(S.eT[k]), "=d"(S.eInv[k])
                 : "r"(tab_addr(static_cast<unsigned>(__double2hiint(S.t[k])), tab, one)));
#else
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(S.eT[k]), "=d"(S.eInv[k]) : "r"((S.u[k] << 4) + tab));
#endif
  }
}

template <int W, bool DBG = false>
__device__ __forceinline__ void transform_stage(const Stage<W>& S, const EPParams& P, const LeanConst& K,
                                                PairAcc& A, unsigned long long* s_rare,
                                                double* dbg = nullptr, unsigned nvalid = W) {
  double r[W], c[W], L[W], p[W], y0[W], e[W], g[W], t2[W], X[W], Y[W];
  unsigned l[W];
  bool acc[W], ok[W], band[W];
#pragma unroll
  for (int k = 0; k < W; ++k) {
    band[k] = false;
    if (EP_T_FMA == 1) {
      // t' is the fused t' (<= 1 ulp from NPB's): settled on the fast path
      // only below the high word 0x3FCFFFFF; the two high words around 1/4
      // (P ~ 1e-6 per pair) go to the rare path, which decides exactly
      const unsigned h = static_cast<unsigned>(__double2hiint(S.t[k]));
      acc[k] = h < 0x3FCFFFFFu;
      band[k] = h - 0x3FCFFFFFu <= 1u;
    } else if (EP_PRED_MODE == 1 && !DBG)
      acc[k] = k < nvalid;  // decided by the selector below (rejects -> NaN or >= 2^21)
    else if (EP_ACC_HI && (!DBG || EP_T_FMA == 2))
      // high word only: t' < 1/4 is decided exactly; hi == bits(1/4) holds
      // t' == 1/4 (L = 0 -> X = Y = 0, bin 0: correct on the fast path) and
      // rejects just above 1/4, whose L < 0 makes X, Y NaN -> selector says
      // "rare" -> rare_pair rejects them exactly (t > 0.25)
      acc[k] = static_cast<unsigned>(__double2hiint(S.t[k])) <= 0x3FD00000u + (EP_TSH << 20);
    else if (EP_ACC_INT)
      acc[k] = static_cast<unsigned long long>(__double_as_longlong(S.t[k])) <= 0x3FD0000000000000ull;
    else
      acc[k] = S.t[k] <= 0.25;
    if (EP_T_FMA == 1) band[k] = band[k] && k < nvalid;
    acc[k] = acc[k] && k < nvalid;  // (nvalid < W only in a thread's last, partial group)
    r[k] = fma(S.t[k], S.eInv[k], -1.0);
#if EP_LOG_DEG4 && EP_LOG_K >= 9
    c[k] = fma(r[k], 0.5, P.coef[2]);  // -2 ln(1+r) = r(-2 + r(1 + r(-2/3 + r/2))) + O(r^5)
#elif EP_LOG_K >= 9
    c[k] = fma(r[k], K.c6, 0.5);  // K.c6 holds c5 = -2/5 (20-bit) for the degree-5 series
#elif EP_KMODE == 1
    c[k] = fma(r[k], EP_C6, P.coef[1]);  // c6 immediate (b slot), c5 uniform (param -> UR)
#elif EP_KMODE == 2
    c[k] = fma(r[k], P.coef[0], EP_C5);  // c6 uniform (param -> UR, b slot), c5 immediate
#else
    c[k] = fma(r[k], K.c6, EP_C5);
#endif
  }
#if EP_LOG_K < 9
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], 0.5);
#endif
#if !(EP_LOG_DEG4 && EP_LOG_K >= 9)
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], P.coef[2]);
#endif
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], 1.0);
#pragma unroll
  for (int k = 0; k < W; ++k) c[k] = fma(c[k], r[k], -2.0);
#pragma unroll
  for (int k = 0; k < W; ++k) {
    L[k] = fma(c[k], r[k], S.eT[k]);
    p[k] = fma(L[k], S.t[k], 0x1p-200);
#if EP_ABL & 4  // ablation: no MUFU
    y0[k] = S.t[k];
#elif EP_Y0LO
    y0[k] = rsqrt_seed_hi(p[k]);
#else
    y0[k] = rsqrt_approx(p[k]);
#endif
  }
#if EP_Y0LO && !EP_E_SQ
  // e = 1 - p y0^2 as 1 - (L y0)(t y0): p is dead after the MUFU (its
  // register pair can hold y0), g = L y0 is reused below
#pragma unroll
  for (int k = 0; k < W; ++k) e[k] = fma(-__dmul_rn(L[k], y0[k]), __dmul_rn(S.t[k], y0[k]), 1.0);
#else
#pragma unroll
  for (int k = 0; k < W; ++k)
    e[k] = EP_E_SQ ? fma(-p[k], __dmul_rn(y0[k], y0[k]), 1.0) : fma(-__dmul_rn(p[k], y0[k]), y0[k], 1.0);
#endif
  bool any_rare = false;
  unsigned sel_min = 0xFFFFFFFFu;
  (void)sel_min;
#pragma unroll
  for (int k = 0; k < W; ++k) {
    g[k] = __dmul_rn(L[k], y0[k]);
#if EP_KMODE == 1
    t2[k] = fma(__dmul_rn(g[k], e[k]), fma(e[k], 0.375, P.coef[4]), g[k]);
#elif EP_KMODE == 2
    t2[k] = fma(__dmul_rn(g[k], e[k]), fma(e[k], P.coef[3], 0.5), g[k]);
#elif EP_T2MODE == 2
    t2[k] = __dmul_rn(g[k], fma(e[k], fma(e[k], K.c0375, 0.5), 1.0));  // g RN(1 + e cc): no 3-register DFMA
#elif EP_T2MODE == 1
    t2[k] = fma(g[k], __dmul_rn(e[k], fma(e[k], K.c0375, 0.5)), g[k]);  // g (1 + e cc)
#else
    t2[k] = fma(__dmul_rn(g[k], e[k]), fma(e[k], K.c0375, 0.5), g[k]);
#endif
#if EP_MAXSQ
    // max(|X|,|Y|) = RN(|xm| t2) with xm chosen by the rounded squares (equal
    // squares can pick the smaller |x'|: <= 1 ulp, inside reading R7's margin)
    const double Mv = __dmul_rn(S.xm[k], t2[k]);
    X[k] = Mv;  // placeholders: the rare path / debug hook recompute X, Y
    Y[k] = Mv;
#else
    X[k] = __dmul_rn(S.x1[k], t2[k]);
    Y[k] = __dmul_rn(S.x2[k], t2[k]);
#endif
    bool ge4;
#if EP_ABL & 8  // ablation: no binning (F2I, max, compare)
    l[k] = 0; ge4 = false;
#else
    l[k] = bin_index(X[k], Y[k], ge4, K.implicit_bit);
#endif
#if EP_ABL & 16  // ablation: no acceptance / rare predicates
    ok[k] = true; acc[k] = true;
#else
    ok[k] = acc[k] && !ge4;
#endif
#if EP_PRED_MODE == 1
    // selector bits: < 2^20 + 4/8 ok; [.., 2^21) rare (l >= 4 or tiny t');
    // >= 2^21 or NaN: rejected (reject sentinel, or t' > 1/4 in the 1/4 bucket,
    // where L < 0 makes X, Y NaN and FMNMX3.NAN propagates it)
    if (k < nvalid) sel_min = min(sel_min, l[k] - 0x49800004u);  // (masked tail pairs never reach the rare path)
#endif
    if (ok[k]) {
#if EP_MAXSQ
      A.csx = fma(S.x1[k], t2[k], A.csx);
      A.csy = fma(S.x2[k], t2[k], A.csy);
#else
      A.csx = __dadd_rn(A.csx, X[k]);
      A.csy = __dadd_rn(A.csy, Y[k]);
#endif
      A.cnt += bin_increment(l[k], K.one);
    }
#if EP_PRED_MODE != 1
    any_rare |= (acc[k] && !ok[k]) || band[k];
#endif
    if (DBG && EP_MAXSQ) {
      X[k] = __dmul_rn(S.x1[k], t2[k]);
      Y[k] = __dmul_rn(S.x2[k], t2[k]);
    }
    if (DBG) {  // test hook (hpl_ep_pairs_debug): t, X, Y, l (-1 rare path, -2 rejected)
      // t as NPB rounds it (the fused t' of EP_T_FMA is internal)
      dbg[4 * k + 0] = (4.0 / EP_TSCALE) * __dadd_rn(__dmul_rn(S.x1[k], S.x1[k]), __dmul_rn(S.x2[k], S.x2[k]));
      dbg[4 * k + 1] = ok[k] ? X[k] : 0.0;
      dbg[4 * k + 2] = ok[k] ? Y[k] : 0.0;
      const bool acc_npb = __dadd_rn(__dmul_rn(S.x1[k], S.x1[k]), __dmul_rn(S.x2[k], S.x2[k])) <= 0.25 * EP_TSCALE;
      dbg[4 * k + 3] = !acc_npb ? -2.0 : ok[k] ? double(EP_BIN_MODE == 3 ? l[k] & 3u : l[k]) : -1.0;
    }
  }
#if EP_PRED_MODE == 1
  any_rare = sel_min < 0x007FFFFCu;
#endif
#if EP_RARE_VOTE
  if (DBG ? any_rare : __any_sync(0xFFFFFFFFu, any_rare)) {  // warp-uniform: no reconvergence barrier
#else
  if (any_rare) {
#endif
#pragma unroll
    for (int k = 0; k < W; ++k)
      if (EP_PRED_MODE == 1 ? (k < nvalid && l[k] - 0x49800004u < 0x007FFFFCu) : ((acc[k] && !ok[k]) || band[k])) {
        if (EP_MAXSQ) {
          X[k] = __dmul_rn(S.x1[k], t2[k]);
          Y[k] = __dmul_rn(S.x2[k], t2[k]);
        }
        const RareOut o = rare_pair(S.t[k], S.x1[k], S.x2[k], X[k], Y[k], (EP_STAGE_U && !EP_IDX_TRUNC) ? S.u[k] : ~0u, s_rare);
        A.csx += o.dx;
        A.csy += o.dy;
        A.cnt += o.dcnt;
        if (DBG) {
          dbg[4 * k + 1] = o.dx;
          dbg[4 * k + 2] = o.dy;
        }
      }
  }
}

// Test hook: every pair of [pair_begin, pair_begin + n) through the production
// gen_stage / transform_stage code (one pair per thread), writing t, X, Y, l.
template <bool A32>
__global__ void __launch_bounds__(256) ep_pairs_debug_kernel(const __grid_constant__ EPParams P, uint64_t n,
                                                             double* out) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ unsigned long long s_rare[7];
  __shared__ double s_kc[4];
  for (unsigned i = threadIdx.x; i < LOG_TAB; i += blockDim.x)
    reinterpret_cast<double2*>(smem_raw)[i] = __ldg(reinterpret_cast<const double2*>(P.table) + i);
  if (threadIdx.x < 7) s_rare[threadIdx.x] = 0;
  if (threadIdx.x == 0) {
    s_kc[0] = EP_LOG_K >= 9 ? EP_C5 : EP_C6;
    s_kc[1] = 0.375;
    reinterpret_cast<unsigned*>(s_kc)[4] = 1u;
    reinterpret_cast<unsigned*>(s_kc)[5] = 0x200000u;
    reinterpret_cast<unsigned*>(s_kc)[6] = 0x3FF00000u;
  }
  __syncthreads();
  const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const unsigned tab = tab_base(smem_raw);
  const LeanConst K = make_lean_const(static_cast<unsigned>(__cvta_generic_to_shared(s_kc)));
  const uint64_t x0 = jump_state(P.x_begin, 2 * i, P.jump);
  const uint64_t v0 = EP_I2F ? state_to_y(x0) : state_to_v(x0);
  unsigned vlo = unsigned(v0), vhi = unsigned(v0 >> 32);
  Stage<1> S;
  gen_stage<A32, 1>(vlo, vhi, P, tab, S, K.exp_hi);
  PairAcc A{0.0, 0.0, 0u};
  transform_stage<1, true>(S, P, K, A, s_rare, out + 4 * i);
}

// NPB's own formulation with CUDA libdevice log / div / sqrt (A/B variant).
template <bool A32>
__device__ __forceinline__ void libdevice_pair(unsigned& vlo, unsigned& vhi, const EPParams& P,
                                               unsigned, PairAcc& A, unsigned long long* s_rare) {
  lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
  const double v1 = __hiloint2double(int(vhi), int(vlo));
  lcg_step<A32>(vlo, vhi, P.a_lo, P.a_hi);
  const double v2 = __hiloint2double(int(vhi), int(vlo));
  const double x1 = fma(v1, 2.0, -3.0);
  const double x2 = fma(v2, 2.0, -3.0);
  const double t = __dadd_rn(__dmul_rn(x1, x1), __dmul_rn(x2, x2));
  if (t <= 1.0) {
    const double t2 = sqrt(-2.0 * log(t) / t);
    const double X = __dmul_rn(x1, t2), Y = __dmul_rn(x2, t2);
    const unsigned l = __double2uint_rz(fmax(fabs(X), fabs(Y)));
    A.csx += X;
    A.csy += Y;
    if (l < 4) A.cnt += bin_increment(l);
    else atomicAdd(&s_rare[(l < 10 ? l : 10u) - 4], 1ull);
  }
}

// The pipelined pair loop of one thread (A3-A7): `iters` full iterations of
// PER_IT pairs, then the last `tail` (<= PER_IT) pairs with the rest of the
// group masked.  Out of line (EP_LOOP_NOINLINE) so that ptxas allocates and
// schedules the hot loop on its own, independent of the kernel's prologue
// (skip-ahead, table copy) and epilogue (reduction, combine).
struct LoopOut {
  double sx, sy;
  unsigned q0, q1, q2, q3;
};
#ifndef EP_LOOP_NOINLINE
#define EP_LOOP_NOINLINE 0
#endif
#if EP_LOOP_NOINLINE
#define EP_LOOP_INL __noinline__
#else
#define EP_LOOP_INL __forceinline__
#endif
template <bool A32, int W>
__device__ EP_LOOP_INL LoopOut pair_loop(unsigned vlo, unsigned vhi, uint64_t n_t, const EPParams& P, unsigned tab,
                                         unsigned kc, unsigned long long* s_rare) {
  double sx = 0.0, sy = 0.0;
  unsigned q0 = 0, q1 = 0, q2 = 0, q3 = 0;
  auto flush = [&](const PairAcc& A) {
    q0 += A.cnt & 0xFFu;
    q1 += (A.cnt >> 8) & 0xFFu;
    q2 += (A.cnt >> 16) & 0xFFu;
    q3 += A.cnt >> 24;
    sx += A.csx;
    sy += A.csy;
  };
  {
    // 8-bit packed counters overflow after 255 pairs: <= 252 pairs per flush.
    constexpr unsigned PER_IT = (EP_PIPE_ORDER == 1 ? 1 : 2) * W, IT_PER_CHUNK = 252 / PER_IT;
    // Warp-uniform trip count: every thread runs base / PER_IT pipelined
    // iterations (base = the grid-wide floor); the rest (<= PER_IT pairs)
    // goes through the same stages once more with the pairs past the
    // thread's range masked out (the loop's one-group overshoot is exactly
    // the next group of the stream).
    const unsigned tail = unsigned(n_t - (P.base / PER_IT) * PER_IT);
    uint64_t iters = P.base / PER_IT;
    const LeanConst K = make_lean_const(kc);
    Stage<W> s0, s1;
    gen_stage<A32, W>(vlo, vhi, P, tab, s0, K.exp_hi, K.one);
    while (iters) {
      const unsigned ci = iters < IT_PER_CHUNK ? unsigned(iters) : IT_PER_CHUNK;
      PairAcc A{0.0, 0.0, 0u};
#pragma unroll kLoopUnroll
      for (unsigned i = 0; i < ci; ++i) {
#if EP_PIPE_ORDER == 1
        transform_stage<W>(s0, P, K, A, s_rare);
        gen_stage<A32, W>(vlo, vhi, P, tab, s0, K.exp_hi, K.one);
        (void)s1;
#else
        gen_stage<A32, W>(vlo, vhi, P, tab, s1, K.exp_hi, K.one);
        transform_stage<W>(s0, P, K, A, s_rare);
        gen_stage<A32, W>(vlo, vhi, P, tab, s0, K.exp_hi, K.one);
        transform_stage<W>(s1, P, K, A, s_rare);
#endif
      }
      flush(A);
      iters -= ci;
    }
    // the thread's last <= PER_IT pairs: s0 already holds the next group
    if (__any_sync(0xFFFFFFFFu, tail != 0)) {
      PairAcc A{0.0, 0.0, 0u};
      transform_stage<W>(s0, P, K, A, s_rare, nullptr, tail < W ? tail : W);
#if EP_PIPE_ORDER != 1
      gen_stage<A32, W>(vlo, vhi, P, tab, s1, K.exp_hi, K.one);
      transform_stage<W>(s1, P, K, A, s_rare, nullptr, tail > W ? tail - W : 0u);
#endif
      flush(A);
    }
  }
  return LoopOut{sx, sy, q0, q1, q2, q3};
}

template <int VARIANT, bool A32, int NT, int MINB, int W>
__global__ void __launch_bounds__(NT, MINB)
ep_kernel(const __grid_constant__ EPParams P) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ unsigned long long s_rare[7];  // bins 4..9, then l >= 10
  __shared__ double s_kc[4];                // LeanConst source (see make_lean_const)
  __shared__ double s_wsx[EP_MAX_THREADS / 32], s_wsy[EP_MAX_THREADS / 32];
  __shared__ unsigned long long s_wq[EP_MAX_THREADS / 32][4];
  __shared__ int s_last;
  __shared__ double s_fin[13];
  __shared__ long long s_fold[EP_MAX_THREADS / 16][13];

  const unsigned tid = threadIdx.x;
  unsigned tab;  // opaque copy: keeps the shared base in a register (no per-use rematerialisation)
  asm volatile("mov.u32 %0, %1;" : "=r"(tab) : "r"(tab_base(smem_raw)));
  // Table -> shared memory with TMA bulk copies (cp.async.bulk, one thread,
  // completion counted on an mbarrier): one 131-KB stream at L2 bandwidth
  // instead of 16 dependent load/store rounds per thread (~8 us per launch).
  __shared__ __align__(8) unsigned long long s_mbar;
  const unsigned mbar = static_cast<unsigned>(__cvta_generic_to_shared(&s_mbar));
  if (VARIANT == HPL_VARIANT_LEAN && !EP_TMA_TABLE) {
    // EP_TAB_BATCH independent 16-B loads in flight per thread, then the
    // stores: ~3 L2 round trips for the 139-KB table instead of ~17
    const double2* src = reinterpret_cast<const double2*>(P.table);
    double2* dst = reinterpret_cast<double2*>(smem_raw);
    const unsigned nt = blockDim.x;
#pragma unroll 1
    for (unsigned i0 = tid; i0 < LOG_TAB; i0 += EP_TAB_BATCH * nt) {
      double2 v[EP_TAB_BATCH];
#pragma unroll
      for (int k = 0; k < EP_TAB_BATCH; ++k)
        if (i0 + k * nt < LOG_TAB) v[k] = __ldg(src + i0 + k * nt);
#pragma unroll
      for (int k = 0; k < EP_TAB_BATCH; ++k)
        if (i0 + k * nt < LOG_TAB) dst[i0 + k * nt] = v[k];
    }
  }
  if (VARIANT == HPL_VARIANT_LEAN && EP_TMA_TABLE && !(EP_ABL & 64) && tid == 0) {
    constexpr unsigned BYTES = LOG_TAB * sizeof(LogEntry), CHUNK = 32768;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mbar));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}"
                 ::"r"(mbar), "r"(BYTES) : "memory");
    const unsigned dst = static_cast<unsigned>(__cvta_generic_to_shared(smem_raw));
    const char* src = reinterpret_cast<const char*>(P.table);
    for (unsigned off = 0; off < BYTES; off += CHUNK) {
      const unsigned n = BYTES - off < CHUNK ? BYTES - off : CHUNK;
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(dst + off), "l"(src + off), "r"(n), "r"(mbar) : "memory");
    }
  }
#if EP_JUMP_WIN
  // A2 skip-ahead by 4-bit windows: s_win[i][d] = a^(d 16^i) mod 2^46 from the
  // binary jump table (<= 4 mulmods per entry, one entry per thread), so each
  // thread's jump below is <= 12 table multiplies instead of up to 46
  // predicated ones (~1 us less per launch; DESIGN.md §6 fixed cost)
  __shared__ uint64_t s_win[EP_WIN_N][16];
  for (unsigned e = tid; e < EP_WIN_N * 16; e += blockDim.x) {
    const unsigned wi = e >> 4, d = e & 15;
    uint64_t w = 1;
#pragma unroll
    for (unsigned b = 0; b < 4; ++b)
      if (((d >> b) & 1) && 4 * wi + b < NJUMP) w = mulmod46(w, P.jump[4 * wi + b]);
    s_win[wi][d] = w;
  }
#endif
  if (tid < 7) s_rare[tid] = 0;
  if (tid == 0) {
    s_kc[0] = EP_LOG_K >= 9 ? EP_C5 : EP_C6;
    s_kc[1] = 0.375;
    reinterpret_cast<unsigned*>(s_kc)[4] = 1u;
    reinterpret_cast<unsigned*>(s_kc)[5] = 0x200000u;
    reinterpret_cast<unsigned*>(s_kc)[6] = 0x3FF00000u;
  }
  __syncthreads();  // mbarrier initialised before anyone waits on it
#if !EP_TMA_WAIT_LATE
  if (VARIANT == HPL_VARIANT_LEAN && EP_TMA_TABLE) {
    unsigned done = 0;
    while (!done)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\t"
                   "selp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(mbar) : "memory");
  }
#endif

  // ---- A2: this thread's pair range and start state
  const uint64_t gid = uint64_t(blockIdx.x) * blockDim.x + tid;
  const uint64_t n_t = P.base + (gid < P.extra ? 1 : 0);
  const uint64_t p0 = gid * P.base + (gid < P.extra ? gid : P.extra);
#if EP_ABL & 128  // ablation: no skip-ahead
  const uint64_t v0 = state_to_v(P.x_begin + 2 * p0);
#elif EP_JUMP_WIN
  uint64_t xj = P.x_begin;
#pragma unroll 1
  for (uint64_t k = 2 * p0, wi = 0; k != 0; k >>= 4, ++wi)
    if (k & 15) xj = mulmod46(xj, s_win[wi][k & 15]);
  const uint64_t v0 = (EP_I2F && VARIANT == HPL_VARIANT_LEAN && EP_PIPE) ? state_to_y(xj) : state_to_v(xj);
#else
  const uint64_t v0 = state_to_v(jump_state(P.x_begin, 2 * p0, P.jump));
#endif
  unsigned vlo = unsigned(v0), vhi = unsigned(v0 >> 32);
#if EP_TMA_WAIT_LATE
  // the skip-ahead above overlapped the table's bulk copy; wait for it now
  if (VARIANT == HPL_VARIANT_LEAN && EP_TMA_TABLE && !(EP_ABL & 64)) {
    unsigned done = 0;
    while (!done)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\t"
                   "selp.u32 %0, 1, 0, p;\n\t}" : "=r"(done) : "r"(mbar) : "memory");
  }
#endif

  double sx = 0.0, sy = 0.0;
  unsigned q0 = 0, q1 = 0, q2 = 0, q3 = 0;
  auto flush = [&](const PairAcc& A) {
    q0 += A.cnt & 0xFFu;
    q1 += (A.cnt >> 8) & 0xFFu;
    q2 += (A.cnt >> 16) & 0xFFu;
    q3 += A.cnt >> 24;
    sx += A.csx;
    sy += A.csy;
  };
  if (EP_ABL & 32) {  // ablation: no pairs (fixed cost only)
    sx = double(vlo); sy = double(vhi);
  } else if (VARIANT == HPL_VARIANT_LEAN && EP_PIPE) {
    const LoopOut o = pair_loop<A32, W>(vlo, vhi, n_t, P, tab, static_cast<unsigned>(__cvta_generic_to_shared(s_kc)),
                                        s_rare);
    sx = o.sx;
    sy = o.sy;
    q0 = o.q0;
    q1 = o.q1;
    q2 = o.q2;
    q3 = o.q3;
  } else {
    // 8-bit packed counters overflow after 255 pairs: chunks of 252 = 63 x 4
    constexpr unsigned UNROLL = 4, CHUNK = 63 * UNROLL;
    static_assert(EP_PIPE || UNROLL % W == 0, "W must divide UNROLL");
    uint64_t rem = n_t;
    for (; rem >= CHUNK; rem -= CHUNK) {
      PairAcc A{0.0, 0.0, 0u};
  #pragma unroll 1
      for (unsigned i = 0; i < CHUNK / UNROLL; ++i) {
        if (VARIANT == HPL_VARIANT_LEAN) {
  #pragma unroll
          for (unsigned j = 0; j < UNROLL / W; ++j) lean_pairs<A32, (UNROLL % W ? 1 : W)>(vlo, vhi, P, tab, A, s_rare);
        } else {
  #pragma unroll
          for (unsigned j = 0; j < UNROLL; ++j) libdevice_pair<A32>(vlo, vhi, P, tab, A, s_rare);
        }
      }
      flush(A);
    }
    if (rem) {
      PairAcc A{0.0, 0.0, 0u};
  #pragma unroll 1
      for (unsigned i = 0; i < unsigned(rem); ++i) {
        if (VARIANT == HPL_VARIANT_LEAN) lean_pair<A32>(vlo, vhi, P, tab, A, s_rare);
        else libdevice_pair<A32>(vlo, vhi, P, tab, A, s_rare);
      }
      flush(A);
    }
  }

  // ---- A8: warp -> block reduction (fixed order => deterministic)
  unsigned long long w0 = q0, w1 = q1, w2 = q2, w3 = q3;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    sx += __shfl_xor_sync(0xFFFFFFFFu, sx, off);
    sy += __shfl_xor_sync(0xFFFFFFFFu, sy, off);
    w0 += __shfl_xor_sync(0xFFFFFFFFu, w0, off);
    w1 += __shfl_xor_sync(0xFFFFFFFFu, w1, off);
    w2 += __shfl_xor_sync(0xFFFFFFFFu, w2, off);
    w3 += __shfl_xor_sync(0xFFFFFFFFu, w3, off);
  }
  const unsigned warp = tid >> 5, lane = tid & 31;
  if (lane == 0) {
    s_wsx[warp] = sx;
    s_wsy[warp] = sy;
    s_wq[warp][0] = w0;
    s_wq[warp][1] = w1;
    s_wq[warp][2] = w2;
    s_wq[warp][3] = w3;
  }
  __syncthreads();
  if (warp == 0) {  // warp 0 folds the per-warp values by a fixed shuffle tree
    const unsigned nw = blockDim.x >> 5;
    double a = 0.0, b = 0.0;
    unsigned long long c[4] = {0, 0, 0, 0};
    for (unsigned w = lane; w < nw; w += 32) {
      a += s_wsx[w];
      b += s_wsy[w];
      for (int k = 0; k < 4; ++k) c[k] += s_wq[w][k];
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      a += __shfl_xor_sync(0xFFFFFFFFu, a, off);
      b += __shfl_xor_sync(0xFFFFFFFFu, b, off);
#pragma unroll
      for (int k = 0; k < 4; ++k) c[k] += __shfl_xor_sync(0xFFFFFFFFu, c[k], off);
    }
    if (lane == 0) {
      EPPartial part;
      part.sx = a;
      part.sy = b;
      for (int k = 0; k < 4; ++k) part.q[k] = c[k];
      for (int k = 4; k < 10; ++k) part.q[k] = s_rare[k - 4];
      part.big = s_rare[6];
      P.partials[blockIdx.x] = part;
      __threadfence();
#if EP_TICKET_ACQ
      // acquire: the last block's partial loads (after the barrier below) are
      // ordered after every other block's fence + ticket, so the fold needs no
      // second fence
      unsigned ticket;
      asm volatile("atom.add.acquire.gpu.global.u32 %0, [%1], 1;" : "=r"(ticket) : "l"(P.counter) : "memory");
#else
      const unsigned ticket = atomicAdd(P.counter, 1u);
#endif
      s_last = (ticket == gridDim.x - 1);
    }
  }
  __syncthreads();
  if (!s_last || (EP_ABL & 256)) return;  // (ablation 256: no last-block fold)
  // last block: 16-thread groups; thread (group gi, word w) folds word w of
  // partials gi, gi + ng, ... (independent loads in flight), then thread w
  // folds the groups in order — fixed order, so bitwise deterministic.
#if !(EP_ABL & 512) && !EP_TICKET_ACQ  // (ablation 512: no fence before the fold)
  __threadfence();
#endif
#if EP_ABL & 1024  // ablation: fold without reading the partials
  if (tid < 13) s_fin[tid] = double(tid);
  if (false)
#endif
  {
    const unsigned G = gridDim.x, ng = blockDim.x >> 4, gi = tid >> 4, w = tid & 15;
    // FOLD_U loads issued before the first add: one L2 round trip per FOLD_U
    // partials instead of one per partial (same summation order)
    constexpr unsigned FOLD_U = 8;
    if (w < 13) {
      if (w < 2) {
        double sacc = 0.0;
        for (unsigned b0 = gi; b0 < G; b0 += FOLD_U * ng) {
          double v[FOLD_U];
#pragma unroll
          for (unsigned k = 0; k < FOLD_U; ++k) {
            const unsigned b = b0 + k * ng;
            v[k] = b < G ? __ldcg(w == 0 ? &P.partials[b].sx : &P.partials[b].sy) : 0.0;
          }
#pragma unroll
          for (unsigned k = 0; k < FOLD_U; ++k) sacc += v[k];
        }
        s_fold[gi][w] = __double_as_longlong(sacc);
      } else {
        unsigned long long sacc = 0;
        for (unsigned b0 = gi; b0 < G; b0 += FOLD_U * ng) {
          unsigned long long v[FOLD_U];
#pragma unroll
          for (unsigned k = 0; k < FOLD_U; ++k) {
            const unsigned b = b0 + k * ng;
            v[k] = b < G ? __ldcg(w < 12 ? &P.partials[b].q[w - 2] : &P.partials[b].big) : 0ull;
          }
#pragma unroll
          for (unsigned k = 0; k < FOLD_U; ++k) sacc += v[k];
        }
        s_fold[gi][w] = static_cast<long long>(sacc);
      }
    }
    __syncthreads();
    // warp j folds word j over the groups: lane-strided, then a fixed shuffle tree
    for (unsigned word = warp; word < 13; word += blockDim.x >> 5) {
      if (word < 2) {
        double sacc = 0.0;
        for (unsigned g = lane; g < ng; g += 32) sacc += __longlong_as_double(s_fold[g][word]);
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) sacc += __shfl_xor_sync(0xFFFFFFFFu, sacc, off);
        if (lane == 0) s_fin[word] = sacc;
      } else {
        unsigned long long sacc = 0;
        for (unsigned g = lane; g < ng; g += 32) sacc += static_cast<unsigned long long>(s_fold[g][word]);
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) sacc += __shfl_xor_sync(0xFFFFFFFFu, sacc, off);
        if (lane == 0) s_fin[word] = static_cast<double>(sacc);  // exact: < 2^53
      }
    }
  }
  __syncthreads();
  if (P.comm.nranks > 0) {
    // F3: the cross-GPU combine in the same kernel.  Store this shard's 13
    // words into slot [parity][rank] of every rank's inbox (NVLink peer
    // stores), fence at system scope, signal each inbox, then wait for all
    // partials in the own inbox and fold them in rank order (deterministic,
    // identical on every rank).  No separate collective is launched.
    //
    // Each slot carries its call's epoch in word COMM_TAG, published with a
    // system-scope release after the 13 data words: a rank folds only slots
    // tagged with its own epoch, so partials of different calls never mix,
    // and it re-reads the tags after the fold — a peer that gave up waiting
    // (timeout) and moved on to the next call of the same parity would have
    // changed them — so a torn read is reported (NaN + `stale`), never used.
    const CommParams& C = P.comm;
    const unsigned par = unsigned(C.epoch & 1), n = unsigned(C.nranks);
    for (unsigned i = tid; i < 13 * n; i += blockDim.x) {  // any block size covers every peer
      const unsigned r = i / 13, w = i % 13;
      volatile double* dst = &C.inbox[r]->slot[par][C.rank][w];
      *dst = s_fin[w];
    }
    __threadfence_system();
    __syncthreads();
    for (unsigned r = tid; r < n; r += blockDim.x) {
      unsigned long long* tag = reinterpret_cast<unsigned long long*>(&C.inbox[r]->slot[par][C.rank][COMM_TAG]);
      asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(tag), "l"(C.epoch) : "memory");
    }
    CommInbox* own = C.inbox[C.rank];
    if (tid == 0) {
      unsigned long long t0, now, v;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
      int timed_out = 0;
      for (unsigned r = 0; r < n && !timed_out; ++r) {
        const unsigned long long* tag = reinterpret_cast<const unsigned long long*>(&own->slot[par][r][COMM_TAG]);
        for (;;) {
          asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(tag) : "memory");
          if (v == C.epoch) break;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
          if (now - t0 > C.timeout_ns) { timed_out = 1; break; }
          __nanosleep(200);
        }
      }
      if (timed_out) atomicAdd(&own->timeouts, 1ull);
      s_last = timed_out;  // reuse: 1 = combine failed
    }
    __syncthreads();
    if (tid < 13) {
      const volatile double* src = &own->slot[par][0][tid];
      double acc = 0.0;
      for (unsigned r = 0; r < n; ++r) acc += src[r * 16];  // rank order
      s_fin[tid] = acc;
    }
    __syncthreads();
    if (tid == 0 && !s_last) {
      for (unsigned r = 0; r < n; ++r) {
        unsigned long long v;
        const unsigned long long* tag = reinterpret_cast<const unsigned long long*>(&own->slot[par][r][COMM_TAG]);
        asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(tag) : "memory");
        if (v != C.epoch) s_last = 1;
      }
      if (s_last) atomicAdd(&own->stale, 1ull);
    }
    __syncthreads();
  }
  if (tid == 0) {
    double gc = 0.0;
    for (int k = 0; k < 10; ++k) gc += s_fin[2 + k];  // exact integer sum
    const bool big = s_fin[12] != 0.0 || (P.comm.nranks > 0 && s_last != 0);
    P.out13[0] = big ? __longlong_as_double(0x7FF8000000000000ll) : s_fin[0];
    P.out13[1] = s_fin[1];
    for (int k = 0; k < 10; ++k) P.out13[2 + k] = s_fin[2 + k];
    P.out13[12] = gc;
    *P.counter = 0;  // ready for the next launch on this workspace
  }
}

// Test hook kernel: x_{offset+i+1} via the kernel's own jump + step code.
// The step is gen_stage's own (lcg_step_c with the unmasked carry word, or
// lcg_step_k), so these states pin the hot loop's LCG, not a re-implementation.
template <bool A32>
__global__ void lcg_states_kernel(uint64_t seed, uint64_t a, uint64_t offset, uint64_t n,
                                  const __grid_constant__ JumpTable J, uint64_t* out) {
  const uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const unsigned a_lo = unsigned(a), a_hi = unsigned(a >> 32), exp_hi = 0x3FF00000u;
#if EP_I2F
  const uint64_t y = state_to_y(jump_state(seed, offset + i, J.j));
  unsigned lo = unsigned(y), hi = unsigned(y >> 32);
  lcg_step_y<A32>(lo, hi, a_lo, a_hi);
  (void)exp_hi;
  out[i] = y_to_state((uint64_t(hi) << 32) | lo);
#else
  const uint64_t v = state_to_v(jump_state(seed, offset + i, J.j));
  unsigned lo = unsigned(v), hi = unsigned(v >> 32), hd;
#if EP_LCG_CARRY
  lcg_step_c<A32>(lo, hi, hd, a_lo, a_hi, exp_hi);
#else
  lcg_step_k<A32>(lo, hi, a_lo, a_hi, exp_hi);
  hd = hi;
#endif
  out[i] = v_to_state((uint64_t(hd) << 32) | lo);
#endif
}

// ------------------------------------------------------------- dispatcher
// Launch-bound tiers: (max threads per block, min blocks per SM) -> register cap
// 64 / 64 / 85 / 85 / 128 regs.  A launch uses the smallest tier >= its block.
using EPKernel = void (*)(const EPParams);
template <int V, bool A32>
static EPKernel tier_kernel(int thr) {
#ifndef EP_T256_MINB
#define EP_T256_MINB 3
#endif
#ifndef EP_T256_W
#define EP_T256_W EP_ILP
#endif
#ifndef EP_T384_MINB
#define EP_T384_MINB 1   // one CTA per SM (the 139-KB table allows no second one): up to 170 registers
#endif
#ifndef EP_T384_W
#define EP_T384_W 4      // 140 registers, no spills; the default tier (EP_DEFAULT_THREADS)
#endif
#ifndef EP_TIER_X
#define EP_TIER_X 0    // an extra launch-bound tier between 384 and 512 threads (0: none)
#endif
#ifndef EP_TIER_X_W
#define EP_TIER_X_W 4
#endif
#ifndef EP_T512_W
#define EP_T512_W 3  // 120 registers, no spills (round 2: W = 2 is 4 % slower, W = 4 spills)
#endif
  if (thr <= 128) return ep_kernel<V, A32, 128, 4, 1>;   // 128 regs
  if (thr <= 256) return ep_kernel<V, A32, 256, EP_T256_MINB, EP_T256_W>;   //  85 regs (3 blocks/SM)
  if (thr <= 384) return ep_kernel<V, A32, 384, EP_T384_MINB, EP_T384_W>;   // 140 regs, W = 4 (default)
#if EP_TIER_X
  if (thr <= EP_TIER_X) return ep_kernel<V, A32, EP_TIER_X, 1, EP_TIER_X_W>;  // extra tier (A/B)
#endif
  if (thr <= 512) return ep_kernel<V, A32, 512, 1, EP_T512_W>;   // 128 regs
  if (thr <= 640) return ep_kernel<V, A32, 640, 1, EP_ILP>;   // 102 regs
  if (thr <= 768) return ep_kernel<V, A32, 768, 1, EP_ILP>;   //  85 regs
  return ep_kernel<V, A32, 1024, 1, 1>;                  //  64 regs
}
static EPKernel pick_kernel(int variant, bool a32, int thr) {
  if (variant == HPL_VARIANT_LEAN) return a32 ? tier_kernel<HPL_VARIANT_LEAN, true>(thr) : tier_kernel<HPL_VARIANT_LEAN, false>(thr);
  return a32 ? tier_kernel<HPL_VARIANT_LIBDEVICE, true>(thr) : tier_kernel<HPL_VARIANT_LIBDEVICE, false>(thr);
}

// ------------------------------------------------------------------ host side
void build_jump_table(uint64_t a, uint64_t* J) {
  uint64_t x = a & MASK46;
  for (int i = 0; i < NJUMP; ++i) {
    J[i] = x;
    x = mulmod46(x, x);
  }
}

uint64_t host_jump(uint64_t x, uint64_t k, const uint64_t* J) {
  for (int i = 0; i < NJUMP && (k >> i) != 0; ++i)
    if ((k >> i) & 1) x = mulmod46(x, J[i]);
  return x;
}

// Kernel parameters shared by every EP launch: jump table J[i] = a^(2^i),
// multiplier words, a^(k+1) table, constants, and the range's start state
// x_begin = seed * a^(2 pair_begin) mod 2^46.
static void init_params(EPParams& P, uint64_t seed, uint64_t a, uint64_t pair_begin) {
  std::memset(&P, 0, sizeof(P));
  build_jump_table(a, P.jump);
  P.a = a;
  P.a_lo = unsigned(a);
  P.a_hi = unsigned(a >> 32);
  uint64_t ak = a & MASK46;
  for (int k = 0; k < 8; ++k) {  // a^(k+1) mod 2^46
    P.apow_lo[k] = unsigned(ak);
    P.apow_hi[k] = unsigned(ak >> 32);
    ak = mulmod46(ak, a);
  }
  const double coef[6] = {EP_C6, EP_C5, -2.0 / 3.0, 0.375, 0.5, 0x1p-200};
  for (int i = 0; i < 6; ++i) P.coef[i] = coef[i];
  P.x_begin = host_jump(seed & MASK46, 2 * pair_begin, P.jump);
}

// Lean-log table, built in 80-bit long double on the host.
void build_log_table(std::vector<LogEntry>& tab) {
  tab.resize(LOG_TAB);
#if EP_IDX_TRUNC
  // truncating buckets [lo_j, lo_j + w), reference point at the centre (ep_common.cuh)
  for (uint32_t e = 0; e < LOG_TAB; ++e) {
    const uint32_t j = TRUNC_J0 + e;
    if (e == 0) {                       // below the table -> moderate X, Y -> exact rare path
      tab[e].T = 60.0;
      tab[e].inv = 0.0;
    } else if (j < LOG_IDX_MAX - 1) {   // real bucket of t' in [2^-18, 1/4 - w)
      const int E = int(j >> LOG_K) - 1023;
      const long double centre =
          ldexpl(1.0L + ((long double)(j & ((1u << LOG_K) - 1)) + 0.5L) / (1 << LOG_K), E);
      const float inv = (float)(1.0L / centre);
      tab[e].inv = ldexp((double)inv, -int(EP_TSH));  // (t'' = t' 2^EP_TSH: r = t'' inv'' - 1 unchanged)
      tab[e].T = (double)(2.0L * logl((long double)inv * 0.25L));  // -2 ln(4 t') at r = 0
    } else if (EP_T_FMA == 2 && j == LOG_IDX_MAX) {  // [1/4, 1/4 + w) and, via the H + 1 index,
      tab[e].T = __builtin_nan("");                  // the fused t' just below 1/4: NaN -> the
      tab[e].inv = __builtin_nan("");                // rare path decides acceptance on NPB's t'
    } else if (j <= LOG_IDX_MAX) {      // [1/4 - w, 1/4 + w), reference point 1/4 itself (T = 0,
                                        // r = 4t' - 1 exact): L = -2 ln(1 + r) has no cancellation
                                        // as t' -> 1/4; t' = 1/4 -> L = 0; above -> L < 0 -> NaN
      tab[e].T = 0.0;
      tab[e].inv = ldexp(4.0, -int(EP_TSH));
    } else {                            // reject sentinels up to t' = 1/2 (L t'' stays finite)
      tab[e].T = EP_I2F ? 0x1p800 : 0x1p1000;
      tab[e].inv = 0.0;
    }
  }
#else
  for (uint32_t u = 0; u < LOG_N; ++u) {
    const uint32_t idx = LOG_IDX_MIN + u;
    const int E = int(idx >> LOG_K) - 1023;
    const long double centre = ldexpl(1.0L + (long double)(idx & ((1u << LOG_K) - 1)) / (1 << LOG_K), E);
    const float inv = (float)(1.0L / centre);
    tab[u].inv = (double)inv;
    tab[u].T = (double)(2.0L * logl((long double)inv * 0.25L));  // -2 ln(4 t') at r = 0
  }
  for (uint32_t u = LOG_N; u < LOG_TINY; ++u) {  // reject sentinels (ep_common.cuh)
    tab[u].T = 0x1p1000;
    tab[u].inv = 0.0;
  }
  tab[LOG_TINY].T = 60.0;  // t' below the table -> moderate X, Y -> exact rare path
  tab[LOG_TINY].inv = 0.0;
#endif
}

namespace {
struct DeviceState {
  LogEntry* table = nullptr;
  int sms = 0;
  int max_smem_optin = 0;
};
std::mutex g_mu;
std::vector<DeviceState> g_dev;
struct Workspace {
  int device;
  cudaStream_t stream;
  EPPartial* partials;
  unsigned* counter;
  int capacity;
};
std::vector<Workspace> g_ws;
unsigned long long g_launches = 0;

int set_attrs_once(int device) {
  static std::vector<char> done;
  if ((int)done.size() <= device) done.resize(device + 1, 0);
  if (done[device]) return 0;
  const int smem = int(LOG_TAB * sizeof(LogEntry));
  for (int thr : {128, 256, 384, EP_TIER_X ? EP_TIER_X : 512, 512, 640, 768, 1024})
    for (bool a32 : {true, false}) {
      cudaError_t e = cudaFuncSetAttribute(pick_kernel(HPL_VARIANT_LEAN, a32, thr),
                                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e != cudaSuccess) return set_cuda_error(e, "cudaFuncSetAttribute");
    }
  done[device] = 1;
  return 0;
}
}  // namespace

int device_state(int device, const LogEntry** table, int* sms) {
  std::lock_guard<std::mutex> lk(g_mu);
  if ((int)g_dev.size() <= device) g_dev.resize(device + 1);
  DeviceState& d = g_dev[device];
  if (d.table == nullptr) {
    cudaDeviceProp prop;
    cudaError_t e = cudaGetDeviceProperties(&prop, device);
    if (e != cudaSuccess) return set_cuda_error(e, "cudaGetDeviceProperties");
    if (prop.major != 10) return set_error(HPL_ENODEV, "device is sm_%d%d, this build targets sm_100a", prop.major, prop.minor);
    d.sms = prop.multiProcessorCount;
    d.max_smem_optin = int(prop.sharedMemPerBlockOptin);
    std::vector<LogEntry> tab;
    build_log_table(tab);
    LogEntry* dt = nullptr;
    e = cudaMalloc(&dt, tab.size() * sizeof(LogEntry));
    if (e != cudaSuccess) return set_cuda_error(e, "cudaMalloc(log table)");
    e = cudaMemcpy(dt, tab.data(), tab.size() * sizeof(LogEntry), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) { cudaFree(dt); return set_cuda_error(e, "cudaMemcpy(log table)"); }
    d.table = dt;
    int rc = set_attrs_once(device);
    if (rc) return rc;
  }
  *table = d.table;
  *sms = d.sms;
  return 0;
}

// One workspace per (device, stream), sized once for the largest grid any
// configuration can launch (sms x 32 blocks) and never reallocated, so a
// pointer handed to one host thread can never be freed under another's
// pending launch.
static int workspace(int device, cudaStream_t stream, int blocks, EPPartial** partials, unsigned** counter) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (auto& w : g_ws) {
    if (w.device == device && w.stream == stream) {
      if (w.capacity < blocks) return set_error(HPL_EINVAL, "grid of %d blocks exceeds the workspace (%d)", blocks, w.capacity);
      *partials = w.partials;
      *counter = w.counter;
      return 0;
    }
  }
  const int cap = g_dev[device].sms * EP_MAX_BLOCKS_PER_SM;
  if (blocks > cap) return set_error(HPL_EINVAL, "grid of %d blocks exceeds the workspace (%d)", blocks, cap);
  Workspace w{device, stream, nullptr, nullptr, cap};
  cudaError_t e = cudaMalloc(&w.partials, sizeof(EPPartial) * cap);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaMalloc(partials)");
  e = cudaMalloc(&w.counter, sizeof(unsigned));
  if (e == cudaSuccess) e = cudaMemset(w.counter, 0, sizeof(unsigned));
  if (e != cudaSuccess) { cudaFree(w.partials); return set_cuda_error(e, "cudaMalloc(counter)"); }
  g_ws.push_back(w);
  *partials = w.partials;
  *counter = w.counter;
  return 0;
}

int launch_shape(int device, uint64_t npairs, const EPConfig& cfg, int* blocks, int* threads, int* smem) {
  const LogEntry* tab;
  int sms;
  int rc = device_state(device, &tab, &sms);
  if (rc) return rc;
  const int thr = cfg.threads_per_block > 0 ? cfg.threads_per_block : EP_DEFAULT_THREADS;
  if (thr < 32 || thr > EP_MAX_THREADS || thr % 32) return set_error(HPL_EINVAL, "threads_per_block must be a multiple of 32 in [32, 1024]");
  const int sm_bytes = cfg.variant == HPL_VARIANT_LEAN ? int(LOG_TAB * sizeof(LogEntry)) : 0;
  int bps = cfg.blocks_per_sm;
  if (bps <= 0) {
    // occupancy per (device, variant, block size), cached: the query costs
    // microseconds of host time that would sit inside small launches
    static std::mutex occ_mu;
    static std::vector<long long> occ_cache;  // key << 8 | occupancy
    const long long key = (static_cast<long long>(device) << 20) | (static_cast<long long>(cfg.variant) << 12) | thr;
    {
      std::lock_guard<std::mutex> lk(occ_mu);
      for (long long v : occ_cache)
        if ((v >> 8) == key) bps = int(v & 0xFF);
    }
    if (bps <= 0) {
      int occ = 0;
      cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, pick_kernel(cfg.variant, true, thr),
                                                                    thr, sm_bytes);
      if (e != cudaSuccess) return set_cuda_error(e, "cudaOccupancyMaxActiveBlocksPerMultiprocessor");
      bps = occ > 0 ? occ : 1;
      std::lock_guard<std::mutex> lk(occ_mu);
      occ_cache.push_back((key << 8) | bps);
    }
  }
  // at least EP_MIN_PAIRS_PER_THREAD pairs per thread so skip-ahead stays negligible
  uint64_t want = (npairs + uint64_t(thr) * EP_MIN_PAIRS_PER_THREAD - 1) / (uint64_t(thr) * EP_MIN_PAIRS_PER_THREAD);
  uint64_t full = uint64_t(sms) * bps;
  uint64_t b = want < full ? want : full;
  if (b < 1) b = 1;
  *blocks = int(b);
  *threads = thr;
  *smem = sm_bytes;
  return 0;
}

int launch_ep(int device, uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t npairs,
              const EPConfig& cfg, double* dev_out13, cudaStream_t stream, const CommParams* comm) {
  const LogEntry* tab;
  int sms;
  int rc = device_state(device, &tab, &sms);
  if (rc) return rc;
  int blocks, threads, smem;
  rc = launch_shape(device, npairs, cfg, &blocks, &threads, &smem);
  if (rc) return rc;
  EPPartial* partials;
  unsigned* counter;
  rc = workspace(device, stream, blocks, &partials, &counter);
  if (rc) return rc;

  EPParams P;
  init_params(P, seed, a, pair_begin);
  P.npairs = npairs;
  const uint64_t T = uint64_t(blocks) * threads;
  P.base = npairs / T;
  P.extra = npairs % T;
  P.table = tab;
  P.partials = partials;
  P.counter = counter;
  P.out13 = dev_out13;
  if (comm) P.comm = *comm;

  const bool a32 = (a >> 32) == 0;
  pick_kernel(cfg.variant, a32, threads)<<<blocks, threads, smem, stream>>>(P);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, "ep_kernel launch");
  {
    std::lock_guard<std::mutex> lk(g_mu);
    ++g_launches;
  }
  return 0;
}

// hpl_shutdown(): free the log tables and EP workspaces of every device
// (each device synchronised first); they are re-created on the next call.
int release_ep_state() {
  std::lock_guard<std::mutex> lk(g_mu);
  int prev = -1;
  cudaGetDevice(&prev);
  cudaError_t first = cudaSuccess;
  for (auto& w : g_ws) {
    cudaSetDevice(w.device);
    cudaError_t e = cudaStreamSynchronize(w.stream);
    if (e != cudaSuccess && first == cudaSuccess) first = e;
    cudaFree(w.partials);
    cudaFree(w.counter);
  }
  g_ws.clear();
  for (size_t d = 0; d < g_dev.size(); ++d)
    if (g_dev[d].table) {
      cudaSetDevice(int(d));
      cudaDeviceSynchronize();
      cudaFree(g_dev[d].table);
      g_dev[d].table = nullptr;
    }
  if (prev >= 0) cudaSetDevice(prev);
  return first == cudaSuccess ? 0 : set_cuda_error(first, "hpl_shutdown: synchronize");
}

unsigned long long launch_count() {
  std::lock_guard<std::mutex> lk(g_mu);
  return g_launches;
}

int launch_pairs_debug(int device, uint64_t seed, uint64_t a, uint64_t pair_begin, uint64_t n,
                       double* dev_out, cudaStream_t stream) {
  const LogEntry* tab;
  int sms;
  int rc = device_state(device, &tab, &sms);
  if (rc) return rc;
  EPParams P;
  init_params(P, seed, a, pair_begin);
  P.table = tab;
  const int smem = int(LOG_TAB * sizeof(LogEntry));
  const bool a32 = (a >> 32) == 0;
  auto k = a32 ? ep_pairs_debug_kernel<true> : ep_pairs_debug_kernel<false>;
  cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return set_cuda_error(e, "cudaFuncSetAttribute(debug)");
  const uint64_t blocks = (n + 255) / 256;
  if (blocks == 0) return 0;
  k<<<unsigned(blocks), 256, smem, stream>>>(P, n, dev_out);
  e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, "ep_pairs_debug_kernel launch");
  return 0;
}

int launch_lcg_states(uint64_t seed, uint64_t a, uint64_t offset, uint64_t n, uint64_t* dev_out,
                      cudaStream_t stream) {
  JumpTable J;
  build_jump_table(a, J.j);
  const int thr = 256;
  const uint64_t blocks = (n + thr - 1) / thr;
  if (blocks == 0) return 0;
  if ((a >> 32) == 0)
    lcg_states_kernel<true><<<unsigned(blocks), thr, 0, stream>>>(seed & MASK46, a, offset, n, J, dev_out);
  else
    lcg_states_kernel<false><<<unsigned(blocks), thr, 0, stream>>>(seed & MASK46, a, offset, n, J, dev_out);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_cuda_error(e, "lcg_states_kernel launch");
  return 0;
}

}  // namespace hplep
