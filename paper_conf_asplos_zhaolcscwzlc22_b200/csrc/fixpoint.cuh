// Deterministic per-channel reductions in 64-bit fixed point (SPOS BatchNorm, spos.cu and
// the GEMM epilogue's fused statistics, gemm.cu).
//
// Every producer reduces its share of the rows in a fixed order to fp32 partials, converts
// them to 64-bit fixed point and adds them with integer atomics into an accumulator
// acc[0 .. 2C) (sum and second sum per channel).  Integer addition is associative, so the
// totals -- and everything computed from them -- are bitwise independent of the order in
// which CTAs arrive: no float atomics, no finalize launch.  acc[2C] is a sticky overflow
// flag: a partial outside the fixed-point range sets it instead of wrapping silently; the
// engine checks it at drain.
//
// Scales: forward sum z 2^32 (|sum| < 2^31), sum z^2 2^24 (< 5.5e11), backward sums 2^40
// (|sum| < 8.4e6); the resolution (2^-32, 2^-24, 2^-40) is far below the fp32 partials'.
#pragma once
#include <cstdint>

namespace naspipe {

constexpr double FIX_S1 = 4294967296.0;    // 2^32
constexpr double FIX_S2 = 16777216.0;      // 2^24
constexpr double FIX_B = 1099511627776.0;  // 2^40

// acc[i] += v * scale (fixed point); flag = &acc[2C]
__device__ __forceinline__ void fix_add(unsigned long long* acc, int i, unsigned long long* flag, float v,
                                        double scale) {
  const double x = (double)v * scale;
  if (!(fabs(x) < 4.0e18)) {  // also catches NaN
    atomicOr(flag, 1ull);
    return;
  }
  atomicAdd(acc + i, (unsigned long long)(long long)__double2ll_rn(x));
}
__device__ __forceinline__ double fix_get(const unsigned long long* acc, int i, double scale) {
  return (double)(long long)acc[i] / scale;
}

}  // namespace naspipe
