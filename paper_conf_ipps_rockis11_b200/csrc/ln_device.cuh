// ln_device.cuh — correctly rounded ln(x) for integer x on the device
// (DESIGN.md §3 reading R9: lnT[k] = RN(ln(k * unit))).
//
// Double-double arithmetic built only from IEEE round-to-nearest intrinsics
// (__dadd_rn, __dmul_rn, __ddiv_rn, __fma_rn), so nothing depends on FMA
// contraction or on the 1-ulp CUDA log():
//   x = 2^e * m, m in [sqrt(1/2), sqrt(2)]
//   ln m = 2 atanh(s), s = (m - 1) / (m + 1), atanh(s) = s * sum_j s^(2j) / (2j+1)
//   ln x = e * ln2 + ln m            (ln2 as a double-double constant)
// Error ~2^-100 relative, far below the 2^-68 distance of the hardest cases
// (ln 9170 is 2e-5 ulp from a rounding midpoint), so hi + lo rounds correctly.
#pragma once
#include <cstdint>

namespace mcts_dev {

struct dd { double hi, lo; };

__device__ __forceinline__ dd dd_two_sum(double a, double b) {
  double s = __dadd_rn(a, b);
  double bb = __dadd_rn(s, -a);
  double err = __dadd_rn(__dadd_rn(a, -__dadd_rn(s, -bb)), __dadd_rn(b, -bb));
  return {s, err};
}

__device__ __forceinline__ dd dd_fast_two_sum(double a, double b) {  // |a| >= |b|
  double s = __dadd_rn(a, b);
  return {s, __dadd_rn(b, -__dadd_rn(s, -a))};
}

__device__ __forceinline__ dd dd_two_prod(double a, double b) {
  double p = __dmul_rn(a, b);
  return {p, __fma_rn(a, b, -p)};
}

__device__ __forceinline__ dd dd_add(dd a, dd b) {
  dd s = dd_two_sum(a.hi, b.hi);
  dd t = dd_two_sum(a.lo, b.lo);
  s.lo = __dadd_rn(s.lo, t.hi);
  s = dd_fast_two_sum(s.hi, s.lo);
  s.lo = __dadd_rn(s.lo, t.lo);
  return dd_fast_two_sum(s.hi, s.lo);
}

__device__ __forceinline__ dd dd_mul(dd a, dd b) {
  dd p = dd_two_prod(a.hi, b.hi);
  double cross = __dadd_rn(__dmul_rn(a.hi, b.lo), __dmul_rn(a.lo, b.hi));
  p.lo = __dadd_rn(p.lo, cross);
  return dd_fast_two_sum(p.hi, p.lo);
}

// a / b for double-doubles: two quotient digits plus a correction.
__device__ __forceinline__ dd dd_div(dd a, dd b) {
  double q1 = __ddiv_rn(a.hi, b.hi);
  dd r = dd_add(a, {-dd_mul({q1, 0.0}, b).hi, -dd_mul({q1, 0.0}, b).lo});
  double q2 = __ddiv_rn(r.hi, b.hi);
  dd q2b = dd_mul({q2, 0.0}, b);
  r = dd_add(r, {-q2b.hi, -q2b.lo});
  double q3 = __ddiv_rn(r.hi, b.hi);
  dd q = dd_fast_two_sum(q1, q2);
  return dd_add(q, {q3, 0.0});
}

// RN(ln(x)) for 1 <= x < 2^53.
__device__ __forceinline__ double ln_rn(unsigned long long x) {
  if (x <= 1ULL) return 0.0;
  const double xd = (double)x;  // exact
  int e;
  double m = frexp(xd, &e);      // xd = m * 2^e, m in [0.5, 1), exact
  m = __dmul_rn(m, 2.0);
  e -= 1;                        // m in [1, 2)
  if (m > 1.4142135623730951) {  // move to [sqrt(1/2), sqrt(2)]
    m = __dmul_rn(m, 0.5);
    e += 1;
  }
  const dd ln2 = {0x1.62e42fefa39efp-1, 0x1.abc9e3b39803fp-56};
  dd el2 = dd_two_prod((double)e, ln2.hi);
  el2.lo = __dadd_rn(el2.lo, __dmul_rn((double)e, ln2.lo));
  el2 = dd_fast_two_sum(el2.hi, el2.lo);
  if (m == 1.0) return __dadd_rn(el2.hi, el2.lo);

  const double num = __dadd_rn(m, -1.0);      // exact (Sterbenz)
  const dd den = dd_two_sum(m, 1.0);
  const dd s = dd_div({num, 0.0}, den);
  const dd t = dd_mul(s, s);                   // s^2 <= 0.0295
  // Horner: P(t) = sum_{j=0}^{N} t^j / (2j+1), N = 24 (t^25/51 < 2^-130).
  const int N = 24;
  dd acc = dd_div({1.0, 0.0}, {(double)(2 * N + 1), 0.0});
  for (int j = N - 1; j >= 0; --j) {
    acc = dd_mul(acc, t);
    acc = dd_add(acc, dd_div({1.0, 0.0}, {(double)(2 * j + 1), 0.0}));
  }
  dd lnm = dd_mul(s, acc);
  lnm.hi = __dmul_rn(lnm.hi, 2.0);
  lnm.lo = __dmul_rn(lnm.lo, 2.0);
  const dd r = dd_add(el2, lnm);
  return __dadd_rn(r.hi, r.lo);
}

}  // namespace mcts_dev
