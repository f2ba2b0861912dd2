// Two-operation exact quotient for a divisor known in advance: host checks.
//
// The fused kernels form a grad3d derivative (reading R1:
// num / d with d the neighbour-centre distance) as
//     q = RN(num * r + RN(num * yl)),  r = RN(1/d),  yl = RN(1/d - r)
// (Brisebarre, Muller and Raina's scheme), two FMA-pipe operations instead
// of Markstein's three.  q equals RN(num / d) for most divisors but not all
// (about 1 % of random fp32 significands fail), so an axis uses the scheme
// only when every divisor of its table is certified.  DESIGN.md section 5.
//
// certify_div2<T>: certification by candidates, for float and double.
//   Error bound (proof).  u = 2^-p.  r = RN(1/d) gives |r - 1/d| <= u/d
//   (|RN(y) - y| <= ulp(y)/2 <= u |y|).  The remainder e = fma(-r, d, 1) =
//   1 - r d is exact (Markstein), so tau = 1/d - r = e/d exactly and
//   yl = RN(e/d) = RN(tau) with |yl - tau| <= u |tau| (tau normal; if
//   yl == 0 we require e == 0, i.e. tau == 0).  Let L = RN(x yl):
//   |L - x yl| <= u |x yl| (x yl normal).  The FMA rounds v = x r + L once,
//   and x/d = x r + x tau, so
//       v - x/d = (L - x yl) + x (yl - tau),
//       |v - x/d| <= u |x| (|yl| + |tau|) <= u (2 + u) |x| |tau|
//                 <= (2 + u) 2^-2p |x/d|.
//   Scale to significands: d = B 2^(e-p), x = A 2^(e-p), B, A in [2^(p-1),
//   2^p) (every quantity scales exactly by powers of two while the products
//   stay normal), q* = x/d = A/B in (1/2, 2).  RN(v) != RN(q*) needs a
//   rounding midpoint m between v and q* (q* itself is never a midpoint;
//   v == m is covered since |q* - m| <= |v - q*| then):
//     q* in [1, 2):   m = N 2^-p,     N odd:  |2^p A - N B| <= (2+u) 2^-p A < 2 + u
//     q* in [1/2, 1): m = N 2^-(p+1), N odd:  |2^(p+1) A - N B| < 4 + 2u
//   (A < 2^p), i.e. k = 2^s A - N B is a nonzero integer with |k| <= 2
//   (s = p) or |k| <= 4 (s = p + 1); the binade ends are out of reach
//   (q* >= 1/2 + 2^-(p+1) - and <= 2 - 2^(1-p), far beyond the error).  For
//   each k with |k| <= W (W = 16 > 4) the congruence N B = -k (mod 2^s)
//   fixes N modulo 2^(s-t) (t = trailing zero bits of B); every N in
//   (2^p, 2^(p+1)) is enumerated and gives the numerator A = (N B + k) / 2^s.
//   So the candidates contain EVERY numerator at which the scheme can
//   differ from RN(x/d): the divisor is certified when the scheme matches
//   IEEE division at each of them (and, for margin, its two neighbours).  A
//   divisor with more than log2(W) trailing zero bits has no candidate at
//   all: such divisors (the RT meshes' spacings, differences of nearby
//   coordinates) always pass.  tests/test_lib_host.py pins the bound with
//   exact rational arithmetic on random fp64 operands and the whole method
//   against exhaustive fp32 enumeration.
//   Preconditions checked here: r == RN(1/d) and yl == RN(1/d - r) formed
//   as RN(e / d); d, r, yl normal, or yl == 0 with e == 0.

// exhaustive_div2_f32: the exhaustive definition for fp32 (all 2^23
// significands), on the host; the device version (kern::verify_div2) decides
// fp32 meshes, this one exists to validate certify_div2.
#pragma once

#include <cmath>
#include <cstdint>
#include <cstring>
#include <limits>

namespace dfg {

template <typename T>
inline T div2_low_part(T d, T r) {
  const T e = std::fma(-r, d, T(1));  // exact: 1 - r d
  return e / d;                       // RN((1 - r d) / d) = RN(1/d - r)
}

template <typename T>
bool certify_div2(T d, T r, T yl, int W = 16, long* tested = nullptr) {
  typedef unsigned __int128 u128;
  typedef __int128 i128;
  const int p = std::numeric_limits<T>::digits;
  long cnt = 0;
  if (tested) *tested = 0;
  if (!(d > T(0)) || !std::isnormal(d) || !std::isnormal(r)) return false;
  if (r != T(1) / d || yl != div2_low_part(d, r)) return false;
  if (yl != T(0) && !std::isnormal(yl)) return false;
  if (yl == T(0) && std::fma(-r, d, T(1)) != T(0)) return false;  // tau != 0 lost to underflow
  int ed = 0;
  const T md = std::frexp(d, &ed);                  // d = md 2^ed, md in [1/2, 1)
  const uint64_t B = uint64_t(std::ldexp(md, p));   // d = B 2^(ed - p)
  int t = 0;
  while (((B >> t) & 1u) == 0) ++t;
  const u128 Bo = u128(B >> t);
  auto passes = [&](u128 A) {
    if (A < (u128(1) << (p - 1)) || A >= (u128(1) << p)) return true;
    ++cnt;
    const T x = std::ldexp(T(uint64_t(A)), ed - p);  // x / d = A / B
    const T lo = x * yl;                             // rounded on its own (-ffp-contract=off)
    return std::fma(x, r, lo) == x / d;
  };
  bool ok = true;
  for (int s = p; s <= p + 1 && ok; ++s) {
    const int m = s - t;  // N Bo = -(k / 2^t) (mod 2^m)
    const u128 mod = u128(1) << m, mask = mod - 1;
    u128 inv = Bo;        // Bo^-1 mod 2^128 (Newton: correct bits double per step)
    for (int i = 0; i < 7; ++i) inv = inv * (2 - Bo * inv);
    for (int k = -W; k <= W && ok; ++k) {
      if (k == 0) continue;
      const long ak = k < 0 ? -k : k;
      if (t >= 62 || ak % (1L << t) != 0) continue;  // 2^t divides N B - 2^s A
      const long kp = k / (1L << t);
      const u128 N0 = ((u128(0) - u128(i128(kp))) * inv) & mask;
      if ((N0 & 1u) == 0) continue;                  // midpoints have odd N
      const u128 lo = u128(1) << p, hi = u128(1) << (p + 1);
      u128 N = N0;
      if (N < lo) N += ((lo - N + mod - 1) / mod) * mod;
      for (; N < hi && ok; N += mod) {
        const i128 num = i128(N) * i128(B) + k;     // = 2^s A
        if (num <= 0 || (num & ((i128(1) << s) - 1)) != 0) continue;
        const u128 A = u128(num >> s);
        ok = passes(A - 1) && passes(A) && passes(A + 1);
      }
    }
  }
  if (tested) *tested = cnt;
  return ok;
}

inline bool exhaustive_div2_f32(float d, float r, float yl) {
  for (uint32_t m = 0; m < (1u << 23); ++m) {
    const uint32_t u = 0x3f800000u | m;
    float a;
    std::memcpy(&a, &u, 4);
    const float lo = a * yl;
    if (std::fma(a, r, lo) != a / d) return false;
  }
  return true;
}

}  // namespace dfg
