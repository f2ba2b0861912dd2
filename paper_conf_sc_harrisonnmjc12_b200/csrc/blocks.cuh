// dfg building blocks: the primitives of PAPER.md L86 ("small ... functions
// ... written once and shared by all execution strategies"), as sm_100a
// __device__ functions.  Included by the precompiled per-primitive kernels
// (kernels.cu: roundtrip + staged) and pasted into every generated fused
// kernel (codegen.cpp -> NVRTC), so the three strategies run the same
// arithmetic instruction for instruction.
//
// Rounding: every block is one IEEE operation rounded to T with the
// explicit _rn intrinsics, so neither nvcc nor NVRTC may contract or
// reassociate across blocks (reading R6).  This header must compile both
// under nvcc and under NVRTC: no #include, builtins only.
#pragma once

#ifndef DFG_DEVICE
#define DFG_DEVICE __device__ __forceinline__
#endif

// --- arithmetic (add, sub, mult, sqrt: L86; div, neg: reading R3) --------
DFG_DEVICE float dfg_add(float a, float b) { return __fadd_rn(a, b); }
DFG_DEVICE double dfg_add(double a, double b) { return __dadd_rn(a, b); }
DFG_DEVICE float dfg_sub(float a, float b) { return __fsub_rn(a, b); }
DFG_DEVICE double dfg_sub(double a, double b) { return __dsub_rn(a, b); }
DFG_DEVICE float dfg_mult(float a, float b) { return __fmul_rn(a, b); }
DFG_DEVICE double dfg_mult(double a, double b) { return __dmul_rn(a, b); }
DFG_DEVICE float dfg_div(float a, float b) { return __fdiv_rn(a, b); }
DFG_DEVICE double dfg_div(double a, double b) { return __ddiv_rn(a, b); }
DFG_DEVICE float dfg_neg(float a) { return -a; }
DFG_DEVICE double dfg_neg(double a) { return -a; }
DFG_DEVICE float dfg_sqrt(float a) { return __fsqrt_rn(a); }
DFG_DEVICE double dfg_sqrt(double a) { return __dsqrt_rn(a); }

// --- comparisons -> T(1)/T(0), NaN compares false; select (intro L19, R7) -
#define DFG_CMP(name, op)                                                        \
  DFG_DEVICE float name(float a, float b) { return (a op b) ? 1.0f : 0.0f; }     \
  DFG_DEVICE double name(double a, double b) { return (a op b) ? 1.0 : 0.0; }
DFG_CMP(dfg_gt, >)
DFG_CMP(dfg_lt, <)
DFG_CMP(dfg_ge, >=)
DFG_CMP(dfg_le, <=)
DFG_CMP(dfg_eq, ==)
DFG_CMP(dfg_ne, !=)
#undef DFG_CMP
DFG_DEVICE float dfg_select(float c, float a, float b) { return (c != 0.0f) ? a : b; }
DFG_DEVICE double dfg_select(double c, double a, double b) { return (c != 0.0) ? a : b; }

// --- grad3d, one axis (reading R1) -------------------------------------
// d f/d axis at cell i = (f[ip] - f[im]) / (c[ip] - c[im]) with
// ip = min(i+1, n-1), im = max(i-1, 0); the caller passes the clamped
// neighbour values fp = f[ip], fm = f[im] and the per-cell table entries
//   d = c[ip] - c[im]   (computed in T exactly as the definition says)
//   r = RN(1 / d)        (correctly rounded reciprocal)
// DFG_DIV_MODE selects how the quotient is formed:
//   0 "ieee"  : IEEE division num / d (div.rn; ~8-10 SASS instructions);
//   1 "exact" : Markstein's correction with the correctly rounded
//               reciprocal: q0 = RN(num*r); t = q0*d - num (exact by FMA);
//               q = RN(q0 - t*r).  Equals RN(num/d) whenever num and the
//               quotient are normal numbers away from overflow (DESIGN.md
//               section 5); 3 instructions.  The correction is formed as
//               -t rather than num - q0*d so that a zero numerator keeps its
//               sign: for num = -0, t = RN(-0*d + +0) = +0 and
//               q = RN(-0 + -0) = -0 (num - q0*d would give +0 + -0 = +0);
//   2 "fast"  : num * r (one rounding more; <= 1 ulp from num / d).
#ifndef DFG_DIV_MODE
#define DFG_DIV_MODE 1
#endif
// Spacing table of an axis: d[n] | r[n] | -d[n] | yl[n].  The fused kernels
// pass segment DFG_NDSEG_<axis> as the first table operand of the quotient:
// -d for the correction, yl for the two-operation form (DFG_DIV2_<axis>).
#ifndef DFG_DIV2_X
#define DFG_DIV2_X 0
#endif
#ifndef DFG_DIV2_Y
#define DFG_DIV2_Y 0
#endif
#ifndef DFG_DIV2_Z
#define DFG_DIV2_Z 0
#endif
#define DFG_NDSEG_X (DFG_DIV2_X ? 3 : 2)
#define DFG_NDSEG_Y (DFG_DIV2_Y ? 3 : 2)
#define DFG_NDSEG_Z (DFG_DIV2_Z ? 3 : 2)
DFG_DEVICE float dfg_grad1q(float num, float d, float r) {
#if DFG_DIV_MODE == 0
  (void)r;
  return __fdiv_rn(num, d);
#elif DFG_DIV_MODE == 1
  float q0 = __fmul_rn(num, r);
  float t = __fmaf_rn(q0, d, -num);
  return __fmaf_rn(-t, r, q0);
#else
  (void)d;
  return __fmul_rn(num, r);
#endif
}
DFG_DEVICE double dfg_grad1q(double num, double d, double r) {
#if DFG_DIV_MODE == 0
  (void)r;
  return __ddiv_rn(num, d);
#elif DFG_DIV_MODE == 1
  double q0 = __dmul_rn(num, r);
  double t = __fma_rn(q0, d, -num);
  return __fma_rn(-t, r, q0);
#else
  (void)d;
  return __dmul_rn(num, r);
#endif
}
DFG_DEVICE float dfg_grad1(float fp, float fm, float d, float r) {
  float num = __fsub_rn(fp, fm);
  return dfg_grad1q(num, d, r);
}
DFG_DEVICE double dfg_grad1(double fp, double fm, double d, double r) {
  double num = __dsub_rn(fp, fm);
  return dfg_grad1q(num, d, r);
}

// --- paired blocks: two cells per instruction ------------------------------
// sm_100 executes FADD2 / FMUL2 / FFMA2 on float2 register pairs.  The fused
// kernels evaluate the network on pairs of cells (float2 for T = float; for
// T = double a "pair" is one double and the blocks are the scalar ones).
// Contraction guard: ptxas contracts f32x2 multiply -> add sequences into
// FFMA2 even with .rn and --fmad=false, which would change the rounding.
// Products are therefore formed as fma(a, b, Z) with Z = (-0, -0) passed in
// at run time (opaque to the compiler): RN(a*b + -0) == RN(a*b) for every a,
// b (including signed zeros, Inf and NaN), and an FFMA2 feeding an add can
// not be contracted further.
#if defined(DFG_PAIRS)
#if DFG_PAIRS_F32
typedef float2 dfg2;
DFG_DEVICE dfg2 dfg2_splat(float a) { return make_float2(a, a); }
DFG_DEVICE dfg2 dfg2_add(dfg2 a, dfg2 b, dfg2) { return __fadd2_rn(a, b); }
DFG_DEVICE dfg2 dfg2_sub(dfg2 a, dfg2 b, dfg2) { return __ffma2_rn(b, make_float2(-1.0f, -1.0f), a); }
DFG_DEVICE dfg2 dfg2_mult(dfg2 a, dfg2 b, dfg2 z) { return __ffma2_rn(a, b, z); }
DFG_DEVICE dfg2 dfg2_neg(dfg2 a, dfg2 z) { return __ffma2_rn(a, make_float2(-1.0f, -1.0f), z); }
// RN(b + c*a) for a power of two c (scale folding: c*a is exact, one rounding)
DFG_DEVICE dfg2 dfg2_axpy(dfg2 a, float c, dfg2 b) { return __ffma2_rn(a, make_float2(c, c), b); }
#define DFG2_LANEWISE1(name, f) \
  DFG_DEVICE dfg2 name(dfg2 a, dfg2) { return make_float2(f(a.x), f(a.y)); }
#define DFG2_LANEWISE2(name, f) \
  DFG_DEVICE dfg2 name(dfg2 a, dfg2 b, dfg2) { return make_float2(f(a.x, b.x), f(a.y, b.y)); }
DFG2_LANEWISE1(dfg2_sqrt, dfg_sqrt)
DFG2_LANEWISE2(dfg2_div, dfg_div)
DFG2_LANEWISE2(dfg2_gt, dfg_gt)
DFG2_LANEWISE2(dfg2_lt, dfg_lt)
DFG2_LANEWISE2(dfg2_ge, dfg_ge)
DFG2_LANEWISE2(dfg2_le, dfg_le)
DFG2_LANEWISE2(dfg2_eq, dfg_eq)
DFG2_LANEWISE2(dfg2_ne, dfg_ne)
DFG_DEVICE dfg2 dfg2_select(dfg2 c, dfg2 a, dfg2 b, dfg2) {
  return make_float2(dfg_select(c.x, a.x, b.x), dfg_select(c.y, a.y, b.y));
}
// grad3d quotient on a pair, num = f[ip] - f[im] already formed; nd = -d
// (the tables carry the exact negation so the correction is one FFMA2)
DFG_DEVICE dfg2 dfg2_gradq(dfg2 num, dfg2 nd, dfg2 r, dfg2 z) {
#if DFG_DIV_MODE == 0
  return make_float2(__fdiv_rn(num.x, -nd.x), __fdiv_rn(num.y, -nd.y));
#elif DFG_DIV_MODE == 1
  const dfg2 q0 = __ffma2_rn(num, r, z);                                                 // RN(num * r)
  const dfg2 t = __ffma2_rn(make_float2(-q0.x, -q0.y), nd, make_float2(-num.x, -num.y));  // q0*d - num, exact
  return __ffma2_rn(t, make_float2(-r.x, -r.y), q0);                                     // RN(q0 - t*r)
#else
  return __ffma2_rn(num, r, z);
#endif
}
// Two-operation exact quotient for a divisor known in advance (Brisebarre,
// Muller and Raina's scheme): yh = r = RN(1/d), yl ~ 1/d - yh, and
//   q = RN(num*yh + RN(num*yl)).
// It is not RN(num/d) for every divisor, so the runtime checks each divisor
// of an axis against IEEE division for all 2^23 significands (kern::
// verify_div2) and emits this block only for axes that passed: there it is
// RN(num/d) under the same normal-range conditions as the correction above.
DFG_DEVICE dfg2 dfg2_gradq2(dfg2 num, dfg2 yl, dfg2 yh, dfg2 z) {
  return __ffma2_rn(num, yh, __ffma2_rn(num, yl, z));
}
#else   // T = double: one cell per "pair", scalar blocks
typedef double dfg2;
DFG_DEVICE dfg2 dfg2_splat(double a) { return a; }
DFG_DEVICE dfg2 dfg2_add(dfg2 a, dfg2 b, dfg2) { return dfg_add(a, b); }
DFG_DEVICE dfg2 dfg2_sub(dfg2 a, dfg2 b, dfg2) { return dfg_sub(a, b); }
DFG_DEVICE dfg2 dfg2_mult(dfg2 a, dfg2 b, dfg2) { return dfg_mult(a, b); }
DFG_DEVICE dfg2 dfg2_neg(dfg2 a, dfg2) { return dfg_neg(a); }
DFG_DEVICE dfg2 dfg2_axpy(dfg2 a, double c, dfg2 b) { return __fma_rn(a, c, b); }
DFG_DEVICE dfg2 dfg2_sqrt(dfg2 a, dfg2) { return dfg_sqrt(a); }
DFG_DEVICE dfg2 dfg2_div(dfg2 a, dfg2 b, dfg2) { return dfg_div(a, b); }
DFG_DEVICE dfg2 dfg2_gt(dfg2 a, dfg2 b, dfg2) { return dfg_gt(a, b); }
DFG_DEVICE dfg2 dfg2_lt(dfg2 a, dfg2 b, dfg2) { return dfg_lt(a, b); }
DFG_DEVICE dfg2 dfg2_ge(dfg2 a, dfg2 b, dfg2) { return dfg_ge(a, b); }
DFG_DEVICE dfg2 dfg2_le(dfg2 a, dfg2 b, dfg2) { return dfg_le(a, b); }
DFG_DEVICE dfg2 dfg2_eq(dfg2 a, dfg2 b, dfg2) { return dfg_eq(a, b); }
DFG_DEVICE dfg2 dfg2_ne(dfg2 a, dfg2 b, dfg2) { return dfg_ne(a, b); }
DFG_DEVICE dfg2 dfg2_select(dfg2 c, dfg2 a, dfg2 b, dfg2) { return dfg_select(c, a, b); }
DFG_DEVICE dfg2 dfg2_gradq(dfg2 num, dfg2 nd, dfg2 r, dfg2) { return dfg_grad1q(num, -nd, r); }
// two-operation quotient (fp64 axes certified by candidates, div2.hpp)
DFG_DEVICE dfg2 dfg2_gradq2(dfg2 num, dfg2 yl, dfg2 yh, dfg2) { return __fma_rn(num, yh, __dmul_rn(num, yl)); }
#endif
#endif  // DFG_PAIRS
