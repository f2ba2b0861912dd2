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
//               reciprocal: q0 = RN(num*r); rem = num - q0*d (exact by FMA);
//               q = RN(q0 + rem*r).  Equals RN(num/d) whenever num and the
//               quotient are normal numbers away from overflow (DESIGN.md
//               section 5); 3 instructions;
//   2 "fast"  : num * r (one rounding more; <= 1 ulp from num / d).
#ifndef DFG_DIV_MODE
#define DFG_DIV_MODE 1
#endif
DFG_DEVICE float dfg_grad1(float fp, float fm, float d, float r) {
  float num = __fsub_rn(fp, fm);
#if DFG_DIV_MODE == 0
  (void)r;
  return __fdiv_rn(num, d);
#elif DFG_DIV_MODE == 1
  float q0 = __fmul_rn(num, r);
  float rem = __fmaf_rn(-q0, d, num);
  return __fmaf_rn(rem, r, q0);
#else
  (void)d;
  return __fmul_rn(num, r);
#endif
}
DFG_DEVICE double dfg_grad1(double fp, double fm, double d, double r) {
  double num = __dsub_rn(fp, fm);
#if DFG_DIV_MODE == 0
  (void)r;
  return __ddiv_rn(num, d);
#elif DFG_DIV_MODE == 1
  double q0 = __dmul_rn(num, r);
  double rem = __fma_rn(-q0, d, num);
  return __fma_rn(rem, r, q0);
#else
  (void)d;
  return __dmul_rn(num, r);
#endif
}
