// Hand-written "reference kernels" ("reference OpenCL kernels
// written for each of the three vortex detection expressions ... able to
// execute the expressions using less memory fetches and floating point
// operations than our strategies").  Each body plugs into the same fused
// skeletons as the generated networks (same I/O, same TMA pipeline), but is
// written directly from the mathematics instead of from the network:
// derivatives as numerator x reciprocal spacing (one rounding more than the
// network's division), FMA contraction, and for Q the identity
//   Q = 1/2 (||Omega||^2 - ||S||^2) = -1/2 tr(J J)
//     = -1/2 (J00^2 + J11^2 + J22^2) - (J01 J10 + J02 J20 + J12 J21)
// (Eq. 2-3).  Results agree with the oracle within the
// floating-point tolerance, not bit for bit.
//
// Field slots: stencil inputs u, v, w are s[0..2] / gn[0..2] (VortMag, Q);
// VelMag reads them point-wise as p[0..2].  DFG_REF selects the body.

#if DFG_PAIRS_F32
__device__ __forceinline__ dfg2 ref_mul(dfg2 a, dfg2 b) { return __fmul2_rn(a, b); }
__device__ __forceinline__ dfg2 ref_fma(dfg2 a, dfg2 b, dfg2 c) { return __ffma2_rn(a, b, c); }
__device__ __forceinline__ dfg2 ref_sqrt(dfg2 a) { return make_float2(__fsqrt_rn(a.x), __fsqrt_rn(a.y)); }
__device__ __forceinline__ dfg2 ref_sub(dfg2 a, dfg2 b) { return __ffma2_rn(b, make_float2(-1.0f, -1.0f), a); }
#else
__device__ __forceinline__ dfg2 ref_mul(dfg2 a, dfg2 b) { return a * b; }
__device__ __forceinline__ dfg2 ref_fma(dfg2 a, dfg2 b, dfg2 c) { return __fma_rn(a, b, c); }
__device__ __forceinline__ dfg2 ref_sqrt(dfg2 a) { return __dsqrt_rn(a); }
__device__ __forceinline__ dfg2 ref_sub(dfg2 a, dfg2 b) { return a - b; }
#endif

__device__ __forceinline__ void dfg_body(const dfg2 (&s)[DFG_NSF_][7], const dfg2 (&gn)[DFG_NSF_][3],
                                         const dfg2 (&p)[DFG_NPF_], const dfg2 ndx, const dfg2 rx,
                                         const dfg2 ndy, const dfg2 ry, const dfg2 ndz, const dfg2 rz,
                                         const dfg2 Z, dfg2 (&o)[DFG_OUTW]) {
  (void)s; (void)gn; (void)p; (void)ndx; (void)rx; (void)ndy; (void)ry; (void)ndz; (void)rz; (void)Z;
#if DFG_REF == 1
  // velocity magnitude |v| = sqrt(u^2 + v^2 + w^2)
  o[0] = ref_sqrt(ref_fma(p[2], p[2], ref_fma(p[1], p[1], ref_mul(p[0], p[0]))));
#elif DFG_REF == 2
  // vorticity magnitude |curl v| (Eq. 1)
  const dfg2 dwdy = ref_mul(gn[2][1], ry), dvdz = ref_mul(gn[1][2], rz);
  const dfg2 dudz = ref_mul(gn[0][2], rz), dwdx = ref_mul(gn[2][0], rx);
  const dfg2 dvdx = ref_mul(gn[1][0], rx), dudy = ref_mul(gn[0][1], ry);
  const dfg2 wx = ref_sub(dwdy, dvdz), wy = ref_sub(dudz, dwdx), wz = ref_sub(dvdx, dudy);
  o[0] = ref_sqrt(ref_fma(wz, wz, ref_fma(wy, wy, ref_mul(wx, wx))));
#elif DFG_REF == 3
  // Q-criterion, Q = -1/2 tr(J^2) with J_ij = d u_i / d x_j
  const dfg2 J00 = ref_mul(gn[0][0], rx), J01 = ref_mul(gn[0][1], ry), J02 = ref_mul(gn[0][2], rz);
  const dfg2 J10 = ref_mul(gn[1][0], rx), J11 = ref_mul(gn[1][1], ry), J12 = ref_mul(gn[1][2], rz);
  const dfg2 J20 = ref_mul(gn[2][0], rx), J21 = ref_mul(gn[2][1], ry), J22 = ref_mul(gn[2][2], rz);
  const dfg2 diag = ref_fma(J22, J22, ref_fma(J11, J11, ref_mul(J00, J00)));
  const dfg2 cross = ref_fma(J12, J21, ref_fma(J02, J20, ref_mul(J01, J10)));
  const dfg2 mhalf = dfg2_splat(DFG_T(-0.5));
  o[0] = ref_fma(mhalf, diag, ref_sub(dfg2_splat(DFG_T(0)), cross));
#endif
}
