// dfg fused-kernel skeletons (the "fusion" strategy).
//
// Compiled by NVRTC (sm_100a) after the generated prologue, which defines
//   DFG_T, DFG_VEC (16 B / sizeof T), DFG_NSF (stencil fields: read by a
//   grad3d), DFG_NPF (fields read only at the cell itself), DFG_OUTW (1 or
//   4), DFG_NCW (consumer warps = tile rows), DFG_STAGES (smem ring depth),
//   DFG_XDEG/YDEG/ZDEG, DFG_HAS_TMA, DFG_DIV_MODE
// and the per-expression body
//   dfg_body(s, p, dx, rx, dy, ry, dz, rz, o)
// where s[f][0..6] are stencil field f at the cell, x-1, x+1, y-1, y+1, z-1,
// z+1 (already clamped at the global mesh ends), p[f] the point-wise
// fields, (d*, r*) the spacing-table entries of the cell (reading R1), and
// o[] the result lanes.  The body is the whole network with intermediates in
// registers (L97); the skeletons only move data.
//
// Kernels:
//   dfg_fused_pointwise -- networks without grad3d: flat, 16-byte I/O.
//   dfg_fused_general   -- any layout: one cell per thread, clamped direct
//                          loads (ragged nx, unaligned buffers).
//   dfg_fused_tma       -- the B200 path: persistent CTAs march z-columns of
//                          (32*VEC) x DFG_NCW cells; one producer warp streams
//                          halo'd x-y tiles of every stencil field into a
//                          DFG_STAGES-deep shared-memory ring with TMA
//                          (cp.async.bulk.tensor.3d + mbarrier complete_tx);
//                          consumer warps keep z-1/z/z+1 centres in
//                          registers, read x/y neighbours from shared memory
//                          and write 16-byte streaming stores.

// DFG_NSF_ / DFG_NPF_ / DFG_NF_ (array extents, at least 1) come from the
// generated prologue because the body's signature uses them.

#if DFG_VEC == 4
typedef float4 dfg_v16;
#else
typedef double2 dfg_v16;
#endif

struct DfgParams {
  const DFG_T* f[DFG_NF_];  // fields: base of T[nzl + 2*ghost][ny][nx]
  DFG_T* out;               // T[nzl][ny][nx][DFG_OUTW]
  const DFG_T* tx;          // x table: d[nx] then r[nx]
  const DFG_T* ty;          // y table: d[ny] then r[ny]
  const DFG_T* tz;          // z table over the GLOBAL mesh: d[NZ] then r[NZ]
  long long nx, ny, nzl, NZ, k0, ghost;
  long long kbeg, kend;     // global planes computed by this launch
  long long items;          // TMA: tiles_x * tiles_y * zchunks
  int tiles_x, tiles_y, kz, vec_ok;
};

__device__ __forceinline__ void dfg_ld16(DFG_T (&d)[DFG_VEC], const DFG_T* p) {
  dfg_v16 v = *reinterpret_cast<const dfg_v16*>(p);
#if DFG_VEC == 4
  d[0] = v.x; d[1] = v.y; d[2] = v.z; d[3] = v.w;
#else
  d[0] = v.x; d[1] = v.y;
#endif
}
__device__ __forceinline__ void dfg_ldg16(DFG_T (&d)[DFG_VEC], const DFG_T* p) {
  dfg_v16 v = __ldcs(reinterpret_cast<const dfg_v16*>(p));
#if DFG_VEC == 4
  d[0] = v.x; d[1] = v.y; d[2] = v.z; d[3] = v.w;
#else
  d[0] = v.x; d[1] = v.y;
#endif
}
__device__ __forceinline__ void dfg_stg16(DFG_T* p, const DFG_T* s) {
  dfg_v16 v;
#if DFG_VEC == 4
  v.x = s[0]; v.y = s[1]; v.z = s[2]; v.w = s[3];
#else
  v.x = s[0]; v.y = s[1];
#endif
  __stcs(reinterpret_cast<dfg_v16*>(p), v);
}

#if DFG_NSF == 0
// ----------------------------------------------------------- point-wise
extern "C" __global__ void __launch_bounds__(256) dfg_fused_pointwise(const DfgParams P) {
  const long long plane = P.nx * P.ny;
  const long long n = plane * (P.kend - P.kbeg);
  const long long in_off = (P.kbeg - P.k0 + P.ghost) * plane;
  const long long out_off = (P.kbeg - P.k0) * plane;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const DFG_T sz[DFG_NSF_][7] = {};
  const long long nv = P.vec_ok ? n / DFG_VEC : 0;
  for (long long v = tid; v < nv; v += stride) {
    DFG_T pv[DFG_NPF_][DFG_VEC];
#pragma unroll
    for (int f = 0; f < DFG_NPF; ++f) dfg_ldg16(pv[f], P.f[DFG_NSF + f] + in_off + v * DFG_VEC);
    DFG_T o[DFG_VEC][DFG_OUTW];
#pragma unroll
    for (int c = 0; c < DFG_VEC; ++c) {
      DFG_T p[DFG_NPF_];
#pragma unroll
      for (int f = 0; f < DFG_NPF; ++f) p[f] = pv[f][c];
      dfg_body(sz, p, DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), o[c]);
    }
    DFG_T* dst = P.out + (out_off + v * DFG_VEC) * DFG_OUTW;
#if DFG_OUTW == 1
    DFG_T t[DFG_VEC];
#pragma unroll
    for (int c = 0; c < DFG_VEC; ++c) t[c] = o[c][0];
    dfg_stg16(dst, t);
#else
#pragma unroll
    for (int c = 0; c < DFG_VEC; ++c)
#pragma unroll
      for (int h = 0; h < DFG_OUTW; h += DFG_VEC) dfg_stg16(dst + c * DFG_OUTW + h, &o[c][h]);
#endif
  }
  for (long long c = nv * DFG_VEC + tid; c < n; c += stride) {
    DFG_T p[DFG_NPF_];
#pragma unroll
    for (int f = 0; f < DFG_NPF; ++f) p[f] = P.f[DFG_NSF + f][in_off + c];
    DFG_T o[DFG_OUTW];
    dfg_body(sz, p, DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), DFG_T(0), o);
#pragma unroll
    for (int h = 0; h < DFG_OUTW; ++h) P.out[(out_off + c) * DFG_OUTW + h] = o[h];
  }
}
#endif

#if DFG_NSF > 0
// ------------------------------------------------------------- general
extern "C" __global__ void __launch_bounds__(256) dfg_fused_general(const DfgParams P) {
  const long long plane = P.nx * P.ny;
  const long long total = plane * (P.kend - P.kbeg);
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long c = (long long)blockIdx.x * blockDim.x + threadIdx.x; c < total; c += stride) {
    const long long i = c % P.nx;
    const long long t = c / P.nx;
    const long long j = t % P.ny;
    const long long kg = P.kbeg + t / P.ny;
    const long long kl = kg - P.k0;
    const long long base = (kl + P.ghost) * plane + j * P.nx + i;
    const long long oxm = i > 0 ? 1 : 0, oxp = i < P.nx - 1 ? 1 : 0;
    const long long oym = j > 0 ? P.nx : 0, oyp = j < P.ny - 1 ? P.nx : 0;
    const long long ozm = kg > 0 ? plane : 0, ozp = kg < P.NZ - 1 ? plane : 0;
    DFG_T s[DFG_NSF_][7];
#pragma unroll
    for (int f = 0; f < DFG_NSF; ++f) {
      const DFG_T* F = P.f[f];
      s[f][0] = F[base];
      s[f][1] = F[base - oxm];
      s[f][2] = F[base + oxp];
      s[f][3] = F[base - oym];
      s[f][4] = F[base + oyp];
      s[f][5] = F[base - ozm];
      s[f][6] = F[base + ozp];
    }
    DFG_T p[DFG_NPF_];
#pragma unroll
    for (int f = 0; f < DFG_NPF; ++f) p[f] = P.f[DFG_NSF + f][base];
    DFG_T o[DFG_OUTW];
    dfg_body(s, p, P.tx[i], P.tx[P.nx + i], P.ty[j], P.ty[P.ny + j], P.tz[kg], P.tz[P.NZ + kg], o);
    const long long ob = (kl * plane + j * P.nx + i) * DFG_OUTW;
#pragma unroll
    for (int h = 0; h < DFG_OUTW; ++h) P.out[ob + h] = o[h];
  }
}
#endif

#if DFG_NSF > 0 && DFG_HAS_TMA
// ----------------------------------------------------------------- TMA
struct __align__(64) DfgTmap { unsigned long long v[16]; };  // CUtensorMap
struct DfgTmaParams {
  DfgTmap map[DFG_NSF_];
  DfgParams p;
};

#define DFG_TX (32 * DFG_VEC)
#define DFG_HX DFG_VEC
#define DFG_ROWW (DFG_TX + 2 * DFG_HX)
#define DFG_ROWS (DFG_NCW + 2)
#define DFG_TILE_ELEMS (DFG_ROWW * DFG_ROWS)
#define DFG_TILE_BYTES ((DFG_TILE_ELEMS * (int)sizeof(DFG_T) + 127) / 128 * 128)
#define DFG_STAGE_BYTES (DFG_TILE_BYTES * DFG_NSF)

__device__ __forceinline__ unsigned dfg_smem(const void* p) {
  return (unsigned)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void dfg_mbar_init(unsigned long long* b, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(dfg_smem(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void dfg_mbar_expect_tx(unsigned long long* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(dfg_smem(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void dfg_mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(dfg_smem(b)) : "memory");
}
__device__ __forceinline__ void dfg_mbar_wait(unsigned long long* b, unsigned parity) {
  unsigned done;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(dfg_smem(b)), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void dfg_tma_load3(void* dst, const DfgTmap* map, unsigned long long* bar,
                                              int x, int y, int z) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dfg_smem(dst)),
      "l"(reinterpret_cast<unsigned long long>(map)), "r"(dfg_smem(bar)), "r"(x), "r"(y), "r"(z)
      : "memory");
}

extern "C" __global__ void __launch_bounds__((DFG_NCW + 1) * 32, 1)
    dfg_fused_tma(const __grid_constant__ DfgTmaParams TP) {
  const DfgParams& P = TP.p;
  // dynamic shared memory starts at the (1024-aligned) base of the CTA's
  // window: no static __shared__ in this kernel
  extern __shared__ __align__(1024) unsigned char dfg_smem_raw[];
  unsigned char* smem = dfg_smem_raw;
  unsigned long long* full = reinterpret_cast<unsigned long long*>(smem + DFG_STAGES * DFG_STAGE_BYTES);
  unsigned long long* empty = full + DFG_STAGES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const long long plane = P.nx * P.ny;

  if (threadIdx.x == 0) {
    for (int s = 0; s < DFG_STAGES; ++s) {
      dfg_mbar_init(&full[s], 1);
      dfg_mbar_init(&empty[s], DFG_NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == DFG_NCW) {
    // ---------------- producer: one elected lane issues all TMA loads
    if (lane == 0) {
      for (int f = 0; f < DFG_NSF; ++f)
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<unsigned long long>(&TP.map[f]))
                     : "memory");
      int stage = 0;
      unsigned phase = 0;
      for (long long item = blockIdx.x; item < P.items; item += gridDim.x) {
        const long long tx_ = item % P.tiles_x;
        const long long rest = item / P.tiles_x;
        const long long ty_ = rest % P.tiles_y;
        const long long zc = rest / P.tiles_y;
        const int x0 = (int)(tx_ * DFG_TX) - DFG_HX;
        const int y0 = (int)(ty_ * DFG_NCW) - 1;
        const long long kb = P.kbeg + zc * P.kz;
        const long long ke = min(kb + (long long)P.kz, P.kend);
        const long long pf = kb > 0 ? kb - 1 : kb;
        const long long pl = ke < P.NZ ? ke : ke - 1;
        for (long long pg = pf; pg <= pl; ++pg) {
          dfg_mbar_wait(&empty[stage], phase ^ 1u);
          dfg_mbar_expect_tx(&full[stage], (unsigned)(DFG_NSF * DFG_TILE_ELEMS * sizeof(DFG_T)));
          const int zl = (int)(pg - P.k0 + P.ghost);
#pragma unroll
          for (int f = 0; f < DFG_NSF; ++f)
            dfg_tma_load3(smem + stage * DFG_STAGE_BYTES + f * DFG_TILE_BYTES, &TP.map[f], &full[stage], x0, y0,
                          zl);
          if (++stage == DFG_STAGES) {
            stage = 0;
            phase ^= 1u;
          }
        }
      }
    }
    return;
  }

  // ------------------- consumers: warp w computes tile row w
  int stage = 0;
  unsigned phase = 0;
  const int c0 = DFG_HX + DFG_VEC * lane;
  const int r = 1 + warp;
  for (long long item = blockIdx.x; item < P.items; item += gridDim.x) {
    const long long tx_ = item % P.tiles_x;
    const long long rest = item / P.tiles_x;
    const long long ty_ = rest % P.tiles_y;
    const long long zc = rest / P.tiles_y;
    const long long i = tx_ * DFG_TX + DFG_VEC * lane;
    const long long j = ty_ * DFG_NCW + warp;
    const long long kb = P.kbeg + zc * P.kz;
    const long long ke = min(kb + (long long)P.kz, P.kend);
    const bool act = (i < P.nx) && (j < P.ny);
    const long long ic = min(i, P.nx - DFG_VEC);
    const long long jc = min(j, P.ny - 1);
    DFG_T dxv[DFG_VEC], rxv[DFG_VEC];
#pragma unroll
    for (int c = 0; c < DFG_VEC; ++c) {
      dxv[c] = P.tx[ic + c];
      rxv[c] = P.tx[P.nx + ic + c];
    }
    const DFG_T dy = P.ty[jc], ry = P.ty[P.ny + jc];
    const int cxm = (i == 0) ? c0 : c0 - 1;
    const int cxp = (i + DFG_VEC >= P.nx) ? c0 + DFG_VEC - 1 : c0 + DFG_VEC;
    const int rm = (j == 0) ? r : r - 1;
    const int rp = (j >= P.ny - 1) ? r : r + 1;

    DFG_T zm[DFG_NSF][DFG_VEC], zcur[DFG_NSF][DFG_VEC], zn[DFG_NSF][DFG_VEC];
#define DFG_TILE(st, f) reinterpret_cast<const DFG_T*>(smem + (st) * DFG_STAGE_BYTES + (f) * DFG_TILE_BYTES)
    if (kb > 0) {
      dfg_mbar_wait(&full[stage], phase);
#pragma unroll
      for (int f = 0; f < DFG_NSF; ++f) dfg_ld16(zm[f], DFG_TILE(stage, f) + r * DFG_ROWW + c0);
      __syncwarp();
      if (lane == 0) dfg_mbar_arrive(&empty[stage]);
      if (++stage == DFG_STAGES) { stage = 0; phase ^= 1u; }
    }
    dfg_mbar_wait(&full[stage], phase);
    int cur = stage;
#pragma unroll
    for (int f = 0; f < DFG_NSF; ++f) dfg_ld16(zcur[f], DFG_TILE(cur, f) + r * DFG_ROWW + c0);
    if (++stage == DFG_STAGES) { stage = 0; phase ^= 1u; }
    if (kb == 0) {
#pragma unroll
      for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
        for (int c = 0; c < DFG_VEC; ++c) zm[f][c] = zcur[f][c];
    }

    for (long long k = kb; k < ke; ++k) {
      int nxt = -1;
      if (k + 1 < P.NZ) {
        dfg_mbar_wait(&full[stage], phase);
        nxt = stage;
#pragma unroll
        for (int f = 0; f < DFG_NSF; ++f) dfg_ld16(zn[f], DFG_TILE(nxt, f) + r * DFG_ROWW + c0);
        if (++stage == DFG_STAGES) { stage = 0; phase ^= 1u; }
      } else {
#pragma unroll
        for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
          for (int c = 0; c < DFG_VEC; ++c) zn[f][c] = zcur[f][c];
      }
      DFG_T xm[DFG_NSF], xp[DFG_NSF], ym[DFG_NSF][DFG_VEC], yp[DFG_NSF][DFG_VEC];
#pragma unroll
      for (int f = 0; f < DFG_NSF; ++f) {
        const DFG_T* t = DFG_TILE(cur, f);
        xm[f] = t[r * DFG_ROWW + cxm];
        xp[f] = t[r * DFG_ROWW + cxp];
        dfg_ld16(ym[f], t + rm * DFG_ROWW + c0);
        dfg_ld16(yp[f], t + rp * DFG_ROWW + c0);
      }
      const DFG_T dz = P.tz[k], rz = P.tz[P.NZ + k];
      const long long cell = (k - P.k0) * plane + j * P.nx + i;
      DFG_T pv[DFG_NPF_][DFG_VEC];
#pragma unroll
      for (int f = 0; f < DFG_NPF; ++f) {
        if (act) dfg_ldg16(pv[f], P.f[DFG_NSF + f] + cell + P.ghost * plane);
        else
#pragma unroll
          for (int c = 0; c < DFG_VEC; ++c) pv[f][c] = DFG_T(0);
      }
      DFG_T o[DFG_VEC][DFG_OUTW];
#pragma unroll
      for (int c = 0; c < DFG_VEC; ++c) {
        DFG_T s[DFG_NSF][7];
#pragma unroll
        for (int f = 0; f < DFG_NSF; ++f) {
          s[f][0] = zcur[f][c];
          s[f][1] = c == 0 ? xm[f] : zcur[f][c == 0 ? 0 : c - 1];
          s[f][2] = c == DFG_VEC - 1 ? xp[f] : zcur[f][c == DFG_VEC - 1 ? c : c + 1];
          s[f][3] = ym[f][c];
          s[f][4] = yp[f][c];
          s[f][5] = zm[f][c];
          s[f][6] = zn[f][c];
        }
        DFG_T p[DFG_NPF_];
#pragma unroll
        for (int f = 0; f < DFG_NPF; ++f) p[f] = pv[f][c];
        dfg_body(s, p, dxv[c], rxv[c], dy, ry, dz, rz, o[c]);
      }
      if (act) {
        DFG_T* dst = P.out + cell * DFG_OUTW;
#if DFG_OUTW == 1
        DFG_T t[DFG_VEC];
#pragma unroll
        for (int c = 0; c < DFG_VEC; ++c) t[c] = o[c][0];
        dfg_stg16(dst, t);
#else
#pragma unroll
        for (int c = 0; c < DFG_VEC; ++c)
#pragma unroll
          for (int h = 0; h < DFG_OUTW; h += DFG_VEC) dfg_stg16(dst + c * DFG_OUTW + h, &o[c][h]);
#endif
      }
      __syncwarp();
      if (lane == 0) {
        dfg_mbar_arrive(&empty[cur]);
        if (k + 1 == ke && nxt >= 0) dfg_mbar_arrive(&empty[nxt]);  // post plane: centre only
      }
      cur = nxt;
#pragma unroll
      for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
        for (int c = 0; c < DFG_VEC; ++c) {
          zm[f][c] = zcur[f][c];
          zcur[f][c] = zn[f][c];
        }
    }
#undef DFG_TILE
  }
}
#endif
