// dfg_fused_tma: the B200 fused-kernel skeleton (PAPER.md L97-L105 fusion,
// re-designed for sm_100a).  Compiled by NVRTC after skeleton.cuh.
//
// Work decomposition: persistent CTAs (grid = #SM x occupancy) walk items
// (x-tile of DFG_TX = 32*VEC/RPW cells) x (y-tile of DFG_TH = NCW*RPW rows)
// x (z-chunk of kz planes), item = blockIdx.x + t*gridDim.x; RPW (rows per
// consumer warp: 1, 2 or 4) is chosen on the host so that narrow meshes do
// not leave lanes idle in a ragged x-tile.  Warp DFG_NCW is the producer:
// one lane streams, per z-plane, one halo'd x-y tile per stencil field
// (box (TX + 2*VEC) x (TH + 2) x 1, cp.async.bulk.tensor.3d) into a
// DFG_STAGES-deep ring of shared-memory stages guarded by full/empty
// mbarriers (complete_tx byte counts; all consumer threads arrive on
// "empty", so no divergent branch).  For every item the producer loads
// kz + 2 planes: the pre-plane max(kb-1, 0), planes kb..ke-1 and the post-plane
// min(ke, NZ-1).  At the global ends these duplicate the first / last plane,
// which is exactly the clamped neighbour of reading R1, so the consumer loop
// has no boundary branch.
// Consumers: warp w owns tile rows w*RPW .. w*RPW+RPW-1 (32/RPW lanes per
// row), a lane owns VEC consecutive x cells of its row;
// the z-1 / z / z+1 centres live in a 3-entry register queue whose roles
// rotate through a 3-way unrolled loop (no register copies); x/y neighbours
// come from shared memory through per-thread clamped offsets; the network
// body runs on pairs of cells (FADD2/FFMA2); results leave as 16-byte
// streaming stores.

#if DFG_NSF > 0 && DFG_HAS_TMA
struct __align__(64) DfgTmap { unsigned long long v[16]; };  // CUtensorMap
// Peer-memory halo of a z-slab: the neighbours' stencil fields, read in place
// (IPC mappings) for the planes outside [k0, k0 + nzl).
struct DfgPeerInfo {
  long long lo_k0, lo_ghost, hi_k0, hi_ghost;
  int lo_on, hi_on;
  // single-launch mode (wait != 0): before loading a neighbour's plane the
  // producer waits in the kernel until that neighbour's "ready" flag (IPC
  // mapped) reaches `epoch`, and the z-chunks at the slab ends run last
  int wait;
  unsigned epoch;
  const unsigned* lo_ready;
  const unsigned* hi_ready;
};
// host image: runtime.cpp tma_blob_* (same order, 64-byte aligned maps)
struct DfgTmaParams {
  DfgTmap map[DFG_NF_];  // stencil fields, then point-wise fields
  DfgTmap map_lo[DFG_NSF_], map_hi[DFG_NSF_];  // neighbours' stencil fields (peer halo)
  DfgPeerInfo peer;
  DfgParams p;
};

#ifndef DFG_RPW
#define DFG_RPW 1
#endif
#define DFG_LPR (32 / DFG_RPW)          // lanes per tile row
#define DFG_TX (DFG_LPR * DFG_VEC)      // tile width (cells)
#define DFG_TH (DFG_NCW * DFG_RPW)      // tile height (rows)
#define DFG_HX DFG_VEC
#define DFG_ROWW (DFG_TX + 2 * DFG_HX)
#define DFG_ROWS (DFG_TH + 2)
#define DFG_TILE_ELEMS (DFG_ROWW * DFG_ROWS)
#define DFG_TILE_BYTES ((DFG_TILE_ELEMS * (int)sizeof(DFG_T) + 127) / 128 * 128)
// every field streams through the ring (point-wise fields: centre only)
#define DFG_NTF (DFG_NSF + DFG_NPF)
#define DFG_STAGE_BYTES (DFG_TILE_BYTES * DFG_NTF)

__device__ __forceinline__ unsigned dfg_smem(const void* p) {
  return (unsigned)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void dfg_mbar_init(unsigned bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void dfg_mbar_expect_tx(unsigned bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void dfg_mbar_arrive(unsigned bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
// try_wait with a suspend-time hint: the thread sleeps in hardware until the
// phase completes (or the hint expires) instead of spinning on issue slots
__device__ __forceinline__ bool dfg_mbar_try(unsigned bar, unsigned parity, unsigned hint_ns) {
  unsigned done;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(done)
      : "r"(bar), "r"(parity), "r"(hint_ns)
      : "memory");
  return done != 0;
}
__device__ __forceinline__ void dfg_mbar_wait(unsigned bar, unsigned parity, unsigned hint_ns) {
  while (!dfg_mbar_try(bar, parity, hint_ns)) {
  }
}
// Shared-memory bounds / alignment check (NVRTC define DFG_CHECK_SMEM; the
// GPU pool has no compute-sanitizer): every shared access of the ring
// kernels must lie inside the CTA's dynamic window and be aligned to its
// size, else the kernel traps (a loud CUDA error, never a silent result).
#ifdef DFG_CHECK_SMEM
__device__ __forceinline__ void dfg_check_smem(unsigned addr, unsigned bytes) {
  extern __shared__ __align__(1024) unsigned char dfg_smem_raw[];
  const unsigned base = (unsigned)__cvta_generic_to_shared(dfg_smem_raw);
  unsigned size;
  asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(size));
  if (addr < base || addr + bytes > base + size || (addr & (bytes - 1u)) != 0u) __trap();
}
#define DFG_SMEM_CHECK(a, b) dfg_check_smem((a), (b))
#else
#define DFG_SMEM_CHECK(a, b)
#endif
__device__ __forceinline__ void dfg_tma_load3(unsigned dst, const DfgTmap* map, unsigned bar, int x, int y, int z) {
  DFG_SMEM_CHECK(dst, 16u);
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<unsigned long long>(map)), "r"(bar), "r"(x), "r"(y), "r"(z)
      : "memory");
}
__device__ __forceinline__ void dfg_lds16(DFG_T (&d)[DFG_VEC], unsigned addr) {
  DFG_SMEM_CHECK(addr, 16u);
#if DFG_VEC == 4
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(d[0]), "=f"(d[1]), "=f"(d[2]), "=f"(d[3])
               : "r"(addr)
               : "memory");
#else
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(d[0]), "=d"(d[1]) : "r"(addr) : "memory");
#endif
}
__device__ __forceinline__ DFG_T dfg_lds1(unsigned addr) {
  DFG_SMEM_CHECK(addr, (unsigned)sizeof(DFG_T));
  DFG_T v;
#if DFG_VEC == 4
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
#else
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr) : "memory");
#endif
  return v;
}

// Ring cursor: shared-memory byte address of the current stage and of its
// full / empty barriers, advanced without multiplies (same sequence as the
// producer's).
template <unsigned SB, int NS>
struct DfgRingT {
  static constexpr unsigned kEmpty = 8u * NS;  // empty[s] = full[s] + kEmpty
  unsigned tile;   // smem byte address of stage s, field 0
  unsigned full;   // smem byte address of full[s]
  unsigned phase;
  int stage;
  unsigned tile0, full0;
  __device__ __forceinline__ void advance() {
    ++stage;
    tile += SB;
    full += 8;
    if (stage == NS) {
      stage = 0;
      tile = tile0;
      full = full0;
      phase ^= 1u;
    }
  }
};
typedef DfgRingT<DFG_STAGE_BYTES, DFG_STAGES> DfgRing;
#define DFG_EMPTY(full_addr) ((full_addr) + 8 * DFG_STAGES)

// per-item, per-thread constants of a consumer thread
struct DfgCol {
  unsigned off_c, off_xm, off_xp, off_ym, off_yp;  // byte offsets in a tile
  dfg2 ndx[DFG_NPAIR], rx[DFG_NPAIR], ndy, ry, Z;  // -d and 1/d spacing entries
  bool act;
  int nvalid;  // tile kernel: cells of this thread inside the mesh (0..VEC)
  bool vst;    // tile kernel: 16-byte output stores allowed (aligned rows)
};

// The TMA kernel's producer warp fills the ring; the tile kernel's consumer
// threads fill it themselves, one stage per consumed stage (DfgFill below).
struct DfgNoFill {
  __device__ __forceinline__ void step() {}
};

// Masked store of the VEC cells of a thread (tile kernel): 16-byte store
// when the row is aligned and every cell is inside the mesh, else one scalar
// store per valid cell.
__device__ __forceinline__ void dfg_store_masked(DFG_T* dst, const dfg2 (&o)[DFG_NPAIR][DFG_OUTW], const DfgCol& C) {
  if (C.nvalid == DFG_VEC && C.vst) {
    dfg_store_cells(dst, o);
    return;
  }
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h)
#pragma unroll
    for (int l = 0; l < DFG_LANES; ++l) {
      const int c = h * DFG_LANES + l;
      if (c < C.nvalid) {
#pragma unroll
        for (int w = 0; w < DFG_OUTW; ++w) __stcs(dst + c * DFG_OUTW + w, dfg2_get(o[h][w], l));
      }
    }
}

// One z-plane.  `cur` = smem address of the plane's stage (tile, full bar);
// the next plane's stage is always present (the producer loads a clamped
// post-plane).  Queue roles are template parameters (no copies).
template <int ZM, int ZC, int ZN, bool MASKED = false, class Fill = DfgNoFill, class Ring = DfgRing>
__device__ __forceinline__ void dfg_plane(const DfgCol& C, Ring& R, unsigned& cur_tile, unsigned& cur_full,
                                          DFG_T (&zq)[3][DFG_NSF][DFG_VEC], DFG_T*& outp,
                                          long long plane, const DFG_T*& tzd, const DFG_T*& tzr, Fill& fill) {
  // x/y neighbours of this plane first (its stage is already resident), then
  // wait for the next plane's stage: the loads overlap the barrier wait
  DFG_T xmv[DFG_NSF], xpv[DFG_NSF], ymv[DFG_NSF][DFG_VEC], ypv[DFG_NSF][DFG_VEC];
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) {
    const unsigned t = cur_tile + f * DFG_TILE_BYTES;
    xmv[f] = dfg_lds1(t + C.off_xm);
    xpv[f] = dfg_lds1(t + C.off_xp);
    dfg_lds16(ymv[f], t + C.off_ym);
    dfg_lds16(ypv[f], t + C.off_yp);
  }
  dfg_mbar_wait(R.full, R.phase, 0x100000u);
  const unsigned nxt_tile = R.tile, nxt_full = R.full;
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) dfg_lds16(zq[ZN][f], nxt_tile + f * DFG_TILE_BYTES + C.off_c);
  R.advance();
  dfg2 s[DFG_NPAIR][DFG_NSF][7], gn[DFG_NPAIR][DFG_NSF][3];
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) {
    const DFG_T xm = xmv[f], xp = xpv[f];
    const DFG_T(&ym)[DFG_VEC] = ymv[f];
    const DFG_T(&yp)[DFG_VEC] = ypv[f];
    DFG_T lft[DFG_VEC], rgt[DFG_VEC];
#pragma unroll
    for (int c = 0; c < DFG_VEC; ++c) {
      lft[c] = c == 0 ? xm : zq[ZC][f][c == 0 ? 0 : c - 1];
      rgt[c] = c == DFG_VEC - 1 ? xp : zq[ZC][f][c == DFG_VEC - 1 ? c : c + 1];
    }
#pragma unroll
    for (int h = 0; h < DFG_NPAIR; ++h) {
      const int a = h * DFG_LANES, b = h * DFG_LANES + DFG_LANES - 1;
      s[h][f][0] = dfg2_mk(zq[ZC][f][a], zq[ZC][f][b]);
      s[h][f][1] = dfg2_mk(lft[a], lft[b]);
      s[h][f][2] = dfg2_mk(rgt[a], rgt[b]);
      s[h][f][3] = dfg2_mk(ym[a], ym[b]);
      s[h][f][4] = dfg2_mk(yp[a], yp[b]);
      s[h][f][5] = dfg2_mk(zq[ZM][f][a], zq[ZM][f][b]);
      s[h][f][6] = dfg2_mk(zq[ZN][f][a], zq[ZN][f][b]);
      // x numerators as scalar subtractions (no pair shuffles), y/z as pairs
      gn[h][f][0] = dfg2_mk(dfg_sub(rgt[a], lft[a]), dfg_sub(rgt[b], lft[b]));
      gn[h][f][1] = dfg2_sub(s[h][f][4], s[h][f][3], C.Z);
      gn[h][f][2] = dfg2_sub(s[h][f][6], s[h][f][5], C.Z);
    }
  }
  const dfg2 ndz = dfg2_splat(__ldg(tzd)), rz = dfg2_splat(__ldg(tzr));
  ++tzd;
  ++tzr;
  dfg2 p[DFG_NPAIR][DFG_NPF_];
#pragma unroll
  for (int f = 0; f < DFG_NPF; ++f) {
    DFG_T pv[DFG_VEC];
    dfg_lds16(pv, cur_tile + (DFG_NSF + f) * DFG_TILE_BYTES + C.off_c);
#pragma unroll
    for (int h = 0; h < DFG_NPAIR; ++h) p[h][f] = dfg2_mk(pv[h * DFG_LANES], pv[h * DFG_LANES + DFG_LANES - 1]);
  }
  dfg2 o[DFG_NPAIR][DFG_OUTW];
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h)
    dfg_body(s[h], gn[h], p[h], C.ndx[h], C.rx[h], C.ndy, C.ry, ndz, rz, C.Z, o[h]);
  if (MASKED) {
    dfg_store_masked(outp, o, C);
  } else if (C.act) {
    dfg_store_cells(outp, o);
  }
  outp += plane * DFG_OUTW;
  dfg_mbar_arrive(cur_full + Ring::kEmpty);  // every consumer thread (count NCW*32)
  fill.step();
  cur_tile = nxt_tile;
  cur_full = nxt_full;
}

// z-chunk of an item.  Single-launch peer halo: the interior chunks first,
// then the chunk at the low slab end, the one at the high end last (their
// boundary planes wait for the neighbours; the interior overlaps that wait).
__device__ __forceinline__ long long dfg_zchunk(const DfgTmaParams& TP, long long zc) {
  if (!TP.peer.wait) return zc;
  const long long n = (TP.p.kend - TP.p.kbeg + TP.p.kz - 1) / TP.p.kz;
  if (n < 3) return zc;
  return zc < n - 2 ? zc + 1 : (zc == n - 2 ? 0 : n - 1);
}

// Wait (producer lane) until a neighbour's IPC-mapped "ready" flag reaches
// the step: acquire at system scope, then order the async proxy (the TMA
// reads that follow) after it.  A neighbour that never arrives within 30 s
// traps: a loud failure, never a silent wrong result or a hung step.
__device__ __forceinline__ void dfg_wait_ready(const unsigned* flag, unsigned epoch) {
  unsigned long long t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    unsigned v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
    if ((int)(v - epoch) >= 0) break;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 30000000000ull) __trap();
    __nanosleep(200);
  }
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// Producer side of one item (x-tile, y-tile, z-chunk) of mesh TP: the
// pre-plane, planes kb..ke-1 and the post-plane, clamped to the global mesh (R1).
__device__ __forceinline__ void dfg_produce_item(const DfgTmaParams& TP, long long item, DfgRing& W) {
  const DfgParams& P = TP.p;
  const long long tx_ = item % P.tiles_x;
  const long long rest = item / P.tiles_x;
  const long long ty_ = rest % P.tiles_y;
  const long long zc = dfg_zchunk(TP, rest / P.tiles_y);
  // input coordinates include the block's x/y ghost columns / rows
  const int x0 = (int)(tx_ * DFG_TX) - DFG_HX + (int)P.gx;
  const int y0 = (int)(ty_ * DFG_TH) - 1 + (int)P.gy;
  const long long kb = P.kbeg + zc * P.kz;
  const long long ke = min(kb + (long long)P.kz, P.kend);
  for (long long q = kb - 1; q <= ke; ++q) {
    const long long pg = max(0LL, min(q, P.NZ - 1));
    // wait until every consumer released this slot (the producer runs
    // ahead; the suspend hint keeps it off the issue slots)
    dfg_mbar_wait(DFG_EMPTY(W.full), W.phase ^ 1u, 0x100000u);
    dfg_mbar_expect_tx(W.full, (unsigned)(DFG_NTF * DFG_TILE_ELEMS * sizeof(DFG_T)));
    const int zl = (int)(pg - P.k0 + P.ghost);
    // planes of the z neighbours come from their own buffers when the slab is
    // linked to peers (stencil fields only; point-wise fields are read at owned planes)
    const bool lo = TP.peer.lo_on && pg < P.k0, hi = TP.peer.hi_on && pg >= P.k0 + P.nzl;
    const int zp = lo ? (int)(pg - TP.peer.lo_k0 + TP.peer.lo_ghost) : (int)(pg - TP.peer.hi_k0 + TP.peer.hi_ghost);
    if (TP.peer.wait && (lo || hi)) dfg_wait_ready(lo ? TP.peer.lo_ready : TP.peer.hi_ready, TP.peer.epoch);
#pragma unroll
    for (int f = 0; f < DFG_NTF; ++f) {
      const bool peer = (lo || hi) && f < DFG_NSF;
      const DfgTmap* map = !peer ? &TP.map[f] : lo ? &TP.map_lo[f < DFG_NSF ? f : 0] : &TP.map_hi[f < DFG_NSF ? f : 0];
      dfg_tma_load3(W.tile + f * DFG_TILE_BYTES, map, W.full, x0, y0, peer ? zp : zl);
    }
    W.advance();
  }
}

// Consumer side of one item: warp w computes tile rows w*RPW .. w*RPW+RPW-1.
__device__ __forceinline__ void dfg_consume_item(const DfgTmaParams& TP, long long item, DfgRing& R, DfgCol& C,
                                                 int warp, int lane) {
  const DfgParams& P = TP.p;
  const long long plane = P.nx * P.ny;
  const int col = lane % DFG_LPR, sub = lane / DFG_LPR;
  const unsigned c0 = DFG_HX + DFG_VEC * col;
  const unsigned r = 1 + warp * DFG_RPW + sub;
  const long long tx_ = item % P.tiles_x;
  const long long rest = item / P.tiles_x;
  const long long ty_ = rest % P.tiles_y;
  const long long zc = dfg_zchunk(TP, rest / P.tiles_y);
  const long long i = tx_ * DFG_TX + DFG_VEC * col;
  const long long j = ty_ * DFG_TH + warp * DFG_RPW + sub;
  const long long kb = P.kbeg + zc * P.kz;
  const long long ke = min(kb + (long long)P.kz, P.kend);
  C.act = (i < P.nx) && (j < P.ny);
  const long long ic = min(i, P.nx - DFG_VEC);
  const long long jc = min(j, P.ny - 1);
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h) {
    // spacing tables are indexed globally (blocks: i0 / j0 offsets)
    const long long a = P.i0 + ic + h * DFG_LANES, b = P.i0 + ic + h * DFG_LANES + DFG_LANES - 1;
    C.ndx[h] = dfg2_mk(__ldg(P.tx + DFG_NDSEG_X * P.NX + a), __ldg(P.tx + DFG_NDSEG_X * P.NX + b));
    C.rx[h] = dfg2_mk(__ldg(P.tx + P.NX + a), __ldg(P.tx + P.NX + b));
  }
  C.ndy = dfg2_splat(__ldg(P.ty + DFG_NDSEG_Y * P.NY + P.j0 + jc));
  C.ry = dfg2_splat(__ldg(P.ty + P.NY + P.j0 + jc));
  // one-sided differences only at the GLOBAL mesh ends (reading R1)
  const long long ig = P.i0 + i, jg = P.j0 + j;
  const unsigned cxm = (ig == 0) ? c0 : c0 - 1;
  const unsigned cxp = (ig + DFG_VEC >= P.NX) ? c0 + DFG_VEC - 1 : c0 + DFG_VEC;
  const unsigned rm = (jg == 0) ? r : r - 1;
  const unsigned rp = (jg >= P.NY - 1) ? r : r + 1;
  const unsigned TS = (unsigned)sizeof(DFG_T);
  C.off_c = (r * DFG_ROWW + c0) * TS;
  C.off_xm = (r * DFG_ROWW + cxm) * TS;
  C.off_xp = (r * DFG_ROWW + cxp) * TS;
  C.off_ym = (rm * DFG_ROWW + c0) * TS;
  C.off_yp = (rp * DFG_ROWW + c0) * TS;
  const long long cell0 = (kb - P.k0) * plane + jc * P.nx + ic;
  DFG_T* outp = P.out + cell0 * DFG_OUTW;
  const DFG_T* tzd = P.tz + DFG_NDSEG_Z * P.NZ + kb;  // -d and 1/d of the plane's z spacing
  const DFG_T* tzr = P.tz + P.NZ + kb;

  DFG_T zq[3][DFG_NSF][DFG_VEC];
  // pre-plane (clamped): its centre becomes z-1 of plane kb
  dfg_mbar_wait(R.full, R.phase, 0x100000u);
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) dfg_lds16(zq[0][f], R.tile + f * DFG_TILE_BYTES + C.off_c);
  dfg_mbar_arrive(DFG_EMPTY(R.full));
  R.advance();
  dfg_mbar_wait(R.full, R.phase, 0x100000u);
  unsigned cur_tile = R.tile, cur_full = R.full;
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) dfg_lds16(zq[1][f], cur_tile + f * DFG_TILE_BYTES + C.off_c);
  R.advance();
  DfgNoFill nf;
  long long k = kb;
  for (; k + 3 <= ke; k += 3) {
    dfg_plane<0, 1, 2>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, nf);
    dfg_plane<1, 2, 0>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, nf);
    dfg_plane<2, 0, 1>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, nf);
  }
  if (k < ke) {
    dfg_plane<0, 1, 2>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, nf);
    if (k + 1 < ke) dfg_plane<1, 2, 0>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, nf);
  }
  // the post-plane stage was read for its centre only
  dfg_mbar_arrive(DFG_EMPTY(cur_full));
}

// full_count: arrivals that complete a "full" phase (1 for the TMA
// producer's arrive.expect_tx; every consumer thread for the tile kernel)
__device__ __forceinline__ unsigned dfg_ring_init(unsigned full_count = 1, unsigned stage_bytes = DFG_STAGE_BYTES,
                                                  int stages = DFG_STAGES, unsigned empty_count = DFG_NCW * 32,
                                                  bool ready = false) {
  // dynamic shared memory starts at the (1024-aligned) base of the CTA's
  // window: no static __shared__ in this kernel
  extern __shared__ __align__(1024) unsigned char dfg_smem_raw[];
  const unsigned smem = dfg_smem(dfg_smem_raw);
  const unsigned full0 = smem + stages * stage_bytes;  // full[s] at full0 + 8s, empty[s] = full[s] + 8*stages
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      dfg_mbar_init(full0 + 8 * s, full_count);
      dfg_mbar_init(full0 + 8 * s + 8 * stages, empty_count);
      if (ready) dfg_mbar_init(full0 + 8 * s + 16 * stages, 1);  // ready[s] = full[s] + 16*stages
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  return smem;
}

extern "C" __global__ void __launch_bounds__((DFG_NCW + 1) * 32, DFG_CTAS)
    dfg_fused_tma(const __grid_constant__ DfgTmaParams TP) {
  const unsigned smem = dfg_ring_init();
  const unsigned full0 = smem + DFG_STAGES * DFG_STAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  if (warp == DFG_NCW) {
    // ---------------- producer: one lane issues all TMA loads
    if (lane == 0) {
      for (int f = 0; f < DFG_NTF; ++f)
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<unsigned long long>(&TP.map[f]))
                     : "memory");
      DfgRing W{smem, full0, 0u, 0, smem, full0};
      for (long long item = blockIdx.x; item < TP.p.items; item += gridDim.x) dfg_produce_item(TP, item, W);
    }
    return;
  }
  // ------------------- consumers
  DfgRing R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(TP.p.nzero);
  for (long long item = blockIdx.x; item < TP.p.items; item += gridDim.x) dfg_consume_item(TP, item, R, C, warp, lane);
}

// Several meshes of one network in one launch (VisIt-style blocks of a
// device, the paper's 12 sub-grids per GPU, L315): block b's parameters and
// tensor maps live in global memory; the persistent CTAs walk the
// concatenated item space, first[b] = first item of block b, first[nb] = total.
struct DfgMulti {
  const DfgTmaParams* blocks;
  const long long* first;
  int nb;
};

extern "C" __global__ void __launch_bounds__((DFG_NCW + 1) * 32, DFG_CTAS)
    dfg_fused_tma_multi(const __grid_constant__ DfgMulti M) {
  const unsigned smem = dfg_ring_init();
  const unsigned full0 = smem + DFG_STAGES * DFG_STAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const long long total = M.first[M.nb];
  if (warp == DFG_NCW) {
    if (lane == 0) {
      DfgRing W{smem, full0, 0u, 0, smem, full0};
      int b = 0;
      for (long long item = blockIdx.x; item < total; item += gridDim.x) {
        while (item >= M.first[b + 1]) ++b;  // items only grow: the block index too
        dfg_produce_item(M.blocks[b], item - M.first[b], W);
      }
    }
    return;
  }
  DfgRing R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(M.blocks[0].p.nzero);
  int b = 0;
  for (long long item = blockIdx.x; item < total; item += gridDim.x) {
    while (item >= M.first[b + 1]) ++b;
    dfg_consume_item(M.blocks[b], item - M.first[b], R, C, warp, lane);
  }
}

// ---------------------------------------------------------------- tile
// Layouts the tensor maps cannot describe: rows that are not a multiple of
// 16 bytes (nx % VEC != 0), packed ghost shells (owned cells from column 1),
// pitched or unaligned buffers.  TMA needs 16-byte global strides and box
// starts (an odd start column faults on B200, tools/tma_probe.cu), so the
// consumer threads fill the same shared-memory ring themselves with 4 / 8-byte
// cp.async copies, every tile element landing at the position the TMA kernel
// reads (LDS.128 stays aligned whatever the global alignment).  Elements past
// the GLOBAL mesh ends are filled with the boundary cell (clamped source
// index), so a ragged last vector of a row and the one-sided differences of
// reading R1 need no per-cell selects; inside a block the ghost shell is read
// as data.  The fill runs STAGES-1 stages ahead of the consumption: every
// consumed stage releases its slot ("empty") and each thread then issues its
// share of the next stage (waiting for the slot released one stage earlier)
// and arrives on that stage's "full" barrier when its copies land
// (cp.async.mbarrier.arrive.noinc; full count = all consumer threads).
#define DFG_NT (DFG_NCW * 32)
#define DFG_FM ((DFG_TILE_ELEMS + DFG_NT - 1) / DFG_NT)  // tile elements per thread

__device__ __forceinline__ void dfg_cp_async(unsigned dst, const DFG_T* src) {
#if DFG_VEC == 4
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst), "l"(src) : "memory");
#else
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(dst), "l"(src) : "memory");
#endif
}
__device__ __forceinline__ void dfg_cp_async_arrive(unsigned bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}

// Fill cursor of one consumer thread: the stage sequence of the CTA's items
// (pre-plane, planes kb..ke-1, post-plane of each), its own ring position.
// Several meshes (dfg_fused_tile_multi): block b's parameters at blocks[b],
// its items first[b] .. first[b+1]-1 of the concatenated item space; a
// single mesh is the case nb = 1 with first = {0, items}.
struct DfgFill {
  const DfgParams* blocks;  // all blocks (single mesh: the kernel parameter)
  const long long* first;   // nullptr: single mesh
  int b;                    // current block
  long long item, end;      // global item; end of the item space
  long long q, qe;
  DfgRing W;
  unsigned off[DFG_FM];  // input element offsets within a plane of this thread's tile elements
  unsigned tid;

  __device__ __forceinline__ long long base() const { return first ? first[b] : 0; }
  __device__ __forceinline__ void setup() {
    if (first)
      while (item >= first[b + 1]) ++b;  // items only grow: the block index too
    const DfgParams& p = blocks[b];
    const long long li = item - base();
    const long long tx_ = li % p.tiles_x;
    const long long rest = li / p.tiles_x;
    const long long ty_ = rest % p.tiles_y;
    const long long zc = rest / p.tiles_y;
    const long long kb = p.kbeg + zc * p.kz;
    q = kb - 1;
    qe = min(kb + (long long)p.kz, p.kend);
    const int x0 = (int)(tx_ * DFG_TX) - DFG_HX + (int)p.gx;  // input column of tile column 0
    const int y0 = (int)(ty_ * DFG_TH) - 1 + (int)p.gy;      // input row of tile row 0
    // clamp to the global mesh ends (R1); elsewhere to the input array
    const int clo = p.i0 == 0 ? (int)p.gx : 0;
    const int chi = p.i0 + p.nx >= p.NX ? (int)(p.gx + p.nx - 1) : (int)(p.px - 1);
    const int rlo = p.j0 == 0 ? (int)p.gy : 0;
    const int rhi = p.j0 + p.ny >= p.NY ? (int)(p.gy + p.ny - 1) : (int)(p.py - 1);
#pragma unroll
    for (int m = 0; m < DFG_FM; ++m) {
      const unsigned e = tid + m * DFG_NT;
      const int row = (int)(e / DFG_ROWW), col = (int)(e % DFG_ROWW);
      const int yy = max(rlo, min(y0 + row, rhi)), xx = max(clo, min(x0 + col, chi));
      off[m] = (unsigned)yy * (unsigned)p.px + (unsigned)xx;
    }
  }
  __device__ __forceinline__ void init(const DfgParams* p, const long long* fst, long long total, unsigned smem,
                                       unsigned full0, unsigned t) {
    blocks = p;
    first = fst;
    b = 0;
    end = total;
    W = DfgRing{smem, full0, 0u, 0, smem, full0};
    tid = t;
    item = blockIdx.x;
    if (item < end) setup();
  }
  // issue this thread's share of the next stage of the sequence
  __device__ __forceinline__ void step() {
    if (item >= end) return;
    const DfgParams& p = blocks[b];
    dfg_mbar_wait(DFG_EMPTY(W.full), W.phase ^ 1u, 0x100000u);
    const long long pg = max(0LL, min(q, p.NZ - 1));
    const long long pbase = (pg - p.k0 + p.ghost) * p.px * p.py;
    const unsigned TS = (unsigned)sizeof(DFG_T);
#pragma unroll
    for (int f = 0; f < DFG_NTF; ++f) {
      const DFG_T* src = p.f[f] + pbase;
      const unsigned dst = W.tile + f * DFG_TILE_BYTES + tid * TS;
#pragma unroll
      for (int m = 0; m < DFG_FM; ++m)
        if (m < DFG_FM - 1 || tid + m * DFG_NT < (unsigned)DFG_TILE_ELEMS) dfg_cp_async(dst + m * DFG_NT * TS, src + off[m]);
    }
    dfg_cp_async_arrive(W.full);
    W.advance();
    if (++q > qe) {
      item += gridDim.x;
      if (item < end) setup();
    }
  }
};

template <class Ring, class Fill>
__device__ __forceinline__ void dfg_consume_tile(const DfgParams& P, long long item, Ring& R, DfgCol& C, int warp,
                                                 int lane, Fill& F) {
  const long long plane = P.nx * P.ny;
  const int col = lane % DFG_LPR, sub = lane / DFG_LPR;
  const unsigned c0 = DFG_HX + DFG_VEC * col;
  const unsigned r = 1 + warp * DFG_RPW + sub;
  const long long tx_ = item % P.tiles_x;
  const long long rest = item / P.tiles_x;
  const long long ty_ = rest % P.tiles_y;
  const long long zc = rest / P.tiles_y;
  const long long i = tx_ * DFG_TX + DFG_VEC * col;
  const long long j = ty_ * DFG_TH + warp * DFG_RPW + sub;
  const long long kb = P.kbeg + zc * P.kz;
  const long long ke = min(kb + (long long)P.kz, P.kend);
  C.nvalid = j < P.ny ? (int)max(0LL, min((long long)DFG_VEC, P.nx - i)) : 0;
  C.act = C.nvalid > 0;
  const long long ic = min(i, P.nx - 1);
  const long long jc = min(j, P.ny - 1);
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h) {
    // per-cell spacing entries (a ragged vector's outside cells reuse the last)
    const long long a = min(P.i0 + i + h * DFG_LANES, P.NX - 1);
    const long long b = min(P.i0 + i + h * DFG_LANES + DFG_LANES - 1, P.NX - 1);
    C.ndx[h] = dfg2_mk(__ldg(P.tx + DFG_NDSEG_X * P.NX + a), __ldg(P.tx + DFG_NDSEG_X * P.NX + b));
    C.rx[h] = dfg2_mk(__ldg(P.tx + P.NX + a), __ldg(P.tx + P.NX + b));
  }
  C.ndy = dfg2_splat(__ldg(P.ty + DFG_NDSEG_Y * P.NY + P.j0 + jc));
  C.ry = dfg2_splat(__ldg(P.ty + P.NY + P.j0 + jc));
  // the fill replicates the boundary cells past the global ends: plain offsets
  const unsigned TS = (unsigned)sizeof(DFG_T);
  C.off_c = (r * DFG_ROWW + c0) * TS;
  C.off_xm = (r * DFG_ROWW + c0 - 1) * TS;
  C.off_xp = (r * DFG_ROWW + c0 + DFG_VEC) * TS;
  C.off_ym = ((r - 1) * DFG_ROWW + c0) * TS;
  C.off_yp = ((r + 1) * DFG_ROWW + c0) * TS;
  DFG_T* outp = P.out + ((kb - P.k0) * plane + jc * P.nx + ic) * DFG_OUTW;
  const DFG_T* tzd = P.tz + DFG_NDSEG_Z * P.NZ + kb;  // -d and 1/d of the plane's z spacing
  const DFG_T* tzr = P.tz + P.NZ + kb;

  DFG_T zq[3][DFG_NSF][DFG_VEC];
  dfg_mbar_wait(R.full, R.phase, 0x100000u);
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) dfg_lds16(zq[0][f], R.tile + f * DFG_TILE_BYTES + C.off_c);
  dfg_mbar_arrive(R.full + Ring::kEmpty);
  F.step();
  R.advance();
  dfg_mbar_wait(R.full, R.phase, 0x100000u);
  unsigned cur_tile = R.tile, cur_full = R.full;
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) dfg_lds16(zq[1][f], cur_tile + f * DFG_TILE_BYTES + C.off_c);
  R.advance();
  long long k = kb;
  for (; k + 3 <= ke; k += 3) {
    dfg_plane<0, 1, 2, true, Fill, Ring>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, F);
    dfg_plane<1, 2, 0, true, Fill, Ring>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, F);
    dfg_plane<2, 0, 1, true, Fill, Ring>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, F);
  }
  if (k < ke) {
    dfg_plane<0, 1, 2, true, Fill, Ring>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, F);
    if (k + 1 < ke) dfg_plane<1, 2, 0, true, Fill, Ring>(C, R, cur_tile, cur_full, zq, outp, plane, tzd, tzr, F);
  }
  dfg_mbar_arrive(cur_full + Ring::kEmpty);
  F.step();
}

extern "C" __global__ void __launch_bounds__(DFG_NCW * 32, DFG_CTAS) dfg_fused_tile(const __grid_constant__ DfgParams P) {
  const unsigned smem = dfg_ring_init(DFG_NCW * 32);
  const unsigned full0 = smem + DFG_STAGES * DFG_STAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  DfgFill F;
  F.init(&P, nullptr, P.items, smem, full0, threadIdx.x);
  for (int n = 0; n < DFG_STAGES - 1; ++n) F.step();
  DfgRing R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(P.nzero);
  C.vst = P.vec_ok != 0;
  for (long long item = blockIdx.x; item < P.items; item += gridDim.x) dfg_consume_tile(P, item, R, C, warp, lane, F);
}

// All blocks of a device in one launch on the cp.async ring (packed ghost
// shells, the paper's VisIt blocks, L315): per-block DfgParams in global
// memory, first[b] = first item of block b, first[nb] = total.
struct DfgTileMulti {
  const DfgParams* blocks;
  const long long* first;
  int nb;
};

extern "C" __global__ void __launch_bounds__(DFG_NCW * 32, DFG_CTAS)
    dfg_fused_tile_multi(const __grid_constant__ DfgTileMulti M) {
  const unsigned smem = dfg_ring_init(DFG_NCW * 32);
  const unsigned full0 = smem + DFG_STAGES * DFG_STAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const long long total = M.first[M.nb];
  DfgFill F;
  F.init(M.blocks, M.first, total, smem, full0, threadIdx.x);
  for (int n = 0; n < DFG_STAGES - 1; ++n) F.step();
  DfgRing R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(M.blocks[0].nzero);
  int b = 0;
  for (long long item = blockIdx.x; item < total; item += gridDim.x) {
    while (item >= M.first[b + 1]) ++b;
    C.vst = M.blocks[b].vec_ok != 0;
    dfg_consume_tile(M.blocks[b], item - M.first[b], R, C, warp, lane, F);
  }
}

#if DFG_ROWS_KERNEL
// ---------------------------------------------------------------- rows
// The tile kernel's layouts (packed VisIt ghost shells, rows that are not a
// multiple of 16 bytes) with the TMA engine doing the loads.  A tensor map
// needs 16-byte global strides and 16-byte-aligned box starts, which a row
// pitch of 194 floats breaks -- but only from row to row: the rows whose
// byte offset y * px * sizeof(T) has the same residue mod 16 form a CLASS,
// and the rows of one class are a regular 3-D tensor with stride
// P * px * sizeof(T), a multiple of 16 (P = the period of the residues: 1, 2
// or 4 rows).  So the producer loads, per field and plane, one box per class
// (2 requests for a 194-float pitch, 4 for an odd pitch): class c's map
// starts at the field base + (c px T) rounded down to 16 bytes (o_c elements
// before row c's first element), its box at the class column of tile column
// HX-1 (the first one read) rounded down to a 16-byte boundary, so every row
// of class c lands shifted by m_c = (x0 + o_c + HX - 1) mod VEC; the box is
// the halo'd tile row wide (TX + 2 VEC), all a row's reads need.
// Consumers read the boxes as they are, with full-warp row ownership (lane l
// owns the cells l + 32 m of each of its RPW rows, below), so every
// shared-memory access of a warp is 32 consecutive 4/8-byte words of one row
// -- conflict-free at any shift -- and the x neighbours are plain loads at
// +-1 element.  Stores are fully coalesced (consecutive lanes, consecutive
// cells).  Mesh-end rules of reading R1: clamped rows in y (as the TMA
// kernel); in x a FIXUP warp writes, once TMA has landed a stage, the first
// / last global cell of every row into the slot its x-1 / x+1 reads, then
// releases the stage to the consumers ("ready" barriers), so the consumers
// carry no x-end code at all.
// Preconditions (host): 16-byte aligned field bases and plane strides, and
// at least P rows per plane.
// Two planes per box: a box of this size (a few KB) costs the TMA unit a
// near-fixed ~240 cycles (tools/tma_rate.cu: 76x16x1 boxes deliver 20 B per
// SM-cycle, 72x13x2 ones 31), so every box spans planes q and q+1 and a ring
// stage holds two planes (slot 0 / slot 1); P x fields boxes per TWO planes.
// box width: the halo'd tile row.  A box starts at the aligned column at or
// below tile column HX-1 (the first one read), so the cells read span at
// most VEC-1 + TX + 2 <= TX + 2 VEC columns from it
#define DFG_SBW DFG_ROWW
#define DFG_SROWS_ALLOC (DFG_ROWS + 3)   // P boxes of ceil(ROWS / P) rows, P <= 4
// class boxes (two planes each) start on 128-byte boundaries (TMA destination alignment)
#define DFG_STILE_BYTES ((2 * DFG_SBW * DFG_SROWS_ALLOC * (int)sizeof(DFG_T) + 127) / 128 * 128 + 4 * 128)
#define DFG_SSTAGE_BYTES (DFG_STILE_BYTES * DFG_NTF)
typedef DfgRingT<DFG_SSTAGE_BYTES, DFG_RSTAGES> DfgRingS;

// host image: runtime.cpp rows_blob (same order, 64-byte aligned maps):
// map[f * 4 + c] = class c of field f
struct DfgRowsInfo {
  int P;      // rows per period of the 16-byte residues (1, 2 or 4)
  int BR;     // box rows: ceil(ROWS / P)
  int o[4];   // o_c: elements between class c's map origin and its rows' first element
  int lgP;    // log2 P
  // one plane of a class box (the offset of slot 1), a two-plane box, its smem stride
  __device__ __forceinline__ unsigned slot() const { return (unsigned)(DFG_SBW * BR * (int)sizeof(DFG_T)); }
  __device__ __forceinline__ unsigned box() const { return 2u * slot(); }
  __device__ __forceinline__ unsigned cstride() const { return (box() + 127u) & ~127u; }
};
struct DfgRowsParams {
  DfgTmap map[DFG_NF_ * 4];
  DfgRowsInfo ri;
  int pad[9];
  DfgParams p;
};

// geometry of an item (the tile kernel's), shared by producer and consumers
struct DfgRowsItem {
  long long kb, ke;
  int x0, y0, tx, ty;
  __device__ __forceinline__ DfgRowsItem(const DfgParams& p, long long item) {
    tx = (int)(item % p.tiles_x);
    const long long rest = item / p.tiles_x;
    ty = (int)(rest % p.tiles_y);
    const long long zc = rest / p.tiles_y;
    kb = p.kbeg + zc * p.kz;
    ke = min(kb + (long long)p.kz, p.kend);
    x0 = tx * DFG_TX - DFG_HX + (int)p.gx;  // input column of tile column 0
    y0 = ty * DFG_TH - 1 + (int)p.gy;       // input row of tile row 0
  }
  // first tile row of class c (rows y = c mod P), and the start of its box:
  // the aligned map column and the class row index (may be -1)
  __device__ __forceinline__ int first(const DfgRowsInfo& ri, int c) const { return (c - y0) & (ri.P - 1); }
  __device__ __forceinline__ int bx(const DfgRowsInfo& ri, int c) const {
    const int v = x0 + ri.o[c] + DFG_HX - 1;  // class column of tile column HX-1
    return v - (v & (DFG_VEC - 1));  // floor to a multiple of VEC (v may be negative)
  }
  __device__ __forceinline__ int by(const DfgRowsInfo& ri, int c) const {
    return (y0 + first(ri, c) - c) >> ri.lgP;  // exact: y0 + first - c is a multiple of P
  }
  // smem byte offset (in a field tile, slot 0) of tile column 0 of tile row r
  // (tile column HX-1 lands at element m of its box row, so column 0 may lie
  // before the row: only columns >= HX-1 are ever read)
  __device__ __forceinline__ unsigned row_col0(const DfgRowsInfo& ri, int r) const {
    const int c = (y0 + r) & (ri.P - 1);
    const int m = (x0 + ri.o[c] + DFG_HX - 1) & (DFG_VEC - 1);
    return (unsigned)((int)c * (int)ri.cstride() +
                      (((r - first(ri, c)) >> ri.lgP) * DFG_SBW + m - (DFG_HX - 1)) * (int)sizeof(DFG_T));
  }
};

// Producer (one lane): per stage, one two-plane TMA box per (field, row
// class): planes q, q + 1 for q = kb-1, kb+1, ... (the item's kz + 2 planes,
// the last stage possibly half used).  Planes past the buffer ends (the
// global ends of a mesh without ghost planes) are zero-filled by TMA and
// never read: the consumers take the one-sided neighbours of R1 from the
// owned plane instead (dfg_consume_rows).
__device__ __forceinline__ void dfg_produce_rows(const DfgRowsParams& RP, long long item, DfgRingS& W) {
  const DfgParams& p = RP.p;
  const DfgRowsInfo& ri = RP.ri;
  const DfgRowsItem I(p, item);
  const unsigned box = ri.box(), cs = ri.cstride();
  int bxc[4], byc[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    bxc[c] = c < ri.P ? I.bx(ri, c) : 0;
    byc[c] = c < ri.P ? I.by(ri, c) : 0;
  }
  for (long long q = I.kb - 1; q <= I.ke; q += 2) {
    dfg_mbar_wait(W.full + DfgRingS::kEmpty, W.phase ^ 1u, 0x100000u);
    dfg_mbar_expect_tx(W.full, (unsigned)(DFG_NTF * ri.P) * box);
    const int zl = (int)(q - p.k0 + p.ghost);
#pragma unroll
    for (int f = 0; f < DFG_NTF; ++f)
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (c < ri.P)
          dfg_tma_load3(W.tile + f * DFG_STILE_BYTES + c * cs, &RP.map[f * 4 + c], W.full, bxc[c], byc[c], zl);
    W.advance();
  }
}

// Cell ownership: a warp owns RPW tile rows of 32 VEC / RPW cells; lane l
// owns, in each of its rows, the cells l + 32 m (m < CPR = VEC / RPW), so
// every shared-memory access of the warp is 32 consecutive words of ONE row
// (conflict-free at any shift).  Thread cell k (0 .. VEC-1) = row k / CPR,
// cell l + 32 (k mod CPR).
#define DFG_CPR (DFG_VEC / DFG_RPW)
// per-item constants of a consumer thread: smem byte offsets (in a field
// tile) of its first cell in each of its rows and of that cell's y-1 / y+1
// neighbours (clamped at the global ends).  Between the thread's own rows the
// y neighbours come from registers (the centres).
struct DfgColS {
  unsigned oc[DFG_RPW], om[DFG_RPW], op[DFG_RPW];
  DFG_T ndy[DFG_RPW], ry[DFG_RPW];  // y spacing entries of each of the thread's rows
};
#define DFG_KREADY (16u * DFG_RSTAGES)  // ready[s] = full[s] + 16 * stages (fixup warp -> consumers)

__device__ __forceinline__ void dfg_sts1(unsigned addr, DFG_T v) {
  DFG_SMEM_CHECK(addr, (unsigned)sizeof(DFG_T));
#if DFG_VEC == 4
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
#else
  asm volatile("st.shared.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
#endif
}

// One z-plane: slot `sg` of the stage R points at.  Its z+1 neighbour is
// slot 1 of the same stage (sg 0) or slot 0 of the next one (sg 1: wait for
// it, and release this stage after the plane); `zend`: the last plane of
// the mesh, whose z+1 is itself (R1).
template <int ZM, int ZC, int ZN>
__device__ __forceinline__ void dfg_plane_rows(const DfgCol& C, const DfgColS& Q, DfgRingS& R, unsigned& sg,
                                               unsigned pslot, DFG_T (&zq)[3][DFG_NSF][DFG_VEC], DFG_T*& outp,
                                               unsigned plane, int rowpitch, const DFG_T*& tzd, const DFG_T*& tzr,
                                               bool zend, unsigned wb) {
  constexpr unsigned TS = (unsigned)sizeof(DFG_T), ST = 32 * TS;  // cell stride within a row
  const unsigned cur = R.tile + (sg ? pslot : 0u);
  // y neighbours before the wait for the next stage (as the TMA kernel; fp64:
  // after it, its doubles need the registers), x neighbours after it
  DFG_T xm[DFG_NSF][DFG_VEC], xp[DFG_NSF][DFG_VEC], ym[DFG_NSF][DFG_VEC], yp[DFG_NSF][DFG_VEC];
  auto load_y = [&]() {
#pragma unroll
    for (int f = 0; f < DFG_NSF; ++f) {
      const unsigned t = cur + f * DFG_STILE_BYTES;
#pragma unroll
      for (int k = 0; k < DFG_VEC; ++k) {
        const int q = k / DFG_CPR;
        if (q == 0) ym[f][k] = dfg_lds1(t + Q.om[0] + (k % DFG_CPR) * ST);
        else ym[f][k] = zq[ZC][f][k - DFG_CPR];  // the row above is this thread's (never a global end)
        // the row below: this thread's next row (a row past the global end
        // holds this row's centres: its offsets are clamped, R1)
        if (q == DFG_RPW - 1) yp[f][k] = dfg_lds1(t + Q.op[q] + (k % DFG_CPR) * ST);
        else yp[f][k] = zq[ZC][f][k + DFG_CPR];
      }
    }
  };
#if DFG_VEC == 4
  load_y();
#endif
  // the stage after R's (ring order), waited for by a slot-1 plane
  const bool wrap = R.stage + 1 == DFG_RSTAGES;
  unsigned nxt = cur + pslot;
  if (sg) {
    dfg_mbar_wait((wrap ? R.full0 : R.full + 8u) + wb, R.phase ^ (wrap ? 1u : 0u), 0x100000u);
    nxt = wrap ? R.tile0 : R.tile + DFG_SSTAGE_BYTES;
  }
  if (zend) nxt = cur;
#if DFG_VEC == 2
  load_y();
#endif
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) {
    const unsigned t = cur + f * DFG_STILE_BYTES;
#pragma unroll
    for (int k = 0; k < DFG_VEC; ++k) {
      const unsigned c = t + Q.oc[k / DFG_CPR] + (k % DFG_CPR) * ST;
      xm[f][k] = dfg_lds1(c - TS);
      xp[f][k] = dfg_lds1(c + TS);
    }
  }
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
    for (int k = 0; k < DFG_VEC; ++k)
      zq[ZN][f][k] = dfg_lds1(nxt + f * DFG_STILE_BYTES + Q.oc[k / DFG_CPR] + (k % DFG_CPR) * ST);
  dfg2 s[DFG_NPAIR][DFG_NSF][7], gn[DFG_NPAIR][DFG_NSF][3];
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f) {
#pragma unroll
    for (int h = 0; h < DFG_NPAIR; ++h) {
      const int a = h * DFG_LANES, b = h * DFG_LANES + DFG_LANES - 1;
      s[h][f][0] = dfg2_mk(zq[ZC][f][a], zq[ZC][f][b]);
      s[h][f][1] = dfg2_mk(xm[f][a], xm[f][b]);
      s[h][f][2] = dfg2_mk(xp[f][a], xp[f][b]);
      s[h][f][3] = dfg2_mk(ym[f][a], ym[f][b]);
      s[h][f][4] = dfg2_mk(yp[f][a], yp[f][b]);
      s[h][f][5] = dfg2_mk(zq[ZM][f][a], zq[ZM][f][b]);
      s[h][f][6] = dfg2_mk(zq[ZN][f][a], zq[ZN][f][b]);
      gn[h][f][0] = dfg2_sub(s[h][f][2], s[h][f][1], C.Z);
      gn[h][f][1] = dfg2_sub(s[h][f][4], s[h][f][3], C.Z);
      gn[h][f][2] = dfg2_sub(s[h][f][6], s[h][f][5], C.Z);
    }
  }
  const dfg2 ndz = dfg2_splat(__ldg(tzd)), rz = dfg2_splat(__ldg(tzr));
  ++tzd;
  ++tzr;
  dfg2 p[DFG_NPAIR][DFG_NPF_];
#pragma unroll
  for (int f = 0; f < DFG_NPF; ++f) {
    DFG_T pv[DFG_VEC];
#pragma unroll
    for (int k = 0; k < DFG_VEC; ++k)
      pv[k] = dfg_lds1(cur + (DFG_NSF + f) * DFG_STILE_BYTES + Q.oc[k / DFG_CPR] + (k % DFG_CPR) * ST);
#pragma unroll
    for (int h = 0; h < DFG_NPAIR; ++h) p[h][f] = dfg2_mk(pv[h * DFG_LANES], pv[h * DFG_LANES + DFG_LANES - 1]);
  }
  dfg2 o[DFG_NPAIR][DFG_OUTW];
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h)
    dfg_body(s[h], gn[h], p[h], C.ndx[h], C.rx[h],
             dfg2_mk(Q.ndy[(h * DFG_LANES) / DFG_CPR], Q.ndy[(h * DFG_LANES + DFG_LANES - 1) / DFG_CPR]),
             dfg2_mk(Q.ry[(h * DFG_LANES) / DFG_CPR], Q.ry[(h * DFG_LANES + DFG_LANES - 1) / DFG_CPR]), ndz, rz, C.Z,
             o[h]);
  // cell k at outp + row(k) * rowpitch + 32 (k mod CPR); bit k of nvalid: valid
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h)
#pragma unroll
    for (int l = 0; l < DFG_LANES; ++l) {
      const int k = h * DFG_LANES + l;
      if ((C.nvalid >> k) & 1) {
        DFG_T* d = outp + ((k / DFG_CPR) * rowpitch + 32 * (k % DFG_CPR)) * DFG_OUTW;
#pragma unroll
        for (int w = 0; w < DFG_OUTW; ++w) __stcs(d + w, dfg2_get(o[h][w], l));
      }
    }
  outp += (size_t)plane * DFG_OUTW;
  if (sg) {
    dfg_mbar_arrive(R.full + DfgRingS::kEmpty);  // both planes done (every consumer thread, count NCW*32)
    R.advance();
  }
  sg ^= 1u;
}

__device__ __forceinline__ void dfg_consume_rows(const DfgRowsParams& RP, long long item, DfgRingS& R, DfgCol& C,
                                                 int warp, int lane) {
  const DfgParams& P = RP.p;
  const DfgRowsInfo& ri = RP.ri;
  const DfgRowsItem I(P, item);
  const unsigned plane = (unsigned)(P.nx * P.ny);  // < 2^32 (host precondition)
  const int r0 = 1 + warp * DFG_RPW;                   // tile row of this thread's row 0
  const long long i = (long long)I.tx * DFG_TX + lane;  // cell of k = 0 (row 0)
  const long long j0 = (long long)I.ty * DFG_TH + warp * DFG_RPW;
  const unsigned TS = (unsigned)sizeof(DFG_T);
  const unsigned cb = (unsigned)(DFG_HX + lane) * TS;  // tile column of cell m = 0
  DfgColS Q;
  C.nvalid = 0;
#pragma unroll
  for (int k = 0; k < DFG_VEC; ++k) {
    const long long ik = i + 32 * (k % DFG_CPR), jk = j0 + k / DFG_CPR;
    C.nvalid |= (ik < P.nx && jk < P.ny ? 1 : 0) << k;
  }
#pragma unroll
  for (int h = 0; h < DFG_NPAIR; ++h) {
    const int ka = h * DFG_LANES, kb = h * DFG_LANES + DFG_LANES - 1;
    const long long a = min(P.i0 + i + 32 * (ka % DFG_CPR), P.NX - 1);
    const long long b = min(P.i0 + i + 32 * (kb % DFG_CPR), P.NX - 1);
    C.ndx[h] = dfg2_mk(__ldg(P.tx + DFG_NDSEG_X * P.NX + a), __ldg(P.tx + DFG_NDSEG_X * P.NX + b));
    C.rx[h] = dfg2_mk(__ldg(P.tx + P.NX + a), __ldg(P.tx + P.NX + b));
  }
#pragma unroll
  for (int q = 0; q < DFG_RPW; ++q) {
    const long long yq = P.j0 + min(j0 + q, P.ny - 1);
    Q.ndy[q] = __ldg(P.ty + DFG_NDSEG_Y * P.NY + yq);
    Q.ry[q] = __ldg(P.ty + P.NY + yq);
  }
#pragma unroll
  for (int q = 0; q < DFG_RPW; ++q) {
    // one-sided differences only at the GLOBAL mesh ends (reading R1)
    const long long jg = P.j0 + j0 + q;
    const int r = r0 + q;
    Q.oc[q] = I.row_col0(ri, r) + cb;
    Q.om[q] = (jg == 0) ? Q.oc[q] : I.row_col0(ri, r - 1) + cb;
    Q.op[q] = (jg >= P.NY - 1) ? Q.oc[q] : I.row_col0(ri, r + 1) + cb;
    // a row past the global end (never stored) reads the row above: the
    // y+1 of the last global row is then itself, from registers (R1)
    if (q > 0 && jg > P.NY - 1) Q.oc[q] = Q.oc[q - 1];
  }
  DFG_T* outp = P.out + ((I.kb - P.k0) * (long long)plane + min(j0, P.ny - 1) * P.nx + min(i, P.nx - 1)) * DFG_OUTW;
  const DFG_T* tzd = P.tz + DFG_NDSEG_Z * P.NZ + I.kb;  // -d and 1/d of the plane's z spacing
  const DFG_T* tzr = P.tz + P.NZ + I.kb;
  constexpr unsigned ST = 32 * (unsigned)sizeof(DFG_T);
  const unsigned pslot = ri.slot();

  // stage 0 of the item: planes kb-1 (slot 0) and kb (slot 1).  At the
  // global z start the z-1 neighbour of plane 0 is plane 0 itself (R1).
  // an item holding a global x end waits for the fixup warp ("ready"), the
  // others take the stage as soon as TMA has landed it ("full")
  const long long tl = P.NX - 1 - P.i0 - (long long)I.tx * DFG_TX;
  const unsigned wb = ((P.i0 == 0 && I.tx == 0) || (P.i0 + P.nx == P.NX && tl >= 0 && tl < DFG_TX)) ? DFG_KREADY : 0u;
  DFG_T zq[3][DFG_NSF][DFG_VEC];
  dfg_mbar_wait(R.full + wb, R.phase, 0x100000u);
  const unsigned pre = R.tile + (I.kb == 0 ? pslot : 0u);
#pragma unroll
  for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
    for (int k = 0; k < DFG_VEC; ++k) {
      zq[0][f][k] = dfg_lds1(pre + f * DFG_STILE_BYTES + Q.oc[k / DFG_CPR] + (k % DFG_CPR) * ST);
      zq[1][f][k] = dfg_lds1(R.tile + pslot + f * DFG_STILE_BYTES + Q.oc[k / DFG_CPR] + (k % DFG_CPR) * ST);
    }
  unsigned sg = 1u;
  const int n = (int)(I.ke - I.kb);
  const int last = I.ke == P.NZ ? n - 1 : -1;  // the mesh's last plane (z+1 = itself, R1)
  int t = 0;
  for (; t + 3 <= n; t += 3) {
    dfg_plane_rows<0, 1, 2>(C, Q, R, sg, pslot, zq, outp, plane, (int)P.nx, tzd, tzr, t == last, wb);
    dfg_plane_rows<1, 2, 0>(C, Q, R, sg, pslot, zq, outp, plane, (int)P.nx, tzd, tzr, t + 1 == last, wb);
    dfg_plane_rows<2, 0, 1>(C, Q, R, sg, pslot, zq, outp, plane, (int)P.nx, tzd, tzr, t + 2 == last, wb);
  }
  if (t < n) {
    dfg_plane_rows<0, 1, 2>(C, Q, R, sg, pslot, zq, outp, plane, (int)P.nx, tzd, tzr, t == last, wb);
    if (t + 1 < n) dfg_plane_rows<1, 2, 0>(C, Q, R, sg, pslot, zq, outp, plane, (int)P.nx, tzd, tzr, t + 1 == last, wb);
  }
  // the stage holding plane ke (the item's post-plane) is read for its centre only
  dfg_mbar_arrive(R.full + DfgRingS::kEmpty);
  R.advance();
}

// Fixup warp (R1 in x): per stage, once TMA has landed it, the first /
// last GLOBAL cell of every owned tile row is copied into the slot its x-1 /
// x+1 neighbour is read from (both planes, every stencil field), then the
// stage goes to the consumers (ready).  Every stage passes through here, so
// the ready barriers advance exactly once per lap, like full.
__device__ __forceinline__ void dfg_fixup_rows(const DfgRowsParams& RP, long long item, DfgRingS& W, int lane) {
  const DfgParams& p = RP.p;
  const DfgRowsInfo& ri = RP.ri;
  const DfgRowsItem I(p, item);
  constexpr unsigned TS = (unsigned)sizeof(DFG_T);
  const bool first = p.i0 == 0 && I.tx == 0;                   // global column 0 at tile column HX
  const long long tl = p.NX - 1 - p.i0 - (long long)I.tx * DFG_TX;  // tile offset of the global last column
  const bool last = p.i0 + p.nx == p.NX && tl >= 0 && tl < DFG_TX;  // this block holds the global last column
  const unsigned pslot = ri.slot();
  for (long long q = I.kb - 1; q <= I.ke; q += 2) {
    dfg_mbar_wait(W.full, W.phase, 0x100000u);
    if (first || last) {
#pragma unroll 1
      for (int r = 1 + lane; r <= DFG_TH; r += 32) {
        const unsigned o = W.tile + I.row_col0(ri, r);
#pragma unroll
        for (int f = 0; f < DFG_NSF; ++f)
#pragma unroll
          for (int sl = 0; sl < 2; ++sl) {
            const unsigned t = o + f * DFG_STILE_BYTES + (sl ? pslot : 0u);
            if (first) dfg_sts1(t + (DFG_HX - 1) * TS, dfg_lds1(t + DFG_HX * TS));
            if (last) dfg_sts1(t + (unsigned)(DFG_HX + tl + 1) * TS, dfg_lds1(t + (unsigned)(DFG_HX + tl) * TS));
          }
      }
      // these generic-proxy writes precede the TMA (async-proxy) refill of the
      // stage a lap later: fence them into the async proxy's order, then the
      // ready -> empty barrier chain orders them before the producer's copy
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
    }
    if (lane == 0) dfg_mbar_arrive(W.full + DFG_KREADY);  // release: the slots are written
    W.advance();
  }
}

extern "C" __global__ void __launch_bounds__((DFG_NCW + 2) * 32, DFG_CTAS)
    dfg_fused_rows(const __grid_constant__ DfgRowsParams RP) {
  const unsigned smem = dfg_ring_init(1, DFG_SSTAGE_BYTES, DFG_RSTAGES, DFG_NCW * 32, true);
  const unsigned full0 = smem + DFG_RSTAGES * DFG_SSTAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  if (warp == DFG_NCW + 1) {
    DfgRingS W{smem, full0, 0u, 0, smem, full0};
    for (long long item = blockIdx.x; item < RP.p.items; item += gridDim.x) dfg_fixup_rows(RP, item, W, lane);
    return;
  }
  if (warp == DFG_NCW) {
    if (lane == 0) {
      for (int f = 0; f < DFG_NTF * 4; ++f)
        if ((f & 3) < RP.ri.P)
          asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<unsigned long long>(&RP.map[f])) : "memory");
      DfgRingS W{smem, full0, 0u, 0, smem, full0};
      for (long long item = blockIdx.x; item < RP.p.items; item += gridDim.x) dfg_produce_rows(RP, item, W);
    }
    return;
  }
  DfgRingS R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(RP.p.nzero);
  for (long long item = blockIdx.x; item < RP.p.items; item += gridDim.x) dfg_consume_rows(RP, item, R, C, warp, lane);
}

// several meshes in one launch: DfgRowsParams images in global memory
struct DfgRowsMulti {
  const DfgRowsParams* blocks;
  const long long* first;
  int nb;
};

extern "C" __global__ void __launch_bounds__((DFG_NCW + 2) * 32, DFG_CTAS)
    dfg_fused_rows_multi(const __grid_constant__ DfgRowsMulti M) {
  const unsigned smem = dfg_ring_init(1, DFG_SSTAGE_BYTES, DFG_RSTAGES, DFG_NCW * 32, true);
  const unsigned full0 = smem + DFG_RSTAGES * DFG_SSTAGE_BYTES;
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const long long total = M.first[M.nb];
  int b = 0;
  if (warp == DFG_NCW + 1) {
    DfgRingS W{smem, full0, 0u, 0, smem, full0};
    for (long long item = blockIdx.x; item < total; item += gridDim.x) {
      while (item >= M.first[b + 1]) ++b;
      dfg_fixup_rows(M.blocks[b], item - M.first[b], W, lane);
    }
    return;
  }
  if (warp == DFG_NCW) {
    if (lane == 0) {
      DfgRingS W{smem, full0, 0u, 0, smem, full0};
      for (long long item = blockIdx.x; item < total; item += gridDim.x) {
        while (item >= M.first[b + 1]) ++b;
        dfg_produce_rows(M.blocks[b], item - M.first[b], W);
      }
    }
    return;
  }
  DfgRingS R{smem, full0, 0u, 0, smem, full0};
  DfgCol C;
  C.Z = dfg2_splat(M.blocks[0].p.nzero);
  // the block index is found again per item (a short search in global
  // memory) rather than kept live across the consumer loop: registers
  for (long long item = blockIdx.x; item < M.first[M.nb]; item += gridDim.x) {
    int bb = 0;
    while (item >= M.first[bb + 1]) ++bb;
    dfg_consume_rows(M.blocks[bb], item - M.first[bb], R, C, warp, lane);
  }
}
#endif  // DFG_ROWS_KERNEL
#endif
