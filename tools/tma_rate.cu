// TMA delivery-rate probe (developer tool): how fast does one SM's TMA unit
// fill a shared-memory ring with the box shapes the fused kernels use?
// One producer lane per CTA streams `boxes` boxes per stage into an S-stage
// ring (full/empty mbarriers); one consumer warp only waits and releases, so
// the time is the load path alone.  Grid = #SMs, each CTA walks its own
// tiles of a 3-D fp32 tensor (dims X x Y x Z, row pitch X floats, the
// stride of one "row class" = P rows: rows of one box are P rows apart).
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tma_rate tma_rate.cu -lcuda
//   ./tma_rate <box_w> <box_h> <box_d> <boxes per stage> <P> [stages]
// prints bytes per SM-cycle, cycles per box and aggregate GB/s.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>

struct alignas(64) Map { CUtensorMap m; };

__device__ __forceinline__ void mbar_init(unsigned b, unsigned n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(n) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned b, unsigned ph) {
  unsigned done = 0;
  while (!done)
    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                 : "=r"(done) : "r"(b), "r"(ph) : "memory");
}

__global__ void __launch_bounds__(64, 1) rate(const __grid_constant__ Map map, int bw, int bh, int bd, int nbox, int P,
                                              int S, int tiles_x, int tiles_y, int planes, unsigned stage_bytes,
                                              unsigned long long* cyc) {
  extern __shared__ __align__(1024) unsigned char smem[];
  const unsigned base = (unsigned)__cvta_generic_to_shared(smem);
  const unsigned bars = base + S * stage_bytes;  // full[s] = bars + 8s, empty[s] = bars + 8(S + s)
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(bars + 8 * s, 1);
      mbar_init(bars + 8 * (S + s), 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const unsigned box_bytes = (unsigned)(bw * bh * bd * 4);
  const int tile = blockIdx.x;
  const int tx = tile % tiles_x, ty = (tile / tiles_x) % tiles_y;
  const int steps = planes / bd;
  unsigned long long t0 = clock64();
  if (threadIdx.x == 0) {
    for (int i = 0; i < steps; ++i) {
      const int s = i % S;
      const unsigned ph = (i / S) & 1;
      mbar_wait(bars + 8 * (S + s), ph ^ 1);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bars + 8 * s),
                   "r"(box_bytes * nbox) : "memory");
      for (int b = 0; b < nbox; ++b) {
        // box b: row class b % P (rows b % P, b % P + P, ...), field b / P
        const int y = ty * bh;  // class-row index of the tile (every class box reads class 0: L2-hot re-reads)
        const int z = (b / P) * planes + i * bd;
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
            ::"r"(base + s * stage_bytes + b * ((box_bytes + 127) / 128 * 128)), "l"(&map), "r"(bars + 8 * s),
            "r"(tx * (bw - 8)), "r"(y), "r"(z)
            : "memory");
      }
    }
  } else if (threadIdx.x >= 32) {
    for (int i = 0; i < steps; ++i) {
      const int s = i % S;
      mbar_wait(bars + 8 * s, (i / S) & 1);
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bars + 8 * (S + s)) : "memory");
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = clock64() - t0;
}

int main(int argc, char** argv) {
  if (argc < 6) { printf("usage: tma_rate bw bh bd boxes P [stages]\n"); return 2; }
  const int bw = atoi(argv[1]), bh = atoi(argv[2]), bd = atoi(argv[3]), nbox = atoi(argv[4]), P = atoi(argv[5]);
  const int S = argc > 6 ? atoi(argv[6]) : 6;
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  // fields = nbox / P, each X x Y x planes fp32, stacked along z
  const int fields = (nbox + P - 1) / P, planes = 240;
  const long long X = 1024, Y = 1024;
  const long long Z = (long long)planes * fields;
  float* g;
  if (cudaMalloc(&g, X * Y * Z * 4) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMemset(g, 0, X * Y * Z * 4);
  Map map;
  // class view: rows P apart (stride P * X floats), dims {X, Y / P, Z}
  cuuint64_t gd[3] = {cuuint64_t(X), cuuint64_t(Y / P), cuuint64_t(Z)};
  cuuint64_t gs[2] = {cuuint64_t(X * 4 * P), cuuint64_t(X * Y * 4)};
  cuuint32_t box[3] = {cuuint32_t(bw), cuuint32_t(bh), cuuint32_t(bd)}, es[3] = {1, 1, 1};
  CUresult r = cuTensorMapEncodeTiled(&map.m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, g, gd, gs, box, es,
                                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { printf("encode failed %d\n", int(r)); return 1; }
  const unsigned box_bytes = bw * bh * bd * 4, stage_bytes = nbox * ((box_bytes + 127) / 128 * 128);
  const size_t smem = size_t(S) * stage_bytes + 16 * S;
  if (smem > 227 * 1024) { printf("smem %zu too large\n", smem); return 1; }
  cudaFuncSetAttribute(rate, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  const int tiles_x = int(X / (bw - 8)), tiles_y = int(Y / P / bh);
  unsigned long long* cyc;
  cudaMalloc(&cyc, sms * 8);
  for (int rep = 0; rep < 2; ++rep) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    rate<<<sms, 64, smem>>>(map, bw, bh, bd, nbox, P, S, tiles_x, tiles_y, planes, stage_bytes, cyc);
    cudaEventRecord(e1);
    cudaError_t e = cudaEventSynchronize(e1);
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long* h = new unsigned long long[sms];
    cudaMemcpy(h, cyc, sms * 8, cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < sms; ++i) avg += double(h[i]) / sms;
    const double boxes = double(planes / bd) * nbox, bytes = boxes * box_bytes;
    if (rep == 1)
      printf("box %dx%dx%d x%d P%d S%d: %.1f B/SM-cycle, %.0f cycles/box, %.0f GB/s aggregate (%.3f ms)\n", bw, bh, bd,
             nbox, P, S, bytes / avg, avg / boxes, bytes * sms / (ms * 1e-3) / 1e9, ms);
    delete[] h;
  }
  return 0;
}
