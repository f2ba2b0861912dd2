// TMA alignment probe (developer tool): does cp.async.bulk.tensor accept a
// box whose start coordinate is not a multiple of 16 bytes?
//   nvcc -gencode arch=compute_100a,code=sm_100a -o tma_probe tma_probe.cu -lcuda
//   ./tma_probe <rank 1|3> <x coordinate>
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

__global__ void probe(const __grid_constant__ CUtensorMap map, int rank, int x, int y, int z, float* out, int n) {
  __shared__ __align__(128) float buf[136 * 4];
  __shared__ __align__(8) unsigned long long bar;
  unsigned b = (unsigned)__cvta_generic_to_shared(&bar);
  unsigned d = (unsigned)__cvta_generic_to_shared(buf);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(n * 4));
    if (rank == 1)
      asm volatile("cp.async.bulk.tensor.1d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3}], [%2];"
                   ::"r"(d), "l"(&map), "r"(b), "r"(x) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
                   ::"r"(d), "l"(&map), "r"(b), "r"(x), "r"(y), "r"(z) : "memory");
  }
  unsigned done = 0;
  while (!done)
    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                 : "=r"(done) : "r"(b) : "memory");
  for (int i = threadIdx.x; i < n; i += blockDim.x) out[i] = buf[i];
}

int main(int argc, char** argv) {
  int rank = argc > 1 ? atoi(argv[1]) : 1;
  int x = argc > 2 ? atoi(argv[2]) : 3;
  const int nx = 67, ny = 5, nz = 3;  // nx * 4 B rows are NOT 16-byte multiples
  const int N = nx * ny * nz;
  std::vector<float> h(N);
  for (int i = 0; i < N; ++i) h[i] = float(i);
  float *g, *o;
  cudaMalloc(&g, N * 4);
  cudaMalloc(&o, 136 * 4 * 4);
  cudaMemcpy(g, h.data(), N * 4, cudaMemcpyHostToDevice);
  CUtensorMap map;
  CUresult r;
  int n;
  if (rank == 1) {
    cuuint64_t gd[1] = {cuuint64_t(N)};
    cuuint32_t box[1] = {136}, es[1] = {1};
    r = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 1, g, gd, nullptr, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    n = 136;
  } else {
    // a 68-wide padded row so the 3-D map is legal; start column x
    cuuint64_t gd[3] = {68, cuuint64_t(ny), cuuint64_t(nz)};
    cuuint64_t gs[2] = {68 * 4, 68 * 4 * ny};
    cuuint32_t box[3] = {16, 2, 1}, es[3] = {1, 1, 1};
    r = cuTensorMapEncodeTiled(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, g, gd, gs, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    n = 32;
  }
  if (r != CUDA_SUCCESS) { printf("encode failed %d\n", int(r)); return 2; }
  probe<<<1, 128>>>(map, rank, x, 1, 1, o, n);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("rank %d x %d: kernel error %s\n", rank, x, cudaGetErrorString(e)); return 1; }
  std::vector<float> got(n);
  cudaMemcpy(got.data(), o, n * 4, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < n; ++i) {
    float want;
    if (rank == 1) { long long gi = x + i; want = (gi < 0 || gi >= N) ? 0.f : h[gi]; }
    else { int col = x + i % 16, row = 1 + i / 16; want = (col < 0 || col >= 68) ? 0.f : float(68 * (row + ny * 1) + col); }
    if (rank == 3) { /* data at padded index: compare against 68-wide layout of the buffer */ }
    if (rank == 1 && got[i] != want) ++bad;
  }
  printf("rank %d x %d: ok, first %g %g %g, mismatches %d\n", rank, x, got[0], got[1], got[2], bad);
  return 0;
}
