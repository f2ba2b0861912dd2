// Microbenchmark: FP32 lane throughput of scalar FFMA vs paired FFMA2 /
// FADD2 on sm_100a (developer tool; numbers go to profiles/).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fma_micro tools/fma_micro.cu && /tmp/fma_micro
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;
constexpr int ACC = 8;

__global__ void k_ffma(float* out, float a, float b) {
  float acc[ACC];
  for (int i = 0; i < ACC; ++i) acc[i] = threadIdx.x * 1e-3f + i;
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < ACC; ++i) acc[i] = __fmaf_rn(acc[i], a, b);
  float s = 0;
  for (int i = 0; i < ACC; ++i) s += acc[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma2(float* out, float a, float b) {
  float2 acc[ACC];
  for (int i = 0; i < ACC; ++i) acc[i] = make_float2(threadIdx.x * 1e-3f + i, i * 0.5f);
  const float2 A = make_float2(a, a), B = make_float2(b, b);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < ACC; ++i) acc[i] = __ffma2_rn(acc[i], A, B);
  float s = 0;
  for (int i = 0; i < ACC; ++i) s += acc[i].x + acc[i].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_fadd2(float* out, float a, float b) {
  float2 acc[ACC];
  for (int i = 0; i < ACC; ++i) acc[i] = make_float2(threadIdx.x * 1e-3f + i, i * 0.5f);
  const float2 B = make_float2(b, b);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < ACC; ++i) acc[i] = __fadd2_rn(acc[i], B);
  float s = 0;
  for (int i = 0; i < ACC; ++i) s += acc[i].x + acc[i].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// mixed: 1 FFMA2 + 1 scalar FFMA per step (can the lite pipe run the scalar?)
__global__ void k_mix(float* out, float a, float b) {
  float2 acc[ACC / 2];
  float sc[ACC / 2];
  for (int i = 0; i < ACC / 2; ++i) {
    acc[i] = make_float2(threadIdx.x * 1e-3f + i, i * 0.5f);
    sc[i] = i;
  }
  const float2 A = make_float2(a, a), B = make_float2(b, b);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < ACC / 2; ++i) {
      acc[i] = __ffma2_rn(acc[i], A, B);
      sc[i] = __fmaf_rn(sc[i], a, b);
    }
  float s = 0;
  for (int i = 0; i < ACC / 2; ++i) s += acc[i].x + acc[i].y + sc[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <typename K>
void run(const char* name, K k, double lane_ops_per_step, float* d, int sms) {
  int blocks = sms * 8, threads = 256;
  k<<<blocks, threads>>>(d, 0.999f, 1e-3f);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 10; ++r) k<<<blocks, threads>>>(d, 0.999f, 1e-3f);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double ops = 10.0 * blocks * threads * double(ITERS) * lane_ops_per_step;
  double per_clk_sm = ops / (ms * 1e-3) / (clk * 1e3) / sms;
  printf("%-8s %8.3f ms  %8.1f Gflop-lanes/s  %6.1f lane-ops/clk/SM (at max clock %d MHz)\n", name, ms / 10,
         ops / (ms * 1e-3) / 1e9, per_clk_sm, clk / 1000);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float* d;
  cudaMalloc(&d, sizeof(float) * sms * 8 * 256);
  run("FFMA", k_ffma, ACC, d, sms);
  run("FFMA2", k_ffma2, 2 * ACC, d, sms);
  run("FADD2", k_fadd2, 2 * ACC, d, sms);
  run("MIX", k_mix, ACC / 2 * 3, d, sms);
  return 0;
}
