// Launchers of the per-primitive kernels (kernels.cu).  Sizes are element
// counts; vector arrays are AoS 4-wide.  All launches are asynchronous on `s`.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "lang.hpp"

namespace dfg {
namespace kern {

void binary(Op op, DType dt, const void* a, const void* b, void* o, long long n, cudaStream_t s);
void unary(Op op, DType dt, const void* a, void* o, long long n, cudaStream_t s);  // Neg, Sqrt
void select(DType dt, const void* c, const void* a, const void* b, void* o, long long n, cudaStream_t s);
void fill(DType dt, double v, void* o, long long n, cudaStream_t s);
void decompose(DType dt, const void* v4, int lane, void* o, long long n, cudaStream_t s);
void compose(DType dt, const void* const* in, int w, void* o4, long long n, cudaStream_t s);
// f: local plane 0 of T[nzl + 2*ghost][ny][nx]; tables d[n] then r[n]; tz global.
void grad3d(DType dt, const void* f, void* o4, const void* tx, const void* ty, const void* tz, long long nx,
            long long ny, long long nzl, long long NZ, long long k0, long long ghost, cudaStream_t s);

// Exhaustive check of the two-operation quotient for n fp32 divisors
// (DESIGN.md section 5): bad[k] = 1 unless, for all 2^23 significands
// a in [1, 2), RN(a*yh[k] + RN(a*yl[k])) == RN(a / d[k]).  Device pointers;
// bad must be zeroed by the caller.
void verify_div2(const float* d, const float* yh, const float* yl, int n, unsigned* bad, cudaStream_t s);

// Peer-halo probe block: kProbeRows rows of kProbeCols 32-bit words, word i =
// probe_word(i), placed kProbeOffset bytes into a mesh's flag allocation.
constexpr int kProbeRows = 32, kProbeCols = 64, kProbeOffset = 256;
inline uint32_t probe_word(uint32_t i) { return (i + 1u) * 2654435761u ^ 0x5bd1e995u; }
// One TMA load of the whole probe box through `map` (host copy of a
// CUtensorMap) into out[kProbeRows * kProbeCols] (device).
void tma_probe(const CUtensorMap* map, uint32_t* out, cudaStream_t s);

}  // namespace kern
}  // namespace dfg
