// synth_gen.cu -- device twins of synth/__init__.py's counter-based generators.
// Input generation only (no lookup, pooling or layout arithmetic of the method).
#include <cuda_runtime.h>
#include <stdint.h>

#include "synth.h"

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;
constexpr uint64_t S_TABLE = 0x7AB1E, S_POOL = 0x9001, S_INDEX = 0x1D3;

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t hash3(uint64_t stream, uint64_t seed, uint64_t a, uint64_t b) {
  uint64_t x = mix64(seed * kGolden + stream);
  x = mix64(x ^ a);
  return mix64(x + b);
}

__global__ void gen_table_kernel(void* w, int64_t rows, int32_t dim, int32_t wdtype, int32_t mode, uint64_t seed,
                                 int64_t t) {
  const int64_t n = rows * dim;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
    float v;
    if (mode == 2) {  // identity
      const int64_t i = e / dim;
      const int k = (int)(e - i * dim);
      int f;
      switch (k) {
        case 0: f = (int)(t & 255); break;
        case 1: f = (int)((t >> 8) & 255); break;
        case 2: f = (int)(i & 255); break;
        case 3: f = (int)((i >> 8) & 255); break;
        case 4: f = (int)((i >> 16) & 255); break;
        case 5: f = (int)((i >> 24) & 255); break;
        default: f = k & 255;
      }
      v = (float)f;
    } else {
      const uint64_t h = hash3(S_TABLE, seed, (uint64_t)t, (uint64_t)e);
      if (mode == 1) v = (float)((int)(h % 17ull) - 8);
      else if (wdtype == 0) v = (float)((int)(h >> 40) - (1 << 23)) * 0x1p-23f;
      else v = (float)((int)(h >> 56) - 128) * 0x1p-7f;
    }
    if (wdtype == 0) reinterpret_cast<float*>(w)[e] = v;
    else reinterpret_cast<uint16_t*>(w)[e] = (uint16_t)(__float_as_uint(v) >> 16);  // exact (values are bf16)
  }
}

__global__ void gen_lengths_kernel(int64_t* out, int64_t batch, uint64_t seed, int64_t t, int64_t pmin, int64_t pmax) {
  for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < batch; b += (int64_t)gridDim.x * blockDim.x) {
    if (pmin == pmax) out[b] = pmin;
    else out[b] = pmin + (int64_t)(hash3(S_POOL, seed, (uint64_t)t, (uint64_t)b) % (uint64_t)(pmax - pmin + 1));
  }
}

__global__ void gen_indices_kernel(int64_t* out, int64_t count, int64_t pos0, uint64_t seed, int64_t t, int64_t M,
                                   int32_t dist, const double* __restrict__ cdf, int64_t a, int64_t c) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < count; j += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = hash3(S_INDEX, seed, (uint64_t)t, (uint64_t)(pos0 + j));
    if (dist == 0) {
      out[j] = (int64_t)(h % (uint64_t)M);
    } else {
      const double u = (double)(h >> 11) * 0x1p-53;
      int64_t lo = 0, hi = M;  // numpy searchsorted(side='right'): first i with cdf[i] > u
      while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (__ldg(cdf + mid) <= u) lo = mid + 1; else hi = mid;
      }
      const int64_t k0 = lo < M - 1 ? lo : M - 1;
      out[j] = (a * k0 + c) % M;
    }
  }
}

int grid_for(int64_t n) {
  int64_t g = (n + 255) / 256;
  if (g > 148 * 32) g = 148 * 32;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace

extern "C" {

int synth_gen_table(void* w, int64_t rows, int32_t dim, int32_t wdtype, int32_t mode, uint64_t seed, int64_t t,
                    void* stream) {
  gen_table_kernel<<<grid_for(rows * dim), 256, 0, (cudaStream_t)stream>>>(w, rows, dim, wdtype, mode, seed, t);
  return (int)cudaGetLastError();
}

int synth_gen_lengths(int64_t* out, int64_t batch, uint64_t seed, int64_t t, int64_t pmin, int64_t pmax, void* stream) {
  gen_lengths_kernel<<<grid_for(batch), 256, 0, (cudaStream_t)stream>>>(out, batch, seed, t, pmin, pmax);
  return (int)cudaGetLastError();
}

int synth_gen_indices(int64_t* out, int64_t count, int64_t pos0, uint64_t seed, int64_t t, int64_t num_rows,
                      int32_t dist, const double* cdf, int64_t a, int64_t c, void* stream) {
  if (count <= 0) return 0;
  gen_indices_kernel<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(out, count, pos0, seed, t, num_rows, dist, cdf,
                                                                         a, c);
  return (int)cudaGetLastError();
}

}  // extern "C"
