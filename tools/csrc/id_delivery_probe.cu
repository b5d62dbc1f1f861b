// id_delivery_probe.cu -- does the row-id delivery cost L1 data-pipe throughput in the
// forward's gather?  (DESIGN.md §5.)  Model: a 512-B row costs 4 LSU data wavefronts, a row
// that misses L1 another ~4 (fill), and the id broadcast (one LDS.128 per 4 rows, split into 4
// quarter-warp phases) ~1 more.  Two gathers of the same zipf-like id stream over an
// L2-resident table, each warp summing its rows (consumed, like the forward):
//   bcast: every lane needs every id -- one broadcast LDS.128 per 4 rows, a row = 32 lanes x 16 B
//   quad : 4 lane groups of 8, each its own row stream -- one LDS.32 (4 distinct addresses)
//          per 4 rows, a row = 8 lanes x 4 x 16 B (4 LDG.128 per lane per row)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/csrc/id_delivery_probe tools/csrc/id_delivery_probe.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <cmath>
#include <vector>

#define CK(x)                                                                   \
  do {                                                                          \
    cudaError_t e = (x);                                                        \
    if (e != cudaSuccess) {                                                     \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
      exit(1);                                                                  \
    }                                                                           \
  } while (0)

constexpr int ROWB = 512;
constexpr int BATCH = 128;   // ids staged per warp per batch

__device__ __forceinline__ void ldg4(const char* p, float4& v) {
  asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
}
// L1::no_allocate: does a load that bypasses L1 allocation skip the fill wavefronts?
__device__ __forceinline__ void ldg4_na(const char* p, float4& v) {
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
}

// ids of this warp's batch -> shared (coalesced LDG + STS), then the gather
template <int WARPS, bool NA = false>
__global__ void __launch_bounds__(WARPS * 32) bcast_kernel(const char* __restrict__ table, const uint32_t* __restrict__ ids,
                                                           long n, float* out) {
  __shared__ __align__(16) uint32_t sid[WARPS][BATCH];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long gw = (long)blockIdx.x * WARPS + warp;
  const uint32_t* my = ids + gw * n;
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(&sid[warp][0]);
  float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  const char* base = table + lane * 16;
  for (long b = 0; b < n; b += BATCH) {
    __syncwarp();
#pragma unroll
    for (int k = 0; k < BATCH / 32; ++k) sid[warp][k * 32 + lane] = __ldg(my + b + k * 32 + lane);
    __syncwarp();
    float4 A[4], Bv[4];
    auto issue = [&](float4 (&r)[4], int j) {
      uint32_t x[4];
      asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3]) : "r"(sb + 4 * j) : "memory");
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        if (NA) ldg4_na(base + (size_t)x[u] * ROWB, r[u]);
        else ldg4(base + (size_t)x[u] * ROWB, r[u]);
      }
    };
    auto consume = [&](float4 (&r)[4]) {
#pragma unroll
      for (int u = 0; u < 4; ++u) { a0 += r[u].x; a1 += r[u].y; a2 += r[u].z; a3 += r[u].w; }
    };
    issue(A, 0);
#pragma unroll 1
    for (int j = 0; j < BATCH; j += 8) {
      issue(Bv, j + 4);
      consume(A);
      if (j + 8 < BATCH) issue(A, j + 8);
      consume(Bv);
    }
  }
  out[gw * 32 + lane] = a0 + a1 + a2 + a3;
}

template <int WARPS>
__global__ void __launch_bounds__(WARPS * 32) quad_kernel(const char* __restrict__ table, const uint32_t* __restrict__ ids,
                                                          long n, float* out) {
  __shared__ __align__(16) uint32_t sid[WARPS][BATCH];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int grp = lane >> 3, gl = lane & 7;
  const long gw = (long)blockIdx.x * WARPS + warp;
  const uint32_t* my = ids + gw * n;
  // group g walks the batch positions g*32 .. g*32+31 (its own stream)
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(&sid[warp][0]) + grp * (BATCH / 4) * 4;
  float acc[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) acc[i] = 0.f;
  const char* base = table + gl * 16;
  for (long b = 0; b < n; b += BATCH) {
    __syncwarp();
#pragma unroll
    for (int k = 0; k < BATCH / 32; ++k) sid[warp][k * 32 + lane] = __ldg(my + b + k * 32 + lane);
    __syncwarp();
    float4 A[4], Bv[4];
    auto issue = [&](float4 (&r)[4], int j) {   // row j of this group's stream
      uint32_t x;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(sb + 4 * j) : "memory");
      const char* rp = base + (size_t)x * ROWB;
#pragma unroll
      for (int k = 0; k < 4; ++k) ldg4(rp + k * 128, r[k]);
    };
    auto consume = [&](float4 (&r)[4]) {
#pragma unroll
      for (int k = 0; k < 4; ++k) { acc[4 * k] += r[k].x; acc[4 * k + 1] += r[k].y; acc[4 * k + 2] += r[k].z; acc[4 * k + 3] += r[k].w; }
    };
    issue(A, 0);
#pragma unroll 1
    for (int j = 0; j < BATCH / 4; j += 2) {
      issue(Bv, j + 1);
      consume(A);
      if (j + 2 < BATCH / 4) issue(A, j + 2);
      consume(Bv);
    }
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < 16; ++i) s += acc[i];
  out[gw * 32 + lane] = s;
}

template <typename F>
static float time_it(F f) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  f();
  CK(cudaDeviceSynchronize());
  cudaEventRecord(e0);
  for (int r = 0; r < 5; ++r) f();
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms / 5;
}

int main(int argc, char** argv) {
  const long rows = argc > 1 ? atol(argv[1]) : 2000000;
  const double s_exp = argc > 2 ? atof(argv[2]) : 1.05;   // zipf exponent (0: uniform)
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const long n = 4096;
  const long maxw = (long)sms * 64;
  char* table;
  uint32_t* ids;
  float* out;
  CK(cudaMalloc(&table, (size_t)rows * ROWB));
  CK(cudaMemset(table, 0, (size_t)rows * ROWB));
  CK(cudaMalloc(&ids, (size_t)maxw * n * 4));
  CK(cudaMalloc(&out, (size_t)maxw * 32 * 4));
  // zipf over ranks 1..rows by inverting the CDF, rank -> row by a fixed odd multiplier
  std::vector<double> cdf(rows);
  double acc = 0;
  for (long k = 0; k < rows; ++k) {
    acc += s_exp > 0 ? std::pow((double)(k + 1), -s_exp) : 1.0;
    cdf[k] = acc;
  }
  std::vector<uint32_t> h((size_t)maxw * n);
  uint64_t x = 88172645463325252ull;
  for (auto& v : h) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    const double u = (double)(x >> 11) * (1.0 / 9007199254740992.0) * acc;
    const long r = std::lower_bound(cdf.begin(), cdf.end(), u) - cdf.begin();
    v = (uint32_t)(((uint64_t)(r < rows ? r : rows - 1) * 2654435761ull) % (uint64_t)rows);
  }
  CK(cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice));
  printf("# rows %ld (%.1f MB), zipf %.2f, %ld rows per warp, %d SMs\n", rows, rows * ROWB / 1e6, s_exp, n, sms);
  for (int cps : {4, 5}) {
    const int grid = sms * cps;
    const double bytes = (double)grid * 8 * n * ROWB;
    float ms = time_it([&] { bcast_kernel<8><<<grid, 256>>>(table, ids, n, out); });
    CK(cudaGetLastError());
    printf("{\"variant\": \"bcast\", \"ctas_per_sm\": %d, \"ms\": %.4f, \"GBps\": %.1f}\n", cps, ms, bytes / (ms * 1e-3) / 1e9);
    ms = time_it([&] { bcast_kernel<8, true><<<grid, 256>>>(table, ids, n, out); });
    CK(cudaGetLastError());
    printf("{\"variant\": \"bcast_no_allocate\", \"ctas_per_sm\": %d, \"ms\": %.4f, \"GBps\": %.1f}\n", cps, ms, bytes / (ms * 1e-3) / 1e9);
    ms = time_it([&] { quad_kernel<8><<<grid, 256>>>(table, ids, n, out); });
    CK(cudaGetLastError());
    printf("{\"variant\": \"quad\", \"ctas_per_sm\": %d, \"ms\": %.4f, \"GBps\": %.1f}\n", cps, ms, bytes / (ms * 1e-3) / 1e9);
  }
  return 0;
}
