// gather4_probe.cu -- how fast can the TMA engine gather random 512-B rows into shared memory
// (cp.async.bulk.tensor.2d ... tile::gather4: 4 rows per instruction), and what does consuming
// them with LDS cost?  The LSU gather's 19-20 TB/s on an L2-resident table is the L1 data
// pipe's limit for missing loads (4 data + 4 fill wavefronts per row), not necessarily L2's
// (DESIGN.md §11 probes); this measures the L2 -> SM rate of the async-proxy path.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/csrc/gather4_probe tools/csrc/gather4_probe.cu -lcuda
// Each warp streams its own id list: lane 0 arms stage s's mbarrier with 2 KB and issues one
// gather4 of 4 rows into it; K stages per warp are in flight; the warp waits on a stage, every
// lane reads its 16 B of each row (LDS.128) and adds, then lane 0 refills the stage.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
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
constexpr int D = ROWB / 4;

template <int K, int WARPS, bool CONSUME>
__global__ void __launch_bounds__(WARPS * 32) g4_kernel(const __grid_constant__ CUtensorMap tmap, const uint32_t* __restrict__ ids,
                                                        long n, float* out) {
  extern __shared__ __align__(1024) unsigned char smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(smem) + warp * K * 4 * ROWB;
  const uint32_t bars = (uint32_t)__cvta_generic_to_shared(smem) + WARPS * K * 4 * ROWB + warp * K * 8;
  if (lane == 0)
    for (int s = 0; s < K; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bars + 8 * s));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const long gw = (long)blockIdx.x * WARPS + warp;
  const uint32_t* my = ids + gw * n;
  auto issue = [&](int s, long i) {   // rows i .. i+3 of this warp's list into stage s
    const uint4 x = *reinterpret_cast<const uint4*>(my + i);
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bars + 8 * s), "r"(4 * ROWB) : "memory");
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(ring + s * 4 * ROWB),
        "l"(&tmap), "r"(0), "r"(x.x), "r"(x.y), "r"(x.z), "r"(x.w), "r"(bars + 8 * s)
        : "memory");
  };
  const long ng = n / 4;
  if (lane == 0)
    for (int s = 0; s < K && s < ng; ++s) issue(s, 4L * s);
  float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  for (long g = 0; g < ng; ++g) {
    const int s = (int)(g % K);
    const uint32_t ph = (uint32_t)((g / K) & 1);
    uint32_t done = 0;
    while (!done)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done)
                   : "r"(bars + 8 * s), "r"(ph)
                   : "memory");
    if (CONSUME) {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        float4 v;
        asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                     : "r"(ring + (s * 4 + u) * ROWB + lane * 16) : "memory");
        a0 += v.x; a1 += v.y; a2 += v.z; a3 += v.w;
      }
    }
    __syncwarp();
    if (lane == 0 && g + K < ng) issue(s, 4 * (g + K));
  }
  out[gw * 32 + lane] = a0 + a1 + a2 + a3;
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

template <int K, int WARPS, bool CONSUME>
static void run(const CUtensorMap& tm, const uint32_t* ids, long n, float* out, int sms, int cps) {
  const int grid = sms * cps;
  const size_t smem = (size_t)WARPS * K * (4 * ROWB + 8) + 1024;
  CK(cudaFuncSetAttribute(g4_kernel<K, WARPS, CONSUME>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const float ms = time_it([&] { g4_kernel<K, WARPS, CONSUME><<<grid, WARPS * 32, smem>>>(tm, ids, n, out); });
  CK(cudaGetLastError());
  const double bytes = (double)grid * WARPS * n * ROWB;
  printf("{\"variant\": \"gather4%s\", \"K\": %d, \"warps_per_cta\": %d, \"ctas_per_sm\": %d, \"ms\": %.4f, \"GBps\": %.1f}\n",
         CONSUME ? "" : "_noconsume", K, WARPS, cps, ms, bytes / (ms * 1e-3) / 1e9);
}

int main(int argc, char** argv) {
  const long rows = argc > 1 ? atol(argv[1]) : 100000;
  const double s_exp = argc > 2 ? atof(argv[2]) : 0.0;
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const long n = 4096;
  const long maxw = (long)sms * 64;
  float* table;
  uint32_t* ids;
  float* out;
  CK(cudaMalloc(&table, (size_t)rows * ROWB));
  CK(cudaMemset(table, 0, (size_t)rows * ROWB));
  CK(cudaMalloc(&ids, (size_t)maxw * n * 4));
  CK(cudaMalloc(&out, (size_t)maxw * 32 * 4));
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
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  auto encode = reinterpret_cast<CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                              const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                              CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill)>(fn);
  CUtensorMap tm;
  cuuint64_t dims[2] = {(cuuint64_t)D, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ROWB};
  cuuint32_t box[2] = {(cuuint32_t)D, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, table, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    fprintf(stderr, "encode failed %d\n", (int)r);
    return 1;
  }
  printf("# rows %ld (%.1f MB), zipf %.2f, %ld rows per warp, %d SMs\n", rows, rows * ROWB / 1e6, s_exp, n, sms);
  run<4, 8, true>(tm, ids, n, out, sms, 2);
  run<4, 8, false>(tm, ids, n, out, sms, 2);
  run<8, 8, true>(tm, ids, n, out, sms, 1);
  run<4, 16, true>(tm, ids, n, out, sms, 1);
  run<2, 16, true>(tm, ids, n, out, sms, 2);
  run<6, 8, true>(tm, ids, n, out, sms, 2);
  run<3, 8, true>(tm, ids, n, out, sms, 4);
  return 0;
}
