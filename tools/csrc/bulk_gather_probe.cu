// bulk_gather_probe.cu -- how fast can B200 gather random 512-B rows into shared memory with
// the bulk-copy (TMA) engine instead of LSU loads?  (the fused forward is bound
// by the L1 data pipe; a bulk-copy gather would move the rows L2 -> smem without LSU
// wavefronts and read them back with LDS only.)  Standalone: nvcc -gencode
// arch=compute_100a,code=sm_100a -O3 -o /tmp/bgp tools/csrc/bulk_gather_probe.cu
//
// Each warp streams its own list of row ids: lane 0 arms a per-slot mbarrier with 512
// expected bytes and issues cp.async.bulk (global -> shared::cta) for the row; K slots per
// warp are in flight; the whole warp waits on the slot's barrier, reads the row with one
// LDS.128 per lane and adds it (so the bytes are really consumed), then lane 0 reuses the
// slot.  Variant "lsu": the same gather with LDG.128 per lane, K rows in flight.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#define CK(x)                                                                                   \
  do {                                                                                          \
    cudaError_t e = (x);                                                                        \
    if (e != cudaSuccess) {                                                                     \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));                 \
      exit(1);                                                                                  \
    }                                                                                           \
  } while (0)

constexpr int ROWB = 512;

template <int K, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) bulk_kernel(const char* __restrict__ table, const uint32_t* __restrict__ ids,
                                                          long n, float* out) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(smem) + warp * K * ROWB;
  const uint32_t bars = (uint32_t)__cvta_generic_to_shared(smem) + WARPS * K * ROWB + warp * K * 8;
  if (lane == 0)
    for (int s = 0; s < K; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(bars + 8 * s));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const long gw = (long)blockIdx.x * WARPS + warp;
  const uint32_t* my = ids + gw * n;
  auto issue = [&](int s, uint32_t id) {
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bars + 8 * s), "r"(ROWB) : "memory");
    asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     ring + s * ROWB),
                 "l"(table + (size_t)id * ROWB), "r"(ROWB), "r"(bars + 8 * s)
                 : "memory");
  };
  if (lane == 0)
    for (int s = 0; s < K && s < n; ++s) issue(s, my[s]);
  float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  for (long i = 0; i < n; ++i) {
    const int s = (int)(i % K);
    const uint32_t ph = (uint32_t)((i / K) & 1);
    uint32_t done = 0;
    while (!done)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(done)
                   : "r"(bars + 8 * s), "r"(ph)
                   : "memory");
    float4 v;
    asm volatile("ld.shared.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                 : "r"(ring + s * ROWB + lane * 16) : "memory");
    a0 += v.x; a1 += v.y; a2 += v.z; a3 += v.w;
    __syncwarp();
    if (lane == 0 && i + K < n) issue(s, my[i + K]);
  }
  out[gw * 32 + lane] = a0 + a1 + a2 + a3;
}

template <int K, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) lsu_kernel(const char* __restrict__ table, const uint32_t* __restrict__ ids,
                                                         long n, float* out) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long gw = (long)blockIdx.x * WARPS + warp;
  const uint32_t* my = ids + gw * n;
  float a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  for (long i = 0; i < n; i += K) {
    float4 v[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const uint32_t id = __ldg(my + i + k);
      v[k] = __ldg(reinterpret_cast<const float4*>(table + (size_t)id * ROWB) + lane);
    }
#pragma unroll
    for (int k = 0; k < K; ++k) { a0 += v[k].x; a1 += v[k].y; a2 += v[k].z; a3 += v[k].w; }
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

template <int K, int WARPS>
static void run(const char* name, const char* table, const uint32_t* ids, long n, float* out, int sms, int ctas_per_sm,
                bool bulk) {
  const int grid = sms * ctas_per_sm;
  const size_t smem = bulk ? (size_t)WARPS * K * (ROWB + 8) : 0;
  if (bulk) CK(cudaFuncSetAttribute(bulk_kernel<K, WARPS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const float ms = time_it([&] {
    if (bulk) bulk_kernel<K, WARPS><<<grid, WARPS * 32, smem>>>(table, ids, n, out);
    else lsu_kernel<K, WARPS><<<grid, WARPS * 32>>>(table, ids, n, out);
  });
  CK(cudaGetLastError());
  const double bytes = (double)grid * WARPS * n * ROWB;
  printf("{\"variant\": \"%s\", \"K\": %d, \"warps_per_cta\": %d, \"ctas_per_sm\": %d, \"ms\": %.4f, \"GBps\": %.1f}\n", name,
         K, WARPS, ctas_per_sm, ms, bytes / (ms * 1e-3) / 1e9);
}

int main(int argc, char** argv) {
  const long rows = argc > 1 ? atol(argv[1]) : 100000;   // 51 MB: L2-resident
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const long n = 4096;                                    // rows per warp
  const long maxw = (long)sms * 64;                       // warps of the largest grid below
  char* table;
  uint32_t* ids;
  float* out;
  CK(cudaMalloc(&table, (size_t)rows * ROWB));
  CK(cudaMemset(table, 0, (size_t)rows * ROWB));
  CK(cudaMalloc(&ids, (size_t)maxw * n * 4));
  CK(cudaMalloc(&out, (size_t)maxw * 32 * 4));
  std::vector<uint32_t> h((size_t)maxw * n);
  uint64_t x = 88172645463325252ull;
  for (auto& v : h) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    v = (uint32_t)(x % (uint64_t)rows);
  }
  CK(cudaMemcpy(ids, h.data(), h.size() * 4, cudaMemcpyHostToDevice));
  printf("# rows %ld (%.1f MB), %ld rows per warp, %d SMs\n", rows, rows * ROWB / 1e6, n, sms);
  run<8, 8>("bulk", table, ids, n, out, sms, 2, true);
  run<16, 8>("bulk", table, ids, n, out, sms, 2, true);
  run<16, 16>("bulk", table, ids, n, out, sms, 1, true);
  run<24, 8>("bulk", table, ids, n, out, sms, 2, true);
  run<12, 16>("bulk", table, ids, n, out, sms, 2, true);
  run<8, 16>("bulk", table, ids, n, out, sms, 3, true);
  run<4, 8>("lsu", table, ids, n, out, sms, 4, false);
  run<8, 8>("lsu", table, ids, n, out, sms, 4, false);
  run<4, 8>("lsu", table, ids, n, out, sms, 8, false);
  run<8, 8>("lsu", table, ids, n, out, sms, 8, false);
  return 0;
}
