// l2_probe.cu -- measurement tool (not product): streaming read bandwidth of a buffer
// with L1-bypassing 16-byte loads (ld.global.cg), every SM reading the whole buffer
// `reps` times.  A buffer well under the 126 MB L2 gives the L2 read bandwidth; one far
// above it gives HBM read bandwidth.  Used as the L2 denominator in DESIGN.md §8.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void l2_read_kernel(const uint4* __restrict__ buf, size_t n16, int reps, unsigned long long* sink) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < reps; ++r) {
    // rotate the start so CTAs do not march in lockstep over the same lines; 4 loads in
    // flight per thread
    const size_t off = ((size_t)blockIdx.x * 977 + r * 131) % n16;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += 4 * stride) {
      uint4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        size_t j = i + u * stride + off;
        while (j >= n16) j -= n16;
        asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w)
                     : "l"(buf + j));
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
  }
  if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

extern "C" int l2_probe(const void* buf, size_t bytes, int reps, int grid, int block, void* sink, void* stream) {
  l2_read_kernel<<<grid, block, 0, (cudaStream_t)stream>>>((const uint4*)buf, bytes / 16, reps,
                                                           (unsigned long long*)sink);
  return (int)cudaGetLastError();
}
