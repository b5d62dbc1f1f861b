// emb_bwd.cuh -- SURVEY row f2: the EMB-layer backward with PGAS-style one-sided access.
//
// PAPER.md §V (L378-382): "during backpropagation, the gradients for these embeddings need
// to be communicated back to the GPUs that own these embeddings ... gradients must be
// aggregated ... replacing multiple rounds of collective calls with atomic PGAS
// direct-GPU remote [accesses]".  Definition (adjoint of sum pooling, L91-95):
//     dW_t[x, :] = sum over bags (t, b), positions j with x_t[j] = x, of dY[b, t, :]
// where dY[b] lives on the rank owning sample b (data parallel) and dW_t on the owner of
// table t (model parallel) -- or, for an f3 row-sharded table, the rows [lo, hi) of dW_t on
// the shard's owner, which reads the table's full bag list and keeps its own ids.
//
// B200 design: the OWNER pulls.  Every rank writes its dY [B_r][T][d] (fp32) into a
// symmetric grad slot and releases a per-source "ready" flag; the owner's fused kernel
// acquires the flags, then per bag loads the bag's gradient vector straight from the DP
// rank's slot (one-sided NVLink load; the load of the next bag is in flight while the
// current one is scattered) and red.add.v4.f32's it into the dW rows of every index of
// the bag (L2 atomics, no sort, no all-to-all, no unpack).  The last CTA releases a
// per-source "done" flag so each DP rank knows when its slot may be refilled.
#pragma once

#include "emb_kernels.cuh"

namespace emb {

struct BwdParams {
  const TableDesc* tables;     // [T_r] (rows, global id)
  float* const* dW;            // [T_r] device pointers, fp32 [M_t][d], accumulated into
  const int64_t* offsets;      // [T_r*B + 1]
  const int64_t* indices;
  int64_t B;
  int64_t bstart[kMaxG + 1];
  const char* gsrc[kMaxG];     // per DP rank: its grad slot of this epoch, [B_dst][T][d] fp32
  uint32_t* peer_ready[kMaxG]; // &ready_p[rank] on peer p
  uint32_t* peer_done[kMaxG];  // &done_p[rank] on peer p
  const uint32_t* my_ready;    // ready_r[G]
  Ctrl* ctrl;                  // uses bwork / bdone
  int64_t timeout_ns;
  int32_t T, T_r, d, G, rank, lanes, chunk_rows;
  int32_t interleave;          // table group size g: chunks interleaved over g tables at a time (1 = table-major)
  uint32_t epoch;
};

template <int VB>
__device__ __forceinline__ void red_add_vec(float* p, const uint32_t* r);
template <>
__device__ __forceinline__ void red_add_vec<16>(float* p, const uint32_t* r) {
  asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(__uint_as_float(r[0])),
               "f"(__uint_as_float(r[1])), "f"(__uint_as_float(r[2])), "f"(__uint_as_float(r[3]))
               : "memory");
}
template <>
__device__ __forceinline__ void red_add_vec<8>(float* p, const uint32_t* r) {
  asm volatile("red.relaxed.gpu.global.add.v2.f32 [%0], {%1,%2};" ::"l"(p), "f"(__uint_as_float(r[0])),
               "f"(__uint_as_float(r[1]))
               : "memory");
}
template <int VB>
__device__ __forceinline__ void ld_vec_relaxed(const void* p, uint32_t* r);
template <>
__device__ __forceinline__ void ld_vec_relaxed<16>(const void* p, uint32_t* r) {
  asm volatile("ld.global.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "l"(p));
}
template <>
__device__ __forceinline__ void ld_vec_relaxed<8>(const void* p, uint32_t* r) {
  asm volatile("ld.global.v2.b32 {%0,%1}, [%2];" : "=r"(r[0]), "=r"(r[1]) : "l"(p));
}

__device__ __forceinline__ bool wait_flags_geq(const uint32_t* flags, int G, int rank, uint32_t epoch, int64_t timeout_ns,
                                               unsigned* err) {
  const uint64_t t0 = globaltimer();
  for (int s = 0; s < G; ++s) {
    if (s == rank) continue;
    unsigned ns = 32;
    while ((int32_t)(ld_relaxed_sys(flags + s) - epoch) < 0) {
      if ((int64_t)(globaltimer() - t0) > timeout_ns) {
        atomicOr(err, 0x1u);
        return false;
      }
      __nanosleep(ns);
      if (ns < 1024) ns <<= 1;
    }
  }
  fence_acq_rel_sys();
  return true;
}

// VB bytes per lane vector, NV vectors per lane (row = 32*VB*NV bytes when all lanes active).
// Each 32-id slice's distinct rows are compacted into a per-warp shared-memory list (row id
// and multiplicity in one word) and scattered from it with broadcast LDS.128 reads, 8
// REDs per iteration -- no SHFL / find-first-set chain per distinct row.
//
// HC > 0: each warp privatizes up to HC dW rows of its current chunk in shared
// memory (direct-mapped by a multiplicative hash of the row id, first come first served,
// a row whose slot is taken goes straight to L2).  A zipf-hot row then costs one RED per
// chunk (the flush at the chunk's end) instead of one per bag slice: same-address
// atomics on the hottest rows are what serialize in the L2.
template <int VB, int NV, int HC = 0>
__global__ void __launch_bounds__(kBlock) emb_bwd_kernel(const __grid_constant__ BwdParams p) {
  static_assert(HC == 0 || (HC <= 32 && (HC & (HC - 1)) == 0), "cache: power of two <= 32 slots");
  constexpr int W = VB / 4;
  const int lane = threadIdx.x & 31;
  const bool active = lane < p.lanes;
  const int64_t rowbytes = (int64_t)p.d * 4;
  const int64_t B = p.B;
  __shared__ __align__(16) uint32_t bwd_ring[kBlock / 32][128];     // per-warp id ring
  __shared__ __align__(16) uint32_t bwd_list[kBlock / 32][80];   // compacted (id|mult) + mult
  const uint32_t list_s = (uint32_t)__cvta_generic_to_shared(&bwd_list[threadIdx.x >> 5][0]);
  // HC: per-warp row cache [HC][32*VB*NV bytes] + tags [HC] in dynamic shared memory
  constexpr uint32_t kRowB = 32u * VB * NV;
  constexpr uint32_t kEmpty = 0xffffffffu;
  constexpr int kLogHC = HC >= 32 ? 5 : HC >= 16 ? 4 : HC >= 8 ? 3 : HC >= 4 ? 2 : HC >= 2 ? 1 : 0;
  extern __shared__ __align__(16) unsigned char bwd_dyn[];
  const uint32_t cache_s = HC ? (uint32_t)__cvta_generic_to_shared(bwd_dyn) + (threadIdx.x >> 5) * (HC * (kRowB + 4u)) : 0u;
  const uint32_t tag_s = cache_s + HC * kRowB;
  if (HC > 0 && lane < HC) asm volatile("st.shared.u32 [%0], %1;" ::"r"(tag_s + 4u * lane), "r"(kEmpty) : "memory");
  __syncwarp();
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(&bwd_ring[threadIdx.x >> 5][0]);
  // acquire every DP rank's dY of this epoch
  if (threadIdx.x == 0 && p.G > 1) wait_flags_geq(p.my_ready, p.G, p.rank, p.epoch, p.timeout_ns, &p.ctrl->err);
  __syncthreads();

  const int64_t nbags = (int64_t)p.T_r * B;
  if (nbags > 0) {
    const int64_t nnz = __ldg(p.offsets + nbags);
    const int64_t cb64 = (nnz > 0) ? ((int64_t)p.chunk_rows * nbags + nnz - 1) / nnz : 31;
    const int cb = (int)(cb64 < 1 ? 1 : (cb64 > 31 ? 31 : cb64));
    const int64_t cpt = (B + cb - 1) / cb;
    const int64_t nchunks = cpt * p.T_r;
    for (;;) {
      unsigned c = 0;
      if (lane == 0) c = atomicAdd(&p.ctrl->bwork, 1u);
      c = __shfl_sync(kFull, c, 0);
      if ((int64_t)c >= nchunks) break;
      // interleave tables (chunk c -> table c mod T_r): a zipf-hot dW row then receives its
      // atomics spread over the whole kernel instead of from every warp at once
      // (in groups of g tables: the touched dW rows of g tables stay live in L2 at once)
      const int g = p.interleave, nfull = p.T_r / g;
      const int64_t nfc = (int64_t)nfull * g * cpt;       // chunks of the full groups
      int t_l;
      int64_t bi;
      if ((int64_t)c < nfc) {
        const int64_t r = (int64_t)c % ((int64_t)g * cpt);
        t_l = (int)((int64_t)c / ((int64_t)g * cpt)) * g + (int)(r % g);
        bi = r / g;
      } else {                                            // the last, smaller group
        const int rem = p.T_r - nfull * g;
        const int64_t r = (int64_t)c - nfc;
        t_l = nfull * g + (int)(r % rem);
        bi = r / rem;
      }
      const int64_t b0 = bi * cb;
      const int nb = (int)min((int64_t)cb, B - b0);
      const int64_t o_l = (lane <= nb) ? ld_stream_i64(p.offsets + (int64_t)t_l * B + b0 + lane) : 0;
      const TableDesc* tdp = p.tables + t_l;
      const int64_t tglob = __ldg(&tdp->tglob);
      const int64_t trows = __ldg(reinterpret_cast<const long long*>(&tdp->rows));
      const bool pack = trows < (1ll << 26);
      // f3 row shards: the CSR lists the table's full bags with global row ids; ids outside
      // this shard's [lo, lo + rows) belong to another shard's owner and are skipped (a whole
      // table has lo = 0, rows = M_t: nothing is skipped)
      const uint32_t tlo = (uint32_t)__ldg(reinterpret_cast<const long long*>(&tdp->lo));
      char* dwl = reinterpret_cast<char*>(__ldg(reinterpret_cast<const unsigned long long*>(p.dW + t_l))) + lane * VB;

      auto gaddr = [&](int bag) -> const char* {        // dY[b][tglob] on the DP rank owning b
        const int64_t b = b0 + bag;
        int dst = 0;
        while (b >= p.bstart[dst + 1]) ++dst;
        return p.gsrc[dst] + ((b - p.bstart[dst]) * p.T + tglob) * rowbytes + lane * VB;
      };
      // Per bag: the bag's gradient vector (prefetched one bag ahead) is added once per DISTINCT row of each 32-id slice, multiplied by the
      // row's multiplicity (match.any): zipf-hot rows repeat inside a bag, and fewer
      // atomics on the same L2 address is what bounds this kernel.
      auto bag_start = [&](int bag) -> int64_t { return __shfl_sync(kFull, o_l, bag); };
      // The chunk's row ids stream through a per-warp shared-memory ring of 4 batches of 32
      // (cp.async of each int64 id's low word, up to 3 batches ahead of the slice being
      // scattered), so no slice waits on an id load from DRAM.
      const int64_t pos0 = bag_start(0);
      const int32_t nrel = (int32_t)(bag_start(nb) - pos0);
      const int64_t* ip = p.indices + pos0;
      const int32_t nbatch = (nrel + 31) >> 5;
      int32_t fetched = 0;
      auto fetch = [&]() {
        const int32_t at = fetched * 32 + lane;
        if (at < nrel)
          asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(ring_s + (uint32_t)(((fetched & 3) * 32 + lane) * 4)),
                       "l"(ip + at) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
        ++fetched;
      };
      uint32_t gn[NV][W];
      if (active && nb > 0) {
        const char* a = gaddr(0);
#pragma unroll
        for (int v = 0; v < NV; ++v) ld_vec_relaxed<VB>(a + v * 32 * VB, gn[v]);
      }
      for (int bag = 0; bag < nb; ++bag) {
        uint32_t g[NV][W];
#pragma unroll
        for (int v = 0; v < NV; ++v)
#pragma unroll
          for (int i = 0; i < W; ++i) g[v][i] = gn[v][i];
        const int64_t s0 = bag_start(bag), e0 = bag_start(bag + 1);
        if (bag + 1 < nb && active) {                     // next bag's gradient in flight
          const char* a = gaddr(bag + 1);
#pragma unroll
          for (int v = 0; v < NV; ++v) ld_vec_relaxed<VB>(a + v * 32 * VB, gn[v]);
        }
        for (int64_t c0 = s0; c0 < e0; c0 += 32) {
          const int32_t r0 = (int32_t)(c0 - pos0);
          const int32_t lo = r0 >> 5, hi = min((r0 + 31) >> 5, nbatch - 1);
          while (fetched < nbatch && fetched <= lo + 3) fetch();
          switch (min(fetched - 1 - hi, 3)) {             // batches lo..hi landed
            case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
            case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
            case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
            default: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
          }
          __syncwarp();
          uint32_t x = 0x80000000u | lane;
          if (c0 + lane < e0) {
            uint32_t xg;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(xg) : "r"(ring_s + (uint32_t)(((r0 + lane) & 127) * 4)) : "memory");
            const uint32_t xs = xg - tlo;                 // shard-local row
            if ((uint64_t)xs < (uint64_t)trows) x = xs;
          }
          const unsigned same = __match_any_sync(kFull, x);
          const bool lead = (x & 0x80000000u) == 0 && (__ffs(same) - 1) == lane;
          const unsigned leaders = __ballot_sync(kFull, lead);
          // row id and multiplicity travel in one word (ids < 2^26): one SHFL per distinct
          // row instead of two -- the leader loop is bound by the MIO pipe
          const uint32_t xm = pack ? (x | ((uint32_t)__popc(same) << 26)) : x;
          const int n = __popc(leaders);
          if (lead) {
            const uint32_t at = list_s + 4u * (uint32_t)__popc(leaders & ((1u << lane) - 1u));
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(at), "r"(xm) : "memory");
            if (!pack) asm volatile("st.shared.u32 [%0], %1;" ::"r"(at + 160u), "r"((uint32_t)__popc(same)) : "memory");
          }
          __syncwarp();
          for (int k = 0; k < n; k += 8) {
            uint32_t wv[8], mv[8];
            asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(wv[0]), "=r"(wv[1]), "=r"(wv[2]), "=r"(wv[3])
                         : "r"(list_s + 4u * k) : "memory");
            asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(wv[4]), "=r"(wv[5]), "=r"(wv[6]), "=r"(wv[7])
                         : "r"(list_s + 4u * k + 16u) : "memory");
            if (!pack) {
              asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(mv[0]), "=r"(mv[1]), "=r"(mv[2]), "=r"(mv[3])
                           : "r"(list_s + 4u * k + 160u) : "memory");
              asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(mv[4]), "=r"(mv[5]), "=r"(mv[6]), "=r"(mv[7])
                           : "r"(list_s + 4u * k + 176u) : "memory");
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              if constexpr (HC > 0) {
                if (k + u < n) {
                  const uint32_t xl = pack ? (wv[u] & 0x03ffffffu) : wv[u];
                  const float m = pack ? (float)(wv[u] >> 26) : (float)mv[u];
                  const uint32_t h = HC == 1 ? 0u : (xl * 2654435761u) >> (32 - kLogHC);
                  // lane 0 alone reads and claims the tag (no cross-lane access to it); the
                  // shuffle hands its decision to the warp
                  uint32_t tg = 0;
                  if (lane == 0) {
                    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(tg) : "r"(tag_s + 4u * h) : "memory");
                    if (tg == kEmpty) asm volatile("st.shared.u32 [%0], %1;" ::"r"(tag_s + 4u * h), "r"(xl) : "memory");
                  }
                  tg = __shfl_sync(kFull, tg, 0);
                  const bool hit = tg == xl, claim = tg == kEmpty;
                  if (active) {
#pragma unroll
                    for (int v = 0; v < NV; ++v) {
                      uint32_t gm[W];
#pragma unroll
                      for (int i = 0; i < W; ++i) gm[i] = __float_as_uint(m == 1.0f ? __uint_as_float(g[v][i]) : m * __uint_as_float(g[v][i]));
                      const uint32_t sa = cache_s + h * kRowB + (uint32_t)(v * 32 + lane) * VB;
                      if (hit) {                            // this lane's columns only: no atomics
                        uint32_t cv[W];
                        lds_bytes<VB>(sa, cv);
#pragma unroll
                        for (int i = 0; i < W; ++i) cv[i] = __float_as_uint(__uint_as_float(cv[i]) + __uint_as_float(gm[i]));
                        sts_bytes<VB>(sa, cv);
                      } else if (claim) {
                        sts_bytes<VB>(sa, gm);
                      } else {
                        red_add_vec<VB>(reinterpret_cast<float*>(dwl + (uint64_t)xl * (uint64_t)rowbytes + v * 32 * VB), gm);
                      }
                    }
                  }
                }
                continue;
              }
              if (k + u < n && active) {
                const uint32_t xl = pack ? (wv[u] & 0x03ffffffu) : wv[u];
                const float m = pack ? (float)(wv[u] >> 26) : (float)mv[u];
                char* rp = dwl + (uint64_t)xl * (uint64_t)rowbytes;
#pragma unroll
                for (int v = 0; v < NV; ++v) {
                  uint32_t gm[W];
#pragma unroll
                  for (int i = 0; i < W; ++i) gm[i] = __float_as_uint(m == 1.0f ? __uint_as_float(g[v][i]) : m * __uint_as_float(g[v][i]));
                  red_add_vec<VB>(reinterpret_cast<float*>(rp + v * 32 * VB), gm);
                }
              }
            }
          }
          __syncwarp();                                 // the list is rewritten by the next slice
        }
      }
      asm volatile("cp.async.wait_group 0;" ::: "memory");   // no copy outlives the chunk
      __syncwarp();
      if constexpr (HC > 0) {                             // flush the chunk's cached rows
        uint32_t tg = kEmpty;
        if (lane < HC) asm volatile("ld.shared.u32 %0, [%1];" : "=r"(tg) : "r"(tag_s + 4u * lane) : "memory");
        unsigned occ = __ballot_sync(kFull, tg != kEmpty);
        while (occ) {
          const int l = __ffs(occ) - 1;
          occ &= occ - 1;
          const uint32_t xl = __shfl_sync(kFull, tg, l);
          if (active) {
#pragma unroll
            for (int v = 0; v < NV; ++v) {
              uint32_t cv[W];
              lds_bytes<VB>(cache_s + (uint32_t)l * kRowB + (uint32_t)(v * 32 + lane) * VB, cv);
              red_add_vec<VB>(reinterpret_cast<float*>(dwl + (uint64_t)xl * (uint64_t)rowbytes + v * 32 * VB), cv);
            }
          }
        }
        if (lane < HC) asm volatile("st.shared.u32 [%0], %1;" ::"r"(tag_s + 4u * lane), "r"(kEmpty) : "memory");
        __syncwarp();
      }
    }
  }
  // completion: every CTA's reads of peer slots are done before the last CTA tells the
  // peers their slots may be refilled
  // (G = 1: no peer waits for "done", so device scope suffices, as in cta_complete)
  __syncthreads();
  if (threadIdx.x != 0) return;
  if (p.G > 1) fence_acq_rel_sys();
  const unsigned prev = atomicAdd(&p.ctrl->bdone, 1u);
  if (prev != gridDim.x - 1) return;
  if (p.G > 1) fence_acq_rel_sys();
  else __threadfence();
  p.ctrl->bdone = 0;
  p.ctrl->bwork = 0;
  for (int q = 1; q < p.G; ++q) st_release_sys(p.peer_done[(p.rank + q) % p.G], p.epoch);
}

#ifdef EMB_RUNTIME_TU
// release "my dY of this epoch is in my grad slot" to every peer (stream-ordered after the
// kernels that wrote it)
__global__ void emb_bwd_signal_kernel(const __grid_constant__ BwdParams p) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  fence_acq_rel_sys();
  for (int q = 1; q < p.G; ++q) st_release_sys(p.peer_ready[(p.rank + q) % p.G], p.epoch);
}
// before a grad slot is refilled: wait until every peer finished reading its previous use
__global__ void emb_bwd_slot_wait_kernel(const uint32_t* my_done, int G, int rank, uint32_t epoch, int64_t timeout_ns,
                                         unsigned* err) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  wait_flags_geq(my_done, G, rank, epoch, timeout_ns, err);
}
#endif

}  // namespace emb
