// emb_bwd_sort.cuh -- SURVEY row f2, second algorithm (option "bwd_algo" = 1): the EMB
// backward as a transpose of the sparse input (an LSD radix sort of the lookups by dW row)
// followed by a segmented gather-sum, so every distinct dW row receives ONE atomic add per
// run of the sorted list instead of one per bag slice.
//
// Same definition as emb_bwd.cuh (§V; adjoint of the sum pooling of
// L91-95):   dW_t[x, :] += sum over bags (t, b), positions j with x_t[j] = x, of dY[b, t, :]
//
// Steps (all stream-ordered on the caller's stream; only the reduce reads peers' memory):
//   1. gen      entries in position order: {dY row code of the bag, global row g =
//               rowbase[t] + x}; the code is (owning DP rank << 28) | (b - s_dst) * T + t
//   2. sort     per 9-bit digit: upsweep of per-tile digit histograms, the 3-kernel scan
//               (tile sums, scan of the tile sums, tile scan + offset) over the digit-major
//               histogram matrix, stable downsweep (3 passes cover 27-bit rows)
//   3. reduce   persistent warps claim tasks of S consecutive sorted entries, gather each
//               entry's dY vector (one-sided load from the DP rank's grad slot), sum runs of
//               equal g in registers and red.add the run into dW_t[x] (two-group software
//               pipeline of row loads as in the forward); the last CTA releases "done".
// The sort is stable, so a run's fp32 sum follows position order; across runs and warps
// the atomics make the order unspecified: results match the oracle within the order-
// independent bound and exactly on integer-valued gradients, like the atomic scatter.
#pragma once

#include "emb_bwd.cuh"

namespace emb {

struct SortParams {
  const int64_t* offsets;      // [T_r*B + 1]
  const int64_t* indices;
  const int64_t* rowbase;      // [T_r + 1] global row base of each local table (device)
  const TableDesc* tables;     // [T_r] (global id)
  uint32_t* cnt;               // [R] counts -> exclusive starts -> ends
  uint32_t* ecode;             // [cap] dY row code of each entry (gen output; sorted: reduce input)
  uint32_t* erow;              // [cap] global dW row g of each entry (the sort key)
  uint32_t* bsum;              // [nblk] scan tile sums
  float* const* dW;            // [T_r] fp32 [M_t][d]
  const char* gsrc[kMaxG];     // per DP rank: its grad slot of this epoch, [B_dst][T][d] fp32
  uint32_t* peer_done[kMaxG];  // &done_p[rank] on peer p
  const uint32_t* my_ready;    // ready_r[G]
  Ctrl* ctrl;                  // bwork / bdone
  int64_t bstart[kMaxG + 1];
  int64_t R, cap, B, timeout_ns;
  int32_t T, T_r, d, G, rank, lanes, chunk_rows;
  uint32_t epoch;
  // bwd_algo 3 (LSD radix sort): ping-pong entry buffers, per-(digit, tile) histogram
  const uint32_t* rin_c;       // this pass's input entries (codes, rows) ...
  const uint32_t* rin_g;
  uint32_t* rout_c;            // ... and output
  uint32_t* rout_g;
  uint32_t* ghist;             // [256][nblk_r], digit-major
  int64_t nblk_r;
  int32_t shift;
};

constexpr int kScanTile = 4096;    // counters per scan tile (256 threads x 16)
constexpr int kSortTask = 512;     // sorted entries per warp task in reduce (multiple of 128)

__device__ __forceinline__ int64_t sort_nnz(const SortParams& p) {
  return __ldg(p.offsets + (int64_t)p.T_r * p.B);
}

// local table of position j: the last t with offsets[t*B] <= j (tb in shared memory)
__device__ __forceinline__ int table_of(const int64_t* tb, int T_r, int64_t j) {
  int lo = 0, hi = T_r - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (tb[mid] <= j) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// 2a. per-tile sums
__global__ void __launch_bounds__(kBlock) emb_bsort_scan_sum_kernel(const __grid_constant__ SortParams p) {
  __shared__ uint32_t red[kBlock / 32];
  const int64_t base = (int64_t)blockIdx.x * kScanTile;
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanTile / kBlock; ++k) {
    const int64_t i = base + (int64_t)k * kBlock + threadIdx.x;
    if (i < p.R) s += p.cnt[i];
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x < 32) {
    s = threadIdx.x < kBlock / 32 ? red[threadIdx.x] : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
    if (threadIdx.x == 0) p.bsum[blockIdx.x] = s;
  }
}

// block-wide exclusive scan of one value per thread (256 threads); returns the block total
__device__ __forceinline__ uint32_t block_exscan(uint32_t v, uint32_t* sh, uint32_t* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sh[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t s = lane < kBlock / 32 ? sh[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, s, o);
      if (lane >= o) s += y;
    }
    if (lane < kBlock / 32) sh[lane] = s;    // inclusive warp totals
  }
  __syncthreads();
  const uint32_t before = (w > 0 ? sh[w - 1] : 0u) + x - v;
  *total = sh[kBlock / 32 - 1];
  __syncthreads();
  return before;
}

// 2b. exclusive scan of the tile sums (one CTA, sequential over 256-wide pieces)
__global__ void __launch_bounds__(kBlock) emb_bsort_scan_top_kernel(uint32_t* bsum, int64_t nblk) {
  __shared__ uint32_t sh[kBlock / 32];
  uint32_t carry = 0;
  for (int64_t b0 = 0; b0 < nblk; b0 += kBlock) {
    const int64_t i = b0 + threadIdx.x;
    const uint32_t v = i < nblk ? bsum[i] : 0u;
    uint32_t tot;
    const uint32_t ex = block_exscan(v, sh, &tot);
    if (i < nblk) bsum[i] = carry + ex;
    carry += tot;
  }
}

// 2c. in-place exclusive scan of each tile plus its offset: 16 coalesced rounds of 256
__global__ void __launch_bounds__(kBlock) emb_bsort_scan_apply_kernel(const __grid_constant__ SortParams p) {
  __shared__ uint32_t sh[kBlock / 32];
  const int64_t base = (int64_t)blockIdx.x * kScanTile + threadIdx.x;
  uint32_t v[kScanTile / kBlock];
#pragma unroll
  for (int k = 0; k < kScanTile / kBlock; ++k) v[k] = (base + k * kBlock < p.R) ? p.cnt[base + k * kBlock] : 0u;
  uint32_t carry = p.bsum[blockIdx.x];
#pragma unroll
  for (int k = 0; k < kScanTile / kBlock; ++k) {
    uint32_t tot;
    const uint32_t ex = block_exscan(v[k], sh, &tot);
    if (base + k * kBlock < p.R) p.cnt[base + k * kBlock] = carry + ex;
    carry += tot;
  }
}

// ---------------------------------------------------------------------------- bwd_algo 3
// LSD radix sort of the {code, g} entries by g, 9-bit digits: per pass an upsweep writes
// each tile's 512-bin digit histogram (shared-memory atomics only), an exclusive scan over
// the digit-major [512][tiles] matrix gives every (digit, tile) its output offset, and a
// stable downsweep ranks each tile's entries per digit (match.any within a warp, per-warp
// digit counts in shared memory across warps and iterations) and scatters them.  No
// global atomics on row counters at all.
constexpr int kRTile = 4096;       // entries per tile (8 warps x 512 contiguous)

// entries in position order: pairs[j] = {dY row code of j's bag, global row of j}
__global__ void __launch_bounds__(kBlock) emb_bradix_gen_kernel(const __grid_constant__ SortParams p) {
  __shared__ int64_t ofs[kBlock / 32][33];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t B = p.B, nbags = (int64_t)p.T_r * B;
  if (nbags == 0) return;
  const int64_t nnz = sort_nnz(p);
  if (nnz > p.cap) {
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicOr(&p.ctrl->err, 0x4u);
    return;
  }
  const int64_t cb64 = nnz > 0 ? ((int64_t)p.chunk_rows * nbags + nnz - 1) / nnz : 31;
  const int cb = (int)(cb64 < 1 ? 1 : (cb64 > 31 ? 31 : cb64));
  const int64_t cpt = (B + cb - 1) / cb, nchunks = cpt * p.T_r;
  const int64_t nw = (int64_t)gridDim.x * (kBlock / 32);
  for (int64_t c = (int64_t)blockIdx.x * (kBlock / 32) + w; c < nchunks; c += nw) {
    const int t_l = (int)(c / cpt);
    const int64_t b0 = (c % cpt) * cb;
    const int nb = (int)min((int64_t)cb, B - b0);
    if (lane <= nb) ofs[w][lane] = ld_stream_i64(p.offsets + (int64_t)t_l * B + b0 + lane);
    __syncwarp();
    const int64_t pos0 = ofs[w][0], pos1 = ofs[w][nb];
    const int64_t rb = __ldg(p.rowbase + t_l);
    const int64_t tglob = __ldg(&p.tables[t_l].tglob);
    for (int64_t j = pos0 + lane; j < pos1; j += 32) {
      int lo = 0, hi = nb - 1;                          // last bag with start <= j
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (ofs[w][mid] <= j) lo = mid;
        else hi = mid - 1;
      }
      const int64_t b = b0 + lo;
      int dst = 0;
      while (b >= p.bstart[dst + 1]) ++dst;
      const uint32_t code = ((uint32_t)dst << 28) | (uint32_t)((b - p.bstart[dst]) * p.T + tglob);
      p.ecode[j] = code;
      p.erow[j] = (uint32_t)(rb + ld_stream_i64(p.indices + j));
    }
    __syncwarp();
  }
}

constexpr int kRBits = 9;                      // digit width: 3 passes cover 27-bit rows
constexpr int kRBins = 1 << kRBits;

__global__ void __launch_bounds__(kBlock) emb_bradix_up_kernel(const __grid_constant__ SortParams p) {
  __shared__ uint32_t hist[kRBins];
  for (int d = threadIdx.x; d < kRBins; d += kBlock) hist[d] = 0;
  __syncthreads();
  const int64_t nnz = sort_nnz(p);
  const int64_t base = (int64_t)blockIdx.x * kRTile;
  if (nnz <= p.cap) {
#pragma unroll 4
    for (int i = 0; i < kRTile / kBlock; ++i) {
      const int64_t idx = base + (int64_t)i * kBlock + threadIdx.x;
      if (idx < nnz) atomicAdd(hist + ((p.rin_g[idx] >> p.shift) & (kRBins - 1)), 1u);
    }
  }
  __syncthreads();
  for (int d = threadIdx.x; d < kRBins; d += kBlock) p.ghist[(int64_t)d * p.nblk_r + blockIdx.x] = hist[d];
}

// stable downsweep: each warp ranks its own contiguous 512 entries with warp-private digit
// counters (match.any groups, the leader's shared-memory atomicAdd returns the group's
// base: no block barrier per step), one block pass turns the counters into per-(warp,
// digit) offsets inside the tile, the tile is staged in shared memory in digit order and
// each digit's run is written out as consecutive 8-B entries (coalesced)
__global__ void __launch_bounds__(kBlock) emb_bradix_down_kernel(const __grid_constant__ SortParams p) {
  extern __shared__ __align__(16) uint32_t rd_smem[];
  uint2* stage = reinterpret_cast<uint2*>(rd_smem);                 // [kRTile]
  uint32_t* lstart = rd_smem + 2 * kRTile;                          // [kRBins] tile-local digit start
  uint32_t* gofs = lstart + kRBins;                                 // [kRBins] global start (scanned)
  uint32_t* wcnt = gofs + kRBins;                                   // [kBlock/32][kRBins]
  __shared__ uint32_t sh[kBlock / 32];
  constexpr int KI = kRTile / kBlock;                               // 16 entries per lane
  constexpr int NW = kBlock / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int d = threadIdx.x; d < kRBins; d += kBlock) {
    gofs[d] = p.ghist[(int64_t)d * p.nblk_r + blockIdx.x];
#pragma unroll
    for (int k = 0; k < NW; ++k) wcnt[k * kRBins + d] = 0;
  }
  __syncthreads();
  const int64_t nnz = sort_nnz(p);
  if (nnz > p.cap) return;
  const int64_t wbase = (int64_t)blockIdx.x * kRTile + (int64_t)w * (32 * KI);   // warp-contiguous
  const unsigned lt = (1u << lane) - 1u;
  uint2 e[KI];
  uint32_t rk[KI];
#pragma unroll
  for (int i = 0; i < KI; ++i) {
    const int64_t idx = wbase + 32 * i + lane;
    e[i] = idx < nnz ? make_uint2(p.rin_c[idx], p.rin_g[idx]) : make_uint2(0u, 0xffffffffu);
  }
#pragma unroll
  for (int i = 0; i < KI; ++i) {
    const bool valid = wbase + 32 * i + lane < nnz;
    const uint32_t d = (e[i].y >> p.shift) & (kRBins - 1);
    const unsigned peers = __match_any_sync(kFull, valid ? d : (0x10000u | (uint32_t)lane));
    const int leader = __ffs(peers) - 1;
    uint32_t b = 0;
    if (valid && leader == lane) b = atomicAdd(wcnt + w * kRBins + d, (uint32_t)__popc(peers));
    rk[i] = __shfl_sync(kFull, b, leader) + (uint32_t)__popc(peers & lt);
  }
  __syncthreads();
  {                                                      // per-(warp, digit) offsets, digit starts
    constexpr int DP = kRBins / kBlock;
    uint32_t tot[DP], sum = 0;
#pragma unroll
    for (int k = 0; k < DP; ++k) {
      const int d = threadIdx.x * DP + k;
      uint32_t run = 0;
#pragma unroll
      for (int q = 0; q < NW; ++q) {
        const uint32_t c = wcnt[q * kRBins + d];
        wcnt[q * kRBins + d] = run;
        run += c;
      }
      tot[k] = run;
      sum += run;
    }
    uint32_t all;
    uint32_t ex = block_exscan(sum, sh, &all);
#pragma unroll
    for (int k = 0; k < DP; ++k) {
      lstart[threadIdx.x * DP + k] = ex;
      ex += tot[k];
    }
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < KI; ++i) {
    if (wbase + 32 * i + lane < nnz) {
      const uint32_t d = (e[i].y >> p.shift) & (kRBins - 1);
      stage[lstart[d] + wcnt[w * kRBins + d] + rk[i]] = e[i];
    }
  }
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kRTile;
  const int cnt = (int)min((int64_t)kRTile, nnz - base);
  for (int k = threadIdx.x; k < cnt; k += kBlock) {      // digit runs leave contiguously
    const uint2 v = stage[k];
    const uint32_t d = (v.y >> p.shift) & (kRBins - 1);
    const uint32_t o = gofs[d] + (uint32_t)k - lstart[d];
    p.rout_c[o] = v.x;
    p.rout_g[o] = v.y;
  }
}

// 5. segmented gather-sum of the sorted entries + one red.add per run of equal rows.
// A warp claims tasks of kSortTask consecutive sorted entries; the next task's codes and
// rows are copied into the warp's shared-memory double buffer (cp.async, 16 B per lane)
// while the current one is summed, so no entry load sits on the critical path.  Per group
// of UR entries one broadcast LDS.128 yields the 4 dY row codes (issue) and one the 4 dW
// rows (consume) -- no per-entry SHFL; dY vectors are gathered in a software pipeline of
// NGRP groups (two in flight while one is consumed for 512-B rows, as in the forward) and
// summed with packed FADD2; a run's sum goes to dW_t[x] with one red.add per lane vector
// when the run ends (runs crossing a task boundary add one partial per task).
template <int VB, int NV, int NGRP = 2, int MB = 1, bool MULTI = true>
__global__ void __launch_bounds__(kBlock, MB) emb_bsort_reduce_kernel(const __grid_constant__ SortParams p) {
  constexpr int W = VB / 4;
  constexpr int UR = 4;                                   // entries per pipeline group
  static_assert(NGRP == 2 || NGRP == 3, "groups of row vectors in registers");
  constexpr int S = kSortTask;
  static_assert(S % (32 * 4) == 0, "a task is whole 16-B pieces per lane");
  constexpr int kPad = (NGRP + 1) * UR;                   // codes read ahead past a task's end
  constexpr uint32_t kCodeB = (S + kPad) * 4u;            // codes + zero padding read by issue-ahead
  constexpr uint32_t kBufB = kCodeB + S * 4u;             // one buffer: codes | rows
  extern __shared__ __align__(16) int64_t bs_smem[];
  int64_t* rb = bs_smem;                                  // [T_r + 1] row bases
  const int lane = threadIdx.x & 31;
  const bool active = lane < p.lanes;
  const uint32_t rowbytes = (uint32_t)p.d * 4u;
  // per-warp entry double buffer after the row bases
  const uint32_t ebase = (((uint32_t)__cvta_generic_to_shared(bs_smem) + (uint32_t)(p.T_r + 1) * 8u + 15u) & ~15u) +
                         (threadIdx.x >> 5) * (2u * kBufB);
  for (int i = threadIdx.x; i <= p.T_r; i += blockDim.x) rb[i] = __ldg(p.rowbase + i);
  if (lane < kPad)                                        // codes past a task's end: row 0 of rank 0
    for (uint32_t b = 0; b < 2; ++b)
      asm volatile("st.shared.u32 [%0], %1;" ::"r"(ebase + b * kBufB + (S + lane) * 4u), "r"(0u) : "memory");
  if (threadIdx.x == 0 && p.G > 1) wait_flags_geq(p.my_ready, p.G, p.rank, p.epoch, p.timeout_ns, &p.ctrl->err);
  __syncthreads();
  const char* g0 = p.gsrc[0] + lane * VB;                 // !MULTI: every code is a row of rank 0's slot
  const int64_t nnz = sort_nnz(p);
  if (nnz <= p.cap) {
    const int64_t ntask = (nnz + S - 1) / S;
    // stage task c's entries into buffer `buf` (the entry arrays hold >= nnz + S slots, so a
    // task's last piece never reads past them; entries past nnz are never consumed)
    auto stage = [&](int64_t c, uint32_t buf) {
      const uint32_t sb = ebase + buf * kBufB;
#pragma unroll
      for (int k = 0; k < S / 128; ++k) {
        const int64_t e = c * S + (int64_t)(k * 32 + lane) * 4;
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sb + (uint32_t)(k * 32 + lane) * 16u),
                     "l"(p.ecode + e) : "memory");
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sb + kCodeB + (uint32_t)(k * 32 + lane) * 16u),
                     "l"(p.erow + e) : "memory");
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
    unsigned c_next = 0;
    if (lane == 0) c_next = atomicAdd(&p.ctrl->bwork, 1u);
    int64_t c = __shfl_sync(kFull, c_next, 0);
    if (c < ntask) stage(c, 0);
    uint32_t buf = 0;
    while (c < ntask) {
      if (lane == 0) c_next = atomicAdd(&p.ctrl->bwork, 1u);
      const int64_t cn = __shfl_sync(kFull, c_next, 0);
      if (cn < ntask) stage(cn, buf ^ 1u);                // next task's entries in flight
      else asm volatile("cp.async.commit_group;" ::: "memory");
      asm volatile("cp.async.wait_group 1;" ::: "memory");   // this task's entries landed
      __syncwarp();
      const uint32_t sc = ebase + buf * kBufB;
      const int n = (int)min((int64_t)S, nnz - c * S);
      if (n < S) {                                        // the list's last task: codes past n -> 0
        for (int k = n + lane; k < S; k += 32) asm volatile("st.shared.u32 [%0], %1;" ::"r"(sc + 4u * k), "r"(0u) : "memory");
        __syncwarp();
      }
      uint32_t cur;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(cur) : "r"(sc + kCodeB) : "memory");
      int t = 0;
      {
        int lo = 0, hi = p.T_r - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (rb[mid] <= (int64_t)cur) lo = mid;
          else hi = mid - 1;
        }
        t = lo;
      }
      float acc[NV * W];
#pragma unroll
      for (int i = 0; i < NV * W; ++i) acc[i] = 0.0f;
      auto emit = [&]() {                                 // run of row `cur` -> dW_t[x]
        while ((int64_t)cur >= rb[t + 1]) ++t;
        if (active) {
          char* dwt = reinterpret_cast<char*>(__ldg(reinterpret_cast<const unsigned long long*>(p.dW + t)));
          char* rp = dwt + (int64_t)((int64_t)cur - rb[t]) * rowbytes + lane * VB;
#pragma unroll
          for (int v = 0; v < NV; ++v) {
            uint32_t u[W];
#pragma unroll
            for (int i = 0; i < W; ++i) u[i] = __float_as_uint(acc[v * W + i]);
            red_add_vec<VB>(reinterpret_cast<float*>(rp + v * 32 * VB), u);
          }
        }
#pragma unroll
        for (int i = 0; i < NV * W; ++i) acc[i] = 0.0f;
      };
      auto add_row = [&](const uint32_t (&r)[NV][W]) {
        if (active) {
#pragma unroll
          for (int v = 0; v < NV; ++v) Widen<float, VB>::add(acc + v * W, r[v]);
        }
      };
      // the UR entries whose codes start at shared address qa: their dY vectors in flight
      // (positions past the task read code 0 -- a valid row, loaded and never added)
      auto issue = [&](uint32_t (&bf)[UR][NV][W], uint32_t qa) {
        uint32_t code[UR];
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(code[0]), "=r"(code[1]), "=r"(code[2]), "=r"(code[3])
                     : "r"(qa) : "memory");
#pragma unroll
        for (int u = 0; u < UR; ++u) {
          if (active) {
            const char* a = MULTI ? p.gsrc[code[u] >> 28] + lane * VB : g0;
            a = row_addr(a, MULTI ? (code[u] & 0x0fffffffu) : code[u], rowbytes);
#pragma unroll
            for (int v = 0; v < NV; ++v) ld_vec_relaxed<VB>(a + v * 32 * VB, bf[u][v]);
          }
        }
      };
      auto consume = [&](const bool PRED, const uint32_t (&bf)[UR][NV][W], uint32_t qa, int q) {
        uint32_t g[UR];
        asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(g[0]), "=r"(g[1]), "=r"(g[2]), "=r"(g[3])
                     : "r"(qa + kCodeB) : "memory");
        if (!PRED && g[UR - 1] == cur) {                  // sorted: the whole group continues the run
#pragma unroll
          for (int u = 0; u < UR; ++u) add_row(bf[u]);
          return;
        }
#pragma unroll
        for (int u = 0; u < UR; ++u) {
          if (!PRED || q + u < n) {
            if (g[u] != cur) {
              emit();
              cur = g[u];
            }
            add_row(bf[u]);
          }
        }
      };
      constexpr uint32_t kG = UR * 4u;                    // bytes of one group's codes
      if constexpr (NGRP == 3) {
        uint32_t A[UR][NV][W], Bv[UR][NV][W], C[UR][NV][W];
        issue(A, sc);
        issue(Bv, sc + kG);
        uint32_t qa = sc;
#pragma unroll 1
        for (int q = 0; q < n; q += 3 * UR, qa += 3 * kG) {
          issue(C, qa + 2 * kG);
          if (q + UR > n) { consume(true, A, qa, q); break; }
          consume(false, A, qa, q);
          issue(A, qa + 3 * kG);
          if (q + 2 * UR > n) { consume(true, Bv, qa + kG, q + UR); break; }
          consume(false, Bv, qa + kG, q + UR);
          issue(Bv, qa + 4 * kG);
          if (q + 3 * UR > n) { consume(true, C, qa + 2 * kG, q + 2 * UR); break; }
          consume(false, C, qa + 2 * kG, q + 2 * UR);
        }
      } else {
        uint32_t A[UR][NV][W], Bv[UR][NV][W];
        issue(A, sc);
        uint32_t qa = sc;
#pragma unroll 1
        for (int q = 0; q < n; q += 2 * UR, qa += 2 * kG) {
          issue(Bv, qa + kG);
          if (q + UR > n) { consume(true, A, qa, q); break; }
          consume(false, A, qa, q);
          issue(A, qa + 2 * kG);
          if (q + 2 * UR > n) { consume(true, Bv, qa + kG, q + UR); break; }
          consume(false, Bv, qa + kG, q + UR);
        }
      }
      emit();                                             // the task's last run
      __syncwarp();                                       // buffer `buf` is restaged two tasks on
      buf ^= 1u;
      c = cn;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
  }
  // completion: every CTA's reads of peer slots are done before the last CTA tells the
  // peers their slots may be refilled
  __syncthreads();
  if (threadIdx.x != 0) return;
  fence_acq_rel_sys();
  const unsigned prev = atomicAdd(&p.ctrl->bdone, 1u);
  if (prev != gridDim.x - 1) return;
  fence_acq_rel_sys();
  p.ctrl->bdone = 0;
  p.ctrl->bwork = 0;
  for (int q = 1; q < p.G; ++q) st_release_sys(p.peer_done[(p.rank + q) % p.G], p.epoch);
}

}  // namespace emb
