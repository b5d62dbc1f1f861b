// emb_inst_bf16_f32.cu -- instantiations of the fused kernel for bf16 tables, f32 output.
#include "emb_dispatch.h"

namespace emb {
namespace {
template <int VB, int NV, typename WT, typename OT, bool CHECK>
KernelFn pick_u(int unroll, int mb, bool full, bool sidx, bool shard, bool tmast) {
  if constexpr (!CHECK && NV == 1) {
    if (tmast && full && !shard) {  // f4: staged vectors shipped by TMA scatter4
      if (unroll == 2) return emb_fwd_kernel<VB, NV, WT, OT, 2, false, 6, true, false, false, true>;
      return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 4, true, false, false, true>;
    }
  }
  if constexpr (!CHECK) {
    if (shard) {  // f3: row-sharded tables (in-kernel id partitioning, partial slots)
      if (!full) return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 4, false, false, true>;
      if (unroll == 2) return emb_fwd_kernel<VB, NV, WT, OT, 2, false, 6, true, false, true>;
      if (NV > 1) return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 1, true, false, true>;
      return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 4, true, false, true>;
    }
  }
  if (!full) return emb_fwd_kernel<VB, NV, WT, OT, 4, CHECK, 4, false>;  // rows narrower than a warp
  if constexpr (!CHECK && NV == 1) {
    if (unroll == 3)  // experiment: 2 groups of 8 rows in flight per warp, 16 warps/SM (128 registers)
      return sidx ? emb_fwd_kernel<VB, NV, WT, OT, 8, false, 2, true, true> : emb_fwd_kernel<VB, NV, WT, OT, 8, false, 2, true, false>;
    if (sidx && unroll == 4 && mb == 4) return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 4, true, true>;
    if (sidx && unroll == 4 && mb == 5) return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 5, true, true>;  // 40 warps/SM
    if (sidx && unroll == 4 && mb == 6) return emb_fwd_kernel<VB, NV, WT, OT, 4, false, 6, true, true>;  // 48 warps/SM
    if (sidx && unroll == 2) return emb_fwd_kernel<VB, NV, WT, OT, 2, false, 6, true, true>;
  }
  if (unroll == 2) return emb_fwd_kernel<VB, NV, WT, OT, 2, CHECK, 6, true>;
  switch (mb) {
    case 1: return emb_fwd_kernel<VB, NV, WT, OT, 4, CHECK, 1, true>;
    case 6: return emb_fwd_kernel<VB, NV, WT, OT, 4, CHECK, 6, true>;
    default: return emb_fwd_kernel<VB, NV, WT, OT, 4, CHECK, 4, true>;
  }
}
template <int VB, int NV, typename WT, typename OT>
KernelFn pick_c(int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast) {
  if constexpr (NV == 1) {  // ring v2: cp.async rows, more rows in flight than registers allow
    if (!check && full && !shard && !tmast && unroll < 0) {
      switch (-unroll) {
        case 8: return emb_fwd_ring_kernel<VB, WT, OT, 8, 6>;
        case 12: return emb_fwd_ring_kernel<VB, WT, OT, 12, 4>;
        case 16: return emb_fwd_ring_kernel<VB, WT, OT, 16, 3>;
        default: return emb_fwd_ring_kernel<VB, WT, OT, 8, 4>;
      }
    }
  }
  if (unroll < 0) unroll = 4;
  if (unroll >= 8 && !shard && !tmast) {  // shared-memory ring (cp.async) with `unroll` rows in flight per warp
    if constexpr (NV == 1) {
      if (unroll == 16)
        return check ? emb_fwd_async_kernel<VB, NV, WT, OT, 16, true, 3> : emb_fwd_async_kernel<VB, NV, WT, OT, 16, false, 3>;
      return check ? emb_fwd_async_kernel<VB, NV, WT, OT, 8, true, 4> : emb_fwd_async_kernel<VB, NV, WT, OT, 8, false, 4>;
    }
    unroll = 4;
  }
  return check ? pick_u<VB, NV, WT, OT, true>(unroll, mb, full, sidx, shard, tmast)
               : pick_u<VB, NV, WT, OT, false>(unroll, mb, full, sidx, shard, tmast);
}
}  // namespace

KernelFn pick_tile_bf16_f32(int vb, int nv, int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast) {
  using WT = __nv_bfloat16;
  using OT = float;
  if (vb == 8) return pick_c<8, 1, WT, OT>(unroll, check, mb, full, sidx, shard, tmast);
  switch (nv) {
    case 2: return pick_c<16, 2, WT, OT>(unroll, check, mb, full, sidx, shard, tmast);
    case 4: return pick_c<16, 4, WT, OT>(unroll, check, mb, full, sidx, shard, tmast);
    case 8: return pick_c<16, 8, WT, OT>(unroll, check, mb, full, sidx, shard, tmast);
    default: return pick_c<16, 1, WT, OT>(unroll, check, mb, full, sidx, shard, tmast);
  }
}
// dual-stream kernel for 256-B rows (two half-warp bag streams per warp)
KernelFn pick_ds_bf16_f32(int mb) { return mb == 3 ? emb_fwd_ds_kernel<__nv_bfloat16, float, 3> : emb_fwd_ds_kernel<__nv_bfloat16, float, 4>; }
}  // namespace emb
