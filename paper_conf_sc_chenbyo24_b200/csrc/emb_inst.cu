// emb_inst.cu -- instantiations of the fused forward kernel for ONE (weight, output) dtype
// pair, selected at compile time: -DEMB_INST_WT=<float|__nv_bfloat16>
// -DEMB_INST_OT=<float|__nv_bfloat16> -DEMB_INST_NAME=pick_fwd_<w>_<o> (build.py compiles
// this file four times).
#include "emb_dispatch.h"

#if !defined(EMB_INST_WT) || !defined(EMB_INST_OT) || !defined(EMB_INST_NAME)
#error "compile with -DEMB_INST_WT=... -DEMB_INST_OT=... -DEMB_INST_NAME=..."
#endif

namespace emb {
namespace {
using WT = EMB_INST_WT;
using OT = EMB_INST_OT;

// CTAs of 256 threads per SM the register budget is sized for (__launch_bounds__ min
// blocks), measured per tile: fp32 rows of one 16-B vector per lane run three
// row groups in flight at 64 registers / 32 warps per SM (weak zipf -2.7 % against two
// groups at 48 registers / 40 warps); bf16 rows need 8 fp32 accumulators per lane and keep
// two groups at 64 registers (three at 76 registers / 24 warps: +8 %); 8-B lanes fit 40
// registers / 48 warps (three groups there: no gain); rows of several vectors per lane are
// unconstrained.  The f3 / bounds-check (kModeFilt) and f4 (kModeTma) variants carry more
// live state and get one step more registers than the direct kernel of the same tile.
template <int VB, int NV, bool FULL, int MODE>
constexpr int min_blocks() {
  constexpr bool f32w = std::is_same<WT, float>::value;
  if (NV > 1) return 1;
  if (VB == 8 && FULL) return MODE == kModeDirect ? 6 : (MODE == kModeTma ? 5 : 4);
  if (VB == 16 && FULL && MODE == kModeFilt && !f32w) return 3;
  return 4;
}
// row groups in flight: 3 for the direct kernel on fp32 rows of one 16-B vector per lane
template <int VB, int NV, bool FULL, int MODE>
constexpr int row_groups() {
  return (VB == 16 && NV == 1 && FULL && MODE == kModeDirect && std::is_same<WT, float>::value) ? 3 : 2;
}
template <int VB, int NV, bool FULL, int MODE>
KernelFn inst() {
  constexpr int UR = NV > 1 ? 2 : 4;                     // rows per pipeline group
  return emb_fwd_kernel<VB, NV, WT, OT, UR, min_blocks<VB, NV, FULL, MODE>(), FULL, MODE,
                        row_groups<VB, NV, FULL, MODE>()>;
}
template <int VB, int NV, bool FULL>
KernelFn by_mode(int mode) {
  if constexpr (NV == 1 && FULL) {
    if (mode == kModeTma) return inst<VB, NV, FULL, kModeTma>();
  }
  if (mode == kModeFilt) return inst<VB, NV, FULL, kModeFilt>();
  if (mode == kModeDirect) return inst<VB, NV, FULL, kModeDirect>();
  return nullptr;
}
}  // namespace

KernelFn EMB_INST_NAME(int vb, int nv, bool full, int mode) {
  if (nv == 1) {
    if (vb == 16) return full ? by_mode<16, 1, true>(mode) : by_mode<16, 1, false>(mode);
    if (vb == 8) return full ? by_mode<8, 1, true>(mode) : by_mode<8, 1, false>(mode);
    return nullptr;
  }
  if (vb != 16 || !full) return nullptr;
  switch (nv) {
    case 2: return by_mode<16, 2, true>(mode);
    case 4: return by_mode<16, 4, true>(mode);
    case 8: return by_mode<16, 8, true>(mode);
    default: return nullptr;
  }
}
}  // namespace emb
