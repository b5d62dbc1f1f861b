// emb_dispatch.h -- kernel selection of the fused forward, split by (weight, output) dtype
// pair across translation units (emb_inst.cu is compiled once per pair; parallel build).
#pragma once
#include "emb_kernels.cuh"

namespace emb {
using KernelFn = void (*)(FwdParams);
// vb: bytes per lane vector (8 or 16); nv: vectors per lane (1, 2, 4, 8); full: the row is
// exactly the warp's 32 lane vectors; mode: kModeDirect / kModeFilt / kModeTma.
// Returns nullptr for a combination that is not instantiated.
KernelFn pick_fwd_f32_f32(int vb, int nv, bool full, int mode);
KernelFn pick_fwd_f32_bf16(int vb, int nv, bool full, int mode);
KernelFn pick_fwd_bf16_f32(int vb, int nv, bool full, int mode);
KernelFn pick_fwd_bf16_bf16(int vb, int nv, bool full, int mode);
}  // namespace emb
