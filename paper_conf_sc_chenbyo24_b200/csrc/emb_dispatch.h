// emb_dispatch.h -- kernel selection split across translation units (parallel build).
#pragma once
#include "emb_kernels.cuh"

namespace emb {
using KernelFn = void (*)(FwdParams);
KernelFn pick_tile_f32_f32(int vb, int nv, int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast);
KernelFn pick_tile_f32_bf16(int vb, int nv, int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast);
KernelFn pick_tile_bf16_f32(int vb, int nv, int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast);
KernelFn pick_tile_bf16_bf16(int vb, int nv, int unroll, bool check, int mb, bool full, bool sidx, bool shard, bool tmast);
KernelFn pick_ds_f32_f32(int mb);
KernelFn pick_ds_f32_bf16(int mb);
KernelFn pick_ds_bf16_f32(int mb);
KernelFn pick_ds_bf16_bf16(int mb);
}  // namespace emb
