// emb_runtime.cu -- the C ABI of include/emb.h: context, validation, symmetric output
// allocator with CUDA-IPC peer mapping, epochs, launches.
//
// PAPER.md passages: the host side of Listing 2 (L235-254: PGAS_EMB_forward launches
// the fused kernel per device on a non-blocking stream, then synchronizes) becomes
// one context per rank process, launching on the caller's stream; the paper's
// symmetric `outputs` array addressed on any PE (L216, L228, L232) becomes a
// cudaMalloc'd buffer per rank whose IPC handle is all-gathered once over the
// caller's process group.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <unistd.h>

#include <algorithm>
#include <type_traits>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/emb.h"
#define EMB_RUNTIME_TU
#include "emb_kernels.cuh"
#include "emb_dispatch.h"
#include "emb_bwd.cuh"
#include "emb_bwd_sort.cuh"

using namespace emb;

namespace {

constexpr uint64_t kMagic = 0x454d42504741531full;  // "EMBPGAS"
// Output ring depth.  Peer p's forward e+3 writes into slot e % 3 of this rank only after
// p's forward e+2 acquired this rank's epoch-(e+2) signal, i.e. after this rank launched
// its forward e+2: so Y_r(e) stays intact until this rank's second subsequent forward, and
// the host path can overlap the D2H of Y_r(e) with forward e+1.
constexpr int kOutSlots = 3;

struct PeerBlob {
  uint64_t magic;
  int32_t rank, pid;
  uint64_t host_hash;
  uint64_t ptr;          // base of the symmetric allocation in the owner's process
  uint64_t bytes;
  uint64_t slot_off;     // byte offset of slot 0
  uint64_t slot_bytes;   // bytes per slot (B_r*T*d*e_o rounded up to 256)
  uint64_t grad_off;     // byte offset of backward grad slot 0 (0 = backward not enabled)
  uint64_t gslot_bytes;  // bytes per grad slot (B_r*T*d*4 rounded up)
  uint64_t part_off;     // f3: byte offset of partial slot 0 (0 = no row-sharded table)
  uint64_t pslot_bytes;  // f3: bytes per partial slot
  int32_t device;
  int32_t pad;
  cudaIpcMemHandle_t handle;
};

std::string g_init_error;

uint64_t host_hash() {
  char name[256] = {0};
  gethostname(name, sizeof(name) - 1);
  uint64_t h = 1469598103934665603ull;
  for (const char* c = name; *c; ++c) h = (h ^ (uint64_t)(unsigned char)*c) * 1099511628211ull;
  return h;
}

size_t round_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

}  // namespace

struct emb_ctx {
  int rank = 0, G = 1, dev = 0, num_sms = 148;
  emb_allgather_fn ag = nullptr;
  void* user = nullptr;
  bool registered = false;
  // tables
  int T = 0, T_r = 0, d = 0;
  emb_dtype_t wdt = EMB_F32, odt = EMB_F32;
  int64_t B = 0;
  std::vector<int64_t> rows;
  std::vector<int32_t> owner;
  std::vector<int64_t> bstart;          // G+1
  std::vector<int32_t> local;           // global table id of each local shard (ascending (t, s))
  // f3 row-wise sharding
  bool has_shard = false;
  int T_sh = 0, S_max = 1;
  size_t part_off = 0, pslot_bytes = 0;
  std::vector<uint64_t> peer_part_off, peer_pslot_bytes;
  int32_t* d_comb_tglob = nullptr;
  int32_t* d_comb_nsh = nullptr;
  int64_t* d_pbase = nullptr;           // f3 comparison path: unpack-combine maps
  int32_t* d_pstride = nullptr;
  int32_t* d_psoff = nullptr;
  std::vector<int32_t> nloc;            // f3: local shards (incl. whole tables) of every rank
  std::vector<int32_t> tables_of[kMaxG];
  TableDesc* d_tables = nullptr;
  // symmetric buffer (flags at offset 0, slots after)
  char* sym = nullptr;
  size_t sym_bytes = 0, slot_off = 0, slot_bytes = 0;
  std::vector<char*> peer_base;         // mapped base per rank
  std::vector<uint64_t> peer_slot_off, peer_slot_bytes;
  std::vector<bool> peer_ipc;           // opened through cudaIpcOpenMemHandle
  Ctrl* ctrl = nullptr;
  uint64_t epoch = 0;
  // options
  int chunk_rows = 0, ctas_per_sm = 0, stagger = 1, carveout = 0;  // 0: auto per tile
  int64_t timeout_ns = 10000000000ll;
  // gather tiling
  int lanes = 32, vb = 16, nv = 1;
  // comparison path
  int64_t* d_unpack_base = nullptr;
  int32_t* d_unpack_stride = nullptr;
  // e2e staging
  int64_t* d_off_stage = nullptr;
  int64_t* d_idx_stage = nullptr;
  size_t idx_cap = 0;
  // pipelined host path: two input stages, copy-in / copy-out streams, events
  char* p_off[2] = {nullptr, nullptr};
  char* p_idx[2] = {nullptr, nullptr};
  size_t p_cap[2] = {0, 0};               // bytes of p_idx[k]
  size_t p_offcap[2] = {0, 0};            // bytes of p_off[k]
  cudaStream_t s_in = nullptr, s_out = nullptr;
  cudaEvent_t ev_in[2] = {nullptr, nullptr}, ev_kern[2] = {nullptr, nullptr};
  cudaEvent_t ev_out[kOutSlots] = {};   // D2H of the output of epoch e, by e % kOutSlots
  bool kern_rec[2] = {false, false}, out_rec[kOutSlots] = {};
  uint64_t host_calls = 0;
  bool wait_pending = false;            // last forward used EMB_FWD_SEPARATE_WAIT and emb_wait is due
  // f2 backward
  bool bwd_enabled = false;
  size_t grad_off = 0, gslot_bytes = 0;
  std::vector<uint64_t> peer_grad_off, peer_gslot_bytes;
  uint64_t bepoch = 0;
  bool bwd_ready_pending = false;
  int bwd_interleave = 1;
  int bwd_cache = 16;              // per-warp dW row cache slots (0 off, 16 on; one vector per lane)
  int bwd_chunk_rows = 0;          // backward chunk target rows (0: chunk_rows, else 256)
  int bwd_group = 8;               // tables interleaved at a time in the backward (0: all T_r)
  int bwd_algo = 0;                // 0: atomic scatter per bag slice; 1: radix sort + segmented sum
  int64_t bs_cap = 0, bs_R = 0;    // bwd_algo 1 workspace: entries, local rows
  int64_t* d_rowbase = nullptr;
  uint32_t* d_pairs = nullptr;     // entries SoA: codes [bs_stride] then rows [bs_stride]
  uint32_t* d_pairs_b = nullptr;   // radix-sort ping-pong buffer (same layout)
  int64_t bs_stride = 0;           // entries per array: cap + one reduce task, 32-aligned
  uint32_t* d_ghist = nullptr;     // [512][tiles] digit histograms
  uint32_t* d_rbsum = nullptr;
  int64_t rs_nblk = 0;
  int fwd_interleave = 0;
  int tail_div = 4;                // guided tail of the forward's chunk schedule
  int64_t d2h_delay_us = 0;        // test hook: stall the host path's copy-out stream before each D2H
  int tma_store = 0;          // f4: stage pooled vectors, ship 4 per TMA scatter4
  void* d_tmaps = nullptr;    // f4: CUtensorMap [kOutSlots][kMaxG] of every rank's output slots
  float** d_dW = nullptr;
  std::vector<void*> h_dW;
  int blanes = 32, bvb = 16, bnv = 1;
  // f1 trace buffer
  unsigned long long* trace = nullptr;
  uint32_t trace_cap = 0;
  std::string err;
  FwdParams last{};
};

#define FAIL(ctx, code, ...)                        \
  do {                                              \
    char _b[512];                                   \
    snprintf(_b, sizeof(_b), __VA_ARGS__);          \
    if (ctx) (ctx)->err = _b; else g_init_error = _b; \
    return code;                                    \
  } while (0)

#define CK(ctx, call)                                                                                   \
  do {                                                                                                  \
    cudaError_t _e = (call);                                                                            \
    if (_e != cudaSuccess) FAIL(ctx, EMB_ERR_CUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(_e), \
                                __FILE__, __LINE__);                                                    \
  } while (0)

static size_t esize(emb_dtype_t t) { return t == EMB_F32 ? 4 : 2; }
// a row exactly covers the warp's 32 lane vectors (lets the row stride be a constant)
static bool full_row(const emb_ctx* c) { return c->lanes == 32 && (int64_t)c->d * (int64_t)esize(c->wdt) == 32LL * c->vb * c->nv; }
// fused-kernel variant: f4 TMA stores, per-id validity (f3 row shards / bounds check), or the
// default direct-store kernel
static int fwd_mode(bool check, bool shard, bool tmast) {
  if (check || shard) return kModeFilt;
  return tmast ? kModeTma : kModeDirect;
}
// dynamic shared memory: the per-warp id ring (+ f4: two staging buffers of 4 output rows per warp)
static size_t fwd_smem(const emb_ctx* c, int mode) {
  size_t s = (size_t)(kBlock / 32) * kSidxWarpBytes + kSidxWarpBytes;   // + alignment slack of the rings
  if (mode == kModeTma) s += (size_t)(kBlock / 32) * 8 * (size_t)c->d * esize(c->odt);
  return mode == kModeFilt ? 0 : s;
}

// ---------------------------------------------------------------------------- kernel dispatch
namespace {

KernelFn pick_kernel(const emb_ctx* c, int mode) {
  const bool full = full_row(c);
  if (c->wdt == EMB_F32 && c->odt == EMB_F32) return pick_fwd_f32_f32(c->vb, c->nv, full, mode);
  if (c->wdt == EMB_F32 && c->odt == EMB_BF16) return pick_fwd_f32_bf16(c->vb, c->nv, full, mode);
  if (c->wdt == EMB_BF16 && c->odt == EMB_F32) return pick_fwd_bf16_f32(c->vb, c->nv, full, mode);
  return pick_fwd_bf16_bf16(c->vb, c->nv, full, mode);
}

// row-gather tiling: VB bytes per lane-vector, NV vectors per lane, `lanes` active lanes
bool choose_tiling(int64_t rowbytes, size_t wsz, size_t osz, int* lanes, int* vb, int* nv) {
  if (rowbytes <= 0) return false;
  if (rowbytes == 256) { *vb = 8; *nv = 1; *lanes = 32; }
  else if (rowbytes % 16 == 0 && rowbytes <= 512) { *vb = 16; *nv = 1; *lanes = (int)(rowbytes / 16); }
  else if (rowbytes % 512 == 0 && rowbytes <= 4096 && (rowbytes / 512 == 2 || rowbytes / 512 == 4 || rowbytes / 512 == 8)) {
    *vb = 16; *nv = (int)(rowbytes / 512); *lanes = 32;
  } else if (rowbytes % 8 == 0 && rowbytes < 256) { *vb = 8; *nv = 1; *lanes = (int)(rowbytes / 8); }
  else return false;
  // output vector per lane must be >= 4 bytes
  const int epv = *vb / (int)wsz;
  return epv * (int)osz >= 4;
}

}  // namespace

// ---------------------------------------------------------------------------- API
extern "C" {

emb_status_t emb_init(int rank, int world_size, int cuda_device, emb_allgather_fn allgather, void* user,
                      emb_ctx_t** out) {
  if (!out) FAIL((emb_ctx_t*)nullptr, EMB_ERR_ARG, "out is NULL");
  *out = nullptr;
  if (world_size < 1 || world_size > kMaxG) FAIL((emb_ctx_t*)nullptr, EMB_ERR_ARG, "world_size %d not in [1, %d]", world_size, kMaxG);
  if (rank < 0 || rank >= world_size) FAIL((emb_ctx_t*)nullptr, EMB_ERR_ARG, "rank %d not in [0, %d)", rank, world_size);
  if (world_size > 1 && !allgather) FAIL((emb_ctx_t*)nullptr, EMB_ERR_ARG, "allgather callback required for world_size > 1");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0)
    FAIL((emb_ctx_t*)nullptr, EMB_ERR_CUDA, "no CUDA device: %s", cudaGetErrorString(e));
  if (cuda_device < 0 || cuda_device >= ndev) FAIL((emb_ctx_t*)nullptr, EMB_ERR_ARG, "cuda_device %d not in [0, %d)", cuda_device, ndev);
  emb_ctx_t* c = new (std::nothrow) emb_ctx_t();
  if (!c) FAIL((emb_ctx_t*)nullptr, EMB_ERR_NOMEM, "host allocation failed");
  c->rank = rank;
  c->G = world_size;
  c->dev = cuda_device;
  c->ag = allgather;
  c->user = user;
  if (const char* s = getenv("EMB_TIMEOUT_MS")) c->timeout_ns = atoll(s) * 1000000ll;
  e = cudaSetDevice(cuda_device);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  if (e == cudaSuccess) e = cudaMalloc(&c->ctrl, sizeof(Ctrl));
  if (e == cudaSuccess) e = cudaMemset(c->ctrl, 0, sizeof(Ctrl));
  if (e != cudaSuccess) {
    g_init_error = std::string("CUDA init failed: ") + cudaGetErrorString(e);
    delete c;
    return EMB_ERR_CUDA;
  }
  *out = c;
  return EMB_OK;
}

static emb_status_t register_impl(emb_ctx_t* c, int32_t num_tables, const int64_t* rows, const int32_t* num_shards,
                                  const int32_t* shard_owner, const int64_t* shard_row_start, int32_t dim,
                                  emb_dtype_t weight_dtype, emb_dtype_t out_dtype, int64_t global_batch,
                                  const void* const* local_weights) {
  if (!c) return EMB_ERR_ARG;
  if (c->registered) FAIL(c, EMB_ERR_STATE, "tables already registered");
  if (num_tables < 1 || !rows || !num_shards || !shard_owner || !shard_row_start)
    FAIL(c, EMB_ERR_ARG, "num_tables/rows/shards invalid");
  if (weight_dtype != EMB_F32 && weight_dtype != EMB_BF16) FAIL(c, EMB_ERR_ARG, "bad weight dtype");
  if (out_dtype != EMB_F32 && out_dtype != EMB_BF16) FAIL(c, EMB_ERR_ARG, "bad out dtype");
  if (global_batch < c->G) FAIL(c, EMB_ERR_ARG, "global_batch %lld < world_size %d", (long long)global_batch, c->G);
  if (dim < 1) FAIL(c, EMB_ERR_ARG, "dim %d < 1", dim);
  // the forward's work counter is 32-bit: (local shards + 1) x B bags bound the chunks
  int64_t nsh = 0;
  for (int t = 0; t < num_tables; ++t) nsh += num_shards[t] > 0 ? num_shards[t] : 0;
  if ((nsh + 1) * global_batch > (int64_t)INT32_MAX)
    FAIL(c, EMB_ERR_ARG, "(table shards + 1) * global_batch = %lld exceeds 2^31 - 1",
         (long long)(nsh + 1) * (long long)global_batch);
  const size_t wsz = esize(weight_dtype), osz = esize(out_dtype);
  int lanes, vb, nv;
  if (!choose_tiling((int64_t)dim * wsz, wsz, osz, &lanes, &vb, &nv))
    FAIL(c, EMB_ERR_ARG, "unsupported row size d*e = %lld bytes (need multiple of 8, <= 512 or 1024/2048/4096)",
         (long long)dim * (long long)wsz);
  if (((int64_t)dim * (int64_t)osz) % 16 != 0 && c->G > 1) {
    // unpack kernel moves 8-byte pieces at least
    if (((int64_t)dim * (int64_t)osz) % 8 != 0) FAIL(c, EMB_ERR_ARG, "output row bytes must be a multiple of 8");
  }
  c->T = num_tables;
  c->d = dim;
  c->wdt = weight_dtype;
  c->odt = out_dtype;
  c->B = global_batch;
  c->lanes = lanes;
  c->vb = vb;
  c->nv = nv;
  c->rows.assign(rows, rows + num_tables);
  c->owner.assign(num_tables, -1);
  c->local.clear();
  for (int g = 0; g < kMaxG; ++g) c->tables_of[g].clear();
  // shards: (t, s) -> rows [lo, hi) on shard_owner; a table with one shard is table-wise
  struct LocalShard { int t, s, part; int64_t lo, hi; };
  std::vector<LocalShard> lsh;
  std::vector<int32_t> comb_tglob, comb_nsh;
  std::vector<int32_t> ent_owner, ent_k, ent_off(1, 0), nloc(c->G, 0);   // every (t, s): owner, its index there
  c->T_sh = 0;
  c->S_max = 1;
  for (int t = 0; t < num_tables; ++t)
    if (num_shards[t] > 1) { ++c->T_sh; c->S_max = std::max(c->S_max, (int)num_shards[t]); }
  int64_t k = 0;
  int ksh = 0;
  for (int t = 0; t < num_tables; ++t) {
    if (rows[t] < 1 || rows[t] > 0x7fffffffLL)
      FAIL(c, EMB_ERR_ARG, "rows[%d] = %lld not in [1, 2^31) (row ids travel as 32-bit)", t, (long long)rows[t]);
    const int S = num_shards[t];
    if (S < 1 || S > 64) FAIL(c, EMB_ERR_ARG, "num_shards[%d] = %d not in [1, 64]", t, S);
    if (S > 1) {
      comb_tglob.push_back(t);
      comb_nsh.push_back(S);
    }
    for (int sh = 0; sh < S; ++sh, ++k) {
      const int32_t o = shard_owner[k];
      const int64_t lo = shard_row_start[k];
      const int64_t hi = (sh + 1 < S) ? shard_row_start[k + 1] : rows[t];
      if (o < 0 || o >= c->G) FAIL(c, EMB_ERR_ARG, "owner of table %d shard %d = %d not in [0, %d)", t, sh, o, c->G);
      if ((sh == 0 && lo != 0) || lo < 0 || hi <= lo || hi > rows[t])
        FAIL(c, EMB_ERR_ARG, "table %d shard %d rows [%lld, %lld) invalid", t, sh, (long long)lo, (long long)hi);
      if (S == 1) {
        c->owner[t] = o;
        c->tables_of[o].push_back(t);
      }
      ent_owner.push_back(o);
      ent_k.push_back(nloc[o]++);
      if (o == c->rank) {
        lsh.push_back({t, sh, S > 1 ? ksh * c->S_max + sh : -1, lo, hi});
        c->local.push_back(t);
      }
    }
    if (S > 1) ++ksh;
    ent_off.push_back((int32_t)ent_owner.size());
  }
  c->has_shard = c->T_sh > 0;
  c->T_r = (int)c->local.size();
  // contiguous batch split (C8)
  c->bstart.assign(c->G + 1, 0);
  {
    const int64_t q = global_batch / c->G, rem = global_batch % c->G;
    for (int r = 0; r < c->G; ++r) c->bstart[r + 1] = c->bstart[r] + q + (r < rem ? 1 : 0);
  }
  CK(c, cudaSetDevice(c->dev));
  // table descriptors
  std::vector<TableDesc> td(std::max(c->T_r, 1));
  for (int i = 0; i < c->T_r; ++i) {
    const void* w = local_weights ? local_weights[i] : nullptr;
    if (!w) FAIL(c, EMB_ERR_ARG, "local_weights[%d] is NULL", i);
    if (((uintptr_t)w) % 16 != 0) FAIL(c, EMB_ERR_ARG, "local_weights[%d] not 16-byte aligned", i);
    td[i].w = w;
    td[i].rows = lsh[i].hi - lsh[i].lo;
    td[i].mrows = rows[lsh[i].t];
    td[i].tglob = lsh[i].t;
    td[i].part = lsh[i].part;
    td[i].lo = lsh[i].lo;
  }
  if (c->has_shard) {
    // f3 comparison path: recv = [G][B_r][T_loc(src)][d] fp32 partials; the partial of shard
    // (t, s) for sample b is vector R0[src] + b * T_loc(src) + k (k = its index on src)
    const int64_t Br0 = c->bstart[c->rank + 1] - c->bstart[c->rank];
    std::vector<int64_t> R0(c->G + 1, 0), pbase(ent_owner.size());
    std::vector<int32_t> pstride(ent_owner.size());
    for (int g = 0; g < c->G; ++g) R0[g + 1] = R0[g] + Br0 * nloc[g];
    for (size_t e = 0; e < ent_owner.size(); ++e) {
      pbase[e] = R0[ent_owner[e]] + ent_k[e];
      pstride[e] = nloc[ent_owner[e]];
    }
    c->nloc = nloc;
    CK(c, cudaMalloc(&c->d_pbase, std::max<size_t>(pbase.size(), 1) * sizeof(int64_t)));
    CK(c, cudaMalloc(&c->d_pstride, std::max<size_t>(pstride.size(), 1) * sizeof(int32_t)));
    CK(c, cudaMalloc(&c->d_psoff, ent_off.size() * sizeof(int32_t)));
    CK(c, cudaMemcpy(c->d_pbase, pbase.data(), pbase.size() * sizeof(int64_t), cudaMemcpyHostToDevice));
    CK(c, cudaMemcpy(c->d_pstride, pstride.data(), pstride.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
    CK(c, cudaMemcpy(c->d_psoff, ent_off.data(), ent_off.size() * sizeof(int32_t), cudaMemcpyHostToDevice));
    CK(c, cudaMalloc(&c->d_comb_tglob, c->T_sh * sizeof(int32_t)));
    CK(c, cudaMalloc(&c->d_comb_nsh, c->T_sh * sizeof(int32_t)));
    CK(c, cudaMemcpy(c->d_comb_tglob, comb_tglob.data(), c->T_sh * sizeof(int32_t), cudaMemcpyHostToDevice));
    CK(c, cudaMemcpy(c->d_comb_nsh, comb_nsh.data(), c->T_sh * sizeof(int32_t), cudaMemcpyHostToDevice));
  }
  CK(c, cudaMalloc(&c->d_tables, td.size() * sizeof(TableDesc)));
  CK(c, cudaMemcpy(c->d_tables, td.data(), td.size() * sizeof(TableDesc), cudaMemcpyHostToDevice));
  // unpack maps: recv = [G][B_r][T_src][d]; vector index of (b, t) = R0[src] + b*T_src + t_l
  if (!c->has_shard) {
    const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
    std::vector<int64_t> base(num_tables);
    std::vector<int32_t> stride(num_tables);
    int64_t R0 = 0;
    for (int s = 0; s < c->G; ++s) {
      const int Ts = (int)c->tables_of[s].size();
      for (int i = 0; i < Ts; ++i) {
        base[c->tables_of[s][i]] = R0 + i;
        stride[c->tables_of[s][i]] = Ts;
      }
      R0 += Br * Ts;
    }
    CK(c, cudaMalloc(&c->d_unpack_base, num_tables * sizeof(int64_t)));
    CK(c, cudaMalloc(&c->d_unpack_stride, num_tables * sizeof(int32_t)));
    CK(c, cudaMemcpy(c->d_unpack_base, base.data(), num_tables * sizeof(int64_t), cudaMemcpyHostToDevice));
    CK(c, cudaMemcpy(c->d_unpack_stride, stride.data(), num_tables * sizeof(int32_t), cudaMemcpyHostToDevice));
  }
  // symmetric buffer: [flags: G u32, padded to 512 B][output slot 0][slot 1][slot 2]
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  // header: [fwd flags G u32 @0][bwd ready G u32 @64][bwd done G u32 @128], 512 B
  c->slot_off = 512;
  c->slot_bytes = round_up((size_t)Br * (size_t)num_tables * (size_t)dim * osz, 512);
  c->sym_bytes = c->slot_off + kOutSlots * c->slot_bytes;
  if (c->has_shard) {  // f3 partial slots [2][B_r][T_sh * S_max][d] fp32
    if (dim % 4 != 0) FAIL(c, EMB_ERR_ARG, "row-sharded tables need dim %% 4 == 0");
    c->part_off = c->sym_bytes;
    c->pslot_bytes = round_up((size_t)Br * (size_t)c->T_sh * (size_t)c->S_max * (size_t)dim * 4, 512);
    c->sym_bytes += 2 * c->pslot_bytes;
  }
  if (c->bwd_enabled) {
    if (!choose_tiling((int64_t)dim * 4, 4, 4, &c->blanes, &c->bvb, &c->bnv) || c->bnv > 4)
      FAIL(c, EMB_ERR_ARG, "backward: unsupported fp32 row size %d bytes", dim * 4);
    c->grad_off = c->sym_bytes;
    c->gslot_bytes = round_up((size_t)Br * (size_t)num_tables * (size_t)dim * 4, 512);
    c->sym_bytes += 2 * c->gslot_bytes;
  }
  {
    cudaError_t e = cudaMalloc(&c->sym, c->sym_bytes);
    if (e == cudaErrorMemoryAllocation) FAIL(c, EMB_ERR_NOMEM, "symmetric buffer of %zu bytes: out of memory", c->sym_bytes);
    CK(c, e);
  }
  CK(c, cudaMemset(c->sym, 0, c->slot_off));
  // exchange
  PeerBlob mine{};
  mine.magic = kMagic;
  mine.rank = c->rank;
  mine.pid = (int32_t)getpid();
  mine.host_hash = host_hash();
  mine.ptr = (uint64_t)(uintptr_t)c->sym;
  mine.bytes = c->sym_bytes;
  mine.slot_off = c->slot_off;
  mine.slot_bytes = c->slot_bytes;
  mine.grad_off = c->grad_off;
  mine.gslot_bytes = c->gslot_bytes;
  mine.part_off = c->part_off;
  mine.pslot_bytes = c->pslot_bytes;
  mine.device = c->dev;
  CK(c, cudaIpcGetMemHandle(&mine.handle, c->sym));
  std::vector<PeerBlob> all(c->G);
  if (c->G == 1) {
    all[0] = mine;
  } else {
    if (c->ag(c->user, &mine, all.data(), sizeof(PeerBlob)) != 0) FAIL(c, EMB_ERR_PEER, "allgather of IPC handles failed");
  }
  c->peer_base.assign(c->G, nullptr);
  c->peer_slot_off.assign(c->G, 0);
  c->peer_slot_bytes.assign(c->G, 0);
  c->peer_ipc.assign(c->G, false);
  c->peer_grad_off.assign(c->G, 0);
  c->peer_gslot_bytes.assign(c->G, 0);
  c->peer_part_off.assign(c->G, 0);
  c->peer_pslot_bytes.assign(c->G, 0);
  for (int p = 0; p < c->G; ++p) {
    const PeerBlob& b = all[p];
    if (b.magic != kMagic || b.rank != p) FAIL(c, EMB_ERR_PEER, "bad peer blob from rank %d", p);
    if (b.host_hash != mine.host_hash) FAIL(c, EMB_ERR_PEER, "rank %d is on another host (multi-node is out of scope)", p);
    c->peer_slot_off[p] = b.slot_off;
    c->peer_slot_bytes[p] = b.slot_bytes;
    c->peer_grad_off[p] = b.grad_off;
    c->peer_gslot_bytes[p] = b.gslot_bytes;
    c->peer_part_off[p] = b.part_off;
    c->peer_pslot_bytes[p] = b.pslot_bytes;
    if ((b.grad_off != 0) != c->bwd_enabled) FAIL(c, EMB_ERR_PEER, "rank %d disagrees on enable_backward", p);
    if (p == c->rank) {
      c->peer_base[p] = c->sym;
    } else if (b.pid == mine.pid) {  // simulated rank in this process: raw pointer
      if (b.device != c->dev) {
        cudaError_t e = cudaDeviceEnablePeerAccess(b.device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(c, e);
        cudaGetLastError();
      }
      c->peer_base[p] = (char*)(uintptr_t)b.ptr;
    } else {
      void* ptr = nullptr;
      cudaError_t e = cudaIpcOpenMemHandle(&ptr, b.handle, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) FAIL(c, EMB_ERR_PEER, "cudaIpcOpenMemHandle(rank %d) failed: %s", p, cudaGetErrorString(e));
      c->peer_base[p] = (char*)ptr;
      c->peer_ipc[p] = true;
    }
  }
  // barrier: every rank mapped everything before anyone writes
  if (c->G > 1) {
    int one = 1;
    std::vector<int> r(c->G);
    if (c->ag(c->user, &one, r.data(), sizeof(int)) != 0) FAIL(c, EMB_ERR_PEER, "registration barrier failed");
  }
  c->registered = true;
  // Load every kernel this context may launch now (CUDA lazy loading would otherwise load
  // a kernel at its first launch, and a module load can wait for a running kernel -- e.g.
  // the in-kernel peer wait of another rank sharing this GPU).
  {
    cudaFuncAttributes a;
    for (int mode : {kModeDirect, kModeFilt, kModeTma}) {
      KernelFn k = pick_kernel(c, mode);
      if (k) cudaFuncGetAttributes(&a, k);
    }
    cudaFuncGetAttributes(&a, emb_wait_kernel);
    cudaFuncGetAttributes(&a, emb_sleep_kernel);
    cudaFuncGetAttributes(&a, emb_unpack_rows_kernel<uint4>);
    cudaFuncGetAttributes(&a, emb_unpack_rows_kernel<uint2>);
    cudaFuncGetAttributes(&a, emb_unpack_partials_kernel<float>);
    cudaFuncGetAttributes(&a, emb_unpack_partials_kernel<__nv_bfloat16>);
    cudaFuncGetAttributes(&a, emb_combine_kernel<float>);
    cudaFuncGetAttributes(&a, emb_combine_kernel<__nv_bfloat16>);
    cudaFuncGetAttributes(&a, emb_bwd_signal_kernel);
    cudaFuncGetAttributes(&a, emb_bwd_slot_wait_kernel);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<8, 1>);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<16, 1>);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<16, 2>);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<16, 4>);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<8, 1, 16>);
    cudaFuncGetAttributes(&a, emb_bwd_kernel<16, 1, 16>);
    cudaFuncGetAttributes(&a, emb_bsort_scan_sum_kernel);
    cudaFuncGetAttributes(&a, emb_bsort_scan_top_kernel);
    cudaFuncGetAttributes(&a, emb_bsort_scan_apply_kernel);
    cudaFuncGetAttributes(&a, emb_bradix_gen_kernel);
    cudaFuncGetAttributes(&a, emb_bradix_up_kernel);
    cudaFuncGetAttributes(&a, emb_bradix_down_kernel);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<8, 1, 2, 1, false>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 1, 2, 4, false>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 2, 2, 1, false>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 4, 2, 1, false>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<8, 1, 2, 1, true>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 1, 2, 4, true>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 2, 2, 1, true>);
    cudaFuncGetAttributes(&a, emb_bsort_reduce_kernel<16, 4, 2, 1, true>);
    cudaGetLastError();
  }
  return EMB_OK;
}

emb_status_t emb_register_tables(emb_ctx_t* c, int32_t num_tables, const int64_t* rows, const int32_t* owner,
                                 int32_t dim, emb_dtype_t weight_dtype, emb_dtype_t out_dtype, int64_t global_batch,
                                 const void* const* local_weights) {
  if (!c) return EMB_ERR_ARG;
  if (num_tables < 1 || !rows || !owner) FAIL(c, EMB_ERR_ARG, "num_tables/rows/owner invalid");
  std::vector<int32_t> ns(num_tables, 1);
  std::vector<int64_t> lo(num_tables, 0);
  return register_impl(c, num_tables, rows, ns.data(), owner, lo.data(), dim, weight_dtype, out_dtype, global_batch,
                       local_weights);
}

emb_status_t emb_register_sharded_tables(emb_ctx_t* c, int32_t num_tables, const int64_t* rows,
                                         const int32_t* num_shards, const int32_t* shard_owner,
                                         const int64_t* shard_row_start, int32_t dim, emb_dtype_t weight_dtype,
                                         emb_dtype_t out_dtype, int64_t global_batch,
                                         const void* const* local_weights) {
  return register_impl(c, num_tables, rows, num_shards, shard_owner, shard_row_start, dim, weight_dtype, out_dtype,
                       global_batch, local_weights);
}

static char* out_slot(emb_ctx_t* c, int g, uint64_t epoch) {   // rank g's output slot of `epoch`
  return c->peer_base[g] + c->peer_slot_off[g] + (size_t)(epoch % kOutSlots) * c->peer_slot_bytes[g];
}

static emb_status_t launch_combine(emb_ctx_t* c, cudaStream_t s) {
  if (!c->has_shard) return EMB_OK;
  const int pslot = (int)(c->epoch & 1);
  const float* part = reinterpret_cast<const float*>(c->sym + c->part_off + (size_t)pslot * c->pslot_bytes);
  char* out = out_slot(c, c->rank, c->epoch);
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  const int64_t total = Br * c->T_sh * (c->d / 4);
  int grid = (int)std::min<int64_t>((total + kBlock - 1) / kBlock, (int64_t)c->num_sms * 8);
  if (grid < 1) return EMB_OK;
  if (c->odt == EMB_F32)
    emb_combine_kernel<float><<<grid, kBlock, 0, s>>>(part, out, c->d_comb_tglob, c->d_comb_nsh, Br, c->T, c->T_sh,
                                                      c->S_max, c->d);
  else
    emb_combine_kernel<__nv_bfloat16><<<grid, kBlock, 0, s>>>(part, out, c->d_comb_tglob, c->d_comb_nsh, Br, c->T,
                                                              c->T_sh, c->S_max, c->d);
  CK(c, cudaGetLastError());
  return EMB_OK;
}

// f4: one 2-D tensor map per (slot, destination rank) over that rank's output slot viewed
// as [B_dst*T rows][d], box = one row; the kernel scatters 4 rows per TMA store
static emb_status_t build_tmaps(emb_ctx_t* c) {
  if (c->d_tmaps) return EMB_OK;
  if (!full_row(c) || c->nv != 1 || c->has_shard || c->d > 256)
    FAIL(c, EMB_ERR_ARG, "tma_store needs full-warp rows with one vector per lane, d <= 256, no row sharding");
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(c, cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  if (!fn || q != cudaDriverEntryPointSuccess) FAIL(c, EMB_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  auto encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  std::vector<CUtensorMap> maps(kOutSlots * kMaxG);
  memset(maps.data(), 0, maps.size() * sizeof(CUtensorMap));
  const size_t eo = esize(c->odt);
  for (int slot = 0; slot < kOutSlots; ++slot)
    for (int g = 0; g < c->G; ++g) {
      void* base = out_slot(c, g, (uint64_t)slot);
      const cuuint64_t rows = (cuuint64_t)(c->bstart[g + 1] - c->bstart[g]) * (cuuint64_t)c->T;
      cuuint64_t dims[2] = {(cuuint64_t)c->d, rows};
      cuuint64_t strides[1] = {(cuuint64_t)c->d * eo};
      cuuint32_t box[2] = {(cuuint32_t)c->d, 1};
      cuuint32_t es[2] = {1, 1};
      CUresult r = encode(&maps[slot * kMaxG + g],
                          c->odt == EMB_F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                          base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                          CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) FAIL(c, EMB_ERR_CUDA, "cuTensorMapEncodeTiled(slot %d, rank %d) failed: %d", slot, g, (int)r);
    }
  CK(c, cudaMalloc(&c->d_tmaps, maps.size() * sizeof(CUtensorMap)));
  CK(c, cudaMemcpy(c->d_tmaps, maps.data(), maps.size() * sizeof(CUtensorMap), cudaMemcpyHostToDevice));
  return EMB_OK;
}

static emb_status_t fill_params(emb_ctx_t* c, const void* offsets, const void* indices, bool i32, bool pgas, char* send,
                                FwdParams* p) {
  memset(p, 0, sizeof(*p));
  p->tables = c->d_tables;
  p->offsets = offsets;
  p->indices = indices;
  p->idx32 = i32 ? 1 : 0;
  p->B = c->B;
  p->T_r = c->T_r;
  p->d = c->d;
  p->G = c->G;
  p->rank = c->rank;
  p->lanes = c->lanes;
  // forward chunk target rows: 0 = auto (192 for fp32 rows, 256 for bf16 rows: measured
  // weak zipf -1.2 %, uniform -0.8 %, single -0.4/-1.5 %, strong -0.6 %; bf16 large_shard
  // +1.4 % at 192)
  p->chunk_rows = c->chunk_rows ? c->chunk_rows : (c->wdt == EMB_F32 ? 192 : 256);
  p->stagger = c->stagger;
  p->interleave = c->fwd_interleave;
  p->tail_div = c->tail_div;
  p->ctrl = c->ctrl;
  p->timeout_ns = c->timeout_ns;
  for (int g = 0; g <= c->G; ++g) p->bstart[g] = c->bstart[g];
  for (int g = c->G + 1; g <= kMaxG; ++g) p->bstart[g] = INT64_MAX;
  p->my_flags = reinterpret_cast<const uint32_t*>(c->sym);
  const size_t osz = esize(c->odt);
  if (pgas) {
    const int pslot = (int)(c->epoch & 1);  // epoch already advanced for this forward
    p->rowstride = c->T;
    p->use_tglob = 1;
    p->signal = 1;
    for (int g = 0; g < c->G; ++g) {
      p->out_base[g] = out_slot(c, g, c->epoch);
      p->peer_flag[g] = (g == c->rank) ? nullptr : reinterpret_cast<uint32_t*>(c->peer_base[g]) + c->rank;
      if (c->has_shard)
        p->part_base[g] = c->peer_base[g] + c->peer_part_off[g] + (size_t)pslot * c->peer_pslot_bytes[g];
    }
    p->part_stride = (int64_t)c->T_sh * c->S_max;
    p->tmaps = (c->tma_store && c->d_tmaps)
                   ? static_cast<const char*>(c->d_tmaps) + (size_t)(c->epoch % kOutSlots) * kMaxG * sizeof(CUtensorMap)
                   : nullptr;
  } else {
    p->rowstride = c->T_r;
    p->use_tglob = 0;
    p->signal = 0;
    for (int g = 0; g < c->G; ++g)  // send = [G][B_dst][T_r][d]: block of dst starts at s_dst*T_r rows
      p->out_base[g] = send + (size_t)c->bstart[g] * (size_t)c->T_r * (size_t)c->d * osz;
  }
  p->ostep = p->rowstride * (int64_t)c->d * (int64_t)osz;
  p->epoch = (uint32_t)c->epoch;
  p->trace = c->trace;
  p->trace_cap = c->trace_cap;
  return EMB_OK;
}

// CTAs of 256 threads the kernel's registers allow per SM (the occupancy it was built for)
static int ctas_by_regs(KernelFn k) {
  cudaFuncAttributes a;
  if (cudaFuncGetAttributes(&a, k) != cudaSuccess || a.numRegs <= 0) return 4;
  const int per_warp = (int)round_up((size_t)a.numRegs * 32, 256);
  return std::max(1, 65536 / (per_warp * (kBlock / 32)));
}

static emb_status_t launch_fwd(emb_ctx_t* c, const FwdParams& p, uint32_t flags, cudaStream_t s) {
  const bool chk = (flags & EMB_FWD_CHECK_BOUNDS) != 0, shard = p.part_stride > 0, tmast = p.tmaps != nullptr;
  const int mode = fwd_mode(chk, shard, tmast);
  KernelFn k = pick_kernel(c, mode);
  if (!k) FAIL(c, EMB_ERR_ARG, "no kernel for this row tiling / mode");
  const size_t smem = fwd_smem(c, mode);
  if (smem > 0) CK(c, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  // the gather lives off L1 hits of zipf-hot rows: ask for the smallest shared-memory
  // carve-out that still fits the occupancy target (the CTAs the registers allow, each
  // with its id ring + 1 KB driver reserve), so the rest of the 256 KB per SM stays L1
  if (c->carveout > 0) {
    CK(c, cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, c->carveout));
  } else if (c->carveout == 0) {
    const size_t want = (size_t)ctas_by_regs(k);
    const int pct = smem == 0 ? 0 : (int)std::min<size_t>(100, (want * (smem + 1024) * 100 + 233471) / 233472);
    CK(c, cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, pct));
  }
  int per_sm = c->ctas_per_sm;
  if (per_sm <= 0) {
    CK(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kBlock, smem));
    if (per_sm < 1) per_sm = 1;
  }
  const int grid = c->num_sms * per_sm;
  k<<<grid, kBlock, smem, s>>>(p);
  CK(c, cudaGetLastError());
  return EMB_OK;
}

static emb_status_t wait_impl(emb_ctx_t* c, cudaStream_t s) {
  c->wait_pending = false;
  if (c->G > 1) {
    emb_wait_kernel<<<1, 32, 0, s>>>(c->last);
    CK(c, cudaGetLastError());
  }
  return launch_combine(c, s);
}

static emb_status_t forward_impl(emb_ctx_t* c, const void* offsets, const void* indices, bool i32, uint32_t flags,
                                 cudaStream_t s, void** out) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered) FAIL(c, EMB_ERR_STATE, "emb_forward before emb_register_tables");
  if (c->T_r > 0 && (!offsets || !indices)) FAIL(c, EMB_ERR_ARG, "offsets/indices NULL");
  if (flags & ~(EMB_FWD_CHECK_BOUNDS | EMB_FWD_SEPARATE_WAIT)) FAIL(c, EMB_ERR_ARG, "unknown flag bits 0x%x", flags);
  CK(c, cudaSetDevice(c->dev));
  if (c->tma_store) {
    emb_status_t st0 = build_tmaps(c);
    if (st0 != EMB_OK) return st0;
  }
  // a previous EMB_FWD_SEPARATE_WAIT forward that was never completed is completed first:
  // the output ring's reuse argument needs every forward's wait before the next launch
  if (c->wait_pending) {
    emb_status_t st0 = wait_impl(c, s);
    if (st0 != EMB_OK) return st0;
  }
  c->epoch += 1;
  FwdParams p;
  fill_params(c, offsets, indices, i32, true, nullptr, &p);
  p.wait = (flags & EMB_FWD_SEPARATE_WAIT) ? 0 : 1;
  p.check = (flags & EMB_FWD_CHECK_BOUNDS) ? 1 : 0;
  c->last = p;
  emb_status_t st = launch_fwd(c, p, flags, s);
  if (st != EMB_OK) return st;
  if (!(flags & EMB_FWD_SEPARATE_WAIT)) {  // f3: partials landed (in-kernel wait) -> combine
    st = launch_combine(c, s);
    if (st != EMB_OK) return st;
  } else {
    c->wait_pending = true;
  }
  if (out) *out = out_slot(c, c->rank, c->epoch);
  return EMB_OK;
}

emb_status_t emb_forward(emb_ctx_t* c, const int64_t* offsets, const int64_t* indices, uint32_t flags, void* stream,
                         void** out) {
  return forward_impl(c, offsets, indices, false, flags, (cudaStream_t)stream, out);
}

emb_status_t emb_forward_i32(emb_ctx_t* c, const int32_t* offsets, const int32_t* indices, uint32_t flags, void* stream,
                             void** out) {
  return forward_impl(c, offsets, indices, true, flags, (cudaStream_t)stream, out);
}

emb_status_t emb_wait(emb_ctx_t* c, void* stream) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered || c->epoch == 0) FAIL(c, EMB_ERR_STATE, "emb_wait without a forward");
  CK(c, cudaSetDevice(c->dev));
  return wait_impl(c, (cudaStream_t)stream);
}

emb_status_t emb_forward_host(emb_ctx_t* c, const int64_t* h_offsets, const int64_t* h_indices, uint32_t flags,
                              void* stream, void* h_out) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered) FAIL(c, EMB_ERR_STATE, "emb_forward_host before emb_register_tables");
  if (!h_offsets || !h_out || (c->T_r > 0 && !h_indices)) FAIL(c, EMB_ERR_ARG, "NULL host buffer");
  CK(c, cudaSetDevice(c->dev));
  cudaStream_t s = (cudaStream_t)stream;
  const size_t noff = (size_t)c->T_r * (size_t)c->B + 1;
  const int64_t nnz = h_offsets[noff - 1];
  if (nnz < 0) FAIL(c, EMB_ERR_ARG, "negative nnz");
  if (!c->d_off_stage) CK(c, cudaMalloc(&c->d_off_stage, noff * sizeof(int64_t)));
  if ((size_t)nnz > c->idx_cap || !c->d_idx_stage) {
    CK(c, cudaStreamSynchronize(s));
    if (c->d_idx_stage) CK(c, cudaFree(c->d_idx_stage));
    c->idx_cap = std::max<size_t>((size_t)nnz, 1) + (size_t)nnz / 4;
    CK(c, cudaMalloc(&c->d_idx_stage, c->idx_cap * sizeof(int64_t)));
  }
  CK(c, cudaMemcpyAsync(c->d_off_stage, h_offsets, noff * sizeof(int64_t), cudaMemcpyHostToDevice, s));
  if (nnz > 0) CK(c, cudaMemcpyAsync(c->d_idx_stage, h_indices, (size_t)nnz * sizeof(int64_t), cudaMemcpyHostToDevice, s));
  void* dout = nullptr;
  emb_status_t st = forward_impl(c, c->d_off_stage, c->d_idx_stage, false, flags & ~EMB_FWD_SEPARATE_WAIT, s, &dout);
  if (st != EMB_OK) return st;
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  CK(c, cudaMemcpyAsync(h_out, dout, (size_t)Br * c->T * c->d * esize(c->odt), cudaMemcpyDeviceToHost, s));
  return EMB_OK;
}

// pipelined host path (both index widths): H2D of call k into stage k & 1 on the copy-in
// stream, the forward on the caller's stream, D2H of Y_r on the copy-out stream
static emb_status_t host_async_impl(emb_ctx_t* c, const void* h_offsets, const void* h_indices, bool i32,
                                    uint32_t flags, cudaStream_t s, void* h_out) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered) FAIL(c, EMB_ERR_STATE, "emb_forward_host_async before emb_register_tables");
  if (!h_offsets || !h_out || (c->T_r > 0 && !h_indices)) FAIL(c, EMB_ERR_ARG, "NULL host buffer");
  CK(c, cudaSetDevice(c->dev));
  if (!c->s_in) {
    CK(c, cudaStreamCreateWithFlags(&c->s_in, cudaStreamNonBlocking));
    CK(c, cudaStreamCreateWithFlags(&c->s_out, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CK(c, cudaEventCreateWithFlags(&c->ev_in[i], cudaEventDisableTiming));
      CK(c, cudaEventCreateWithFlags(&c->ev_kern[i], cudaEventDisableTiming));
    }
    for (int i = 0; i < kOutSlots; ++i) CK(c, cudaEventCreateWithFlags(&c->ev_out[i], cudaEventDisableTiming));
  }
  const size_t isz = i32 ? 4 : 8;
  const int k = (int)(c->host_calls & 1);
  const size_t noff = (size_t)c->T_r * (size_t)c->B + 1;
  const int64_t nnz = i32 ? (int64_t) static_cast<const int32_t*>(h_offsets)[noff - 1]
                          : static_cast<const int64_t*>(h_offsets)[noff - 1];
  if (nnz < 0) FAIL(c, EMB_ERR_ARG, "negative nnz");
  if (!c->p_off[k] || noff * isz > c->p_offcap[k] || (size_t)nnz * isz > c->p_cap[k]) {
    // (re)allocate stage k: drain everything first
    CK(c, cudaStreamSynchronize(c->s_in));
    CK(c, cudaStreamSynchronize(c->s_out));
    CK(c, cudaStreamSynchronize(s));
    if (c->p_off[k]) CK(c, cudaFree(c->p_off[k]));
    if (c->p_idx[k]) CK(c, cudaFree(c->p_idx[k]));
    c->p_offcap[k] = noff * 8;
    c->p_cap[k] = (std::max<size_t>((size_t)nnz, 1) + (size_t)nnz / 4) * 8;
    CK(c, cudaMalloc(&c->p_off[k], c->p_offcap[k]));
    CK(c, cudaMalloc(&c->p_idx[k], c->p_cap[k]));
  }
  // 1. H2D into stage k once the kernel that last read it (two calls ago) is done
  if (c->kern_rec[k]) CK(c, cudaStreamWaitEvent(c->s_in, c->ev_kern[k], 0));
  CK(c, cudaMemcpyAsync(c->p_off[k], h_offsets, noff * isz, cudaMemcpyHostToDevice, c->s_in));
  if (nnz > 0) CK(c, cudaMemcpyAsync(c->p_idx[k], h_indices, (size_t)nnz * isz, cudaMemcpyHostToDevice, c->s_in));
  CK(c, cudaEventRecord(c->ev_in[k], c->s_in));
  // 2. forward e on the caller's stream after its inputs landed and after the D2H of
  //    Y_r(e-2) finished: a peer's forward e+1 may overwrite slot (e-2) % 3 as soon as
  //    this rank's forward e has signalled (kOutSlots ring argument)
  const uint64_t e = c->epoch + 1;
  CK(c, cudaStreamWaitEvent(s, c->ev_in[k], 0));
  if (e >= 3 && c->out_rec[(e - 2) % kOutSlots]) CK(c, cudaStreamWaitEvent(s, c->ev_out[(e - 2) % kOutSlots], 0));
  void* dout = nullptr;
  emb_status_t st = forward_impl(c, c->p_off[k], c->p_idx[k], i32, flags & ~EMB_FWD_SEPARATE_WAIT, s, &dout);
  if (st != EMB_OK) return st;
  CK(c, cudaEventRecord(c->ev_kern[k], s));
  c->kern_rec[k] = true;
  // 3. D2H of Y_r(e) on the copy-out stream, overlapping the next call's H2D and kernel
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  CK(c, cudaStreamWaitEvent(c->s_out, c->ev_kern[k], 0));
  if (c->d2h_delay_us > 0) emb_sleep_kernel<<<1, 1, 0, c->s_out>>>((uint64_t)c->d2h_delay_us * 1000ull);
  CK(c, cudaMemcpyAsync(h_out, dout, (size_t)Br * c->T * c->d * esize(c->odt), cudaMemcpyDeviceToHost, c->s_out));
  CK(c, cudaEventRecord(c->ev_out[e % kOutSlots], c->s_out));
  c->out_rec[e % kOutSlots] = true;
  c->host_calls += 1;
  return EMB_OK;
}

emb_status_t emb_forward_host_async(emb_ctx_t* c, const int64_t* h_offsets, const int64_t* h_indices, uint32_t flags,
                                    void* stream, void* h_out) {
  return host_async_impl(c, h_offsets, h_indices, false, flags, (cudaStream_t)stream, h_out);
}

emb_status_t emb_forward_host_async_i32(emb_ctx_t* c, const int32_t* h_offsets, const int32_t* h_indices,
                                        uint32_t flags, void* stream, void* h_out) {
  return host_async_impl(c, h_offsets, h_indices, true, flags, (cudaStream_t)stream, h_out);
}

emb_status_t emb_host_drain(emb_ctx_t* c, void* stream) {
  if (!c) return EMB_ERR_ARG;
  if (!c->s_in) return EMB_OK;
  CK(c, cudaSetDevice(c->dev));
  cudaStream_t s = (cudaStream_t)stream;
  for (int i = 0; i < kOutSlots; ++i)
    if (c->out_rec[i]) CK(c, cudaStreamWaitEvent(s, c->ev_out[i], 0));
  return EMB_OK;
}

static void fill_bwd_params(emb_ctx_t* c, BwdParams* p) {
  memset(p, 0, sizeof(*p));
  p->tables = c->d_tables;
  p->dW = c->d_dW;
  p->B = c->B;
  for (int g = 0; g <= c->G; ++g) p->bstart[g] = c->bstart[g];
  for (int g = c->G + 1; g <= kMaxG; ++g) p->bstart[g] = INT64_MAX;
  const int slot = (int)(c->bepoch & 1);
  for (int g = 0; g < c->G; ++g) {
    p->gsrc[g] = c->peer_base[g] + c->peer_grad_off[g] + (size_t)slot * c->peer_gslot_bytes[g];
    p->peer_ready[g] = (g == c->rank) ? nullptr : reinterpret_cast<uint32_t*>(c->peer_base[g] + 64) + c->rank;
    p->peer_done[g] = (g == c->rank) ? nullptr : reinterpret_cast<uint32_t*>(c->peer_base[g] + 128) + c->rank;
  }
  p->my_ready = reinterpret_cast<const uint32_t*>(c->sym + 64);
  p->ctrl = c->ctrl;
  p->timeout_ns = c->timeout_ns;
  p->T = c->T;
  p->T_r = c->T_r;
  p->d = c->d;
  p->G = c->G;
  p->rank = c->rank;
  p->lanes = c->blanes;
  p->chunk_rows = c->bwd_chunk_rows > 0 ? c->bwd_chunk_rows : (c->chunk_rows ? c->chunk_rows : 256);
  // chunk order: table groups of `bwd_group` tables, chunks interleaved inside a group
  // (1 = table-major, T_r = every table interleaved)
  p->interleave = c->bwd_interleave ? ((c->bwd_group > 0 && c->bwd_group < c->T_r) ? c->bwd_group : std::max(c->T_r, 1)) : 1;
  p->epoch = (uint32_t)c->bepoch;
}

emb_status_t emb_backward_grad_slot(emb_ctx_t* c, void* stream, void** dY) {
  if (!c || !dY) return EMB_ERR_ARG;
  if (!c->registered || !c->bwd_enabled) FAIL(c, EMB_ERR_STATE, "backward not enabled (set enable_backward before registering)");
  CK(c, cudaSetDevice(c->dev));
  const uint64_t next = c->bepoch + 1;
  // the slot of epoch `next` was last read by the peers at epoch next-2
  if (c->G > 1 && next > 2) {
    emb_bwd_slot_wait_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(reinterpret_cast<const uint32_t*>(c->sym + 128), c->G,
                                                                  c->rank, (uint32_t)(next - 2), c->timeout_ns,
                                                                  &c->ctrl->err);
    CK(c, cudaGetLastError());
  }
  *dY = c->sym + c->grad_off + (size_t)(next & 1) * c->gslot_bytes;
  return EMB_OK;
}

emb_status_t emb_backward_grad_ready(emb_ctx_t* c, void* stream) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered || !c->bwd_enabled) FAIL(c, EMB_ERR_STATE, "backward not enabled (set enable_backward before registering)");
  if (c->bwd_ready_pending) FAIL(c, EMB_ERR_STATE, "emb_backward_grad_ready called twice without emb_backward");
  CK(c, cudaSetDevice(c->dev));
  c->bepoch += 1;
  c->bwd_ready_pending = true;
  if (c->G > 1) {
    BwdParams p;
    fill_bwd_params(c, &p);
    emb_bwd_signal_kernel<<<1, 32, 0, (cudaStream_t)stream>>>(p);
    CK(c, cudaGetLastError());
  }
  return EMB_OK;
}

// f2, bwd_algo 1 (emb_bwd_sort.cuh): workspace of the radix sort, allocated before the
// step is committed (a failure here must still release the peers, see emb_backward)
static emb_status_t sorted_workspace(emb_ctx_t* c, const int64_t* offsets, cudaStream_t s) {
  if (!c->d_rowbase) {                                  // workspace sized by the local rows
    std::vector<int64_t> rb(c->T_r + 1, 0);
    for (int i = 0; i < c->T_r; ++i) rb[i + 1] = rb[i] + c->rows[c->local[i]];
    if (rb[c->T_r] >= (1ll << 27)) FAIL(c, EMB_ERR_ARG, "bwd_algo 1: more than 2^27 local rows (3 radix passes)");
    for (int g = 0; g < c->G; ++g)
      if ((c->bstart[g + 1] - c->bstart[g]) * (int64_t)c->T >= (1ll << 28))
        FAIL(c, EMB_ERR_ARG, "bwd_algo 1: B_r * T must be < 2^28 (rank %d)", g);
    c->bs_R = rb[c->T_r];
    CK(c, cudaMalloc(&c->d_rowbase, rb.size() * sizeof(int64_t)));
    CK(c, cudaMemcpy(c->d_rowbase, rb.data(), rb.size() * sizeof(int64_t), cudaMemcpyHostToDevice));
  }
  if (!c->d_pairs) {                                    // entry lists: sized from the first CSR
    if (c->bs_cap <= 0) {                               // (one host sync, first call only)
      int64_t nnz = 0;
      CK(c, cudaMemcpyAsync(&nnz, offsets + (int64_t)c->T_r * c->B, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
      CK(c, cudaStreamSynchronize(s));
      c->bs_cap = std::min<int64_t>(nnz + nnz / 4 + 4096, 0xffffffffll);
    }
    c->rs_nblk = (c->bs_cap + kRTile - 1) / kRTile;
    const int64_t nh = (int64_t)kRBins * c->rs_nblk;
    c->bs_stride = (c->bs_cap + kSortTask + 31) / 32 * 32;   // a reduce task's staging never reads past
    CK(c, cudaMalloc(&c->d_pairs, (size_t)c->bs_stride * 2 * sizeof(uint32_t)));
    CK(c, cudaMalloc(&c->d_pairs_b, (size_t)c->bs_stride * 2 * sizeof(uint32_t)));
    CK(c, cudaMalloc(&c->d_ghist, (size_t)nh * sizeof(uint32_t)));
    CK(c, cudaMalloc(&c->d_rbsum, (size_t)((nh + kScanTile - 1) / kScanTile) * sizeof(uint32_t)));
  }
  const size_t dsm = (size_t)(2 * kRTile + (2 + kBlock / 32) * kRBins) * sizeof(uint32_t);
  CK(c, cudaFuncSetAttribute(emb_bradix_down_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm));
  return EMB_OK;
}

// f2, bwd_algo 1: LSD radix sort of the lookups by dW row, then a segmented gather-sum
// with one red.add per run of equal rows (workspace prepared by sorted_workspace)
static emb_status_t backward_sorted(emb_ctx_t* c, const BwdParams& bp, const int64_t* offsets, const int64_t* indices,
                                    cudaStream_t s) {
  SortParams q;
  memset(&q, 0, sizeof(q));
  q.offsets = offsets;
  q.indices = indices;
  q.rowbase = c->d_rowbase;
  q.tables = c->d_tables;
  q.ecode = c->d_pairs;
  q.erow = c->d_pairs + c->bs_stride;
  q.dW = bp.dW;
  for (int g = 0; g < kMaxG; ++g) {
    q.gsrc[g] = bp.gsrc[g];
    q.peer_done[g] = bp.peer_done[g];
  }
  for (int g = 0; g <= kMaxG; ++g) q.bstart[g] = bp.bstart[g];
  q.my_ready = bp.my_ready;
  q.ctrl = c->ctrl;
  q.R = c->bs_R;
  q.cap = c->bs_cap;
  q.B = c->B;
  q.timeout_ns = c->timeout_ns;
  q.T = c->T;
  q.T_r = c->T_r;
  q.d = c->d;
  q.G = c->G;
  q.rank = c->rank;
  q.lanes = c->blanes;
  q.chunk_rows = bp.chunk_rows;
  q.epoch = bp.epoch;
  const int grid = c->num_sms * 8;
  emb_bradix_gen_kernel<<<grid, kBlock, 0, s>>>(q);
  int bits = 1;
  while (bits < 32 && (1ll << bits) < c->bs_R) ++bits;
  const int passes = (bits + kRBits - 1) / kRBits;
  const int64_t nh = (int64_t)kRBins * c->rs_nblk, nb2 = (nh + kScanTile - 1) / kScanTile;
  const size_t dsm = (size_t)(2 * kRTile + (2 + kBlock / 32) * kRBins) * sizeof(uint32_t);
  uint32_t* in = c->d_pairs;
  uint32_t* out = c->d_pairs_b;
  q.ghist = c->d_ghist;
  q.nblk_r = c->rs_nblk;
  SortParams qs = q;                                    // the scan runs over the histograms
  qs.cnt = c->d_ghist;
  qs.R = nh;
  qs.bsum = c->d_rbsum;
  for (int ps = 0; ps < passes; ++ps) {
    q.rin_c = in;
    q.rin_g = in + c->bs_stride;
    q.rout_c = out;
    q.rout_g = out + c->bs_stride;
    q.shift = kRBits * ps;
    emb_bradix_up_kernel<<<(unsigned)c->rs_nblk, kBlock, 0, s>>>(q);
    emb_bsort_scan_sum_kernel<<<(unsigned)nb2, kBlock, 0, s>>>(qs);
    emb_bsort_scan_top_kernel<<<1, kBlock, 0, s>>>(c->d_rbsum, nb2);
    emb_bsort_scan_apply_kernel<<<(unsigned)nb2, kBlock, 0, s>>>(qs);
    emb_bradix_down_kernel<<<(unsigned)c->rs_nblk, kBlock, dsm, s>>>(q);
    std::swap(in, out);
  }
  q.ecode = in;                                         // sorted by row
  q.erow = in + c->bs_stride;
  void (*k)(SortParams) = nullptr;
  const bool multi = c->G > 1;
  if (c->bvb == 8) k = multi ? emb_bsort_reduce_kernel<8, 1, 2, 1, true> : emb_bsort_reduce_kernel<8, 1, 2, 1, false>;
  else if (c->bnv == 2) k = multi ? emb_bsort_reduce_kernel<16, 2, 2, 1, true> : emb_bsort_reduce_kernel<16, 2, 2, 1, false>;
  else if (c->bnv == 4) k = multi ? emb_bsort_reduce_kernel<16, 4, 2, 1, true> : emb_bsort_reduce_kernel<16, 4, 2, 1, false>;
  else k = multi ? emb_bsort_reduce_kernel<16, 1, 2, 4, true> : emb_bsort_reduce_kernel<16, 1, 2, 4, false>;
  // row bases + per-warp double buffer of one task's codes and rows
  const size_t rsm = ((size_t)(c->T_r + 1) * 8 + 15) / 16 * 16 + (size_t)(kBlock / 32) * 2 * (2 * kSortTask + 16) * 4;
  CK(c, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)rsm));
  int per_sm = 0;
  CK(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kBlock, rsm));
  k<<<c->num_sms * std::max(per_sm, 1), kBlock, rsm, s>>>(q);
  CK(c, cudaGetLastError());
  return EMB_OK;
}

// the kernel launches of emb_backward's chosen path (gpu_launches accounting)
static int backward_launches(const emb_ctx_t* c) {
  if (c->bwd_algo != 1 || c->T_r == 0) return 1;
  int64_t R = 0;
  for (int i = 0; i < c->T_r; ++i) R += c->rows[c->local[i]];
  int bits = 1;
  while (bits < 32 && (1ll << bits) < R) ++bits;
  return 2 + 5 * ((bits + kRBits - 1) / kRBits);      // gen + passes x (up, 3 scan, down) + reduce
}

emb_status_t emb_backward(emb_ctx_t* c, const int64_t* offsets, const int64_t* indices, void* const* dW,
                          uint32_t flags, void* stream) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered || !c->bwd_enabled) FAIL(c, EMB_ERR_STATE, "backward not enabled (set enable_backward before registering)");
  if (!c->bwd_ready_pending) FAIL(c, EMB_ERR_STATE, "emb_backward without emb_backward_grad_ready");
  if (flags != 0) FAIL(c, EMB_ERR_ARG, "emb_backward takes no flags (got 0x%x)", flags);
  CK(c, cudaSetDevice(c->dev));
  cudaStream_t s = (cudaStream_t)stream;
  BwdParams p;
  fill_bwd_params(c, &p);
  // Everything that can fail is checked and allocated BEFORE the step is committed; if it
  // fails, the step still releases the "done" flags so the peers' next grad_slot does not
  // time out, and the pending state is cleared so the next step can proceed.
  auto abandon = [&](emb_status_t st) -> emb_status_t {
    const std::string msg = c->err;
    c->bwd_ready_pending = false;
    if (c->G > 1) {
      BwdParams r = p;
      for (int g = 0; g < kMaxG; ++g) r.peer_ready[g] = p.peer_done[g];   // release "done reading"
      emb_bwd_signal_kernel<<<1, 32, 0, s>>>(r);
      cudaGetLastError();
    }
    c->err = msg;
    return st;
  };
  if (c->T_r > 0 && (!offsets || !indices || !dW)) {
    c->err = "NULL buffer";
    return abandon(EMB_ERR_ARG);
  }
  if (!c->d_dW) {
    cudaError_t e = cudaMalloc(&c->d_dW, std::max(c->T_r, 1) * sizeof(float*));
    if (e != cudaSuccess) { c->err = cudaGetErrorString(e); return abandon(EMB_ERR_CUDA); }
  }
  bool same = (int)c->h_dW.size() == c->T_r;
  for (int i = 0; same && i < c->T_r; ++i) same = c->h_dW[i] == dW[i];
  if (!same) {
    for (int i = 0; i < c->T_r; ++i)
      if (!dW[i] || ((uintptr_t)dW[i]) % 16) {
        c->err = "dW[" + std::to_string(i) + "] NULL or not 16-byte aligned";
        return abandon(EMB_ERR_ARG);
      }
    c->h_dW.assign(dW, dW + c->T_r);
    cudaError_t e = cudaStreamSynchronize(s);
    if (e == cudaSuccess) e = cudaMemcpy(c->d_dW, c->h_dW.data(), c->T_r * sizeof(float*), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) { c->err = cudaGetErrorString(e); return abandon(EMB_ERR_CUDA); }
  }
  p.dW = c->d_dW;
  const bool sorted = c->bwd_algo == 1 && c->T_r > 0;
  if (sorted && c->has_shard) {
    c->err = "bwd_algo 1 does not support row-sharded tables (use bwd_algo 0)";
    return abandon(EMB_ERR_ARG);
  }
  if (sorted) {
    emb_status_t st = sorted_workspace(c, offsets, s);
    if (st != EMB_OK) return abandon(st);
  }
  c->bwd_ready_pending = false;
  if (sorted) return backward_sorted(c, p, offsets, indices, s);
  p.offsets = offsets;
  p.indices = indices;
  void (*k)(BwdParams) = nullptr;
  size_t smem = 0;
  if (c->bwd_cache && c->bnv == 1) {                     // cache variants: 256-B and 512-B rows
    k = c->bvb == 16 ? emb_bwd_kernel<16, 1, 16> : emb_bwd_kernel<8, 1, 16>;
    smem = (size_t)(kBlock / 32) * 16 * (32 * c->bvb + 4);
    CK(c, cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  } else if (c->bvb == 8) k = emb_bwd_kernel<8, 1>;
  else if (c->bnv == 2) k = emb_bwd_kernel<16, 2>;
  else if (c->bnv == 4) k = emb_bwd_kernel<16, 4>;
  else k = emb_bwd_kernel<16, 1>;
  int per_sm = 0;
  CK(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kBlock, smem));
  k<<<c->num_sms * std::max(per_sm, 1), kBlock, smem, s>>>(p);
  CK(c, cudaGetLastError());
  return EMB_OK;
}

emb_status_t emb_trace_read(emb_ctx_t* c, uint64_t* host, int64_t capacity, int64_t* count) {
  if (!c || !count || (capacity > 0 && !host)) return EMB_ERR_ARG;
  CK(c, cudaSetDevice(c->dev));
  CK(c, cudaDeviceSynchronize());
  unsigned n = 0;
  CK(c, cudaMemcpy(&n, &c->ctrl->trace_n, sizeof(unsigned), cudaMemcpyDeviceToHost));
  const int64_t have = std::min<int64_t>((int64_t)n, (int64_t)c->trace_cap);
  const int64_t m = std::min<int64_t>(have, capacity);
  if (m > 0) CK(c, cudaMemcpy(host, c->trace, (size_t)m * 2 * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  *count = m;
  CK(c, cudaMemset(&c->ctrl->trace_n, 0, sizeof(unsigned)));
  return EMB_OK;
}

emb_status_t emb_finalize(emb_ctx_t* c) {
  if (!c) return EMB_ERR_ARG;
  cudaSetDevice(c->dev);
  cudaDeviceSynchronize();
  emb_status_t st = EMB_OK;
  if (c->registered && c->G > 1) {  // nobody may still write into our buffer
    int one = 1;
    std::vector<int> r(c->G);
    if (c->ag(c->user, &one, r.data(), sizeof(int)) != 0) st = EMB_ERR_PEER;
  }
  for (int p = 0; p < (int)c->peer_base.size(); ++p)
    if (c->peer_ipc[p]) cudaIpcCloseMemHandle(c->peer_base[p]);
  if (c->sym) cudaFree(c->sym);
  if (c->d_tables) cudaFree(c->d_tables);
  if (c->ctrl) cudaFree(c->ctrl);
  if (c->d_unpack_base) cudaFree(c->d_unpack_base);
  if (c->d_comb_tglob) cudaFree(c->d_comb_tglob);
  if (c->d_tmaps) cudaFree(c->d_tmaps);
  if (c->d_comb_nsh) cudaFree(c->d_comb_nsh);
  if (c->d_pbase) cudaFree(c->d_pbase);
  if (c->d_pstride) cudaFree(c->d_pstride);
  if (c->d_psoff) cudaFree(c->d_psoff);
  if (c->d_unpack_stride) cudaFree(c->d_unpack_stride);
  if (c->d_off_stage) cudaFree(c->d_off_stage);
  if (c->d_idx_stage) cudaFree(c->d_idx_stage);
  for (int i = 0; i < 2; ++i) {
    if (c->p_off[i]) cudaFree(c->p_off[i]);
    if (c->p_idx[i]) cudaFree(c->p_idx[i]);
    if (c->ev_in[i]) cudaEventDestroy(c->ev_in[i]);
    if (c->ev_kern[i]) cudaEventDestroy(c->ev_kern[i]);
  }
  for (int i = 0; i < kOutSlots; ++i)
    if (c->ev_out[i]) cudaEventDestroy(c->ev_out[i]);
  if (c->s_in) cudaStreamDestroy(c->s_in);
  if (c->trace) cudaFree(c->trace);
  if (c->d_dW) cudaFree(c->d_dW);
  if (c->d_rowbase) cudaFree(c->d_rowbase);
  if (c->d_pairs) cudaFree(c->d_pairs);
  if (c->d_pairs_b) cudaFree(c->d_pairs_b);
  if (c->d_ghist) cudaFree(c->d_ghist);
  if (c->d_rbsum) cudaFree(c->d_rbsum);
  if (c->s_out) cudaStreamDestroy(c->s_out);
  delete c;
  return st;
}

emb_status_t emb_local_batch(const emb_ctx_t* c, int rank, int64_t* start, int64_t* count) {
  if (!c || !start || !count) return EMB_ERR_ARG;
  if (!c->registered) return EMB_ERR_STATE;
  if (rank < 0 || rank >= c->G) return EMB_ERR_ARG;
  *start = c->bstart[rank];
  *count = c->bstart[rank + 1] - c->bstart[rank];
  return EMB_OK;
}

emb_status_t emb_get_info(const emb_ctx_t* c, emb_info_t* i) {
  if (!c || !i) return EMB_ERR_ARG;
  memset(i, 0, sizeof(*i));
  i->rank = c->rank;
  i->world_size = c->G;
  i->device = c->dev;
  i->num_sms = c->num_sms;
  i->num_tables = c->T;
  i->num_local_tables = c->T_r;
  i->dim = c->d;
  i->weight_dtype = c->wdt;
  i->out_dtype = c->odt;
  i->global_batch = c->B;
  if (c->registered) {
    i->local_batch_start = c->bstart[c->rank];
    i->local_batch = c->bstart[c->rank + 1] - c->bstart[c->rank];
    i->out_slot_bytes = i->local_batch * c->T * c->d * (int64_t)esize(c->odt);
  }
  i->epoch = c->epoch;
  int per_sm = c->ctas_per_sm;
  if (per_sm <= 0 && c->registered) {
    KernelFn k = pick_kernel(c, fwd_mode(false, c->has_shard, c->tma_store != 0));
    const size_t smem = fwd_smem(c, fwd_mode(false, c->has_shard, c->tma_store != 0));
    if (smem > 0) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, kBlock, smem);
  }
  i->grid = c->num_sms * std::max(per_sm, 1);
  i->block = kBlock;
  i->lanes = c->lanes;
  i->vec_bytes = c->vb;
  i->vecs_per_lane = c->nv;
  i->out_slots = kOutSlots;
  // kernels one call launches: the fused forward (+ the f3 combine); emb_backward's path
  i->fwd_launches = 1 + (c->has_shard ? 1 : 0);
  i->bwd_launches = c->registered && c->bwd_enabled ? backward_launches(c) : 0;
  return EMB_OK;
}

emb_status_t emb_set_option(emb_ctx_t* c, const char* key, int64_t v) {
  if (!c || !key) return EMB_ERR_ARG;
  if (!strcmp(key, "chunk_rows")) { if (v < 0) FAIL(c, EMB_ERR_ARG, "chunk_rows < 0"); c->chunk_rows = (int)v; }
  else if (!strcmp(key, "ctas_per_sm")) { if (v < 0 || v > 32) FAIL(c, EMB_ERR_ARG, "ctas_per_sm"); c->ctas_per_sm = (int)v; }
  else if (!strcmp(key, "stagger")) c->stagger = v ? 1 : 0;
  else if (!strcmp(key, "timeout_ms")) { if (v < 1) FAIL(c, EMB_ERR_ARG, "timeout_ms < 1"); c->timeout_ns = v * 1000000ll; }
  else if (!strcmp(key, "bwd_interleave")) c->bwd_interleave = v ? 1 : 0;
  else if (!strcmp(key, "bwd_algo")) { if (v < 0 || v > 1) FAIL(c, EMB_ERR_ARG, "bwd_algo must be 0 or 1"); c->bwd_algo = (int)v; }
  else if (!strcmp(key, "bwd_max_nnz")) {
    if (v < 0 || v >= (1ll << 32)) FAIL(c, EMB_ERR_ARG, "bwd_max_nnz not in [0, 2^32)");
    if (c->d_pairs) { cudaFree(c->d_pairs); c->d_pairs = nullptr; }
    if (c->d_pairs_b) { cudaFree(c->d_pairs_b); c->d_pairs_b = nullptr; }
    if (c->d_ghist) { cudaFree(c->d_ghist); c->d_ghist = nullptr; }
    if (c->d_rbsum) { cudaFree(c->d_rbsum); c->d_rbsum = nullptr; }
    c->bs_cap = v;
  }
  else if (!strcmp(key, "bwd_cache")) {
    if (v != 0 && v != 16) FAIL(c, EMB_ERR_ARG, "bwd_cache must be 0 or 16");
    c->bwd_cache = (int)v;
  }
  else if (!strcmp(key, "bwd_chunk_rows")) { if (v < 0 || v > 65536) FAIL(c, EMB_ERR_ARG, "bwd_chunk_rows not in [0, 65536]"); c->bwd_chunk_rows = (int)v; }
  else if (!strcmp(key, "bwd_group")) { if (v < 0 || v > 4096) FAIL(c, EMB_ERR_ARG, "bwd_group not in [0, 4096]"); c->bwd_group = (int)v; }
  else if (!strcmp(key, "fwd_interleave")) c->fwd_interleave = v ? 1 : 0;
  else if (!strcmp(key, "tail_div")) { if (v < 1 || v > 64) FAIL(c, EMB_ERR_ARG, "tail_div not in [1, 64]"); c->tail_div = (int)v; }
  else if (!strcmp(key, "tma_store")) c->tma_store = v ? 1 : 0;
  else if (!strcmp(key, "debug_d2h_delay_us")) {
    if (v < 0 || v > 10000000) FAIL(c, EMB_ERR_ARG, "debug_d2h_delay_us not in [0, 1e7]");
    c->d2h_delay_us = v;
  }
  else if (!strcmp(key, "carveout")) {
    if (v < -1 || v > 100) FAIL(c, EMB_ERR_ARG, "carveout in [-1 (driver default), 100] percent");
    c->carveout = (int)v;
  }
  else if (!strcmp(key, "enable_backward")) {
    if (c->registered) FAIL(c, EMB_ERR_STATE, "enable_backward must be set before emb_register_tables");
    c->bwd_enabled = v != 0;
  }
  else if (!strcmp(key, "trace_capacity")) {
    if (v < 0 || v > (1 << 26)) FAIL(c, EMB_ERR_ARG, "trace_capacity in [0, 2^26]");
    CK(c, cudaSetDevice(c->dev));
    CK(c, cudaDeviceSynchronize());
    if (c->trace) CK(c, cudaFree(c->trace));
    c->trace = nullptr;
    c->trace_cap = 0;
    if (v > 0) {
      CK(c, cudaMalloc(&c->trace, (size_t)v * 2 * sizeof(unsigned long long)));
      c->trace_cap = (uint32_t)v;
    }
    CK(c, cudaMemset(&c->ctrl->trace_n, 0, sizeof(unsigned)));
  }
  else FAIL(c, EMB_ERR_ARG, "unknown option '%s'", key);
  return EMB_OK;
}

emb_status_t emb_query_device_error(emb_ctx_t* c, uint32_t* word, int clear) {
  if (!c || !word) return EMB_ERR_ARG;
  CK(c, cudaSetDevice(c->dev));
  CK(c, cudaMemcpy(word, &c->ctrl->err, sizeof(uint32_t), cudaMemcpyDeviceToHost));
  if (clear) CK(c, cudaMemset(&c->ctrl->err, 0, sizeof(uint32_t)));
  return EMB_OK;
}

const char* emb_last_error(const emb_ctx_t* c) { return c ? c->err.c_str() : g_init_error.c_str(); }

emb_status_t emb_baseline_splits(const emb_ctx_t* c, int64_t* send_counts, int64_t* recv_counts) {
  if (!c || !send_counts || !recv_counts) return EMB_ERR_ARG;
  if (!c->registered) return EMB_ERR_STATE;
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  if (c->has_shard) {                   // fp32 partials of every local shard (incl. whole tables)
    for (int g = 0; g < c->G; ++g) {
      send_counts[g] = (c->bstart[g + 1] - c->bstart[g]) * c->T_r * c->d;
      recv_counts[g] = Br * (int64_t)c->nloc[g] * c->d;
    }
    return EMB_OK;
  }
  for (int g = 0; g < c->G; ++g) {
    send_counts[g] = (c->bstart[g + 1] - c->bstart[g]) * c->T_r * c->d;
    recv_counts[g] = Br * (int64_t)c->tables_of[g].size() * c->d;
  }
  return EMB_OK;
}

static emb_status_t baseline_pool_impl(emb_ctx_t* c, const void* offsets, const void* indices, bool i32, uint32_t flags,
                                       cudaStream_t s, void* send) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered) FAIL(c, EMB_ERR_STATE, "emb_baseline_pool before emb_register_tables");
  if (c->T_r > 0 && (!offsets || !indices || !send)) FAIL(c, EMB_ERR_ARG, "NULL buffer");
  CK(c, cudaSetDevice(c->dev));
  FwdParams p;
  fill_params(c, offsets, indices, i32, false, (char*)send, &p);
  p.check = (flags & EMB_FWD_CHECK_BOUNDS) ? 1 : 0;
  if (c->has_shard) {                   // f3: every local shard's fp32 partial, destination-major
    p.all_partial = 1;
    p.part_stride = c->T_r;
    for (int g = 0; g < c->G; ++g)
      p.part_base[g] = (char*)send + (size_t)c->bstart[g] * (size_t)c->T_r * (size_t)c->d * 4;
  }
  return launch_fwd(c, p, flags & EMB_FWD_CHECK_BOUNDS, s);
}

emb_status_t emb_baseline_pool(emb_ctx_t* c, const int64_t* offsets, const int64_t* indices, uint32_t flags,
                               void* stream, void* send) {
  return baseline_pool_impl(c, offsets, indices, false, flags, (cudaStream_t)stream, send);
}

emb_status_t emb_baseline_pool_i32(emb_ctx_t* c, const int32_t* offsets, const int32_t* indices, uint32_t flags,
                                   void* stream, void* send) {
  return baseline_pool_impl(c, offsets, indices, true, flags, (cudaStream_t)stream, send);
}

emb_status_t emb_baseline_unpack(emb_ctx_t* c, const void* recv, void* stream, void* out) {
  if (!c) return EMB_ERR_ARG;
  if (!c->registered) FAIL(c, EMB_ERR_STATE, "emb_baseline_unpack before emb_register_tables");
  if (!recv || !out) FAIL(c, EMB_ERR_ARG, "NULL buffer");
  CK(c, cudaSetDevice(c->dev));
  const int64_t Br = c->bstart[c->rank + 1] - c->bstart[c->rank];
  const int rowbytes = c->d * (int)esize(c->odt);
  const int64_t rows = Br * c->T;
  int grid = (int)std::min<int64_t>((rows + (kBlock / 32) - 1) / (kBlock / 32), (int64_t)c->num_sms * 8);
  if (grid < 1) grid = 1;
  if (c->has_shard) {                   // f3: sum the shards' partials in shard order, then pack
    if (c->odt == EMB_F32)
      emb_unpack_partials_kernel<float><<<grid, kBlock, 0, (cudaStream_t)stream>>>(
          (const float*)recv, (char*)out, c->d_pbase, c->d_pstride, c->d_psoff, Br, c->T, c->d);
    else
      emb_unpack_partials_kernel<__nv_bfloat16><<<grid, kBlock, 0, (cudaStream_t)stream>>>(
          (const float*)recv, (char*)out, c->d_pbase, c->d_pstride, c->d_psoff, Br, c->T, c->d);
    CK(c, cudaGetLastError());
    return EMB_OK;
  }
  if (rowbytes % 16 == 0)
    emb_unpack_rows_kernel<uint4><<<grid, kBlock, 0, (cudaStream_t)stream>>>((const char*)recv, (char*)out,
                                                                           c->d_unpack_base, c->d_unpack_stride, Br,
                                                                           c->T, rowbytes);
  else
    emb_unpack_rows_kernel<uint2><<<grid, kBlock, 0, (cudaStream_t)stream>>>((const char*)recv, (char*)out,
                                                                           c->d_unpack_base, c->d_unpack_stride, Br,
                                                                           c->T, rowbytes);
  CK(c, cudaGetLastError());
  return EMB_OK;
}

}  // extern "C"
