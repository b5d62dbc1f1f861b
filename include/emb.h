/*
 * emb.h -- C ABI of libemb: the B200-native PGAS-style EMB-layer forward.
 *
 * What it computes (PAPER.md, /root/reference/PAPER.md):
 *   - lookup + sum pooling of embedding rows per (table, sample) bag
 *     (L91-95, §II-B, Fig. 3);
 *   - table-wise model parallelism with the batch-sharded data-parallel output
 *     layout (L99-113, §II-C, Fig. 4): rank r ends with Y_r[B_r][T][d], the pooled
 *     vectors of ALL T tables for its contiguous mini-batch;
 *   - the paper's PGAS fused retrieval (L129-147, §III-B/C, Listing 2):
 *     each pooled vector is stored by the kernel straight into its final slot of
 *     the owning rank's output (one-sided peer stores over NVLink), replacing the
 *     NCCL all-to-all + unpack of the baseline (L155, L193, §IV);
 *   - the conventional comparison path's two kernels (pool into a send buffer,
 *     unpack the received buffer); the all-to-all between them is NCCL, called by
 *     the caller (PyTorch) -- L155/L193.
 *
 * The paper's user-facing call is forward(weights, offsets, indices, outputs)
 * (Listing 1; Listing 2).  This ABI keeps those four
 * roles per rank process and stream-ordered; output storage is library-owned
 * (symmetric across ranks, PGAS style, L216/L228/L232).
 *
 * Conventions
 *   - One context per rank process (or per simulated rank, see emb_init).  All
 *     calls on a context come from one host thread.  No C++ exception crosses the
 *     ABI; every call returns an emb_status_t and, on failure, a message is kept
 *     for emb_last_error().
 *   - "stream" arguments are cudaStream_t handles passed as void* (NULL = legacy
 *     default stream).  All device work is stream-ordered and asynchronous.
 *   - Device pointers are plain CUDA device addresses of the context's device.
 *   - Collective calls (emb_register_tables, emb_forward, emb_finalize) must be
 *     entered by every rank, in the same order.
 *   - One forward-type launch (emb_forward / emb_baseline_pool) in flight per context at a
 *     time: they share the context's device work counters (stream order provides this when
 *     they are issued on one stream).
 *   - Readings of points the paper leaves open are listed in DESIGN.md (C1..C29).
 */
#ifndef EMB_H_
#define EMB_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct emb_ctx emb_ctx_t;

typedef enum {
  EMB_OK = 0,
  EMB_ERR_ARG = 1,      /* invalid argument (message in emb_last_error)            */
  EMB_ERR_STATE = 2,    /* call out of order (e.g. forward before register)        */
  EMB_ERR_CUDA = 3,     /* a CUDA runtime call failed                              */
  EMB_ERR_NOMEM = 4,    /* device or host allocation failed                        */
  EMB_ERR_PEER = 5,     /* peer exchange / IPC mapping failed                      */
  EMB_ERR_TIMEOUT = 6,  /* a device-side peer wait timed out (see device error)    */
  EMB_ERR_BOUNDS = 7    /* an out-of-range index was seen under CHECK_BOUNDS       */
} emb_status_t;

typedef enum { EMB_F32 = 0, EMB_BF16 = 1 } emb_dtype_t;

/* emb_forward / emb_baseline_pool flags */
#define EMB_FWD_CHECK_BOUNDS 0x1u  /* skip indices outside [0, M_t) and set EMB_DEVERR_BOUNDS */
#define EMB_FWD_SEPARATE_WAIT 0x2u /* fused kernel only signals; call emb_wait() to complete  */

/* sticky device error word bits (emb_query_device_error) */
#define EMB_DEVERR_TIMEOUT 0x1u
#define EMB_DEVERR_BOUNDS 0x2u
#define EMB_DEVERR_CAPACITY 0x4u /* emb_backward (bwd_algo 1): more lookups than the entry workspace; step skipped */

/* Index width (SURVEY reading C12).  The paper's listing passes int64 offsets and indices
 * (Listing 2), the default of every call below.  The *_i32 entry points take the
 * same CSR as int32 arrays (offsets[T_r*B] < 2^31): half the index bytes in HBM and over
 * PCIe, identical results. */

/* All-gather over the caller's process group.  send: `bytes` bytes of this rank;
 * recv: world_size*bytes, rank order.  Return 0 on success.  Called only from
 * emb_register_tables and emb_finalize (once each, plus a barrier-style call). */
typedef int (*emb_allgather_fn)(void* user, const void* send, void* recv, size_t bytes);

typedef struct {
  int32_t rank, world_size, device, num_sms;
  int32_t num_tables;         /* T (global)                                   */
  int32_t num_local_tables;   /* T_r                                          */
  int32_t dim;                /* d                                            */
  int32_t weight_dtype, out_dtype;
  int64_t global_batch;       /* B                                            */
  int64_t local_batch_start;  /* s_r                                          */
  int64_t local_batch;        /* B_r                                          */
  uint64_t epoch;             /* number of emb_forward calls so far           */
  int32_t grid, block;        /* fused kernel launch shape                    */
  int32_t lanes, vec_bytes, vecs_per_lane; /* row-gather tiling                */
  int64_t out_slot_bytes;     /* B_r*T*d*e_o                                  */
  int32_t out_slots;          /* depth of the symmetric output ring (3)       */
  int32_t fwd_launches;       /* kernels one emb_forward launches             */
  int32_t bwd_launches;       /* kernels one emb_backward launches            */
  int32_t reserved;
} emb_info_t;

/* Create a context for `rank` of `world_size` on CUDA device `cuda_device`.
 * `allgather` (+ opaque `user`) is the process-group all-gather used to exchange
 * the 64-byte CUDA IPC handles of the symmetric output buffers (may be NULL
 * only when world_size == 1).  Several contexts may live in one process
 * (single-process simulation of G ranks): peers in the same process are mapped
 * by raw pointer instead of IPC.  Errors: EMB_ERR_ARG, EMB_ERR_CUDA, EMB_ERR_NOMEM. */
emb_status_t emb_init(int rank, int world_size, int cuda_device, emb_allgather_fn allgather, void* user,
                      emb_ctx_t** out);

/* Collective.  Describe ALL T tables and register this rank's local ones.
 *   rows[T]    : rows M_t of every table (host), 1 <= M_t < 2^31
 *   owner[T]   : rank holding table t, in [0, world_size) (host)  -- table-wise MP (L99-101)
 *   dim        : embedding dim d; d*sizeof(weight) must be a multiple of 8 and either
 *                <= 512 bytes or a multiple of 512 bytes up to 4096
 *   weight_dtype / out_dtype : EMB_F32 or EMB_BF16 (accumulation is always fp32, C5;
 *                bf16 output is RNE-rounded once, C6)
 *   global_batch: B >= world_size; rank r's mini-batch is the contiguous block
 *                [s_r, s_r + B_r), first B mod G ranks one extra sample (C8);
 *                (T + 1) * B <= 2^31 - 1, T counting every row shard (the fused
 *                kernel's 32-bit work counter)
 *   local_weights[T_r] : device pointers of this rank's tables in ascending global id,
 *                row-major [M_t][d], 16-byte aligned; zero-copy: the caller keeps them
 *                alive until emb_finalize.
 * Allocates the symmetric output (a ring of 3 slots of [B_r][T][d]) + flag words, exchanges IPC
 * handles through `allgather`, maps every peer.  Errors: EMB_ERR_ARG, EMB_ERR_STATE
 * (already registered), EMB_ERR_CUDA/NOMEM, EMB_ERR_PEER. */
emb_status_t emb_register_tables(emb_ctx_t* ctx, int32_t num_tables, const int64_t* rows, const int32_t* owner,
                                 int32_t dim, emb_dtype_t weight_dtype, emb_dtype_t out_dtype, int64_t global_batch,
                                 const void* const* local_weights);

/* Collective.  f3 (§V "partitioning by rows ... merge the
 * sparse input partitioning into the computation kernel"): like emb_register_tables but
 * every table t is split into num_shards[t] contiguous row ranges.  shard_owner[] and
 * shard_row_start[] list the shards of table 0, then table 1, ... (sum(num_shards)
 * entries); shard s of t holds global rows [shard_row_start, next start or rows[t]) on
 * rank shard_owner (first start 0, strictly increasing).  A table with one shard is
 * table-wise.  local_weights[] lists this rank's shards in ascending (t, s), each pointing
 * at the shard's first row.  The CSR passed to emb_forward lists, for every local shard
 * in the same order, the FULL bag list of its table with GLOBAL row ids; the kernel skips
 * other shards' ids (in-kernel partitioning), stores each bag's fp32 partial sum into the
 * owner's partial slot (one-sided, like the pooled vectors), and after the exchange a
 * combine kernel sums the partials in shard order into Y_r (bf16 out: RNE once).
 * EMB_FWD_CHECK_BOUNDS checks ids against the whole table's [0, rows[t]).  Backward (f2,
 * bwd_algo 0): the same CSR; each shard owner accumulates into its shard's rows only (dW of a
 * local shard is [hi - lo][d], shard-local rows).  Comparison path: emb_baseline_pool writes
 * every local shard's fp32 partial (whole tables too) destination-major, the splits count fp32
 * elements, and emb_baseline_unpack sums each table's partials in shard order (then RNE for
 * bf16 out) -- the same result as the fused path, bit for bit.  Not supported with row-sharded
 * tables: bwd_algo 1.  Errors as emb_register_tables. */
emb_status_t emb_register_sharded_tables(emb_ctx_t* ctx, int32_t num_tables, const int64_t* rows,
                                         const int32_t* num_shards, const int32_t* shard_owner,
                                         const int64_t* shard_row_start, int32_t dim, emb_dtype_t weight_dtype,
                                         emb_dtype_t out_dtype, int64_t global_batch,
                                         const void* const* local_weights);

/* Collective, stream-ordered, asynchronous: the fused PGAS forward (Listing 2).
 *   offsets : device int64[T_r*B + 1], table-major CSR: bag (t_l, b) spans
 *             indices[offsets[t_l*B+b] .. offsets[t_l*B+b+1]) (C11; L212-215)
 *   indices : device int64 local row ids in [0, M_t) (C1, C12)
 *   *out    : receives the device pointer of Y_r = [B_r][T][d] (out dtype) for this
 *             epoch e; library-owned slot e % 3 of the symmetric ring.  Every read of it
 *             must be ordered before this rank's forward e+2 is launched (on `stream`,
 *             or on another stream that `stream` waits on before that launch): a peer
 *             can overwrite the slot with its forward e+3 as soon as this rank's forward
 *             e+2 has signalled.  Valid until then or emb_finalize.
 * Without EMB_FWD_SEPARATE_WAIT the kernel completes only when every peer's
 * pooled vectors for this rank have landed (in-kernel acquire wait), so any later
 * work on `stream` sees the whole Y_r.  With it, emb_wait completes the forward; a
 * forward issued while the previous one's emb_wait is still due enqueues that wait on its
 * own `stream` first (if the two forwards use different streams, the caller orders them).  Empty bags produce +0.0 (C2).  IEEE fp32 adds, no flush-to-zero; NaN and
 * Inf propagate (C7).  Unknown flag bits: EMB_ERR_ARG.
 * Errors: EMB_ERR_STATE (not registered), EMB_ERR_ARG, EMB_ERR_CUDA.  Device-side
 * failures (peer timeout, bounds) set the sticky device error word instead. */
emb_status_t emb_forward(emb_ctx_t* ctx, const int64_t* offsets, const int64_t* indices, uint32_t flags,
                         void* stream, void** out);
/* emb_forward with int32 offsets / indices (C12 option, see above). */
emb_status_t emb_forward_i32(emb_ctx_t* ctx, const int32_t* offsets, const int32_t* indices, uint32_t flags,
                             void* stream, void** out);

/* Complete a forward issued with EMB_FWD_SEPARATE_WAIT: enqueue the acquire wait on
 * every peer's flag for the latest epoch on `stream`. */
emb_status_t emb_wait(emb_ctx_t* ctx, void* stream);

/* End-to-end convenience: host CSR in, host Y_r out (e2e measurement).  Copies
 * h_offsets[T_r*B+1] and h_indices[h_offsets[T_r*B]] into library-owned device
 * staging (grown on demand), runs emb_forward, copies Y_r into h_out
 * (B_r*T*d*e_o bytes).  Host buffers should be pinned for asynchrony; the caller
 * synchronizes `stream` before reading h_out. */
emb_status_t emb_forward_host(emb_ctx_t* ctx, const int64_t* h_offsets, const int64_t* h_indices, uint32_t flags,
                              void* stream, void* h_out);

/* Pipelined end-to-end path (same inputs/outputs as emb_forward_host): call k's H2D
 * (internal copy-in stream, two alternating device stages) overlaps call k-1's kernel
 * (on `stream`) and call k-1's D2H (internal copy-out stream); the forward of call k
 * waits for the D2H of call k-2 (output-ring rule of emb_forward).  The peer wait is
 * always in-kernel here (EMB_FWD_SEPARATE_WAIT is ignored).  h_out of a call is
 * complete once emb_host_drain(ctx, s) has been called and `s` synchronized (or after a
 * later call's drain).  The host input buffers of a call must stay unchanged, and its
 * h_out must not be reused by another in-flight call, until then; h_out buffers should
 * be pinned.  Two calls in flight at most per stage (the library waits on events). */
emb_status_t emb_forward_host_async(emb_ctx_t* ctx, const int64_t* h_offsets, const int64_t* h_indices,
                                    uint32_t flags, void* stream, void* h_out);
/* Same with int32 host offsets / indices (C12 option). */
emb_status_t emb_forward_host_async_i32(emb_ctx_t* ctx, const int32_t* h_offsets, const int32_t* h_indices,
                                        uint32_t flags, void* stream, void* h_out);

/* Make `stream` wait for every outstanding copy of emb_forward_host_async. */
emb_status_t emb_host_drain(emb_ctx_t* ctx, void* stream);

/* Collective: waits for the device, unmaps peers, frees everything, destroys ctx. */
emb_status_t emb_finalize(emb_ctx_t* ctx);

/* Mini-batch [*start, *start + *count) of `rank` (C8). */
emb_status_t emb_local_batch(const emb_ctx_t* ctx, int rank, int64_t* start, int64_t* count);

emb_status_t emb_get_info(const emb_ctx_t* ctx, emb_info_t* info);

/* Tunables (take effect on the next launch): "chunk_rows" (target rows per claimed
 * work chunk; 0 = auto, the default: 192 for fp32 rows and 256 for bf16 rows in the
 * forward, 256 in the backward), "ctas_per_sm" (0 = occupancy max), "stagger" (1 =
 * destination-staggered chunk order, default), "timeout_ms" (peer wait, default
 * 10000 or env EMB_TIMEOUT_MS), "fwd_interleave" (1 = forward chunks interleaved across
 * tables instead of table-major), "tail_div" (the last table's chunks are this many times
 * smaller, default 4; 1 = off), "carveout" (shared-memory carve-out percent; 0 = auto, the
 * default: the smallest that fits the kernel's occupancy; -1 = driver default),
 * "tma_store" (f4, PAPER.md L386 aggregated stores: 1 = pooled vectors are staged per
 * warp in shared memory and shipped 4 at a time to 4 arbitrary output rows with one TMA
 * scatter4; needs full-warp rows with one vector per lane and d <= 256),
 * "enable_backward" (f2: 1 before emb_register_tables adds two fp32 grad slots
 * [B_r][T][d] to the symmetric buffer for emb_backward), f2 backward tunables:
 * "bwd_interleave" (1 = chunks interleaved across tables, default; 0 = table-major),
 * "bwd_group" (tables interleaved at a time, default 8; 0 = all local tables),
 * "bwd_cache" (per-warp shared-memory dW row cache: 16 slots (default) or 0; rows of one
 * vector per lane), "bwd_chunk_rows" (0 = chunk_rows),
 * "bwd_algo" (0 = atomic scatter per bag slice, default; 1 = LSD radix sort of the lookups
 * by dW row + segmented gather-sum, one red.add per run of equal rows: library-owned
 * workspace of 16 B per lookup, sized on the first call from the CSR (one host sync) or
 * preset by "bwd_max_nnz"; a later CSR with more lookups sets EMB_DEVERR_CAPACITY and
 * skips the step; needs fewer than 2^27 local rows),
 * "debug_d2h_delay_us" (test hook: the pipelined host path stalls its copy-out stream this
 * long before every D2H, to exercise the output-ring rule under a slow consumer),
 * "trace_capacity" (f1 instrumentation: > 0 allocates a device buffer
 * of that many records and makes every warp append {globaltimer ns, bytes stored to
 * peers << 32 | bytes stored locally} after each claimed chunk; 0 disables).
 * Errors: EMB_ERR_ARG for an unknown key or value. */
emb_status_t emb_set_option(emb_ctx_t* ctx, const char* key, int64_t value);

/* ---- f2: backward (§V) ---------------------------------------------
 * dW_t[x, :] += sum over bags (t, b) and positions j with x_t[j] = x of dY[b, t, :].
 * Usage per step (collective, every rank in the same order):
 *   emb_backward_grad_slot(ctx, stream, &dY)  -> device fp32 [B_r][T][d] slot of THIS
 *       rank's gradient w.r.t. its outputs; write it with work on `stream` (the call
 *       enqueues a wait until every peer finished reading the slot's previous use);
 *   emb_backward_grad_ready(ctx, stream) -> releases "my dY is written" to every peer
 *       (stream-ordered after the fill);
 *   emb_backward(ctx, offsets, indices, dW, flags = 0, stream) -> one fused kernel acquires
 *       every peer's "ready" flag and, per local bag, loads the
 *       bag's gradient vector from the DP rank's slot (one-sided NVLink load) and
 *       atomically adds it (red.add.f32, FTZ per the hardware atomic; a warp may first
 *       sum a hot row's contributions of one chunk in shared memory) into the rows of
 *       dW[t_l] (caller-owned device fp32 [M_t][d], NOT zeroed by the library; 16-byte
 *       aligned) for every index of the bag.  Same CSR as emb_forward.  Accumulation
 *       order is unspecified (atomics): results match the oracle within the fp32
 *       tolerance, exactly for integer-valued gradients.
 * Every CTA of the fused kernel waits for the peers' "ready" flags before it starts, so
 * when several ranks share ONE GPU (test harnesses) all ranks' grad_ready calls must be
 * issued before any rank's emb_backward.  The last CTA releases "done reading" into each
 * peer (emb_backward_grad_slot waits on it before a slot is refilled).
 * Requires "enable_backward" before emb_register_tables.  Errors: EMB_ERR_STATE (also for
 * emb_backward without a preceding grad_ready), EMB_ERR_ARG, EMB_ERR_CUDA; peer timeouts
 * set EMB_DEVERR_TIMEOUT.  If emb_backward fails after a grad_ready, it still releases
 * the peers ("done" flags) and clears the pending state, so the next step can proceed. */
emb_status_t emb_backward_grad_slot(emb_ctx_t* ctx, void* stream, void** dY);
emb_status_t emb_backward_grad_ready(emb_ctx_t* ctx, void* stream);
emb_status_t emb_backward(emb_ctx_t* ctx, const int64_t* offsets, const int64_t* indices, void* const* dW,
                          uint32_t flags, void* stream);

/* f1: synchronize the device, copy up to `capacity` trace records (2 x uint64 each,
 * see "trace_capacity") into `host`, set *count, and reset the trace. */
emb_status_t emb_trace_read(emb_ctx_t* ctx, uint64_t* host, int64_t capacity, int64_t* count);

/* Read (after synchronizing the forward's stream) and optionally clear the sticky
 * device error word (EMB_DEVERR_* bits). */
emb_status_t emb_query_device_error(emb_ctx_t* ctx, uint32_t* word, int clear);

/* Last error message of this context (or of the last failed emb_init when ctx is NULL). */
const char* emb_last_error(const emb_ctx_t* ctx);

/* ---- comparison path (L155, L193) -------------------------------
 * Split sizes (in ELEMENTS of out dtype; fp32 elements with row-sharded tables) for
 * torch.distributed.all_to_all_single: send_counts[dst] = B_dst*T_r*d,
 * recv_counts[src] = B_r*T_src*d (T_r, T_src: local tables or, sharded, local shards). */
emb_status_t emb_baseline_splits(const emb_ctx_t* ctx, int64_t* send_counts, int64_t* recv_counts);

/* Same gather+pool core as emb_forward, written destination-major into the
 * caller-owned device buffer send = [G][B_dst][T_r][d] (out dtype). */
emb_status_t emb_baseline_pool(emb_ctx_t* ctx, const int64_t* offsets, const int64_t* indices, uint32_t flags,
                               void* stream, void* send);
emb_status_t emb_baseline_pool_i32(emb_ctx_t* ctx, const int32_t* offsets, const int32_t* indices, uint32_t flags,
                                   void* stream, void* send);

/* Unpack/rearrange after the all-to-all: recv = [G][B_r][T_src][d] (blocks in
 * source-rank order, tables of each source in ascending global id) into
 * out = [B_r][T][d] (caller-owned device buffers, out dtype). */
emb_status_t emb_baseline_unpack(emb_ctx_t* ctx, const void* recv, void* stream, void* out);

#ifdef __cplusplus
}
#endif
#endif /* EMB_H_ */
