/*
 * ttemb.h -- C ABI of libttemb.so: the B200 (sm_100a) TT-EmbeddingBag hot path.
 *
 * What it computes (PAPER.md, cited P:<line>; DESIGN.md for the readings R1..R24):
 *   A table W_t in R^{M_t x N} is stored as three TT cores (Eq. 1-2):
 *     C1[m1][n1][R], C2[m2][R][n2][R], C3[m3][R][n3],   N = n1 n2 n3,  m1 m2 m3 >= M_t
 *   Row i has digits i1 = floor(i/(m2 m3)), i2 = floor(i/m3) mod m2, i3 = i mod m3
 *   (Eq. 3, pinned by the Fig. 5(b) example P:164) and
 *     W_t[i, (j1 n2 + j2) n3 + j3] = sum_{r1,r2} C1[i1,j1,r1] C2[i2,r1,j2,r2] C3[i3,r2,j3].
 *   forward:  out[b][t][:] = sum_{j in bag(t,b)} W_t[indices[j], :]   (sum pooling, Eq. 4,
 *             P:164-167; a drop-in for nn.EmbeddingBag(mode="sum"))
 *   backward: dL/dC_k of L = sum(out * grad_out)  (Eq. 6 read as left^T dL/de right^T,
 *             P:185-191), gradients aggregated per unique row first
 *   update:   SGD  C -= lr g;  Adagrad  S += g^2, C -= lr g / (sqrt(S) + eps)
 * Inside, the forward computes each shared prefix product C1[i1] C2[i2] once per
 * batch (the Reuse buffer) and the backward reduces per unique core slice.
 *
 * Conventions
 *   * Every call returns int: 0 = TTEMB_OK, < 0 = ttemb_status.  Host-detectable
 *     errors return before anything is enqueued.
 *   * "device" pointers are CUDA global memory on the handle's device; "host"
 *     pointers are CPU memory (pinned for asynchronous copies).
 *   * `stream` is a cudaStream_t (NULL = legacy default stream).  Every call is
 *     asynchronous on it; nothing synchronises the host except ttemb_check,
 *     ttemb_read_counts and ttemb_stage_times.
 *   * Offsets are table-major: bag (t,b) = indices[offsets[t*B+b] .. offsets[t*B+b+1]),
 *     offsets[0] = 0, non-decreasing, offsets[T*B] = nnz.  out / grad_out are
 *     [B][T][dim] float32, row-major (DLRM's concatenated embedding layer).
 *   * Ownership: the caller allocates every buffer (cores, optimizer state,
 *     gradients, workspace) and keeps it alive until ttemb_destroy; the library
 *     never allocates device memory on the hot path.  Not thread-safe per handle;
 *     one forward may be in flight per handle (its plan is kept for backward).
 *   * Device-detectable input errors (id < 0 or id >= M_t, including padding ids
 *     in [M_t, m1 m2 m3), malformed offsets) set a flag in device memory; outputs
 *     of that step are unspecified (but memory-safe) and ttemb_check reports
 *     TTEMB_ERR_INDEX_RANGE / TTEMB_ERR_INVALID_ARG.
 */
#ifndef TTEMB_H
#define TTEMB_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TTEMB_OK = 0,
  TTEMB_ERR_INVALID_ARG = -1,   /* bad config / argument / offsets                */
  TTEMB_ERR_UNSUPPORTED = -2,   /* num_cores != 3, rank/factor limits exceeded    */
  TTEMB_ERR_INDEX_RANGE = -3,   /* an id outside [0, M_t) (reported by ttemb_check) */
  TTEMB_ERR_STATE = -4,         /* backward without forward, update when fused    */
  TTEMB_ERR_CUDA = -5,          /* a CUDA runtime error                           */
  TTEMB_ERR_CAPACITY = -6       /* nnz > max_nnz or batch > max_batch             */
} ttemb_status;

typedef enum { TTEMB_SGD = 0, TTEMB_ADAGRAD = 1 } ttemb_opt;

/* ttemb_config.flags */
#define TTEMB_FUSED_UPDATE 1u   /* backward applies the update (single replica) */
#define TTEMB_FP32_CORES 2u     /* force the FP32 CUDA-core contraction path (no tcgen05) */
/* Ablation switches (Fig. 14 / 17 / 18 of the paper).  Results are unchanged
 * (same outputs and gradients up to fp32 rounding order); only the amount of work grows. */
#define TTEMB_NO_PREFIX_REUSE 4u  /* every unique row computes its own prefix product
                                     C1[i1] C2[i2] (disables batch-level intermediate-result
                                     reuse) */
#define TTEMB_MEAN_POOLING 16u   /* nn.EmbeddingBag mode="mean": out = sum / |bag| (empty
                                     bag -> 0); default is mode="sum" (P:48, P:306 drop-in) */
#define TTEMB_NO_AGGREGATION 8u   /* every lookup occurrence is its own row in forward and
                                     backward (disables row dedup and the in-advance gradient
                                     aggregation) */

typedef struct {
  int64_t num_rows;        /* M_t >= 1 */
  int32_t row_factors[3];  /* (m1, m2, m3), m1 m2 m3 >= M_t  (R10); ignored if dense */
  int32_t dense;           /* != 0: hybrid placement (only tables with more than 1 M
                              rows are TT-compressed) -- the table is a plain EmbeddingBag
                              table W[M_t][dim] in the cores buffer (ttemb_core_layout core 0,
                              shape {M_t, dim, 1, 1}; cores 1 and 2 are empty), looked up,
                              pooled, aggregated and updated by the same call */
} ttemb_table;

typedef struct {
  int32_t num_tables;            /* T >= 1 (T = 1 is a plain EmbeddingBag)            */
  const ttemb_table* tables;     /* [T], host memory, copied by ttemb_create          */
  int32_t num_cores;             /* must be 3 (the paper's design)         */
  int32_t dim;                   /* N = col_factors[0]*col_factors[1]*col_factors[2]  */
  int32_t col_factors[3];        /* (n1, n2, n3), shared by all tables                */
  int32_t rank;                  /* R1 = R2 = rank (1..128), R0 = R3 = 1; the
                                    tensor-core path runs R = 32, 64, 128 natively and STORES
                                    a rank 16..31 / 33..63 zero-padded to 32 / 64
                                    (ttemb_core_layout reports the storage shapes; padding
                                    entries must be 0 and stay 0)                         */
  int32_t index_bits;            /* 64 (int64 ids, PyTorch default) or 32             */
  int32_t max_batch;             /* B capacity (workspace sizing)                     */
  int64_t max_nnz;               /* nnz capacity, <= 2^30                             */
  int32_t optimizer;             /* ttemb_opt                                         */
  float adagrad_eps;             /* Adagrad eps (PyTorch default 1e-10)               */
  uint32_t flags;                /* TTEMB_FUSED_UPDATE | TTEMB_FP32_CORES | ablations */
} ttemb_config;

typedef struct ttemb_ctx* ttemb_t;

/* Byte sizes of the caller-owned buffers for `cfg`.  core_bytes == grad_bytes;
 * state_bytes is 0 for SGD.  Pure host computation. */
int ttemb_query_sizes(const ttemb_config* cfg, size_t* core_bytes, size_t* state_bytes,
                      size_t* grad_bytes, size_t* workspace_bytes);

/* Validate `cfg` and bind the caller's device buffers (sizes from
 * ttemb_query_sizes; 256-byte aligned): cores (parameters, initialised by the
 * caller via ttemb_core_layout), state (Adagrad accumulator, zero-initialised
 * by the caller; may be NULL for SGD), grads (dense dL/dC, same layout as
 * cores, ZERO-initialised by the caller; written by ttemb_backward, read by
 * ttemb_update; safe to all-reduce in place between the two; with
 * TTEMB_FUSED_UPDATE the backward keeps it zero between steps), workspace
 * (scratch).  ttemb_create enqueues no device work and never touches these
 * buffers, so a second handle on the same cores / state / grads (cross-step
 * pipelining, ttemb_plan_batch) may be created at any time.  `device` is the
 * CUDA ordinal the buffers live on.  On success *out is a new handle.
 * Errors: INVALID_ARG (null / misaligned pointers, bad factors, Adagrad with
 * adagrad_eps <= 0), UNSUPPORTED (limits), CUDA. */
int ttemb_create(const ttemb_config* cfg, int device, void* cores, void* state, void* grads,
                 void* workspace, ttemb_t* out);
int ttemb_destroy(ttemb_t h);

/* Where core `core` (0, 1, 2) of table `table` lives: float offset into the
 * cores / grads / state buffers and its shape:
 *   core 0: {m1, n1, R, 1}   core 1: {m2, R, n2, R}   core 2: {m3, R, n3, 1}. */
int ttemb_core_layout(ttemb_t h, int table, int core, int64_t* offset_floats,
                      int32_t shape[4]);

/* Forward (device buffers): indices [nnz] (int64 or int32 per index_bits),
 * offsets [T*batch+1] int64, out [batch][T][dim] float32 (fully overwritten).
 * Runs the index stage (sort / unique / inverse / prefixes), the prefix and
 * row contractions and the pooling; keeps the plan for ttemb_backward. */
int ttemb_forward(ttemb_t h, const void* indices, const int64_t* offsets, int64_t nnz,
                  int32_t batch, float* out, void* stream);

/* Backward of the last forward: grad_out [batch][T][dim] float32 (device).
 * Without TTEMB_FUSED_UPDATE it overwrites the whole grads buffer with dL/dC
 * (untouched slices 0); with it, it applies the update with `lr` instead
 * (grads then stays zero).  Exactly one backward per forward: a second call
 * (or one without a forward) returns TTEMB_ERR_STATE. */
int ttemb_backward(ttemb_t h, const float* grad_out, float lr, void* stream);

/* Optimizer step from the grads buffer (after an optional all-reduce SUM).
 * TTEMB_ERR_STATE when the handle was created with TTEMB_FUSED_UPDATE. */
int ttemb_update(ttemb_t h, float lr, void* stream);

/* Data-parallel plumbing ("the only communication is the
 * gradient all-reduce").
 * ttemb_grad_buckets: the gradient buffer as contiguous float ranges in the order the
 * (unfused) backward finalises them, so a caller can start the all-reduce of a bucket while the
 * backward is still computing the next: bucket 0 = the dense (hybrid) tables (final after the
 * aggregation), bucket 1 = every C3 core (final after the row stage), bucket 2 = every C1 and
 * C2 core (final at the end of the backward).  Writes up to max_buckets (begin, count) pairs
 * (float offsets into grads; count 0 = empty bucket) and returns the number of buckets (3).
 * ttemb_set_bucket_events: `events` is an array of n (<= 3) cudaEvent_t (host handles, owned by
 * the caller; NULL / n = 0 switches it off); every later unfused ttemb_backward records event i
 * on its stream as soon as bucket i is final (the tcgen05 path records them at those points,
 * the FFMA path after its last gradient kernel).  Capturable in a CUDA graph.
 * ttemb_update_range: the optimizer step restricted to the float range [begin, begin + count)
 * of cores / state / grads (a rank's shard after a reduce-scatter: sharded update, then the
 * caller all-gathers the cores).  TTEMB_ERR_STATE with TTEMB_FUSED_UPDATE, INVALID_ARG for a
 * range outside the buffers. */
int ttemb_grad_buckets(ttemb_t h, int64_t* begin, int64_t* count, int max_buckets);
int ttemb_set_bucket_events(ttemb_t h, void* const* events, int n);
int ttemb_update_range(ttemb_t h, float lr, int64_t begin, int64_t count, void* stream);

/* Offline index-bijection generator (Sec. IV-C), host code: modularity-based
 * community detection (Louvain method, the paper's refs [34], [35]) of an undirected weighted
 * graph with n vertices and m edges (u[e], v[e], w[e] > 0; every edge listed once).  Writes a
 * community label per vertex (0 .. C-1, numbered by first vertex) into labels[n] (host memory,
 * caller-owned).  Deterministic.  INVALID_ARG for null pointers or vertex ids outside [0, n).
 * Used by paper_conf_sc_wangwfmmd22_b200/reorder.py to build the index bijection that
 * ttemb_set_bijection applies at run time. */
int ttemb_louvain(int64_t n, int64_t m, const int64_t* u, const int64_t* v, const double* w, int64_t* labels);

/* ---- Host-memory tier (PAPER §V) ----------------------------------
 * Tables too large for HBM stay in host memory (float32 [n_rows][dim], caller-owned); a CPU
 * parameter server pre-fetches the rows of the next batches and applies the gradients
 * the GPU worker pushes back; the GPU embedding cache below keeps rows that recent batches
 * updated, so a batch pre-fetched before those updates reached host memory is synchronised
 * (the read-after-write conflict).  A batch's host rows travel as a block
 * rows[U][dim] with ids[U] = the distinct global host-row numbers (unique within the batch).
 *
 * ttemb_ht_cache: caller-allocated device buffers (the "index table" and the cached rows):
 *   index[n_rows]        int32, cache slot of a host row or -1
 *   rows[capacity][dim]  float32 cached rows;  lc[capacity] int32 life cycles (0 = free slot)
 *   owner[capacity]      int64 host row of a slot;  free_list[capacity] int32;  top[2] int32
 *                        (free-list size, overflow flag).
 * Capacity: at most `life` batches' rows are live, so life * max(U) slots always suffice; an
 * insert that finds no free slot sets the overflow flag (ttemb_ht_cache_stats) and that row is
 * not cached (later reads of it may then be stale).
 * All device calls are asynchronous on `stream` (cudaStream_t, NULL = legacy default) and return
 * TTEMB_ERR_INVALID_ARG (null pointers, negative sizes) before enqueuing anything. */
typedef struct {
  int32_t* index;
  float* rows;
  int32_t* lc;
  int64_t* owner;
  int32_t* free_list;
  int32_t* top;
  int64_t n_rows;
  int32_t capacity;
  int32_t dim;
} ttemb_ht_cache;

/* Empty cache: index = -1, every slot free. */
int ttemb_ht_cache_init(const ttemb_ht_cache* c, void* stream);
/* Step 1 of P:290 / P:298: rows[u] = the cached row of ids[u] where one exists (device ids[n],
 * rows[n][dim]); other rows keep the pre-fetched values. */
int ttemb_ht_sync(const ttemb_ht_cache* c, const int64_t* ids, int64_t n, float* rows, void* stream);
/* Sum pooling over the block: bag (t,b) = positions offsets[t*batch+b] .. offsets[t*batch+b+1]
 * (int64, table-major like ttemb_forward), ridx[j] = block row of position j (int32);
 * out[b][t][:] = sum of rows[ridx[j]] in position order (float32, written in full). */
int ttemb_ht_pool(const float* rows, const int32_t* ridx, const int64_t* offsets, int32_t num_tables,
                  int32_t batch, int32_t dim, float* out, void* stream);
/* Row gradients of L = sum(out * grad_out): g[u] = sum over k in [occ_ptr[u], occ_ptr[u+1]) of
 * grad_out[b][t] with bag occ_bag[k] = t*batch + b (the positions of row u, in position order). */
int ttemb_ht_grad(const float* grad_out, const int64_t* occ_ptr, const int32_t* occ_bag, int64_t n,
                  int32_t num_tables, int32_t batch, int32_t dim, float* g, void* stream);
/* One pull from the gradient queue: every live entry's LC decreases by 1; an entry that
 * reaches 0 is evicted (index entry -1, slot freed). */
int ttemb_ht_tick(const ttemb_ht_cache* c, void* stream);
/* SGD on the block, rows[u] = rows[u] - rn(lr * g[u]) (two roundings, the server's arithmetic),
 * then, for life > 0, insert / refresh each row in the cache with LC = life ("the
 * maximum length of the Requests Queue").  life = 0 updates without caching. */
int ttemb_ht_update_push(const ttemb_ht_cache* c, float* rows, const float* g, const int64_t* ids, int64_t n,
                         float lr, int32_t life, void* stream);
/* Live entries and the overflow flag (synchronises `stream`). */
int ttemb_ht_cache_stats(const ttemb_ht_cache* c, int32_t* live, int32_t* overflow, void* stream);
/* Parameter-server side, host memory, `nthreads` worker threads (<= 0: up to 16):
 * gather out[u] = table[ids[u]] (the pre-fetch) and apply table[ids[u]] -= rn(lr * g[u]).
 * TTEMB_ERR_INDEX_RANGE (nothing written) for an id outside [0, n_rows); ids must be distinct. */
int ttemb_ht_host_gather(const float* table, int64_t n_rows, int32_t dim, const int64_t* ids, int64_t n,
                         float* out, int32_t nthreads);
int ttemb_ht_host_sgd(float* table, int64_t n_rows, int32_t dim, const int64_t* ids, int64_t n, const float* g,
                      float lr, int32_t nthreads);

/* Host-buffer variants (end-to-end path): copy the inputs from host memory
 * into the workspace staging area, run the step, and copy `out` back to the
 * host, all on `stream`.  Pinned host memory keeps the copies asynchronous. */
int ttemb_forward_host(ttemb_t h, const void* host_indices, const int64_t* host_offsets,
                       int64_t nnz, int32_t batch, float* host_out, void* stream);
int ttemb_backward_host(ttemb_t h, const float* host_grad_out, float lr, void* stream);

/* Synchronise `stream` and report deferred device errors of the last calls
 * (TTEMB_ERR_INDEX_RANGE, TTEMB_ERR_INVALID_ARG for malformed offsets). */
int ttemb_check(ttemb_t h, void* stream);

/* Device-resident results of the index stage of the last forward (valid until
 * the next forward).  Counts live on the device (read them with
 * ttemb_read_counts).  Arrays are uint32; sizes in brackets. */
typedef struct {
  int64_t nnz;
  int32_t batch;
  const uint32_t* counts;    /* [16] U, P, NG, error flags, ... (ttemb_read_counts)    */
  const uint32_t* skey;      /* [nnz] sorted plan keys (R29): for a TT table
                                 key = kbase_t + (i2 m1 + i1) m3 + i3 with the digits of
                                 Eq. 3 and kbase_t = sum of m1 m2 m3 over earlier TT
                                 tables; dense (hybrid) tables follow all TT keys with
                                 key = kbase_t + id.  A bijection of (t, row) for valid ids,
                                 ordered by (t, i2, i1, i3)                                */
  const uint32_t* spos;      /* [nnz] stable argsort of the keys                       */
  const uint32_t* bag_of;    /* [nnz] output row b*T + t of position j                 */
  const uint32_t* ukey;      /* [U] distinct plan keys, ascending                       */
  const uint32_t* seg_off;   /* [U+1] sorted-position segment of each unique row        */
  const uint32_t* inverse;   /* [nnz] unique slot of position j                         */
  const uint32_t* row_pfx;   /* [U] prefix slot of each unique row                      */
  const uint32_t* row_i3;    /* [U] third digit                                         */
  const uint32_t* pfx_t;     /* [P] table of each unique prefix (t, floor(row/m3))      */
  const uint32_t* pfx_i1;    /* [P] first digit                                         */
  const uint32_t* pfx_i2;    /* [P] second digit                                        */
  const uint32_t* row_seg;   /* [P+1] unique rows of each prefix                        */
  const uint32_t* grp_pfx;   /* [P] prefix slot of the q-th prefix in (t, i2, i1) order;
                                 the identity, because the plan key already orders the
                                 prefixes that way (kept for ABI stability)            */
  const uint32_t* grp_off;   /* [NG+1] i2-groups (one C2 slice each)                    */
  const uint32_t* grp_t;     /* [NG] */
  const uint32_t* grp_i2;    /* [NG] */
  const float* rows;         /* [U][dim] W rows of the unique ids                       */
} ttemb_plan;

int ttemb_get_plan(ttemb_t h, ttemb_plan* plan);

/* The forward in two halves, so that the index stage of the NEXT batch (a1-a4: key build, sort,
 * unique rows / prefixes / groups -- it reads no parameters) can run on another stream while the
 * current batch's forward compute / backward / update run (cross-step pipelining).
 * ttemb_plan_batch: the index stage for (indices, offsets[, per_sample_weights]) into this handle's
 * workspace (same arguments and errors as ttemb_forward_weighted minus `out`); `offsets` must stay
 * valid until ttemb_forward_planned.  ttemb_forward_planned: the contractions + pooling of the
 * planned batch (TTEMB_ERR_STATE without a preceding ttemb_plan_batch).  ttemb_forward = both.
 * To pipeline, create two handles on the SAME cores / state / grads buffers (each with its own
 * workspace) and alternate them; order the streams so that a handle's plan starts after its
 * previous backward and the forward after its plan. */
int ttemb_plan_batch(ttemb_t h, const void* indices, const int64_t* offsets, const float* per_sample_weights,
               int64_t nnz, int32_t batch, void* stream);
int ttemb_forward_planned(ttemb_t h, float* out, void* stream);

/* ttemb_forward with per-sample weights (nn.EmbeddingBag(mode="sum") per_sample_weights):
 * out[b][t] = sum_j w[j] W_t[idx_j]; `per_sample_weights` is a DEVICE float array [nnz]
 * aligned with `indices` (NULL = all ones, i.e. ttemb_forward).  The weights are copied into
 * the workspace by the key-build kernel, so the caller may reuse the buffer once the call's
 * work has run; the following ttemb_backward differentiates the weighted bags
 * (G_u = sum_j w[j] grad_out[bag(j)]; the weights themselves get no gradient).
 * TTEMB_ERR_INVALID_ARG with TTEMB_MEAN_POOLING (PyTorch allows weights only with "sum"). */
int ttemb_forward_weighted(ttemb_t h, const void* indices, const int64_t* offsets,
                           const float* per_sample_weights, int64_t nnz, int32_t batch, float* out,
                           void* stream);

/* Runtime index bijection (Sec. IV-B: "all indices will first be transformed into
 * new indices based on the index bijection function ... New_Batch = {index(i_j)}").
 * `bijection` is a DEVICE array of uint32 with one entry per row of every table,
 * concatenated in table order (table t occupies [rowbase_t, rowbase_t + M_t), rowbase_t =
 * M_0 + ... + M_{t-1}; ttemb_total_rows gives the length): every later forward looks up
 * row bijection[rowbase_t + i] of table t for id i.  The caller owns the buffer and keeps
 * it alive and unchanged while forwards run; NULL switches the mapping off.  The map must
 * send [0, M_t) into [0, M_t) (a bijection for the method's purpose); a mapped id >= M_t
 * raises TTEMB_ERR_INDEX_RANGE through ttemb_check like a raw out-of-range id.  Applied
 * inside the key-build kernel (no extra pass).  Generate one offline, e.g. with the
 * frequency ordering of Alg. 2 lines 1-4 (paper_conf_sc_wangwfmmd22_b200/reorder.py). */
int ttemb_set_bijection(ttemb_t h, const uint32_t* bijection);
uint64_t ttemb_total_rows(ttemb_t h);   /* sum of M_t (length of a bijection buffer); 0 for NULL */

/* Synchronous helper: copy {U, P, NG, error flags} of the last forward to host. */
int ttemb_read_counts(ttemb_t h, int64_t counts[4], void* stream);

/* Per-stage device timing (CUDA events on the launching stream).  While
 * enabled, every stage of forward/backward/update records an event pair;
 * ttemb_stage_times synchronises and returns, per stage id, the summed
 * milliseconds and launch count since the last reset; names via
 * ttemb_stage_name.  Returns the number of stages. */
int ttemb_set_timing(ttemb_t h, int enable);
int ttemb_stage_times(ttemb_t h, double* ms, int64_t* launches, int max_stages);
const char* ttemb_stage_name(int stage);

const char* ttemb_status_string(int status);

#ifdef __cplusplus
}
#endif
#endif /* TTEMB_H */
