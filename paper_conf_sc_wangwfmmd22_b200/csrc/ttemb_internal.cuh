// ttemb_internal.cuh -- shared host/device definitions of libttemb.so (B200, sm_100a).
//
// Data layout in HBM:
//   cores / grads / state: [all tables' C1][all tables' C2][all tables' C3], fp32,
//   C1_t[m1][n1][R], C2_t[m2][R][n2][R], C3_t[m3][R][n3]; each table's block starts
//   16-byte aligned so slices can be moved as float4.
//   workspace: the index-stage plan (u32 arrays), the prefix products (Reuse buffer,
//   P:178), unique rows, aggregated row gradients, dP, dC1 partials, the per-step
//   zeroed scan/sort state, and host staging buffers.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include <vector>

#include "../../include/ttemb.h"

namespace ttemb {

// ---- error flags in counts[3] ------------------------------------------------
constexpr uint32_t kErrRange = 1u;     // an id outside [0, M_t)
constexpr uint32_t kErrOffsets = 2u;   // malformed offsets

// counts[] slots (device)
constexpr int kCntU = 0, kCntP = 1, kCntNG = 2, kCntErr = 3, kCntMulti = 4, kCntUtt1 = 5,
              kCntNCh = 6, kCntNSplit = 7, kNumCounts = 16;

// FFMA group kernels: an i2-group is processed in units of at most kGroupChunk prefixes, so a
// Zipf-hot group is spread over many CTAs (dC2 partials of split groups meet by reductions).
constexpr uint32_t kGroupChunk = 128;

// Unique rows [0, Utt) belong to TT tables, [Utt, U) to dense (hybrid) tables: plan keys number
// the TT tables first.  counts[kCntUtt1] = Utt + 1 when a dense row exists, else 0.
__host__ __device__ inline uint32_t tt_rows(const uint32_t* counts) {
  return counts[kCntUtt1] ? counts[kCntUtt1] - 1 : counts[kCntU];
}

// ---- stage ids for per-stage timing ----------------------------------------------
enum Stage : int {
  ST_ZERO = 0, ST_KEYS, ST_SORT_HIST, ST_SORT_PASS, ST_UNIQUE, ST_PREFIX, ST_GSORT_HIST,
  ST_GSORT_PASS, ST_GROUPS, ST_FWD_PREFIX, ST_FWD_ROWS, ST_POOL, ST_BWD_ZERO, ST_AGG,
  ST_AGG_FIX, ST_BWD_ROWS, ST_BWD_PREFIX, ST_DC1, ST_UPD_C3, ST_UPDATE, ST_H2D, ST_D2H,
  ST_COUNT
};

// Debug / experiment knobs from the environment, read ONCE per process (never on the launch
// path): TTEMB_EXP bits switch parts of k_prefix_bwd off (timing experiments, results invalid),
// TTEMB_DBG likewise for the forward kernels, TTEMB_TRACE enables role timers (trace builds),
// TTEMB_PF_BWD sets an L2 prefetch distance in k_prefix_bwd; TTEMB_NO_PDL=1 launches the main
// chain without programmatic dependent launch (bench.py sets it for N > 1, where the step graph
// interleaves NCCL kernels and no multi-GPU box was available to validate PDL next to them).
struct Knobs {
  int exp = 0, dbg = 0, trace = 0, pf_bwd = 0, no_pdl = 0;
};
inline const Knobs& knobs() {
  static const Knobs k = [] {
    auto num = [](const char* n) { const char* e = getenv(n); return e ? atoi(e) : 0; };
    Knobs r;
    r.exp = num("TTEMB_EXP"); r.dbg = num("TTEMB_DBG"); r.trace = getenv("TTEMB_TRACE") ? 1 : 0;
    r.pf_bwd = num("TTEMB_PF_BWD"); r.no_pdl = num("TTEMB_NO_PDL");
    return r;
  }();
  return k;
}
inline int exp_bits() { return knobs().exp; }

// Index of the key range holding `key` (kbase[0..T-1] ascending, in key order).
__device__ __forceinline__ int table_of_key(const uint64_t* kbase, int T, uint32_t key) {
  int lo = 0, hi = T - 1;   // last range with kbase[i] <= key
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (__ldg(kbase + mid) <= key) lo = mid; else hi = mid - 1;
  }
  return lo;
}

struct TableMeta {
  uint32_t m1, m2, m3, M;      // row factors, rows (M <= 2^32-1 checked on host)
  uint64_t rowbase;            // exclusive prefix sum of M (row numbering across tables)
  uint64_t kbase;              // first plan key of the table: exclusive prefix sum of m1 m2 m3
  uint64_t c1_off, c2_off, c3_off;  // float offsets into cores / grads / state
  uint32_t grpbase;            // first (t, i2) bucket id = sum of m2 of earlier TT tables
  uint32_t dense;              // hybrid placement: plain table W[M][N] at c1_off
};

// Per-step plan pointers (all device).
struct PlanDev {
  uint32_t* counts;
  uint32_t *keysA, *valsA, *keysB, *valsB;     // radix ping-pong (sort 1), reused by sort 2
  uint32_t *skey, *spos;                       // -> final sort-1 buffers
  uint32_t *bag_of, *sbag, *inverse;           // [nnz]
  uint32_t *ukey, *seg_off, *row_pfx, *row_i3; // [U]
  uint32_t* row_c3;                            // [U] C3 slice of the row: (C3 float offset - c3_begin) / (R n3)
  uint32_t *pfx_t, *pfx_i1, *pfx_i2, *row_seg; // [P]
  uint32_t *gkeyA, *gvalA, *gkeyB, *gvalB;     // group sort ping-pong [P]
  uint32_t *gkey, *gval;                       // -> final sort-2 buffers
  uint32_t *grp_pfx, *grp_off, *grp_t, *grp_i2;
  uint32_t *hist1, *dbase1, *hist2, *dbase2;   // [4][256]
  uint32_t *rs1_counter, *rs1_status;          // sort-1 look-back state [4][tiles][256]
  uint32_t *rs2_counter, *rs2_status;
  uint32_t *sc_counter, *sc_status;            // scans [3][tiles]
  uint32_t* work;                              // dynamic group schedulers [2]
  float *rows, *gbuf, *dabuf, *aggpart;
  float* wpos;                                 // [nnz] bag weight of every position (weighted/mean bags)
  float *pbuf, *dpbuf;                         // tensor-core path: P and dL/dP per prefix
  float* dc2buf;                               // fused Adagrad (tensor-core path): dC2 per group [NG][R NC]
  uint32_t* grp_arow;                          // [P]  C1 row (float offset / R) of sorted prefix q, j1 = 0
  uint32_t *chunk_off, *split_list;            // FFMA path: [NG+1] first unit of group g; [NG] split groups
  unsigned long long* grp_c2;                  // [NG] float offset of the C2 slice of group g
  uint32_t *unit_sorted, *unit_snake;          // [NU] prefix-kernel work units by tile count (desc) /
                                               // that order dealt to the backward grid boustrophedon
};

struct Ctx {
  // configuration
  int device = 0, sm_count = 148;
  int T = 0, n1 = 0, n2 = 0, n3 = 0, N = 0, R = 0, NC = 0;
  int R_user = 0;                    // the configured rank (R may be the zero-padded storage rank)
  int index_bits = 64, opt = 0;
  float eps = 1e-10f;
  uint32_t flags = 0;
  int64_t max_nnz = 0;
  int32_t max_batch = 0;
  uint64_t total_rows = 0, total_keys = 0;
  uint32_t total_buckets = 0;
  int key_passes = 1, gkey_passes = 1;
  int64_t U_cap = 0, P_cap = 0, NG_cap = 0;
  int64_t rs1_tiles = 0, rs2_tiles = 0, sc_tiles = 0;
  std::vector<TableMeta> meta;
  size_t core_floats = 0, c1_floats = 0, c3_begin = 0, c3_floats = 0;

  // caller buffers
  float* cores = nullptr;
  float* state = nullptr;
  float* grads = nullptr;
  uint8_t* ws = nullptr;
  const uint32_t* bij = nullptr;     // runtime index bijection [sum M_t], or null

  // workspace carve
  TableMeta* d_meta = nullptr;
  uint64_t* d_kbase = nullptr;       // [T+1] plan-key base of every table (+ total)
  uint32_t* d_grpbase = nullptr;     // [T+1]
  uint32_t* d_kmap = nullptr;        // [T] user table of the i-th key range (d_kbase is in key order)
  int n_dense = 0;                   // hybrid placement: number of dense tables
  uint64_t tt_keys = 0;              // plan keys of the TT tables (dense keys follow)
  size_t dense_begin = 0, dense_floats = 0;   // dense tables' region of cores / grads / state
  PlanDev p{};
  uint8_t* zero_begin = nullptr;
  size_t zero_bytes = 0;
  void* st_idx = nullptr;
  int64_t* st_off = nullptr;
  float* st_out = nullptr;
  float* st_grad = nullptr;
  size_t ws_bytes = 0;

  // step state
  int64_t nnz = 0;
  int32_t B = 0;
  bool fwd_done = false;
  bool bwd_done = false;             // the last forward's backward ran (one backward per forward)
  bool planned = false;              // ttemb_plan ran; ttemb_forward_planned may follow
  const int64_t* offsets = nullptr;  // the planned batch's offsets (device; caller keeps alive)
  const float* psw = nullptr;        // per-sample weights of the current forward (device) or null
  bool weighted = false;             // this step's bags carry weights (psw or mean): p.wpos valid

  // data-parallel gradient buckets (ttemb_set_bucket_events): event i recorded when bucket i is final
  cudaEvent_t bucket_ev[3] = {nullptr, nullptr, nullptr};
  void mark_bucket(int i, cudaStream_t s) const {
    if (bucket_ev[i]) cudaEventRecord(bucket_ev[i], s);
  }

  // TMA tensor maps of the prefix-backward kernel (dP stash, C2 region), encoded on first use
  // (the buffers never move)
  CUtensorMap tm_dp{}, tm_c2{};
  bool tm_bwd_ready = false;

  // timing
  bool timing = false;
  std::vector<cudaEvent_t> ev_pool;
  struct Pending { int stage; cudaEvent_t a, b; };
  std::vector<Pending> pending;
  double stage_ms[ST_COUNT] = {};
  int64_t stage_n[ST_COUNT] = {};
};

// ---- stage timing helpers (host) ---------------------------------------------------
struct StageScope {
  Ctx& c; int stage; cudaStream_t s; cudaEvent_t a = nullptr, b = nullptr;
  StageScope(Ctx& c_, int st, cudaStream_t s_);
  ~StageScope();
};

// ---- launchers (host) ----------------------------------------------------------------
cudaError_t run_index_stage(Ctx& c, const void* indices, const int64_t* offsets, cudaStream_t s);
cudaError_t run_forward_compute(Ctx& c, float* out, const int64_t* offsets, cudaStream_t s);
cudaError_t run_backward(Ctx& c, const float* grad_out, float lr, cudaStream_t s);
cudaError_t run_update(Ctx& c, float lr, cudaStream_t s);
cudaError_t run_update_range(Ctx& c, float lr, size_t begin, size_t count, cudaStream_t s);
cudaError_t configure_group(Ctx& c);
cudaError_t configure_tc(Ctx& c);
bool tc_eligible(const Ctx& c);
cudaError_t run_tc_fwd(Ctx& c, float* out, cudaStream_t s);
cudaError_t run_tc_bwd(Ctx& c, float lr, cudaStream_t s);
bool fused_eligible(const Ctx& c);
cudaError_t run_dp_zero(Ctx& c, cudaStream_t s);
cudaError_t run_unit_order(Ctx& c, cudaStream_t s);
int prefix_units_per_group(const Ctx& c);
int prefix_bwd_grid(const Ctx& c);
cudaError_t run_plan_tail(Ctx& c, cudaStream_t s);
cudaError_t configure_fused(Ctx& c);
cudaError_t run_fused_fwd(Ctx& c, float* out, cudaStream_t s);
cudaError_t run_rows_bwd2(Ctx& c, cudaStream_t s);
cudaError_t configure_bwdtc(Ctx& c);
cudaError_t run_prefix_bwd(Ctx& c, float lr, cudaStream_t s);

// ---- small helpers -------------------------------------------------------------------
static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Programmatic dependent launch along the step's main chain (forward: prefix -> rows -> pooling;
// backward: aggregation -> rows -> prefix -> update).  A kernel launched with launch_pdl may be
// scheduled while its predecessor on the stream is still draining; it calls pdl_wait() before
// its first access to anything the predecessor wrote (every such kernel does so on entry), so
// results are those of plain stream order.  The successor is released when the predecessor's CTAs
// exit (implicit trigger): c4 step 433 -> 430 us in an interleaved A/B.  Triggering on entry
// (pdl_trigger, built only with TTEMB_PDL_EARLY_TRIGGER) measured 483 us: early successor CTAs
// took SMs from the predecessors' later waves and from the pipelined index stage.  TTEMB_EXP bit
// 32768 launches without the attribute (plain stream order) for comparison.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() {
#ifdef TTEMB_PDL_EARLY_TRIGGER
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid; cfg.blockDim = block; cfg.dynamicSmemBytes = smem; cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = ((exp_bits() & 32768) || knobs().no_pdl) ? 0 : 1;
  cfg.attrs = at; cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}
inline cudaError_t launch_pdl_ptr(const void* kernel, dim3 grid, dim3 block, size_t smem, cudaStream_t s, void** args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid; cfg.blockDim = block; cfg.dynamicSmemBytes = smem; cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = ((exp_bits() & 32768) || knobs().no_pdl) ? 0 : 1;
  cfg.attrs = at; cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, kernel, args);
}
static inline int grid_for(const Ctx& c, int64_t items, int threads, int per_sm = 32) {
  int64_t g = cdiv(items, threads);
  int64_t cap = (int64_t)c.sm_count * per_sm;
  if (g > cap) g = cap;
  if (g < 1) g = 1;
  return (int)g;
}

}  // namespace ttemb
