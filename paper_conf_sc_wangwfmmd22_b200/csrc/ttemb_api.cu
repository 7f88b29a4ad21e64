// ttemb_api.cu -- the C ABI of libttemb.so (include/ttemb.h): configuration checks,
// buffer layout, workspace carving, stage sequencing, deferred error reporting and
// per-stage CUDA-event timing.  No kernel arithmetic lives here.
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <new>

#include "ttemb_internal.cuh"

namespace ttemb {
int64_t radix_tiles(int64_t n);
int64_t scan_tiles(int64_t n);
int64_t agg_chunks(int64_t nnz);
int64_t dc1_chunks(int64_t P);

StageScope::StageScope(Ctx& c_, int st, cudaStream_t s_) : c(c_), stage(st), s(s_) {
  if (!c.timing) return;
  if (c.ev_pool.size() < 2) {
    for (int i = 0; i < 64; ++i) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) == cudaSuccess) c.ev_pool.push_back(e);
    }
  }
  if (c.ev_pool.size() < 2) return;
  a = c.ev_pool.back(); c.ev_pool.pop_back();
  b = c.ev_pool.back(); c.ev_pool.pop_back();
  cudaEventRecord(a, s);
}
StageScope::~StageScope() {
  if (!a) return;
  cudaEventRecord(b, s);
  c.pending.push_back({stage, a, b});
}

static const char* kStageNames[ST_COUNT] = {
    "zero_state", "build_keys", "sort_hist", "sort_pass", "unique", "prefix", "gsort_hist",
    "gsort_pass", "groups", "fwd_prefix", "fwd_rows", "pool", "bwd_zero", "agg", "agg_fix",
    "bwd_rows", "bwd_prefix", "dc1", "update_c3", "update", "h2d", "d2h"};

namespace {

struct Carver {
  uint8_t* base;
  size_t off = 0;
  explicit Carver(uint8_t* b) : base(b) {}
  template <typename T>
  T* take(size_t count) {
    off = (off + 255) & ~(size_t)255;
    T* p = base ? reinterpret_cast<T*>(base + off) : nullptr;
    off += sizeof(T) * (count ? count : 1);
    return p;
  }
};

int bits_for(uint64_t max_value) {
  int b = 0;
  while (b < 64 && (max_value >> b) != 0) ++b;
  return b;
}

int validate(const ttemb_config* cfg) {
  if (!cfg || !cfg->tables || cfg->num_tables < 1) return TTEMB_ERR_INVALID_ARG;
  if (cfg->num_cores != 3) return TTEMB_ERR_UNSUPPORTED;
  const int n1 = cfg->col_factors[0], n2 = cfg->col_factors[1], n3 = cfg->col_factors[2];
  if (n1 < 1 || n2 < 1 || n3 < 1 || (int64_t)n1 * n2 * n3 != cfg->dim) return TTEMB_ERR_INVALID_ARG;
  if (cfg->rank < 1) return TTEMB_ERR_INVALID_ARG;
  if (cfg->rank > 128) return TTEMB_ERR_UNSUPPORTED;
  if (n1 > 8 || n3 > 8 || cfg->dim > 4096) return TTEMB_ERR_UNSUPPORTED;
  if (cfg->index_bits != 64 && cfg->index_bits != 32) return TTEMB_ERR_INVALID_ARG;
  if (cfg->max_batch < 0 || cfg->max_nnz < 0) return TTEMB_ERR_INVALID_ARG;
  if (cfg->max_nnz > (int64_t(1) << 30)) return TTEMB_ERR_UNSUPPORTED;
  if ((int64_t)cfg->num_tables * cfg->max_batch > (int64_t(1) << 31)) return TTEMB_ERR_UNSUPPORTED;
  if (cfg->optimizer != TTEMB_SGD && cfg->optimizer != TTEMB_ADAGRAD) return TTEMB_ERR_INVALID_ARG;
  // Adagrad divides by sqrt(S) + eps; the fused C2 pass also visits zero-gradient entries, so
  // eps = 0 would turn untouched (e.g. rank-padding) entries into 0/0
  if (cfg->optimizer == TTEMB_ADAGRAD && !(cfg->adagrad_eps > 0.f)) return TTEMB_ERR_INVALID_ARG;
  // pooled output / gradient element counts stay below 2^31 (32-bit element indexing)
  if ((int64_t)cfg->num_tables * cfg->max_batch * cfg->dim >= (int64_t(1) << 31)) return TTEMB_ERR_UNSUPPORTED;
  if (cfg->flags & ~(TTEMB_FUSED_UPDATE | TTEMB_FP32_CORES | TTEMB_NO_PREFIX_REUSE | TTEMB_NO_AGGREGATION |
                     TTEMB_MEAN_POOLING))
    return TTEMB_ERR_INVALID_ARG;
  uint64_t total = 0, buckets = 0, keys = 0;
  for (int t = 0; t < cfg->num_tables; ++t) {
    const ttemb_table& tb = cfg->tables[t];
    if (tb.dense) {                       // hybrid placement: plain table, factors ignored
      if (tb.num_rows < 1) return TTEMB_ERR_INVALID_ARG;
      total += (uint64_t)tb.num_rows;
      keys += (uint64_t)tb.num_rows;
      continue;
    }
    const int64_t m1 = tb.row_factors[0], m2 = tb.row_factors[1], m3 = tb.row_factors[2];
    if (tb.num_rows < 1 || m1 < 1 || m2 < 1 || m3 < 1) return TTEMB_ERR_INVALID_ARG;
    if (m1 * m2 * m3 < tb.num_rows) return TTEMB_ERR_INVALID_ARG;
    if (m1 > (1 << 24) || m2 > (1 << 24) || m3 > (1 << 24)) return TTEMB_ERR_UNSUPPORTED;
    total += (uint64_t)tb.num_rows;
    buckets += (uint64_t)m2;
    keys += (uint64_t)(m1 * m2 * m3);
  }
  if (total > 0xFFFFFFFFull || buckets > 0xFFFFFFFFull || keys > 0xFFFFFFFFull) return TTEMB_ERR_UNSUPPORTED;
  return TTEMB_OK;
}

#ifndef TTEMB_PAD_MIN_RANK
#define TTEMB_PAD_MIN_RANK 16   // c2 (R = 16) 1.56x faster padded; c1 (R = 8) is not
#endif
constexpr int kPadMinRank = TTEMB_PAD_MIN_RANK;   // smallest rank run zero-padded on tcgen05

// Fills every size-derived field of c (no device pointers).
void plan_sizes(const ttemb_config* cfg, Ctx& c) {
  c.T = cfg->num_tables;
  c.n1 = cfg->col_factors[0]; c.n2 = cfg->col_factors[1]; c.n3 = cfg->col_factors[2];
  c.N = cfg->dim; c.R = cfg->rank;
  // kPadMinRank <= R < 32 / 32 < R < 64: store the cores zero-padded to rank 32 / 64 and run the
  // tcgen05 path (native kernels exist for R = 32, 64, 128).  Exact: the padded rows / columns of
  // C1, C2, C3 multiply only zeros, so every padded entry of dC_k is exactly 0 and SGD / Adagrad
  // keep it 0 (R28).
  c.R_user = c.R;
  if (!(cfg->flags & TTEMB_FP32_CORES) && c.R >= kPadMinRank && c.R < 64 && c.R != 32 && (c.n3 == 4 || c.n3 == 8) &&
      (c.n1 == 1 || c.n1 == 2 || c.n1 == 4 || c.n1 == 8) && c.n1 * c.n2 <= 16) {
    const int padded = c.R < 32 ? 32 : 64;
    if (c.n2 * padded <= 256) c.R = padded;
  }
  c.NC = c.n2 * c.R;
  c.index_bits = cfg->index_bits; c.opt = cfg->optimizer;
  c.eps = cfg->adagrad_eps; c.flags = cfg->flags;
  c.max_nnz = cfg->max_nnz; c.max_batch = cfg->max_batch;
  c.meta.assign(c.T, TableMeta{});
  const size_t s1 = (size_t)c.n1 * c.R, s2 = (size_t)c.R * c.n2 * c.R, s3 = (size_t)c.R * c.n3;
  auto up4 = [](size_t x) { return (x + 3) & ~(size_t)3; };
  size_t off = 0;
  uint64_t rb = 0, pfx = 0, kb = 0;
  uint32_t gb = 0;
  c.n_dense = 0;
  for (int t = 0; t < c.T; ++t) {   // [C1 of all TT tables]
    const ttemb_table& tb = cfg->tables[t];
    TableMeta& m = c.meta[t];
    m.dense = tb.dense ? 1u : 0u;
    m.M = (uint32_t)tb.num_rows;
    m.rowbase = rb; rb += (uint64_t)tb.num_rows;     // user table order (bijection layout)
    if (m.dense) {
      m.m1 = m.m2 = m.m3 = 1;
      ++c.n_dense;
      continue;
    }
    m.m1 = tb.row_factors[0]; m.m2 = tb.row_factors[1]; m.m3 = tb.row_factors[2];
    m.kbase = kb; kb += (uint64_t)m.m1 * m.m2 * m.m3;   // plan keys: TT tables first
    m.grpbase = gb; gb += m.m2;
    pfx += (uint64_t)((tb.num_rows + m.m3 - 1) / m.m3);
    m.c1_off = off; off += up4(m.m1 * s1);
  }
  c.tt_keys = kb;
  for (int t = 0; t < c.T; ++t)                     // then the dense tables' keys
    if (c.meta[t].dense) { c.meta[t].kbase = kb; kb += c.meta[t].M; }
  c.c1_floats = off;
  for (int t = 0; t < c.T; ++t)
    if (!c.meta[t].dense) { c.meta[t].c2_off = off; off += up4(c.meta[t].m2 * s2); }
  c.c3_begin = off;
  for (int t = 0; t < c.T; ++t)
    if (!c.meta[t].dense) { c.meta[t].c3_off = off; off += up4(c.meta[t].m3 * s3); }
  c.c3_floats = off - c.c3_begin;
  c.dense_begin = off;                               // [W of the dense tables]
  for (int t = 0; t < c.T; ++t)
    if (c.meta[t].dense) { c.meta[t].c1_off = off; c.meta[t].c2_off = c.meta[t].c3_off = 0; off += up4((size_t)c.meta[t].M * c.N); }
  c.dense_floats = off - c.dense_begin;
  c.core_floats = off;
  c.total_rows = rb;
  c.total_keys = kb;
  c.total_buckets = gb;
  c.key_passes = std::max(1, (bits_for(kb ? kb - 1 : 0) + 7) / 8);
  c.gkey_passes = std::max(1, (bits_for(gb ? gb - 1 : 0) + 7) / 8);
  // Ablations (TTEMB_NO_*): every occurrence a row / every row a prefix.
  c.U_cap = (c.flags & TTEMB_NO_AGGREGATION) ? c.max_nnz : std::min<int64_t>(c.max_nnz, (int64_t)rb);
  c.P_cap = (c.flags & TTEMB_NO_PREFIX_REUSE) ? c.U_cap : std::min<int64_t>(c.U_cap, (int64_t)pfx);
  c.NG_cap = std::min<int64_t>(c.P_cap, (int64_t)gb);
  c.rs1_tiles = radix_tiles(c.max_nnz);
  c.rs2_tiles = radix_tiles(c.P_cap);
  c.sc_tiles = std::max<int64_t>(1, scan_tiles(c.max_nnz));
}

// Carves the workspace; with base == nullptr only computes the size.
size_t carve(Ctx& c, uint8_t* base) {
  Carver k(base);
  const int64_t nnz = std::max<int64_t>(c.max_nnz, 1);
  const int64_t U = std::max<int64_t>(c.U_cap, 1), P = std::max<int64_t>(c.P_cap, 1);
  const int64_t NG = std::max<int64_t>(c.NG_cap, 1);
  const int64_t bags = (int64_t)c.T * c.max_batch;
  PlanDev& p = c.p;
  c.d_meta = k.take<TableMeta>(c.T);
  c.d_kbase = k.take<uint64_t>(c.T + 1);
  c.d_grpbase = k.take<uint32_t>(c.T + 1);
  c.d_kmap = k.take<uint32_t>(c.T);
  // --- zeroed every forward ---
  k.off = (k.off + 255) & ~(size_t)255;
  const size_t zb = k.off;
  p.counts = k.take<uint32_t>(kNumCounts);
  p.hist1 = k.take<uint32_t>(4 * 256);
  p.hist2 = k.take<uint32_t>(4 * 256);
  p.rs1_counter = k.take<uint32_t>(4);
  p.rs2_counter = k.take<uint32_t>(4);
  p.sc_counter = k.take<uint32_t>(4);
  p.work = k.take<uint32_t>(4);
  p.rs1_status = k.take<uint32_t>((size_t)c.key_passes * std::max<int64_t>(c.rs1_tiles, 1) * 256);
  p.rs2_status = k.take<uint32_t>((size_t)c.gkey_passes * std::max<int64_t>(c.rs2_tiles, 1) * 256);
  p.sc_status = k.take<uint32_t>((size_t)3 * c.sc_tiles);
  k.off = (k.off + 255) & ~(size_t)255;
  c.zero_bytes = k.off - zb;
  c.zero_begin = base ? base + zb : nullptr;
  // --- plan ---
  p.dbase1 = k.take<uint32_t>(4 * 256);
  p.dbase2 = k.take<uint32_t>(4 * 256);
  p.keysA = k.take<uint32_t>(nnz); p.valsA = k.take<uint32_t>(nnz);
  p.keysB = k.take<uint32_t>(nnz); p.valsB = k.take<uint32_t>(nnz);
  p.bag_of = k.take<uint32_t>(nnz); p.sbag = k.take<uint32_t>(nnz); p.inverse = k.take<uint32_t>(nnz);
  p.ukey = k.take<uint32_t>(U); p.seg_off = k.take<uint32_t>(U + 1);
  p.row_pfx = k.take<uint32_t>(U); p.row_i3 = k.take<uint32_t>(U); p.row_c3 = k.take<uint32_t>(U);
  p.pfx_t = k.take<uint32_t>(P); p.pfx_i1 = k.take<uint32_t>(P); p.pfx_i2 = k.take<uint32_t>(P);
  p.row_seg = k.take<uint32_t>(P + 1);
  p.gkeyB = k.take<uint32_t>(P); p.gvalB = k.take<uint32_t>(P);
  p.grp_pfx = k.take<uint32_t>(P); p.grp_off = k.take<uint32_t>(NG + 1);
  p.grp_t = k.take<uint32_t>(NG); p.grp_i2 = k.take<uint32_t>(NG);
  p.grp_arow = k.take<uint32_t>(P);
  p.chunk_off = k.take<uint32_t>(NG + 1);
  p.split_list = k.take<uint32_t>(NG);
  p.grp_c2 = k.take<unsigned long long>(NG);
  p.unit_sorted = k.take<uint32_t>((size_t)NG * 4);   // <= 4 units per group (R = 128, NC <= 512)
  p.unit_snake = k.take<uint32_t>((size_t)NG * 4);
  // --- float intermediates ---
  p.dabuf = k.take<float>((size_t)P * c.n1 * c.R);
  const size_t pf = tc_eligible(c) ? (size_t)P * c.n1 * c.NC : 1;
  p.pbuf = k.take<float>(pf);
  p.dpbuf = k.take<float>(pf);
  // dC2 per group for the fused Adagrad pass (overwritten every step, so the C2 part of the
  // gradient buffer stays zero and needs no clearing); only the tensor-core path with Adagrad
  p.dc2buf = k.take<float>(tc_eligible(c) && c.opt == TTEMB_ADAGRAD && (c.flags & TTEMB_FUSED_UPDATE)
                               ? (size_t)NG * c.R * c.NC : 1);
  p.wpos = k.take<float>(nnz);
  p.rows = k.take<float>((size_t)U * c.N);
  p.gbuf = k.take<float>((size_t)U * c.N);
  p.aggpart = k.take<float>(std::max<size_t>((size_t)2 * agg_chunks(nnz) * c.N,
                                              (size_t)2 * dc1_chunks(P) * c.n1 * c.R));
  // --- host staging (end-to-end API) ---
  c.st_idx = k.take<uint8_t>((size_t)nnz * (c.index_bits / 8));
  c.st_off = k.take<int64_t>(bags + 1);
  c.st_out = k.take<float>((size_t)std::max<int64_t>(bags, 1) * c.N);
  c.st_grad = k.take<float>((size_t)std::max<int64_t>(bags, 1) * c.N);
  return (k.off + 255) & ~(size_t)255;
}

int map_cuda(cudaError_t e) { return e == cudaSuccess ? TTEMB_OK : TTEMB_ERR_CUDA; }

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace
}  // namespace ttemb

using namespace ttemb;

struct ttemb_ctx {
  Ctx c;
};

extern "C" {

const char* ttemb_status_string(int status) {
  switch (status) {
    case TTEMB_OK: return "ok";
    case TTEMB_ERR_INVALID_ARG: return "invalid argument";
    case TTEMB_ERR_UNSUPPORTED: return "unsupported configuration";
    case TTEMB_ERR_INDEX_RANGE: return "index out of range";
    case TTEMB_ERR_STATE: return "invalid call order";
    case TTEMB_ERR_CUDA: return "CUDA error";
    case TTEMB_ERR_CAPACITY: return "capacity exceeded";
    default: return "unknown status";
  }
}

const char* ttemb_stage_name(int stage) {
  return (stage >= 0 && stage < ST_COUNT) ? kStageNames[stage] : "?";
}

int ttemb_query_sizes(const ttemb_config* cfg, size_t* core_bytes, size_t* state_bytes,
                      size_t* grad_bytes, size_t* workspace_bytes) {
  const int rc = validate(cfg);
  if (rc) return rc;
  Ctx c;
  plan_sizes(cfg, c);
  const size_t cb = sizeof(float) * c.core_floats;
  if (core_bytes) *core_bytes = cb;
  if (grad_bytes) *grad_bytes = cb;
  if (state_bytes) *state_bytes = cfg->optimizer == TTEMB_ADAGRAD ? cb : 0;
  if (workspace_bytes) *workspace_bytes = carve(c, nullptr);
  return TTEMB_OK;
}

int ttemb_create(const ttemb_config* cfg, int device, void* cores, void* state, void* grads,
                 void* workspace, ttemb_t* out) {
  if (!out) return TTEMB_ERR_INVALID_ARG;
  *out = nullptr;
  int rc = validate(cfg);
  if (rc) return rc;
  if (!cores || !grads || !workspace) return TTEMB_ERR_INVALID_ARG;
  if (cfg->optimizer == TTEMB_ADAGRAD && !state) return TTEMB_ERR_INVALID_ARG;
  if (((uintptr_t)cores | (uintptr_t)grads | (uintptr_t)workspace | (uintptr_t)state) & 255)
    return TTEMB_ERR_INVALID_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return TTEMB_ERR_CUDA;
  }
  DeviceGuard dg(device);
  ttemb_ctx* h = new (std::nothrow) ttemb_ctx;
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  plan_sizes(cfg, c);
  c.device = device;
  c.cores = (float*)cores; c.state = (float*)state; c.grads = (float*)grads;
  c.ws = (uint8_t*)workspace;
  c.ws_bytes = carve(c, c.ws);
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) { delete h; return TTEMB_ERR_CUDA; }
  c.sm_count = prop.multiProcessorCount;
  std::vector<uint64_t> rb(c.T + 1);
  std::vector<uint32_t> gb(c.T + 1), km(c.T);
  {   // key ranges in key order (TT tables, then dense tables) -> user table
    int i = 0;
    for (int pass = 0; pass < 2; ++pass)
      for (int t = 0; t < c.T; ++t)
        if ((int)c.meta[t].dense == pass) { rb[i] = c.meta[t].kbase; km[i] = (uint32_t)t; ++i; }
  }
  for (int t = 0; t < c.T; ++t) gb[t] = c.meta[t].grpbase;
  rb[c.T] = c.total_keys; gb[c.T] = c.total_buckets;
  cudaError_t e = cudaMemcpy(c.d_meta, c.meta.data(), sizeof(TableMeta) * c.T, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c.d_kbase, rb.data(), sizeof(uint64_t) * (c.T + 1), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c.d_grpbase, gb.data(), sizeof(uint32_t) * (c.T + 1), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c.d_kmap, km.data(), sizeof(uint32_t) * c.T, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = configure_group(c);
  if (e == cudaSuccess) e = configure_tc(c);
  if (e == cudaSuccess) e = configure_fused(c);
  if (e == cudaSuccess) e = configure_bwdtc(c);
  // (the caller hands in a zeroed grads buffer -- include/ttemb.h; the fused backward keeps the
  // C1 / C3 accumulators zero between steps, so a second handle on the same buffers, created
  // mid-training, must not and does not touch them)
  if (e != cudaSuccess) {
    fprintf(stderr, "ttemb_create: %s\n", cudaGetErrorString(e));
    delete h;
    return TTEMB_ERR_CUDA;
  }
  *out = h;
  return TTEMB_OK;
}

int ttemb_destroy(ttemb_t h) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  for (auto& p : h->c.pending) { cudaEventDestroy(p.a); cudaEventDestroy(p.b); }
  for (auto e : h->c.ev_pool) cudaEventDestroy(e);
  delete h;
  return TTEMB_OK;
}

int ttemb_core_layout(ttemb_t h, int table, int core, int64_t* offset_floats, int32_t shape[4]) {
  if (!h || table < 0 || table >= h->c.T || core < 0 || core > 2) return TTEMB_ERR_INVALID_ARG;
  const Ctx& c = h->c;
  const TableMeta& m = c.meta[table];
  int32_t s[4];
  int64_t off;
  if (m.dense) {   // hybrid: core 0 = W[M][N], cores 1, 2 empty
    off = core == 0 ? (int64_t)m.c1_off : 0;
    if (core == 0) { s[0] = (int32_t)m.M; s[1] = c.N; s[2] = 1; s[3] = 1; }
    else if (core == 1) { s[0] = 0; s[1] = c.R; s[2] = c.n2; s[3] = c.R; }
    else { s[0] = 0; s[1] = c.R; s[2] = c.n3; s[3] = 1; }
    if (offset_floats) *offset_floats = off;
    if (shape) memcpy(shape, s, sizeof(s));
    return TTEMB_OK;
  }
  if (core == 0) { off = m.c1_off; s[0] = m.m1; s[1] = c.n1; s[2] = c.R; s[3] = 1; }
  else if (core == 1) { off = m.c2_off; s[0] = m.m2; s[1] = c.R; s[2] = c.n2; s[3] = c.R; }
  else { off = m.c3_off; s[0] = m.m3; s[1] = c.R; s[2] = c.n3; s[3] = 1; }
  if (offset_floats) *offset_floats = off;
  if (shape) memcpy(shape, s, sizeof(s));
  return TTEMB_OK;
}

int ttemb_forward(ttemb_t h, const void* indices, const int64_t* offsets, int64_t nnz,
                  int32_t batch, float* out, void* stream) {
  return ttemb_forward_weighted(h, indices, offsets, nullptr, nnz, batch, out, stream);
}

int ttemb_forward_weighted(ttemb_t h, const void* indices, const int64_t* offsets,
                           const float* per_sample_weights, int64_t nnz, int32_t batch, float* out,
                           void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  if (!out && batch > 0) return TTEMB_ERR_INVALID_ARG;
  const int rc = ttemb_plan_batch(h, indices, offsets, per_sample_weights, nnz, batch, stream);
  if (rc) return rc;
  return ttemb_forward_planned(h, out, stream);
}

int ttemb_plan_batch(ttemb_t h, const void* indices, const int64_t* offsets, const float* per_sample_weights,
               int64_t nnz, int32_t batch, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (per_sample_weights && (c.flags & TTEMB_MEAN_POOLING)) return TTEMB_ERR_INVALID_ARG;
  if (nnz < 0 || batch < 0 || !offsets || (nnz > 0 && !indices)) return TTEMB_ERR_INVALID_ARG;
  if (nnz > c.max_nnz || batch > c.max_batch) return TTEMB_ERR_CAPACITY;
  if (batch == 0 && nnz != 0) return TTEMB_ERR_INVALID_ARG;
  c.psw = nnz > 0 ? per_sample_weights : nullptr;
  c.weighted = c.psw != nullptr || (c.flags & TTEMB_MEAN_POOLING) != 0;
  DeviceGuard dg(c.device);
  cudaStream_t s = (cudaStream_t)stream;
  c.nnz = nnz;
  c.B = batch;
  c.offsets = offsets;
  c.fwd_done = false;
  c.planned = false;
  cudaError_t e = run_index_stage(c, indices, offsets, s);
  if (e != cudaSuccess) {
    fprintf(stderr, "ttemb_plan_batch: %s\n", cudaGetErrorString(e));
    return TTEMB_ERR_CUDA;
  }
  c.planned = true;
  return TTEMB_OK;
}

int ttemb_forward_planned(ttemb_t h, float* out, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (!c.planned) return TTEMB_ERR_STATE;
  if (!out && c.B > 0) return TTEMB_ERR_INVALID_ARG;
  DeviceGuard dg(c.device);
  cudaError_t e = run_forward_compute(c, out, c.offsets, (cudaStream_t)stream);
  if (e != cudaSuccess) {
    fprintf(stderr, "ttemb_forward: %s\n", cudaGetErrorString(e));
    return TTEMB_ERR_CUDA;
  }
  c.planned = false;
  c.fwd_done = true;
  c.bwd_done = false;
  return TTEMB_OK;
}

int ttemb_backward(ttemb_t h, const float* grad_out, float lr, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  // one backward per forward: the plan-dependent accumulators (aggregated rows, straddling dP
  // rows) are zeroed by the index stage and consumed by the backward
  if (!c.fwd_done || c.bwd_done) return TTEMB_ERR_STATE;
  if (!grad_out && c.B > 0) return TTEMB_ERR_INVALID_ARG;
  DeviceGuard dg(c.device);
  cudaError_t e = run_backward(c, grad_out, lr, (cudaStream_t)stream);
  if (e != cudaSuccess) {
    fprintf(stderr, "ttemb_backward: %s\n", cudaGetErrorString(e));
    return TTEMB_ERR_CUDA;
  }
  c.bwd_done = true;
  return TTEMB_OK;
}

int ttemb_update(ttemb_t h, float lr, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (c.flags & TTEMB_FUSED_UPDATE) return TTEMB_ERR_STATE;
  DeviceGuard dg(c.device);
  return map_cuda(run_update(c, lr, (cudaStream_t)stream));
}

int ttemb_update_range(ttemb_t h, float lr, int64_t begin, int64_t count, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (c.flags & TTEMB_FUSED_UPDATE) return TTEMB_ERR_STATE;
  if (begin < 0 || count < 0 || (uint64_t)(begin + count) > (uint64_t)c.core_floats) return TTEMB_ERR_INVALID_ARG;
  if (count == 0) return TTEMB_OK;
  DeviceGuard dg(c.device);
  return map_cuda(run_update_range(c, lr, (size_t)begin, (size_t)count, (cudaStream_t)stream));
}

int ttemb_grad_buckets(ttemb_t h, int64_t* begin, int64_t* count, int max_buckets) {
  if (!h || max_buckets < 0 || (max_buckets > 0 && (!begin || !count))) return TTEMB_ERR_INVALID_ARG;
  const Ctx& c = h->c;
  const int64_t b[3] = {(int64_t)c.dense_begin, (int64_t)c.c3_begin, 0};
  const int64_t n[3] = {(int64_t)c.dense_floats, (int64_t)c.c3_floats, (int64_t)c.c3_begin};
  for (int i = 0; i < 3 && i < max_buckets; ++i) { begin[i] = b[i]; count[i] = n[i]; }
  return 3;
}

int ttemb_set_bucket_events(ttemb_t h, void* const* events, int n) {
  if (!h || n < 0 || n > 3 || (n > 0 && !events)) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  for (int i = 0; i < 3; ++i) c.bucket_ev[i] = i < n ? (cudaEvent_t)events[i] : nullptr;
  return TTEMB_OK;
}

int ttemb_forward_host(ttemb_t h, const void* host_indices, const int64_t* host_offsets,
                       int64_t nnz, int32_t batch, float* host_out, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (nnz < 0 || batch < 0 || !host_offsets || (nnz > 0 && !host_indices) || (!host_out && batch > 0))
    return TTEMB_ERR_INVALID_ARG;
  if (nnz > c.max_nnz || batch > c.max_batch) return TTEMB_ERR_CAPACITY;
  DeviceGuard dg(c.device);
  cudaStream_t s = (cudaStream_t)stream;
  {
    StageScope sc(c, ST_H2D, s);
    if (nnz > 0)
      cudaMemcpyAsync(c.st_idx, host_indices, (size_t)nnz * (c.index_bits / 8), cudaMemcpyHostToDevice, s);
    cudaMemcpyAsync(c.st_off, host_offsets, sizeof(int64_t) * ((size_t)c.T * batch + 1),
                    cudaMemcpyHostToDevice, s);
  }
  int rc = ttemb_forward(h, c.st_idx, c.st_off, nnz, batch, c.st_out, stream);
  if (rc) return rc;
  {
    StageScope sc(c, ST_D2H, s);
    if (batch > 0)
      cudaMemcpyAsync(host_out, c.st_out, sizeof(float) * (size_t)batch * c.T * c.N,
                      cudaMemcpyDeviceToHost, s);
  }
  return map_cuda(cudaGetLastError());
}

int ttemb_backward_host(ttemb_t h, const float* host_grad_out, float lr, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  if (!c.fwd_done || c.bwd_done) return TTEMB_ERR_STATE;
  if (!host_grad_out && c.B > 0) return TTEMB_ERR_INVALID_ARG;
  DeviceGuard dg(c.device);
  cudaStream_t s = (cudaStream_t)stream;
  {
    StageScope sc(c, ST_H2D, s);
    if (c.B > 0)
      cudaMemcpyAsync(c.st_grad, host_grad_out, sizeof(float) * (size_t)c.B * c.T * c.N,
                      cudaMemcpyHostToDevice, s);
  }
  return ttemb_backward(h, c.st_grad, lr, stream);
}

int ttemb_set_bijection(ttemb_t h, const uint32_t* bijection) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  h->c.bij = bijection;
  return TTEMB_OK;
}

uint64_t ttemb_total_rows(ttemb_t h) { return h ? h->c.total_rows : 0; }

int ttemb_check(ttemb_t h, void* stream) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  DeviceGuard dg(c.device);
  uint32_t err = 0;
  cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
  if (e == cudaSuccess) e = cudaMemcpy(&err, c.p.counts + kCntErr, sizeof(uint32_t), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    fprintf(stderr, "ttemb_check: %s\n", cudaGetErrorString(e));
    return TTEMB_ERR_CUDA;
  }
  if (err & kErrRange) return TTEMB_ERR_INDEX_RANGE;
  if (err & kErrOffsets) return TTEMB_ERR_INVALID_ARG;
  return TTEMB_OK;
}

int ttemb_get_plan(ttemb_t h, ttemb_plan* plan) {
  if (!h || !plan) return TTEMB_ERR_INVALID_ARG;
  const Ctx& c = h->c;
  if (!c.fwd_done) return TTEMB_ERR_STATE;
  const PlanDev& p = c.p;
  plan->nnz = c.nnz; plan->batch = c.B;
  plan->counts = p.counts; plan->skey = p.skey; plan->spos = p.spos; plan->bag_of = p.bag_of;
  plan->ukey = p.ukey; plan->seg_off = p.seg_off; plan->inverse = p.inverse;
  plan->row_pfx = p.row_pfx; plan->row_i3 = p.row_i3; plan->pfx_t = p.pfx_t;
  plan->pfx_i1 = p.pfx_i1; plan->pfx_i2 = p.pfx_i2; plan->row_seg = p.row_seg;
  plan->grp_pfx = p.grp_pfx; plan->grp_off = p.grp_off; plan->grp_t = p.grp_t;
  plan->grp_i2 = p.grp_i2; plan->rows = (knobs().dbg & 1024) ? p.pbuf : p.rows;   // debug: the P stash
  return TTEMB_OK;
}

int ttemb_read_counts(ttemb_t h, int64_t counts[4], void* stream) {
  if (!h || !counts) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  DeviceGuard dg(c.device);
  uint32_t v[4];
  cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
  if (e == cudaSuccess) e = cudaMemcpy(v, c.p.counts, sizeof(v), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return TTEMB_ERR_CUDA;
  for (int i = 0; i < 4; ++i) counts[i] = v[i];
  return TTEMB_OK;
}

int ttemb_set_timing(ttemb_t h, int enable) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  DeviceGuard dg(c.device);
  c.timing = enable != 0;
  if (c.timing && c.ev_pool.size() < 4096) {
    for (size_t i = c.ev_pool.size(); i < 4096; ++i) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) != cudaSuccess) return TTEMB_ERR_CUDA;
      c.ev_pool.push_back(e);
    }
  }
  return TTEMB_OK;
}

int ttemb_stage_times(ttemb_t h, double* ms, int64_t* launches, int max_stages) {
  if (!h) return TTEMB_ERR_INVALID_ARG;
  Ctx& c = h->c;
  DeviceGuard dg(c.device);
  for (auto& p : c.pending) {
    if (cudaEventSynchronize(p.b) != cudaSuccess) return TTEMB_ERR_CUDA;
    float t = 0.f;
    cudaEventElapsedTime(&t, p.a, p.b);
    c.stage_ms[p.stage] += t;
    c.stage_n[p.stage] += 1;
    c.ev_pool.push_back(p.a);
    c.ev_pool.push_back(p.b);
  }
  c.pending.clear();
  for (int i = 0; i < ST_COUNT && i < max_stages; ++i) {
    if (ms) ms[i] = c.stage_ms[i];
    if (launches) launches[i] = c.stage_n[i];
    c.stage_ms[i] = 0.0;
    c.stage_n[i] = 0;
  }
  return ST_COUNT;
}

}  // extern "C"
