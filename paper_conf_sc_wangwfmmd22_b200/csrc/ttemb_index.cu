// ttemb_index.cu -- the index stage, sm_100a.
//
//   a1 key build + range check: the group-major plan key
//        key_j = kbase_t + (i2 m1 + i1) m3 + i3     ((i1, i2, i3) = Eq. 3 digits of id_j)
//      and bag_of_j = b*T + t.  Sorting by this key puts duplicates, then rows of one prefix
//      (i1, i2) (Alg. 1's Buf_idx = idx / length_3), then prefixes of one C2 slice
//      (the i2-groups) next to each other, so one sort yields the whole plan.
//   a2 stable LSD radix sort of the 32-bit keys carrying positions (onesweep: an
//      upfront digit histogram, then one kernel per 8-bit pass with warp-level
//      match_any ranking and decoupled look-back across tiles)
//   a3 unique rows, segment offsets, inverse map (single-pass scan with warp
//      ballots and decoupled look-back) -- "compute the unique embeddings within a
//      batch"
//   a4 TT digits, unique prefixes (runs of (t, i2, i1)) and i2-groups (runs of (t, i2))
//      as two more single-pass scans, so one CTA owns each C2 slice (replaces Alg. 1's
//      flag array).
// Everything here is integer work and bit-exact against oracle/ttemb_oracle.c.
#include <algorithm>
#include <stdlib.h>

#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr uint32_t FULL = 0xffffffffu;
constexpr uint32_t kFlagAgg = 1u << 30, kFlagPfx = 2u << 30, kValMask = (1u << 30) - 1;

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
// Look-back status words carry (flag, value) in one 32-bit word, so a relaxed load sees a
// consistent pair and nothing else published by the predecessor is read: relaxed ordering
// suffices (no acquire round trips in the look-back chain).
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Decoupled look-back (one thread per status word): publish `agg` for tile `tile` in
// status[tile*stride], walk back over predecessors in windows of W independent acquire
// loads, publish the inclusive prefix, return the exclusive prefix.  When all tiles run
// concurrently the inclusive prefixes propagate ~W tiles per round trip.
template <int W>
__device__ __forceinline__ uint32_t lookback(uint32_t* status, size_t stride, uint32_t tile,
                                             uint32_t agg) {
  uint32_t* me = status + (size_t)tile * stride;
  if (tile == 0) {
    st_release(me, kFlagPfx | agg);
    return 0;
  }
  st_release(me, kFlagAgg | agg);
  uint32_t excl = 0;
  int64_t j = (int64_t)tile - 1;
  bool done = false;
  while (!done) {
    uint32_t v[W];
#pragma unroll
    for (int i = 0; i < W; ++i)
      v[i] = (j - i >= 0) ? ld_acquire(status + (size_t)(j - i) * stride) : kFlagPfx;
#pragma unroll
    for (int i = 0; i < W; ++i) {
      if (!done) {
        while ((v[i] >> 30) == 0) v[i] = ld_acquire(status + (size_t)(j - i) * stride);
        excl += v[i] & kValMask;
        if (v[i] & kFlagPfx) done = true;
      }
    }
    j -= W;
  }
  st_release(me, kFlagPfx | (excl + agg));
  return excl;
}

// Warp-wide look-back for a single status word per tile (call with the whole warp):
// each round reads 32 predecessors in parallel.
__device__ __forceinline__ uint32_t lookback_warp(uint32_t* status, uint32_t tile, uint32_t agg) {
  const int lane = threadIdx.x & 31;
  if (tile == 0) {
    if (lane == 0) st_release(status, kFlagPfx | agg);
    return 0;
  }
  if (lane == 0) st_release(status + tile, kFlagAgg | agg);
  uint32_t excl = 0;
  int64_t j = (int64_t)tile - 1;
  for (;;) {
    const int64_t idx = j - lane;
    uint32_t v = idx >= 0 ? ld_acquire(status + idx) : kFlagPfx;
    while (__any_sync(FULL, (v >> 30) == 0)) {
      if ((v >> 30) == 0) v = ld_acquire(status + idx);
    }
    const uint32_t pfx = __ballot_sync(FULL, (v & kFlagPfx) != 0);
    const int stop = pfx ? __ffs(pfx) - 1 : 31;          // nearest inclusive prefix
    uint32_t x = lane <= stop ? (v & kValMask) : 0u;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(FULL, x, o);
    excl += x;
    if (pfx) break;
    j -= 32;
  }
  if (lane == 0) st_release(status + tile, kFlagPfx | (excl + agg));
  return excl;
}

// Exclusive scan of one value per thread over a 256-thread block.
__device__ __forceinline__ uint32_t block_excl_scan_256(uint32_t v, uint32_t* s_warp,
                                                        uint32_t& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_warp[w] = x;
  __syncthreads();
  if (w == 0) {
    uint32_t s = lane < 8 ? s_warp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, s, o);
      if (lane >= o) s += y;
    }
    if (lane < 8) s_warp[lane] = s;
  }
  __syncthreads();
  total = s_warp[7];
  const uint32_t wpre = w ? s_warp[w - 1] : 0;
  return wpre + x - v;
}

// ------------------------------------------------------------------------------------
// a1: keys
// ------------------------------------------------------------------------------------
// Bag-parallel: thread per bag writes the keys / bag ids of its positions and counts the
// radix digits of every pass (the sort's upfront histogram, fused here).  keys / bag_of
// are zeroed beforehand so malformed offsets (flagged) leave only in-range values.
template <typename IdxT>
__global__ void __launch_bounds__(256)
k_build_keys(const IdxT* __restrict__ indices, const int64_t* __restrict__ offsets, int64_t nnz,
             int32_t B, int T, const TableMeta* __restrict__ meta, uint32_t* __restrict__ keys,
             uint32_t* __restrict__ bag_of, uint32_t* __restrict__ counts, int passes,
             uint32_t* __restrict__ hist, const uint32_t* __restrict__ bij,
             const float* __restrict__ psw, int mean, float* __restrict__ wpos) {
  __shared__ uint32_t sh[4][256];
  for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) (&sh[0][0])[i] = 0;
  __syncthreads();
  const int64_t nbags = (int64_t)T * B;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int lane = threadIdx.x & 31;
  uint32_t err = 0, multi = 0;
  // whole warps iterate together (the digit histogram below is warp-aggregated)
  for (int64_t b0 = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); b0 < nbags; b0 += stride) {
    const int64_t b = b0 + lane;
    const bool bval = b < nbags;
    int64_t s = bval ? __ldg(offsets + b) : 0, e = bval ? __ldg(offsets + b + 1) : 0;
    if (s < 0 || e > nnz || e < s) { err |= kErrOffsets; s = 0; e = 0; }
    if (b == 0 && s != 0) err |= kErrOffsets;
    if (b == nbags - 1 && e != nnz) err |= kErrOffsets;
    if (bval && e - s != 1) multi = 1u;
    const int t = bval ? (int)(b / B) : 0;
    const int64_t bb = b - (int64_t)t * B;
    const TableMeta& mt = meta[t];
    const uint32_t kb = (uint32_t)mt.kbase, M = mt.M, m1 = mt.m1, m2 = mt.m2, m3 = mt.m3;
    const uint32_t bo = (uint32_t)(bb * T + t);
    const uint32_t* bt = bij ? bij + mt.rowbase : nullptr;   // table t's bijection
    const float wmean = e > s ? 1.0f / (float)(e - s) : 0.f; // nn.EmbeddingBag mode="mean"
    const int64_t len = e - s;
    int64_t rounds = len;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) rounds = max(rounds, __shfl_xor_sync(0xffffffffu, rounds, o));
    for (int64_t r = 0; r < rounds; ++r) {
      const int64_t j = s + r;
      const bool act = r < len;
      uint32_t key = 0xFFFFFFFFu;
      if (act) {
      const int64_t id = (int64_t)indices[j];
      key = kb;
      if (id < 0 || (uint64_t)id >= M) err |= kErrRange;
      else {
        const uint32_t r = bt ? __ldg(bt + id) : (uint32_t)id;   // New_Batch = {index(i_j)}
        if (r >= M) {
          err |= kErrRange;
        } else if (mt.dense) {                  // hybrid: plain table, key = row id
          key = kb + r;
        } else {
          const uint32_t p = r / m3, i3 = r - p * m3, i1 = p / m2, i2 = p - i1 * m2;
          key = kb + (i2 * m1 + i1) * m3 + i3;
        }
      }
      keys[j] = key;
      bag_of[j] = bo;
      if (wpos) wpos[j] = psw ? __ldg(psw + j) : wmean;
      }
      // digit histograms: one shared-memory atomic per distinct digit per warp (Zipf-hot keys
      // share their high digits, so per-key atomics would serialise)
      for (int p = 0; p < passes; ++p) {
        const uint32_t d = act ? ((key >> (8 * p)) & 255u) : 256u;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        if (d < 256 && (__ffs(peers) - 1) == lane) atomicAdd(&sh[p][d], __popc(peers));
      }
    }
  }
  if (nbags == 0 && nnz != 0 && blockIdx.x == 0 && threadIdx.x == 0) err |= kErrOffsets;
  if (err) atomicOr(counts + kCntErr, err);
  if (multi) atomicOr(counts + kCntMulti, 1u);
  __syncthreads();
  for (int i = threadIdx.x; i < passes * 256; i += blockDim.x) {
    const uint32_t v = (&sh[0][0])[i];
    if (v) atomicAdd(hist + i, v);
  }
}

// ------------------------------------------------------------------------------------
// a2: onesweep LSD radix sort, 8-bit digits
#ifndef TTEMB_KEYS_PER_SM
#define TTEMB_KEYS_PER_SM 4   // k_build_keys grid cap, CTAs per SM
#endif
#ifndef TTEMB_RS_IPT
#define TTEMB_RS_IPT 8    // keys per thread (tile = 256 x RS_IPT; 8 beats 16 and 4 at C4)
#endif
// ------------------------------------------------------------------------------------
constexpr int RS_T = 256, RS_IPT = TTEMB_RS_IPT, RS_WARPS = RS_T / 32, RS_TILE = RS_T * RS_IPT;

// Digit histograms of all passes in one read of the keys.
__global__ void __launch_bounds__(256)
k_radix_hist(const uint32_t* __restrict__ keys, const uint32_t* n_dev, uint32_t n_static,
             int passes, uint32_t* __restrict__ hist) {
  __shared__ uint32_t sh[4][256];
  for (int i = threadIdx.x; i < 4 * 256; i += blockDim.x) (&sh[0][0])[i] = 0;
  __syncthreads();
  const uint32_t n = n_dev ? *n_dev : n_static;
  const int lane = threadIdx.x & 31;
  for (uint32_t base = blockIdx.x * blockDim.x; base < n; base += gridDim.x * blockDim.x) {
    const uint32_t i = base + threadIdx.x;
    const bool ok = i < n;
    const uint32_t k = ok ? keys[i] : 0u;
    for (int p = 0; p < passes; ++p) {
      const uint32_t d = ok ? ((k >> (8 * p)) & 255u) : 256u;
      const uint32_t peers = __match_any_sync(FULL, d);      // warp-aggregated increments
      if (d < 256 && (__ffs(peers) - 1) == lane) atomicAdd(&sh[p][d], __popc(peers));
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < passes * 256; i += blockDim.x) {
    const uint32_t v = (&sh[0][0])[i];
    if (v) atomicAdd(hist + i, v);
  }
}

__global__ void __launch_bounds__(256)
k_hist_scan(const uint32_t* __restrict__ hist, uint32_t* __restrict__ dbase, int passes) {
  __shared__ uint32_t s_warp[8];
  for (int p = 0; p < passes; ++p) {
    uint32_t tot;
    const uint32_t e = block_excl_scan_256(hist[p * 256 + threadIdx.x], s_warp, tot);
    dbase[p * 256 + threadIdx.x] = e;
    __syncthreads();
  }
}

__global__ void __launch_bounds__(RS_T)
k_radix_pass(const uint32_t* __restrict__ kin, const uint32_t* __restrict__ vin,
             uint32_t* __restrict__ kout, uint32_t* __restrict__ vout, const uint32_t* n_dev,
             uint32_t n_static, int shift, const uint32_t* __restrict__ dbase,
             uint32_t* status, uint32_t* counter) {
  __shared__ uint32_t s_wc[RS_WARPS][256];
  __shared__ uint32_t s_k[RS_TILE];
  __shared__ uint32_t s_v[RS_TILE];
  __shared__ uint32_t s_bstart[256], s_gbase[256], s_warp[8], s_tile;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(counter, 1u);
  for (int i = tid; i < RS_WARPS * 256; i += RS_T) (&s_wc[0][0])[i] = 0;
  __syncthreads();
  const uint32_t n = n_dev ? *n_dev : n_static;
  const uint32_t tile = s_tile;
  const uint32_t base = tile * RS_TILE;
  if (base >= n) return;

  uint32_t key[RS_IPT], val[RS_IPT], rank[RS_IPT];
  uint32_t dig[RS_IPT];
#pragma unroll
  for (int k = 0; k < RS_IPT; ++k) {
    const uint32_t i = base + w * 32 * RS_IPT + k * 32 + lane;
    const bool ok = i < n;
    key[k] = ok ? kin[i] : 0u;
    val[k] = ok ? (vin ? vin[i] : i) : 0u;
    dig[k] = ok ? ((key[k] >> shift) & 255u) : 256u;
  }
  // warp-level stable ranking: items in (k, lane) order == element order
#pragma unroll
  for (int k = 0; k < RS_IPT; ++k) {
    const uint32_t d = dig[k];
    const uint32_t peers = __match_any_sync(FULL, d);
    const uint32_t lt = __popc(peers & lanemask_lt());
    uint32_t c = 0;
    if (d < 256) c = s_wc[w][d];
    __syncwarp();
    if (d < 256 && lt == 0) s_wc[w][d] = c + __popc(peers);
    __syncwarp();
    rank[k] = c + lt;
  }
  __syncthreads();
  // per digit: exclusive offsets over warps, tile count
  uint32_t run = 0;
#pragma unroll
  for (int ww = 0; ww < RS_WARPS; ++ww) {
    const uint32_t c = s_wc[ww][tid];
    s_wc[ww][tid] = run;
    run += c;
  }
  uint32_t tot;
  const uint32_t bstart = block_excl_scan_256(run, s_warp, tot);
  s_bstart[tid] = bstart;
  const uint32_t excl = lookback<16>(status + tid, 256, tile, run);
  s_gbase[tid] = dbase[tid] + excl;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < RS_IPT; ++k) {
    const uint32_t d = dig[k];
    if (d < 256) {
      const uint32_t pos = s_bstart[d] + s_wc[w][d] + rank[k];
      s_k[pos] = key[k];
      s_v[pos] = val[k];
    }
  }
  __syncthreads();
  const uint32_t cnt = min((uint32_t)RS_TILE, n - base);
  for (uint32_t i = tid; i < cnt; i += RS_T) {
    const uint32_t k = s_k[i];
    const uint32_t d = (k >> shift) & 255u;
    const uint32_t o = s_gbase[d] + i - s_bstart[d];
    kout[o] = k;
    vout[o] = s_v[i];
  }
}

// ------------------------------------------------------------------------------------
// Plan scan tiles: 256 threads x 8 occurrences (SC_IPT * 8 == 64 warp counts).
// ------------------------------------------------------------------------------------
constexpr int SC_T = 256, SC_IPT = 8, SC_TILE = SC_T * SC_IPT;   // SC_IPT * 8 == 64 warp counts

// a3 + a4 in ONE pass over the sorted occurrences: position k starts a unique row (key change), a unique prefix (change of (t, i2 m1 + i1)
// on a TT row) and an i2-group (change of (t, i2)).  Three flag ballots, three warp-count
// scans and three decoupled look-backs (warps 0-2 in parallel) give every position its row
// slot u, prefix slot q and group slot g; the emits write the same arrays the three scans did.
struct PlanScanArgs {
  const uint32_t *skey, *spos, *bag_of;
  const uint64_t* kbase; const uint32_t* kmap; const TableMeta* meta; int T;
  uint32_t *ukey, *seg_off, *inverse, *sbag, *counts;
  uint32_t *row_pfx, *row_i3, *pfx_t, *pfx_i1, *pfx_i2, *row_seg;
  uint32_t *grp_pfx, *grp_off, *grp_t, *grp_i2;
  uint32_t* row_c3;                 // [U] C3 slice index of the row (row kernels: one load per row)
  uint64_t c3_begin, s3;            // C3 region start, floats per C3 slice (R n3)
  uint32_t nnz, every_row, every_pfx;
  uint64_t tt_keys;
};

struct KeyInfo { uint32_t t, pq, i3, dense; };

__device__ __forceinline__ KeyInfo decode_key(const PlanScanArgs& a, uint32_t key) {
  KeyInfo r;
  const int it = table_of_key(a.kbase, a.T, key);
  r.t = __ldg(a.kmap + it);
  const uint32_t local = (uint32_t)(key - __ldg(a.kbase + it));
  r.dense = key >= a.tt_keys ? 1u : 0u;
  const uint32_t m3 = r.dense ? 1u : a.meta[r.t].m3;
  r.pq = local / m3;
  r.i3 = local - r.pq * m3;
  return r;
}

__global__ void __launch_bounds__(SC_T) k_plan_scan(PlanScanArgs a, uint32_t* status, uint32_t* counter) {
  __shared__ uint32_t s_wc[3][SC_IPT * 8];
  __shared__ uint32_t s_tile, s_base[3], s_total[3];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(counter, 1u);
  __syncthreads();
  const uint32_t n = a.nnz;
  const uint32_t tile = s_tile, base = tile * SC_TILE;
  if (n == 0) {
    if (tile == 0 && tid == 0) {
      a.counts[kCntU] = 0; a.seg_off[0] = 0; a.counts[kCntP] = 0; a.row_seg[0] = 0;
      a.counts[kCntNG] = 0; a.grp_off[0] = 0;
    }
    return;
  }
  if (base >= n) return;
  uint32_t bal[3][SC_IPT];
  KeyInfo ki[SC_IPT];
#pragma unroll
  for (int k = 0; k < SC_IPT; ++k) {
    const uint32_t i = base + k * SC_T + tid;
    bool fr = false, fp = false, fg = false;
    ki[k] = KeyInfo{0, 0, 0, 1};
    if (i < n) {
      const uint32_t key = a.skey[i];
      const bool newkey = i == 0 || a.skey[i - 1] != key;
      fr = a.every_row || newkey;
      ki[k].dense = key >= a.tt_keys ? 1u : 0u;
      if (fr) ki[k] = decode_key(a, key);          // digits are needed at row starts only
      if (fr && !ki[k].dense) {
        if (i == 0) {
          fp = fg = true;
        } else {
          const KeyInfo pv = newkey ? decode_key(a, a.skey[i - 1]) : ki[k];
          const bool newgrp = pv.dense || pv.t != ki[k].t || pv.pq / a.meta[pv.t].m1 != ki[k].pq / a.meta[ki[k].t].m1;
          fp = a.every_pfx || newgrp || pv.pq != ki[k].pq;
          fg = newgrp;
        }
      }
    }
    bal[0][k] = __ballot_sync(FULL, fr);
    bal[1][k] = __ballot_sync(FULL, fp);
    bal[2][k] = __ballot_sync(FULL, fg);
    if (lane == 0) {
      s_wc[0][k * 8 + w] = __popc(bal[0][k]);
      s_wc[1][k * 8 + w] = __popc(bal[1][k]);
      s_wc[2][k * 8 + w] = __popc(bal[2][k]);
    }
  }
  __syncthreads();
  if (w < 3) {   // exclusive scan of the 64 warp counts (k-major) of flag w, then its look-back
    const uint32_t x0 = s_wc[w][2 * lane], x1 = s_wc[w][2 * lane + 1];
    uint32_t x = x0 + x1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    const uint32_t ex = x - x0 - x1;
    s_wc[w][2 * lane] = ex;
    s_wc[w][2 * lane + 1] = ex + x0;
    const uint32_t tot = __shfl_sync(FULL, x, 31);
    const uint32_t b = lookback_warp(status + (size_t)w * gridDim.x, tile, tot);
    if (lane == 0) { s_base[w] = b; s_total[w] = tot; }
  }
  __syncthreads();
  const uint32_t lt = lanemask_lt();
#pragma unroll
  for (int k = 0; k < SC_IPT; ++k) {
    const uint32_t i = base + k * SC_T + tid;
    if (i >= n) continue;
    // inclusive counts - 1 = this position's row / prefix / group slot
    const uint32_t u = s_base[0] + s_wc[0][k * 8 + w] + __popc(bal[0][k] & lt) + ((bal[0][k] >> lane) & 1u) - 1u;
    const uint32_t q = s_base[1] + s_wc[1][k * 8 + w] + __popc(bal[1][k] & lt) + ((bal[1][k] >> lane) & 1u) - 1u;
    const uint32_t g = s_base[2] + s_wc[2][k * 8 + w] + __popc(bal[2][k] & lt) + ((bal[2][k] >> lane) & 1u) - 1u;
    const uint32_t pos = a.spos[i];
    a.inverse[pos] = u;
    a.sbag[i] = __ldg(a.bag_of + pos);
    if ((bal[0][k] >> lane) & 1u) {
      const uint32_t key = a.skey[i];
      a.ukey[u] = key;
      a.seg_off[u] = i;
      if (ki[k].dense) {
        a.row_pfx[u] = 0xFFFFFFFFu;
        a.row_i3[u] = 0;
        a.row_c3[u] = 0;
        if (i == 0 || a.skey[i - 1] < a.tt_keys) {   // first dense row: TT rows / prefixes end here
          a.counts[kCntUtt1] = u + 1;
          a.row_seg[q + 1] = u;
        }
      } else {
        a.row_pfx[u] = q;
        a.row_i3[u] = ki[k].i3;
        a.row_c3[u] = (uint32_t)((a.meta[ki[k].t].c3_off - a.c3_begin) / a.s3) + ki[k].i3;
      }
    }
    if ((bal[1][k] >> lane) & 1u) {
      const uint32_t m1 = a.meta[ki[k].t].m1;
      const uint32_t i2 = ki[k].pq / m1;
      a.pfx_t[q] = ki[k].t; a.pfx_i1[q] = ki[k].pq - i2 * m1; a.pfx_i2[q] = i2;
      a.row_seg[q] = u;
      a.grp_pfx[q] = q;
      if ((bal[2][k] >> lane) & 1u) { a.grp_off[g] = q; a.grp_t[g] = ki[k].t; a.grp_i2[g] = i2; }
    }
  }
  if (base + SC_TILE >= n && tid == 0) {
    const uint32_t U = s_base[0] + s_total[0], P = s_base[1] + s_total[1], NG = s_base[2] + s_total[2];
    a.counts[kCntU] = U; a.seg_off[U] = n;
    a.counts[kCntP] = P; a.counts[kCntNG] = NG; a.grp_off[NG] = P;
    if (a.skey[n - 1] < a.tt_keys) a.row_seg[P] = U;   // no dense rows (else written above)
  }
}

// Host: full LSD sort; returns which buffer pair holds the result (0 = A, 1 = B).
int radix_sort(Ctx& c, uint32_t* kA, uint32_t* vA, uint32_t* kB, uint32_t* vB,
               const uint32_t* n_dev, uint32_t n_static, int64_t n_max, int passes,
               uint32_t* hist, uint32_t* dbase, uint32_t* counters, uint32_t* status,
               int64_t tiles, int st_hist, int st_pass, cudaStream_t s, bool have_hist = false) {
  {
    StageScope sc(c, st_hist, s);
    if (!have_hist)
      k_radix_hist<<<grid_for(c, n_max, 256, 4), 256, 0, s>>>(kA, n_dev, n_static, passes, hist);
    k_hist_scan<<<1, 256, 0, s>>>(hist, dbase, passes);
  }
  uint32_t *ki = kA, *vi = vA, *ko = kB, *vo = vB;
  const int64_t grid = tiles > 0 ? tiles : 1;
  for (int p = 0; p < passes; ++p) {
    StageScope sc(c, st_pass, s);
    k_radix_pass<<<(unsigned)grid, RS_T, 0, s>>>(ki, p == 0 ? nullptr : vi, ko, vo, n_dev, n_static,
                                                  8 * p, dbase + 256 * p,
                                                  status + (size_t)p * tiles * 256, counters + p);
    uint32_t* t;
    t = ki; ki = ko; ko = t;
    t = vi; vi = vo; vo = t;
  }
  return (passes & 1) ? 1 : 0;
}

}  // namespace

int64_t radix_tiles(int64_t n) { return cdiv(n, RS_TILE); }
int64_t scan_tiles(int64_t n) { return cdiv(n, SC_TILE); }

cudaError_t run_index_stage(Ctx& c, const void* indices, const int64_t* offsets, cudaStream_t s) {
  PlanDev& p = c.p;
  const int64_t nnz = c.nnz;
  {
    StageScope sc(c, ST_ZERO, s);
    cudaMemsetAsync(c.zero_begin, 0, c.zero_bytes, s);
  }
  {
    StageScope sc(c, ST_KEYS, s);
    if (nnz > 0) {
      cudaMemsetAsync(p.keysA, 0, sizeof(uint32_t) * nnz, s);
      cudaMemsetAsync(p.bag_of, 0, sizeof(uint32_t) * nnz, s);
    }
    const int64_t bags = (int64_t)c.T * c.B;
    // fewer CTAs than bags (grid-stride): each CTA flushes up to passes x 256 histogram atomics
    const int g = grid_for(c, bags > 0 ? bags : 1, 256, TTEMB_KEYS_PER_SM);
    if (c.index_bits == 64)
      k_build_keys<int64_t><<<g, 256, 0, s>>>((const int64_t*)indices, offsets, nnz, c.B, c.T,
                                              c.d_meta, p.keysA, p.bag_of, p.counts,
                                              c.key_passes, p.hist1, c.bij, c.psw,
                                              (c.flags & TTEMB_MEAN_POOLING) ? 1 : 0,
                                              c.weighted ? p.wpos : nullptr);
    else
      k_build_keys<int32_t><<<g, 256, 0, s>>>((const int32_t*)indices, offsets, nnz, c.B, c.T,
                                              c.d_meta, p.keysA, p.bag_of, p.counts,
                                              c.key_passes, p.hist1, c.bij, c.psw,
                                              (c.flags & TTEMB_MEAN_POOLING) ? 1 : 0,
                                              c.weighted ? p.wpos : nullptr);
  }
  // a2: sort (key, position)
  const int64_t tiles1 = radix_tiles(nnz);
  const int which = radix_sort(c, p.keysA, p.valsA, p.keysB, p.valsB, nullptr, (uint32_t)nnz, nnz,
                               c.key_passes, p.hist1, p.dbase1, p.rs1_counter, p.rs1_status, tiles1,
                               ST_SORT_HIST, ST_SORT_PASS, s, /*have_hist=*/true);
  p.skey = which ? p.keysB : p.keysA;
  p.spos = which ? p.valsB : p.valsA;
  {   // a3 + a4 in one scan
    StageScope sc(c, ST_UNIQUE, s);
    PlanScanArgs a;
    a.skey = p.skey; a.spos = p.spos; a.bag_of = p.bag_of; a.kbase = c.d_kbase; a.kmap = c.d_kmap;
    a.meta = c.d_meta; a.T = c.T; a.ukey = p.ukey; a.seg_off = p.seg_off; a.inverse = p.inverse;
    a.sbag = p.sbag; a.counts = p.counts; a.row_pfx = p.row_pfx; a.row_i3 = p.row_i3; a.pfx_t = p.pfx_t;
    a.pfx_i1 = p.pfx_i1; a.pfx_i2 = p.pfx_i2; a.row_seg = p.row_seg; a.grp_pfx = p.grp_pfx;
    a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2; a.nnz = (uint32_t)nnz;
    a.every_row = (c.flags & TTEMB_NO_AGGREGATION) ? 1u : 0u;
    a.every_pfx = (c.flags & TTEMB_NO_PREFIX_REUSE) ? 1u : 0u;
    a.tt_keys = c.tt_keys;
    a.row_c3 = p.row_c3; a.c3_begin = c.c3_begin; a.s3 = (uint64_t)c.R * c.n3;
    const int64_t tiles = std::max<int64_t>(1, scan_tiles(nnz));
    k_plan_scan<<<(unsigned)tiles, SC_T, 0, s>>>(a, p.sc_status, p.sc_counter + 0);
  }
  return run_plan_tail(c, s);
}

}  // namespace ttemb
