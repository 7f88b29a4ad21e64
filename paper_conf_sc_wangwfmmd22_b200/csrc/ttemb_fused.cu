// ttemb_fused.cu -- fused forward contraction kernel (SURVEY 8(a) rows a5 + a6), sm_100a.
//
// One persistent CTA per SM walks the i2-groups g = (t, i2) (dynamic claim).  Per group:
//   a5  P^T[c][m] = sum_r1 C2[i2][r1][c] . C1[i1_m][j1_m][r1]     (Reuse buffer)
//       on tcgen05 kind::tf32, 3xTF32 split, with the C2 slice held TRANSPOSED IN TENSOR
//       MEMORY as the A operand (lane = c, column = r1; scripts/tc_probe3.cu) and the group's
//       C1 rows (m = (prefix, j1)) as the K-major B operand in shared memory.  M = 128 c per
//       block, N = tile rows (<= 64), K = R = 64.
//   a6  E_u = P_q (n1 n2 x R) . C3[i3_u] (R x n3)  (Eq. 2, Fig. 5(b) step 3) on FFMA:
//       the accumulator is drained TMEM -> shared memory (P_s[m][c]) and the group's unique
//       rows are split evenly over the row warps (Zipf-hot prefixes spread over all warps).
// The C2 slice streams HBM -> shared memory (bulk copy, one group ahead) -> registers (one
// more group ahead) -> TMEM, so two groups' loads are always in flight.
//
// Warp roles (544 threads):  0-7 loaders (C2 column c = thread, C1 rows -> B),  8 MMA issuer,
// 9-16 row warps (TMEM drain of one c-block quarter each, then the row contraction).
// Pipelines (mbarriers): raw (bulk copy), A (TMEM C2, per group), B[2] (C1 rows, per tile),
// D[2] (TMEM accumulators, per tile), unit ring[4] (tile descriptors for MMA + row warps).
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <type_traits>
#include <vector>

#include "tc.cuh"
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int XT = 64;                         // tile rows (prefix, j1) = MMA N (max)
constexpr int X_LW = 8, X_RW = 4;   // loaders, epilogue warps
constexpr int X_THREADS = (X_LW + 1 + X_RW) * 32;
constexpr int X_MMA_W = X_LW, X_ROW_W0 = X_LW + 1;
constexpr uint32_t X_RAW_BYTES = 65536;        // R x NC fp32, NC <= 256

struct XArgs {
  float* cores;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_i1, *pfx_t, *row_seg, *row_i3, *row_pfx;
  uint32_t* grp_arow;                 // [P]  C1 row index (floats / R) of sorted prefix q, j1 = 0
  const uint32_t* unit_sorted;        // [NU] work units, largest first (claim k -> unit_sorted[k])
  unsigned long long* grp_c2;         // [NG] float offset of group g's C2 slice
  float* rows;                        // [U][N]
  float* pbuf;                        // [P][n1][NC] (consumed by the backward row stage)
  uint32_t* work;
  int dbg;                            // TTEMB_DBG bit mask (timing experiments only; results invalid)
  unsigned long long* trace;          // optional per-CTA role timers (TTEMB_TRACE): 32 slots per CTA
  int n1, n1s, n2, n3, N, NC, nblk, tpp, R;
};

// TTEMB_TRACE instrumentation: clock64 intervals accumulated per role leader.
#define XT0() long long _tt = a.trace ? clock64() : 0
#define XTA(k)                                           \
  do {                                                   \
    if (a.trace) {                                       \
      const long long _n = clock64();                    \
      trc[k] += (unsigned long long)(_n - _tt);          \
      _tt = _n;                                          \
    }                                                    \
  } while (0)

struct XCtl {
  uint64_t raw_full, a_full, a_free;
  uint64_t b_full[2], b_free[2], d_full[2], d_free[2];
  uint64_t u_full[4], u_empty[4];
  uint32_t ring[4][8];                // group, first prefix, #prefixes, flags (1 first, 2 last, 4 done), unit block
  uint32_t claim[2];
  uint32_t tmem;
};

__global__ void k_fused_prep(XArgs a) {
  pdl_wait();
  const uint32_t P = a.counts[kCntP], NG = a.counts[kCntNG];
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < max(P, NG); q += gridDim.x * blockDim.x) {
    if (q < P) {
      const uint32_t p = a.grp_pfx[q];
      a.grp_arow[q] = (uint32_t)(a.meta[a.pfx_t[p]].c1_off / a.R) + (a.pfx_i1[p] << a.n1s);
    }
    if (q < NG) a.grp_c2[q] = a.meta[a.grp_t[q]].c2_off + (unsigned long long)a.grp_i2[q] * a.R * a.NC;
  }
}

__device__ __forceinline__ float tf32_lo(float x) { return x - tc::tf32_trunc(x); }

// Work unit = (i2-group, c-range of BPU 128-wide c-blocks): at R = 64 one unit covers the group's
// whole C2 slice (C2^T of both c-blocks fills TMEM columns [0, 256)); at R = 128 (K = 128) one
// c-block's C2^T hi + lo already takes 256 columns, so a group is split into NC / 128 units and
// the C1 rows of a tile are staged once per unit.
template <int KR, int NC_T>   // NC_T = n2 R when fixed at compile time (immediate store offsets), else 0
__global__ void __launch_bounds__(X_THREADS, 1) k_prefix_fwd(XArgs a) {
  pdl_wait();
  pdl_trigger();
  const int NCT = NC_T ? NC_T : a.NC;
  constexpr int BPU = KR <= 64 ? 2 : 1;            // c-blocks per work unit
  constexpr uint32_t BSLOT = 2u * XT * KR * 4;    // one B slot: C1 tile hi + lo (K = KR)
  constexpr uint32_t BHALF = XT * KR * 4;
  extern __shared__ __align__(128) char smem_raw[];
  __shared__ XCtl ctl;
  char* const smem = smem_raw + ((128u - (tc::smem_u32(smem_raw) & 127u)) & 127u);
  float* const raw = reinterpret_cast<float*>(smem);
  char* const bbuf = smem + X_RAW_BYTES;
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const uint32_t NG = a.counts[kCntNG];
  const uint32_t UPG = (uint32_t)(a.nblk + BPU - 1) / BPU;   // units per group
  const uint32_t NU = NG * UPG;
  // raw staging: R = 64 the whole C2 slice [KR][NC] (contiguous); R = 128 the unit's block,
  // KR rows of 128 columns (row stride RS)
  const int RS = BPU == 2 ? a.NC : 128;
  if (tid == 0) {
    tc::mbar_init(&ctl.raw_full, 1);
    tc::mbar_init(&ctl.a_full, X_LW * 32);
    tc::mbar_init(&ctl.a_free, 1);
    for (int s = 0; s < 2; ++s) {
      tc::mbar_init(&ctl.b_full[s], X_LW * 32);
      tc::mbar_init(&ctl.b_free[s], 1);
      tc::mbar_init(&ctl.d_full[s], 1);
      tc::mbar_init(&ctl.d_free[s], X_RW * 32);
    }
    for (int s = 0; s < 4; ++s) { tc::mbar_init(&ctl.u_full[s], 1); tc::mbar_init(&ctl.u_empty[s], 1 + X_RW); }
    tc::fence_mbar_init();
  }
  if (w == X_MMA_W) tc::tmem_alloc(&ctl.tmem, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = ctl.tmem;
  // TMEM columns: [0,128) C2^T hi (KR per c-block), [128,256) lo, [256,512) D[2] (128 each:
  // 64 per c-block).
  const int tpp = a.tpp;
  unsigned long long trc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  const long long t_start = a.trace ? clock64() : 0;
  const unsigned long long g_start = a.trace ? tc::globaltimer_ns() : 0;

  if (w < X_LW) {
    // ------------------------------- loaders -------------------------------
    // thread = C2^T row (column c of the slice) x 64 r1 values: R = 64 warps 0-3 / 4-7 take the
    // two c-blocks, R = 128 they take r1 [0, 64) / [64, 128) of the unit's block
    const int wb = w >> 2, Q = w & 3;
    const int blk = BPU == 2 ? wb : 0, r0 = BPU == 2 ? 0 : 64 * wb;
    const int cl = blk * 128 + Q * 32 + lane;      // column inside the staged raw block
    float xa[32], xb[32];
    uint32_t ui = 0, gs = 0, rawk = 0;
    bool cval = false;
    auto col_valid = [&](uint32_t u) { return ((int)(u % UPG) * BPU * 128 + cl) < a.NC; };
    auto load_raw = [&]() {          // regs <- raw (this thread's column, 64 r1)
#pragma unroll
      for (int r = 0; r < 32; ++r) {
        xa[r] = cval ? raw[(r0 + r) * RS + cl] : 0.f;
        xb[r] = (cval && KR > 32) ? raw[(r0 + r + 32) * RS + cl] : 0.f;
      }
    };
    auto issue_raw = [&](uint32_t u) {   // thread 0: the unit's C2 columns -> raw
      const uint32_t g = u / UPG, ub = u % UPG;
      const float* src = a.cores + a.grp_c2[g];
      if (BPU == 2) {
        const uint32_t bytes = (uint32_t)KR * a.NC * 4u;
        tc::mbar_arrive_tx(&ctl.raw_full, bytes);
        tc::bulk_g2s(tc::smem_u32(raw), src, bytes, &ctl.raw_full);
      } else {
        const int c0 = (int)ub * 128, nc = min(128, a.NC - c0);
        tc::mbar_arrive_tx(&ctl.raw_full, (uint32_t)(KR * nc * 4));
        for (int r = 0; r < KR; ++r)
          tc::bulk_g2s(tc::smem_u32(raw + r * 128), src + (size_t)r * a.NC + c0, (uint32_t)(nc * 4), &ctl.raw_full);
      }
    };
    // thread 0: the next unit in group order (claiming the largest-first order of unit_sorted
    // instead measured 1.5 us slower at c4: TTEMB_DBG bit 64 selects it for comparison)
    auto claim = [&]() {
      const uint32_t k = atomicAdd(a.work, 1u);
      return k < NU ? ((a.dbg & 64) ? a.unit_sorted[k] : k) : NU;
    };
    if (tid == 0) {
      ctl.claim[0] = claim();
      ctl.claim[1] = claim();
      if (ctl.claim[0] < NU) issue_raw(ctl.claim[0]);
    }
    tc::named_sync(1, X_LW * 32);
    uint32_t cur = ctl.claim[0], nxt = ctl.claim[1];
    if (cur < NU) {
      tc::mbar_wait(&ctl.raw_full, rawk & 1);
      ++rawk;
      cval = col_valid(cur);
      load_raw();
    }
    tc::named_sync(1, X_LW * 32);
    if (tid == 0 && nxt < NU) issue_raw(nxt);
    // The C1 row of this thread's B row in the NEXT tile (its grp_arow entry, loaded one tile ahead)
    // is prefetched into L1 at the end of the current tile, and the next unit's group bounds are
    // loaded one unit ahead, so a tile's C1 loads neither wait on grp_arow nor on DRAM.
    const int m = tid & 63;
    const uint32_t jm = (uint32_t)(m & ((1 << a.n1s) - 1));
    auto arow_of = [&](uint32_t qa, uint32_t q1) {   // C1 row of B row m of the tile at qa, or ~0
      const uint32_t np = qa < q1 ? min((uint32_t)tpp, q1 - qa) : 0u;
      return m < (int)(np << a.n1s) ? a.grp_arow[qa + (m >> a.n1s)] + jm : 0xffffffffu;
    };
    uint32_t q0n = 0, q1n = 0;
    if (nxt < NU) { q0n = a.grp_off[nxt / UPG]; q1n = a.grp_off[nxt / UPG + 1]; }
    uint32_t q0 = 0, q1 = 0;
    if (cur < NU) { q0 = a.grp_off[cur / UPG]; q1 = a.grp_off[cur / UPG + 1]; }
    uint32_t arow_n = arow_of(q0, q1);
    while (cur < NU) {
      const uint32_t g = cur / UPG, ub = cur % UPG;
      for (uint32_t qa = q0; qa < q1; qa += tpp, ++ui) {
        const uint32_t np = min((uint32_t)tpp, q1 - qa);
        const int rows = (int)np << a.n1s;
        const uint32_t fl = (qa == q0 ? 1u : 0u) | (qa + tpp >= q1 ? 2u : 0u);
        XT0();
        if (tid == 0) {
          tc::mbar_wait(&ctl.u_empty[ui & 3], ((ui >> 2) & 1) ^ 1);
          ctl.ring[ui & 3][0] = g; ctl.ring[ui & 3][1] = qa; ctl.ring[ui & 3][2] = np; ctl.ring[ui & 3][3] = fl;
          ctl.ring[ui & 3][4] = ub;
          tc::mbar_arrive(&ctl.u_full[ui & 3]);
        }
        // C1 rows of the tile -> registers (B = CM(m, r1), m = tid & 63, KR / 16 float4 of r1)
        float4 bv[KR / 16];
        {
          const uint32_t arow = arow_n;
          const bool ok = arow != 0xffffffffu;
          const float4* src = reinterpret_cast<const float4*>(a.cores + (size_t)(ok ? arow : 0u) * KR);
#pragma unroll
          for (int k = 0; k < KR / 16; ++k) bv[k] = (ok && !(a.dbg & 2)) ? __ldg(src + (tid >> 6) + 4 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
          (void)rows;
          // the next tile's grp_arow entry (this group's next tile, else the next unit's first)
          arow_n = qa + tpp < q1 ? arow_of(qa + tpp, q1) : (nxt < NU ? arow_of(q0n, q1n) : 0xffffffffu);
        }
        XTA(0);
        if (fl & 1u) {   // the unit's C2^T -> TMEM (hi = raw fp32, lo = x - trunc_tf32(x))
          tc::mbar_wait(&ctl.a_free, (gs & 1) ^ 1);
          XTA(1);
          tc::fence_after();
          if (BPU == 1 || blk < a.nblk) {
            tc::tmem_st32(tc::taddr(tm + blk * KR + r0, 32 * Q, 0), xa);
            if (KR > 32) tc::tmem_st32(tc::taddr(tm + blk * KR + r0 + 32, 32 * Q, 0), xb);
#pragma unroll
            for (int r = 0; r < 32; ++r) { xa[r] = tf32_lo(xa[r]); xb[r] = tf32_lo(xb[r]); }
            tc::tmem_st32(tc::taddr(tm + 128 + blk * KR + r0, 32 * Q, 0), xa);
            if (KR > 32) tc::tmem_st32(tc::taddr(tm + 128 + blk * KR + r0 + 32, 32 * Q, 0), xb);
            tc::tmem_wait_st();
          }
          tc::fence_before();
          tc::mbar_arrive(&ctl.a_full);
          XTA(2);
        }
        {
          const uint32_t s = ui & 1;
          tc::mbar_wait(&ctl.b_free[s], ((ui >> 1) & 1) ^ 1);
          XTA(3);
          char* bh = bbuf + s * BSLOT;
          char* bl = bh + BHALF;
#pragma unroll
          for (int k = 0; k < KR / 16; ++k) {
            const uint32_t off = tc::cm_off(m, 4 * ((tid >> 6) + 4 * k), XT / 8);
            const float4 v = bv[k];
            *reinterpret_cast<float4*>(bh + off) = v;
            *reinterpret_cast<float4*>(bl + off) = make_float4(tf32_lo(v.x), tf32_lo(v.y), tf32_lo(v.z), tf32_lo(v.w));
          }
          tc::fence_async_smem();
          tc::mbar_arrive(&ctl.b_full[s]);
          XTA(4);
        }
        if (arow_n != 0xffffffffu && !(a.dbg & 256)) {   // next tile's C1 row lines -> L1
          const float* pf = a.cores + (size_t)arow_n * KR + 4 * (tid >> 6);
#pragma unroll
          for (int k = 0; k < KR / 16; k += 2) asm volatile("prefetch.global.L1 [%0];" ::"l"(pf + 16 * k));
        }
      }
      XT0();
      // next unit: registers <- raw (nxt); raw <- the unit after (claimed now)
      if (tid == 0) ctl.claim[gs & 1] = claim();
      if (nxt < NU) {
        tc::mbar_wait(&ctl.raw_full, rawk & 1);
        ++rawk;
        XTA(5);
        cval = col_valid(nxt);
        load_raw();
      }
      tc::named_sync(1, X_LW * 32);
      XTA(6);
      const uint32_t nn = ctl.claim[gs & 1];
      if (tid == 0 && nn < NU) issue_raw(nn);
      ++gs;
      cur = nxt;
      nxt = nn;
      q0 = q0n; q1 = q1n;
      if (nn < NU) { q0n = a.grp_off[nn / UPG]; q1n = a.grp_off[nn / UPG + 1]; }
    }
    if (tid == 0) {
      tc::mbar_wait(&ctl.u_empty[ui & 3], ((ui >> 2) & 1) ^ 1);
      ctl.ring[ui & 3][3] = 4u;
      tc::mbar_arrive(&ctl.u_full[ui & 3]);
    }
  } else if (w == X_MMA_W) {
    // ------------------------------- MMA issuer -------------------------------
    uint32_t gs = 0;
    for (uint32_t ui = 0;; ++ui) {
      XT0();
      tc::mbar_wait(&ctl.u_full[ui & 3], (ui >> 2) & 1);
      XTA(0);
      const uint32_t np = ctl.ring[ui & 3][2], fl = ctl.ring[ui & 3][3], ub = ctl.ring[ui & 3][4];
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&ctl.u_empty[ui & 3]);
      if (fl & 4u) break;
      const int rows = (int)np << a.n1s;
      const int n16 = (rows + 15) & ~15;
      const uint32_t s = ui & 1;
      if (fl & 1u) tc::mbar_wait(&ctl.a_full, gs & 1);
      XTA(1);
      tc::mbar_wait(&ctl.b_full[s], (ui >> 1) & 1);
      XTA(2);
      tc::mbar_wait(&ctl.d_free[s], ((ui >> 1) & 1) ^ 1);
      XTA(3);
      tc::fence_after();
      if (lane == 0) {
        const uint32_t id = tc::idesc_tf32(128, n16, false, false);
        const uint32_t bh = tc::smem_u32(bbuf + s * BSLOT), bl = bh + BHALF;
        for (int blk = 0; blk < BPU && (int)ub * BPU + blk < a.nblk; ++blk) {
          const uint32_t d = tm + 256 + s * 128 + blk * 64;
#pragma unroll
          for (int kk = 0; kk < KR / 8; ++kk) {
            const uint32_t o = kk * 2 * (XT / 8) * 128;
            const uint64_t dbh = tc::sdesc(bh + o, (XT / 8) * 128, 128);
            const uint64_t dbl = tc::sdesc(bl + o, (XT / 8) * 128, 128);
            const uint32_t ah = tm + blk * KR + kk * 8, al = tm + 128 + blk * KR + kk * 8;
            if (a.dbg & 4) continue;
            tc::mma_tf32_ts(d, ah, dbh, id, kk > 0 ? 1u : 0u);
            if (a.dbg & 8) continue;
            tc::mma_tf32_ts(d, ah, dbl, id, 1u);
            tc::mma_tf32_ts(d, al, dbh, id, 1u);
          }
        }
        tc::commit(&ctl.b_free[s]);
        tc::commit(&ctl.d_full[s]);
        if (fl & 2u) tc::commit(&ctl.a_free);
      }
      __syncwarp();
      XTA(4);
      trc[9] += 1;
      if (fl & 2u) ++gs;
    }
  } else {
    // ------------------------- epilogue: TMEM -> P stash -------------------------
    // warp w drains lane quarter Q = w % 4 of every c-block of the unit: thread = column c, 32
    // tile rows per tcgen05.ld; pbuf[(q n1 + j1)][c] rows of one tile are contiguous
    const int Q = w & 3;
    for (uint32_t ui = 0;; ++ui) {
      XT0();
      tc::mbar_wait(&ctl.u_full[ui & 3], (ui >> 2) & 1);
      XTA(0);
      const uint32_t qa = ctl.ring[ui & 3][1], np = ctl.ring[ui & 3][2], fl = ctl.ring[ui & 3][3];
      const uint32_t ub = ctl.ring[ui & 3][4];
      __syncwarp();
      if (fl & 4u) break;
      const int rows = (int)np << a.n1s;
      const uint32_t s = ui & 1;
      tc::mbar_wait(&ctl.d_full[s], (ui >> 1) & 1);
      XTA(1);
      tc::fence_after();
      float* dst = a.pbuf + (size_t)qa * a.n1 * a.NC;
      for (int blk = 0; blk < BPU; ++blk) {
        const int c = ((int)ub * BPU + blk) * 128 + Q * 32 + lane;
        for (int j0 = 0; j0 < rows; j0 += 32) {
          float v[32];
          tc::tmem_ld32(tc::taddr(tm + 256 + s * 128 + blk * 64 + j0, 32 * Q, 0), v);
          const int lim = min(32, rows - j0);
          if (c < a.NC && !(a.dbg & 1)) {
            float* d = dst + (size_t)j0 * a.NC + c;
            if (lim == 32) {   // full 32-row chunk: no per-element predicates / branches
#pragma unroll
              for (int j = 0; j < 32; ++j) d[(size_t)j * NCT] = v[j];
            } else {
#pragma unroll
              for (int j = 0; j < 32; ++j)
                if (j < lim) d[(size_t)j * NCT] = v[j];
            }
          }
        }
      }
      tc::fence_before();
      tc::mbar_arrive(&ctl.d_free[s]);
      XTA(2);
      if (lane == 0) tc::mbar_arrive(&ctl.u_empty[ui & 3]);
    }
  }
  if (a.trace) {
    const int role = tid == 0 ? 0 : tid == X_MMA_W * 32 ? 1 : tid == X_ROW_W0 * 32 ? 2 : -1;
    if (role >= 0)
      for (int k = 0; k < 10; ++k) a.trace[32 * blockIdx.x + 10 * role + k] = trc[k];
    if (tid == 0) a.trace[32 * blockIdx.x + 30] = (unsigned long long)(clock64() - t_start);
    if (tid == X_ROW_W0 * 32) {
      a.trace[32 * blockIdx.x + 31] = tc::globaltimer_ns();
      a.trace[32 * blockIdx.x + 29] = g_start;
    }
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (w == X_MMA_W) tc::tmem_dealloc(tm, 512);
}

template <int KR> constexpr size_t prefix_smem() { return 128 + X_RAW_BYTES + 2 * (2u * XT * KR * 4); }

// ------------------------------------------------------------------------------------
// Row contraction a6 (Eq. 2, Fig. 5(b) step 3): E_u = P_q (n1 n2 x R) . C3[i3_u] (R x n3)
// on FFMA, high occupancy (8 warps per CTA, 4 CTAs per SM).  A warp owns RCH consecutive
// unique rows (rows of one prefix are consecutive, so P_q is reloaded only at prefix
// changes).  Lane map: jq = lane >> 3 owns j12 = 4 jq .. 4 jq + 3, rp = lane & 7 owns
// r = 8 rp .. 8 rp + 7 (P_q slice in 32 registers); the C3 slice of each row is streamed
// into a per-warp 3-slot shared-memory ring by cp.async two rows ahead, with rows skewed by
// 4 floats per 8 so the 8 rp lanes of an LDS.128 phase hit distinct banks; the 4 j12 x n3
// partial sums are reduced over rp by recursive halving (3 shuffle levels) and each lane
// stores n3/2 consecutive outputs.
// ------------------------------------------------------------------------------------
// Packed fp32 pairs on sm_100 (FFMA2): d = a * b + c lane by lane, each an ordinary
// round-to-nearest fp32 fma; ptxas folds a {s, s} pair into a scalar operand.
__device__ __forceinline__ void ffma2(float2& d, float2 a, float2 b) {
  asm("fma.rn.f32x2 %0, %1, %2, %0;"
      : "+l"(*reinterpret_cast<unsigned long long*>(&d))
      : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)));
}
__device__ __forceinline__ void ffma2s(float2& d, float s, float2 b) { ffma2(d, make_float2(s, s), b); }

#ifndef TTEMB_FWD_ROWS_GRID
#define TTEMB_FWD_ROWS_GRID 4     // k_rows_fwd2 grid cap, CTAs per SM
#endif
#ifndef TTEMB_FWD_ROWS_BLOCKS
#define TTEMB_FWD_ROWS_BLOCKS 3   // k_rows_fwd2 CTAs per SM at n3 = 4, R = 64 (register cap 85)
#endif
#ifndef TTEMB_RF_NSL
#define TTEMB_RF_NSL 3   // ring slots of k_rows_fwd2 (rows in flight + 1)
#endif
#ifndef TTEMB_RB_NSL
#define TTEMB_RB_NSL 3   // ring slots of k_rows_bwd2
#endif
constexpr int RW_WARPS = 8, RW_RCH = 16, RW_NSL = TTEMB_RF_NSL, RB_NSL = TTEMB_RB_NSL;

struct RowArgs {
  const float* cores;
  const TableMeta* meta;
  const uint32_t *counts, *row_pfx, *row_c3, *pfx_t, *seg_off, *sbag;
  unsigned long long c3_begin;   // float offset of the C3 region (row_c3 counts R n3 slices from it)
  const float* pbuf;          // [P][n1][NC]
  float* rows;                // [U][N]
  float* out;                 // [B][T][N]: written directly when every bag holds one id (a7)
  int n1, n1s, n2, N, NC;
};

template <int N3, int RPL>   // RPL = R / 8: r values per lane (8 at R = 64, 16 at R = 128)
__global__ void __launch_bounds__(RW_WARPS * 32, (RPL == 8 && N3 == 4) ? TTEMB_FWD_ROWS_BLOCKS : 2) k_rows_fwd2(RowArgs a) {
  pdl_wait();
  pdl_trigger();
  constexpr int KR = 8 * RPL;
  constexpr int SLOT = KR * N3 + KR / 2;       // + 4 floats of skew per 8 rows of r
  constexpr int C3L = KR * N3 / 4 / 32;
  extern __shared__ __align__(16) float rw_smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float* const ringp = rw_smem + w * (RW_NSL * SLOT);
  const uint32_t ring = tc::smem_u32(ringp);
  const uint32_t U = tt_rows(a.counts);   // TT rows only (hybrid: dense rows follow)
  const int J12 = a.n1 * a.n2;
  const int jq = lane >> 3, rp = lane & 7;
  // per-lane P offsets inside a prefix block [n1][NC] for e = 0..3 (j12 = 4 jq + e)
  int poff[4];
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const int j12 = 4 * jq + e, j1 = j12 / a.n2, j2 = j12 - j1 * a.n2;
    poff[e] = j12 < J12 ? j1 * a.NC + j2 * KR + RPL * rp : -1;
  }
  const int64_t nch = ((int64_t)U + RW_RCH - 1) / RW_RCH;
  const int64_t gw = (int64_t)blockIdx.x * RW_WARPS + w, nw = (int64_t)gridDim.x * RW_WARPS;
  for (int64_t ch = gw; ch < nch; ch += nw) {
    const uint32_t u0 = (uint32_t)ch * RW_RCH;
    const int nr = (int)min((uint32_t)RW_RCH, U - u0);
    uint32_t ql = 0;
    unsigned long long o3l = 0;
    if (lane < nr) {
      ql = __ldg(a.row_pfx + u0 + lane);
      o3l = a.c3_begin + (unsigned long long)__ldg(a.row_c3 + u0 + lane) * KR * N3;
    }
    auto issue = [&](int j) {
      const unsigned long long o3 = __shfl_sync(0xffffffffu, o3l, j);
      const float4* src = reinterpret_cast<const float4*>(a.cores + o3);
      const uint32_t dst = ring + (uint32_t)((j % RW_NSL) * SLOT * 4);
#pragma unroll
      for (int i = 0; i < C3L; ++i) {
        const int f = lane + 32 * i, r = f / (N3 / 4);
        tc::cp_async16(dst + 4u * (uint32_t)(4 * f + 4 * (r >> 3)), src + f);
      }
    };
#pragma unroll
    for (int j = 0; j < RW_NSL - 1; ++j) {
      if (j < nr) issue(j);
      tc::cp_commit();
    }
    uint32_t curq = 0xffffffffu;
    float pr[4][RPL];
    for (int j = 0; j < nr; ++j) {
      const uint32_t q = __shfl_sync(0xffffffffu, ql, j);
      if (q != curq) {
        const float* pq = a.pbuf + (size_t)q * a.n1 * a.NC;
#pragma unroll
        for (int e = 0; e < 4; ++e)
#pragma unroll
          for (int h = 0; h < RPL; h += 4) {
            const float4 x0 = poff[e] >= 0 ? __ldg(reinterpret_cast<const float4*>(pq + poff[e] + h))
                                           : make_float4(0.f, 0.f, 0.f, 0.f);
            pr[e][h] = x0.x; pr[e][h + 1] = x0.y; pr[e][h + 2] = x0.z; pr[e][h + 3] = x0.w;
          }
        curq = q;
      }
      tc::cp_wait<RW_NSL - 2>();
      __syncwarp();
      float2 acc2[2 * N3];   // (E[j12][b], E[j12][b + 1]) partial pairs: packed FFMA2, P scalar
#pragma unroll
      for (int i = 0; i < 2 * N3; ++i) acc2[i] = make_float2(0.f, 0.f);
      const float* slot3 = ringp + (j % RW_NSL) * SLOT;
#pragma unroll
      for (int x = 0; x < RPL; ++x) {
        const int r = RPL * rp + x;
        const float* c3 = slot3 + r * N3 + 4 * (r >> 3);   // the ring's per-8-row skew
        float2 cv[N3 / 2];
#pragma unroll
        for (int b = 0; b < N3; b += 4) {
          const float4 t4 = *reinterpret_cast<const float4*>(c3 + b);
          cv[b / 2] = make_float2(t4.x, t4.y); cv[b / 2 + 1] = make_float2(t4.z, t4.w);
        }
#pragma unroll
        for (int e = 0; e < 4; ++e)
#pragma unroll
          for (int b2 = 0; b2 < N3 / 2; ++b2) ffma2s(acc2[e * (N3 / 2) + b2], pr[e][x], cv[b2]);
      }
      float acc[4 * N3];
#pragma unroll
      for (int i = 0; i < 2 * N3; ++i) { acc[2 * i] = acc2[i].x; acc[2 * i + 1] = acc2[i].y; }
      __syncwarp();
      if (j + RW_NSL - 1 < nr) issue(j + RW_NSL - 1);
      tc::cp_commit();
#pragma unroll
      for (int lv = 0; lv < 3; ++lv) {
        const int mask = 4 >> lv, half = (4 * N3) >> (lv + 1);
        const bool hi = (lane & mask) != 0;
#pragma unroll
        for (int i = 0; i < half; ++i) {
          const float snd = hi ? acc[i] : acc[i + half];
          const float kp = hi ? acc[i + half] : acc[i];
          acc[i] = kp + __shfl_xor_sync(0xffffffffu, snd, mask);
        }
      }
      // this lane holds E[j12 = 4 jq + rp / 2][j3 = (rp & 1) n3/2 .. + n3/2 - 1]
      if (4 * jq + (rp >> 1) < J12) {
        float* d = a.rows + (size_t)(u0 + j) * a.N + (4 * jq) * N3 + rp * (N3 / 2);
        if (N3 == 4) *reinterpret_cast<float2*>(d) = make_float2(acc[0], acc[1]);
        else *reinterpret_cast<float4*>(d) = make_float4(acc[0], acc[1], acc[2], acc[3]);
      }
    }
    tc::cp_wait<0>();
    __syncwarp();
  }
}

size_t rows_smem(int n3, int R) { return (size_t)RW_WARPS * RW_NSL * (R * n3 + R / 2) * 4; }

// ------------------------------------------------------------------------------------
// Row backward a9 (Eq. 6 read as left^T . dL/de . right^T).  A warp owns 16
// consecutive unique rows (rows of one prefix are consecutive) and one SW-wide slice of r;
// lane l owns r = rb + RL l + x (x < RL) for ALL j12 and j3, so neither product needs a
// cross-lane reduction:
//   dP_q[j12][r] += sum_j3 G_u[j12][j3] C3_u[r][j3]     registers (16 j12 x RL per lane),
//                                                       flushed to dpbuf at prefix changes
//   dC3[i3_u][r][j3] += sum_j12 P_q[j12][r] G_u[j12][j3]  (RL x n3 per lane, red.global.add.v4
//                                                         into the L2-resident gradient)
// The C3 slice (r-slice of the row) and G_u stream into a per-warp 3-slot shared-memory ring by
// cp.async two rows ahead; the C3 part is stored [x][j3/4][l] in 16-byte pieces so a lane's
// loads are conflict-free, and G_u is read as broadcasts.  dP of a prefix whose rows straddle a
// chunk boundary is accumulated with vector reductions into rows zeroed by k_dp_zero2;
// prefixes inside one chunk are stored directly.
// ------------------------------------------------------------------------------------
struct RowBwdArgs {
  const float* cores;
  float* grads;
  const TableMeta* meta;
  const uint32_t *counts, *row_pfx, *row_c3, *pfx_t, *row_seg;
  unsigned long long c3_begin;   // float offset of the C3 region (row_c3 counts R n3 slices from it)
  const float* pbuf;          // [P][n1][NC]
  const float* gbuf;          // [U][N]
  float* dpbuf;               // [P][n1][NC]
  int n1, n2, N, NC, R;
  int exp;                    // TTEMB_EXP bits (timing experiments only; results invalid)
};

__global__ void __launch_bounds__(256) k_dp_zero2(RowBwdArgs a) {
  const uint32_t P = a.counts[kCntP];
  const int blk = a.n1 * a.NC / 4;
  const int lane = threadIdx.x & 31;
  for (uint32_t q = blockIdx.x * 8 + (threadIdx.x >> 5); q < P; q += gridDim.x * 8) {
    const uint32_t r0 = a.row_seg[q], r1 = a.row_seg[q + 1];
    if (r0 / RW_RCH == (r1 - 1) / RW_RCH) continue;
    float4* d = reinterpret_cast<float4*>(a.dpbuf + (size_t)q * a.n1 * a.NC);
    for (int f = lane; f < blk; f += 32) d[f] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

__device__ __forceinline__ void red_v4(float* addr, float4 v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
               : "memory");
}
__device__ __forceinline__ void red_v2(float* addr, float x, float y) {
  asm volatile("red.global.add.v2.f32 [%0], {%1, %2};" ::"l"(addr), "f"(x), "f"(y) : "memory");
}

constexpr int RB_J12 = 16;   // n1 n2 <= 16


// P_q[j12][r] sits at pbuf[(q J12 + j12) R + r] (NC = n2 R), so with R a template constant every
// per-j12 access is an immediate offset from one base pointer.
template <int N3, int RL, int KR, int J12T>   // RL = r per lane: 1 (R = 32) or 2 (R = 64, 128 in two
                                              // slices); J12T = n1 n2 (0: runtime, <= 16)
__global__ void __launch_bounds__(RW_WARPS * 32, RL == 1 ? 3 : 2) k_rows_bwd2(RowBwdArgs a) {
  pdl_wait();
  pdl_trigger();
  constexpr int SW = 32 * RL;                   // r width of a work item (a slice of R)
  constexpr int NSL = KR / SW;                  // slices per row
  constexpr int C3S = SW * N3;                  // C3 part of a slot
  constexpr int SLOT = C3S + RB_J12 * N3;       // + G_u (N <= 16 n3)
  constexpr int H4 = N3 / 4;                    // 16-byte pieces per r row
  constexpr int C3L = RL * H4;                  // 16-byte pieces of the C3 slice per lane
  constexpr int JM = J12T ? J12T : RB_J12;      // unrolled j12 extent
  extern __shared__ __align__(16) float rw_smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float* const ringp = rw_smem + w * (RB_NSL * SLOT);
  const uint32_t ring = tc::smem_u32(ringp);
  const uint32_t U = tt_rows(a.counts);   // TT rows only (hybrid: dense rows follow)
  const int J12 = J12T ? J12T : a.n1 * a.n2;
  const int64_t nch = ((int64_t)U + RW_RCH - 1) / RW_RCH;
  const int64_t gw = (int64_t)blockIdx.x * RW_WARPS + w, nw = (int64_t)gridDim.x * RW_WARPS;
  // work item metadata (row prefix, C3 slice) is loaded one item ahead
  auto load_meta = [&](int64_t it, uint32_t& q, uint32_t& c3) {
    q = 0; c3 = 0;
    if (it < nch * NSL) {
      const uint32_t u = (uint32_t)(NSL == 1 ? it : it / NSL) * RW_RCH + lane;
      if (u < U) { q = __ldg(a.row_pfx + u); c3 = __ldg(a.row_c3 + u); }
    }
  };
  uint32_t nql, nc3;
  load_meta(gw, nql, nc3);
  for (int64_t it = gw; it < nch * NSL; it += nw) {
    const int64_t ch = NSL == 1 ? it : it / NSL;
    const int rb = SW * (int)(it - ch * NSL);     // first r of the slice (R = 128: two slices)
    const int rl = rb + RL * lane;                // this lane's first r
    const uint32_t u0 = (uint32_t)ch * RW_RCH;
    const int nr = (int)min((uint32_t)RW_RCH, U - u0);
    const uint32_t ql = nql;
    // the row's C3 slice, this work item's r-slice
    const unsigned long long o3l = a.c3_begin + (unsigned long long)nc3 * KR * N3 + (unsigned long long)rb * N3;
    load_meta(it + nw, nql, nc3);
    const uint32_t prevq = u0 > 0 ? __ldg(a.row_pfx + u0 - 1) : 0xffffffffu;
    const uint32_t nextq = u0 + nr < U ? __ldg(a.row_pfx + u0 + nr) : 0xffffffffu;
    // slot layout: C3 piece (x, h) of lane l at [(x H4 + h) 32 + l] (16 bytes each: the warp's
    // cp.async stores and a lane's loads are contiguous / conflict-free), then G_u
    auto issue = [&](int j) {
      if (a.exp & 512) return;
      const unsigned long long o3 = __shfl_sync(0xffffffffu, o3l, j) + (unsigned long long)(RL * lane) * N3;
      const float4* src = reinterpret_cast<const float4*>(a.cores + o3);
      const uint32_t dst = ring + (uint32_t)((j % RB_NSL) * SLOT * 4) + 16u * lane;
#pragma unroll
      for (int i = 0; i < C3L; ++i) tc::cp_async16(dst + 16u * 32u * i, src + i);
      if (lane < a.N / 4)
        tc::cp_async16(ring + (uint32_t)(((j % RB_NSL) * SLOT + C3S) * 4) + 16u * lane,
                       reinterpret_cast<const float4*>(a.gbuf + (size_t)(u0 + j) * a.N) + lane);
    };
#pragma unroll
    for (int j = 0; j < RB_NSL - 1; ++j) {
      if (j < nr) issue(j);
      tc::cp_commit();
    }
    uint32_t curq = 0xffffffffu;
    // lane's P_q[j12][rl .. rl + RL) and dP accumulators: one fp32 (RL = 1) or a packed pair
    using PV = typename std::conditional<RL == 2, float2, float>::type;
    PV pr[JM], dp[JM];
    auto flush = [&]() {
      if (a.exp & 128) return;
      const bool red = curq == prevq || curq == nextq;
      float* d = a.dpbuf + (size_t)curq * J12 * KR + rl;
#pragma unroll
      for (int j12 = 0; j12 < JM; ++j12) {
        if (!J12T && j12 >= J12) break;
        float* e = d + j12 * KR;
        if constexpr (RL == 2) {
          if (red) red_v2(e, dp[j12].x, dp[j12].y);
          else *reinterpret_cast<float2*>(e) = dp[j12];
        } else {
          if (red) atomicAdd(e, dp[j12]);
          else *e = dp[j12];
        }
      }
    };
    for (int j = 0; j < nr; ++j) {
      const uint32_t q = __shfl_sync(0xffffffffu, ql, j);
      if (q != curq) {
        if (curq != 0xffffffffu) flush();
        {   // L1 prefetch of the next prefix of the item (its P slice: 16 j12 x SW floats)
          const unsigned later = __ballot_sync(0xffffffffu, lane > j && lane < nr && ql != q);
          if (later) {
            const uint32_t qn = __shfl_sync(0xffffffffu, ql, __ffs(later) - 1);
            if ((lane >> 1) < J12)
              asm volatile("prefetch.global.L1 [%0];" ::"l"(a.pbuf + (size_t)qn * J12 * KR + (lane >> 1) * KR + rb + 32 * (lane & 1)));
          }
        }
        const float* pq = a.pbuf + (size_t)q * J12 * KR + rl;
#pragma unroll
        for (int j12 = 0; j12 < JM; ++j12) {
          if constexpr (RL == 2) {
            pr[j12] = ((J12T || j12 < J12) && !(a.exp & 256)) ? __ldg(reinterpret_cast<const float2*>(pq + j12 * KR)) : make_float2(0.f, 0.f);
            dp[j12] = make_float2(0.f, 0.f);
          } else {
            pr[j12] = (J12T || j12 < J12) ? __ldg(pq + j12 * KR) : 0.f;
            dp[j12] = 0.f;
          }
        }
        curq = q;
      }
      tc::cp_wait<RB_NSL - 2>();
      __syncwarp();
      const float* slot = ringp + (j % RB_NSL) * SLOT;
      // C3[rl + x][b] for the lane's r; c3x[b] = (C3[rl][b], C3[rl + 1][b]) pairs the lane's two r
      float c3[RL][N3];
      float2 dc[RL][N3 / 2];
#pragma unroll
      for (int i = 0; i < C3L; ++i) {   // piece i = (x, h): r = rl + x, j3 = 4h .. 4h + 3
        const int x = i / H4, h = i - x * H4;
        const float4 t4 = *reinterpret_cast<const float4*>(slot + 4 * (i * 32 + lane));
        c3[x][4 * h] = t4.x; c3[x][4 * h + 1] = t4.y; c3[x][4 * h + 2] = t4.z; c3[x][4 * h + 3] = t4.w;
        dc[x][2 * h] = make_float2(0.f, 0.f); dc[x][2 * h + 1] = make_float2(0.f, 0.f);
      }
#pragma unroll
      for (int j12 = 0; j12 < JM; ++j12) {
        if (J12T || j12 < J12) {
          float2 g[N3 / 2];
#pragma unroll
          for (int h = 0; h < H4; ++h) {   // broadcast read of G_u[j12][4h .. 4h + 3]
            const float4 t4 = *reinterpret_cast<const float4*>(slot + C3S + j12 * N3 + 4 * h);
            g[2 * h] = make_float2(t4.x, t4.y); g[2 * h + 1] = make_float2(t4.z, t4.w);
          }
          // dP: scalar FFMA (a packed form would need (C3[rl][b], C3[rl + 1][b]) pairs, which cost
          // more register moves than they save); dC3: packed pairs (FFMA2) of G[j12][b], G[j12][b + 1]
#pragma unroll
          for (int b = 0; b < N3; ++b) {   // dP[j12][rl + x] += G[j12][b] C3[rl + x][b]
            const float gb = (b & 1) ? g[b >> 1].y : g[b >> 1].x;
            if constexpr (RL == 2) {
              dp[j12].x = fmaf(gb, c3[0][b], dp[j12].x);
              dp[j12].y = fmaf(gb, c3[1][b], dp[j12].y);
            } else {
              dp[j12] = fmaf(gb, c3[0][b], dp[j12]);
            }
          }
#pragma unroll
          for (int b2 = 0; b2 < N3 / 2; ++b2) {   // dC3[rl + x][2 b2 .. 2 b2 + 1] += P[j12][rl + x] G[j12][2 b2 ..]
            if constexpr (RL == 2) {
              ffma2s(dc[0][b2], pr[j12].x, g[b2]);
              ffma2s(dc[1][b2], pr[j12].y, g[b2]);
            } else {
              ffma2s(dc[0][b2], pr[j12], g[b2]);
            }
          }
        }
      }
      __syncwarp();
      if (j + RB_NSL - 1 < nr) issue(j + RB_NSL - 1);
      tc::cp_commit();
      // dC3[i3_u][rl + x][0 .. n3): RL n3 consecutive floats per lane
      float* d3 = a.grads + __shfl_sync(0xffffffffu, o3l, j) + (size_t)(RL * lane) * N3;
      if (!(a.exp & 64))
#pragma unroll
      for (int x = 0; x < RL; ++x)
#pragma unroll
        for (int b2 = 0; b2 < N3 / 2; b2 += 2)
          red_v4(d3 + x * N3 + 2 * b2, make_float4(dc[x][b2].x, dc[x][b2].y, dc[x][b2 + 1].x, dc[x][b2 + 1].y));
    }
    if (curq != 0xffffffffu) flush();
    tc::cp_wait<0>();
    __syncwarp();
  }
}

size_t rows_bwd_smem(int n3, int sw) { return (size_t)RW_WARPS * RB_NSL * (sw * n3 + RB_J12 * n3) * 4; }   // per sw-wide r slice

// (n3, R, n1 n2) -> k_rows_bwd2 instantiation (n1 n2 = 16 unrolled exactly, others predicated)
template <int N3, int RL, int KR> const void* rows_bwd_pick(int j12) {
  return j12 == 16 ? (const void*)k_rows_bwd2<N3, RL, KR, 16> : (const void*)k_rows_bwd2<N3, RL, KR, 0>;
}
const void* rows_bwd_kernel(int n3, int R, int j12) {
  if (n3 == 4) {
    if (R == 32) return rows_bwd_pick<4, 1, 32>(j12);
    if (R == 64) return rows_bwd_pick<4, 2, 64>(j12);
    if (R == 128) return rows_bwd_pick<4, 2, 128>(j12);
  } else if (n3 == 8) {
    if (R == 32) return rows_bwd_pick<8, 1, 32>(j12);
    if (R == 64) return rows_bwd_pick<8, 2, 64>(j12);
    if (R == 128) return rows_bwd_pick<8, 2, 128>(j12);
  }
  return nullptr;
}
const void* rows_bwd_kernel_rl1(int n3, int R, int j12) {
  if (n3 == 4) {
    if (R == 32) return rows_bwd_pick<4, 1, 32>(j12);
    if (R == 64) return rows_bwd_pick<4, 1, 64>(j12);
    if (R == 128) return rows_bwd_pick<4, 1, 128>(j12);
  } else if (n3 == 8) {
    if (R == 32) return rows_bwd_pick<8, 1, 32>(j12);
    if (R == 64) return rows_bwd_pick<8, 1, 64>(j12);
    if (R == 128) return rows_bwd_pick<8, 1, 128>(j12);
  }
  return nullptr;
}
template <class F> void for_rows_bwd(F&& f) {
  for (int n3 : {4, 8})
    for (int R : {32, 64, 128})
      for (int j12 : {16, 4}) f(rows_bwd_kernel_rl1(n3, R, j12), n3, 32);
  for (int n3 : {4, 8})
    for (int R : {32, 64, 128})
      for (int j12 : {16, 4}) f(rows_bwd_kernel(n3, R, j12), n3, R == 32 ? 32 : 64);
}

// Work-unit order of the prefix kernels (plan-dependent, run with the index stage): units (i2-group,
// c-block range) sorted by their tile count, largest first (a counting sort; the order inside one
// count is arbitrary and only changes which CTA does what).  k_prefix_bwd deals it to its G
// CTAs round by round in alternating directions (round r, CTA c takes sorted unit r G + c for even
// r, r G + G - 1 - c for odd r), which balances its static schedule: at c4 the most loaded CTA
// had 22 tiles against a mean of 18.3 in group order (bwd_prefix 150 -> 135 us).  k_prefix_fwd
// keeps claiming in group order (dynamic claims already balance it; see its claim()).
__global__ void __launch_bounds__(1024) k_unit_order(const uint32_t* __restrict__ counts, const uint32_t* __restrict__ grp_off,
                                                     int tpp, int upg, int G, uint32_t* __restrict__ sorted,
                                                     uint32_t* __restrict__ snake) {
  __shared__ uint32_t hist[256];
  const uint32_t NU = counts[kCntNG] * (uint32_t)upg;
  for (int i = threadIdx.x; i < 256; i += blockDim.x) hist[i] = 0;
  __syncthreads();
  auto bucket = [&](uint32_t u) {   // 255 - min(tiles, 255): ascending bucket = descending size
    const uint32_t g = u / upg, np = grp_off[g + 1] - grp_off[g];
    return 255u - min((np + tpp - 1) / tpp, 255u);
  };
  for (uint32_t u = threadIdx.x; u < NU; u += blockDim.x) atomicAdd(&hist[bucket(u)], 1u);
  __syncthreads();
  if (threadIdx.x < 32) {   // exclusive scan of 256 buckets by one warp (8 per lane)
    const int l = threadIdx.x;
    uint32_t v[8], t = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) { v[i] = hist[8 * l + i]; t += v[i]; }
    uint32_t x = t;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (l >= o) x += y;
    }
    uint32_t run = x - t;
#pragma unroll
    for (int i = 0; i < 8; ++i) { hist[8 * l + i] = run; run += v[i]; }
  }
  __syncthreads();
  for (uint32_t u = threadIdx.x; u < NU; u += blockDim.x) sorted[atomicAdd(&hist[bucket(u)], 1u)] = u;
  __syncthreads();
  for (uint32_t p = threadIdx.x; p < NU; p += blockDim.x) {
    const uint32_t r = p / (uint32_t)G, c = p - r * (uint32_t)G, base = r * (uint32_t)G;
    const uint32_t m = min((uint32_t)G, NU - base);   // units in this round
    snake[p] = sorted[base + ((r & 1u) ? m - 1u - c : c)];
  }
}

}  // namespace

int prefix_units_per_group(const Ctx& c) { return c.R <= 64 ? 1 : (c.NC + 127) / 128; }
int prefix_bwd_grid(const Ctx& c) {
  const int64_t units = c.NG_cap * prefix_units_per_group(c);
  return (int)std::max<int64_t>(1, std::min<int64_t>(units, (int64_t)c.sm_count));
}

cudaError_t run_unit_order(Ctx& c, cudaStream_t s) {
  k_unit_order<<<1, 1024, 0, s>>>(c.p.counts, c.p.grp_off, XT / c.n1, prefix_units_per_group(c), prefix_bwd_grid(c),
                                  c.p.unit_sorted, c.p.unit_snake);
  return cudaGetLastError();
}

bool fused_eligible(const Ctx& c) {
  // R = 32 / 64 (ranks 16..63 stored padded to 32 or 64) with n2 R <= 256; R = 128 with n2 R <= 512
  return !(c.flags & TTEMB_FP32_CORES) && (c.R == 32 || c.R == 64 || c.R == 128) &&
         c.NC <= (c.R == 128 ? 512 : 256) &&
         (c.n3 == 4 || c.n3 == 8) && (c.n1 == 1 || c.n1 == 2 || c.n1 == 4 || c.n1 == 8) && c.n1 * c.n2 <= 16;
}
bool tc_eligible(const Ctx& c) { return fused_eligible(c); }
cudaError_t configure_tc(Ctx&) { return cudaSuccess; }

cudaError_t configure_fused(Ctx& c) {
  if (!fused_eligible(c)) return cudaSuccess;
  cudaError_t e = cudaSuccess;
  auto set = [&](const void* f, size_t bytes) {
    if (e == cudaSuccess) e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  };
  set((const void*)k_prefix_fwd<32, 0>, prefix_smem<32>());
  set((const void*)k_prefix_fwd<64, 0>, prefix_smem<64>());
  set((const void*)k_prefix_fwd<128, 0>, prefix_smem<128>());
  set((const void*)k_prefix_fwd<32, 128>, prefix_smem<32>());
  set((const void*)k_prefix_fwd<64, 256>, prefix_smem<64>());
  set((const void*)k_prefix_fwd<128, 512>, prefix_smem<128>());
  set((const void*)k_rows_fwd2<4, 8>, rows_smem(4, 64));
  set((const void*)k_rows_fwd2<8, 8>, rows_smem(8, 64));
  set((const void*)k_rows_fwd2<4, 4>, rows_smem(4, 32));
  set((const void*)k_rows_fwd2<8, 4>, rows_smem(8, 32));
  set((const void*)k_rows_fwd2<4, 16>, rows_smem(4, 128));
  set((const void*)k_rows_fwd2<8, 16>, rows_smem(8, 128));
  for_rows_bwd([&](const void* f, int n3, int sw) { set(f, rows_bwd_smem(n3, sw)); });
  return e;
}

cudaError_t run_fused_fwd(Ctx& c, float* out, cudaStream_t s) {
  const PlanDev& p = c.p;
  XArgs a;
  a.cores = c.cores; a.meta = c.d_meta; a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t;
  a.grp_i2 = p.grp_i2; a.grp_pfx = p.grp_pfx; a.pfx_i1 = p.pfx_i1; a.pfx_t = p.pfx_t; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.row_pfx = p.row_pfx; a.grp_arow = p.grp_arow; a.grp_c2 = p.grp_c2; a.rows = p.rows; a.pbuf = p.pbuf;
  a.unit_sorted = p.unit_sorted;
  a.work = p.work + 0;
  a.dbg = knobs().dbg;
  a.n1 = c.n1; a.n1s = c.n1 == 1 ? 0 : c.n1 == 2 ? 1 : c.n1 == 4 ? 2 : 3;
  a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.NC = c.NC; a.nblk = (c.NC + 127) / 128; a.tpp = XT / c.n1; a.R = c.R;
  {
    StageScope sc(c, ST_FWD_PREFIX, s);
    launch_pdl(k_fused_prep, dim3(grid_for(c, std::max(c.P_cap, c.NG_cap), 256, 4)), dim3(256), 0, s, a);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count));
    static unsigned long long* trace = nullptr;
    a.trace = nullptr;
    if (knobs().trace) {
      if (!trace) cudaMalloc(&trace, sizeof(unsigned long long) * 32 * grid);
      cudaMemsetAsync(trace, 0, sizeof(unsigned long long) * 32 * grid, s);
      a.trace = trace;
    }
    const bool n2_4 = c.n2 == 4;   // the c4 / c5 shapes: NC = 4 R as a compile-time constant
    if (c.R == 32) {
      if (n2_4) launch_pdl(k_prefix_fwd<32, 128>, dim3(grid), dim3(X_THREADS), prefix_smem<32>(), s, a);
      else launch_pdl(k_prefix_fwd<32, 0>, dim3(grid), dim3(X_THREADS), prefix_smem<32>(), s, a);
    } else if (c.R == 64) {
      if (n2_4) launch_pdl(k_prefix_fwd<64, 256>, dim3(grid), dim3(X_THREADS), prefix_smem<64>(), s, a);
      else launch_pdl(k_prefix_fwd<64, 0>, dim3(grid), dim3(X_THREADS), prefix_smem<64>(), s, a);
    } else {
      if (n2_4) launch_pdl(k_prefix_fwd<128, 512>, dim3(grid), dim3(X_THREADS), prefix_smem<128>(), s, a);
      else launch_pdl(k_prefix_fwd<128, 0>, dim3(grid), dim3(X_THREADS), prefix_smem<128>(), s, a);
    }
    if (a.trace) {
      std::vector<unsigned long long> hb(32 * grid);
      cudaMemcpyAsync(hb.data(), trace, hb.size() * 8, cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
      double m[32] = {};
      for (int b = 0; b < grid; ++b) for (int k = 0; k < 29; ++k) m[k] += (double)hb[32 * b + k] / grid;
      unsigned long long s0 = ~0ull, s1 = ~0ull, e0 = 0, e1 = ~0ull;
      double tmax = 0;
      for (int b = 0; b < grid; ++b) {
        s0 = std::min(s0, hb[32 * b + 29]); s1 = s1 == ~0ull ? hb[32 * b + 29] : std::max(s1, hb[32 * b + 29]);
        e0 = std::max(e0, hb[32 * b + 31]); e1 = std::min(e1, hb[32 * b + 31]);
        tmax = std::max(tmax, (double)hb[32 * b + 30]);
      }
      fprintf(stderr, "[trace fused] span: first start -> last start %.1f us, first end %.1f us, last end %.1f us; max CTA cycles %.0f\n",
              (s1 - s0) * 1e-3, (e1 - s0) * 1e-3, (e0 - s0) * 1e-3, tmax);
      fprintf(stderr, "[trace fused] total %.0f | loader: ring+bload %.0f a_free %.0f a_store %.0f b_free %.0f b_store %.0f "
              "raw_wait %.0f raw_sync %.0f | mma: u_full %.0f a_full %.0f b_full %.0f d_free %.0f issue %.0f units %.1f | "
              "rows: u_full %.0f plist %.0f d_full %.0f [fa %.0f loop %.0f] fb+arrive %.0f sync1 %.0f rows %.0f sync2 %.0f nrows %.0f (cycles/CTA)\n",
              m[30], m[0], m[1], m[2], m[3], m[4], m[5], m[6], m[10], m[11], m[12], m[13], m[14], m[19], m[20], m[21],
              m[22], m[27], m[29], m[23], m[24], m[25], m[26], m[28]);
    }
  }
  {
    StageScope sc(c, ST_FWD_ROWS, s);
    RowArgs r;
    r.cores = c.cores; r.meta = c.d_meta; r.counts = p.counts; r.row_pfx = p.row_pfx; r.row_c3 = p.row_c3;
    r.c3_begin = c.c3_begin; r.pfx_t = p.pfx_t; r.pbuf = p.pbuf; r.rows = p.rows; r.seg_off = p.seg_off; r.sbag = p.sbag; r.out = out;
    r.n1 = c.n1; r.n1s = a.n1s; r.n2 = c.n2; r.N = c.N; r.NC = c.NC;
    const int grid = grid_for(c, cdiv(c.U_cap, RW_RCH), RW_WARPS, TTEMB_FWD_ROWS_GRID);
    const dim3 g(grid), b(RW_WARPS * 32);
    if (c.R == 32) {
      if (c.n3 == 4) launch_pdl(k_rows_fwd2<4, 4>, g, b, rows_smem(4, 32), s, r);
      else launch_pdl(k_rows_fwd2<8, 4>, g, b, rows_smem(8, 32), s, r);
    } else if (c.R == 64) {
      if (c.n3 == 4) launch_pdl(k_rows_fwd2<4, 8>, g, b, rows_smem(4, 64), s, r);
      else launch_pdl(k_rows_fwd2<8, 8>, g, b, rows_smem(8, 64), s, r);
    } else {
      if (c.n3 == 4) launch_pdl(k_rows_fwd2<4, 16>, g, b, rows_smem(4, 128), s, r);
      else launch_pdl(k_rows_fwd2<8, 16>, g, b, rows_smem(8, 128), s, r);
    }
  }
  return cudaGetLastError();
}

// Backward row stage (dP stash + dC3) for the fused-eligible shapes.
// Zero the dP rows the backward row kernel accumulates with reductions (plan-dependent, reads
// no parameters: runs at the end of the index stage, i.e. on the pipelined side stream).
cudaError_t run_dp_zero(Ctx& c, cudaStream_t s) {
  const PlanDev& p = c.p;
  RowBwdArgs r;
  r.cores = c.cores; r.grads = c.grads; r.meta = c.d_meta; r.counts = p.counts; r.row_pfx = p.row_pfx;
  r.row_c3 = p.row_c3; r.c3_begin = c.c3_begin; r.pfx_t = p.pfx_t; r.row_seg = p.row_seg; r.pbuf = p.pbuf; r.gbuf = p.gbuf;
  r.dpbuf = p.dpbuf; r.n1 = c.n1; r.n2 = c.n2; r.N = c.N; r.NC = c.NC; r.R = c.R;
  k_dp_zero2<<<grid_for(c, c.P_cap, 8, 8), 256, 0, s>>>(r);
  return cudaGetLastError();
}

cudaError_t run_rows_bwd2(Ctx& c, cudaStream_t s) {
  const PlanDev& p = c.p;
  RowBwdArgs r;
  r.cores = c.cores; r.grads = c.grads; r.meta = c.d_meta; r.counts = p.counts; r.row_pfx = p.row_pfx;
  r.row_c3 = p.row_c3; r.c3_begin = c.c3_begin; r.pfx_t = p.pfx_t; r.row_seg = p.row_seg; r.pbuf = p.pbuf; r.gbuf = p.gbuf;
  r.dpbuf = p.dpbuf; r.n1 = c.n1; r.n2 = c.n2; r.N = c.N; r.NC = c.NC; r.R = c.R;
  r.exp = exp_bits();
  // (the dP rows of chunk-straddling prefixes were zeroed at the end of the index stage)
  // 32-wide r slices (RL = 1, 24 warps / SM) for n3 = 4: at c4 88 us vs 98.7 us for 64-wide slices
  // (RL = 2, 16 warps / SM); 64-wide for n3 = 8 (c5 R = 64: 3.83 vs 3.99 ms, R = 128: 7.61 vs
  // 7.94 ms); TTEMB_EXP bit 2048 flips the choice for comparison
  const bool narrow = c.R == 32 || ((c.n3 == 4) != ((exp_bits() & 2048) != 0));
  const int sw = narrow ? 32 : 64;
  const int grid = grid_for(c, cdiv(c.U_cap, RW_RCH) * (c.R / sw), RW_WARPS, narrow ? 3 : 2);
  const void* f = narrow ? rows_bwd_kernel_rl1(c.n3, c.R, c.n1 * c.n2) : rows_bwd_kernel(c.n3, c.R, c.n1 * c.n2);
  if (!f) return cudaErrorInvalidValue;
  void* args[] = {&r};
  return launch_pdl_ptr(f, dim3(grid), dim3(RW_WARPS * 32), rows_bwd_smem(c.n3, sw), s, args);
}

// Forward contractions on tcgen05: P (k_prefix_fwd) then rows (k_rows_fwd2).
cudaError_t run_tc_fwd(Ctx& c, float* out, cudaStream_t s) { return run_fused_fwd(c, out, s); }

// Backward contractions: dP / dC3 row stage, then the prefix GEMMs (dC2, dA) with the fused update.
cudaError_t run_tc_bwd(Ctx& c, float lr, cudaStream_t s) {
  cudaError_t e;
  {
    StageScope sc(c, ST_BWD_ROWS, s);
    e = run_rows_bwd2(c, s);
  }
  if (!(c.flags & TTEMB_FUSED_UPDATE)) c.mark_bucket(1, s);   // every C3 gradient is final
  if (e == cudaSuccess) e = run_prefix_bwd(c, lr, s);
  return e;
}

}  // namespace ttemb
