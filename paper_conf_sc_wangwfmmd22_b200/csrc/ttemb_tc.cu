// ttemb_tc.cu -- rank-64 tensor-core path (sm_100a): the rank-R contractions on tcgen05
// (kind::tf32, 3xTF32 split, fp32 accumulate in TMEM) and the row stages as
// high-occupancy warp-per-row-chunk kernels.  SURVEY 8(a) rows a5, a6, a9, a10, a12.
//
//   forward   k_tc_fwd    P^T = C2^T . A1^T per group  (Reuse buffer) -> Pbuf
//             k_rows_fwd  E_u = P_q . C3[i3_u]         (Eq. 2)  -> out (one id per bag)
//                                                               or rows[u] (pooled later)
//   backward  k_rows_bwd  dP_q += G_u . C3[i3_u]^T     (Eq. 6)    -> dPbuf
//                         dC3[i3_u] += P_q^T G_u       (red.global.add.v4, L2-resident)
//             k_tc_bwd2   dC2[i2] += A2 . D2^T,  dA^T = X2 . D1^T  per i2-group
//                         (dC2 reduced in TMEM over the whole group, no atomics; fused
//                          SGD/Adagrad update of the C2 slice the CTA owns)
// Operands are staged as K-major "CM" core-matrix layouts (tc.cuh):
//   A1 = CM(m, r1)  X1 = CM(c, r1)  X2 = CM(r1, c)  A2 = CM(r1, m)  D1 = CM(m, c)  D2 = CM(c, m)
// Tiles: 64 rows (q, j1) x one j2 block (64 columns of C2) x K = 64.  The next chunk's
// operands are prefetched into registers while the current chunk's MMAs run, and the
// next group is claimed one ahead.  The row kernels walk 16 consecutive unique rows per
// warp, so Zipf-hot prefixes (hundreds of rows) spread over many warps.
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <vector>

#include "tc.cuh"
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int TR = 64, TMT = 64, TCW = 64, TNRB = 8, TNT = 256;
constexpr uint32_t TCM = 64 * 64 * 4;          // bytes of one 64x64 fp32 CM matrix
constexpr int RCH = 16;                        // unique rows per warp item
constexpr int SPS = TR + 4;                    // smem P row stride (floats)

struct TcArgs {
  float* cores;
  float* grads;
  float* state;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_i1, *pfx_t, *row_seg, *row_i3,
      *row_pfx, *seg_off, *sbag;
  uint32_t* grp_arow;   // [P]  C1 row index (floats / R) of sorted prefix q at j1 = 0
  unsigned long long* grp_c2;   // [NG] float offset of group g's C2 slice
  float* pbuf;          // [P][n1][NC]  prefix products (Reuse buffer)
  float* dpbuf;         // [P][n1][NC]  dL/dP per prefix
  float* rows;          // [U][N]
  const float* gbuf;    // [U][N]  aggregated row gradients
  float* dabuf;         // [P][n1][R] dC1 partials
  float* out;           // [B][T][N]
  uint32_t* work;
  int n1, n2, n3, N, NC, n1s;
  unsigned long long* trace;   // optional per-CTA role timers (TTEMB_TRACE), 16 slots per CTA
  int dbg;                     // TTEMB_DBG bit mask (timing experiments only; results invalid)
  int f_nmb, f_trm, f_nst;   // forward GEMM geometry (k_tc_fwd): M blocks, tile rows, raw slots
  float lr, eps;
  int opt, fused;
};

__device__ __forceinline__ float* fat(float* base, uint32_t off) {
  return reinterpret_cast<float*>(reinterpret_cast<char*>(base) + off);
}
__device__ __forceinline__ void st_split4(float* hi, float* lo, uint32_t off, float4 v) {
  const float4 h = make_float4(tc::tf32_hi(v.x), tc::tf32_hi(v.y), tc::tf32_hi(v.z), tc::tf32_hi(v.w));
  *reinterpret_cast<float4*>(fat(hi, off)) = h;
  *reinterpret_cast<float4*>(fat(lo, off)) = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
}
__device__ __forceinline__ void red_add_v4(float* addr, float4 v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(v.x), "f"(v.y),
               "f"(v.z), "f"(v.w)
               : "memory");
}

// 3xTF32 64x64 (K = 64) product of two K-major CM matrices into TMEM column base d.
__device__ __forceinline__ void mma3(uint32_t d, const float* ah, const float* al, const float* bh,
                                     const float* bl, bool accumulate) {
  const uint32_t id = tc::idesc_tf32(64, 64, false, false);
  const uint32_t sah = tc::smem_u32(ah), sal = tc::smem_u32(al);
  const uint32_t sbh = tc::smem_u32(bh), sbl = tc::smem_u32(bl);
#pragma unroll
  for (int kk = 0; kk < 8; ++kk) {
    const uint32_t o = kk * 2 * TNRB * 128;
    const uint64_t dah = tc::sdesc(sah + o, TNRB * 128, 128), dal = tc::sdesc(sal + o, TNRB * 128, 128);
    const uint64_t dbh = tc::sdesc(sbh + o, TNRB * 128, 128), dbl = tc::sdesc(sbl + o, TNRB * 128, 128);
    tc::mma_tf32(d, dah, dbh, id, (accumulate || kk > 0) ? 1u : 0u);
    tc::mma_tf32(d, dah, dbl, id, 1u);
    tc::mma_tf32(d, dal, dbh, id, 1u);
  }
}

__device__ __forceinline__ void publish() {   // generic smem writes -> tensor-core reads
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
}

// Float4 "pattern" loads of a 64x64 tile of a row-major matrix (row stride ld) at
// (row0, col0): ROWQ = 4 rows of one column (for CM(col, row)), COLQ = 4 columns of one row
// (for CM(row, col)).  Element e = tid + 256 k, k < 4.
__device__ __forceinline__ void load_rowq(float4 (&v)[4], const float* base, size_t ld, int nrows) {
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int e = threadIdx.x + TNT * k;
    const int c = e & 63, rq = e >> 6;
    float x[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) x[i] = (4 * rq + i < nrows) ? __ldg(base + (size_t)(4 * rq + i) * ld + c) : 0.f;
    v[k] = make_float4(x[0], x[1], x[2], x[3]);
  }
}
__device__ __forceinline__ void load_colq(float4 (&v)[4], const float* base, size_t ld, int nrows) {
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int e = threadIdx.x + TNT * k;
    const int r = e & 63, cq = e >> 6;
    v[k] = r < nrows ? __ldg(reinterpret_cast<const float4*>(base + (size_t)r * ld + 4 * cq))
                     : make_float4(0.f, 0.f, 0.f, 0.f);
  }
}
// Store a pattern into its CM layout: rowq -> CM(col, 4 rows), colq -> CM(row, 4 cols).
__device__ __forceinline__ void store_pat(float* hi, float* lo, const float4 (&v)[4]) {
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int e = threadIdx.x + TNT * k;
    st_split4(hi, lo, tc::cm_off(e & 63, 4 * (e >> 6), TNRB), v[k]);
  }
}

// Per-m-tile row table in shared memory: for tile row m = (q, j1):
//   rowp[m] = p * n1 + j1      (row of pbuf / dpbuf / dabuf)
//   rowa[m] = i1_p * n1 + j1   (row of C1)        -- 0xffffffff past the tile
__device__ __forceinline__ void fill_table(const TcArgs& a, uint32_t* rowp, uint32_t* rowa,
                                           uint32_t qa, int npq) {
  const int m = threadIdx.x;
  if (m < 64) {
    const int rows = npq << a.n1s;
    uint32_t vp = 0xffffffffu, va = 0xffffffffu;
    if (m < rows) {
      const uint32_t p = a.grp_pfx[qa + (m >> a.n1s)];
      const uint32_t j1 = m & ((1 << a.n1s) - 1);
      vp = (p << a.n1s) + j1;
      va = (a.pfx_i1[p] << a.n1s) + j1;
    }
    rowp[m] = vp;
    rowa[m] = va;
  }
}

// Tile matrix X[m][col] with row m at src + tab[m] * ld (rows with tab == ~0 read as 0):
// ROWQ = 4 consecutive m of one column (for CM(col, m)), COLQ = 4 columns of one m (CM(m, col)).
__device__ __forceinline__ void load_tab(float4 (&v)[4], const float* src, size_t ld, const uint32_t* tab,
                                         bool rowq) {
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int e = threadIdx.x + TNT * k;
    if (rowq) {
      const int c = e & 63, mq = e >> 6;
      float x[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t r = tab[4 * mq + i];
        x[i] = r != 0xffffffffu ? __ldg(src + (size_t)r * ld + c) : 0.f;
      }
      v[k] = make_float4(x[0], x[1], x[2], x[3]);
    } else {
      const int m = e & 63, cq = e >> 6;
      const uint32_t r = tab[m];
      v[k] = r != 0xffffffffu ? __ldg(reinterpret_cast<const float4*>(src + (size_t)r * ld + 4 * cq))
                              : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
}

__device__ __forceinline__ const float* c2_slice(const TcArgs& a, uint32_t g) {
  return a.cores + a.meta[a.grp_t[g]].c2_off + (size_t)a.grp_i2[g] * TR * a.NC;
}

// ------------------------------------------------------------------------------------
// Forward GEMM, transposed so the prefix rows are the MMA N dimension:
//   P^T[c][m] = sum_r1 C2[i2][r1][c] . C1[i1_m][j1_m][r1]      (Reuse buffer)
// M = c (blocks of 128, MN-major operand straight from the row-major C2 slice),
// N = tile rows rounded up to 16 (K-major C1 rows), K = r1 in stages of 16.
// Warp roles (288 threads): warps 0-3 load stages with cp.async (no register staging)
// and write the 3xTF32 "lo" copies; warp 8 issues the MMAs; warps 4-7 drain the TMEM
// accumulator (double-buffered across tiles) into pbuf[(p, j1)][c] with coalesced stores.
// Rows of a tile are whole prefixes of one i2-group (up to fg.trm rows).
// ------------------------------------------------------------------------------------
constexpr int F_LOAD = 128, F_THREADS = 288, F_KS = 16, F_MAXNS = 8;

// Per-step gather tables for the group GEMMs: C1 row of every sorted prefix and the C2
// slice offset of every group (one level of indirection for the pipelined loaders).
__global__ void k_tc_prep(TcArgs a) {
  const uint32_t P = a.counts[kCntP], NG = a.counts[kCntNG];
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < max(P, NG); q += gridDim.x * blockDim.x) {
    if (q < P) {
      const uint32_t p = a.grp_pfx[q];
      a.grp_arow[q] = (uint32_t)(a.meta[a.pfx_t[p]].c1_off / TR) + (a.pfx_i1[p] << a.n1s);
    }
    if (q < NG) a.grp_c2[q] = a.meta[a.grp_t[q]].c2_off + (unsigned long long)a.grp_i2[q] * TR * a.NC;
  }
}

// TTEMB_TRACE instrumentation: clock64 intervals accumulated in registers (trc[k]) and
// written by each role's leader thread at kernel end to trace[16 * blockIdx.x + k].
#define TT_T0(v) long long v = a.trace ? clock64() : 0
#define TT_ADD(k, v, cond)                                                        \
  do {                                                                            \
    if (a.trace) {                                                                \
      const long long _n = clock64();                                             \
      trc[k] += (unsigned long long)(_n - (v));                                   \
      v = _n;                                                                     \
    }                                                                             \
  } while (0)

struct FwdSmemCtl {
  uint64_t landed[F_MAXNS], full[2], empty[2], accfull[2], accempty[2], tfull[4], tempty[4];
  uint32_t cmd[8][4];        // per stage (s & 7): acc slot, k-stage, N, flags (1 last, 2 done)
  uint32_t srows[8];         // per stage (s & 7): tile rows
  uint32_t tinfo[4][2];      // tile ring (loaders -> epilogue): first prefix, rows (~0 = done)
  uint32_t tmem;
  uint32_t rowp[2][128];     // per accumulator slot: pbuf row of each tile row (epilogue-built)
};

// Shared memory: NS linear staging slots filled by the bulk-copy (TMA) engine -- stage =
// 16 consecutive r1 rows of the C2 slice (one contiguous 16*NC*4-byte copy) + 16 r1 of
// every tile row's C1 row (one 64-byte copy per row) -- then 2 converted slots of "hi"
// (raw fp32 in MMA layouts: C2 part MN-major mn32_off, C1 part K-major CM) and 2 of "lo"
// (x - trunc_tf32(x), same layouts).  The loaders convert stage s - LAG while up to LAG
// newer stages are in flight; the MMA warp consumes converted stages.
__global__ void __launch_bounds__(F_THREADS, 1) k_tc_fwd(TcArgs a) {
  extern __shared__ __align__(1024) char smem_raw[];
  __shared__ FwdSmemCtl ctl;
  char* const smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);   // swizzle atoms
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const int NS = a.f_nst, TRM = a.f_trm, MNX = a.f_nmb * 128;
  const uint32_t SS = 64u * (a.NC + TRM);            // staging bytes per stage (C2 rows, C1 rows)
  const uint32_t SC = 64u * (MNX + TRM);             // converted bytes per stage (hi or lo)
  const uint32_t C1OFF = 64u * MNX;                  // C1 part offset inside a converted stage
  const uint32_t HIB = (uint32_t)NS * SS, LOB = HIB + 2 * SC;
  if (tid == 0) {
    for (int b = 0; b < NS; ++b) tc::mbar_init(&ctl.landed[b], 1);
    for (int b = 0; b < 2; ++b) { tc::mbar_init(&ctl.full[b], F_LOAD); tc::mbar_init(&ctl.empty[b], 1); }
    for (int s = 0; s < 2; ++s) { tc::mbar_init(&ctl.accfull[s], 1); tc::mbar_init(&ctl.accempty[s], 128); }
    for (int s = 0; s < 4; ++s) { tc::mbar_init(&ctl.tfull[s], 1); tc::mbar_init(&ctl.tempty[s], 128); }
    tc::fence_mbar_init();
  }
  if (w == 8) tc::tmem_alloc(&ctl.tmem, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t sbase = tc::smem_u32(smem);
  const uint32_t NG = a.counts[kCntNG];
  const int TPP = TRM >> a.n1s;                        // prefixes per tile
  unsigned long long trc[14];
#pragma unroll
  for (int k = 0; k < 14; ++k) trc[k] = 0;
  const long long t_start = a.trace ? clock64() : 0;

  if (w < 4) {
    // ------------------------------- loaders -------------------------------
    const int t = tid;
    const uint32_t LAG = (uint32_t)NS - 2;             // stages in flight behind the newest
    uint32_t s = 0, i = 0;
    auto convert = [&](uint32_t sf) {                  // staging -> hi / lo MMA layouts
      const uint32_t b = sf % NS, l = sf & 1;
      TT_T0(tt);
      tc::named_sync(1, F_LOAD);                       // previous convert done (staging reuse)
      tc::mbar_wait(&ctl.landed[b], (sf / NS) & 1);
      TT_ADD(2, tt, t == 0);
      tc::mbar_wait(&ctl.empty[l], ((sf >> 1) & 1) ^ 1);
      TT_ADD(3, tt, t == 0);
      const char* st = smem + (size_t)b * SS;
      char* hi = smem + HIB + (size_t)l * SC;
      char* lo = smem + LOB + (size_t)l * SC;
      if (!(a.dbg & 2)) {
        const int cpr = a.NC >> 2;
        for (int e = t; e < F_KS * cpr; e += F_LOAD) {
          const int k = e / cpr, c4 = e - k * cpr;
          const float4 x = *reinterpret_cast<const float4*>(st + 16 * e);
          const uint32_t off = tc::mn32_off(4 * c4, k, MNX);
          *reinterpret_cast<float4*>(hi + off) = x;
          *reinterpret_cast<float4*>(lo + off) =
              make_float4(x.x - tc::tf32_trunc(x.x), x.y - tc::tf32_trunc(x.y), x.z - tc::tf32_trunc(x.z),
                          x.w - tc::tf32_trunc(x.w));
        }
        if (t < (int)ctl.srows[sf & 7]) {
#pragma unroll
          for (int u = 0; u < F_KS / 4; ++u) {
            const float4 x = *reinterpret_cast<const float4*>(st + 64 * a.NC + 64 * t + 16 * u);
            const uint32_t off = C1OFF + tc::cm_off(t, 4 * u, TRM >> 3);
            *reinterpret_cast<float4*>(hi + off) = x;
            *reinterpret_cast<float4*>(lo + off) =
                make_float4(x.x - tc::tf32_trunc(x.x), x.y - tc::tf32_trunc(x.y), x.z - tc::tf32_trunc(x.z),
                            x.w - tc::tf32_trunc(x.w));
          }
        }
      }
      tc::fence_async_smem();
      tc::mbar_arrive(&ctl.full[l]);
      TT_ADD(4, tt, t == 0);
    };
    // Static round-robin group schedule; the next tile's metadata is loaded two stages
    // ahead of its use so no dependent global-load chain sits between tiles.
    const uint32_t j1 = t & ((1u << a.n1s) - 1);
    uint32_t g = blockIdx.x, q0 = 0, q1 = 0, qa = 0;
    unsigned long long c2o = 0;
    uint32_t arow = 0;                                 // C1 row index of this thread's tile row
    if (g < NG) {
      q0 = a.grp_off[g]; q1 = a.grp_off[g + 1]; c2o = a.grp_c2[g]; qa = q0;
      if ((int)t < (int)(min((uint32_t)TPP, q1 - qa) << a.n1s)) arow = a.grp_arow[qa + (t >> a.n1s)] + j1;
    }
    while (g < NG) {
      const int rows = (int)min((uint32_t)TPP, q1 - qa) << a.n1s;
      const int n16 = (rows + 15) & ~15;
      const uint32_t slot = i & 1;
      if (t == 0) {                                    // tile ring entry for the epilogue
        tc::mbar_wait(&ctl.tempty[i & 3], ((i >> 2) & 1) ^ 1);
        ctl.tinfo[i & 3][0] = qa; ctl.tinfo[i & 3][1] = (uint32_t)rows;
        tc::mbar_arrive(&ctl.tfull[i & 3]);
      }
      const float* C2s = a.cores + c2o;
      const float* A1r = a.cores + (size_t)arow * TR;
      // next tile
      const bool same = qa + TPP < q1;
      const uint32_t ng = same ? g : g + gridDim.x;
      uint32_t nq0 = q0, nq1 = q1, narow = 0;
      unsigned long long nc2 = c2o;
#pragma unroll 1
      for (int ks = 0; ks < TR / F_KS; ++ks, ++s) {
        const uint32_t b = s % NS;
        TT_T0(tt);
        if (t == 0) {
          ctl.cmd[s & 7][0] = slot; ctl.cmd[s & 7][1] = (uint32_t)ks; ctl.cmd[s & 7][2] = (uint32_t)n16;
          ctl.cmd[s & 7][3] = ks == TR / F_KS - 1 ? 1u : 0u;
          ctl.srows[s & 7] = (uint32_t)rows;
          tc::mbar_arrive_tx(&ctl.landed[b], 64u * (a.NC + rows));
          if (!(a.dbg & 4)) tc::bulk_g2s(sbase + b * SS, C2s + (size_t)ks * F_KS * a.NC, 64u * a.NC, &ctl.landed[b]);
          else tc::bulk_g2s(sbase + b * SS, C2s, 64u * a.NC, &ctl.landed[b]);
        }
        if (t < rows) tc::bulk_g2s(sbase + b * SS + 64u * a.NC + 64u * t, A1r + ks * F_KS, 64u, &ctl.landed[b]);
        TT_ADD(0, tt, t == 0);
        if (ks == 0 && !same && ng < NG) { nq0 = a.grp_off[ng]; nq1 = a.grp_off[ng + 1]; nc2 = a.grp_c2[ng]; }
        if (ks == 2 && ng < NG) {
          const uint32_t nqa = same ? qa + TPP : nq0;
          if ((int)t < (int)(min((uint32_t)TPP, nq1 - nqa) << a.n1s)) narow = a.grp_arow[nqa + (t >> a.n1s)] + j1;
        }
        TT_ADD(1, tt, t == 0);
        if (s >= LAG) convert(s - LAG);
      }
      ++i;
      if (same) { qa += TPP; }
      else { g = ng; q0 = nq0; q1 = nq1; qa = nq0; c2o = nc2; }
      arow = narow;
    }
    for (uint32_t sf = s >= LAG ? s - LAG : 0; sf < s; ++sf) convert(sf);
    // termination: a "done" tile for the epilogue, a done command for the MMA warp
    if (t == 0) {
      tc::mbar_wait(&ctl.tempty[i & 3], ((i >> 2) & 1) ^ 1);
      ctl.tinfo[i & 3][1] = 0xffffffffu;
      tc::mbar_arrive(&ctl.tfull[i & 3]);
    }
    tc::mbar_wait(&ctl.empty[s & 1], ((s >> 1) & 1) ^ 1);
    if (t == 0) ctl.cmd[s & 7][3] = 2u;
    tc::mbar_arrive(&ctl.full[s & 1]);
  } else if (w == 8) {
    // ------------------------------- MMA issuer -------------------------------
    const uint32_t tacc = ctl.tmem;
    uint32_t i = 0;
    for (uint32_t s = 0;; ++s) {
      const uint32_t l = s & 1;
      TT_T0(tt);
      tc::mbar_wait(&ctl.full[l], (s >> 1) & 1);
      TT_ADD(6, tt, lane == 0);
      tc::fence_after();
      const uint32_t slot = ctl.cmd[s & 7][0], ks = ctl.cmd[s & 7][1], n16 = ctl.cmd[s & 7][2], fl = ctl.cmd[s & 7][3];
      if (fl & 2u) break;
      if (ks == 0) { tc::mbar_wait(&ctl.accempty[slot], ((i >> 1) & 1) ^ 1); tc::fence_after(); }
      TT_ADD(7, tt, lane == 0);
      if (lane == 0 && !(a.dbg & 8)) {
        const uint32_t id = tc::idesc_tf32(128, (int)n16, true, false);
        const uint32_t rh = sbase + HIB + l * SC, rl = sbase + LOB + l * SC;
        const uint32_t sboA = (uint32_t)(MNX >> 5) * 512, lboB = (uint32_t)(TRM >> 3) * 128;
#pragma unroll
        for (int kk = 0; kk < F_KS / 8; ++kk) {
          const uint32_t ao = kk * 2 * sboA, bo = C1OFF + kk * 2 * lboB;
          const uint64_t bh = tc::sdesc(rh + bo, lboB, 128), bl = tc::sdesc(rl + bo, lboB, 128);
          for (int mb = 0; mb < a.f_nmb; ++mb) {
            const uint64_t ah = tc::sdesc_l(rh + ao + mb * 2048, 512, sboA, 1);
            const uint64_t al = tc::sdesc_l(rl + ao + mb * 2048, 512, sboA, 1);
            const uint32_t d = tacc + slot * 256 + mb * TRM;
            tc::mma_tf32(d, ah, bh, id, (ks > 0 || kk > 0) ? 1u : 0u);
            tc::mma_tf32(d, ah, bl, id, 1u);
            tc::mma_tf32(d, al, bh, id, 1u);
          }
        }
      }
      if (lane == 0) {
        tc::commit(&ctl.empty[l]);
        if (fl & 1u) tc::commit(&ctl.accfull[slot]);
      }
      __syncwarp();
      TT_ADD(8, tt, lane == 0);
      if (fl & 1u) ++i;
    }
  } else {
    // ------------------------------- epilogue -------------------------------
    const uint32_t tacc = ctl.tmem;
    const int q = w & 3;
    const int et = tid - 128;
    for (uint32_t i = 0;; ++i) {
      const uint32_t slot = i & 1;
      TT_T0(tt);
      tc::mbar_wait(&ctl.tfull[i & 3], (i >> 2) & 1);
      TT_ADD(9, tt, et == 0);
      const uint32_t qa = ctl.tinfo[i & 3][0], rows = ctl.tinfo[i & 3][1];
      tc::mbar_arrive(&ctl.tempty[i & 3]);
      if (rows == 0xffffffffu) break;
      if (et < (int)rows) ctl.rowp[slot][et] = (a.grp_pfx[qa + (et >> a.n1s)] << a.n1s) + (et & ((1 << a.n1s) - 1));
      tc::named_sync(2, 128);
      TT_ADD(10, tt, et == 0);
      tc::mbar_wait(&ctl.accfull[slot], (i >> 1) & 1);
      TT_ADD(11, tt, et == 0);
      tc::fence_after();
      for (int mb = 0; mb < a.f_nmb; ++mb) {
        const int c = mb * 128 + 32 * q + lane;
        for (int j0 = 0; j0 < (int)rows; j0 += 32) {
          float v[32];
          tc::tmem_ld32(tc::taddr(tacc + slot * 256 + mb * TRM + j0, 32 * q, 0), v);
          if (c < a.NC && !(a.dbg & 1)) {
#pragma unroll
            for (int j = 0; j < 32; ++j)
              if (j0 + j < (int)rows) a.pbuf[(size_t)ctl.rowp[slot][j0 + j] * a.NC + c] = v[j];
          }
        }
      }
      tc::fence_before();
      tc::mbar_arrive(&ctl.accempty[slot]);
      TT_ADD(12, tt, et == 0);
      if (a.trace) trc[13] += 1;
    }
  }
  if (a.trace) {
    const bool lead = tid == 0 || tid == 256 || tid == 128;
    if (lead)
      for (int k = 0; k < 14; ++k)
        if (trc[k]) a.trace[16 * blockIdx.x + k] = trc[k];
    if (tid == 0) a.trace[16 * blockIdx.x + 14] = (unsigned long long)(clock64() - t_start);
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (w == 8) tc::tmem_dealloc(ctl.tmem, 512);
}

// ------------------------------------------------------------------------------------
// Row stages: one warp per chunk of RCH consecutive unique rows; the next row's C3 slice,
// G row and (on a prefix change) P_q are prefetched into registers while the current row
// computes from shared memory.
// ------------------------------------------------------------------------------------
struct WarpSmem {
  float sP[16 * SPS];      // P_q rows j12 < 16, r < 64
  float sC3[TR * 8];       // C3[i3_u] : [r][j3], n3 <= 8
  float sG[128];           // G_u : [j12][j3]
};

template <int N3>
struct RowPref {
  static constexpr int C3L = TR * N3 / 4 / 32;   // float4 of a C3 slice per lane
  float4 c3[C3L];
  float4 p[8];                                  // P_q: J12 * 16 float4 <= 256
  float4 g;                                     // G_u: J12 * N3 / 4 <= 32 float4
  uint32_t q;
};

template <int N3>
__device__ __forceinline__ void row_prefetch(RowPref<N3>& f, const TcArgs& a, uint32_t u, int J12,
                                             bool load_p, bool load_g, uint32_t cur) {
  const int lane = threadIdx.x & 31;
  const uint32_t q = a.row_pfx[u];
  const float4* c3 = reinterpret_cast<const float4*>(a.cores + a.meta[a.pfx_t[q]].c3_off +
                                                     (size_t)a.row_i3[u] * TR * N3);
#pragma unroll
  for (int i = 0; i < RowPref<N3>::C3L; ++i) f.c3[i] = __ldg(c3 + lane + 32 * i);
  if (load_p && q != cur) {
    const float4* src = reinterpret_cast<const float4*>(a.pbuf + (size_t)q * J12 * TR);
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int e = lane + 32 * i;
      if (e < J12 * (TR / 4)) f.p[i] = __ldg(src + e);
    }
  }
  if (load_g && lane < J12 * N3 / 4) f.g = __ldg(reinterpret_cast<const float4*>(a.gbuf + (size_t)u * a.N) + lane);
  f.q = q;
}

template <int N3>
__device__ __forceinline__ void row_stage(WarpSmem& ws, const RowPref<N3>& f, int J12, bool store_p,
                                          bool store_g) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int i = 0; i < RowPref<N3>::C3L; ++i) reinterpret_cast<float4*>(ws.sC3)[lane + 32 * i] = f.c3[i];
  if (store_p) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int e = lane + 32 * i;
      if (e < J12 * (TR / 4)) {
        const int j = e >> 4, r4 = e & 15;
        *reinterpret_cast<float4*>(ws.sP + j * SPS + 4 * r4) = f.p[i];
      }
    }
  }
  if (store_g && lane < J12 * N3 / 4) reinterpret_cast<float4*>(ws.sG)[lane] = f.g;
}

// forward: E_u[j12][j3] = sum_r P_q[j12][r] C3_u[r][j3]; lane = (j12 = lane / 2, r half)
template <int N3>
__global__ void __launch_bounds__(128) k_rows_fwd(TcArgs a) {
  __shared__ __align__(16) WarpSmem ws_all[4];
  WarpSmem& ws = ws_all[threadIdx.x >> 5];
  const int lane = threadIdx.x & 31, J12 = a.n1 * a.n2;
  const uint32_t U = tt_rows(a.counts);   // TT rows only (hybrid: dense rows follow)
  const int j12 = lane >> 1, rh = lane & 1;
  const int64_t nch = (U + RCH - 1) / RCH;
  for (int64_t ch = (int64_t)blockIdx.x * 4 + (threadIdx.x >> 5); ch < nch; ch += (int64_t)gridDim.x * 4) {
    const uint32_t u0 = (uint32_t)ch * RCH, u1 = min(u0 + RCH, U);
    RowPref<N3> f;
    uint32_t cur = 0xffffffffu;
    row_prefetch<N3>(f, a, u0, J12, true, false, cur);
    for (uint32_t u = u0; u < u1; ++u) {
      const bool newp = f.q != cur;
      __syncwarp();
      row_stage<N3>(ws, f, J12, newp, false);
      cur = f.q;
      __syncwarp();
      if (u + 1 < u1) row_prefetch<N3>(f, a, u + 1, J12, true, false, cur);
      float acc[N3];
#pragma unroll
      for (int j = 0; j < N3; ++j) acc[j] = 0.f;
      if (j12 < J12) {
        const float* pr = ws.sP + j12 * SPS + 32 * rh;
        const float* c3 = ws.sC3 + 32 * rh * N3;
#pragma unroll 8
        for (int r = 0; r < 32; r += 4) {
          const float4 p4 = *reinterpret_cast<const float4*>(pr + r);
          const float pv[4] = {p4.x, p4.y, p4.z, p4.w};
#pragma unroll
          for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < N3; j += 4) {
              const float4 c4 = *reinterpret_cast<const float4*>(c3 + (r + i) * N3 + j);
              acc[j] = fmaf(pv[i], c4.x, acc[j]);
              acc[j + 1] = fmaf(pv[i], c4.y, acc[j + 1]);
              acc[j + 2] = fmaf(pv[i], c4.z, acc[j + 2]);
              acc[j + 3] = fmaf(pv[i], c4.w, acc[j + 3]);
            }
        }
      }
#pragma unroll
      for (int j = 0; j < N3; ++j) acc[j] += __shfl_xor_sync(0xffffffffu, acc[j], 1);
      if (rh == 0 && j12 < J12) {
        float* d = a.rows + (size_t)u * a.N + j12 * N3;
#pragma unroll
        for (int j = 0; j < N3; j += 4) *reinterpret_cast<float4*>(d + j) = make_float4(acc[j], acc[j + 1], acc[j + 2], acc[j + 3]);
      }
    }
  }
}

// dPbuf rows of prefixes whose rows straddle a chunk boundary are accumulated with atomics:
// zero them first.
__global__ void __launch_bounds__(256) k_dp_zero(TcArgs a) {
  const uint32_t P = a.counts[kCntP];
  const int J12R = a.n1 * a.n2 * TR;
  const int lane = threadIdx.x & 31;
  for (uint32_t q = blockIdx.x * 8 + (threadIdx.x >> 5); q < P; q += gridDim.x * 8) {
    const uint32_t r0 = a.row_seg[q], r1 = a.row_seg[q + 1];
    if (r0 / RCH == (r1 - 1) / RCH) continue;
    float4* d = reinterpret_cast<float4*>(a.dpbuf + (size_t)q * J12R);
    for (int f = lane; f < J12R / 4; f += 32) d[f] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

// backward row stage: dP_q[j12][r] += sum_j3 G_u[j12][j3] C3_u[r][j3]   (lane = j12, r half)
//                     dC3[i3][r][j3] += sum_j12 P_q[j12][r] G_u[j12][j3] (lane = r pair)
template <int N3>
__global__ void __launch_bounds__(128) k_rows_bwd(TcArgs a) {
  __shared__ __align__(16) WarpSmem ws_all[4];
  WarpSmem& ws = ws_all[threadIdx.x >> 5];
  const int lane = threadIdx.x & 31, J12 = a.n1 * a.n2;
  const uint32_t U = tt_rows(a.counts);   // TT rows only (hybrid: dense rows follow)
  const int j12 = lane >> 1, rh = lane & 1;
  const int64_t nch = (U + RCH - 1) / RCH;
  for (int64_t ch = (int64_t)blockIdx.x * 4 + (threadIdx.x >> 5); ch < nch; ch += (int64_t)gridDim.x * 4) {
    const uint32_t u0 = (uint32_t)ch * RCH, u1 = min(u0 + RCH, U);
    uint32_t cur = 0xffffffffu;
    float dp[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) dp[i] = 0.f;
    auto flush = [&](uint32_t q) {
      if (j12 >= J12) return;
      const uint32_t r0 = a.row_seg[q], r1 = a.row_seg[q + 1];
      float* d = a.dpbuf + ((size_t)q * J12 + j12) * TR + 32 * rh;
      const bool whole = (r0 / RCH == (r1 - 1) / RCH);
#pragma unroll
      for (int i = 0; i < 32; i += 4) {
        const float4 v = make_float4(dp[i], dp[i + 1], dp[i + 2], dp[i + 3]);
        if (whole) *reinterpret_cast<float4*>(d + i) = v;
        else red_add_v4(d + i, v);
      }
#pragma unroll
      for (int i = 0; i < 32; ++i) dp[i] = 0.f;
    };
    RowPref<N3> f;
    row_prefetch<N3>(f, a, u0, J12, true, true, cur);
    for (uint32_t u = u0; u < u1; ++u) {
      const uint32_t q = f.q;
      const size_t c3o = a.meta[a.pfx_t[q]].c3_off + (size_t)a.row_i3[u] * TR * N3;
      if (q != cur && cur != 0xffffffffu) flush(cur);
      const bool newp = q != cur;
      __syncwarp();
      row_stage<N3>(ws, f, J12, newp, true);
      cur = q;
      __syncwarp();
      if (u + 1 < u1) row_prefetch<N3>(f, a, u + 1, J12, true, true, cur);
      if (j12 < J12) {     // dP: 32 r of this lane's half
        float gg[N3];
#pragma unroll
        for (int j = 0; j < N3; j += 4) {
          const float4 g4 = *reinterpret_cast<const float4*>(ws.sG + j12 * N3 + j);
          gg[j] = g4.x; gg[j + 1] = g4.y; gg[j + 2] = g4.z; gg[j + 3] = g4.w;
        }
        const float* c3 = ws.sC3 + 32 * rh * N3;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
#pragma unroll
          for (int j = 0; j < N3; j += 4) {
            const float4 c4 = *reinterpret_cast<const float4*>(c3 + i * N3 + j);
            dp[i] = fmaf(gg[j], c4.x, dp[i]);
            dp[i] = fmaf(gg[j + 1], c4.y, dp[i]);
            dp[i] = fmaf(gg[j + 2], c4.z, dp[i]);
            dp[i] = fmaf(gg[j + 3], c4.w, dp[i]);
          }
        }
      }
      {                    // dC3: r = 2 lane, 2 lane + 1
        float acc[2][N3];
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
          for (int j = 0; j < N3; ++j) acc[i][j] = 0.f;
        for (int jj = 0; jj < J12; ++jj) {
          const float2 p2 = *reinterpret_cast<const float2*>(ws.sP + jj * SPS + 2 * lane);
#pragma unroll
          for (int j = 0; j < N3; j += 4) {
            const float4 g4 = *reinterpret_cast<const float4*>(ws.sG + jj * N3 + j);
            acc[0][j] = fmaf(p2.x, g4.x, acc[0][j]); acc[0][j + 1] = fmaf(p2.x, g4.y, acc[0][j + 1]);
            acc[0][j + 2] = fmaf(p2.x, g4.z, acc[0][j + 2]); acc[0][j + 3] = fmaf(p2.x, g4.w, acc[0][j + 3]);
            acc[1][j] = fmaf(p2.y, g4.x, acc[1][j]); acc[1][j + 1] = fmaf(p2.y, g4.y, acc[1][j + 1]);
            acc[1][j + 2] = fmaf(p2.y, g4.z, acc[1][j + 2]); acc[1][j + 3] = fmaf(p2.y, g4.w, acc[1][j + 3]);
          }
        }
        float* d = a.grads + c3o + (size_t)(2 * lane) * N3;
#pragma unroll
        for (int i = 0; i < 2; ++i)
#pragma unroll
          for (int j = 0; j < N3; j += 4)
            red_add_v4(d + i * N3 + j, make_float4(acc[i][j], acc[i][j + 1], acc[i][j + 2], acc[i][j + 3]));
      }
    }
    if (cur != 0xffffffffu) flush(cur);
  }
}

// Backward GEMMs per i2-group, warp-specialised: warps 0-7 (256 threads) stage operands,
// run the epilogues and the fused C2 update; warp 8 issues the tcgen05 MMAs.
//   dA^T [r1][m]  = X2 . D1^T   (TMEM, accumulated over the tile's chunks)
//   dC2  [r1][c] += A2 . D2^T   (TMEM per chunk, accumulated over the group's m-tiles)
// X2 / D1 / D2 are double-buffered; full[b] (one arrival per producer thread) hands a staged step
// to the MMA warp together with a small command word, empty[b] (tcgen05.commit) hands the
// buffer back.  Row addresses of a tile are computed once per tile, so the per-chunk
// prefetch is a plain burst of loads.
constexpr int WS_PROD = 256, WS_ALL = 288;

__global__ void __launch_bounds__(WS_ALL, 1) k_tc_bwd2(TcArgs a) {
  extern __shared__ __align__(128) char smem[];
  float* const base = reinterpret_cast<float*>(smem);
  constexpr int MF = TCM / 4;
  auto x2h = [&](int b) { return base + (6 * b + 0) * MF; };
  auto x2l = [&](int b) { return base + (6 * b + 1) * MF; };
  auto d1h = [&](int b) { return base + (6 * b + 2) * MF; };
  auto d1l = [&](int b) { return base + (6 * b + 3) * MF; };
  auto d2h = [&](int b) { return base + (6 * b + 4) * MF; };
  auto d2l = [&](int b) { return base + (6 * b + 5) * MF; };
  float* a2h = base + 12 * MF;
  float* a2l = base + 13 * MF;
  __shared__ uint64_t full[2], empty[2];
  __shared__ uint32_t cmd[2][2];
  __shared__ uint32_t s_tmem, s_g[2], s_rowp[2][64], s_rowa[2][64];
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    for (int b = 0; b < 2; ++b) {
      tc::mbar_init(&full[b], WS_PROD);
      tc::mbar_init(&empty[b], 1);
    }
    tc::fence_mbar_init();
    s_g[0] = atomicAdd(a.work, 1u);
    s_g[1] = atomicAdd(a.work, 1u);
  }
  if (w == 0) tc::tmem_alloc(&s_tmem, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tDA = s_tmem, tDC2 = s_tmem + 64;
  const uint32_t NG = a.counts[kCntNG];
  const int PPT = TMT >> a.n1s, NCH = a.NC / TCW;

  if (w == 8) {
    // ------------------------------ MMA issuer ------------------------------
    uint32_t fph0 = 0, fph1 = 0;
    for (uint32_t s = 0;; ++s) {
      const int b = s & 1;
      tc::mbar_wait(&full[b], b ? fph1 : fph0);
      if (b) fph1 ^= 1u; else fph0 ^= 1u;
      tc::fence_after();
      const uint32_t c0 = cmd[b][0], c1 = cmd[b][1];
      if (c0 == 0xffffffffu) break;
      if (lane == 0) {
        const int k = (int)c0;
        mma3(tDA, x2h(b), x2l(b), d1h(b), d1l(b), k > 0);               // dA^T [r1][m]
        mma3(tDC2 + 64 * k, a2h, a2l, d2h(b), d2l(b), c1 != 0);          // dC2  [r1][c]
        tc::commit(&empty[b]);
      }
      __syncwarp();
    }
  } else {
    // --------------------------- producers / epilogue ---------------------------
    const int q4 = w & 3, half = w >> 2;
    uint32_t eph0 = 0, eph1 = 0;
    int pend0 = 0, pend1 = 0;
    auto wait_buf = [&](int b) {
      if (b == 0 ? pend0 : pend1) {
        tc::mbar_wait(&empty[b], b == 0 ? eph0 : eph1);
        if (b == 0) { eph0 ^= 1u; pend0 = 0; } else { eph1 ^= 1u; pend1 = 0; }
        tc::fence_after();
      }
    };
    auto finish_chunk = [&](int kc, int b, size_t c2o) {
      float v[32];
      tc::tmem_ld32(tc::taddr(tDC2 + 64 * kc, 32 * q4, 32 * half), v);
      if (lane < 16) {
        const int r1 = 16 * q4 + lane;
        const size_t b0 = c2o + (size_t)r1 * a.NC + kc * TCW + 32 * half;
        if (a.fused) {
          float x[32];
#pragma unroll
          for (int j = 0; j < 32; j += 4) {
            const uint32_t off = tc::cm_off(r1, 32 * half + j, TNRB);
            const float4 h = *reinterpret_cast<const float4*>(fat(x2h(b), off));
            const float4 l = *reinterpret_cast<const float4*>(fat(x2l(b), off));
            x[j] = h.x + l.x; x[j + 1] = h.y + l.y; x[j + 2] = h.z + l.z; x[j + 3] = h.w + l.w;
          }
          if (a.opt == TTEMB_SGD) {
#pragma unroll
            for (int j = 0; j < 32; j += 4)
              *reinterpret_cast<float4*>(a.cores + b0 + j) =
                  make_float4(x[j] - a.lr * v[j], x[j + 1] - a.lr * v[j + 1], x[j + 2] - a.lr * v[j + 2],
                              x[j + 3] - a.lr * v[j + 3]);
          } else {
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              const float4 s4 = *reinterpret_cast<const float4*>(a.state + b0 + j);
              const float s0 = s4.x + v[j] * v[j], s1 = s4.y + v[j + 1] * v[j + 1];
              const float s2 = s4.z + v[j + 2] * v[j + 2], s3 = s4.w + v[j + 3] * v[j + 3];
              *reinterpret_cast<float4*>(a.state + b0 + j) = make_float4(s0, s1, s2, s3);
              *reinterpret_cast<float4*>(a.cores + b0 + j) =
                  make_float4(x[j] - a.lr * v[j] / (sqrtf(s0) + a.eps), x[j + 1] - a.lr * v[j + 1] / (sqrtf(s1) + a.eps),
                              x[j + 2] - a.lr * v[j + 2] / (sqrtf(s2) + a.eps), x[j + 3] - a.lr * v[j + 3] / (sqrtf(s3) + a.eps));
            }
          }
        } else {
#pragma unroll
          for (int j = 0; j < 32; j += 4)
            *reinterpret_cast<float4*>(a.grads + b0 + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
        }
      }
      tc::fence_before();
    };
    // hand step (buffer b) to the MMA warp
    auto post = [&](int b, uint32_t c0, uint32_t c1) {
      tc::fence_async_smem();
      tc::fence_before();
      if (tid == 0) { cmd[b][0] = c0; cmd[b][1] = c1; }
      tc::mbar_arrive(&full[b]);
    };
    // per-tile row offsets: COLQ row (one per thread), ROWQ rows (4 per k)
    uint32_t rcol = 0, racol = 0;
    uint32_t rrow[16];
    auto tile_rows = [&](int tbuf) {
      rcol = s_rowp[tbuf][tid & 63];
      racol = s_rowa[tbuf][tid & 63];
#pragma unroll
      for (int k = 0; k < 4; ++k)
#pragma unroll
        for (int i = 0; i < 4; ++i) rrow[4 * k + i] = s_rowp[tbuf][4 * ((tid >> 6) + 4 * k) + i];
    };
    auto load_d = [&](float4 (&p1)[4], float4 (&p2)[4], int c0) {
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int cq = (tid >> 6) + 4 * k;
        p1[k] = rcol != 0xffffffffu ? __ldg(reinterpret_cast<const float4*>(a.dpbuf + (size_t)rcol * a.NC + c0 + 4 * cq))
                                   : make_float4(0.f, 0.f, 0.f, 0.f);
        float x[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const uint32_t r = rrow[4 * k + i];
          x[i] = r != 0xffffffffu ? __ldg(a.dpbuf + (size_t)r * a.NC + c0 + (tid & 63)) : 0.f;
        }
        p2[k] = make_float4(x[0], x[1], x[2], x[3]);
      }
    };
    auto load_a2 = [&](float4 (&p)[4], const float* C1t, int tbuf) {   // A2 = CM(r1, m): 4 m of one r1
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float x[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const uint32_t r = s_rowa[tbuf][4 * ((tid >> 6) + 4 * k) + i];
          x[i] = r != 0xffffffffu ? __ldg(C1t + (size_t)r * TR + (tid & 63)) : 0.f;
        }
        p[k] = make_float4(x[0], x[1], x[2], x[3]);
      }
    };
    uint32_t g = s_g[0], gnext = s_g[1];
    int tb = 0;
    uint32_t s = 0;
    float4 px[4], pd1[4], pd2[4], pa[4];
    if (g < NG) {
      if (tid < 64) fill_table(a, s_rowp[0], s_rowa[0], a.grp_off[g], (int)min((uint32_t)PPT, a.grp_off[g + 1] - a.grp_off[g]));
      tc::named_sync(1, WS_PROD);
      tile_rows(0);
      load_colq(px, c2_slice(a, g), a.NC, TR);
      load_d(pd1, pd2, 0);
      load_a2(pa, a.cores + a.meta[a.grp_t[g]].c1_off, 0);
    }
    while (g < NG) {
      const uint32_t i2 = a.grp_i2[g];
      const uint32_t q0 = a.grp_off[g], q1 = a.grp_off[g + 1];
      const size_t c2o = a.meta[a.grp_t[g]].c2_off + (size_t)i2 * TR * a.NC;
      const float* C2s = a.cores + c2o;
      const uint32_t nmt = (q1 - q0 + PPT - 1) / PPT;
      for (uint32_t mt = 0; mt < nmt; ++mt) {
        const bool last_tile = (mt + 1 == nmt);
        wait_buf(0);
        wait_buf(1);
        tc::named_sync(1, WS_PROD);                            // previous tile's epilogue done
        store_pat(a2h, a2l, pa);                               // A2 = CM(r1, m)
        const uint32_t s0 = s;
        for (int k = 0; k < NCH; ++k, ++s) {
          const int b = s & 1;
          wait_buf(b);                                         // MMA(s-2) done: buffer b free
          if (last_tile && k >= 2) finish_chunk(k - 2, b, c2o);
          store_pat(x2h(b), x2l(b), px);                       // X2 = CM(r1, c)
          store_pat(d1h(b), d1l(b), pd1);                      // D1 = CM(m, c)
          store_pat(d2h(b), d2l(b), pd2);                      // D2 = CM(c, m)
          post(b, (uint32_t)k, mt > 0 ? 1u : 0u);
          if (b == 0) pend0 = 1; else pend1 = 1;
          if (k + 1 < NCH) {                                   // prefetch the next step
            load_colq(px, C2s + (k + 1) * TCW, a.NC, TR);
            load_d(pd1, pd2, (k + 1) * TCW);
          } else {
            uint32_t ng = g, nqa = q0 + (mt + 1) * PPT;
            if (mt + 1 >= nmt) { ng = gnext; nqa = ng < NG ? a.grp_off[ng] : 0; }
            if (ng < NG) {
              if (tid < 64) fill_table(a, s_rowp[tb ^ 1], s_rowa[tb ^ 1], nqa, (int)min((uint32_t)PPT, a.grp_off[ng + 1] - nqa));
              tc::named_sync(1, WS_PROD);
              tile_rows(tb ^ 1);
              load_colq(px, c2_slice(a, ng), a.NC, TR);
              load_d(pd1, pd2, 0);
              load_a2(pa, a.cores + a.meta[a.grp_t[ng]].c1_off, tb ^ 1);
            }
          }
        }
        // drain the tile: last two steps (their buffers hold chunks NCH-2, NCH-1)
        for (int kc = (NCH >= 2 ? NCH - 2 : 0); kc < NCH; ++kc) {
          const int b = (int)((s0 + kc) & 1);
          wait_buf(b);
          if (last_tile) finish_chunk(kc, b, c2o);
        }
        {   // dA^T -> dabuf[(p, j1)][r1]
          float v[32];
          tc::tmem_ld32(tc::taddr(tDA, 32 * q4, 32 * half), v);
          if (lane < 16) {
            const int r1 = 16 * q4 + lane;
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              const uint32_t r = s_rowp[tb][32 * half + j];
              if (r != 0xffffffffu) a.dabuf[(size_t)r * TR + r1] = v[j];
            }
          }
          tc::fence_before();
        }
        tb ^= 1;
      }
      tc::named_sync(1, WS_PROD);
      if (tid == 0) s_g[1] = atomicAdd(a.work, 1u);
      tc::named_sync(1, WS_PROD);
      g = gnext;
      gnext = s_g[1];
    }
    const int b = s & 1;                                       // tell the MMA warp to stop
    wait_buf(b);
    post(b, 0xffffffffu, 0u);
    wait_buf(b ^ 1);
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (w == 0) tc::tmem_dealloc(tDA, 512);
}

TcArgs make_tc_args(Ctx& c, float lr, uint32_t* work, float* out) {
  const PlanDev& p = c.p;
  TcArgs a;
  a.cores = c.cores; a.grads = c.grads; a.state = c.state; a.meta = c.d_meta;
  a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2;
  a.grp_pfx = p.grp_pfx; a.pfx_i1 = p.pfx_i1; a.pfx_t = p.pfx_t; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.row_pfx = p.row_pfx; a.seg_off = p.seg_off; a.sbag = p.sbag;
  a.grp_arow = p.grp_arow; a.grp_c2 = p.grp_c2;
  a.pbuf = p.pbuf; a.dpbuf = p.dpbuf; a.rows = p.rows; a.gbuf = p.gbuf; a.dabuf = p.dabuf;
  a.out = out; a.work = work; a.trace = nullptr;
  a.dbg = knobs().dbg;
  a.n1 = c.n1; a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.NC = c.NC;
  a.n1s = c.n1 == 1 ? 0 : c.n1 == 2 ? 1 : c.n1 == 4 ? 2 : 3;
  a.f_nmb = (c.NC + 127) / 128;
  a.f_trm = a.f_nmb <= 2 ? 128 : a.f_nmb == 3 ? 80 : 64;
  {   // staging slots: NS * 64 (NC + TRM) + 4 * 64 (MNX + TRM) bytes <= 220 KB
    const size_t sc = 64u * (a.f_nmb * 128 + a.f_trm), ss = 64u * (c.NC + a.f_trm);
    a.f_nst = (int)std::min<size_t>(F_MAXNS, (220 * 1024 - 4 * sc) / ss);
  }
  a.lr = lr; a.eps = c.eps; a.opt = c.opt; a.fused = (c.flags & TTEMB_FUSED_UPDATE) ? 1 : 0;
  return a;
}

size_t fwd_smem(const TcArgs& a) {
  return (size_t)a.f_nst * 64u * (a.NC + a.f_trm) + 4u * 64u * (a.f_nmb * 128 + a.f_trm) + 1024;
}
constexpr size_t kTcBwdSmem = 14 * TCM;

}  // namespace

bool tc_eligible(const Ctx& c) {
  return !(c.flags & TTEMB_FP32_CORES) && c.R == TR && (c.n3 == 4 || c.n3 == 8) &&
         (c.n1 == 1 || c.n1 == 2 || c.n1 == 4 || c.n1 == 8) && c.n1 * c.n2 <= 16 && c.n2 <= 7;
}

cudaError_t configure_tc(Ctx& c) {
  if (!tc_eligible(c)) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(k_tc_fwd, cudaFuncAttributeMaxDynamicSharedMemorySize, 222 * 1024);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_tc_bwd2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTcBwdSmem);
}

// Forward contractions: P (tcgen05) then rows / direct output.
cudaError_t run_tc_fwd(Ctx& c, float* out, cudaStream_t s) {
  if (fused_eligible(c)) return run_fused_fwd(c, out, s);
  TcArgs a = make_tc_args(c, 0.f, c.p.work + 0, out);
  {
    StageScope sc(c, ST_FWD_PREFIX, s);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count));
    static unsigned long long* trace = nullptr;
    if (knobs().trace) {
      if (!trace) cudaMalloc(&trace, sizeof(unsigned long long) * 16 * grid);
      cudaMemsetAsync(trace, 0, sizeof(unsigned long long) * 16 * grid, s);
      a.trace = trace;
    }
    k_tc_prep<<<grid_for(c, std::max(c.P_cap, c.NG_cap), 256, 4), 256, 0, s>>>(a);
    k_tc_fwd<<<grid, F_THREADS, fwd_smem(a), s>>>(a);
    if (a.trace) {
      std::vector<unsigned long long> h(16 * grid);
      cudaMemcpyAsync(h.data(), trace, h.size() * 8, cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
      double m[16] = {};
      for (int b = 0; b < grid; ++b) for (int k = 0; k < 16; ++k) m[k] += (double)h[16 * b + k] / grid;
      fprintf(stderr, "[trace fwd] tiles/CTA %.1f loader-total %.0f | loader: issue %.0f prefetch %.0f landed %.0f empty %.0f convert %.0f other %.0f"
              " | mma: full %.0f accempty %.0f issue %.0f | epi: tinfo %.0f table %.0f accfull %.0f drain %.0f (cycles/CTA)\n",
              m[13], m[14], m[0], m[1], m[2], m[3], m[4], m[5], m[6], m[7], m[8], m[9], m[10], m[11], m[12]);
    }
  }
  {
    StageScope sc(c, ST_FWD_ROWS, s);
    const int grid = grid_for(c, cdiv(c.U_cap, RCH), 4, 8);
    if (c.n3 == 4) k_rows_fwd<4><<<grid, 128, 0, s>>>(a);
    else k_rows_fwd<8><<<grid, 128, 0, s>>>(a);
  }
  return cudaGetLastError();
}

// Backward contractions: dP / dC3 row stage, then the group GEMMs (dC2, dA).
cudaError_t run_tc_bwd(Ctx& c, float lr, cudaStream_t s) {
  if (fused_eligible(c)) {
    cudaError_t e;
    {
      StageScope sc(c, ST_BWD_ROWS, s);
      e = run_rows_bwd2(c, s);
    }
    if (e == cudaSuccess) e = run_prefix_bwd(c, lr, s);
    return e;
  }
  TcArgs a = make_tc_args(c, lr, c.p.work + 1, nullptr);
  {
    StageScope sc(c, ST_BWD_ROWS, s);
    k_dp_zero<<<grid_for(c, c.P_cap, 8, 8), 256, 0, s>>>(a);
    const int grid = grid_for(c, cdiv(c.U_cap, RCH), 4, 8);
    if (c.n3 == 4) k_rows_bwd<4><<<grid, 128, 0, s>>>(a);
    else k_rows_bwd<8><<<grid, 128, 0, s>>>(a);
  }
  {
    StageScope sc(c, ST_BWD_PREFIX, s);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count));
    k_tc_bwd2<<<grid, WS_ALL, kTcBwdSmem, s>>>(a);
  }
  return cudaGetLastError();
}

}  // namespace ttemb
