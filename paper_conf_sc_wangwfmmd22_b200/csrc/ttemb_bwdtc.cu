// ttemb_bwdtc.cu -- prefix backward on tcgen05, sm_100a.
//
// One persistent CTA per SM walks the i2-groups g = (t, i2) (static round robin).  Per tile
// of <= 64 rows m = (prefix q, j1) of the group, with dP = dL/dP from the row stage (dpbuf):
//   dC2[i2]^T[c][r1] += sum_m dP[m][c] . C1[i1_m][j1_m][r1]      (Eq. 6 read as left^T . dL/de
//                       . right^T; the left factor of C2 is the C1 slice)
//       M = 128 c per block, N = 64 r1, K = 64 m: A = dP^T held in TENSOR MEMORY (lane = c,
//       column = m, written by the loader threads), B = C1^T as an MN-major
//       SWIZZLE_128B_BASE32B operand in shared memory (the C1 row pieces stored as loaded);
//       accumulated in TMEM over all tiles of the group (no atomics, no partial buffers).
//   dA[m][r1] = sum_c dP[m][c] . C2[i2][r1][c]                  (the C1 gradient partials)
//       one SS MMA per K step: M = 128 = the tile's dP rows stacked as [dP_hi; dP_lo] (rows
//       0-63 as the TMA landed them, 64-127 the lo parts the loaders wrote next to them),
//       N = 2 KR = [C2_hi | C2_lo] rows (likewise), K = c, both K-major SWIZZLE_128B operands in
//       shared memory; the accumulator holds dP_{hi,lo} . C2_{hi,lo} in its four quadrants (3xTF32
//       plus the lo.lo term) and the epilogue sums them.  (Round 2 measured this 1.10x faster
//       than dP in TMEM written by the loaders with two N = KR MMAs per K step: the loaders'
//       tensor-memory stores were on the critical path.)
//       The epilogue adds dA straight into the C1 gradient (red.global.add.v4, L2-resident).
// At the group's last tile the dC2 accumulator is drained: with TTEMB_FUSED_UPDATE and SGD the
// C2 slice is updated in place by reductions straight from TMEM (the paper's fused TT core
// update; the slice has no other reader once its last tile's MMAs completed); for
// Adagrad (read-modify-write of the slice and its state) or unfused, dC2 is stored and fused
// Adagrad writes dC2 to a per-group scratch and finishes in k_c2_update.
// fp32 accuracy: 3xTF32 (hi = raw fp32, read by the tensor core with truncation; lo =
// x - trunc_tf32(x)); scripts/tc_probe3.cu measures the TMEM-A form.
//
// Warp roles (448 threads): 0-7 loaders (lo rows of the dP and C2 chunks, C1^T hi / lo, dP^T ->
// TMEM with the lo part computed in registers), 8 MMA issuer, 9-12 epilogue (dA -> dC1 reductions, dC2 -> gradient /
// fused update), 13 TMA producer (per K-chunk: 2-D TMA loads of the tile's dP rows and the C2
// slice rows, SWIZZLE_128B, up to Y_NST chunks ahead).
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <vector>

#include "tc.cuh"
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int YT = 64;                          // tile rows (prefix, j1)
constexpr int Y_LW = 8, Y_EW = 4;
constexpr int Y_THREADS = (Y_LW + 1 + Y_EW + 1) * 32;
constexpr int Y_MMA_W = Y_LW;
constexpr int Y_TMA_W = Y_LW + 1 + Y_EW;           // the TMA producer warp
constexpr int Y_NST = 3;                        // chunk stages (TMA)
constexpr int Y_GI = 64;                        // work units per CTA whose metadata is staged in shared memory

// Shape of the kernel for rank KR: a work unit is (i2-group, BPU c-blocks of 128); K-chunks of
// CK columns of c.  R = 64: one unit per group (both c-blocks), 64-column chunks.  R = 128: one
// unit per c-block (the dC2 / dA accumulators are N = 128 wide), 32-column chunks (the C2 chunk
// [CK][KR] hi + lo then fits three stages).
template <int KR> struct YShape {
  static constexpr int BPU = KR <= 64 ? 2 : 1;
  static constexpr int CK = KR <= 64 ? 64 : 32;
  // stage = [dP chunk | C2 chunk] as TMA SWIZZLE_128B boxes of 32 columns (tc::sw128_off); box h
  // of the dP chunk = [hi rows m = 0..63 | lo rows 64..127] (the dA A operand, M = 128), box h of
  // the C2 chunk = [hi rows r1 = 0..KR-1 | lo rows KR..2KR-1] (the dA B operand, N = 2 KR)
  static constexpr uint32_t A2BOX = 2u * YT * 128, B2BOX = 2u * KR * 128;
  static constexpr uint32_t A2 = 2u * YT * CK * 4;                      // dP chunk hi + lo
  static constexpr uint32_t B2 = 2u * KR * CK * 4;                      // C2 chunk hi + lo
  static constexpr uint32_t STAGE = A2 + B2;
  static constexpr uint32_t B1 = 2u * KR * YT * 4;                      // C1^T hi + lo (MN-major)
  static constexpr size_t SMEM = 1024 + B1 + Y_NST * STAGE;
  // TMEM columns
  static constexpr uint32_t T_DPT = 0;                                  // dP^T hi [64 BPU), lo [64 BPU, 128 BPU)
  static constexpr uint32_t T_DC2 = 128 * BPU;                          // dC2^T, KR per c-block
  static constexpr uint32_t T_DA = T_DC2 + KR * BPU;                    // dA quadrants (N = 2 KR)
  static_assert(T_DA + 2 * KR <= 512, "TMEM budget");
  static_assert(SMEM <= 227 * 1024, "shared memory budget");
};

struct YArgs {
  float* cores;
  float* grads;
  float* state;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *pfx_i1, *pfx_t;
  const uint32_t* grp_arow;               // [P]  C1 row index (floats / R) of prefix q, j1 = 0
  const unsigned long long* grp_c2;       // [NG] float offset of the group's C2 slice
  unsigned long long c2_begin;            // float offset of the C2 region (tm_c2 row 0)
  const float* dpbuf;                     // [P][n1][NC]
  float* dc2buf;                          // fused Adagrad: dC2 of group g at g R NC (slice layout)
  const uint32_t* unit_snake;             // [NU] unit at static position p (balanced by tile count)
  uint32_t* work;
  int n1, n1s, NC, nblk, tpp, nchunk, R;
  float lr, eps;
  int opt, fused;
  unsigned long long* trace;              // TTEMB_TRACE: 32 cycle counters per CTA (timing only)
  int pf;                                 // L2 prefetch distance in groups (0 = off)
  int exp;                                // TTEMB_EXP bits (timing experiments only; results invalid)
};

struct YCtl {
  uint64_t a1_full, a1_free;              // dP^T in TMEM + C1^T in smem (per tile)
  uint64_t s_full[Y_NST], s_free[Y_NST];  // K-chunk stages (loaders done / MMAs done)
  uint64_t s_tma[Y_NST];                  // K-chunk stage landed (TMA transactions)
  uint64_t d1_full, d1_free;              // dC2 accumulator (per group)
  uint64_t d2_full, d2_free;              // dA accumulator (per tile)
  uint64_t u_full[4], u_empty[4];
  uint32_t ring[4][5];                    // group, first prefix, #prefixes, flags (1 first, 2 last, 4 done), unit block
  uint32_t claim[2];
  uint32_t tmem;
  // this CTA's work units (static round robin) loaded once, in parallel, at kernel start: first /
  // last prefix and C2 slice offset of the unit's group, so no unit boundary waits on a
  // global-memory round trip
  uint32_t gq0[Y_GI], gq1[Y_GI], gu[Y_GI];
  unsigned long long gc2[Y_GI];
};

__device__ __forceinline__ float lo32(float x) { return x - tc::tf32_trunc(x); }

template <int KR>
__global__ void __launch_bounds__(Y_THREADS, 1)
k_prefix_bwd(const __grid_constant__ CUtensorMap tm_dp, const __grid_constant__ CUtensorMap tm_c2, YArgs a) {
  pdl_wait();
  pdl_trigger();
  using S = YShape<KR>;
  constexpr int BPU = S::BPU, CK = S::CK;
  extern __shared__ __align__(128) char smem_raw[];
  __shared__ YCtl ctl;
  char* const smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);
  char* const b1 = smem;                                 // C1^T hi | lo
  char* const stg = smem + S::B1;                        // stages: [A2 | B2 hi | B2 lo]
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const uint32_t NG = a.counts[kCntNG];
  const uint32_t UPG = (uint32_t)(a.nblk + BPU - 1) / BPU;   // work units per group
  const uint32_t NU = NG * UPG;
  if (tid == 0) {
    tc::mbar_init(&ctl.a1_full, Y_LW * 32);
    tc::mbar_init(&ctl.a1_free, 1);
    for (int s = 0; s < Y_NST; ++s) {
      tc::mbar_init(&ctl.s_full[s], Y_LW * 32); tc::mbar_init(&ctl.s_free[s], 1); tc::mbar_init(&ctl.s_tma[s], 1);
    }
    tc::mbar_init(&ctl.d1_full, 1);
    tc::mbar_init(&ctl.d1_free, Y_EW * 32);
    tc::mbar_init(&ctl.d2_full, 1);
    tc::mbar_init(&ctl.d2_free, Y_EW * 32);
    for (int s = 0; s < 4; ++s) { tc::mbar_init(&ctl.u_full[s], 1); tc::mbar_init(&ctl.u_empty[s], 1 + Y_EW); }
    tc::fence_mbar_init();
  }
  if (w == Y_MMA_W) tc::tmem_alloc(&ctl.tmem, 512);
  for (int i = tid; i < Y_GI; i += blockDim.x) {
    const uint32_t pu = blockIdx.x + (uint32_t)i * gridDim.x;   // static position -> unit
    if (pu < NU) {
      const uint32_t u = a.unit_snake[pu], g = u / UPG;
      ctl.gu[i] = u; ctl.gq0[i] = a.grp_off[g]; ctl.gq1[i] = a.grp_off[g + 1]; ctl.gc2[i] = a.grp_c2[g];
    }
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = ctl.tmem;
#ifdef TTEMB_TRACE_BUILD   // role timers (build with TTEMB_NVCC_FLAGS=-DTTEMB_TRACE_BUILD, run with TTEMB_TRACE=1)
  unsigned long long trc[32] = {};
  long long _tt = 0;
  const long long t_start = a.trace ? clock64() : 0;
#define YT0() do { if (a.trace) _tt = clock64(); } while (0)
#define YTA(k) do { if (a.trace) { const long long _n = clock64(); trc[k] += (unsigned long long)(_n - _tt); _tt = _n; } } while (0)
#else
#define YT0() do { } while (0)
#define YTA(k) do { } while (0)
#endif
  // TMEM columns (YShape): dP^T hi / lo of the unit's c-blocks (lane = c, column = m), the dC2^T
  // accumulators (lane = c, column = r1), dA (lanes m: dP_hi rows, 64 + m: dP_lo rows; column =
  // r1) and the current chunk's [dP_hi; dP_lo] (dA A operand, column = c of the chunk).
  const int tpp = a.tpp, NC = a.NC;

  // Jobs = (unit, tile, K-chunk) in a static round-robin unit order (loaders, TMA producer)
  // Job.u = static position (G0 + k GS), Job.unit = the unit dealt to it (unit_snake)
  struct Job { uint32_t u, unit, q0, q1, qa; int ck, crow; unsigned long long c2; };
  const uint32_t G0 = blockIdx.x, GS = gridDim.x;
  auto start = [&](Job& j, uint32_t u) {   // unit metadata (staged in shared memory)
    j.u = u; j.ck = 0;
    if (u < NU) {
      const uint32_t k = (u - G0) / GS;
      if (k < (uint32_t)Y_GI) { j.unit = ctl.gu[k]; j.q0 = j.qa = ctl.gq0[k]; j.q1 = ctl.gq1[k]; j.c2 = ctl.gc2[k]; }
      else {
        j.unit = a.unit_snake[u];
        const uint32_t g = j.unit / UPG;
        j.q0 = j.qa = a.grp_off[g]; j.q1 = a.grp_off[g + 1]; j.c2 = a.grp_c2[g];
      }
      j.crow = (int)((j.c2 - a.c2_begin) / (unsigned long long)NC);   // C2 region row of r1 = 0
    }
  };
  auto advance = [&](Job& j) {
    if (++j.ck < a.nchunk) return;
    j.ck = 0;
    j.qa += tpp;
    if (j.qa >= j.q1) start(j, j.u + GS);
  };
  if (w < Y_LW) {
    // ------------------------------- loaders -------------------------------
    // Per K-chunk the TMA producer has landed the tile's 64 dP rows (rows past the tile belong to
    // the next group or lie past the stash; they are masked to zero here) and the KR rows of the
    // C2 slice in the B operand's K-major SWIZZLE_128B layout (hi); each thread writes the lo parts
    // of its share of the C2 chunk, and dP (lanes m) and dP^T (lanes c) go to tensor memory with
    // their lo parts made in registers.
    const int mb = tid & 63;                  // C1^T staging map: row mb, float4 columns (tid >> 6) + 4 k
    constexpr int C2F = KR * CK / 4 / 256;    // float4 of the C2 chunk per thread (lo split)
    uint32_t ui = 0, sp = 0;                  // tile counter, processed chunk counter
    Job P;
    start(P, G0);
    // C1 rows of a tile (row mb of the tile, float4 columns (tid >> 6) + 4 k), loaded one tile
    // ahead (NT = the next tile of the processing job) so their latency overlaps a whole tile.
    constexpr int C1F = KR / 16;
    float4 cvn[C1F];
    auto load_c1 = [&](const Job& j, float4* cv) {
      const uint32_t np = j.u < NU ? min((uint32_t)tpp, j.q1 - j.qa) : 0u;
      const bool ok = mb < (int)(np << a.n1s) && !(a.exp & 16);
      const float4* src = reinterpret_cast<const float4*>(
          a.cores + (size_t)(ok ? a.grp_arow[j.qa + (mb >> a.n1s)] + (mb & ((1 << a.n1s) - 1)) : 0u) * KR);
#pragma unroll
      for (int k = 0; k < C1F; ++k) cv[k] = ok ? __ldg(src + (tid >> 6) + 4 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
    };
    load_c1(P, cvn);
    while (P.u < NU) {
      YT0();
      const uint32_t np = min((uint32_t)tpp, P.q1 - P.qa);
      const int rows = (int)(np << a.n1s);              // valid dP rows of the tile
      if (P.ck == 0) {
        const uint32_t fl = (P.qa == P.q0 ? 1u : 0u) | (P.qa + tpp >= P.q1 ? 2u : 0u);
        if (tid == 0) {
          tc::mbar_wait(&ctl.u_empty[ui & 3], ((ui >> 2) & 1) ^ 1);
          ctl.ring[ui & 3][0] = P.unit / UPG; ctl.ring[ui & 3][1] = P.qa; ctl.ring[ui & 3][2] = np;
          ctl.ring[ui & 3][3] = fl; ctl.ring[ui & 3][4] = P.unit % UPG;
          tc::mbar_arrive(&ctl.u_full[ui & 3]);
        }
        // C1^T -> B1 (element (r1, m) = C1 row m, column r1); zero past the tile
        float4 cv[C1F];
#pragma unroll
        for (int k = 0; k < C1F; ++k) cv[k] = cvn[k];
        {   // prefetch the next tile's C1 rows
          Job NT = P;
          NT.qa += tpp;
          if (NT.qa >= NT.q1) start(NT, NT.u + GS);
          load_c1(NT, cvn);
        }
        YTA(0);
        tc::mbar_wait(&ctl.a1_free, (ui & 1) ^ 1);      // previous tile's dC2 GEMM done
        YTA(1);
        tc::fence_after();
        // C1^T as the MN-major (N = r1 contiguous) SWIZZLE_128B_BASE32B operand: the C1 row
        // pieces are stored as they were loaded, one 16-byte store each (hi and lo)
#pragma unroll
        for (int k = 0; k < C1F; ++k) {
          const int r0 = 4 * ((tid >> 6) + 4 * k);
          const uint32_t off = tc::mn32_off(r0, mb, KR);
          const float4 v = cv[k];
          *reinterpret_cast<float4*>(b1 + off) = v;
          *reinterpret_cast<float4*>(b1 + S::B1 / 2 + off) = make_float4(lo32(v.x), lo32(v.y), lo32(v.z), lo32(v.w));
        }
      }
      // chunk P landed
      YTA(2);
      const uint32_t sidx = sp % Y_NST;
      tc::mbar_wait(&ctl.s_tma[sidx], (sp / Y_NST) & 1);
      YTA(3);
      char* a2 = stg + sidx * S::STAGE;
      char* b2 = a2 + S::A2;
      // dP^T first (it reads only the TMA-landed hi rows), so its tensor-memory stores complete
      // while the lo rows are written; no loader-wide barrier: every thread fences its own
      // shared-memory writes and arrives on s_full itself
      {   // dP^T of this chunk -> TMEM (dC2 A operand): thread = column, 32 tile rows; lo in
          // registers.  R = 64: chunk ck covers c-block ck / 2, lane quarters 2 (ck & 1) + {0, 1};
          // R = 128: the unit's block, lane quarter ck & 3.
        const int Q = w & 3;
        const int blk = BPU == 2 ? (P.ck >> 1) : 0;
        const bool mine = BPU == 2 ? ((Q >> 1) == (P.ck & 1) && blk < a.nblk) : (Q == (P.ck & 3));
        if (mine && !(a.exp & 8)) {
          const int cc = BPU == 2 ? 32 * (Q & 1) + lane : lane;   // column inside the chunk
          const int m0 = 32 * (w >> 2);                           // warps 0-3: rows 0..31, 4-7: 32..63
          float x[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            const float v = *reinterpret_cast<const float*>(a2 + tc::sw128_off(m0 + i, cc, 2 * YT));
            x[i] = m0 + i < rows ? v : 0.f;
          }
          tc::tmem_st32(tc::taddr(tm + S::T_DPT + blk * 64 + m0, 32 * Q, 0), x);
#pragma unroll
          for (int i = 0; i < 32; ++i) x[i] = lo32(x[i]);
          tc::tmem_st32(tc::taddr(tm + S::T_DPT + 64 * BPU + blk * 64 + m0, 32 * Q, 0), x);
        }
      }
      YTA(5);
      if (!(a.exp & 4)) {   // lo rows of both chunks: row n + 64 (dP) / n + KR (C2) of a box = lo of
                            // row n (same swizzle phase: 64 % 8 == KR % 8 == 0), elementwise
        constexpr int AF = YT * CK / 4 / 256;
        float4 q[AF + C2F];
        uint32_t o[AF + C2F];
#pragma unroll
        for (int k = 0; k < AF; ++k) {
          const uint32_t e = tid + 256 * k;
          o[k] = (e / (YT * 8)) * S::A2BOX + (e % (YT * 8)) * 16;
          q[k] = *reinterpret_cast<const float4*>(a2 + o[k]);
        }
#pragma unroll
        for (int k = 0; k < C2F; ++k) {
          const uint32_t e = tid + 256 * k;
          o[AF + k] = S::A2 + (e / (KR * 8)) * S::B2BOX + (e % (KR * 8)) * 16;
          q[AF + k] = *reinterpret_cast<const float4*>(a2 + o[AF + k]);
        }
#pragma unroll
        for (int k = 0; k < AF + C2F; ++k)
          *reinterpret_cast<float4*>(a2 + o[k] + (k < AF ? YT * 128 : KR * 128)) =
              make_float4(lo32(q[k].x), lo32(q[k].y), lo32(q[k].z), lo32(q[k].w));
      }
      YTA(6);
      tc::tmem_wait_st();
      tc::fence_async_smem();
      tc::fence_before();
      tc::mbar_arrive(&ctl.s_full[sidx]);
      if (P.ck == a.nchunk - 1) {
        tc::mbar_arrive(&ctl.a1_full);
        ++ui;
      }
      ++sp;
      advance(P);
    }
    if (tid == 0) {
      tc::mbar_wait(&ctl.u_empty[ui & 3], ((ui >> 2) & 1) ^ 1);
      ctl.ring[ui & 3][3] = 4u;
      tc::mbar_arrive(&ctl.u_full[ui & 3]);
    }
  } else if (w == Y_MMA_W) {
    // ------------------------------- MMA issuer -------------------------------
    uint32_t sk = 0, gs = 0;
    for (uint32_t ui = 0;; ++ui) {
      YT0();
      tc::mbar_wait(&ctl.u_full[ui & 3], (ui >> 2) & 1);
      YTA(10);
      const uint32_t fl = ctl.ring[ui & 3][3], ub = ctl.ring[ui & 3][4];
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&ctl.u_empty[ui & 3]);
      if (fl & 4u) break;
      // dA = [dP_hi; dP_lo] . C2_{hi,lo}^T over the K chunks (as they land); N = KR
      tc::mbar_wait(&ctl.d2_free, (ui & 1) ^ 1);
      YTA(11);
      tc::fence_after();
      for (int ck = 0; ck < a.nchunk; ++ck, ++sk) {
        const uint32_t s = sk % Y_NST;
        YTA(13);
        tc::mbar_wait(&ctl.s_full[s], (sk / Y_NST) & 1);
        YTA(12);
        tc::fence_after();
        if (lane == 0) {
          const uint32_t id = tc::idesc_tf32(128, 2 * KR, false, false);
          const uint32_t a2 = tc::smem_u32(stg + s * S::STAGE), b2 = a2 + S::A2;
#pragma unroll
          for (int kk = 0; kk < CK / 8; ++kk) {
            // K-major SWIZZLE_128B: 8 K-columns = 32 bytes inside a 32-column box
            const uint64_t da = tc::sdesc_l(a2 + (kk >> 2) * S::A2BOX + (kk & 3) * 32, 16, 1024, 2);
            const uint64_t db = tc::sdesc_l(b2 + (kk >> 2) * S::B2BOX + (kk & 3) * 32, 16, 1024, 2);
            if (!(a.exp & 32)) tc::mma_tf32(tm + S::T_DA, da, db, id, (ck > 0 || kk > 0) ? 1u : 0u);
          }
          tc::commit(&ctl.s_free[s]);
          if (ck + 1 == a.nchunk) tc::commit(&ctl.d2_full);
        }
        __syncwarp();
      }
      // dC2^T += dP^T . C1  (K = 64 tile rows, N = KR), after the whole tile's dP^T reached TMEM
      YTA(13);
      tc::mbar_wait(&ctl.a1_full, ui & 1);
      YTA(14);
      YTA(15);
      if (fl & 1u) tc::mbar_wait(&ctl.d1_free, (gs & 1) ^ 1);
      tc::fence_after();
      if (lane == 0) {
        const uint32_t id = tc::idesc_tf32(128, KR, false, true);    // B = C1^T MN-major
        const uint32_t bh = tc::smem_u32(b1), bl = bh + S::B1 / 2;
        for (int blk = 0; blk < BPU && (int)ub * BPU + blk < a.nblk; ++blk) {
          const uint32_t d = tm + S::T_DC2 + blk * KR;
#pragma unroll
          for (int kk = 0; kk < YT / 8; ++kk) {
            const uint32_t sbo = (KR / 32) * 512, o = kk * 2 * sbo;   // MN-major, K groups of 4 outermost
            const uint64_t dbh = tc::sdesc_l(bh + o, 512, sbo, 1);
            const uint64_t dbl = tc::sdesc_l(bl + o, 512, sbo, 1);
            const uint32_t ah = tm + S::T_DPT + blk * 64 + kk * 8, al = ah + 64 * BPU;
            if (a.exp & 32) continue;
            tc::mma_tf32_ts(d, ah, dbh, id, ((fl & 1u) && kk == 0) ? 0u : 1u);
            tc::mma_tf32_ts(d, ah, dbl, id, 1u);
            tc::mma_tf32_ts(d, al, dbh, id, 1u);
          }
        }
        tc::commit(&ctl.a1_free);
        if (fl & 2u) tc::commit(&ctl.d1_full);
      }
      __syncwarp();
      YTA(16);
      if (fl & 2u) ++gs;
    }
  } else if (w < Y_TMA_W) {
    // ------------------------------- epilogue -------------------------------
    const int Q = w & 3;
    uint32_t gs = 0;
    for (uint32_t ui = 0;; ++ui) {
      YT0();
      tc::mbar_wait(&ctl.u_full[ui & 3], (ui >> 2) & 1);
      YTA(20);
      const uint32_t g = ctl.ring[ui & 3][0], qa = ctl.ring[ui & 3][1];
      const uint32_t np = ctl.ring[ui & 3][2], fl = ctl.ring[ui & 3][3], ub = ctl.ring[ui & 3][4];
      __syncwarp();
      if (fl & 4u) break;
      const int rows = (int)np << a.n1s;
      // dA: lanes m hold dP_hi (C2_hi + C2_lo), lanes 64 + m dP_lo (C2_hi + C2_lo); both add into dC1
      YTA(25);
      tc::mbar_wait(&ctl.d2_full, ui & 1);
      YTA(21);
      tc::fence_after();
      {
        const int m = (Q & 1) * 32 + lane;               // tile row of this lane
        float v[32];
        float* dst = nullptr;
        if (m < rows)   // grp_arow = C1 row of (prefix, j1 = 0): one load
          dst = a.grads + ((size_t)__ldg(a.grp_arow + qa + (m >> a.n1s)) + (m & ((1 << a.n1s) - 1))) * KR;
        for (int h = 0; h < KR / 32; ++h) {
          tc::tmem_ld32(tc::taddr(tm + S::T_DA + 32 * h, 32 * Q, 0), v);
          {   // + the C2_lo quadrant
            float v2[32];
            tc::tmem_ld32(tc::taddr(tm + S::T_DA + KR + 32 * h, 32 * Q, 0), v2);
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] += v2[i];
          }
          if (dst && !(a.exp & 2)) {
#pragma unroll
            for (int i = 0; i < 32; i += 4)
              asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(dst + 32 * h + i), "f"(v[i]),
                           "f"(v[i + 1]), "f"(v[i + 2]), "f"(v[i + 3])
                           : "memory");
          }
        }
      }
      tc::fence_before();
      tc::mbar_arrive(&ctl.d2_free);
      YTA(22);
      if (fl & 2u) {
        // unit complete: dC2^T [c][r1] -> gradient or fused C2 update (this CTA owns the columns)
        tc::mbar_wait(&ctl.d1_full, gs & 1);
        YTA(23);
        tc::fence_after();
        const unsigned long long so = a.grp_c2[g];
        for (int blk = 0; blk < BPU; ++blk) {
          const int c = ((int)ub * BPU + blk) * 128 + Q * 32 + lane;
          for (int h = 0; h < KR / 32; ++h) {
            float v[32];
            tc::tmem_ld32(tc::taddr(tm + S::T_DC2 + blk * KR + 32 * h, 32 * Q, 0), v);
            if (c < NC && !(a.exp & 1)) {
              const size_t base = so + (size_t)(32 * h) * NC + c;
              if (!a.fused) {
                // unfused: dC2 to the gradient buffer (plain coalesced stores)
#pragma unroll
                for (int i = 0; i < 32; ++i) a.grads[base + (size_t)i * NC] = v[i];
              } else if (a.opt != TTEMB_SGD) {
                // fused Adagrad: dC2 to the per-group scratch (same slice layout); the read-modify-
                // write of C2 and its state runs after the kernel as a bandwidth-bound pass over the
                // touched slices (k_c2_update), which never has to clear it
                float* d = a.dc2buf + (size_t)g * KR * NC + (base - so);
#pragma unroll
                for (int i = 0; i < 32; ++i) d[(size_t)i * NC] = v[i];
              } else {
                // C2 -= lr dC2 as fire-and-forget reductions (each warp instruction covers 32
                // consecutive floats): no read of the old slice, no load latency on this path
#pragma unroll
                for (int i = 0; i < 32; ++i)
                  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(a.cores + base + (size_t)i * NC),
                               "f"(-a.lr * v[i]) : "memory");
              }
            }
          }
        }
        tc::fence_before();
        tc::mbar_arrive(&ctl.d1_free);
        YTA(24);
        ++gs;
      }
      if (lane == 0) tc::mbar_arrive(&ctl.u_empty[ui & 3]);
    }
  } else {
    // ------------------------------- TMA producer -------------------------------
    auto issue = [&](const Job& j, uint32_t sidx) {
      const int c0 = (int)(j.unit % UPG) * BPU * 128 + j.ck * CK;   // first slice column of the chunk
      const uint32_t st = sidx % Y_NST;
      const uint32_t a2 = tc::smem_u32(stg + st * S::STAGE), b2 = a2 + S::A2;
      const int prow = (int)(j.qa << a.n1s);                      // dP stash row of tile row 0
      tc::mbar_arrive_tx(&ctl.s_tma[st], S::A2 / 2 + S::B2 / 2);
#pragma unroll
      for (int h = 0; h < CK / 32; ++h) {
        tc::tma_load_2d(a2 + h * S::A2BOX, &tm_dp, c0 + 32 * h, prow, &ctl.s_tma[st]);
        tc::tma_load_2d(b2 + h * S::B2BOX, &tm_c2, c0 + 32 * h, j.crow, &ctl.s_tma[st]);
      }
    };
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_dp) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(&tm_c2) : "memory");
      Job I;
      start(I, G0);
      for (uint32_t si = 0; I.u < NU; ++si) {
        tc::mbar_wait(&ctl.s_free[si % Y_NST], ((si / Y_NST) & 1) ^ 1);
        issue(I, si);
        advance(I);
      }
    }
    __syncwarp();
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (w == Y_MMA_W) tc::tmem_dealloc(tm, 512);
#ifdef TTEMB_TRACE_BUILD
  if (a.trace) {
    unsigned long long* tb = a.trace + 32 * blockIdx.x;
    if (tid == 0) { for (int k = 0; k < 10; ++k) tb[k] = trc[k]; tb[30] = (unsigned long long)(clock64() - t_start); }
    if (w == Y_MMA_W && lane == 0) for (int k = 10; k < 17; ++k) tb[k] = trc[k];
    if (w == Y_LW + 1 && lane == 0) for (int k = 20; k < 26; ++k) tb[k] = trc[k];
  }
#endif
#undef YT0
#undef YTA
}

}  // namespace

// Fused Adagrad for the C2 slices, from the dC2 the prefix-backward kernel wrote to the per-group
// scratch: s += g^2, C2 -= lr g / (sqrt(s) + eps).
__global__ void __launch_bounds__(256)
k_c2_update(float* __restrict__ cores, float* __restrict__ state, const float* __restrict__ dc2,
            const unsigned long long* __restrict__ grp_c2, const uint32_t* __restrict__ counts,
            uint32_t slice, float lr, float eps) {
  const size_t n4 = (size_t)counts[kCntNG] * (slice / 4);
  for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < n4; e += (size_t)gridDim.x * blockDim.x) {
    const size_t gi = e / (slice / 4), o = grp_c2[gi] + 4 * (e % (slice / 4));
    const float4 g = __ldcs(reinterpret_cast<const float4*>(dc2) + e);
    float4 p = *reinterpret_cast<float4*>(cores + o);
    float4 st = *reinterpret_cast<float4*>(state + o);
    st.x += g.x * g.x; st.y += g.y * g.y; st.z += g.z * g.z; st.w += g.w * g.w;
    p.x -= lr * g.x / (sqrtf(st.x) + eps); p.y -= lr * g.y / (sqrtf(st.y) + eps);
    p.z -= lr * g.z / (sqrtf(st.z) + eps); p.w -= lr * g.w / (sqrtf(st.w) + eps);
    *reinterpret_cast<float4*>(state + o) = st;
    *reinterpret_cast<float4*>(cores + o) = p;
  }
}

cudaError_t configure_bwdtc(Ctx& c) {
  if (!fused_eligible(c)) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(k_prefix_bwd<64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)YShape<64>::SMEM);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(k_prefix_bwd<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)YShape<32>::SMEM);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(k_prefix_bwd<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)YShape<128>::SMEM);
  return e;
}

namespace {
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// fp32 matrix [rows][cols] (row stride cols), boxes of 32 columns x box_rows rows, SWIZZLE_128B,
// out-of-range elements read as zero
bool encode_rows(CUtensorMap* m, const float* base, uint64_t cols, uint64_t rows, uint32_t box_rows) {
  static EncodeTiledFn enc = nullptr;
  if (!enc) {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      enc = nullptr;
    if (!enc) return false;
  }
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)std::max<uint64_t>(rows, 1)};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
  cuuint32_t box[2] = {32, box_rows}, es[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
}  // namespace

// dC2 (fused update) and dC1 partials from the dP stash; requires run_fused_fwd's per-step
// tables (grp_arow, grp_c2).
cudaError_t run_prefix_bwd(Ctx& c, float lr, cudaStream_t s) {
  const PlanDev& p = c.p;
  if (!c.tm_bwd_ready) {   // dP stash [P_cap n1][NC]; C2 region [sum m2 R][NC] (contiguous, NC-aligned)
    if (!encode_rows(&c.tm_dp, p.dpbuf, (uint64_t)c.NC, (uint64_t)c.P_cap * c.n1, YT) ||
        !encode_rows(&c.tm_c2, c.cores + c.c1_floats, (uint64_t)c.NC, (c.c3_begin - c.c1_floats) / c.NC,
                     (uint32_t)c.R))
      return cudaErrorInvalidValue;
    c.tm_bwd_ready = true;
  }
  YArgs a;
  a.cores = c.cores; a.grads = c.grads; a.state = c.state; a.meta = c.d_meta; a.counts = p.counts;
  a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.pfx_i1 = p.pfx_i1; a.pfx_t = p.pfx_t; a.grp_arow = p.grp_arow;
  a.grp_c2 = p.grp_c2; a.dpbuf = p.dpbuf; a.work = p.work + 2; a.c2_begin = c.c1_floats; a.dc2buf = p.dc2buf;
  a.unit_snake = p.unit_snake;
  a.n1 = c.n1; a.n1s = c.n1 == 1 ? 0 : c.n1 == 2 ? 1 : c.n1 == 4 ? 2 : 3;
  a.NC = c.NC; a.nblk = (c.NC + 127) / 128; a.tpp = YT / c.n1; a.R = c.R;
  // K-chunks per work unit: R = 64 the whole slice in 64-column chunks, R = 128 one c-block in
  // 32-column chunks
  a.nchunk = c.R <= 64 ? (c.NC + 63) / 64 : 128 / YShape<128>::CK;
  a.lr = lr; a.eps = c.eps; a.opt = c.opt; a.fused = (c.flags & TTEMB_FUSED_UPDATE) ? 1 : 0;
  a.exp = exp_bits();
  a.pf = knobs().pf_bwd;
  StageScope sc(c, ST_BWD_PREFIX, s);
  const int grid = prefix_bwd_grid(c);   // (the unit_snake deal was made for this grid)
  static unsigned long long* trace = nullptr;
  a.trace = nullptr;
  if (knobs().trace) {
    if (!trace) cudaMalloc(&trace, sizeof(unsigned long long) * 32 * grid);
    cudaMemsetAsync(trace, 0, sizeof(unsigned long long) * 32 * grid, s);
    a.trace = trace;
  }
  if (c.R == 32) launch_pdl(k_prefix_bwd<32>, dim3(grid), dim3(Y_THREADS), YShape<32>::SMEM, s, c.tm_dp, c.tm_c2, a);
  else if (c.R == 64) launch_pdl(k_prefix_bwd<64>, dim3(grid), dim3(Y_THREADS), YShape<64>::SMEM, s, c.tm_dp, c.tm_c2, a);
  else launch_pdl(k_prefix_bwd<128>, dim3(grid), dim3(Y_THREADS), YShape<128>::SMEM, s, c.tm_dp, c.tm_c2, a);
  if (a.fused && a.opt != TTEMB_SGD)
    k_c2_update<<<c.sm_count * 8, 256, 0, s>>>(c.cores, c.state, p.dc2buf, p.grp_c2, p.counts,
                                               (uint32_t)(c.R * c.NC), lr, c.eps);
  if (a.trace) {
    std::vector<unsigned long long> hb(32 * grid);
    cudaMemcpyAsync(hb.data(), trace, hb.size() * 8, cudaMemcpyDeviceToHost, s);
    cudaStreamSynchronize(s);
    double m[32] = {};
    for (int b = 0; b < grid; ++b) for (int k = 0; k < 32; ++k) m[k] += (double)hb[32 * b + k] / grid;
    fprintf(stderr, "[trace bwd] total %.0f | loader: tile-start %.0f a1_free %.0f b1+misc %.0f cp_wait %.0f lo %.0f "
            "sync %.0f tmem %.0f fence+arrive %.0f s_free %.0f issue %.0f | mma: u_full %.0f d2_free %.0f s_full %.0f "
            "dA-issue %.0f a1_full %.0f d1_free %.0f dC2-issue %.0f | epi: u_full %.0f d2_full %.0f dA-drain %.0f "
            "d1_full %.0f dC2-drain %.0f misc %.0f (cycles/CTA)\n",
            m[30], m[0], m[1], m[2], m[3], m[4], m[5], m[6], m[7], m[8], m[9], m[10], m[11], m[12], m[13], m[14],
            m[15], m[16], m[20], m[21], m[22], m[23], m[24], m[25]);
  }
  return cudaGetLastError();
}

}  // namespace ttemb
