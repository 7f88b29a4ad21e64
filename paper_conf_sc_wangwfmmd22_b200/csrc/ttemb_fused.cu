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
#include <vector>

#include "tc.cuh"
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int XR = 64;                         // TT rank = K of the prefix GEMM
constexpr int XT = 64;                         // tile rows (prefix, j1) = MMA N (max)
constexpr int X_LW = 8, X_RW = 7;   // 16 warps total: 128 registers per thread
constexpr int X_THREADS = (X_LW + 1 + X_RW) * 32;
constexpr int X_MMA_W = X_LW, X_ROW_W0 = X_LW + 1;
constexpr int XPSTR = 256;                     // P_s row stride (floats); columns XOR-swizzled
constexpr uint32_t XB_SLOT = 2u * XT * XR * 4; // one B slot: hi + lo CM matrices (32 KB)
constexpr uint32_t XB_HALF = XT * XR * 4;
constexpr uint32_t X_RAW_BYTES = 65536;        // R x NC fp32, NC <= 256

struct XArgs {
  float* cores;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_i1, *pfx_t, *row_seg, *row_i3, *row_pfx;
  uint32_t* grp_arow;                 // [P]  C1 row index (floats / R) of sorted prefix q, j1 = 0
  unsigned long long* grp_c2;         // [NG] float offset of group g's C2 slice
  float* rows;                        // [U][N]
  float* pbuf;                        // [P][n1][NC] (consumed by the backward row stage)
  uint32_t* work;
  int dbg;                            // TTEMB_DBG bit mask (timing experiments only; results invalid)
  unsigned long long* trace;          // optional per-CTA role timers (TTEMB_TRACE): 32 slots per CTA
  int n1, n1s, n2, n3, N, NC, nblk, tpp;
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
  uint32_t ring[4][8];                // group, first prefix, #prefixes, flags (1 first, 2 last, 4 done), u0, u1
  uint32_t claim[2];
  uint32_t tmem;
};

__global__ void k_fused_prep(XArgs a) {
  const uint32_t P = a.counts[kCntP], NG = a.counts[kCntNG];
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < max(P, NG); q += gridDim.x * blockDim.x) {
    if (q < P) {
      const uint32_t p = a.grp_pfx[q];
      a.grp_arow[q] = (uint32_t)(a.meta[a.pfx_t[p]].c1_off / XR) + (a.pfx_i1[p] << a.n1s);
    }
    if (q < NG) a.grp_c2[q] = a.meta[a.grp_t[q]].c2_off + (unsigned long long)a.grp_i2[q] * XR * a.NC;
  }
}

__device__ __forceinline__ float tf32_lo(float x) { return x - tc::tf32_trunc(x); }

template <int N3>
__global__ void __launch_bounds__(X_THREADS, 1) k_fused_fwd(XArgs a) {
  extern __shared__ __align__(128) char smem_raw[];
  __shared__ XCtl ctl;
  char* const smem = smem_raw + ((128u - (tc::smem_u32(smem_raw) & 127u)) & 127u);
  float* const raw = reinterpret_cast<float*>(smem);
  char* const bbuf = smem + X_RAW_BYTES;
  float* const ps = reinterpret_cast<float*>(smem + X_RAW_BYTES + 2 * XB_SLOT);
  float* const c3s = ps + XT * XPSTR;
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const uint32_t NG = a.counts[kCntNG];
  const uint32_t raw_bytes = (uint32_t)XR * a.NC * 4u;
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
    for (int s = 0; s < 4; ++s) { tc::mbar_init(&ctl.u_full[s], 1); tc::mbar_init(&ctl.u_empty[s], 2); }
    tc::fence_mbar_init();
  }
  if (w == X_MMA_W) tc::tmem_alloc(&ctl.tmem, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = ctl.tmem;
  // TMEM columns: [0,128) C2^T hi (64 per c-block), [128,256) lo, [256,512) D[2] (128 each:
  // 64 per c-block).
  const int tpp = a.tpp;
  unsigned long long trc[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
  const long long t_start = a.trace ? clock64() : 0;

  if (w < X_LW) {
    // ------------------------------- loaders -------------------------------
    const int blk = w >> 2, Q = w & 3;
    const int c = blk * 128 + Q * 32 + lane;
    const bool cval = c < a.NC;
    const bool bact = blk < a.nblk;
    float xa[32], xb[32];
    uint32_t ui = 0, gs = 0, rawk = 0;
    auto load_raw = [&]() {          // regs <- raw (this thread's column c, all r1)
#pragma unroll
      for (int r = 0; r < 32; ++r) {
        xa[r] = cval ? raw[r * a.NC + c] : 0.f;
        xb[r] = cval ? raw[(r + 32) * a.NC + c] : 0.f;
      }
    };
    auto issue_raw = [&](uint32_t g) {
      tc::mbar_arrive_tx(&ctl.raw_full, raw_bytes);
      tc::bulk_g2s(tc::smem_u32(raw), a.cores + a.grp_c2[g], raw_bytes, &ctl.raw_full);
    };
    if (tid == 0) {
      ctl.claim[0] = atomicAdd(a.work, 1u);
      ctl.claim[1] = atomicAdd(a.work, 1u);
      if (ctl.claim[0] < NG) issue_raw(ctl.claim[0]);
    }
    tc::named_sync(1, X_LW * 32);
    uint32_t cur = ctl.claim[0], nxt = ctl.claim[1];
    if (cur < NG) {
      tc::mbar_wait(&ctl.raw_full, rawk & 1);
      ++rawk;
      load_raw();
    }
    tc::named_sync(1, X_LW * 32);
    if (tid == 0 && nxt < NG) issue_raw(nxt);
    while (cur < NG) {
      const uint32_t q0 = a.grp_off[cur], q1 = a.grp_off[cur + 1];
      for (uint32_t qa = q0; qa < q1; qa += tpp, ++ui) {
        const uint32_t np = min((uint32_t)tpp, q1 - qa);
        const int rows = (int)np << a.n1s;
        const uint32_t fl = (qa == q0 ? 1u : 0u) | (qa + tpp >= q1 ? 2u : 0u);
        XT0();
        if (tid == 0) {
          tc::mbar_wait(&ctl.u_empty[ui & 3], ((ui >> 2) & 1) ^ 1);
          ctl.ring[ui & 3][0] = cur; ctl.ring[ui & 3][1] = qa; ctl.ring[ui & 3][2] = np; ctl.ring[ui & 3][3] = fl;
          ctl.ring[ui & 3][4] = a.row_seg[qa]; ctl.ring[ui & 3][5] = a.row_seg[qa + np];
          tc::mbar_arrive(&ctl.u_full[ui & 3]);
        }
        // C1 rows of the tile -> registers (B = CM(m, r1), m = tid & 63, 4 float4 of r1)
        const int m = tid & 63;
        float4 bv[4];
        {
          const bool ok = m < rows;
          const uint32_t arow = ok ? a.grp_arow[qa + (m >> a.n1s)] + (m & ((1 << a.n1s) - 1)) : 0u;
          const float4* src = reinterpret_cast<const float4*>(a.cores + (size_t)arow * XR);
#pragma unroll
          for (int k = 0; k < 4; ++k) bv[k] = ok ? __ldg(src + (tid >> 6) + 4 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
        }
        XTA(0);
        if (fl & 1u) {   // the group's C2^T -> TMEM (hi = raw fp32, lo = x - trunc_tf32(x))
          tc::mbar_wait(&ctl.a_free, (gs & 1) ^ 1);
          XTA(1);
          tc::fence_after();
          if (bact) {
            tc::tmem_st32(tc::taddr(tm + blk * 64, 32 * Q, 0), xa);
            tc::tmem_st32(tc::taddr(tm + blk * 64 + 32, 32 * Q, 0), xb);
#pragma unroll
            for (int r = 0; r < 32; ++r) { xa[r] = tf32_lo(xa[r]); xb[r] = tf32_lo(xb[r]); }
            tc::tmem_st32(tc::taddr(tm + 128 + blk * 64, 32 * Q, 0), xa);
            tc::tmem_st32(tc::taddr(tm + 128 + blk * 64 + 32, 32 * Q, 0), xb);
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
          char* bh = bbuf + s * XB_SLOT;
          char* bl = bh + XB_HALF;
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint32_t off = tc::cm_off(m, 4 * ((tid >> 6) + 4 * k), XT / 8);
            const float4 v = bv[k];
            *reinterpret_cast<float4*>(bh + off) = v;
            *reinterpret_cast<float4*>(bl + off) = make_float4(tf32_lo(v.x), tf32_lo(v.y), tf32_lo(v.z), tf32_lo(v.w));
          }
          tc::fence_async_smem();
          tc::mbar_arrive(&ctl.b_full[s]);
          XTA(4);
        }
        {   // L2 prefetch of the tile's C3 slices (the row warps read them about two tiles later);
            // the tile's unique rows are one contiguous range (group-major plan)
          const float* c3base = a.cores + a.meta[a.grp_t[cur]].c3_off;
          const uint32_t u0 = a.row_seg[qa], u1 = a.row_seg[qa + np];
          for (uint32_t u = u0 + tid; u < u1; u += X_LW * 32) {
            const char* p3 = reinterpret_cast<const char*>(c3base + (size_t)__ldg(a.row_i3 + u) * XR * N3);
#pragma unroll
            for (int l = 0; l < XR * N3 * 4 / 128; ++l) asm volatile("prefetch.global.L2 [%0];" ::"l"(p3 + 128 * l));
          }
        }
      }
      XT0();
      // next group: registers <- raw (nxt); raw <- the group after (claimed now)
      if (tid == 0) ctl.claim[gs & 1] = atomicAdd(a.work, 1u);
      if (nxt < NG) {
        tc::mbar_wait(&ctl.raw_full, rawk & 1);
        ++rawk;
        XTA(5);
        load_raw();
      }
      tc::named_sync(1, X_LW * 32);
      XTA(6);
      const uint32_t nn = ctl.claim[gs & 1];
      if (tid == 0 && nn < NG) issue_raw(nn);
      ++gs;
      cur = nxt;
      nxt = nn;
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
      const uint32_t np = ctl.ring[ui & 3][2], fl = ctl.ring[ui & 3][3];
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
        const uint32_t bh = tc::smem_u32(bbuf + s * XB_SLOT), bl = bh + XB_HALF;
        for (int blk = 0; blk < a.nblk; ++blk) {
          const uint32_t d = tm + 256 + s * 128 + blk * 64;
#pragma unroll
          for (int kk = 0; kk < XR / 8; ++kk) {
            const uint32_t o = kk * 2 * (XT / 8) * 128;
            const uint64_t dbh = tc::sdesc(bh + o, (XT / 8) * 128, 128);
            const uint64_t dbl = tc::sdesc(bl + o, (XT / 8) * 128, 128);
            const uint32_t ah = tm + blk * 64 + kk * 8, al = tm + 128 + blk * 64 + kk * 8;
            tc::mma_tf32_ts(d, ah, dbh, id, kk > 0 ? 1u : 0u);
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
    // ------------------------------- row warps -------------------------------
    constexpr int C3L = XR * N3 / 4 / 32;        // float4 of a C3 slice per lane
    constexpr int NSL = N3 == 4 ? 3 : 2;         // per-warp C3 ring slots (cp.async)
    const int rw = w - X_ROW_W0, rtid = tid - X_ROW_W0 * 32;
    const int Q = w & 3;
    // drain assignment: (c-block, lane quarter) pairs; warps rw 0-3 take block 0 (quarters
    // 1,2,3,0), rw 4-6 block 1 (quarters 1,2,3), rw 3 (quarter 0) also block 1
    const int blk0 = rw < 4 ? 0 : 1, blk_step = rw == 3 ? 1 : 2;
    const uint32_t ring3 = tc::smem_u32(c3s + rw * (NSL * XR * N3));
    const float* ring3p = c3s + rw * (NSL * XR * N3);
    const int J12 = a.n1 * a.n2;
    const int j12 = lane >> 1, h = lane & 1;
    const int j1 = j12 / a.n2, j2 = j12 - j1 * a.n2;
    const bool jval = j12 < J12;
    // P_s(m, c) lives at m * XPSTR + (c ^ 4 ((c >> 5) & 7)): conflict-free for the drain (32
    // consecutive c per warp store) and for the row loads (8 column blocks per LDS.128 phase).
    const int pb = (j2 * XR + 32 * h) >> 5;
    const int pxor = pb & 7;
    for (uint32_t ui = 0;; ++ui) {
      XT0();
      tc::mbar_wait(&ctl.u_full[ui & 3], (ui >> 2) & 1);
      XTA(0);
      const uint32_t g = ctl.ring[ui & 3][0], qa = ctl.ring[ui & 3][1];
      const uint32_t np = ctl.ring[ui & 3][2], fl = ctl.ring[ui & 3][3];
      const uint32_t u0 = ctl.ring[ui & 3][4], u1 = ctl.ring[ui & 3][5];
      if (fl & 4u) break;
      const int rows = (int)np << a.n1s;
      const uint32_t s = ui & 1;
      const uint32_t Rt = u1 - u0;
      const float* c3base = a.cores + a.meta[a.grp_t[g]].c3_off;
      // ---- drain D[s]: this warp's c-block quarter -> P_s ----
      XTA(1);
      tc::mbar_wait(&ctl.d_full[s], (ui >> 1) & 1);
      XTA(2);
      tc::fence_after();
      XTA(7);
      for (int blk = blk0; blk < a.nblk; blk += blk_step) {
        const int c = blk * 128 + Q * 32 + lane;
        const int dcol = c ^ (4 * ((c >> 5) & 7));
        for (int j0 = 0; j0 < rows; j0 += 32) {
          float v[32];
          tc::tmem_ld32(tc::taddr(tm + 256 + s * 128 + blk * 64 + j0, 32 * Q, 0), v);
          if (c < a.NC) {
            float* dst = ps + j0 * XPSTR + dcol;
#pragma unroll
            for (int j = 0; j < 32; ++j) dst[j * XPSTR] = v[j];
          }
        }
      }
      XTA(9);
      tc::fence_before();
      tc::mbar_arrive(&ctl.d_free[s]);
      XTA(3);
      tc::named_sync(2, X_RW * 32);
      XTA(4);
      // ---- P stash for the backward row stage: pbuf[q][j1][c] <- P_s (float4); the tile's
      //      prefixes qa .. qa+np-1 are consecutive, so this is one contiguous block ----
      if (a.pbuf) {
        const int nc4 = a.NC >> 2, tot = rows * nc4;
        float* dst = a.pbuf + (size_t)qa * a.n1 * a.NC;
        for (int f = rtid; f < tot; f += X_RW * 32) {
          const int mm = f / nc4, c4 = (f - mm * nc4) * 4;
          *reinterpret_cast<float4*>(dst + (size_t)mm * a.NC + c4) =
              *reinterpret_cast<const float4*>(ps + mm * XPSTR + (c4 ^ (4 * ((c4 >> 5) & 7))));
        }
      }
      // ---- rows: this warp's share [r0, r1) of the tile's Rt unique rows u0 .. u1-1 ----
      const uint32_t r0 = (uint32_t)(((uint64_t)Rt * rw) / X_RW), r1 = (uint32_t)(((uint64_t)Rt * (rw + 1)) / X_RW);
      int curk = -1;
      float4 pv[8];
      for (uint32_t rb = r0; rb < r1; rb += 32) {
        const int nr = (int)min(32u, r1 - rb);
        // lane-parallel: row u0 + rb + lane -> (tile prefix k, i3)
        const uint32_t ul = u0 + rb + lane;
        int kl = 0;
        uint32_t i3l = 0;
        if (lane < nr) {
          kl = (int)(__ldg(a.row_pfx + ul) - qa);
          i3l = __ldg(a.row_i3 + ul);
        }
        auto issue = [&](int j) {   // C3 slice of row rb + j -> ring slot j % NSL
          const uint32_t i3 = __shfl_sync(0xffffffffu, i3l, j);
          const float4* src = reinterpret_cast<const float4*>(c3base + (size_t)i3 * XR * N3);
          const uint32_t dst = ring3 + (uint32_t)((j % NSL) * XR * N3 * 4);
#pragma unroll
          for (int i = 0; i < C3L; ++i) tc::cp_async16(dst + 16u * (lane + 32 * i), src + lane + 32 * i);
        };
#pragma unroll
        for (int j = 0; j < NSL - 1; ++j) {
          if (j < nr) issue(j);
          tc::cp_commit();
        }
        for (int j = 0; j < nr; ++j) {
          tc::cp_wait<NSL - 2>();
          __syncwarp();
          const int k = __shfl_sync(0xffffffffu, kl, j);
          const uint32_t u = u0 + rb + j;
          if (k != curk) {
            const float* prow = ps + ((k << a.n1s) + j1) * XPSTR + 32 * pb;
#pragma unroll
            for (int i = 0; i < 8; ++i)
              pv[i] = jval ? *reinterpret_cast<const float4*>(prow + 4 * (i ^ pxor)) : make_float4(0.f, 0.f, 0.f, 0.f);
            curk = k;
          }
          float acc[N3];
#pragma unroll
          for (int q = 0; q < N3; ++q) acc[q] = 0.f;
          const float* c3 = ring3p + (j % NSL) * XR * N3 + 32 * h * N3;
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const float pr[4] = {pv[i].x, pv[i].y, pv[i].z, pv[i].w};
#pragma unroll
            for (int e = 0; e < 4; ++e)
#pragma unroll
              for (int q = 0; q < N3; q += 4) {
                const float4 c4 = *reinterpret_cast<const float4*>(c3 + (4 * i + e) * N3 + q);
                acc[q] = fmaf(pr[e], c4.x, acc[q]);
                acc[q + 1] = fmaf(pr[e], c4.y, acc[q + 1]);
                acc[q + 2] = fmaf(pr[e], c4.z, acc[q + 2]);
                acc[q + 3] = fmaf(pr[e], c4.w, acc[q + 3]);
              }
          }
          __syncwarp();
          if (j + NSL - 1 < nr) issue(j + NSL - 1);
          tc::cp_commit();
#pragma unroll
          for (int q = 0; q < N3; ++q) acc[q] += __shfl_xor_sync(0xffffffffu, acc[q], 1);
          if (h == 0 && jval) {
            float* d = a.rows + (size_t)u * a.N + j12 * N3;
#pragma unroll
            for (int q = 0; q < N3; q += 4) *reinterpret_cast<float4*>(d + q) = make_float4(acc[q], acc[q + 1], acc[q + 2], acc[q + 3]);
          }
        }
        tc::cp_wait<0>();
        __syncwarp();
      }
      XTA(5);
      tc::named_sync(2, X_RW * 32);      // P_s free for the next tile's drain
      XTA(6);
      trc[8] += Rt;
      if (rtid == 0) tc::mbar_arrive(&ctl.u_empty[ui & 3]);
    }
  }
  if (a.trace) {
    const int role = tid == 0 ? 0 : tid == X_MMA_W * 32 ? 1 : tid == X_ROW_W0 * 32 ? 2 : -1;
    if (role >= 0)
      for (int k = 0; k < 10; ++k) a.trace[32 * blockIdx.x + 10 * role + k] = trc[k];
    if (tid == 0) a.trace[32 * blockIdx.x + 30] = (unsigned long long)(clock64() - t_start);
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (w == X_MMA_W) tc::tmem_dealloc(tm, 512);
}

size_t fused_smem(int n3) {
  return 128 + X_RAW_BYTES + 2 * XB_SLOT + (size_t)XT * XPSTR * 4 + (size_t)X_RW * (n3 == 4 ? 3 : 2) * XR * n3 * 4;
}

}  // namespace

bool fused_eligible(const Ctx& c) {
  return !(c.flags & TTEMB_FP32_CORES) && !getenv("TTEMB_OLD_FWD") && c.R == XR && c.NC <= 256 &&
         (c.n3 == 4 || c.n3 == 8) && (c.n1 == 1 || c.n1 == 2 || c.n1 == 4 || c.n1 == 8) && c.n1 * c.n2 <= 16;
}

cudaError_t configure_fused(Ctx& c) {
  if (!fused_eligible(c)) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(k_fused_fwd<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fused_smem(4));
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(k_fused_fwd<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fused_smem(8));
  return e;
}

cudaError_t run_fused_fwd(Ctx& c, cudaStream_t s) {
  const PlanDev& p = c.p;
  XArgs a;
  a.cores = c.cores; a.meta = c.d_meta; a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t;
  a.grp_i2 = p.grp_i2; a.grp_pfx = p.grp_pfx; a.pfx_i1 = p.pfx_i1; a.pfx_t = p.pfx_t; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.row_pfx = p.row_pfx; a.grp_arow = p.grp_arow; a.grp_c2 = p.grp_c2; a.rows = p.rows; a.pbuf = p.pbuf;
  a.work = p.work + 0;
  a.dbg = getenv("TTEMB_DBG") ? atoi(getenv("TTEMB_DBG")) : 0;
  a.n1 = c.n1; a.n1s = c.n1 == 1 ? 0 : c.n1 == 2 ? 1 : c.n1 == 4 ? 2 : 3;
  a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.NC = c.NC; a.nblk = (c.NC + 127) / 128; a.tpp = XT / c.n1;
  {
    StageScope sc(c, ST_FWD_PREFIX, s);
    k_fused_prep<<<grid_for(c, std::max(c.P_cap, c.NG_cap), 256, 4), 256, 0, s>>>(a);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count));
    static unsigned long long* trace = nullptr;
    a.trace = nullptr;
    if (getenv("TTEMB_TRACE")) {
      if (!trace) cudaMalloc(&trace, sizeof(unsigned long long) * 32 * grid);
      cudaMemsetAsync(trace, 0, sizeof(unsigned long long) * 32 * grid, s);
      a.trace = trace;
    }
    if (c.n3 == 4) k_fused_fwd<4><<<grid, X_THREADS, fused_smem(4), s>>>(a);
    else k_fused_fwd<8><<<grid, X_THREADS, fused_smem(8), s>>>(a);
    if (a.trace) {
      std::vector<unsigned long long> hb(32 * grid);
      cudaMemcpyAsync(hb.data(), trace, hb.size() * 8, cudaMemcpyDeviceToHost, s);
      cudaStreamSynchronize(s);
      double m[32] = {};
      for (int b = 0; b < grid; ++b) for (int k = 0; k < 32; ++k) m[k] += (double)hb[32 * b + k] / grid;
      fprintf(stderr, "[trace fused] total %.0f | loader: ring+bload %.0f a_free %.0f a_store %.0f b_free %.0f b_store %.0f "
              "raw_wait %.0f raw_sync %.0f | mma: u_full %.0f a_full %.0f b_full %.0f d_free %.0f issue %.0f units %.1f | "
              "rows: u_full %.0f plist %.0f d_full %.0f [fa %.0f loop %.0f] fb+arrive %.0f sync1 %.0f rows %.0f sync2 %.0f nrows %.0f (cycles/CTA)\n",
              m[30], m[0], m[1], m[2], m[3], m[4], m[5], m[6], m[10], m[11], m[12], m[13], m[14], m[19], m[20], m[21],
              m[22], m[27], m[29], m[23], m[24], m[25], m[26], m[28]);
    }
  }
  return cudaGetLastError();
}

}  // namespace ttemb
