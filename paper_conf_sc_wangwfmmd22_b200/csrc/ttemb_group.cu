// ttemb_group.cu -- fused per-i2-group forward and backward kernels (SURVEY 8(a) a5, a6,
// a9, a10, a12), sm_100a.
//
// One CTA owns one i2-group g = (t, i2) at a time (dynamic scheduler): it stages the
// C2[i2] slice (R x n2 R) in shared memory once (column chunks of whole j2 blocks) and
// walks the group's prefixes in m-tiles of MT rows (q, j1):
//
//   forward   P_tile  = A_tile . C2chunk          (A rows = C1[i1_q][j1,:];  the Reuse
//                                                  buffer of P:178, kept on chip)
//             E_u     = P_q . C3[i3_u]  for every unique row u of the tile's prefixes
//                                                 (Eq. 2; written to rows[u])
//   backward  P_tile  recomputed (no HBM stash)
//             dP_q    = sum_{u in q} G_u . C3[i3_u]^T             (Eq. 6)
//             dC3[i3] += P_q^T G_u                  (vector atomics, L2-resident)
//             dC2    += A_tile^T . dP_tile          (registers, whole group, no atomics)
//             dA      = dP_tile . C2chunk^T         (per-prefix dC1 partials)
//             end of group: dC2[i2] written, or the fused update applied in place
//                                                 (the group is the only reader)
// Row-stage loops are templated on upper bounds of n1 / n3 so accumulators stay in
// registers; the three contractions of size MT x CW x R are CUDA-core FFMA here.
#include <algorithm>

#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

struct GroupArgs {
  float* cores;
  float* grads;
  float* state;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_i1, *row_seg, *row_i3;
  float* rows;          // forward output  [U][N]
  const float* gbuf;    // backward input  [U][N]
  float* dabuf;         // backward output [P][n1][R]
  uint32_t* work;       // dynamic unit counter
  const uint32_t *chunk_off, *split_list;
  int n1, n2, n3, N, R, NC, CW, CWs, CWp, MT, PPT;
  float lr, eps;
  int opt, fused;
};

__device__ __forceinline__ void upd(float* p, float* s, float g, float lr, float eps, int opt) {
  if (opt == TTEMB_SGD) {
    *p = *p - lr * g;
  } else {
    const float v = *s + g * g;
    *s = v;
    *p = *p - lr * g / (sqrtf(v) + eps);
  }
}

__device__ __forceinline__ void red_add_v4(float* addr, float a, float b, float c, float d) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(a), "f"(b),
               "f"(c), "f"(d)
               : "memory");
}

// Work unit k -> (group g, prefixes [q0, q1), #units of g); false when k is past the last unit.
__device__ __forceinline__ bool claim_unit(const GroupArgs& a, uint32_t k, uint32_t& g, uint32_t& q0,
                                           uint32_t& q1, uint32_t& nch) {
  const uint32_t NG = a.counts[kCntNG];
  if (k >= a.counts[kCntNCh]) return false;
  uint32_t lo = 0, hi = NG - 1;                 // last g with chunk_off[g] <= k
  while (lo < hi) {
    const uint32_t mid = (lo + hi + 1) >> 1;
    if (a.chunk_off[mid] <= k) lo = mid; else hi = mid - 1;
  }
  g = lo;
  nch = a.chunk_off[g + 1] - a.chunk_off[g];
  const uint32_t gq0 = a.grp_off[g], gq1 = a.grp_off[g + 1];
  q0 = gq0 + (k - a.chunk_off[g]) * kGroupChunk;
  q1 = min(gq1, q0 + kGroupChunk);
  return true;
}

// Units of every group (one block): chunk_off = exclusive scan of ceil(#prefixes / kGroupChunk),
// and the list of split groups (more than one unit).
__global__ void __launch_bounds__(1024) k_group_chunks(uint32_t* counts, const uint32_t* __restrict__ grp_off,
                                                       uint32_t* chunk_off, uint32_t* split_list) {
  __shared__ uint32_t s_w[32], s_carry;
  const uint32_t NG = counts[kCntNG];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  if (tid == 0) s_carry = 0;
  __syncthreads();
  for (uint32_t base = 0; base < NG; base += 1024) {
    const uint32_t g = base + tid;
    uint32_t n = 0;
    if (g < NG) {
      n = (grp_off[g + 1] - grp_off[g] + kGroupChunk - 1) / kGroupChunk;
      if (n > 1) split_list[atomicAdd(counts + kCntNSplit, 1u)] = g;
    }
    uint32_t x = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) s_w[w] = x;
    __syncthreads();
    if (w == 0) {
      uint32_t v = s_w[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += y;
      }
      s_w[lane] = v;
    }
    __syncthreads();
    const uint32_t excl = s_carry + (w ? s_w[w - 1] : 0u) + x - n;
    if (g < NG) chunk_off[g] = excl;
    __syncthreads();
    if (tid == 0) s_carry += s_w[31];
    __syncthreads();
  }
  if (tid == 0) { chunk_off[NG] = s_carry; counts[kCntNCh] = s_carry; }
}

// Fused update of split groups' C2 slices from their accumulated dC2 (then cleared).
__global__ void __launch_bounds__(256) k_split_update(GroupArgs a) {
  const uint32_t ns = a.counts[kCntNSplit];
  const size_t per = (size_t)a.R * a.NC, total = (size_t)ns * per;
  for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (size_t)gridDim.x * blockDim.x) {
    const uint32_t g = a.split_list[e / per];
    const size_t idx = a.meta[a.grp_t[g]].c2_off + (size_t)a.grp_i2[g] * per + e % per;
    const float gr = a.grads[idx];
    upd(a.cores + idx, a.state + idx, gr, a.lr, a.eps, a.opt);
    a.grads[idx] = 0.f;
  }
}

// Shared-memory plan of one CTA (floats unless noted).
struct Smem {
  float* sC2;    // [R][CWs]     C2 chunk, odd stride
  float* sAT;    // [R][MT]      A transposed
  float* sA;     // [MT][R]      A (backward)
  float* sP;     // [MT][CWp]    P tile
  float* sdP;    // [MT][CWs]    dP tile (backward)
  float* sdPT;   // [CW][MT]     dP transposed (backward)
  uint32_t* rs;  // [PPT+1] row start of each prefix of the tile, then cumulative counts
  uint32_t* rc;  // [PPT+1]
  uint32_t* pf;  // [PPT]   prefix ids of the tile
  uint32_t* misc;
};

__host__ __device__ inline size_t up4(size_t x) { return (x + 3) & ~(size_t)3; }

__host__ __device__ inline size_t smem_floats(int R, int CW, int MT, int PPT, bool bwd) {
  const int CWs = CW | 1, CWp = (CW + 3) & ~3;
  size_t f = up4((size_t)R * CWs) + up4((size_t)R * MT) + up4((size_t)MT * CWp);
  if (bwd) f += up4((size_t)MT * R) + up4((size_t)MT * CWs) + up4((size_t)CW * MT);
  f += 3 * up4((size_t)(PPT + 1)) + 8;
  return f;
}

__device__ __forceinline__ Smem carve_smem(float* base, const GroupArgs& a, bool bwd) {
  Smem s;
  float* p = base;
  s.sC2 = p; p += up4((size_t)a.R * a.CWs);
  s.sAT = p; p += up4((size_t)a.R * a.MT);
  s.sP = p; p += up4((size_t)a.MT * a.CWp);
  if (bwd) {
    s.sA = p; p += up4((size_t)a.MT * a.R);
    s.sdP = p; p += up4((size_t)a.MT * a.CWs);
    s.sdPT = p; p += up4((size_t)a.CW * a.MT);
  } else {
    s.sA = s.sdP = s.sdPT = nullptr;
  }
  s.rs = reinterpret_cast<uint32_t*>(p); p += up4(a.PPT + 1);
  s.rc = reinterpret_cast<uint32_t*>(p); p += up4(a.PPT + 1);
  s.pf = reinterpret_cast<uint32_t*>(p); p += up4(a.PPT + 1);
  s.misc = reinterpret_cast<uint32_t*>(p);
  return s;
}

// Stage the C2 chunk [R][cw] of slice C2s (row stride NC) at column c0.
__device__ __forceinline__ void stage_c2(const GroupArgs& a, const Smem& s, const float* C2s,
                                         int c0, int cw) {
  for (int e = threadIdx.x; e < a.R * cw; e += blockDim.x) {
    const int r = e / cw, c = e - r * cw;
    s.sC2[r * a.CWs + c] = __ldg(C2s + (size_t)r * a.NC + c0 + c);
  }
}

// Stage the m-tile's prefixes: ids, row ranges (cumulative), and A rows (sAT and
// optionally sA).  npq prefixes starting at position qa of the group list.
__device__ __forceinline__ void stage_tile(const GroupArgs& a, const Smem& s, const float* C1t,
                                           uint32_t qa, int npq, bool want_sA) {
  const int tid = threadIdx.x;
  if (tid < npq) {
    const uint32_t p = a.grp_pfx[qa + tid];
    s.pf[tid] = p;
    const uint32_t r0 = a.row_seg[p], r1 = a.row_seg[p + 1];
    s.rs[tid] = r0;
    s.rc[tid] = r1 - r0;
  }
  __syncthreads();
  if (tid < 32) {   // exclusive scan of row counts (npq <= PPT <= 64)
    uint32_t v0 = tid < npq ? s.rc[tid] : 0, v1 = tid + 32 < npq ? s.rc[tid + 32] : 0;
    uint32_t x0 = v0, x1 = v1;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y0 = __shfl_up_sync(0xffffffffu, x0, o);
      const uint32_t y1 = __shfl_up_sync(0xffffffffu, x1, o);
      if (tid >= o) { x0 += y0; x1 += y1; }
    }
    const uint32_t tot0 = __shfl_sync(0xffffffffu, x0, 31);
    if (tid < npq) s.rc[tid] = x0 - v0;
    if (tid + 32 < npq) s.rc[tid + 32] = tot0 + x1 - v1;
    if (tid == 31) s.rc[npq] = tot0 + x1;
  }
  const int rowsA = npq * a.n1;
  for (int e = tid; e < a.R * a.MT; e += blockDim.x) {
    const int k = e / a.MT, m = e - k * a.MT;
    float v = 0.f;
    if (m < rowsA) {
      const uint32_t p = a.grp_pfx[qa + m / a.n1];
      v = __ldg(C1t + ((size_t)a.pfx_i1[p] * a.n1 + (m % a.n1)) * a.R + k);
    }
    s.sAT[e] = v;
    if (want_sA) s.sA[m * a.R + k] = v;
  }
  __syncthreads();
}

// GEMM1: sP[m][c] = sum_k sAT[k][m] sC2[k][c], m < MT, c < cw.
template <int RM>   // rows per thread = MT / 8
__device__ __forceinline__ void gemm_p(const GroupArgs& a, const Smem& s, int cw) {
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float acc[RM][4];
#pragma unroll
  for (int i = 0; i < RM; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
  for (int k = 0; k < a.R; ++k) {
    float av[RM], bv[4];
    const float* ar = s.sAT + k * a.MT + w * RM;
#pragma unroll
    for (int i = 0; i < RM; i += 4) {
      const float4 t4 = *reinterpret_cast<const float4*>(ar + i);
      av[i] = t4.x; av[i + 1] = t4.y; av[i + 2] = t4.z; av[i + 3] = t4.w;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int c = lane + 32 * j;
      bv[j] = c < cw ? s.sC2[k * a.CWs + c] : 0.f;
    }
#pragma unroll
    for (int i = 0; i < RM; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
  }
#pragma unroll
  for (int i = 0; i < RM; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int c = lane + 32 * j;
      if (c < cw) s.sP[(w * RM + i) * a.CWp + c] = acc[i][j];
    }
}

__device__ __forceinline__ int find_prefix(const uint32_t* rc, int npq, uint32_t ri) {
  int lo = 0, hi = npq - 1;   // last q with rc[q] <= ri
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (rc[mid] <= ri) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// Forward row stage: E_u[j1][j2][j3] for j2 in the chunk, item = (row, j2l).
template <int MN1, int MN3, bool VEC>
__device__ __forceinline__ void fwd_rows(const GroupArgs& a, const Smem& s, const float* C3t,
                                         int npq, int j2b, int n2c) {
  const uint32_t nr = s.rc[npq];
  const int R = a.R, n1 = a.n1, n3 = a.n3;
  for (uint32_t it = threadIdx.x; it < nr * n2c; it += blockDim.x) {
    const uint32_t ri = it / n2c;
    const int j2l = (int)(it - ri * n2c);
    const int ql = find_prefix(s.rc, npq, ri);
    const uint32_t u = s.rs[ql] + (ri - s.rc[ql]);
    const float* c3 = C3t + (size_t)a.row_i3[u] * R * n3;
    float acc[MN1][MN3];
#pragma unroll
    for (int i = 0; i < MN1; ++i)
#pragma unroll
      for (int j = 0; j < MN3; ++j) acc[i][j] = 0.f;
    const float* pr = s.sP + (size_t)(ql * n1) * a.CWp + j2l * R;
    if constexpr (VEC) {
      for (int r = 0; r < R; r += 4) {
        float cv[4][MN3];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < MN3; j += 4) {
            const float4 t4 = __ldg(reinterpret_cast<const float4*>(c3 + (r + i) * n3 + j));
            cv[i][j] = t4.x; cv[i][j + 1] = t4.y; cv[i][j + 2] = t4.z; cv[i][j + 3] = t4.w;
          }
#pragma unroll
        for (int j1 = 0; j1 < MN1; ++j1) {
          if (j1 < n1) {
            const float4 p4 = *reinterpret_cast<const float4*>(pr + j1 * a.CWp + r);
            const float pv[4] = {p4.x, p4.y, p4.z, p4.w};
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
              for (int j = 0; j < MN3; ++j) acc[j1][j] = fmaf(pv[i], cv[i][j], acc[j1][j]);
          }
        }
      }
    } else {
      for (int r = 0; r < R; ++r) {
        float cv[MN3];
#pragma unroll
        for (int j = 0; j < MN3; ++j) cv[j] = j < n3 ? __ldg(c3 + r * n3 + j) : 0.f;
#pragma unroll
        for (int j1 = 0; j1 < MN1; ++j1) {
          if (j1 < n1) {
            const float pv = pr[j1 * a.CWp + r];
#pragma unroll
            for (int j = 0; j < MN3; ++j) acc[j1][j] = fmaf(pv, cv[j], acc[j1][j]);
          }
        }
      }
    }
    const int j2 = j2b + j2l;
    float* dst = a.rows + (size_t)u * a.N;
#pragma unroll
    for (int j1 = 0; j1 < MN1; ++j1) {
      if (j1 >= n1) continue;
      float* d = dst + (j1 * a.n2 + j2) * n3;
      if constexpr (VEC) {
#pragma unroll
        for (int j = 0; j < MN3; j += 4)
          *reinterpret_cast<float4*>(d + j) = make_float4(acc[j1][j], acc[j1][j + 1], acc[j1][j + 2], acc[j1][j + 3]);
      } else {
#pragma unroll
        for (int j = 0; j < MN3; ++j)
          if (j < n3) d[j] = acc[j1][j];
      }
    }
  }
}

template <int MN1, int MN3, bool VEC>
__global__ void __launch_bounds__(256) k_group_fwd(GroupArgs a) {
  extern __shared__ __align__(16) float smem[];
  const Smem s = carve_smem(smem, a, false);
  const int tid = threadIdx.x;
  for (;;) {
    __syncthreads();
    if (tid == 0) s.misc[0] = atomicAdd(a.work, 1u);
    __syncthreads();
    uint32_t g, q0, q1, nch;
    if (!claim_unit(a, s.misc[0], g, q0, q1, nch)) break;
    const uint32_t t = a.grp_t[g], i2 = a.grp_i2[g];
    const TableMeta tm = a.meta[t];
    const float* C2s = a.cores + tm.c2_off + (size_t)i2 * a.R * a.NC;
    const float* C1t = a.cores + tm.c1_off;
    const float* C3t = a.cores + tm.c3_off;
    for (int c0 = 0; c0 < a.NC; c0 += a.CW) {
      const int cw = min(a.CW, a.NC - c0);
      __syncthreads();
      stage_c2(a, s, C2s, c0, cw);
      for (uint32_t qa = q0; qa < q1; qa += a.PPT) {
        const int npq = (int)min((uint32_t)a.PPT, q1 - qa);
        __syncthreads();
        stage_tile(a, s, C1t, qa, npq, false);
        if (a.MT == 64) gemm_p<8>(a, s, cw); else gemm_p<4>(a, s, cw);
        __syncthreads();
        fwd_rows<MN1, MN3, VEC>(a, s, C3t, npq, c0 / a.R, cw / a.R);
      }
    }
  }
}

// ------------------------------------------------------------------------------------
// Backward
// ------------------------------------------------------------------------------------

// dP tile: sdP[(ql,j1)][j2l*R + r] = sum_{u in ql} sum_j3 G_u[j1][j2][j3] C3[i3_u][r][j3].
// Item = (ql, j2l, r-block of 4).
template <int MN1, int MN3, bool VEC>
__device__ __forceinline__ void bwd_dp(const GroupArgs& a, const Smem& s, const float* C3t,
                                       int npq, int j2b, int n2c) {
  const int R = a.R, n1 = a.n1, n3 = a.n3;
  constexpr int RB = VEC ? 4 : 1;
  const int nrb = R / RB;
  const int items = npq * n2c * nrb;
  for (int it = threadIdx.x; it < items; it += blockDim.x) {
    const int ql = it / (n2c * nrb);
    const int rem = it - ql * n2c * nrb;
    const int j2l = rem / nrb;
    const int r0 = (rem - j2l * nrb) * RB;
    const int j2 = j2b + j2l;
    float acc[MN1][RB];
#pragma unroll
    for (int i = 0; i < MN1; ++i)
#pragma unroll
      for (int j = 0; j < RB; ++j) acc[i][j] = 0.f;
    const uint32_t u0 = s.rs[ql], nu = s.rc[ql + 1] - s.rc[ql];
    for (uint32_t k = 0; k < nu; ++k) {
      const uint32_t u = u0 + k;
      const float* c3 = C3t + (size_t)a.row_i3[u] * R * n3 + (size_t)r0 * n3;
      const float* gu = a.gbuf + (size_t)u * a.N + j2 * n3;
      float cv[RB][MN3];
#pragma unroll
      for (int i = 0; i < RB; ++i)
#pragma unroll
        for (int j = 0; j < MN3; ++j) cv[i][j] = 0.f;
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        if constexpr (VEC) {
#pragma unroll
          for (int j = 0; j < MN3; j += 4) {
            const float4 t4 = __ldg(reinterpret_cast<const float4*>(c3 + i * n3 + j));
            cv[i][j] = t4.x; cv[i][j + 1] = t4.y; cv[i][j + 2] = t4.z; cv[i][j + 3] = t4.w;
          }
        } else {
#pragma unroll
          for (int j = 0; j < MN3; ++j) cv[i][j] = j < n3 ? __ldg(c3 + i * n3 + j) : 0.f;
        }
      }
#pragma unroll
      for (int j1 = 0; j1 < MN1; ++j1) {
        if (j1 >= n1) continue;
        float gv[MN3];
        const float* g = gu + j1 * a.n2 * n3;
        if constexpr (VEC) {
#pragma unroll
          for (int j = 0; j < MN3; j += 4) {
            const float4 t4 = __ldg(reinterpret_cast<const float4*>(g + j));
            gv[j] = t4.x; gv[j + 1] = t4.y; gv[j + 2] = t4.z; gv[j + 3] = t4.w;
          }
        } else {
#pragma unroll
          for (int j = 0; j < MN3; ++j) gv[j] = j < n3 ? __ldg(g + j) : 0.f;
        }
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
          for (int j = 0; j < MN3; ++j) acc[j1][i] = fmaf(gv[j], cv[i][j], acc[j1][i]);
      }
    }
#pragma unroll
    for (int j1 = 0; j1 < MN1; ++j1) {
      if (j1 >= n1) continue;
      const int m = ql * n1 + j1;
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        const int c = j2l * R + r0 + i;
        s.sdP[m * a.CWs + c] = acc[j1][i];
        s.sdPT[c * a.MT + m] = acc[j1][i];
      }
    }
  }
}

// dC3[i3_u][r][j3] += sum_{j1, j2 in chunk} P[(ql,j1)][j2l*R + r] G_u[j1][j2][j3].
// Item = (row, r-block of 4); vector atomics into the L2-resident dense gradient.
template <int MN1, int MN3, bool VEC>
__device__ __forceinline__ void bwd_dc3(const GroupArgs& a, const Smem& s, size_t c3off,
                                        int npq, int j2b, int n2c) {
  const int R = a.R, n1 = a.n1, n3 = a.n3;
  constexpr int RB = VEC ? 4 : 1;
  const int nrb = R / RB;
  const uint32_t nr = s.rc[npq];
  for (uint32_t it = threadIdx.x; it < nr * nrb; it += blockDim.x) {
    const uint32_t ri = it / nrb;
    const int r0 = (int)(it - ri * nrb) * RB;
    const int ql = find_prefix(s.rc, npq, ri);
    const uint32_t u = s.rs[ql] + (ri - s.rc[ql]);
    float acc[RB][MN3];
#pragma unroll
    for (int i = 0; i < RB; ++i)
#pragma unroll
      for (int j = 0; j < MN3; ++j) acc[i][j] = 0.f;
    for (int j2l = 0; j2l < n2c; ++j2l) {
      const float* gu = a.gbuf + (size_t)u * a.N + (j2b + j2l) * n3;
#pragma unroll
      for (int j1 = 0; j1 < MN1; ++j1) {
        if (j1 >= n1) continue;
        float gv[MN3];
        const float* g = gu + j1 * a.n2 * n3;
        if constexpr (VEC) {
#pragma unroll
          for (int j = 0; j < MN3; j += 4) {
            const float4 t4 = __ldg(reinterpret_cast<const float4*>(g + j));
            gv[j] = t4.x; gv[j + 1] = t4.y; gv[j + 2] = t4.z; gv[j + 3] = t4.w;
          }
        } else {
#pragma unroll
          for (int j = 0; j < MN3; ++j) gv[j] = j < n3 ? __ldg(g + j) : 0.f;
        }
        const float* pr = s.sP + (size_t)(ql * n1 + j1) * a.CWp + j2l * R + r0;
        float pv[RB];
        if constexpr (VEC) {
          const float4 p4 = *reinterpret_cast<const float4*>(pr);
          pv[0] = p4.x; pv[1] = p4.y; pv[2] = p4.z; pv[3] = p4.w;
        } else {
          pv[0] = pr[0];
        }
#pragma unroll
        for (int i = 0; i < RB; ++i)
#pragma unroll
          for (int j = 0; j < MN3; ++j) acc[i][j] = fmaf(pv[i], gv[j], acc[i][j]);
      }
    }
    float* dst = a.grads + c3off + (size_t)a.row_i3[u] * R * n3 + (size_t)r0 * n3;
#pragma unroll
    for (int i = 0; i < RB; ++i) {
      if constexpr (VEC) {
#pragma unroll
        for (int j = 0; j < MN3; j += 4)
          red_add_v4(dst + i * n3 + j, acc[i][j], acc[i][j + 1], acc[i][j + 2], acc[i][j + 3]);
      } else {
#pragma unroll
        for (int j = 0; j < MN3; ++j)
          if (j < n3) atomicAdd(dst + i * n3 + j, acc[i][j]);
      }
    }
  }
}

// GEMM2: acc2[r1][c] += sum_m sA[m][r1] sdP[m][c]   (r1 = ty2 + 16 i, c = tx2 + 16 j)
__device__ __forceinline__ void gemm_dc2(const GroupArgs& a, const Smem& s, int mrows, int cw,
                                         float (&acc2)[8][8]) {
  const int ty2 = threadIdx.x >> 4, tx2 = threadIdx.x & 15;
  for (int m = 0; m < mrows; ++m) {
    float av[8], dv[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r1 = ty2 + 16 * i;
      av[i] = r1 < a.R ? s.sA[m * a.R + r1] : 0.f;
    }
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int c = tx2 + 16 * j;
      dv[j] = c < cw ? s.sdP[m * a.CWs + c] : 0.f;
    }
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc2[i][j] = fmaf(av[i], dv[j], acc2[i][j]);
  }
}

// GEMM3: dA[m][r1] (+)= sum_c sdPT[c][m] sC2[r1][c]; m = w*RM + i, r1 = lane + 32 j.
template <int RM>
__device__ __forceinline__ void gemm_da(const GroupArgs& a, const Smem& s, uint32_t qa,
                                        int npq, int cw, bool first_chunk) {
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float acc[RM][4];
#pragma unroll
  for (int i = 0; i < RM; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
  for (int c = 0; c < cw; ++c) {
    float dv[RM], bv[4];
    const float* dr = s.sdPT + c * a.MT + w * RM;
#pragma unroll
    for (int i = 0; i < RM; i += 4) {
      const float4 t4 = *reinterpret_cast<const float4*>(dr + i);
      dv[i] = t4.x; dv[i + 1] = t4.y; dv[i + 2] = t4.z; dv[i + 3] = t4.w;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int r1 = lane + 32 * j;
      bv[j] = r1 < a.R ? s.sC2[r1 * a.CWs + c] : 0.f;
    }
#pragma unroll
    for (int i = 0; i < RM; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(dv[i], bv[j], acc[i][j]);
  }
  const int rowsA = npq * a.n1;
#pragma unroll
  for (int i = 0; i < RM; ++i) {
    const int m = w * RM + i;
    if (m >= rowsA) continue;
    float* dst = a.dabuf + ((size_t)s.pf[m / a.n1] * a.n1 + (m % a.n1)) * a.R;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int r1 = lane + 32 * j;
      if (r1 < a.R) dst[r1] = first_chunk ? acc[i][j] : dst[r1] + acc[i][j];
    }
  }
}

template <int MN1, int MN3, bool VEC>
__global__ void __launch_bounds__(256) k_group_bwd(GroupArgs a) {
  extern __shared__ __align__(16) float smem[];
  const Smem s = carve_smem(smem, a, true);
  const int tid = threadIdx.x;
  const int ty2 = tid >> 4, tx2 = tid & 15;
  for (;;) {
    __syncthreads();
    if (tid == 0) s.misc[0] = atomicAdd(a.work, 1u);
    __syncthreads();
    uint32_t g, q0, q1, nch;
    if (!claim_unit(a, s.misc[0], g, q0, q1, nch)) break;
    const uint32_t t = a.grp_t[g], i2 = a.grp_i2[g];
    const TableMeta tm = a.meta[t];
    const size_t c2o = tm.c2_off + (size_t)i2 * a.R * a.NC;
    const float* C1t = a.cores + tm.c1_off;
    const float* C3t = a.cores + tm.c3_off;
    for (int c0 = 0; c0 < a.NC; c0 += a.CW) {
      const int cw = min(a.CW, a.NC - c0);
      const int j2b = c0 / a.R, n2c = cw / a.R;
      __syncthreads();
      stage_c2(a, s, a.cores + c2o, c0, cw);
      float acc2[8][8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc2[i][j] = 0.f;
      for (uint32_t qa = q0; qa < q1; qa += a.PPT) {
        const int npq = (int)min((uint32_t)a.PPT, q1 - qa);
        __syncthreads();
        stage_tile(a, s, C1t, qa, npq, true);
        if (a.MT == 64) gemm_p<8>(a, s, cw); else gemm_p<4>(a, s, cw);
        bwd_dp<MN1, MN3, VEC>(a, s, C3t, npq, j2b, n2c);
        __syncthreads();
        bwd_dc3<MN1, MN3, VEC>(a, s, tm.c3_off, npq, j2b, n2c);
        gemm_dc2(a, s, npq * a.n1, cw, acc2);
        if (a.MT == 64) gemm_da<8>(a, s, qa, npq, cw, c0 == 0);
        else gemm_da<4>(a, s, qa, npq, cw, c0 == 0);
      }
      // this CTA owns C2[t][i2]: gradient or fused update of the chunk
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r1 = ty2 + 16 * i;
        if (r1 >= a.R) continue;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int c = tx2 + 16 * j;
          if (c >= cw) continue;
          const size_t idx = c2o + (size_t)r1 * a.NC + c0 + c;
          if (nch > 1) atomicAdd(a.grads + idx, acc2[i][j]);   // split group: partial dC2
          else if (a.fused) upd(a.cores + idx, a.state + idx, acc2[i][j], a.lr, a.eps, a.opt);
          else a.grads[idx] = acc2[i][j];
        }
      }
    }
  }
}

template <int MN1, int MN3, bool VEC>
cudaError_t set_attrs(size_t fwd_bytes, size_t bwd_bytes) {
  cudaError_t e = cudaFuncSetAttribute(k_group_fwd<MN1, MN3, VEC>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)fwd_bytes);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_group_bwd<MN1, MN3, VEC>,
                              cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bwd_bytes);
}

template <int MN1, int MN3, bool VEC>
void launch(bool bwd, int grid, size_t bytes, const GroupArgs& a, cudaStream_t s) {
  if (bwd) k_group_bwd<MN1, MN3, VEC><<<grid, 256, bytes, s>>>(a);
  else k_group_fwd<MN1, MN3, VEC><<<grid, 256, bytes, s>>>(a);
}

struct Shape {
  int CW, MT, PPT;
  bool vec;
  int mn1, mn3;
};

Shape shape_of(const Ctx& c) {
  Shape sh;
  const int per = c.R <= 128 ? 128 / c.R : 1;
  sh.CW = std::min(c.NC, per * c.R);
  sh.MT = c.R <= 64 ? 64 : 32;
  sh.PPT = sh.MT / c.n1;
  sh.vec = (c.R % 4 == 0) && (c.n3 % 4 == 0);
  sh.mn1 = c.n1 <= 2 ? 2 : (c.n1 <= 4 ? 4 : 8);
  sh.mn3 = sh.vec ? (c.n3 <= 4 ? 4 : 8) : (c.n3 <= 4 ? 4 : 8);
  return sh;
}

template <bool VEC>
cudaError_t dispatch_attrs(int mn1, int mn3, size_t fb, size_t bb) {
  if (mn1 == 2 && mn3 == 4) return set_attrs<2, 4, VEC>(fb, bb);
  if (mn1 == 4 && mn3 == 4) return set_attrs<4, 4, VEC>(fb, bb);
  if (mn1 == 4 && mn3 == 8) return set_attrs<4, 8, VEC>(fb, bb);
  if (mn1 == 2 && mn3 == 8) return set_attrs<2, 8, VEC>(fb, bb);
  if (mn1 == 8 && mn3 == 4) return set_attrs<8, 4, VEC>(fb, bb);
  return set_attrs<8, 8, VEC>(fb, bb);
}

template <bool VEC>
void dispatch_launch(int mn1, int mn3, bool bwd, int grid, size_t bytes, const GroupArgs& a,
                     cudaStream_t s) {
  if (mn1 == 2 && mn3 == 4) return launch<2, 4, VEC>(bwd, grid, bytes, a, s);
  if (mn1 == 4 && mn3 == 4) return launch<4, 4, VEC>(bwd, grid, bytes, a, s);
  if (mn1 == 4 && mn3 == 8) return launch<4, 8, VEC>(bwd, grid, bytes, a, s);
  if (mn1 == 2 && mn3 == 8) return launch<2, 8, VEC>(bwd, grid, bytes, a, s);
  if (mn1 == 8 && mn3 == 4) return launch<8, 4, VEC>(bwd, grid, bytes, a, s);
  return launch<8, 8, VEC>(bwd, grid, bytes, a, s);
}

GroupArgs make_args(Ctx& c, float lr, uint32_t* work) {
  const Shape sh = shape_of(c);
  const PlanDev& p = c.p;
  GroupArgs a;
  a.cores = c.cores; a.grads = c.grads; a.state = c.state; a.meta = c.d_meta;
  a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2;
  a.grp_pfx = p.grp_pfx; a.pfx_i1 = p.pfx_i1; a.row_seg = p.row_seg; a.row_i3 = p.row_i3;
  a.rows = p.rows; a.gbuf = p.gbuf; a.dabuf = p.dabuf; a.work = work;
  a.chunk_off = p.chunk_off; a.split_list = p.split_list;
  a.n1 = c.n1; a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.R = c.R; a.NC = c.NC;
  a.CW = sh.CW; a.CWs = sh.CW | 1; a.CWp = (sh.CW + 3) & ~3; a.MT = sh.MT; a.PPT = sh.PPT;
  a.lr = lr; a.eps = c.eps; a.opt = c.opt; a.fused = (c.flags & TTEMB_FUSED_UPDATE) ? 1 : 0;
  return a;
}

size_t group_smem_bytes(const Ctx& c, bool bwd) {
  const Shape sh = shape_of(c);
  return sizeof(float) * smem_floats(c.R, sh.CW, sh.MT, sh.PPT, bwd);
}

}  // namespace

cudaError_t configure_group(Ctx& c) {
  const Shape sh = shape_of(c);
  const size_t fb = group_smem_bytes(c, false), bb = group_smem_bytes(c, true);
  if (bb > 227 * 1024) return cudaErrorInvalidConfiguration;
  return sh.vec ? dispatch_attrs<true>(sh.mn1, sh.mn3, fb, bb)
                : dispatch_attrs<false>(sh.mn1, sh.mn3, fb, bb);
}

cudaError_t run_group_fwd(Ctx& c, cudaStream_t s) {
  const Shape sh = shape_of(c);
  GroupArgs a = make_args(c, 0.f, c.p.work + 0);
  StageScope sc(c, ST_FWD_PREFIX, s);
  k_group_chunks<<<1, 1024, 0, s>>>(c.p.counts, c.p.grp_off, c.p.chunk_off, c.p.split_list);
  const size_t bytes = group_smem_bytes(c, false);
  const int per_sm = bytes > 110 * 1024 ? 1 : 2;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count * per_sm));
  if (sh.vec) dispatch_launch<true>(sh.mn1, sh.mn3, false, grid, bytes, a, s);
  else dispatch_launch<false>(sh.mn1, sh.mn3, false, grid, bytes, a, s);
  return cudaGetLastError();
}

cudaError_t run_group_bwd(Ctx& c, float lr, cudaStream_t s) {
  const Shape sh = shape_of(c);
  GroupArgs a = make_args(c, lr, c.p.work + 1);
  StageScope sc(c, ST_BWD_PREFIX, s);
  const size_t bytes = group_smem_bytes(c, true);
  const int per_sm = bytes > 110 * 1024 ? 1 : 2;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(c.NG_cap, (int64_t)c.sm_count * per_sm));
  if (sh.vec) dispatch_launch<true>(sh.mn1, sh.mn3, true, grid, bytes, a, s);
  else dispatch_launch<false>(sh.mn1, sh.mn3, true, grid, bytes, a, s);
  if (a.fused)   // split groups: their C2 slices were reduced into the (zero) gradient buffer
    k_split_update<<<c.sm_count * 8, 256, 0, s>>>(a);
  return cudaGetLastError();
}

}  // namespace ttemb
