// ttemb_bwd.cu -- backward and update, sm_100a.
//
//   a8  in-advance aggregation G_u = sum_{positions of row u} grad_out[bag]
//       as a fixed-chunk segmented reduction over the sorted occurrence list (no atomics,
//       deterministic; long Zipf segments are split across chunks and re-joined)
//   a9  per prefix p: dP_p = sum_{u in p} G_u . C3[i3]^T, dC3[i3] += P_p^T G_u   (Eq. 6 read
//       as left^T . dL/de . right^T; dP aggregated per prefix = exact algebra)
//   a10 per i2-group g: dC2[i2] = A_g^T . dP_g  (reduced inside the CTA, no atomics),
//       dA_g = dP_g . C2[i2]^T  (per-prefix dC1 partials)
//   a11 dC1[t][i1] = sum of the partials of the contiguous (t, i1) prefix run
//   a12 SGD / Adagrad; with TTEMB_FUSED_UPDATE the C2 slices are updated by the group
//       CTA that owns them and C1 by the run reduction ("fused TT core update")
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int AGG_CS = 32;   // sorted positions per aggregation chunk
constexpr int GM = 32;       // rows (prefix, j1) per m-tile
constexpr int GCW = 128;     // max C2 columns per chunk

__device__ __forceinline__ void apply_update(float* param, float* state, float g, float lr,
                                             float eps, int opt) {
  if (opt == TTEMB_SGD) {
    *param = *param - lr * g;
  } else {
    const float s = *state + g * g;
    *state = s;
    *param = *param - lr * g / (sqrtf(s) + eps);
  }
}

// a8 part 1: thread = (chunk of AGG_CS sorted positions, column)
__global__ void __launch_bounds__(256)
k_agg(const float* __restrict__ grad_out, const uint32_t* __restrict__ skey,
      const uint32_t* __restrict__ sbag, const uint32_t* __restrict__ spos,
      const uint32_t* __restrict__ inverse, const uint32_t* __restrict__ seg_off, int64_t nnz,
      int N, float* __restrict__ gbuf, float* __restrict__ part) {
  const int64_t nchunks = (nnz + AGG_CS - 1) / AGG_CS;
  const int64_t total = nchunks * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t ch = e / N;
    const int col = (int)(e - ch * N);
    const int64_t k0 = ch * AGG_CS, k1 = min(k0 + AGG_CS, nnz);
    float acc = 0.f;
    for (int64_t k = k0; k < k1; ++k) {
      acc += __ldg(grad_out + (size_t)sbag[k] * N + col);
      const bool seg_end = (k + 1 == nnz) || skey[k + 1] != skey[k];
      if (seg_end || k + 1 == k1) {
        const uint32_t u = inverse[spos[k]];
        const int64_t s0 = seg_off[u], s1 = seg_off[u + 1];
        if (s0 >= k0 && s1 <= k1) gbuf[(size_t)u * N + col] = acc;
        else if (s0 < k0) part[((size_t)ch * 2 + 0) * N + col] = acc;   // head: began earlier
        else part[((size_t)ch * 2 + 1) * N + col] = acc;                // tail: continues
        acc = 0.f;
      }
    }
  }
}

// a8 part 2: rows whose segment spans several chunks: tail(c0) + heads(c0+1..c1)
__global__ void __launch_bounds__(256)
k_agg_fix(const uint32_t* __restrict__ seg_off, const uint32_t* __restrict__ counts, int N,
          const float* __restrict__ part, float* __restrict__ gbuf) {
  const int64_t total = (int64_t)counts[kCntU] * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t u = e / N;
    const int col = (int)(e - u * N);
    const int64_t c0 = seg_off[u] / AGG_CS, c1 = (seg_off[u + 1] - 1) / AGG_CS;
    if (c0 == c1) continue;
    float acc = part[((size_t)c0 * 2 + 1) * N + col];
    for (int64_t ch = c0 + 1; ch <= c1; ++ch) acc += part[((size_t)ch * 2 + 0) * N + col];
    gbuf[(size_t)u * N + col] = acc;
  }
}

struct BwdArgs {
  float* cores;
  float* grads;
  float* state;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_t, *pfx_i1, *row_seg, *row_i3;
  const float* pbuf;
  const float* gbuf;
  float* dpbuf;
  float* dabuf;
  int n1, n2, n3, N, R, NC, CW, CWs;
  float lr, eps;
  int opt, fused;
};

// a9: per prefix, dP_p and dC3 contributions (CTA per prefix)
__global__ void __launch_bounds__(128) k_bwd_rows(BwdArgs a) {
  extern __shared__ __align__(16) float smem[];
  const int R = a.R, N = a.N, n3 = a.n3, J12 = a.n1 * a.n2, ldp = R + 1;
  float* sP = smem;                  // [J12][R+1]
  float* sdP = sP + J12 * ldp;       // [J12][R]
  float* sG = sdP + J12 * R;         // [N]
  const uint32_t P = a.counts[kCntP];
  for (uint32_t p = blockIdx.x; p < P; p += gridDim.x) {
    __syncthreads();
    const float* src = a.pbuf + (size_t)p * J12 * R;
    for (int e = threadIdx.x; e < J12 * R; e += blockDim.x) {
      const int j = e / R, r = e - j * R;
      sP[j * ldp + r] = src[e];
      sdP[e] = 0.f;
    }
    const uint32_t u0 = a.row_seg[p], u1 = a.row_seg[p + 1];
    const TableMeta tm = a.meta[a.pfx_t[p]];
    for (uint32_t u = u0; u < u1; ++u) {
      __syncthreads();
      for (int e = threadIdx.x; e < N; e += blockDim.x) sG[e] = a.gbuf[(size_t)u * N + e];
      __syncthreads();
      const size_t c3o = tm.c3_off + (size_t)a.row_i3[u] * R * n3;
      const float* c3 = a.cores + c3o;
      for (int e = threadIdx.x; e < J12 * R; e += blockDim.x) {      // dP += G C3^T
        const int j12 = e / R, r = e - j12 * R;
        float acc = 0.f;
        for (int j3 = 0; j3 < n3; ++j3) acc = fmaf(sG[j12 * n3 + j3], __ldg(c3 + r * n3 + j3), acc);
        sdP[e] += acc;
      }
      for (int e = threadIdx.x; e < R * n3; e += blockDim.x) {       // dC3 += P^T G
        const int r = e / n3, j3 = e - r * n3;
        float acc = 0.f;
        for (int j12 = 0; j12 < J12; ++j12) acc = fmaf(sP[j12 * ldp + r], sG[j12 * n3 + j3], acc);
        atomicAdd(a.grads + c3o + e, acc);
      }
    }
    __syncthreads();
    float* dst = a.dpbuf + (size_t)p * J12 * R;
    for (int e = threadIdx.x; e < J12 * R; e += blockDim.x) dst[e] = sdP[e];
  }
}

// a10: per i2-group: dC2[i2] = A^T dP (in registers), dA = dP C2[i2]^T (to dabuf)
__global__ void __launch_bounds__(256) k_bwd_prefix(BwdArgs a) {
  extern __shared__ __align__(16) float smem[];
  const int R = a.R, NC = a.NC, CWs = a.CWs, n1 = a.n1;
  float* sB = smem;                 // [R][CWs]   C2 chunk
  float* sA = sB + R * CWs;         // [GM][R]    C1 rows of the m-tile
  float* sD = sA + GM * R;          // [GM][CWs]  dP rows of the m-tile
  const int tid = threadIdx.x;
  const int ty2 = tid >> 4, tx2 = tid & 15;      // dC2 tile: r1 = ty2 + 16 i, c = tx2 + 16 j
  const int ty = tid >> 5, tx = tid & 31;        // dA tile:  m = ty*4 + i,  r1 = tx + 32 j
  const uint32_t NG = a.counts[kCntNG];
  for (uint32_t g = blockIdx.x; g < NG; g += gridDim.x) {
    const uint32_t t = a.grp_t[g], i2 = a.grp_i2[g];
    const uint32_t q0 = a.grp_off[g], q1 = a.grp_off[g + 1];
    const int Mrows = (int)(q1 - q0) * n1;
    const TableMeta tm = a.meta[t];
    const size_t c2o = tm.c2_off + (size_t)i2 * R * NC;
    const float* C1t = a.cores + tm.c1_off;
    for (int c0 = 0; c0 < NC; c0 += a.CW) {
      const int cw = min(a.CW, NC - c0);
      __syncthreads();
      for (int e = tid; e < R * cw; e += 256) {
        const int r = e / cw, cc = e - r * cw;
        sB[r * CWs + cc] = a.cores[c2o + (size_t)r * NC + c0 + cc];
      }
      float acc2[8][8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc2[i][j] = 0.f;
      for (int m0 = 0; m0 < Mrows; m0 += GM) {
        __syncthreads();
        for (int e = tid; e < GM * R; e += 256) {
          const int m = e / R, k = e - m * R;
          const int mr = m0 + m;
          float v = 0.f;
          if (mr < Mrows) {
            const uint32_t p = a.grp_pfx[q0 + mr / n1];
            v = __ldg(C1t + ((size_t)a.pfx_i1[p] * n1 + (mr % n1)) * R + k);
          }
          sA[e] = v;
        }
        for (int e = tid; e < GM * cw; e += 256) {
          const int m = e / cw, cc = e - m * cw;
          const int mr = m0 + m;
          float v = 0.f;
          if (mr < Mrows) {
            const uint32_t p = a.grp_pfx[q0 + mr / n1];
            v = a.dpbuf[((size_t)p * n1 + (mr % n1)) * NC + c0 + cc];
          }
          sD[m * CWs + cc] = v;
        }
        __syncthreads();
        const int mcount = min(GM, Mrows - m0);
        // dC2[r1][c] += sum_m A[m][r1] dP[m][c]
        for (int m = 0; m < mcount; ++m) {
          float av[8], dv[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int r1 = ty2 + 16 * i;
            av[i] = r1 < R ? sA[m * R + r1] : 0.f;
          }
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int cc = tx2 + 16 * j;
            dv[j] = cc < cw ? sD[m * CWs + cc] : 0.f;
          }
#pragma unroll
          for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc2[i][j] = fmaf(av[i], dv[j], acc2[i][j]);
        }
        // dA[m][r1] (+)= sum_c dP[m][c] C2[r1][c] over this chunk
        float accA[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) accA[i][j] = 0.f;
        for (int cc = 0; cc < cw; ++cc) {
          float dv[4], bv[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) dv[i] = sD[(ty * 4 + i) * CWs + cc];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int r1 = tx + 32 * j;
            bv[j] = r1 < R ? sB[r1 * CWs + cc] : 0.f;
          }
#pragma unroll
          for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) accA[i][j] = fmaf(dv[i], bv[j], accA[i][j]);
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int mr = m0 + ty * 4 + i;
          if (mr >= Mrows) continue;
          const uint32_t p = a.grp_pfx[q0 + mr / n1];
          float* dst = a.dabuf + ((size_t)p * n1 + (mr % n1)) * R;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int r1 = tx + 32 * j;
            if (r1 < R) dst[r1] = (c0 == 0) ? accA[i][j] : dst[r1] + accA[i][j];
          }
        }
      }
      // the group owns C2[t][i2]: write its gradient, or apply the fused update
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r1 = ty2 + 16 * i;
        if (r1 >= R) continue;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int cc = tx2 + 16 * j;
          if (cc >= cw) continue;
          const size_t idx = c2o + (size_t)r1 * NC + c0 + cc;
          if (a.fused) apply_update(a.cores + idx, a.state + idx, acc2[i][j], a.lr, a.eps, a.opt);
          else a.grads[idx] = acc2[i][j];
        }
      }
    }
  }
}

// a11: dC1[t][i1] = sum of dA partials over the contiguous prefix run with equal (t, i1)
__global__ void __launch_bounds__(256) k_dc1(BwdArgs a) {
  const int S1 = a.n1 * a.R;
  const uint32_t P = a.counts[kCntP];
  const int64_t total = (int64_t)P * S1;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t p = (uint32_t)(e / S1);
    const int k = (int)(e - (int64_t)p * S1);
    const uint32_t t = a.pfx_t[p], i1 = a.pfx_i1[p];
    if (p > 0 && a.pfx_t[p - 1] == t && a.pfx_i1[p - 1] == i1) continue;   // not a run head
    float acc = 0.f;
    for (uint32_t q = p; q < P && a.pfx_t[q] == t && a.pfx_i1[q] == i1; ++q)
      acc += a.dabuf[(size_t)q * S1 + k];
    const size_t idx = a.meta[t].c1_off + (size_t)i1 * S1 + k;
    if (a.fused) apply_update(a.cores + idx, a.state + idx, acc, a.lr, a.eps, a.opt);
    else a.grads[idx] = acc;
  }
}

// a12: dense update over [begin, begin+n) floats; a zero gradient leaves C and S unchanged
__global__ void __launch_bounds__(256)
k_update(float* __restrict__ cores, float* __restrict__ state, const float* __restrict__ grads,
         size_t begin, size_t n, float lr, float eps, int opt) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (size_t)gridDim.x * blockDim.x) {
    const float g = grads[begin + i];
    if (g != 0.f) apply_update(cores + begin + i, state ? state + begin + i : nullptr, g, lr, eps, opt);
  }
}

}  // namespace

static int bwd_cw(const Ctx& c) { return c.NC < GCW ? c.NC : GCW; }
static size_t bwd_prefix_smem(const Ctx& c) {
  const int CW = bwd_cw(c);
  const int CWs = CW | 1;
  return sizeof(float) * ((size_t)c.R * CWs + (size_t)GM * c.R + (size_t)GM * CWs);
}
static size_t bwd_rows_smem(const Ctx& c) {
  const int J12 = c.n1 * c.n2;
  return sizeof(float) * ((size_t)J12 * (c.R + 1) + (size_t)J12 * c.R + c.N);
}

cudaError_t configure_bwd(Ctx& c) {
  cudaError_t e = cudaFuncSetAttribute(k_bwd_prefix, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)bwd_prefix_smem(c));
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_bwd_rows, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)bwd_rows_smem(c));
}

int64_t agg_chunks(int64_t nnz) { return (nnz + AGG_CS - 1) / AGG_CS; }

cudaError_t run_backward(Ctx& c, const float* grad_out, float lr, cudaStream_t s) {
  const PlanDev& p = c.p;
  const bool fused = (c.flags & TTEMB_FUSED_UPDATE) != 0;
  {
    StageScope sc(c, ST_BWD_ZERO, s);
    if (fused) cudaMemsetAsync(c.grads + c.c3_begin, 0, sizeof(float) * c.c3_floats, s);
    else cudaMemsetAsync(c.grads, 0, sizeof(float) * c.core_floats, s);
  }
  if (c.nnz > 0) {
    StageScope sc(c, ST_AGG, s);
    const int64_t total = agg_chunks(c.nnz) * c.N;
    k_agg<<<grid_for(c, total, 256, 8), 256, 0, s>>>(grad_out, p.skey, p.sbag, p.spos, p.inverse,
                                                     p.seg_off, c.nnz, c.N, p.gbuf, p.aggpart);
  }
  if (c.nnz > 0) {
    StageScope sc(c, ST_AGG_FIX, s);
    k_agg_fix<<<grid_for(c, c.U_cap * c.N, 256, 8), 256, 0, s>>>(p.seg_off, p.counts, c.N, p.aggpart,
                                                                 p.gbuf);
  }
  BwdArgs a;
  a.cores = c.cores; a.grads = c.grads; a.state = c.state; a.meta = c.d_meta;
  a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2;
  a.grp_pfx = p.grp_pfx; a.pfx_t = p.pfx_t; a.pfx_i1 = p.pfx_i1; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.pbuf = p.pbuf; a.gbuf = p.gbuf; a.dpbuf = p.dpbuf; a.dabuf = p.dabuf;
  a.n1 = c.n1; a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.R = c.R; a.NC = c.NC;
  a.CW = bwd_cw(c); a.CWs = a.CW | 1;
  a.lr = lr; a.eps = c.eps; a.opt = c.opt; a.fused = fused ? 1 : 0;
  if (c.nnz > 0) {
    {
      StageScope sc(c, ST_BWD_ROWS, s);
      k_bwd_rows<<<grid_for(c, c.P_cap, 1, 8), 128, bwd_rows_smem(c), s>>>(a);
    }
    {
      StageScope sc(c, ST_BWD_PREFIX, s);
      k_bwd_prefix<<<grid_for(c, c.NG_cap, 1, 2), 256, bwd_prefix_smem(c), s>>>(a);
    }
    {
      StageScope sc(c, ST_DC1, s);
      k_dc1<<<grid_for(c, c.P_cap * c.n1 * c.R, 256, 8), 256, 0, s>>>(a);
    }
  }
  if (fused) {
    StageScope sc(c, ST_UPD_C3, s);
    k_update<<<grid_for(c, (int64_t)c.c3_floats, 256, 8), 256, 0, s>>>(
        c.cores, c.state, c.grads, c.c3_begin, c.c3_floats, lr, c.eps, c.opt);
  }
  return cudaGetLastError();
}

cudaError_t run_update(Ctx& c, float lr, cudaStream_t s) {
  StageScope sc(c, ST_UPDATE, s);
  k_update<<<grid_for(c, (int64_t)c.core_floats, 256, 8), 256, 0, s>>>(
      c.cores, c.state, c.grads, 0, c.core_floats, lr, c.eps, c.opt);
  return cudaGetLastError();
}

}  // namespace ttemb
