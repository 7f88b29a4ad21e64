// ttemb_fwd.cu -- forward contractions and pooling, sm_100a.
//
//   a5 prefix contraction, one CTA per i2-group g = (t, i2):
//        P_g = A_g . C2[i2]     A_g = the C1[i1] slices of the group's prefixes stacked
//        ((Q n1) x R), C2[i2] viewed as (R x n2 R); the result rows are the Reuse buffer
//        entries P_p[j1][j2][r2] = sum_r1 C1[i1,j1,r1] C2[i2,r1,j2,r2]
//      C2[i2] is staged in shared memory once per group (column chunks of <= 128).
//   a6 row contraction E_u = P_p (n1 n2 x R) . C3[i3] (R x n3)  (Eq. 2, P:164 step 3)
//   a7 sum pooling out[b][t] = sum_{j in bag} E_{inverse[j]}     (Eq. 4, P:164 step 4)
// FP32 FFMA on CUDA cores (tensor cores only where ncu shows the rank-R
// contraction is the bottleneck).
#include "ttemb_internal.cuh"

namespace ttemb {

namespace {

constexpr int GM = 32;      // rows (prefix, j1) per m-tile
constexpr int GCW = 128;    // max C2 columns per chunk

struct FwdArgs {
  const float* cores;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_t, *pfx_i1, *row_seg, *row_i3;
  float* pbuf;
  float* rows;
  int n1, n2, n3, N, R, NC, CW, CWp;
};

// a5: P_g = A_g . C2[i2], tile 32 rows x CW columns, 4x4 outputs per thread
__global__ void __launch_bounds__(256) k_fwd_prefix(FwdArgs a) {
  extern __shared__ __align__(16) float smem[];
  const int R = a.R, NC = a.NC, CWp = a.CWp, n1 = a.n1;
  float* sB = smem;                 // [R][CWp]
  float* sAT = smem + R * CWp;      // [R][GM]  (A transposed)
  const int tid = threadIdx.x, ty = tid >> 5, tx = tid & 31;
  const uint32_t NG = a.counts[kCntNG];
  for (uint32_t g = blockIdx.x; g < NG; g += gridDim.x) {
    const uint32_t t = a.grp_t[g], i2 = a.grp_i2[g];
    const uint32_t q0 = a.grp_off[g], q1 = a.grp_off[g + 1];
    const int Mrows = (int)(q1 - q0) * n1;
    const TableMeta tm = a.meta[t];
    const float* C2s = a.cores + tm.c2_off + (size_t)i2 * R * NC;
    const float* C1t = a.cores + tm.c1_off;
    for (int c0 = 0; c0 < NC; c0 += a.CW) {
      const int cw = min(a.CW, NC - c0);
      __syncthreads();
      for (int e = tid; e < R * CWp; e += 256) {
        const int r = e / CWp, cc = e - r * CWp;
        sB[e] = cc < cw ? __ldg(C2s + (size_t)r * NC + c0 + cc) : 0.f;
      }
      for (int m0 = 0; m0 < Mrows; m0 += GM) {
        __syncthreads();
        for (int e = tid; e < R * GM; e += 256) {
          const int k = e / GM, m = e - k * GM;
          const int mr = m0 + m;
          float v = 0.f;
          if (mr < Mrows) {
            const uint32_t p = a.grp_pfx[q0 + mr / n1];
            const uint32_t i1 = a.pfx_i1[p];
            v = __ldg(C1t + ((size_t)i1 * n1 + (mr % n1)) * R + k);
          }
          sAT[e] = v;
        }
        __syncthreads();
        float acc[4][4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
        if (tx * 4 < cw) {
          for (int k = 0; k < R; ++k) {
            const float4 av = *reinterpret_cast<const float4*>(sAT + k * GM + ty * 4);
            const float4 bv = *reinterpret_cast<const float4*>(sB + k * CWp + tx * 4);
            const float ar[4] = {av.x, av.y, av.z, av.w};
            const float br[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
              for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(ar[i], br[j], acc[i][j]);
          }
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int mr = m0 + ty * 4 + i;
          if (mr >= Mrows) continue;
          const uint32_t p = a.grp_pfx[q0 + mr / n1];
          float* dst = a.pbuf + ((size_t)p * n1 + (mr % n1)) * NC + c0;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int cc = tx * 4 + j;
            if (cc < cw) dst[cc] = acc[i][j];
          }
        }
      }
    }
  }
}

// a6: E_u = P_p . C3[i3] for every unique row of prefix p; one CTA per prefix
__global__ void __launch_bounds__(128) k_fwd_rows(FwdArgs a) {
  extern __shared__ __align__(16) float smem[];
  const int R = a.R, N = a.N, n3 = a.n3, J12 = a.n1 * a.n2, ldp = R + 1;
  float* sP = smem;   // [J12][R+1]
  const uint32_t P = a.counts[kCntP];
  for (uint32_t p = blockIdx.x; p < P; p += gridDim.x) {
    __syncthreads();
    const float* src = a.pbuf + (size_t)p * J12 * R;
    for (int e = threadIdx.x; e < J12 * R; e += blockDim.x) {
      const int j = e / R, r = e - j * R;
      sP[j * ldp + r] = src[e];
    }
    __syncthreads();
    const uint32_t u0 = a.row_seg[p], u1 = a.row_seg[p + 1];
    const TableMeta tm = a.meta[a.pfx_t[p]];
    const int total = (int)(u1 - u0) * N;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int ul = e / N, col = e - ul * N;
      const int j12 = col / n3, j3 = col - j12 * n3;
      const uint32_t u = u0 + ul;
      const float* c3 = a.cores + tm.c3_off + (size_t)a.row_i3[u] * R * n3;
      float acc = 0.f;
      for (int r = 0; r < R; ++r) acc = fmaf(sP[j12 * ldp + r], __ldg(c3 + r * n3 + j3), acc);
      a.rows[(size_t)u * N + col] = acc;
    }
  }
}

// a7: out[b][t][:] = sum over the bag's positions (index order); empty bag -> 0
__global__ void __launch_bounds__(256)
k_pool(const float* __restrict__ rows, const uint32_t* __restrict__ inverse,
       const int64_t* __restrict__ offsets, int64_t nnz, int T, int B, int N, float* __restrict__ out) {
  const int64_t total = (int64_t)T * B * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t bag = e / N;
    const int col = (int)(e - bag * N);
    const int t = (int)(bag / B);
    const int64_t b = bag - (int64_t)t * B;
    int64_t s = offsets[bag], f = offsets[bag + 1];
    s = s < 0 ? 0 : (s > nnz ? nnz : s);
    f = f < s ? s : (f > nnz ? nnz : f);
    float acc = 0.f;
    for (int64_t j = s; j < f; ++j) acc += rows[(size_t)inverse[j] * N + col];
    out[((size_t)b * T + t) * N + col] = acc;
  }
}

}  // namespace

static size_t fwd_prefix_smem(const Ctx& c) {
  const int CW = c.NC < GCW ? c.NC : GCW;
  const int CWp = (CW + 3) & ~3;
  return sizeof(float) * ((size_t)c.R * CWp + (size_t)c.R * GM);
}
static size_t fwd_rows_smem(const Ctx& c) { return sizeof(float) * (size_t)c.n1 * c.n2 * (c.R + 1); }

cudaError_t configure_fwd(Ctx& c) {
  cudaError_t e = cudaFuncSetAttribute(k_fwd_prefix, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)fwd_prefix_smem(c));
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_fwd_rows, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)fwd_rows_smem(c));
}

cudaError_t run_forward_compute(Ctx& c, float* out, const int64_t* offsets, cudaStream_t s) {
  const PlanDev& p = c.p;
  FwdArgs a;
  a.cores = c.cores; a.meta = c.d_meta;
  a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2;
  a.grp_pfx = p.grp_pfx; a.pfx_t = p.pfx_t; a.pfx_i1 = p.pfx_i1; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.pbuf = p.pbuf; a.rows = p.rows;
  a.n1 = c.n1; a.n2 = c.n2; a.n3 = c.n3; a.N = c.N; a.R = c.R; a.NC = c.NC;
  a.CW = c.NC < GCW ? c.NC : GCW;
  a.CWp = (a.CW + 3) & ~3;
  {
    StageScope sc(c, ST_FWD_PREFIX, s);
    k_fwd_prefix<<<grid_for(c, c.NG_cap, 1, 2), 256, fwd_prefix_smem(c), s>>>(a);
  }
  {
    StageScope sc(c, ST_FWD_ROWS, s);
    k_fwd_rows<<<grid_for(c, c.P_cap, 1, 8), 128, fwd_rows_smem(c), s>>>(a);
  }
  {
    StageScope sc(c, ST_POOL, s);
    const int64_t total = (int64_t)c.T * c.B * c.N;
    if (total > 0)
      k_pool<<<grid_for(c, total, 256, 8), 256, 0, s>>>(p.rows, p.inverse, offsets, c.nnz, c.T, c.B,
                                                        c.N, out);
  }
  return cudaGetLastError();
}

}  // namespace ttemb
