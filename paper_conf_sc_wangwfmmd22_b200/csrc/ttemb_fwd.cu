// ttemb_fwd.cu -- forward driver, pooling and the dense (hybrid) rows (SURVEY 8(a) row a7,
// 8(f3)), sm_100a.
//
//   a5 + a6 run in the tensor-core kernels (ttemb_fused.cu, R = 64) or the FFMA group kernels
//   (ttemb_group.cu); this file dispatches them, copies the rows of dense (hybrid) tables
//   (k_dense_fwd) and pools:
//   a7 out[b][t] = sum_{j in bag} w_j E_{inverse[j]}   (Eq. 4, P:164 step 4; w_j = 1, the
//      per-sample weight or 1/|bag| for nn.EmbeddingBag "mean", P:48 / P:306)
#include <type_traits>

#include "ttemb_internal.cuh"

#ifndef TTEMB_POOL_MODE
#define TTEMB_POOL_MODE 1     // one-hot pooling: 1 = output-ordered, 0 = position-ordered scatter
#endif
#ifndef TTEMB_POOL_IPT
#define TTEMB_POOL_IPT 2      // independent float4 items per thread (output-ordered kernel)
#endif
#ifndef TTEMB_POOL_STCS
#define TTEMB_POOL_STCS 1     // 1 = streaming (evict-first) stores of the pooled output
#endif
#ifndef TTEMB_POOL_PER_SM
#define TTEMB_POOL_PER_SM 16  // grid cap, CTAs per SM (16 vs 32: one-hot pool 33.5 vs 34.9 us at c4)
#endif

namespace ttemb {

namespace {

// the pooled output is written once and not re-read by this step: optionally streamed past L2
__device__ __forceinline__ void pool_store(float4* p, float4 v) {
#if TTEMB_POOL_STCS
  __stcs(p, v);
#else
  *p = v;
#endif
}

// a7: out[b][t][:] = sum over the bag's positions (index order); empty bag -> 0.
// Thread = (bag, VW-wide column group); 4 independent items per thread are processed
// together so their index -> row loads overlap.
template <int VW>
__global__ void __launch_bounds__(256)
k_pool(const float* __restrict__ rows, const uint32_t* __restrict__ inverse,
       const int64_t* __restrict__ offsets, int64_t nnz, int T, int B, int N, float* __restrict__ out,
       const uint32_t* __restrict__ counts, int skip_single, const float* __restrict__ wpos) {
  pdl_wait();
  if (skip_single && counts[kCntMulti] == 0) return;   // one id per bag: written directly
  using V = typename std::conditional<VW == 4, float4, float>::type;
  const uint32_t NV = (uint32_t)(N / VW);
  const uint32_t total = (uint32_t)T * (uint32_t)B * NV;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t e0 = blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += 4 * stride) {
    int64_t s[4], f[4];
    uint32_t bag[4], col[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const uint32_t e = e0 + i * stride;
      bag[i] = e / NV;
      col[i] = (e - bag[i] * NV) * VW;
      s[i] = f[i] = 0;
      if (e < total) {
        s[i] = __ldg(offsets + bag[i]);
        f[i] = __ldg(offsets + bag[i] + 1);
        s[i] = s[i] < 0 ? 0 : (s[i] > nnz ? nnz : s[i]);
        f[i] = f[i] < s[i] ? s[i] : (f[i] > nnz ? nnz : f[i]);
      }
    }
    V acc[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      acc[i] = V{};
      for (int64_t j = s[i]; j < f[i]; ++j) {
        const V v = __ldg(reinterpret_cast<const V*>(rows + (size_t)__ldg(inverse + j) * N + col[i]));
        const float w = wpos ? __ldg(wpos + j) : 1.f;   // per-sample weight / 1 / |bag|
        if constexpr (VW == 4) { acc[i].x += w * v.x; acc[i].y += w * v.y; acc[i].z += w * v.z; acc[i].w += w * v.w; }
        else acc[i] += w * v;
      }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      if (e0 + i * stride >= total) continue;
      const uint32_t t = bag[i] / (uint32_t)B, b = bag[i] - t * (uint32_t)B;
      *reinterpret_cast<V*>(out + ((size_t)b * T + t) * N + col[i]) = acc[i];
    }
  }
}

// a7 when every bag holds exactly one id (the one-hot configs): out[bag_of[j]] = E_{inverse[j]}
// -- thread = (position, float4 column), four independent items per thread.
__global__ void __launch_bounds__(256)
k_pool_single(const float* __restrict__ rows, const uint32_t* __restrict__ inverse,
              const uint32_t* __restrict__ bag_of, int64_t nnz, int N, float* __restrict__ out,
              const uint32_t* __restrict__ counts, const float* __restrict__ wpos) {
  if (counts[kCntMulti] != 0) return;
  const int NV = N >> 2;
  const int64_t total = nnz * NV, stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += 4 * stride) {
    float4 v[4];
    int64_t dst[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int64_t e = e0 + i * stride;
      dst[i] = -1;
      if (e < total) {
        const int64_t j = e / NV;
        const int f = (int)(e - j * NV);
        v[i] = __ldg(reinterpret_cast<const float4*>(rows + (size_t)__ldg(inverse + j) * N) + f);
        if (wpos) {
          const float w = __ldg(wpos + j);
          v[i].x *= w; v[i].y *= w; v[i].z *= w; v[i].w *= w;
        }
        dst[i] = (int64_t)__ldg(bag_of + j) * NV + f;
      }
    }
#pragma unroll
    for (int i = 0; i < 4; ++i)
      if (dst[i] >= 0) pool_store(reinterpret_cast<float4*>(out) + dst[i], v[i]);
  }
}

// a7 one-hot, output-ordered: with one id per bag the validated offsets are the identity
// (offsets[bag] = bag), so output row o = b*T + t reads position j = t*B + b directly and the
// 109 MB (C4) output is written in address order.  Thread = (output row, float4 column).
// Index math in I (uint32_t whenever the float4 count fits, the common case: a 64-bit division
// is a long software sequence and made this copy ALU-bound), float4 columns per row NV = 2^nvs.
template <typename I>
__global__ void __launch_bounds__(256)
k_pool_single_out(const float* __restrict__ rows, const uint32_t* __restrict__ inverse, int64_t nnz,
                  int T, int B, int N, int nvs, float* __restrict__ out, const uint32_t* __restrict__ counts,
                  const float* __restrict__ wpos) {
  pdl_wait();
  if (counts[kCntMulti] != 0) return;
  const I NV = (I)(N >> 2), uT = (I)T, uB = (I)B;
  const I total = (I)T * (I)B * NV, stride = (I)gridDim.x * blockDim.x;
  for (I e0 = (I)blockIdx.x * blockDim.x + threadIdx.x; e0 < total; e0 += TTEMB_POOL_IPT * stride) {
    float4 v[TTEMB_POOL_IPT];
#pragma unroll
    for (int i = 0; i < TTEMB_POOL_IPT; ++i) {
      const I e = e0 + (I)i * stride;
      v[i] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (e < total) {
        const I o = nvs >= 0 ? (e >> nvs) : e / NV;
        const I f = e - o * NV;
        const I b = o / uT, t = o - b * uT, j = t * uB + b;
        if ((int64_t)j < nnz) {
          v[i] = __ldg(reinterpret_cast<const float4*>(rows + (size_t)__ldg(inverse + j) * N) + f);
          if (wpos) {
            const float w = __ldg(wpos + j);
            v[i].x *= w; v[i].y *= w; v[i].z *= w; v[i].w *= w;
          }
        }
      }
    }
#pragma unroll
    for (int i = 0; i < TTEMB_POOL_IPT; ++i)
      if (e0 + (I)i * stride < total) pool_store(reinterpret_cast<float4*>(out) + e0 + (I)i * stride, v[i]);
  }
}

// Hybrid placement: the unique rows of dense tables, [Utt, U), are plain table rows:
// rows[u] = W_t[row].  Thread = (row, column); coalesced along the row.
__global__ void __launch_bounds__(256)
k_dense_fwd(const float* __restrict__ cores, const TableMeta* __restrict__ meta,
            const uint64_t* __restrict__ kbase, const uint32_t* __restrict__ kmap, int T,
            const uint32_t* __restrict__ ukey, const uint32_t* __restrict__ counts, int N,
            float* __restrict__ rows) {
  const uint32_t U = counts[kCntU], u0 = tt_rows(counts);
  const int64_t total = (int64_t)(U - u0) * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t u = u0 + (uint32_t)(e / N);
    const int col = (int)(e % N);
    const uint32_t key = __ldg(ukey + u);
    const int it = table_of_key(kbase, T, key);
    const TableMeta& m = meta[__ldg(kmap + it)];
    rows[(size_t)u * N + col] = __ldg(cores + m.c1_off + (size_t)(key - __ldg(kbase + it)) * N + col);
  }
}

}  // namespace

cudaError_t run_dense_fwd(Ctx& c, cudaStream_t s) {
  StageScope sc(c, ST_FWD_ROWS, s);
  k_dense_fwd<<<grid_for(c, (int64_t)c.U_cap * c.N, 256, 8), 256, 0, s>>>(
      c.cores, c.d_meta, c.d_kbase, c.d_kmap, c.T, c.p.ukey, c.p.counts, c.N, c.p.rows);
  return cudaGetLastError();
}

cudaError_t run_group_fwd(Ctx& c, cudaStream_t s);

cudaError_t run_forward_compute(Ctx& c, float* out, const int64_t* offsets, cudaStream_t s) {
  const PlanDev& p = c.p;
  const bool tc = tc_eligible(c);
  if (c.nnz > 0) {
    cudaError_t e = tc ? run_tc_fwd(c, out, s) : run_group_fwd(c, s);
    if (e == cudaSuccess && c.n_dense > 0) e = run_dense_fwd(c, s);
    if (e != cudaSuccess) return e;
  }
  {
    StageScope sc(c, ST_POOL, s);
    const int64_t total = (int64_t)c.T * c.B * c.N;
    if (total > 0) {
      if (c.N % 4 == 0) {
        // one id per bag (device flag): a position-parallel copy; otherwise the bag-parallel sum
        if (c.nnz > 0) {
          if (TTEMB_POOL_MODE == 1) {
            const int grid = grid_for(c, total / (4 * TTEMB_POOL_IPT), 256, TTEMB_POOL_PER_SM);
            const int nv = c.N / 4, nvs = (nv & (nv - 1)) == 0 ? __builtin_ctz(nv) : -1;
            const int64_t span = total / 4 + (int64_t)TTEMB_POOL_IPT * grid * 256;   // largest index formed
            const float* wp = c.weighted ? p.wpos : nullptr;
            if (span < ((int64_t)1 << 32))
              launch_pdl(k_pool_single_out<uint32_t>, dim3(grid), dim3(256), 0, s, (const float*)p.rows,
                         (const uint32_t*)p.inverse, (int64_t)c.nnz, c.T, c.B, c.N, nvs, out, (const uint32_t*)p.counts, wp);
            else
              launch_pdl(k_pool_single_out<uint64_t>, dim3(grid), dim3(256), 0, s, (const float*)p.rows,
                         (const uint32_t*)p.inverse, (int64_t)c.nnz, c.T, c.B, c.N, nvs, out, (const uint32_t*)p.counts, wp);
          } else
            k_pool_single<<<grid_for(c, c.nnz * c.N / 16, 256, TTEMB_POOL_PER_SM), 256, 0, s>>>(
                p.rows, p.inverse, p.bag_of, c.nnz, c.N, out, p.counts, c.weighted ? p.wpos : nullptr);
        }
        // the multi-hot sum exits at once on one-hot batches: one wave of CTAs, not four
        launch_pdl(k_pool<4>, dim3(grid_for(c, total / 16, 256, 8)), dim3(256), 0, s, (const float*)p.rows,
                   (const uint32_t*)p.inverse, offsets, (int64_t)c.nnz, c.T, c.B, c.N, out, (const uint32_t*)p.counts, 1,
                   (const float*)(c.weighted ? p.wpos : nullptr));
      }
      else
        k_pool<1><<<grid_for(c, total / 4, 256, 32), 256, 0, s>>>(p.rows, p.inverse, offsets, c.nnz, c.T,
                                                             c.B, c.N, out, p.counts, 0,
                                                             c.weighted ? p.wpos : nullptr);
    }
  }
  return cudaGetLastError();
}

}  // namespace ttemb
