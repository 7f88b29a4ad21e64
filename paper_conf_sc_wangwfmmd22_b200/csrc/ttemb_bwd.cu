// ttemb_bwd.cu -- backward driver, aggregation and updates, sm_100a.
//
//   a8  in-advance aggregation G_u = sum_{positions of row u} w_j grad_out[bag]:
//       k_agg_scatter (warp per 32 sorted occurrences, vector reductions) or the deterministic
//       fixed-chunk segmented reduction k_agg + k_agg_fix (other dims)
//   a9-a11 in the tensor-core kernels (ttemb_fused.cu / ttemb_bwdtc.cu) or the FFMA group
//       kernels (ttemb_group.cu; k_dc1 reduces their per-prefix dC1 partials)
//   a12 SGD / Adagrad: fused on one replica (C2 by its owning CTA, C1 + C3 by k_update_zero,
//       dense tables by k_dense_bwd; "fused TT core update"), else k_update after
//       the caller's gradient all-reduce
#include <type_traits>

#include "ttemb_internal.cuh"

#ifndef TTEMB_AGG_LDCS
#define TTEMB_AGG_LDCS 1      // 1 = streaming loads of grad_out in the one-hot aggregation
#endif

namespace ttemb {

namespace {

constexpr int AGG_CS = 32;   // sorted positions per aggregation chunk
#ifndef TTEMB_UPD_GRID
#define TTEMB_UPD_GRID 8    // fused C1 / C3 update grid cap, CTAs per SM
#endif
#ifndef TTEMB_AGG_GRID
#define TTEMB_AGG_GRID 32   // k_agg_scatter grid cap, CTAs per SM
#endif
#ifndef TTEMB_AGG_B
#define TTEMB_AGG_B 8
#endif
constexpr int AGG_B = TTEMB_AGG_B;   // grad_out rows per lane group loaded ahead in k_agg_scatter

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

// a8 part 1: thread = (chunk of AGG_CS sorted positions, VW-wide column group)
template <int VW>
__global__ void __launch_bounds__(256)
k_agg(const float* __restrict__ grad_out, const uint32_t* __restrict__ skey,
      const uint32_t* __restrict__ sbag, const uint32_t* __restrict__ spos,
      const uint32_t* __restrict__ inverse, const uint32_t* __restrict__ seg_off, int64_t nnz,
      int N, float* __restrict__ gbuf, float* __restrict__ part, const float* __restrict__ wpos) {
  using V = typename std::conditional<VW == 4, float4, float>::type;
  const int NV = N / VW;
  const uint32_t nchunks = (uint32_t)((nnz + AGG_CS - 1) / AGG_CS);
  const uint32_t total = nchunks * NV;
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < total; e += gridDim.x * blockDim.x) {
    const uint32_t ch = e / NV;
    const int col = (int)(e - ch * NV) * VW;
    const int64_t k0 = ch * AGG_CS, k1 = min(k0 + AGG_CS, nnz);
    V acc = V{};
    for (int64_t k = k0; k < k1; ++k) {
      const V v = __ldg(reinterpret_cast<const V*>(grad_out + (size_t)__ldg(sbag + k) * N + col));
      const float w = wpos ? __ldg(wpos + __ldg(spos + k)) : 1.f;   // d out / d row_j = w_j
      if constexpr (VW == 4) { acc.x += w * v.x; acc.y += w * v.y; acc.z += w * v.z; acc.w += w * v.w; }
      else acc += w * v;
      const bool seg_end = (k + 1 == nnz) || __ldg(skey + k + 1) != __ldg(skey + k);
      if (seg_end || k + 1 == k1) {
        const uint32_t u = inverse[spos[k]];
        const int64_t s0 = seg_off[u], s1 = seg_off[u + 1];
        float* dst;
        if (s0 >= k0 && s1 <= k1) dst = gbuf + (size_t)u * N + col;
        else if (s0 < k0) dst = part + ((size_t)ch * 2 + 0) * N + col;   // head: began earlier
        else dst = part + ((size_t)ch * 2 + 1) * N + col;                // tail: continues
        *reinterpret_cast<V*>(dst) = acc;
        acc = V{};
      }
    }
  }
}

// a8 part 2: a row whose segment spans chunks c0..c1 is finished by the warp of chunk c1
// (the chunk where it ends): G = tail(c0) + heads(c0+1..c1).  Lanes split the chunk range
// (fixed strided partition + butterfly), so Zipf-hot rows spanning hundreds of chunks
// stay cheap; the summation order is fixed, hence deterministic.
__global__ void __launch_bounds__(256)
k_agg_fix(const uint32_t* __restrict__ skey, const uint32_t* __restrict__ spos,
          const uint32_t* __restrict__ inverse, const uint32_t* __restrict__ seg_off, int64_t nnz,
          int N, const float* __restrict__ part, float* __restrict__ gbuf) {
  const int64_t nchunks = (nnz + AGG_CS - 1) / AGG_CS;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t ch = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); ch < nchunks;
       ch += warps) {
    const int64_t k = ch * AGG_CS;
    if (ch == 0 || skey[k] != skey[k - 1]) continue;      // chunk starts a fresh segment
    const uint32_t u = inverse[spos[k]];
    const int64_t c0 = seg_off[u] / AGG_CS, c1 = (seg_off[u + 1] - 1) / AGG_CS;
    if (c1 != ch) continue;                                // not the segment's last chunk
    // G = tail(c0) + heads(c0+1 .. c1).  N % 4 == 0: lanes = (float4 column group cq < 16,
    // half h of the chunk range); 4 independent accumulators each; one shuffle joins halves.
    if ((N & 3) == 0) {
      const int cq = lane & 15, h = lane >> 4;
      for (int c4 = cq; c4 < N / 4; c4 += 16) {
        float4 acc[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) acc[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (h == 0) acc[0] = *reinterpret_cast<const float4*>(part + ((size_t)c0 * 2 + 1) * N + 4 * c4);
        int64_t c = c0 + 1 + h;
        int i = 0;
        for (; c <= c1; c += 2, i = (i + 1) & 3) {
          const float4 v = *reinterpret_cast<const float4*>(part + ((size_t)c * 2) * N + 4 * c4);
          acc[i].x += v.x; acc[i].y += v.y; acc[i].z += v.z; acc[i].w += v.w;
        }
        float4 r;
        r.x = (acc[0].x + acc[1].x) + (acc[2].x + acc[3].x);
        r.y = (acc[0].y + acc[1].y) + (acc[2].y + acc[3].y);
        r.z = (acc[0].z + acc[1].z) + (acc[2].z + acc[3].z);
        r.w = (acc[0].w + acc[1].w) + (acc[2].w + acc[3].w);
        r.x += __shfl_xor_sync(0xffffffffu, r.x, 16);
        r.y += __shfl_xor_sync(0xffffffffu, r.y, 16);
        r.z += __shfl_xor_sync(0xffffffffu, r.z, 16);
        r.w += __shfl_xor_sync(0xffffffffu, r.w, 16);
        if (h == 0) *reinterpret_cast<float4*>(gbuf + (size_t)u * N + 4 * c4) = r;
      }
    } else {
      for (int col = lane; col < N; col += 32) {
        float acc = part[((size_t)c0 * 2 + 1) * N + col];
        for (int64_t c = c0 + 1; c <= c1; ++c) acc += part[((size_t)c * 2) * N + col];
        gbuf[(size_t)u * N + col] = acc;
      }
    }
  }
}


// a8 (in-advance gradient aggregation): G_u = sum of grad_out over the occurrences of
// unique row u.  Warp = 32 consecutive sorted occurrences; each half-warp walks every other
// occurrence (lanes = float4 columns) and adds its running sum into G_u with one vector
// reduction per (half-warp, segment piece).  Zipf-hot rows (thousands of occurrences) are
// spread over many warps; G is zeroed first (rows [0, U) only).
__global__ void __launch_bounds__(256) k_zero_rows(float* __restrict__ buf, const uint32_t* __restrict__ counts, int N) {
  const int64_t n4 = (int64_t)counts[kCntU] * N / 4;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
    reinterpret_cast<float4*>(buf)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
}

__global__ void __launch_bounds__(256)
k_agg_scatter(const float* __restrict__ grad_out, const uint32_t* __restrict__ sbag,
              const uint32_t* __restrict__ spos, const uint32_t* __restrict__ inverse, int64_t nnz, int N,
              float* __restrict__ gbuf, const float* __restrict__ wpos, const uint32_t* __restrict__ counts) {
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int NV = N >> 2, P = 32 / NV;   // float4 columns; occurrences in flight per step
  // one id per bag: every grad_out row is read exactly once -> evict-first loads keep L2 for G
  const bool once = TTEMB_AGG_LDCS && __ldg(counts + kCntMulti) == 0;
  const int f = lane % NV, p = lane / NV;
  const int64_t nch = (nnz + 31) / 32;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t ch = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); ch < nch; ch += nw) {
    const int64_t k0 = ch * 32;
    const int cnt = (int)min((int64_t)32, nnz - k0);
    uint32_t bl = 0, ul = 0xffffffffu;
    float wl = 1.f;
    if (lane < cnt) {
      bl = __ldg(sbag + k0 + lane);
      const uint32_t pos = __ldg(spos + k0 + lane);
      ul = __ldg(inverse + pos);
      if (wpos) wl = __ldg(wpos + pos);
    }
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    uint32_t cur = 0xffffffffu;
    // AGG_B occurrences of this lane group are loaded before any is added (AGG_B loads in flight
    // per lane instead of one dependent load per step)
    for (int i0 = 0; i0 < cnt; i0 += AGG_B * P) {
      float4 v[AGG_B];
#pragma unroll
      for (int t = 0; t < AGG_B; ++t) {
        const int i = i0 + t * P + p;
        const uint32_t bag = __shfl_sync(0xffffffffu, bl, i & 31);
        v[t] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (i < cnt) {
          const float4* gp = reinterpret_cast<const float4*>(grad_out + (size_t)bag * N) + f;
          v[t] = once ? __ldcs(gp) : __ldg(gp);
        }
      }
#pragma unroll
      for (int t = 0; t < AGG_B; ++t) {
        const int i = i0 + t * P + p;
        const uint32_t u = __shfl_sync(0xffffffffu, ul, i & 31);
        const float w = __shfl_sync(0xffffffffu, wl, i & 31);
        if (i < cnt) {
          if (u != cur) {
            if (cur != 0xffffffffu)
              asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(gbuf + (size_t)cur * N + 4 * f),
                           "f"(acc.x), "f"(acc.y), "f"(acc.z), "f"(acc.w) : "memory");
            acc = make_float4(0.f, 0.f, 0.f, 0.f);
            cur = u;
          }
          acc.x += w * v[t].x; acc.y += w * v[t].y; acc.z += w * v[t].z; acc.w += w * v[t].w;
        }
      }
    }
    if (cur != 0xffffffffu)
      asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(gbuf + (size_t)cur * N + 4 * f),
                   "f"(acc.x), "f"(acc.y), "f"(acc.z), "f"(acc.w) : "memory");
  }
}

struct BwdArgs {
  float* cores;
  float* grads;
  float* state;
  const TableMeta* meta;
  const uint32_t *counts, *grp_off, *grp_t, *grp_i2, *grp_pfx, *pfx_t, *pfx_i1, *row_seg, *row_i3;
  const float* gbuf;
  float* dabuf;
  int n1, N, R;
  float lr, eps;
  int opt, fused;
};

// a11: dC1[t][i1] = sum of the dA partials of every prefix with that (t, i1).  In the
// group-major plan those prefixes are spread over the i2-groups, so the partials are added
// into the (zeroed, L2-resident) C1 gradient region with vector reductions (Fig. 6(a) step 2,
// P:191); the fused path then updates C1 densely together with C3.
__global__ void __launch_bounds__(256) k_dc1(BwdArgs a) {
  const int S4 = (a.n1 * a.R) >> 2;
  const uint32_t P = a.counts[kCntP];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < (int64_t)P * S4;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t q = (uint32_t)(e / S4);
    const int k4 = (int)(e - (int64_t)q * S4);
    const float4 v = __ldg(reinterpret_cast<const float4*>(a.dabuf) + e);
    float* dst = a.grads + a.meta[a.pfx_t[q]].c1_off + (size_t)a.pfx_i1[q] * (4 * S4) + 4 * k4;
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(dst), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w)
                 : "memory");
  }
}

__global__ void __launch_bounds__(256) k_dc1_scalar(BwdArgs a) {
  const int S1 = a.n1 * a.R;
  const uint32_t P = a.counts[kCntP];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < (int64_t)P * S1;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t q = (uint32_t)(e / S1);
    const int k = (int)(e - (int64_t)q * S1);
    atomicAdd(a.grads + a.meta[a.pfx_t[q]].c1_off + (size_t)a.pfx_i1[q] * S1 + k, __ldg(a.dabuf + e));
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

// Fused update of the C1 and C3 regions (one launch over both): apply, then clear the gradient
// accumulator, so the next backward starts from zero without a memset (the buffer is zeroed once
// by ttemb_create).
__global__ void __launch_bounds__(256)
k_update_zero(float* __restrict__ cores, float* __restrict__ state, float* __restrict__ grads, size_t n1,
              size_t begin2, size_t n2, float lr, float eps, int opt) {
  const size_t n = n1 + n2;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const size_t e = i < n1 ? i : begin2 + (i - n1);
    const float g = grads[e];
    if (g != 0.f) {
      apply_update(cores + e, state ? state + e : nullptr, g, lr, eps, opt);
      grads[e] = 0.f;
    }
  }
}

// k_update_zero on float4 (both regions are multiples of 4 floats): the mostly-zero gradient is
// streamed once and the parameters / state are read only for float4 groups that carry a gradient;
// per element the same arithmetic as k_update_zero.
__global__ void __launch_bounds__(256)
k_update_zero4(float* __restrict__ cores, float* __restrict__ state, float* __restrict__ grads, size_t n1,
               size_t begin2, size_t n2, float lr, float eps, int opt) {
  pdl_wait();
  pdl_trigger();
  const size_t n = (n1 + n2) / 4;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    const size_t e = 4 * i < n1 ? 4 * i : begin2 + (4 * i - n1);
    const float4 g = *reinterpret_cast<const float4*>(grads + e);
    if (g.x == 0.f && g.y == 0.f && g.z == 0.f && g.w == 0.f) continue;
    const float gv[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if (gv[k] != 0.f) apply_update(cores + e + k, state ? state + e + k : nullptr, gv[k], lr, eps, opt);
    *reinterpret_cast<float4*>(grads + e) = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

}  // namespace

cudaError_t run_group_bwd(Ctx& c, float lr, cudaStream_t s);

int64_t agg_chunks(int64_t nnz) { return (nnz + AGG_CS - 1) / AGG_CS; }
int64_t dc1_chunks(int64_t P) { return 1; }

// Hybrid placement: dense-table rows [Utt, U) take their aggregated gradient G_u
// directly: dW[row] = G_u (written to the gradient buffer), or -- fused, one replica -- the
// row is updated in place (each unique row is owned by one thread per column: no races).
__global__ void __launch_bounds__(256)
k_dense_bwd(float* __restrict__ cores, float* __restrict__ state, float* __restrict__ grads,
            const TableMeta* __restrict__ meta, const uint64_t* __restrict__ kbase,
            const uint32_t* __restrict__ kmap, int T, const uint32_t* __restrict__ ukey,
            const uint32_t* __restrict__ counts, int N, const float* __restrict__ gbuf, int fused,
            float lr, float eps, int opt) {
  const uint32_t U = counts[kCntU], u0 = tt_rows(counts);
  const int64_t total = (int64_t)(U - u0) * N;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t u = u0 + (uint32_t)(e / N);
    const int col = (int)(e % N);
    const uint32_t key = __ldg(ukey + u);
    const int it = table_of_key(kbase, T, key);
    const TableMeta& m = meta[__ldg(kmap + it)];
    const size_t dst = m.c1_off + (size_t)(key - __ldg(kbase + it)) * N + col;
    const float g = gbuf[(size_t)u * N + col];
    if (fused) apply_update(cores + dst, state ? state + dst : nullptr, g, lr, eps, opt);
    else grads[dst] = g;
  }
}

bool agg_scatter_path(const Ctx& c) { return c.N % 4 == 0 && c.N <= 128 && (128 % c.N) == 0; }

// Plan-dependent zeroing for the coming backward (G rows for the scatter aggregation, dP rows for
// the row kernel): reads no parameters, so it runs with the index stage (pipelined side stream).
cudaError_t run_plan_tail(Ctx& c, cudaStream_t s) {
  if (c.nnz > 0 && agg_scatter_path(c))
    k_zero_rows<<<grid_for(c, c.U_cap * c.N / 4, 256, 8), 256, 0, s>>>(c.p.gbuf, c.p.counts, c.N);
  if (c.nnz > 0 && fused_eligible(c)) {
    cudaError_t e = run_unit_order(c, s);
    if (e != cudaSuccess) return e;
    return run_dp_zero(c, s);
  }
  return cudaGetLastError();
}

cudaError_t run_backward(Ctx& c, const float* grad_out, float lr, cudaStream_t s) {
  const PlanDev& p = c.p;
  const bool fused = (c.flags & TTEMB_FUSED_UPDATE) != 0;
  {
    StageScope sc(c, ST_BWD_ZERO, s);
    if (fused) {
      // the C1 / C3 accumulators were cleared by the previous fused update (k_update_zero)
    } else {
      cudaMemsetAsync(c.grads, 0, sizeof(float) * c.core_floats, s);
    }
  }
  if (c.nnz > 0) {
    StageScope sc(c, ST_AGG, s);
    if (agg_scatter_path(c)) {
      // (G was zeroed at the end of the index stage: run_plan_tail)
      launch_pdl(k_agg_scatter, dim3(grid_for(c, cdiv(c.nnz, 32), 8, TTEMB_AGG_GRID)), dim3(256), 0, s, grad_out,
                 (const uint32_t*)p.sbag, (const uint32_t*)p.spos, (const uint32_t*)p.inverse, (int64_t)c.nnz, c.N,
                 p.gbuf, (const float*)(c.weighted ? p.wpos : nullptr), (const uint32_t*)p.counts);
    } else {
      const int64_t total = agg_chunks(c.nnz) * c.N;
      if (c.N % 4 == 0)
        k_agg<4><<<grid_for(c, total / 4, 256, 32), 256, 0, s>>>(grad_out, p.skey, p.sbag, p.spos,
                                                                p.inverse, p.seg_off, c.nnz, c.N,
                                                                p.gbuf, p.aggpart, c.weighted ? p.wpos : nullptr);
      else
        k_agg<1><<<grid_for(c, total, 256, 32), 256, 0, s>>>(grad_out, p.skey, p.sbag, p.spos, p.inverse,
                                                            p.seg_off, c.nnz, c.N, p.gbuf, p.aggpart,
                                                            c.weighted ? p.wpos : nullptr);
      k_agg_fix<<<grid_for(c, agg_chunks(c.nnz) * 32, 256, 32), 256, 0, s>>>(
          p.skey, p.spos, p.inverse, p.seg_off, c.nnz, c.N, p.aggpart, p.gbuf);
    }
  }
  if (c.nnz > 0 && c.n_dense > 0) {   // hybrid placement: dense-table rows
    StageScope sc(c, ST_BWD_ROWS, s);
    k_dense_bwd<<<grid_for(c, (int64_t)c.U_cap * c.N, 256, 8), 256, 0, s>>>(
        c.cores, c.state, c.grads, c.d_meta, c.d_kbase, c.d_kmap, c.T, p.ukey, p.counts, c.N, p.gbuf,
        fused ? 1 : 0, lr, c.eps, c.opt);
  }
  if (!fused) c.mark_bucket(0, s);      // the dense tables' gradients are final
  BwdArgs a;
  a.cores = c.cores; a.grads = c.grads; a.state = c.state; a.meta = c.d_meta;
  a.counts = p.counts; a.grp_off = p.grp_off; a.grp_t = p.grp_t; a.grp_i2 = p.grp_i2;
  a.grp_pfx = p.grp_pfx; a.pfx_t = p.pfx_t; a.pfx_i1 = p.pfx_i1; a.row_seg = p.row_seg;
  a.row_i3 = p.row_i3; a.gbuf = p.gbuf; a.dabuf = p.dabuf;
  a.n1 = c.n1; a.N = c.N; a.R = c.R;
  a.lr = lr; a.eps = c.eps; a.opt = c.opt; a.fused = fused ? 1 : 0;
  if (c.nnz > 0) {
    cudaError_t e = tc_eligible(c) ? run_tc_bwd(c, lr, s) : run_group_bwd(c, lr, s);
    if (e != cudaSuccess) return e;
    if (!fused_eligible(c)) {   // (the tcgen05 prefix-backward kernel adds dA into dC1 itself)
      StageScope sc(c, ST_DC1, s);
      if ((c.n1 * c.R) % 4 == 0)
        k_dc1<<<grid_for(c, c.P_cap * c.n1 * c.R / 4, 256, 32), 256, 0, s>>>(a);
      else
        k_dc1_scalar<<<grid_for(c, c.P_cap * c.n1 * c.R, 256, 32), 256, 0, s>>>(a);
    }
  }
  if (!fused) {   // (the tcgen05 path marked the C3 bucket after its row stage)
    if (!tc_eligible(c) || c.nnz == 0) c.mark_bucket(1, s);
    c.mark_bucket(2, s);
  }
  if (fused) {   // C2 was updated inside the group kernel; C1 and C3 densely here
    StageScope sc(c, ST_UPD_C3, s);
    if (c.c1_floats % 4 == 0 && c.c3_begin % 4 == 0 && c.c3_floats % 4 == 0)
      launch_pdl(k_update_zero4, dim3(grid_for(c, (int64_t)(c.c1_floats + c.c3_floats) / 4, 256, TTEMB_UPD_GRID)), dim3(256), 0, s,
                 c.cores, c.state, c.grads, (size_t)c.c1_floats, (size_t)c.c3_begin, (size_t)c.c3_floats, lr, c.eps, c.opt);
    else
      k_update_zero<<<grid_for(c, (int64_t)(c.c1_floats + c.c3_floats), 256, 32), 256, 0, s>>>(
          c.cores, c.state, c.grads, c.c1_floats, c.c3_begin, c.c3_floats, lr, c.eps, c.opt);
  }
  return cudaGetLastError();
}

cudaError_t run_update_range(Ctx& c, float lr, size_t begin, size_t count, cudaStream_t s) {
  StageScope sc(c, ST_UPDATE, s);
  k_update<<<grid_for(c, (int64_t)count, 256, 32), 256, 0, s>>>(c.cores, c.state, c.grads, begin, count, lr,
                                                                c.eps, c.opt);
  return cudaGetLastError();
}

cudaError_t run_update(Ctx& c, float lr, cudaStream_t s) {
  StageScope sc(c, ST_UPDATE, s);
  k_update<<<grid_for(c, (int64_t)c.core_floats, 256, 32), 256, 0, s>>>(
      c.cores, c.state, c.grads, 0, c.core_floats, lr, c.eps, c.opt);
  return cudaGetLastError();
}

}  // namespace ttemb
