// ttemb_hosttier.cu -- the host-memory tier of EL-Rec's pipeline training system (
// PAPER §V; Fig. 16 setup P:417): embedding tables that do not fit in HBM live in host
// memory behind a CPU parameter server; the GPU worker trains the rows a batch touches and a GPU
// embedding cache with life-cycle (LC) eviction resolves the read-after-write conflict of
// pipelined pre-fetching.
//
// Device side (one worker): the pre-fetched rows of batch k arrive as a compact block
// rows[U][dim] (U = unique host rows of the batch, ids[U] = their global host row numbers):
//   k_ht_sync         "the embedding cache will search the indices from the index table; if the
//                     index is found ... [the row] needs to synchronize"
//   k_ht_pool         sum pooling of the bags over the block (Eq. 4 for plain rows)
//   k_ht_grad         dL/drow_u = sum of grad_out over u's occurrences (in occurrence order)
//   k_ht_tick         one gradient-queue pull: every live entry's LC -= 1, evicted at 0
//   k_ht_update_push  SGD on the block, then "pushed into the cache ... assigned with LC values
//                     equal to the maximum length of the Requests Queue"
// The index table is direct-mapped (one int32 slot number per host row: 4 B next to a 4*dim B
// row), slots come from a free list, so search / insert / evict are O(1) without probing.
//
// Host side (the parameter server): multi-threaded gather of rows into pinned staging
// (the pre-fetch) and the SGD apply of a pulled gradient batch.  The SGD arithmetic is the same
// two roundings on both sides (w - rn(lr*g), no FMA contraction), so a row the server updates in
// host memory and the copy the worker pushed into the cache are bitwise equal.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <thread>
#include <vector>

#include "../../include/ttemb.h"

namespace {

inline int grid_1d(int64_t n, int block) {
  int64_t g = (n + block - 1) / block;
  return (int)std::max<int64_t>(1, std::min<int64_t>(g, 148 * 32));
}

__global__ void k_ht_init(int32_t* __restrict__ index, int64_t n_rows, int32_t* __restrict__ lc,
                          int32_t* __restrict__ free_list, int32_t* __restrict__ top, int capacity) {
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < n_rows; i += nth) index[i] = -1;
  for (int64_t s = tid; s < capacity; s += nth) {
    lc[s] = 0;
    free_list[s] = (int32_t)s;
  }
  if (tid == 0) {
    top[0] = capacity;
    top[1] = 0;
  }
}

// warp per unique row: a cached row replaces the (possibly stale) pre-fetched copy
__global__ void k_ht_sync(const int32_t* __restrict__ index, const float* __restrict__ crows,
                          const int64_t* __restrict__ ids, int64_t n, int dim, float* __restrict__ rows) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = w0; u < n; u += nw) {
    const int32_t s = index[ids[u]];
    if (s < 0) continue;
    for (int c = lane; c < dim; c += 32) rows[u * dim + c] = crows[(int64_t)s * dim + c];
  }
}

// thread per (bag, column); bag = t * B + b, out is [B][T][dim]; summed in bag order from 0
__global__ void k_ht_pool(const float* __restrict__ rows, const int32_t* __restrict__ ridx,
                          const int64_t* __restrict__ offsets, int T, int B, int dim, float* __restrict__ out) {
  const int64_t total = (int64_t)T * B * dim;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t bag = e / dim;
    const int c = (int)(e - bag * dim);
    const int t = (int)(bag / B), b = (int)(bag - (int64_t)t * B);
    float acc = 0.f;
    for (int64_t j = offsets[bag]; j < offsets[bag + 1]; ++j) acc = __fadd_rn(acc, rows[(int64_t)ridx[j] * dim + c]);
    out[((int64_t)b * T + t) * dim + c] = acc;
  }
}

// thread per (unique row, column): g_u = sum over u's occurrences (CSR occ_ptr / occ_bag, in
// occurrence order) of grad_out[b][t]
__global__ void k_ht_grad(const float* __restrict__ grad_out, const int64_t* __restrict__ occ_ptr,
                          const int32_t* __restrict__ occ_bag, int64_t n, int T, int B, int dim,
                          float* __restrict__ g) {
  const int64_t total = n * dim;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t u = e / dim;
    const int c = (int)(e - u * dim);
    float acc = 0.f;
    for (int64_t k = occ_ptr[u]; k < occ_ptr[u + 1]; ++k) {
      const int bag = occ_bag[k];
      const int t = bag / B, b = bag - t * B;
      acc = __fadd_rn(acc, grad_out[((int64_t)b * T + t) * dim + c]);
    }
    g[e] = acc;
  }
}

// one gradient-queue pull: LC -= 1 for every live entry; an entry reaching 0 leaves the
// index table and its slot returns to the free list
__global__ void k_ht_tick(int32_t* __restrict__ index, int32_t* __restrict__ lc, const int64_t* __restrict__ owner,
                          int32_t* __restrict__ free_list, int32_t* __restrict__ top, int capacity) {
  for (int s = blockIdx.x * blockDim.x + threadIdx.x; s < capacity; s += gridDim.x * blockDim.x) {
    const int l = lc[s];
    if (l <= 0) continue;
    lc[s] = l - 1;
    if (l == 1) {
      index[owner[s]] = -1;
      free_list[atomicAdd(top, 1)] = s;
    }
  }
}

// warp per unique row: SGD w <- w - rn(lr * g) on the block, then (life > 0) insert / refresh
// the row in the cache with LC = life.  ids are unique within a batch, so no two warps touch the
// same index-table entry; slots are popped from the free list atomically.
__global__ void k_ht_update_push(float* __restrict__ rows, const float* __restrict__ g,
                                 const int64_t* __restrict__ ids, int64_t n, int dim, float lr, int life,
                                 int32_t* __restrict__ index, float* __restrict__ crows, int32_t* __restrict__ lc,
                                 int64_t* __restrict__ owner, const int32_t* __restrict__ free_list,
                                 int32_t* __restrict__ top) {
  const int lane = threadIdx.x & 31;
  const int64_t w0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t u = w0; u < n; u += nw) {
    int32_t s = -1;
    if (life > 0 && lane == 0) {
      const int64_t id = ids[u];
      s = index[id];
      if (s < 0) {
        const int pos = atomicSub(top, 1) - 1;
        if (pos < 0) {
          atomicAdd(top, 1);
          top[1] = 1;                     // capacity exhausted: reported by ttemb_ht_cache_stats
        } else {
          s = free_list[pos];
          index[id] = s;
          owner[s] = id;
        }
      }
      if (s >= 0) lc[s] = life;
    }
    s = __shfl_sync(0xffffffffu, s, 0);
    for (int c = lane; c < dim; c += 32) {
      const int64_t e = u * dim + c;
      const float w = __fsub_rn(rows[e], __fmul_rn(lr, g[e]));
      rows[e] = w;
      if (s >= 0) crows[(int64_t)s * dim + c] = w;
    }
  }
}

bool cache_ok(const ttemb_ht_cache* c) {
  return c && c->index && c->rows && c->lc && c->owner && c->free_list && c->top && c->n_rows >= 0 &&
         c->capacity > 0 && c->dim > 0;
}

int status(cudaError_t e) { return e == cudaSuccess ? TTEMB_OK : TTEMB_ERR_CUDA; }

// rows split over up to `nthreads` threads, at least 16384 rows each (a thread start costs about
// as much as copying that many rows)
template <class F>
void parallel_for(int64_t n, int nthreads, F f) {
  if (nthreads <= 0) nthreads = (int)std::min(16u, std::max(1u, std::thread::hardware_concurrency()));
  nthreads = (int)std::max<int64_t>(1, std::min<int64_t>(nthreads, n / 16384));
  if (nthreads == 1) {
    f(0, n);
    return;
  }
  std::vector<std::thread> th;
  const int64_t chunk = (n + nthreads - 1) / nthreads;
  for (int i = 0; i < nthreads; ++i) {
    const int64_t b = i * chunk, e = std::min(n, b + chunk);
    if (b < e) th.emplace_back([=] { f(b, e); });
  }
  for (auto& t : th) t.join();
}

}  // namespace

extern "C" int ttemb_ht_cache_init(const ttemb_ht_cache* c, void* stream) {
  if (!cache_ok(c)) return TTEMB_ERR_INVALID_ARG;
  k_ht_init<<<grid_1d(std::max<int64_t>(c->n_rows, c->capacity), 256), 256, 0, (cudaStream_t)stream>>>(
      c->index, c->n_rows, c->lc, c->free_list, c->top, c->capacity);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_sync(const ttemb_ht_cache* c, const int64_t* ids, int64_t n, float* rows, void* stream) {
  if (!cache_ok(c) || n < 0 || (n > 0 && (!ids || !rows))) return TTEMB_ERR_INVALID_ARG;
  if (n == 0) return TTEMB_OK;
  k_ht_sync<<<grid_1d(n * 32, 256), 256, 0, (cudaStream_t)stream>>>(c->index, c->rows, ids, n, c->dim, rows);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_pool(const float* rows, const int32_t* ridx, const int64_t* offsets, int32_t num_tables,
                             int32_t batch, int32_t dim, float* out, void* stream) {
  if (num_tables < 0 || batch < 0 || dim <= 0 || !offsets || (num_tables * (int64_t)batch > 0 && !out))
    return TTEMB_ERR_INVALID_ARG;
  const int64_t total = (int64_t)num_tables * batch * dim;
  if (total == 0) return TTEMB_OK;
  k_ht_pool<<<grid_1d(total, 256), 256, 0, (cudaStream_t)stream>>>(rows, ridx, offsets, num_tables, batch, dim, out);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_grad(const float* grad_out, const int64_t* occ_ptr, const int32_t* occ_bag, int64_t n,
                             int32_t num_tables, int32_t batch, int32_t dim, float* g, void* stream) {
  if (n < 0 || num_tables <= 0 || batch <= 0 || dim <= 0 || (n > 0 && (!grad_out || !occ_ptr || !occ_bag || !g)))
    return TTEMB_ERR_INVALID_ARG;
  if (n == 0) return TTEMB_OK;
  k_ht_grad<<<grid_1d(n * dim, 256), 256, 0, (cudaStream_t)stream>>>(grad_out, occ_ptr, occ_bag, n, num_tables,
                                                                      batch, dim, g);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_tick(const ttemb_ht_cache* c, void* stream) {
  if (!cache_ok(c)) return TTEMB_ERR_INVALID_ARG;
  k_ht_tick<<<grid_1d(c->capacity, 256), 256, 0, (cudaStream_t)stream>>>(c->index, c->lc, c->owner, c->free_list,
                                                                         c->top, c->capacity);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_update_push(const ttemb_ht_cache* c, float* rows, const float* g, const int64_t* ids,
                                    int64_t n, float lr, int32_t life, void* stream) {
  if (!cache_ok(c) || n < 0 || life < 0 || (n > 0 && (!rows || !g || !ids))) return TTEMB_ERR_INVALID_ARG;
  if (n == 0) return TTEMB_OK;
  k_ht_update_push<<<grid_1d(n * 32, 256), 256, 0, (cudaStream_t)stream>>>(
      rows, g, ids, n, c->dim, lr, life, c->index, c->rows, c->lc, c->owner, c->free_list, c->top);
  return status(cudaGetLastError());
}

extern "C" int ttemb_ht_host_gather(const float* table, int64_t n_rows, int32_t dim, const int64_t* ids, int64_t n,
                                    float* out, int32_t nthreads) {
  if (!table || dim <= 0 || n < 0 || (n > 0 && (!ids || !out))) return TTEMB_ERR_INVALID_ARG;
  for (int64_t u = 0; u < n; ++u)
    if (ids[u] < 0 || ids[u] >= n_rows) return TTEMB_ERR_INDEX_RANGE;
  parallel_for(n, nthreads, [&](int64_t b, int64_t e) {
    for (int64_t u = b; u < e; ++u) std::copy_n(table + ids[u] * dim, dim, out + u * dim);
  });
  return TTEMB_OK;
}

extern "C" int ttemb_ht_host_sgd(float* table, int64_t n_rows, int32_t dim, const int64_t* ids, int64_t n,
                                 const float* g, float lr, int32_t nthreads) {
  if (!table || dim <= 0 || n < 0 || (n > 0 && (!ids || !g))) return TTEMB_ERR_INVALID_ARG;
  for (int64_t u = 0; u < n; ++u)
    if (ids[u] < 0 || ids[u] >= n_rows) return TTEMB_ERR_INDEX_RANGE;
  parallel_for(n, nthreads, [&](int64_t b, int64_t e) {
    for (int64_t u = b; u < e; ++u) {
      float* w = table + ids[u] * dim;
      const float* gu = g + u * dim;
      // rounded product, then rounded difference: built with -ffp-contract=off (build.py), so
      // the compiler vectorises this without fusing it into an FMA
      for (int c = 0; c < dim; ++c) w[c] = w[c] - lr * gu[c];
    }
  });
  return TTEMB_OK;
}

extern "C" int ttemb_ht_cache_stats(const ttemb_ht_cache* c, int32_t* live, int32_t* overflow, void* stream) {
  if (!cache_ok(c) || !live || !overflow) return TTEMB_ERR_INVALID_ARG;
  int32_t top[2];
  cudaError_t e = cudaMemcpyAsync(top, c->top, sizeof(top), cudaMemcpyDeviceToHost, (cudaStream_t)stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize((cudaStream_t)stream);
  if (e != cudaSuccess) return TTEMB_ERR_CUDA;
  *live = c->capacity - top[0];
  *overflow = top[1];
  return TTEMB_OK;
}
