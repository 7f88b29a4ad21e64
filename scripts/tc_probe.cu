// tc_probe.cu -- standalone check of the hand-written tcgen05 TF32 (3xTF32) MMAs and the
// CM shared-memory layouts used by the prefix contractions (csrc/tc.cuh).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o scripts/tc_probe scripts/tc_probe.cu
// Modes (fp64 CPU reference):
//   1: D[c][m]  = sum_k C2[k][c] X[m][k]     (A = C2 MN-major, B = X K-major)
//   2: D[r][c]  = sum_m X[m][r] Y[m][c]      (A = X^T MN-major, B = Y MN-major)
//   3: D[r][m]  = sum_c C2[r][c] Y[m][c]     (A = C2 K-major,  B = Y^T K-major)
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <cmath>
#include <vector>

#include "../paper_conf_sc_wangwfmmd22_b200/csrc/tc.cuh"

using namespace ttemb;

__device__ void stage_cm(float* hi, float* lo, const float* src, int rows, int cols, bool rowmajor_rc) {
  // src element (r, c): rowmajor_rc ? src[r*cols + c] : src[c*rows + r]
  const int NRB = rows / 8;
  for (int e = threadIdx.x; e < rows * cols; e += blockDim.x) {
    const int r = e / cols, c = e % cols;
    const float x = rowmajor_rc ? src[r * cols + c] : src[c * rows + r];
    const float h = tc::tf32_hi(x);
    const uint32_t off = tc::cm_off(r, c, NRB);
    *reinterpret_cast<float*>(reinterpret_cast<char*>(hi) + off) = h;
    *reinterpret_cast<float*>(reinterpret_cast<char*>(lo) + off) = x - h;
  }
}

__global__ void probe(int mode, int M, int N, int K, const float* a_src, const float* b_src, float* out,
                      int three, int swap) {
  extern __shared__ __align__(1024) float sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tmem_base;
  float *Ahi, *Alo, *Bhi, *Blo;
  int a_rows, a_cols, b_rows, b_cols;
  // natural sources:  mode1: a = C2[K][M] (rows K, cols M), b = X[N][K];
  //                   mode2: a = X[K][M] (rows m=K, cols r=M), b = Y[K][N];
  //                   mode3: a = C2[M][K], b = Y[N][K]
  if (mode == 1) { a_rows = K; a_cols = M; b_rows = N; b_cols = K; }
  else if (mode == 2) { a_rows = K; a_cols = M; b_rows = K; b_cols = N; }
  else { a_rows = M; a_cols = K; b_rows = N; b_cols = K; }
  Ahi = sm; Alo = Ahi + a_rows * a_cols; Bhi = Alo + a_rows * a_cols; Blo = Bhi + b_rows * b_cols;
  stage_cm(Ahi, Alo, a_src, a_rows, a_cols, true);
  stage_cm(Bhi, Blo, b_src, b_rows, b_cols, true);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (threadIdx.x < 32) tc::tmem_alloc(&tmem_base, 256);
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = tmem_base;
  if (threadIdx.x == 0) {
    const int anrb = a_rows / 8, bnrb = b_rows / 8;
    uint32_t alo_, asbo, astep, blo_, bsbo, bstep;
    bool amn, bmn;
    if (mode == 1) {        // A MN-major (M = cols), B K-major (N = rows)
      amn = true; asbo = swap ? 128 : anrb * 128; alo_ = swap ? anrb * 128 : 128; astep = 128;
      bmn = false; bsbo = 128; blo_ = bnrb * 128; bstep = 2 * bnrb * 128;
    } else if (mode == 2) { // A MN-major, B MN-major
      amn = true; asbo = swap ? 128 : anrb * 128; alo_ = swap ? anrb * 128 : 128; astep = 128;
      bmn = true; bsbo = swap ? 128 : bnrb * 128; blo_ = swap ? bnrb * 128 : 128; bstep = 128;
    } else {                // A K-major (M = rows), B K-major (N = rows)
      amn = false; asbo = 128; alo_ = anrb * 128; astep = 2 * anrb * 128;
      bmn = false; bsbo = 128; blo_ = bnrb * 128; bstep = 2 * bnrb * 128;
    }
    const uint32_t id = tc::idesc_tf32(M, N, amn, bmn);
    for (int kk = 0; kk < K / 8; ++kk) {
      const uint64_t ah = tc::sdesc(tc::smem_u32(Ahi) + kk * astep, alo_, asbo);
      const uint64_t al = tc::sdesc(tc::smem_u32(Alo) + kk * astep, alo_, asbo);
      const uint64_t bh = tc::sdesc(tc::smem_u32(Bhi) + kk * bstep, blo_, bsbo);
      const uint64_t bl = tc::sdesc(tc::smem_u32(Blo) + kk * bstep, blo_, bsbo);
      tc::mma_tf32(tb, ah, bh, id, kk > 0);
      if (three) {
        tc::mma_tf32(tb, ah, bl, id, 1);
        tc::mma_tf32(tb, al, bh, id, 1);
      }
    }
    tc::commit(&mbar);
  }
  tc::mbar_wait(&mbar, 0);
  tc::fence_after();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (w < 4) {
    for (int c0 = 0; c0 < N; c0 += 32) {
      float v[32];
      tc::tmem_ld32(tc::taddr(tb, 32 * w, c0), v);
      const int l = 32 * w + lane;
      int row = -1;
      if (M == 128) row = l;
      else if ((l & 31) < 16) row = (l & 15) + 16 * (l >> 5);
      if (row >= 0)
        for (int j = 0; j < 32 && c0 + j < N; ++j) out[row * N + c0 + j] = v[j];
    }
  }
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tb, 256);
}

int timing_main();
int main(int argc, char** argv) {
  if (argc > 1) return timing_main();
  struct Case { int mode, M, N, K; };
  Case cases[] = {{1, 128, 64, 64}, {1, 128, 64, 8}, {1, 128, 48, 32}, {2, 64, 128, 64},
                  {2, 128, 128, 64}, {2, 64, 128, 8}, {3, 64, 64, 128}, {3, 128, 48, 128},
                  {3, 64, 128, 64}};
  int fails = 0;
  for (int swap = 0; swap < 2; ++swap)
  for (auto cs : cases) {
    for (int three = 1; three < 2; ++three) {
      const int M = cs.M, N = cs.N, K = cs.K;
      int ar, ac, br, bc;
      if (cs.mode == 1) { ar = K; ac = M; br = N; bc = K; }
      else if (cs.mode == 2) { ar = K; ac = M; br = K; bc = N; }
      else { ar = M; ac = K; br = N; bc = K; }
      std::vector<float> a(ar * ac), b(br * bc), o(M * N, -7.f);
      srand(cs.mode * 100 + M + N + K);
      for (auto& x : a) x = (rand() / (float)RAND_MAX - 0.5f) * 2.f;
      for (auto& x : b) x = (rand() / (float)RAND_MAX - 0.5f) * 2.f;
      float *da, *db, *dout;
      cudaMalloc(&da, a.size() * 4); cudaMalloc(&db, b.size() * 4); cudaMalloc(&dout, o.size() * 4);
      cudaMemcpy(da, a.data(), a.size() * 4, cudaMemcpyHostToDevice);
      cudaMemcpy(db, b.data(), b.size() * 4, cudaMemcpyHostToDevice);
      cudaMemcpy(dout, o.data(), o.size() * 4, cudaMemcpyHostToDevice);
      const size_t smem = (size_t)2 * 4 * (ar * ac + br * bc);
      cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      probe<<<1, 256, smem>>>(cs.mode, M, N, K, da, db, dout, three, swap);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("mode %d: CUDA error %s\n", cs.mode, cudaGetErrorString(e)); return 2; }
      cudaMemcpy(o.data(), dout, o.size() * 4, cudaMemcpyDeviceToHost);
      double maxrel = 0, maxabs_ref = 0;
      int bad = 0;
      for (int i = 0; i < M; ++i)
        for (int j = 0; j < N; ++j) {
          double s = 0, sa = 0;
          for (int k = 0; k < K; ++k) {
            double x, y;
            if (cs.mode == 1) { x = a[k * M + i]; y = b[j * K + k]; }
            else if (cs.mode == 2) { x = a[k * M + i]; y = b[k * N + j]; }
            else { x = a[i * K + k]; y = b[j * K + k]; }
            s += x * y; sa += std::fabs(x * y);
          }
          const double err = std::fabs(o[i * N + j] - s) / (sa + 1e-30);
          if (err > maxrel) maxrel = err;
          if (sa > maxabs_ref) maxabs_ref = sa;
          if (err > (three ? 1e-5 : 5e-3)) ++bad;
        }
      printf("swap %d mode %d M=%3d N=%3d K=%3d %s: max err/|ref| = %.3e  bad=%d\n", swap, cs.mode, M, N, K,
             three ? "3xTF32" : "1xTF32", maxrel, bad);
      if (bad) ++fails;
      cudaFree(da); cudaFree(db); cudaFree(dout);
    }
  }
  printf(fails ? "TC PROBE FAILED\n" : "TC PROBE OK\n");
  return fails ? 1 : 0;
}

// ---- timing microbenchmark: NM back-to-back 3xTF32 K=64 products (24 MMAs each) ----
__global__ void mma_timing(int M, int N, int reps, int precomp, long long* cycles) {
  extern __shared__ __align__(1024) float sm[];
  __shared__ uint64_t mbar;
  __shared__ uint32_t tmem_base;
  for (int i = threadIdx.x; i < 4 * 64 * 64 * 2; i += blockDim.x) sm[i] = 0.001f * (i % 97);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (threadIdx.x < 32) tc::tmem_alloc(&tmem_base, 256);
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = tmem_base;
  long long t0 = 0, t1 = 0;
  if (threadIdx.x == 0) {
    const int MR = M / 8;    // row blocks of A (M rows), B has N rows
    const uint32_t id = tc::idesc_tf32(M, N, false, false);
    const uint32_t ah = tc::smem_u32(sm), al = ah + M * 64 * 4, bh = al + M * 64 * 4, bl = bh + N * 64 * 4;
    t0 = clock64();
    for (int rep = 0; rep < reps; ++rep) {
      if (precomp) {
        const uint64_t dah = tc::sdesc(ah, MR * 128, 128), dal = tc::sdesc(al, MR * 128, 128);
        const uint64_t dbh = tc::sdesc(bh, (N / 8) * 128, 128), dbl = tc::sdesc(bl, (N / 8) * 128, 128);
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint64_t oa = (uint64_t)((kk * 2 * MR * 128) >> 4), ob = (uint64_t)((kk * 2 * (N / 8) * 128) >> 4);
          tc::mma_tf32(tb, dah + oa, dbh + ob, id, (rep > 0 || kk > 0) ? 1u : 0u);
          tc::mma_tf32(tb, dah + oa, dbl + ob, id, 1u);
          tc::mma_tf32(tb, dal + oa, dbh + ob, id, 1u);
        }
      } else {
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t oa = kk * 2 * MR * 128, ob = kk * 2 * (N / 8) * 128;
          const uint64_t dah = tc::sdesc(ah + oa, MR * 128, 128), dal = tc::sdesc(al + oa, MR * 128, 128);
          const uint64_t dbh = tc::sdesc(bh + ob, (N / 8) * 128, 128), dbl = tc::sdesc(bl + ob, (N / 8) * 128, 128);
          tc::mma_tf32(tb, dah, dbh, id, (rep > 0 || kk > 0) ? 1u : 0u);
          tc::mma_tf32(tb, dah, dbl, id, 1u);
          tc::mma_tf32(tb, dal, dbh, id, 1u);
        }
      }
    }
    t1 = clock64();
    tc::commit(&mbar);
  }
  tc::mbar_wait(&mbar, 0);
  if (threadIdx.x == 0) { cycles[0] = t1 - t0; cycles[1] = clock64() - t0; }
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tb, 256);
}

int timing_main() {
  long long* d;
  cudaMalloc(&d, 16);
  cudaFuncSetAttribute(mma_timing, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 64 * 64 * 4 * 2 + 1024);
  int shapes[][2] = {{64, 64}, {128, 64}, {64, 128}, {128, 128}, {64, 256}, {128, 256}};
  for (auto& sh : shapes)
    for (int pre = 0; pre < 2; ++pre) {
      const int reps = 50;
      mma_timing<<<1, 128, 4 * 64 * 64 * 4 * 2 + 1024>>>(sh[0], sh[1], reps, pre, d);
      cudaError_t e = cudaDeviceSynchronize();
      long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      const double n = reps * 24.0;
      printf("M=%3d N=%3d precomp=%d: issue %.1f cyc/MMA, complete %.1f cyc/MMA (%.0f MAC/cyc) %s\n", sh[0], sh[1], pre,
             h[0] / n, h[1] / n, (double)sh[0] * sh[1] * 8 / (h[1] / n), e == cudaSuccess ? "" : cudaGetErrorString(e));
    }
  return 0;
}
