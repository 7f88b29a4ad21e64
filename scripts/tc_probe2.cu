// tc_probe2.cu -- probe of tcgen05 kind::tf32 operand layouts beyond the K-major interleaved
// "CM" layout: MN-major SWIZZLE_128B_BASE32B (the only MN-major layout tf32 accepts), the
// "raw fp32 as hi" 3xTF32 split, and MMA throughput for small N.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o scripts/tc_probe2 scripts/tc_probe2.cu
//   ./scripts/tc_probe2          correctness table
//   ./scripts/tc_probe2 time     throughput table
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <cmath>
#include <vector>

#include "../paper_conf_sc_wangwfmmd22_b200/csrc/tc.cuh"

using namespace ttemb;

enum Lay { CMK = 0, MN32 = 1, MN32B = 2, KSW128 = 3 };

// byte offset of element (mn, k) of an MNx x Kx operand
__host__ __device__ uint32_t lay_off(int lay, int mn, int k, int MNx, int Kx) {
  if (lay == CMK) return (uint32_t)(((k >> 2) * (MNx / 8) + (mn >> 3)) * 128 + (mn & 7) * 16 + (k & 3) * 4);
  if (lay == KSW128) {   // rows = mn, 128B = 32 k; 8-row atoms (1024B), 16B chunk ^= row%8
    const int atom = (k >> 5) * (MNx / 8) + (mn >> 3);
    const int chunk = ((k & 31) >> 2) ^ (mn & 7);
    return (uint32_t)(atom * 1024 + (mn & 7) * 128 + chunk * 16 + (k & 3) * 4);
  }
  const int g = (((mn & 31) >> 3) ^ (k & 3));
  const uint32_t in = (uint32_t)((k & 3) * 128 + g * 32 + (mn & 7) * 4);
  if (lay == MN32) return (uint32_t)(((k >> 2) * (MNx / 32) + (mn >> 5)) * 512) + in;
  return (uint32_t)(((mn >> 5) * (Kx / 4) + (k >> 2)) * 512) + in;
}

struct DescP { uint32_t lbo, sbo, kstep, type, katom; bool mn; };
// byte offset of k-step kk (K = 8 per MMA)
__host__ __device__ uint32_t koff(const struct DescP& d, int kk);
__host__ __device__ DescP lay_desc(int lay, int MNx, int Kx, int swap) {
  DescP d;
  d.katom = 0;
  if (lay == CMK) { d.lbo = (MNx / 8) * 128; d.sbo = 128; d.kstep = 2 * (MNx / 8) * 128; d.type = 0; d.mn = false; }
  else if (lay == KSW128) { d.lbo = 16; d.sbo = 1024; d.kstep = 32; d.type = 2; d.mn = false; d.katom = (MNx / 8) * 1024; }
  else if (lay == MN32) {
    d.lbo = 512; d.sbo = (MNx / 32) * 512; d.kstep = 2 * (MNx / 32) * 512; d.type = 1; d.mn = true;
    if (swap) { uint32_t t = d.lbo; d.lbo = d.sbo; d.sbo = t; }
  } else {
    d.lbo = (Kx / 4) * 512; d.sbo = 512; d.kstep = 1024; d.type = 1; d.mn = true;
    if (swap) { uint32_t t = d.lbo; d.lbo = d.sbo; d.sbo = t; }
  }
  return d;
}

__host__ __device__ uint32_t koff(const DescP& d, int kk) {
  return d.katom ? (kk >> 2) * d.katom + (kk & 3) * d.kstep : kk * d.kstep;
}

__device__ uint64_t mkdesc(uint32_t saddr, const DescP& p) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((p.lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((p.sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)p.type << 61;
  return d;
}

__device__ float trunc_tf32(float x) { return __uint_as_float(__float_as_uint(x) & 0xffffe000u); }

// split variant: 0 hi = rna(x), lo = x - hi;  1 hi = x (raw), lo = x - trunc(x);  2 hi = x, lo = x - rna(x)
__device__ void stage(float* hi, float* lo, const float* src, int MNx, int Kx, int lay, int var) {
  for (int e = threadIdx.x; e < MNx * Kx; e += blockDim.x) {
    const int mn = e / Kx, k = e % Kx;
    const float x = src[mn * Kx + k];
    float h, l;
    if (var == 0) { h = tc::tf32_hi(x); l = x - h; }
    else if (var == 1) { h = x; l = x - trunc_tf32(x); }
    else { h = x; l = x - tc::tf32_hi(x); }
    const uint32_t off = lay_off(lay, mn, k, MNx, Kx);
    *reinterpret_cast<float*>(reinterpret_cast<char*>(hi) + off) = h;
    *reinterpret_cast<float*>(reinterpret_cast<char*>(lo) + off) = l;
  }
}

__global__ void probe(int M, int N, int K, int la, int lb, int swap, int var, const float* A, const float* B,
                      float* out) {
  extern __shared__ __align__(1024) char smraw[];
  float* sm = reinterpret_cast<float*>(smraw);
  __shared__ uint64_t mbar;
  __shared__ uint32_t tmem_base;
  float *Ahi = sm, *Alo = Ahi + M * K, *Bhi = Alo + M * K, *Blo = Bhi + N * K;
  stage(Ahi, Alo, A, M, K, la, var);
  stage(Bhi, Blo, B, N, K, lb, var);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (threadIdx.x < 32) tc::tmem_alloc(&tmem_base, 512);
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = tmem_base;
  if (threadIdx.x == 0) {
    const DescP da = lay_desc(la, M, K, swap), db = lay_desc(lb, N, K, swap);
    const uint32_t id = tc::idesc_tf32(M, N, da.mn, db.mn);
    for (int kk = 0; kk < K / 8; ++kk) {
      const uint64_t ah = mkdesc(tc::smem_u32(Ahi) + koff(da, kk), da);
      const uint64_t al = mkdesc(tc::smem_u32(Alo) + koff(da, kk), da);
      const uint64_t bh = mkdesc(tc::smem_u32(Bhi) + koff(db, kk), db);
      const uint64_t bl = mkdesc(tc::smem_u32(Blo) + koff(db, kk), db);
      tc::mma_tf32(tb, ah, bh, id, kk > 0);
      tc::mma_tf32(tb, ah, bl, id, 1);
      tc::mma_tf32(tb, al, bh, id, 1);
    }
    tc::commit(&mbar);
  }
  tc::mbar_wait(&mbar, 0);
  tc::fence_after();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (w < 4) {
    for (int c0 = 0; c0 < N; c0 += 8) {
      float v[8];
      tc::tmem_ld8(tc::taddr(tb, 32 * w, c0), v);
      const int l = 32 * w + lane;
      int row = -1;
      if (M == 128) row = l;
      else if ((l & 31) < 16) row = (l & 15) + 16 * (l >> 5);
      if (row >= 0)
        for (int j = 0; j < 8 && c0 + j < N; ++j) out[row * N + c0 + j] = v[j];
    }
  }
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tb, 512);
}

static double run_case(int M, int N, int K, int la, int lb, int swap, int var, bool* err) {
  std::vector<float> a(M * K), b(N * K), o(M * N, -7.f);
  srand(M * 7 + N * 13 + K + la * 3 + lb);
  for (auto& x : a) x = (rand() / (float)RAND_MAX - 0.5f) * 2.f;
  for (auto& x : b) x = (rand() / (float)RAND_MAX - 0.5f) * 2.f;
  float *da, *db, *dout;
  cudaMalloc(&da, a.size() * 4); cudaMalloc(&db, b.size() * 4); cudaMalloc(&dout, o.size() * 4);
  cudaMemcpy(da, a.data(), a.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(db, b.data(), b.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dout, o.data(), o.size() * 4, cudaMemcpyHostToDevice);
  const size_t smem = (size_t)2 * 4 * (M * K + N * K);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  probe<<<1, 256, smem>>>(M, N, K, la, lb, swap, var, da, db, dout);
  cudaError_t e = cudaDeviceSynchronize();
  *err = e != cudaSuccess;
  if (*err) { printf("  CUDA error %s\n", cudaGetErrorString(e)); exit(2); }
  cudaMemcpy(o.data(), dout, o.size() * 4, cudaMemcpyDeviceToHost);
  double maxrel = 0;
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N; ++j) {
      double s = 0, sa = 0;
      for (int k = 0; k < K; ++k) { s += (double)a[i * K + k] * b[j * K + k]; sa += std::fabs((double)a[i * K + k] * b[j * K + k]); }
      maxrel = std::max(maxrel, std::fabs(o[i * N + j] - s) / (sa + 1e-30));
    }
  cudaFree(da); cudaFree(db); cudaFree(dout);
  return maxrel;
}

// ---- throughput: reps x (K=64: 8 k-steps x 3 MMAs), one CTA ----
__global__ void mma_timing(int M, int N, int la, int lb, int reps, long long* cycles, int nd = 1) {
  extern __shared__ __align__(1024) char smraw[];
  float* sm = reinterpret_cast<float*>(smraw);
  __shared__ uint64_t mbar;
  __shared__ uint32_t tmem_base;
  const int K = 64;
  for (int i = threadIdx.x; i < 2 * (M + N) * K; i += blockDim.x) sm[i] = 0.001f * (i % 97);
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (threadIdx.x < 32) tc::tmem_alloc(&tmem_base, 512);
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = tmem_base;
  long long t0 = 0, t1 = 0;
  if (threadIdx.x == 0) {
    const DescP da = lay_desc(la, M, K, 0), db = lay_desc(lb, N, K, 0);
    const uint32_t id = tc::idesc_tf32(M, N, da.mn, db.mn);
    const uint32_t ah = tc::smem_u32(sm), al = ah + M * K * 4, bh = al + M * K * 4, bl = bh + N * K * 4;
    t0 = clock64();
    for (int rep = 0; rep < reps; ++rep) {
#pragma unroll
      for (int kk = 0; kk < 8; ++kk) {
        const uint64_t dah = mkdesc(ah + koff(da, kk), da), dal = mkdesc(al + koff(da, kk), da);
        const uint64_t dbh = mkdesc(bh + koff(db, kk), db), dbl = mkdesc(bl + koff(db, kk), db);
        // nd independent accumulators: the 3 split MMAs of K step kk go to D[(kk % nd)]
        const uint32_t td = tb + (uint32_t)((kk % nd) * N);
        tc::mma_tf32(td, dah, dbh, id, (rep > 0 || kk >= nd) ? 1u : 0u);
        tc::mma_tf32(td, dah, dbl, id, 1u);
        tc::mma_tf32(td, dal, dbh, id, 1u);
      }
    }
    t1 = clock64();
    tc::commit(&mbar);
  }
  tc::mbar_wait(&mbar, 0);
  if (threadIdx.x == 0) { cycles[0] = t1 - t0; cycles[1] = clock64() - t0; }
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tb, 512);
}

static int timing_nd() {
  long long* d;
  cudaMalloc(&d, 16);
  const int smem = 2 * (128 + 256) * 64 * 4;
  cudaFuncSetAttribute(mma_timing, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (int N : {16, 32, 64, 128})
    for (int nd : {1, 2, 4, 8}) {
      if (nd * N > 512) continue;
      const int reps = 40;
      mma_timing<<<1, 128, smem>>>(128, N, KSW128, KSW128, reps, d, nd);
      cudaError_t e = cudaDeviceSynchronize();
      long long h[2];
      cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
      const double n = reps * 24.0;
      printf("M=128 N=%3d, %d independent accumulators: issue %5.1f cyc/MMA, complete %6.1f cyc/MMA (%6.0f MAC/cyc) %s\n", N, nd,
             h[0] / n, h[1] / n, 128.0 * N * 8 / (h[1] / n), e == cudaSuccess ? "" : cudaGetErrorString(e));
    }
  return 0;
}

static int timing_main() {
  long long* d;
  cudaMalloc(&d, 16);
  const int smem = 2 * (128 + 256) * 64 * 4;
  cudaFuncSetAttribute(mma_timing, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int Ms[] = {64, 128};
  const int Ns[] = {8, 16, 32, 64, 128, 256};
  const char* ln[] = {"CMK", "MN32", "MN32B", "KSW128"};
  const int lays[][2] = {{CMK, CMK}, {MN32, MN32}, {MN32, CMK}, {KSW128, KSW128}};
  for (auto& L : lays)
    for (int M : Ms)
      for (int N : Ns) {
        if (L[1] != CMK && L[1] != KSW128 && N < 32) continue;   // MN32 needs N % 32 == 0
        if (L[0] != CMK && L[0] != KSW128 && M < 32) continue;
        const int reps = 40;
        mma_timing<<<1, 128, smem>>>(M, N, L[0], L[1], reps, d);
        cudaError_t e = cudaDeviceSynchronize();
        long long h[2];
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        const double n = reps * 24.0;
        printf("A %-6s B %-6s M=%3d N=%3d: issue %5.1f cyc/MMA, complete %6.1f cyc/MMA (%6.0f MAC/cyc) %s\n", ln[L[0]],
               ln[L[1]], M, N, h[0] / n, h[1] / n, (double)M * N * 8 / (h[1] / n),
               e == cudaSuccess ? "" : cudaGetErrorString(e));
      }
  return 0;
}

int main(int argc, char** argv) {
  if (argc > 1 && argv[1][0] == 'n') return timing_nd();
  if (argc > 1) return timing_main();
  struct Case { int M, N, K, la, lb; };
  const Case cases[] = {
      {64, 64, 64, CMK, CMK},     {64, 8, 64, CMK, CMK},     {64, 24, 64, CMK, CMK},   {128, 16, 64, CMK, CMK},
      {64, 64, 64, MN32, MN32},   {64, 256, 64, MN32, MN32}, {128, 64, 64, MN32, MN32}, {64, 64, 32, MN32, MN32},
      {128, 64, 64, MN32B, MN32B}, {128, 16, 64, MN32, CMK}, {128, 48, 64, MN32, CMK}, {64, 32, 16, MN32, CMK},
      {64, 64, 64, KSW128, KSW128}, {128, 64, 64, KSW128, CMK}};
  const char* ln[] = {"CMK", "MN32", "MN32B", "KSW128"};
  for (int swap = 0; swap < 2; ++swap)
    for (const Case& c : cases) {
      if (swap && c.la != MN32 && c.la != MN32B && c.lb != MN32 && c.lb != MN32B) continue;
      printf("swap %d A %-6s B %-6s M=%3d N=%3d K=%3d:", swap, ln[c.la], ln[c.lb], c.M, c.N, c.K);
      for (int var = 0; var < 3; ++var) {
        bool err;
        const double r = run_case(c.M, c.N, c.K, c.la, c.lb, swap, var, &err);
        printf("  v%d %.2e", var, r);
      }
      printf("\n");
    }
  return 0;
}
