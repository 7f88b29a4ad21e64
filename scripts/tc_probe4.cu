// tc_probe4.cu -- probes for the r02 fused kernels (run on a B200):
//   1. K-major tf32 operands in the SWIZZLE_128B_BASE32B layout (descriptor layout type 1):
//      can one smem arrangement ("rows of 128 B = 32 elements, 32-byte granules XOR row % 4")
//      serve as a K-major AND an MN-major operand?
//   2. the byte arrangement a 2-D TMA load with CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B produces
//   3. cp.reduce.async.bulk .add.f32 (shared -> global bulk reduction)
//   4. tcgen05.ld throughput (4 warps, 32x32b.x32)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o scripts/tc_probe4 scripts/tc_probe4.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <cmath>
#include <vector>

#include "../paper_conf_sc_wangwfmmd22_b200/csrc/tc.cuh"

using namespace ttemb;

// ---------------------------------------------------------------------------------------------
// 1. K-major BASE32B
// ---------------------------------------------------------------------------------------------
// variant v: how the 32-byte granule of (row, k) is permuted inside the 128-byte row
__host__ __device__ uint32_t kmaj_off(int v, int row, int k, int rows) {
  const int ka = k >> 5;                 // 32-element K atom
  const int g = (k & 31) >> 3, w = k & 7;
  int gs = g;
  if (v == 0) gs = g ^ (row & 3);
  if (v == 1) gs = g ^ ((row >> 1) & 3);
  if (v == 2) gs = g;
  if (v == 3) gs = g ^ ((row >> 2) & 3);
  if (v == 4) {   // control: standard SWIZZLE_128B (16-byte chunks XOR row % 8), layout type 2
    const int ch = ((k & 31) >> 2) ^ (row & 7);
    return (uint32_t)(ka * rows * 128 + row * 128 + ch * 16 + (k & 3) * 4);
  }
  return (uint32_t)(ka * rows * 128 + row * 128 + gs * 32 + w * 4);
}
// MN-major BASE32B (measured in r01): element (mn, k) of an MNx-wide operand
__device__ uint32_t mn_off(int mn, int k, int MNx) { return tc::mn32_off(mn, k, MNx); }

__device__ uint64_t desc(uint32_t saddr, uint32_t lbo, uint32_t sbo, uint32_t type) {
  return tc::sdesc_l(saddr, lbo, sbo, type);
}

// D[M][N] = sum_k A[M][K] B[N][K], A K-major (variant v, SBO sbo), B K-major CM (known good) or
// B = "same buffer as A" (bsame: B is the A matrix used as MN-major B: D = A^T-ish, see host).
__global__ void kmaj_probe(int v, int sbo, int M, int N, int K, const float* A, const float* B, float* out,
                           int bmode) {
  extern __shared__ __align__(1024) char smraw[];
  char* sm = smraw + ((1024u - (tc::smem_u32(smraw) & 1023u)) & 1023u);
  __shared__ uint64_t mbar;
  __shared__ uint32_t tbase;
  char* sa = sm;                            // A: M x K
  char* sb = sm + M * K * 4;                // B: N x K
  for (int e = threadIdx.x; e < M * K; e += blockDim.x) {
    const int r = e / K, k = e % K;
    *reinterpret_cast<float*>(sa + kmaj_off(v, r, k, M)) = A[e];
  }
  for (int e = threadIdx.x; e < N * K; e += blockDim.x) {
    const int n = e / K, k = e % K;
    if (bmode == 0) *reinterpret_cast<float*>(sb + tc::cm_off(n, k, N / 8)) = B[e];
    else *reinterpret_cast<float*>(sb + mn_off(n, k, N)) = B[e];   // MN-major B (N contiguous)
  }
  if (threadIdx.x == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (threadIdx.x < 32) tc::tmem_alloc(&tbase, 256);
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tb = tbase;
  if (threadIdx.x == 0) {
    const uint32_t id = tc::idesc_tf32(M, N, false, bmode != 0);
    for (int kk = 0; kk < K / 8; ++kk) {
      const uint32_t aoff = (kk >> 2) * M * 128 + (kk & 3) * 32;
      const uint64_t da = desc(tc::smem_u32(sa) + aoff, 16, sbo, v == 4 ? 2 : 1);
      uint64_t dbb;
      if (bmode == 0) dbb = tc::sdesc(tc::smem_u32(sb) + kk * 2 * (N / 8) * 128, (N / 8) * 128, 128);
      else {
        const uint32_t s2 = (N / 32) * 512;
        dbb = tc::sdesc_l(tc::smem_u32(sb) + kk * 2 * s2, 512, s2, 1);
      }
      tc::mma_tf32(tb, da, dbb, id, kk > 0);
    }
    tc::commit(&mbar);
  }
  tc::mbar_wait(&mbar, 0);
  tc::fence_after();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (w < 4) {
    for (int c0 = 0; c0 < N; c0 += 8) {
      float vv[8];
      tc::tmem_ld8(tc::taddr(tb, 32 * w, c0), vv);
      const int l = 32 * w + lane;
      int row = -1;
      if (M == 128) row = l;
      else if ((l & 31) < 16) row = (l & 15) + 16 * (l >> 5);
      if (row >= 0)
        for (int j = 0; j < 8 && c0 + j < N; ++j) out[row * N + c0 + j] = vv[j];
    }
  }
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tb, 256);
}

static double kmaj_case(int v, int sbo, int M, int N, int K, int bmode) {
  std::vector<float> a(M * K), b(N * K), o(M * N, -7.f);
  srand(1234 + M + N + K);
  for (auto& x : a) x = (float)(rand() % 17 - 8) / 8.f;   // exact in tf32
  for (auto& x : b) x = (float)(rand() % 17 - 8) / 8.f;
  float *da, *db, *dout;
  cudaMalloc(&da, a.size() * 4); cudaMalloc(&db, b.size() * 4); cudaMalloc(&dout, o.size() * 4);
  cudaMemcpy(da, a.data(), a.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(db, b.data(), b.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dout, o.data(), o.size() * 4, cudaMemcpyHostToDevice);
  const int smem = 4 * (M * K + N * K) + 2048;
  cudaFuncSetAttribute(kmaj_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  kmaj_probe<<<1, 256, smem>>>(v, sbo, M, N, K, da, db, dout, bmode);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { cudaDeviceReset(); return -1.0; }
  cudaMemcpy(o.data(), dout, o.size() * 4, cudaMemcpyDeviceToHost);
  double maxerr = 0;
  for (int i = 0; i < M; ++i)
    for (int j = 0; j < N; ++j) {
      double s = 0;
      for (int k = 0; k < K; ++k) s += (double)a[i * K + k] * b[j * K + k];
      maxerr = std::max(maxerr, std::fabs(o[i * N + j] - s));
    }
  cudaFree(da); cudaFree(db); cudaFree(dout);
  return maxerr;
}

// ---------------------------------------------------------------------------------------------
// 2. TMA 2-D load with SWIZZLE_128B_ATOM_32B: dump the smem bytes
// ---------------------------------------------------------------------------------------------
__global__ void tma_probe(const __grid_constant__ CUtensorMap map, float* dump, int nfloats) {
  extern __shared__ __align__(1024) char smraw0[];
  char* smraw = smraw0 + ((1024u - (tc::smem_u32(smraw0) & 1023u)) & 1023u);
  __shared__ uint64_t mbar;
  if (threadIdx.x == 0) {
    tc::mbar_init(&mbar, 1);
    tc::fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    tc::mbar_arrive_tx(&mbar, nfloats * 4);
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        ::"r"(tc::smem_u32(smraw)), "l"(&map), "r"(0), "r"(0), "r"(tc::smem_u32(&mbar))
        : "memory");
  }
  tc::mbar_wait(&mbar, 0);
  for (int i = threadIdx.x; i < nfloats; i += blockDim.x) dump[i] = reinterpret_cast<float*>(smraw)[i];
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static void tma_main() {
  EncodeFn enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  if (!enc) { printf("no cuTensorMapEncodeTiled\n"); return; }
  const int rows = 16, cols = 64;            // global [rows][cols] fp32, value = r * 1000 + c
  std::vector<float> h(rows * cols);
  for (int r = 0; r < rows; ++r)
    for (int c = 0; c < cols; ++c) h[r * cols + c] = r * 1000 + c;
  float *dg, *dd;
  cudaMalloc(&dg, h.size() * 4);
  cudaMalloc(&dd, h.size() * 4);
  cudaMemcpy(dg, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  for (int sw : {(int)CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B, (int)CU_TENSOR_MAP_SWIZZLE_128B}) {
    CUtensorMap map;
    cuuint64_t gdim[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
    cuuint64_t gstr[1] = {(cuuint64_t)cols * 4};
    cuuint32_t box[2] = {32, (cuuint32_t)rows};     // 128-byte inner box
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dg, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     (CUtensorMapSwizzle)sw, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("encode failed %d for swizzle %d\n", (int)r, sw); continue; }
    const int nf = 32 * rows;
    cudaFuncSetAttribute(tma_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 9216);
    tma_probe<<<1, 128, 9216>>>(map, dd, nf);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("tma error %s\n", cudaGetErrorString(e)); exit(2); }
    std::vector<float> o(nf);
    cudaMemcpy(o.data(), dd, nf * 4, cudaMemcpyDeviceToHost);
    printf("swizzle %d: smem float index -> (row, col) of the first 8 rows, granule view:\n", sw);
    for (int r = 0; r < 8; ++r) {
      printf("  smem row %d:", r);
      for (int g = 0; g < 4; ++g) {
        const float v = o[r * 32 + g * 8];
        printf("  g%d=(%d,%d)", g, (int)v / 1000, (int)v % 1000);
      }
      printf("   | 16B chunks:");
      for (int g = 0; g < 8; ++g) { const float v = o[r * 32 + g * 4]; printf(" %d", ((int)v % 1000) / 4); }
      printf("\n");
    }
  }
  cudaFree(dg); cudaFree(dd);
}

// ---------------------------------------------------------------------------------------------
// 3. bulk reduction shared -> global
// ---------------------------------------------------------------------------------------------
__global__ void bulk_red_probe(float* g, int n) {
  extern __shared__ __align__(128) float sf[];
  for (int i = threadIdx.x; i < n; i += blockDim.x) sf[i] = (float)(blockIdx.x + 1) * 0.5f + i;
  tc::fence_async_smem();
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(g),
                 "r"(tc::smem_u32(sf)), "r"(n * 4)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

// ---------------------------------------------------------------------------------------------
// 4. tcgen05.ld throughput
// ---------------------------------------------------------------------------------------------
__global__ void tmem_ld_probe(int reps, int nwarps, long long* cyc, float* sink) {
  __shared__ uint32_t tbase;
  if (threadIdx.x < 32) tc::tmem_alloc(&tbase, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const int w = threadIdx.x >> 5;
  float acc = 0.f;
  long long t0 = clock64();
  if (w < nwarps) {
    for (int r = 0; r < reps; ++r) {
      float v[32];
      tc::tmem_ld32(tc::taddr(tbase, 32 * (w & 3), (uint32_t)((r * 32 + 128 * (w >> 2)) & 511)), v);
#pragma unroll
      for (int i = 0; i < 32; ++i) acc += v[i];
    }
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
  sink[threadIdx.x] = acc;
  tc::fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tc::tmem_dealloc(tbase, 512);
}

int main(int argc, char** argv) {
  const int sec = argc > 1 ? atoi(argv[1]) : 0;
  if (sec == 1) {
  printf("== 1. K-major tf32 with layout type 1 (128B_BASE32B); exact inputs, error must be 0\n");
  const int bsel = argc > 2 ? atoi(argv[2]) : -1, vsel = argc > 3 ? atoi(argv[3]) : -1,
            ssel = argc > 4 ? atoi(argv[4]) : -1;
  for (int bmode = 0; bmode < 2; ++bmode)
    for (int v = 0; v < 5; ++v)
      for (int sbo : {512, 1024}) {
        if ((bsel >= 0 && bmode != bsel) || (vsel >= 0 && v != vsel) || (ssel >= 0 && sbo != ssel)) continue;
        const int M = 128, N = 64, K = 64;
        const double e1 = kmaj_case(v, sbo, M, N, K, bmode);
        const double e2 = kmaj_case(v, sbo, 64, 32, 128, bmode);
        printf("  B=%s variant %d SBO %4d: M128N64K64 err %.3g | M64N32K128 err %.3g\n",
               bmode ? "MN32" : "CM  ", v, sbo, e1, e2);
      }
  }
  if (sec == 2) {
  printf("== 2. TMA 2-D load, 128-byte inner box\n");
  tma_main();
  }
  if (sec == 3) {
  printf("== 3. cp.reduce.async.bulk add.f32\n");
  {
    const int n = 256, nb = 64;
    float* g;
    cudaMalloc(&g, n * 4);
    cudaMemset(g, 0, n * 4);
    bulk_red_probe<<<nb, 128, n * 4>>>(g, n);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<float> o(n);
    cudaMemcpy(o.data(), g, n * 4, cudaMemcpyDeviceToHost);
    double maxerr = 0;
    for (int i = 0; i < n; ++i) {
      double s = 0;
      for (int b = 0; b < nb; ++b) s += (b + 1) * 0.5 + i;
      maxerr = std::max(maxerr, std::fabs(o[i] - s));
    }
    printf("  %s, max err %.3g\n", e == cudaSuccess ? "ok" : cudaGetErrorString(e), maxerr);
  }
  }
  if (sec == 4) {
  printf("== 4. tcgen05.ld.32x32b.x32 throughput\n");
  {
    long long* c;
    float* sink;
    cudaMalloc(&c, 8);
    cudaMalloc(&sink, 4096);
    for (int nw : {1, 4, 8, 16}) {
      const int reps = 256;
      tmem_ld_probe<<<1, 512, 0>>>(reps, nw, c, sink);
      cudaDeviceSynchronize();
      long long h;
      cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
      printf("  %2d warps x %d lds of 4 KB: %lld cycles -> %.1f B/cycle\n", nw, reps, h, nw * reps * 4096.0 / h);
    }
  }
  }
  return 0;
}
