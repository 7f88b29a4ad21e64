// tc_probe3.cu -- probe of the "A operand in TMEM" form of tcgen05.mma kind::tf32 (the
// fused forward kernel keeps C2^T there): layout (lane = M row, one fp32 per column = K),
// tcgen05.st 32x32b staging, 3xTF32 accuracy with raw-fp32-as-hi, and MMA issue rate.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o scripts/tc_probe3 scripts/tc_probe3.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <cmath>
#include <vector>

#include "../paper_conf_sc_wangwfmmd22_b200/csrc/tc.cuh"

using namespace ttemb;

constexpr int M = 128, K = 64;

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const float (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]), "f"(v[8]),
      "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15]), "f"(v[16]),
      "f"(v[17]), "f"(v[18]), "f"(v[19]), "f"(v[20]), "f"(v[21]), "f"(v[22]), "f"(v[23]), "f"(v[24]),
      "f"(v[25]), "f"(v[26]), "f"(v[27]), "f"(v[28]), "f"(v[29]), "f"(v[30]), "f"(v[31])
      : "memory");
}

__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}\n" ::"r"(d),
      "r"(a), "l"(bdesc), "r"(idesc), "r"(acc));
}

// A [M][K] row-major, B [N][K] row-major (K-major), out [M][N]. mode 0: 3xTF32, 1: 1xTF32
__global__ void __launch_bounds__(128, 1) k_probe(const float* A, const float* B, float* out, int N, int mode,
                                                  int reps, unsigned long long* cyc) {
  extern __shared__ __align__(128) char smem[];
  float* bh = reinterpret_cast<float*>(smem);
  float* bl = bh + 256 * K;
  __shared__ uint64_t mbar;
  __shared__ uint32_t s_tmem;
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const int NRB = N / 8;
  for (int e = tid; e < N * K; e += 128) {
    const int n = e / K, k = e % K;
    const float x = B[e];
    const uint32_t off = tc::cm_off(n, k, NRB);
    *reinterpret_cast<float*>(reinterpret_cast<char*>(bh) + off) = x;
    *reinterpret_cast<float*>(reinterpret_cast<char*>(bl) + off) = x - tc::tf32_trunc(x);
  }
  if (tid == 0) { tc::mbar_init(&mbar, 1); tc::fence_mbar_init(); }
  if (w == 0) tc::tmem_alloc(&s_tmem, 512);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tm = s_tmem;
  // A row m = 32 w + lane: hi at columns [0, K), lo at [K, 2K)
  const int m = 32 * w + lane;
  for (int k0 = 0; k0 < K; k0 += 32) {
    float v[32], l[32];
    for (int i = 0; i < 32; ++i) { v[i] = A[m * K + k0 + i]; l[i] = v[i] - tc::tf32_trunc(v[i]); }
    tmem_st32(tc::taddr(tm, 32 * w, k0), v);
    tmem_st32(tc::taddr(tm, 32 * w, K + k0), l);
  }
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  tc::fence_async_smem();
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t D = tm + 256;
  if (tid == 0) {
    const uint32_t id = tc::idesc_tf32(M, N, false, false);
    const long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
      for (int kk = 0; kk < K / 8; ++kk) {
        const uint32_t bo = kk * 2 * NRB * 128;
        const uint64_t dbh = tc::sdesc(tc::smem_u32(bh) + bo, NRB * 128, 128);
        const uint64_t dbl = tc::sdesc(tc::smem_u32(bl) + bo, NRB * 128, 128);
        mma_ts(D, tm + kk * 8, dbh, id, kk > 0 ? 1u : 0u);
        if (mode == 0) {
          mma_ts(D, tm + kk * 8, dbl, id, 1u);
          mma_ts(D, tm + K + kk * 8, dbh, id, 1u);
        }
      }
    }
    tc::commit(&mbar);
    tc::mbar_wait(&mbar, 0);
    if (cyc) *cyc = (unsigned long long)(clock64() - t0);
  }
  __syncthreads();
  tc::fence_after();
  for (int n0 = 0; n0 < N; n0 += 32) {
    float v[32];
    tc::tmem_ld32(tc::taddr(D + n0, 32 * w, 0), v);
    for (int i = 0; i < 32; ++i)
      if (n0 + i < N) out[m * N + n0 + i] = v[i];
  }
  tc::fence_before();
  __syncthreads();
  if (w == 0) tc::tmem_dealloc(tm, 512);
}

int main() {
  srand(1);
  int bad = 0;
  for (int N : {16, 64, 128, 256}) {
    std::vector<float> A(M * K), B(N * K), O(M * N);
    for (auto& x : A) x = (float)rand() / RAND_MAX * 2 - 1;
    for (auto& x : B) x = (float)rand() / RAND_MAX * 2 - 1;
    float *dA, *dB, *dO;
    unsigned long long* dc;
    cudaMalloc(&dA, A.size() * 4); cudaMalloc(&dB, B.size() * 4); cudaMalloc(&dO, O.size() * 4);
    cudaMalloc(&dc, 8);
    cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 256 * K * 4);
    for (int mode = 0; mode < 2; ++mode) {
      k_probe<<<1, 128, 2 * 256 * K * 4>>>(dA, dB, dO, N, mode, 1, nullptr);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("N=%d mode=%d CUDA error %s\n", N, mode, cudaGetErrorString(e)); return 1; }
      cudaMemcpy(O.data(), dO, O.size() * 4, cudaMemcpyDeviceToHost);
      double maxrel = 0;
      for (int m = 0; m < M; ++m)
        for (int n = 0; n < N; ++n) {
          double s = 0, sa = 0;
          for (int k = 0; k < K; ++k) { s += (double)A[m * K + k] * B[n * K + k]; sa += fabs((double)A[m * K + k] * B[n * K + k]); }
          maxrel = std::max(maxrel, fabs(O[m * N + n] - s) / sa);
        }
      printf("N=%3d %s: max |err|/sum|ab| = %.3e\n", N, mode == 0 ? "3xTF32" : "1xTF32", maxrel);
      if (mode == 0 && maxrel > 1e-6) bad = 1;
      if (mode == 1 && maxrel > 5e-3) bad = 1;
    }
    // issue rate: reps x 8 k-steps x 3 MMAs
    const int reps = 64;
    k_probe<<<1, 128, 2 * 256 * K * 4>>>(dA, dB, dO, N, 0, reps, dc);
    cudaDeviceSynchronize();
    unsigned long long c;
    cudaMemcpy(&c, dc, 8, cudaMemcpyDeviceToHost);
    const double per = (double)c / (reps * 24);
    printf("N=%3d TS MMA 128x%dx8: %.1f cycles each (%.0f MAC/clk)\n", N, N, per, 128.0 * N * 8 / per);
    cudaFree(dA); cudaFree(dB); cudaFree(dO); cudaFree(dc);
  }
  printf(bad ? "PROBE FAILED\n" : "PROBE OK\n");
  return bad;
}
