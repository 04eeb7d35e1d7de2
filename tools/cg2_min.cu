// Minimal CTA-pair (tcgen05.mma.cta_group::2) probe: one cluster of two CTAs, D[256 x 128] = A[256 x 64] *
// B[128 x 64]^T with A rows 0-127 / 128-255 in CTA 0 / 1 and B rows 0-63 / 64-127 in CTA 0 / 1, K-major SW128
// tiles written by threads.  Mode 0: each CTA runs its own cta_group::1 M = 128, N = 64 MMA (control).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -DVISTA_HANG_DEBUG -I paper_conf_sigmod_nakandalak20_b200/csrc
//        -o tools/ab/cg2_min tools/cg2_min.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>
#include <cuda_runtime.h>
#include "ptx.cuh"
using namespace vista;

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128) probe(const __nv_bfloat16* A, const __nv_bfloat16* B,
                                                                         float* D, int mode) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sA = smem;                 // 128 rows x 128 B
  uint8_t* sB = smem + 16384;         // 64 rows x 128 B
  uint64_t* bar = (uint64_t*)(smem + 16384 + 8192);
  uint32_t* slot = (uint32_t*)(bar + 2);
  const uint32_t rank = cluster_rank();
  const int t = threadIdx.x, warp = t / 32, lane = t % 32;
  // fill (SW128: 16-byte chunk c of row r at r * 128 + ((c ^ (r & 7)) << 4))
  for (int i = t; i < 128 * 8; i += 128) {
    const int r = i / 8, c = i % 8;
    *(uint4*)(sA + r * 128 + ((c ^ (r & 7)) << 4)) = *(const uint4*)(A + (size_t)(rank * 128 + r) * 64 + c * 8);
  }
  for (int i = t; i < 64 * 8; i += 128) {
    const int r = i / 8, c = i % 8;
    *(uint4*)(sB + r * 128 + ((c ^ (r & 7)) << 4)) = *(const uint4*)(B + (size_t)(rank * 64 + r) * 64 + c * 8);
  }
  fence_proxy_async_smem();
  if (t == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
  }
  cluster_sync_all();
  if (warp == 0) {
    if (mode == 1) tmem_alloc_cg2(slot, 128);
    else tmem_alloc(slot, 128);
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tmem = *slot;
  if (warp == 1) {
    if (mode == 1) {
      if (rank == 0) {
        const uint32_t idesc = umma_idesc_bf16(256, 128);
        const uint32_t a = umma_desc_lo_sw128(smem_u32(sA)), b = umma_desc_lo_sw128(smem_u32(sB));
        for (int k = 0; k < 4; ++k) tc_mma_bf16_lo_warp_cg2(tmem, a + 2 * k, b + 2 * k, idesc, k != 0);
        tc_commit_cg2_warp(bar, (uint16_t)3);
      }
    } else {
      const uint32_t idesc = umma_idesc_bf16(128, 64);
      const uint32_t a = umma_desc_lo_sw128(smem_u32(sA)), b = umma_desc_lo_sw128(smem_u32(sB));
      for (int k = 0; k < 4; ++k) tc_mma_bf16_lo_warp(tmem, a + 2 * k, b + 2 * k, idesc, k != 0);
      tc_commit_warp(bar);
    }
  }
  mbar_wait(bar, 0);
  tc_fence_after();
  const int ncols = mode == 1 ? 128 : 64;
  for (int c0 = 0; c0 < ncols; c0 += 32) {
    uint32_t r[32];
    tmem_ld_32x32b_x32(tmem + ((uint32_t)(warp * 32) << 16) + c0, r);
    tc_wait_ld();
    const int row = rank * 128 + warp * 32 + lane;
    for (int j = 0; j < 32; ++j) D[(size_t)row * 128 + (mode == 1 ? c0 + j : rank * 64 + c0 + j)] = __uint_as_float(r[j]);
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync_all();
  if (warp == 0) {
    if (mode == 1) tmem_dealloc_cg2(tmem, 128);
    else tmem_dealloc(tmem, 128);
  }
}

int main(int argc, char** argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 1;
  std::vector<__nv_bfloat16> hA(256 * 64), hB(128 * 64);
  std::vector<float> fA(256 * 64), fB(128 * 64);
  srand(1);
  for (int i = 0; i < 256 * 64; ++i) { hA[i] = __float2bfloat16((rand() % 17 - 8) / 8.f); fA[i] = __bfloat162float(hA[i]); }
  for (int i = 0; i < 128 * 64; ++i) { hB[i] = __float2bfloat16((rand() % 17 - 8) / 8.f); fB[i] = __bfloat162float(hB[i]); }
  __nv_bfloat16 *dA, *dB;
  float* dD;
  cudaMalloc(&dA, hA.size() * 2);
  cudaMalloc(&dB, hB.size() * 2);
  cudaMalloc(&dD, 256 * 128 * 4);
  cudaMemcpy(dA, hA.data(), hA.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB.data(), hB.size() * 2, cudaMemcpyHostToDevice);
  cudaMemset(dD, 0, 256 * 128 * 4);
  const int smem = 16384 + 8192 + 64 + 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  probe<<<2, 128, smem>>>(dA, dB, dD, mode);
  cudaError_t e = cudaDeviceSynchronize();
  printf("mode %d: %s\n", mode, cudaGetErrorString(e));
  if (e != cudaSuccess) return 1;
  std::vector<float> hD(256 * 128);
  cudaMemcpy(hD.data(), dD, hD.size() * 4, cudaMemcpyDeviceToHost);
  // mode 1: D = A B^T over all 256 x 128; mode 0: CTA r computes rows r*128.. against B rows r*64..
  double maxerr = 0;
  for (int m = 0; m < 256; ++m)
    for (int n = 0; n < 128; ++n) {
      if (mode == 0 && (n / 64) != (m / 128)) continue;
      double s = 0;
      for (int k = 0; k < 64; ++k) s += (double)fA[m * 64 + k] * fB[n * 64 + k];
      maxerr = std::max(maxerr, std::fabs(s - hD[m * 128 + n]));
    }
  printf("mode %d: max |err| = %g\n", mode, maxerr);
  return maxerr < 1e-3 ? 0 : 2;
}
